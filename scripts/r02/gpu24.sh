# epilogue waits suspended vs spinning; fused vs materialised lo (tf32), f16 headline tile
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
T=scripts/time_kernel.py
for f in 1 0; do r=$(EATSS_TCM_FUSE=$f timeout 120 python $T gemm 4000,4000,4000 256,256,32 --engine 2 --iters 50 2>&1 | tail -1); echo "sleep fuse $f tf32: $r"; done
r=$(timeout 120 python $T gemm 4000,4000,4000 256,256,64 --engine 4 --iters 50 2>&1 | tail -1); echo "sleep f16: $r"
EATSS_TCM_PROF=1 timeout 120 python $T gemm 4000,4000,4000 256,256,32 --engine 2 --iters 2 2>&1 | grep prof | tail -1
EATSS_TCM_PROF=1 timeout 120 python $T gemm 4000,4000,4000 256,256,64 --engine 4 --iters 2 2>&1 | grep prof | tail -1
EATSS_DEV_NVCC_FLAGS=-DEATSS_DEVTOOLS python paper_conf_cgo_jayaweerakwk24_b200/build.py --force -j 32 > /dev/null 2>&1 || echo BUILD FAILED
for f in 1 0; do r=$(EATSS_TCM_DBG=32 EATSS_TCM_FUSE=$f timeout 120 python $T gemm 4000,4000,4000 256,256,32 --engine 2 --iters 50 2>&1 | tail -1); echo "spin fuse $f tf32: $r"; done
r=$(EATSS_TCM_DBG=32 timeout 120 python $T gemm 4000,4000,4000 256,256,64 --engine 4 --iters 50 2>&1 | tail -1); echo "spin f16: $r"
