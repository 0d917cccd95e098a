# cost isolation of the 128-k accumulator chunks (development build with -DEATSS_DEVTOOLS, results wrong)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
EATSS_DEV_NVCC_FLAGS=-DEATSS_DEVTOOLS python paper_conf_cgo_jayaweerakwk24_b200/build.py --force -j 32 > /dev/null 2>&1
T=scripts/time_kernel.py
for dbg in 0 1 3 7 4; do for c in 128 512; do echo "dbg=$dbg chunk=$c"; EATSS_TCM_DBG=$dbg EATSS_TCM_CHUNK_K=$c python $T gemm 4000,4000,4000 256,256,32 --engine 2 --iters 50 2>&1 | tail -1; done; done
