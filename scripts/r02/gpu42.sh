# tc_mma: 608 threads (no idle warp) at 104 registers + drain of 8 TMEM columns per wait (fewer accumulator spills)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
timeout 1500 python -m pytest tests/test_gpu_f16.py tests/test_gpu_tensor.py tests/test_gpu_fullsize.py -q -x -p no:cacheprovider 2>&1 | tail -2
T="scripts/time_kernel.py gemm 4000,4000,4000 256,256,64 --engine 4 --iters 100 --kernel-ms"
T2="scripts/time_kernel.py gemm 4000,4000,4000 256,256,32 --engine 2 --iters 100 --kernel-ms"
for rep in 1 2 3; do for v in 1 0; do echo "== drain16=$v (x8 vs guarded x4)"; EATSS_TCM_DRAIN16=$v timeout 120 python $T 2>&1 | tail -2; done; done
for v in 1 0; do echo "== tf32 drain16=$v"; EATSS_TCM_DRAIN16=$v timeout 120 python $T2 2>&1 | tail -2; done
EATSS_DEV_NVCC_FLAGS=-DEATSS_TCM_DRAIN_W=16 python paper_conf_cgo_jayaweerakwk24_b200/build.py --force -j 32 > /dev/null 2>&1
for rep in 1 2; do echo "== x16 build"; timeout 120 python $T 2>&1 | tail -2; done
