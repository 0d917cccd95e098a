cd $GRAFT_REPO_ROOT
timeout 1200 python -m pytest tests -m gpu -q --timeout 600 -p no:cacheprovider 2>&1 | tail -4
T="timeout 120 python scripts/time_kernel.py"
$T gemm 4000,4000,4000 16,1024,16; EATSS_KSUB=1 EATSS_STAGES=1 $T gemm 4000,4000,4000 16,1024,16
EATSS_STAGES=2 $T gemm 4000,4000,4000 16,1024,16; EATSS_KSUB=4 $T gemm 4000,4000,4000 16,1024,16
timeout 120 python scripts/debug_tc.py 4000 16,1024,16
$T gemm 4000,4000,4000 16,1024,16 --engine 2
$T jacobi-2d 16384 16,1024 --tsteps 20 --iters 3; $T jacobi-2d 4000 16,1024 --tsteps 500 --iters 3
$T heat-3d 512 16,16,32 --tsteps 10 --iters 3; $T heat-3d 120 16,16,32 --tsteps 500 --iters 3
