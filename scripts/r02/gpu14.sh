cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
timeout 900 python -m pytest tests/test_gpu_f16.py -q -x --timeout 600 -p no:cacheprovider 2>&1 | tail -3
T=scripts/time_kernel.py
for t in 256,256,64 256,192,128; do timeout 120 python $T gemm 4000,4000,4000 $t --engine 4 --iters 30 2>&1 | tail -1; done
timeout 120 python $T syrk 4000,4000 256,256,64 --engine 4 --iters 30 2>&1 | tail -1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 30 --csv python $T gemm 4000,4000,4000 256,256,64 --engine 4 --iters 3 2>/dev/null | grep -E "prep|colmax|tc_mma" | cut -c1-220 | tail -8
