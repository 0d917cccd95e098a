cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out; T=scripts/time_kernel.py
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_host.py -x -q -k "syrk" --timeout 600 -p no:cacheprovider > gpurun_out/pytest_syrk.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_syrk.log
{ for t in 16,1024,16 32,512,48 32,512,32 64,256,32; do timeout 120 python $T syrk 4000,4000 $t --engine 1 --iters 5 2>&1 | tail -1; EATSS_SYRK_TRANSB=1 timeout 120 python $T syrk 4000,4000 $t --engine 1 --iters 5 2>&1 | tail -1 | sed 's/^/transB /'; done
  timeout 120 python $T gemm 4000,4000,4000 16,1024,16 --engine 1 --iters 5 2>&1 | tail -1; } > gpurun_out/syrk_times.txt 2>&1
tail -3 gpurun_out/pytest_syrk.log; cat gpurun_out/syrk_times.txt
