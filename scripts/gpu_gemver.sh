cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out; T=scripts/time_kernel.py
timeout 600 python -m pytest tests/test_gpu_lowdim.py -x -q -k gemver --timeout 300 -p no:cacheprovider > gpurun_out/pytest_gemver.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gemver.log
{ for n2 in 0 1; do for t in 16,1024 816,16 64,512; do EATSS_GEMVER_NEST2=$n2 timeout 120 python $T gemver 16384 $t --engine 1 --iters 10 2>&1 | tail -1 | sed "s/^/nest2=$n2 /"; done; done; } > gpurun_out/gemver_times.txt 2>&1
tail -2 gpurun_out/pytest_gemver.log; cat gpurun_out/gemver_times.txt
