cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out; T=scripts/time_kernel.py
{ for t in 16,64,5,5 8,152,5,5 4,480,4,4 32,32,5,5 8,512,5,5 16,1024,5,5; do timeout 120 python $T conv-2d 8192,5 $t --iters 20 2>&1 | tail -1; done; } > gpurun_out/conv_times.txt 2>&1
timeout 600 python -m pytest tests/test_gpu_fourd.py -x -q -k "conv2d" --timeout 600 -p no:cacheprovider > gpurun_out/pytest_conv.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_conv.log
cat gpurun_out/conv_times.txt; tail -2 gpurun_out/pytest_conv.log
