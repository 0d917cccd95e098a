# Round-2 baseline on a fresh box: GPU tests, smoke, default bench.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw,temperature.gpu --format=csv > gpurun_out/r02/smi.txt 2>&1
lscpu | head -20 > gpurun_out/r02/lscpu.txt
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/r02/pytest_gpu_base.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r02/pytest_gpu_base.log
timeout 900 python bench.py > gpurun_out/r02/bench_base.log 2>&1; echo "bench rc=$?" >> gpurun_out/r02/bench_base.log
tail -3 gpurun_out/r02/pytest_gpu_base.log; tail -c 600 gpurun_out/r02/bench_base.log
