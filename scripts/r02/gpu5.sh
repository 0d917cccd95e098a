cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
timeout 600 python scripts/r02/chunk_ab.py > gpurun_out/r02/chunk_ab3.jsonl 2>&1
timeout 900 python bench.py --no-configs > gpurun_out/r02/bench5.log 2>&1; echo "bench rc=$?" >> gpurun_out/r02/bench5.log
timeout 900 python -m pytest tests/test_gpu_tensor.py tests/test_gpu_host.py tests/test_gpu_fullsize.py -q --timeout 900 -p no:cacheprovider > gpurun_out/r02/pytest_gpu5.log 2>&1; echo "rc=$?" >> gpurun_out/r02/pytest_gpu5.log
cat gpurun_out/r02/chunk_ab3.jsonl; tail -2 gpurun_out/r02/pytest_gpu5.log; tail -c 1500 gpurun_out/r02/bench5.log
