cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_fourd.py -x -q -k mttkrp --timeout 600 -p no:cacheprovider > gpurun_out/pytest_mt.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_mt.log
bash scripts/gpu_mt.sh
tail -2 gpurun_out/pytest_mt.log
