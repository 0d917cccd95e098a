cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python harness/tensor_sweep.py --out gpurun_out/tensor_sweep_r01.jsonl > gpurun_out/tensor_sweep.log 2>&1; echo "tsweep $?"
timeout 900 python harness/space4d.py --out gpurun_out/space4d_r01.jsonl > gpurun_out/space4d.log 2>&1; echo "space4d $?"
tail -5 gpurun_out/tensor_sweep.log; tail -4 gpurun_out/space4d.log
