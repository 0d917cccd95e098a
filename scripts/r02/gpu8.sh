# Round-2 measurement batch: reading -> tile -> PPW, tensor tile space sweep, candidate protocol (WAF + exact carve-out)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
timeout 1500 python harness/readings.py --out gpurun_out/r02/readings_r02.jsonl > gpurun_out/r02/readings.log 2>&1; echo "readings rc=$?"
timeout 1800 python harness/tensor_sweep.py --kinds gemm --repeats 5 --window 1.0 --out gpurun_out/r02/tensor_sweep_r02.jsonl > gpurun_out/r02/tensor_sweep.log 2>&1; echo "tsweep rc=$?"
timeout 2400 python harness/candidates.py --out gpurun_out/r02/candidates_r02.jsonl > gpurun_out/r02/candidates.log 2>&1; echo "cand rc=$?"
tail -5 gpurun_out/r02/readings.log gpurun_out/r02/tensor_sweep.log gpurun_out/r02/candidates.log
