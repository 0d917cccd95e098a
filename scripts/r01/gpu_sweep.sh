cd $GRAFT_REPO_ROOT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw,temperature.gpu --format=csv > gpurun_out/sweep_gemm4000_r01.gpu.txt
timeout 5200 python harness/sweep.py --window 0.5 --out gpurun_out/sweep_gemm4000_r01.jsonl > gpurun_out/sweep_gemm4000_r01.log 2>&1
echo "sweep exit $?"
python harness/report.py gpurun_out/sweep_gemm4000_r01.jsonl --json gpurun_out/sweep_gemm4000_r01.summary.json | head -80
