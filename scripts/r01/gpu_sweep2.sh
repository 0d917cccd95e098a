# Round-1 re-run of the full 3,375-variant gemm N=4000 sweep with the current SIMT executor (split wave tail,
# staged paths), then the interleaved confirmation of the top candidates.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw,temperature.gpu --format=csv > gpurun_out/sweep_gemm4000_r01b.gpu.txt
timeout 4800 python harness/sweep.py --window 0.5 --out gpurun_out/sweep_gemm4000_r01b.jsonl > gpurun_out/sweep_gemm4000_r01b.log 2>&1
echo "sweep exit $?"
python harness/report.py gpurun_out/sweep_gemm4000_r01b.jsonl --json gpurun_out/sweep_gemm4000_r01b.summary.json > gpurun_out/sweep_report_r01b.txt 2>&1
head -60 gpurun_out/sweep_report_r01b.txt
