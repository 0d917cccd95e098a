cd $GRAFT_REPO_ROOT
timeout 900 python harness/sweep.py --tiles "64,256,128;32,384,48;32,512,48;24,512,32;48,256,64;24,512,48;32,384,64;32,512,24;48,192,64;16,1024,16;32,32,32;48,256,48" --repeats 7 --window 1.0 --no-parity --out gpurun_out/sweep_confirm_r01.jsonl 2>&1 | tail -2
python harness/report.py --confirm gpurun_out/sweep_confirm_r01.jsonl --json gpurun_out/sweep_confirm_r01.summary.json | head -40
timeout 1200 python -m pytest tests -m gpu -q --timeout 600 -p no:cacheprovider 2>&1 | tail -3
T="timeout 120 python scripts/time_kernel.py"
$T heat-3d 512 16,16,32 --tsteps 10 --iters 3; $T heat-3d 120 16,16,32 --tsteps 500 --iters 3; $T gemm 4000,4000,4000 16,1024,16
