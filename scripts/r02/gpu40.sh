# headline after: parked B split, PDL off inside timed-kernel windows; 3 bench runs + a PDL A/B without events
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm,power.draw,temperature.gpu,clocks_throttle_reasons.active --format=csv
for rep in 1 2 3; do
timeout 300 python bench.py --steps 200 --warmup 10 --no-configs --no-secondary --no-cpu-baseline --e2e-steps 2 2>&1 | grep '^{' | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('bench', round(d['ms_per_step'],4), round(d['value'],1), round(r['frac'],3), round(r['call_frac'],3), d['clocks'])"
done
for v in 1 0; do echo "== call pdl=$v"; EATSS_TCM_PDL=$v timeout 120 python scripts/time_kernel.py gemm 4000,4000,4000 256,256,64 --engine 4 --iters 100 2>&1 | tail -1; done
timeout 300 python scripts/time_kernel.py conv-2d 8192,5 16,64,5,5 --iters 50 2>&1 | tail -1
