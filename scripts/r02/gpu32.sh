# SIMT spread parity failure details (product build), SIMT A/B on the bench's own plan, revised heat resident
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
for v in 1 0; do
  echo "== simt parity spread=$v"
  EATSS_SIMT_BULK_SPREAD=$v timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_waf.py -q -p no:cacheprovider -k "gemm or 2mm or syrk" 2>&1 | grep -E "FAILED|passed|failed|Error|assert" | head -20
done
for rep in 1 2; do for v in 1 0; do
  echo "== simt bench-plan spread=$v"
  EATSS_SIMT_BULK_SPREAD=$v timeout 300 python bench.py --engine simt --steps 20 --warmup 3 --no-configs --no-secondary --no-cpu-baseline --e2e-steps 1 2>&1 | grep '^{' | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['value'], d['roofline']['frac'])"
done; done
timeout 600 python -m pytest tests/test_gpu_heat_resident.py tests/test_gpu_parity.py -k "heat" -q -x -p no:cacheprovider 2>&1 | tail -3
for rep in 1 2; do for r in 1 0; do
  echo "== heat resident=$r"; EATSS_HEAT_RESIDENT=$r timeout 120 python scripts/time_kernel.py heat-3d 120 16,16,32 --tsteps 500 --iters 5 2>&1 | tail -1
done; done
