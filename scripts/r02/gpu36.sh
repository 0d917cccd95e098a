# programmatic dependent launch across the tensor engines' launch chain: parity, A/B (call time and bench)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
timeout 1200 python -m pytest tests/test_gpu_f16.py tests/test_gpu_tensor.py tests/test_gpu_fullsize.py -q -x -p no:cacheprovider 2>&1 | tail -2
T="scripts/time_kernel.py gemm 4000,4000,4000 256,256,64 --engine 4 --iters 50"
for rep in 1 2 3; do for v in 1 0; do echo "== pdl=$v"; EATSS_TCM_PDL=$v timeout 120 python $T 2>&1 | tail -1; done; done
for v in 1 0; do echo "== tf32 pdl=$v"; EATSS_TCM_PDL=$v timeout 120 python scripts/time_kernel.py gemm 4000,4000,4000 256,256,32 --engine 2 --iters 50 2>&1 | tail -1; done
for rep in 1 2; do for v in 1 0; do
  echo "== bench pdl=$v"
  EATSS_TCM_PDL=$v timeout 300 python bench.py --steps 100 --warmup 5 --no-configs --no-secondary --no-cpu-baseline --e2e-steps 2 2>&1 | grep '^{' | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print(d['ms_per_step'], d['value'], r['frac'], r['call_frac'])"
done; done
