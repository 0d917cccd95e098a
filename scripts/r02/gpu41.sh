# ccsd_tc: finer t3 slices (h2 plane x p6 part) -- parity, then A/B at dims 48 (2 = h2 halves, 6 = default now)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
timeout 1200 python -m pytest tests/test_gpu_tensor.py tests/test_gpu_parity.py -k "ccsd" -q -x -p no:cacheprovider 2>&1 | tail -2
EATSS_CCSD_TC_SLICES=2 timeout 600 python -m pytest tests/test_gpu_tensor.py -k "ccsd" -q -x -p no:cacheprovider 2>&1 | tail -1
T="scripts/time_kernel.py ccsd_t_d1 48,48,48,48,48,48,48 1,2,1,48,2,48,48 --engine 2 --iters 5"
for rep in 1 2 3; do for v in 6 2 0; do echo "== slices=$v"; EATSS_CCSD_TC_SLICES=$v timeout 300 python $T 2>&1 | tail -1; done; done
