cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests/test_gpu_parity.py -q -k "ccsd" --timeout 300 -p no:cacheprovider 2>&1 | tail -2
T="timeout 120 python scripts/time_kernel.py ccsd_t_d1 48"
$T 4,4,4,4,4,32,4 --iters 3; EATSS_CCSD_GROUP=2 $T 4,4,4,4,4,32,4 --iters 3; EATSS_CCSD_GROUP=1 $T 4,4,4,4,4,32,4 --iters 3
EATSS_CCSD_NOPREFETCH=1 $T 4,4,4,4,4,32,4 --iters 3
$T 8,4,4,4,4,16,8 --iters 3
