cd $GRAFT_REPO_ROOT
T=scripts/time_kernel.py
timeout 900 python -m pytest tests/test_gpu_tensor.py tests/test_gpu_host.py -q --timeout 600 -p no:cacheprovider -k "ccsd or host" 2>&1 | tail -3
for t in 1,2,1,48,2,48,48; do echo "== $t"; EATSS_CCSD_TC_PROF=1 timeout 300 python $T ccsd_t_d1 48 $t --engine 2 --iters 1 2>&1 | tail -2; done
for t in 1,2,1,48,2,48,48 1,1,1,48,2,48,48; do timeout 300 python $T ccsd_t_d1 48 $t --engine 2 --iters 5 2>&1 | tail -1; done
for xb in 1; do EATSS_CCSD_TC_XB=$xb timeout 300 python $T ccsd_t_d1 48 1,1,1,48,2,48,48 --engine 2 --iters 5 2>&1 | tail -1; done
