cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out; T=scripts/time_kernel.py
{ for t in 1,2,1,48,2,48,48 1,1,1,48,2,48,48 1,3,1,48,2,48,48 1,4,1,48,2,48,48 1,5,1,48,2,48,48 1,2,1,48,1,48,48 1,4,1,48,1,48,48; do
    timeout 120 python $T ccsd_t_d1 8,48,48,48,48,48,48 $t --engine 2 --iters 3 2>&1 | tail -1; done
  for xb in 1 2; do for vs in 2 4 8; do EATSS_CCSD_TC_XB=$xb EATSS_CCSD_TC_VSTAGES=$vs timeout 120 python $T ccsd_t_d1 8,48,48,48,48,48,48 1,2,1,48,2,48,48 --engine 2 --iters 3 2>&1 | tail -1 | sed "s/^/xb$xb vs$vs /"; done; done
  EATSS_CCSD_TC_PROF=1 timeout 120 python $T ccsd_t_d1 8,48,48,48,48,48,48 1,2,1,48,2,48,48 --engine 2 --iters 1 2>&1 | grep -E "prof|ccsd" | tail -3
} > gpurun_out/ccsd_sweep.txt 2>&1
cat gpurun_out/ccsd_sweep.txt
