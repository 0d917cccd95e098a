cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out; T=scripts/time_kernel.py
{ for pf in 1 0; do EATSS_CCSD_TC_PF=$pf timeout 120 python $T ccsd_t_d1 8,48,48,48,48,48,48 1,2,1,48,2,48,48 --engine 2 --iters 3 2>&1 | tail -1 | sed "s/^/pf$pf /"; done
  for pf in 1 0; do EATSS_CCSD_TC_PF=$pf timeout 300 python $T ccsd_t_d1 48,48,48,48,48,48,48 1,2,1,48,2,48,48 --engine 2 --iters 2 2>&1 | tail -1 | sed "s/^/pf$pf /"; done
  EATSS_CCSD_TC_PROF=1 timeout 120 python $T ccsd_t_d1 8,48,48,48,48,48,48 1,2,1,48,2,48,48 --engine 2 --iters 1 2>&1 | grep -E "prof" | tail -1
} > gpurun_out/ccsd_pf.txt 2>&1
timeout 900 python -m pytest tests/test_gpu_tensor.py -x -q -k "ccsd" --timeout 600 -p no:cacheprovider > gpurun_out/pytest_ccsd.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_ccsd.log
cat gpurun_out/ccsd_pf.txt; tail -2 gpurun_out/pytest_ccsd.log
