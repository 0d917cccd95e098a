cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_tensor.py -q -x --timeout 300 -p no:cacheprovider -k "ccsd" 2>&1 | tail -3
timeout 900 python scripts/ccsd_variants.py
timeout 600 ncu --set full --clock-control none -k regex:ccsd_tc -c 1 -o gpurun_out/prof_ccsdtc2 python scripts/time_kernel.py ccsd_t_d1 8,48,48,48,48,48,48 1,1,1,48,2,48,48 --engine 2 --iters 1 > /dev/null 2>&1; echo "ncu $?"
