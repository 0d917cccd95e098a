cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_tensor.py -q --timeout 600 -p no:cacheprovider -k "ccsd or syrk" 2>&1 | tail -3
T=scripts/time_kernel.py
timeout 120 python $T syrk 4000,4000 16,1024,16 --engine 1 --iters 10 2>&1 | tail -1
timeout 120 python $T gemm 4000,4000,4000 16,1024,16 --engine 1 --iters 10 2>&1 | tail -1
timeout 900 python scripts/ccsd_variants.py
timeout 900 python harness/l2power.py --phase power --count 120 2>&1 | tail -2
timeout 900 ncu --metrics lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_op_read.sum,gpu__time_duration.sum --clock-control none -k regex:'contract|jacobi2d' --csv --log-file gpurun_out/l2power_l2.csv python harness/l2power.py --phase l2 > /dev/null 2>&1; echo "ncu l2 $?"
python harness/l2power.py --phase report 2>&1 | tail -30
