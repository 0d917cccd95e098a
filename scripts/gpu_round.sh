cd $GRAFT_REPO_ROOT
timeout 600 python bench.py > gpurun_out/bench_r01.json 2> gpurun_out/bench_r01.err; echo "bench exit $?"; cat gpurun_out/bench_r01.json
timeout 600 python bench.py --impl reference --steps 5 --warmup 1 > gpurun_out/bench_ref_r01.json 2>&1; cat gpurun_out/bench_ref_r01.json | tail -1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/launches_r01.csv python bench.py --steps 10 --warmup 3 --e2e-steps 2 --no-cpu-baseline > /dev/null 2>&1; echo "ncu1 $?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:contract_staged -s 3 -c 1 -o gpurun_out/prof_gemm_r01b python bench.py --steps 3 --warmup 3 --e2e-steps 1 --no-cpu-baseline > /dev/null 2>&1; echo "ncu2 $?"
timeout 600 ncu --set full --clock-control none -k regex:jacobi2d_sweep -s 5 -c 1 -o gpurun_out/prof_jacobi_r01b python scripts/time_kernel.py jacobi-2d 16384 16,1024 --tsteps 10 --iters 1 > /dev/null 2>&1; echo "ncu3 $?"
timeout 600 ncu --set full --clock-control none -k regex:heat3d_sweep -s 5 -c 1 -o gpurun_out/prof_heat_r01 python scripts/time_kernel.py heat-3d 512 16,16,32 --tsteps 5 --iters 1 > /dev/null 2>&1; echo "ncu4 $?"
timeout 600 ncu --set full --clock-control none -k regex:ccsd -s 1 -c 1 -o gpurun_out/prof_ccsd_r01b python scripts/time_kernel.py ccsd_t_d1 48 4,4,4,4,4,32,4 --iters 1 > /dev/null 2>&1; echo "ncu5 $?"
