cd $GRAFT_REPO_ROOT
T="python scripts/time_kernel.py"
$T gemm 4000,4000,4000 16,1024,16; $T gemm 4000,4000,4000 32,32,32
$T 2mm 4000,4000,4000,4000 16,1024,16; $T 3mm 4000,4000,4000,4000,4000 16,1024,16; $T syrk 4000,4000 16,1024,16
$T jacobi-2d 4000 16,1024 --tsteps 500 --iters 3; $T jacobi-2d 4000 32,32 --tsteps 500 --iters 3
$T jacobi-2d 16384 16,1024 --tsteps 20 --iters 3
$T heat-3d 120 16,16,32 --tsteps 500 --iters 3; $T heat-3d 120 32,32,32 --tsteps 500 --iters 3; $T heat-3d 512 16,16,32 --tsteps 10 --iters 3
$T ccsd_t_d1 48 4,4,4,4,4,32,4 --iters 2; $T ccsd_t_d1 48 32,32,32,32,32,32,32 --iters 1
timeout 600 python bench.py --steps 200 --warmup 10 > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench exit $?"; cat gpurun_out/bench.json
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/launches.csv python bench.py --steps 10 --warmup 3 --e2e-steps 2 --no-cpu-baseline > /dev/null 2>&1; echo "ncu1 $?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:contract_staged -s 3 -c 1 -o gpurun_out/prof_gemm_r01 python bench.py --steps 3 --warmup 3 --e2e-steps 1 --no-cpu-baseline > /dev/null 2>&1; echo "ncu2 $?"
timeout 600 ncu --set full --clock-control none -k regex:jacobi2d_sweep -s 5 -c 1 -o gpurun_out/prof_jacobi_r01 python scripts/time_kernel.py jacobi-2d 16384 16,1024 --tsteps 10 --iters 1 > /dev/null 2>&1; echo "ncu3 $?"
timeout 600 ncu --set full --clock-control none -k regex:ccsd -s 1 -c 1 -o gpurun_out/prof_ccsd_r01 python scripts/time_kernel.py ccsd_t_d1 48 4,4,4,4,4,32,4 --iters 1 > /dev/null 2>&1; echo "ncu4 $?"
