# Evidence pass: per-config device timings (both engines) and ncu captures of the top kernels.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
T=scripts/time_kernel.py
{
for cfg in "gemm 4000,4000,4000" "2mm 4000,4000,4000,4000" "3mm 4000,4000,4000,4000,4000" "syrk 4000,4000"; do
  timeout 120 python $T $cfg 128,256,32 --engine 2 --iters 20 2>&1 | tail -1
  timeout 120 python $T $cfg 16,1024,16 --engine 1 --iters 10 2>&1 | tail -1
done
timeout 120 python $T jacobi-2d 4000 16,1024 --tsteps 500 --iters 3 2>&1 | tail -1
timeout 120 python $T jacobi-2d 16384 16,1024 --tsteps 1 --iters 20 2>&1 | tail -1
timeout 120 python $T heat-3d 120 16,16,32 --tsteps 500 --iters 3 2>&1 | tail -1
timeout 120 python $T heat-3d 512 16,16,32 --tsteps 1 --iters 20 2>&1 | tail -1
timeout 300 python $T ccsd_t_d1 48 1,1,1,48,2,48,48 --engine 2 --iters 5 2>&1 | tail -1
timeout 300 python $T ccsd_t_d1 48 4,4,4,4,4,32,4 --engine 1 --iters 2 2>&1 | tail -1
} > gpurun_out/evidence_times.txt 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tc_mma -s 3 -c 1 -o gpurun_out/prof_tcm_r01c -f python bench.py --steps 3 --warmup 3 --e2e-steps 1 --no-cpu-baseline --no-secondary > /dev/null 2>&1; echo "ncu tcm $?"
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 40 --csv --log-file gpurun_out/ccsd_launches.csv python $T ccsd_t_d1 48 1,1,1,48,2,48,48 --engine 2 --iters 2 > /dev/null 2>&1; echo "ncu ccsd list $?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ccsd_tc -c 1 -o gpurun_out/prof_ccsdtc_r01c -f python $T ccsd_t_d1 8,48,48,48,48,48,48 1,1,1,48,2,48,48 --engine 2 --iters 1 > /dev/null 2>&1; echo "ncu ccsd $?"
cat gpurun_out/evidence_times.txt
