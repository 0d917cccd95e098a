# Full evidence pass (round 1): tests, smoke, bench + reference arm, launch list, ncu captures, f-row harnesses.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
T=scripts/time_kernel.py
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw,temperature.gpu --format=csv > gpurun_out/smi.txt 2>&1
timeout 1800 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 900 python bench.py > gpurun_out/bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench.log
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 5 --warmup 3 --e2e-steps 1 --no-cpu-baseline --no-secondary --no-configs > gpurun_out/bench_ncu.log 2>&1; echo "ncu list $?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tc_mma -s 3 -c 1 -o gpurun_out/prof_tcm_r01f -f python bench.py --steps 3 --warmup 3 --e2e-steps 1 --no-cpu-baseline --no-secondary --no-configs > /dev/null 2>&1; echo "ncu tcm $?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ccsd_tc -c 1 -o gpurun_out/prof_ccsdtc_r01f -f python $T ccsd_t_d1 8,48,48,48,48,48,48 1,2,1,48,2,48,48 --engine 2 --iters 1 > /dev/null 2>&1; echo "ncu ccsd $?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:jacobi2d_staged -s 2 -c 1 -o gpurun_out/prof_jacobi_r01f -f python $T jacobi-2d 16384 16,1024 --tsteps 2 --iters 1 > /dev/null 2>&1; echo "ncu jacobi $?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:heat3d_staged -s 2 -c 1 -o gpurun_out/prof_heat_r01f -f python $T heat-3d 512 16,16,32 --tsteps 2 --iters 1 > /dev/null 2>&1; echo "ncu heat $?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:lowdim_kernel -s 1 -c 1 -o gpurun_out/prof_mvt_r01f -f python $T mvt 16384 16,1024 --iters 1 > /dev/null 2>&1; echo "ncu mvt $?"
{
for k in "mvt 16384" "atax 16384,16384" "bicg 16384,16384" "gemver 16384"; do set -- $k; timeout 120 python $T $1 $2 16,1024 --engine 1 --iters 10 2>&1 | tail -1; done
timeout 120 python $T gemver 16384 816,16 --engine 1 --iters 5 2>&1 | tail -1
} > gpurun_out/lowdim_times.txt 2>&1
timeout 1500 python harness/candidates.py --out gpurun_out/candidates_r01f.jsonl > gpurun_out/candidates.log 2>&1; echo "cand $?"
timeout 900 python harness/l2power.py --phase power --count 120 --kinds mvt --power gpurun_out/l2power_mvt_power.jsonl > /dev/null 2>&1
timeout 900 ncu --metrics lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_op_read.sum,gpu__time_duration.sum --clock-control none -k regex:'lowdim_kernel' --csv --log-file gpurun_out/l2power_mvt_l2.csv python harness/l2power.py --phase l2 --kinds mvt --power gpurun_out/l2power_mvt_power.jsonl > /dev/null 2>&1; echo "ncu l2 $?"
tail -3 gpurun_out/pytest_gpu.log; tail -2 gpurun_out/smoke.log; tail -c 600 gpurun_out/bench.log
