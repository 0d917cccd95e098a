# Evidence pass: all GPU tests, smoke, bench + reference arm, launch list, ncu capture of the headline kernel.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw,temperature.gpu --format=csv > gpurun_out/smi.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 900 python bench.py > gpurun_out/bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench.log
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 5 --warmup 3 --e2e-steps 1 --no-cpu-baseline --no-secondary --no-configs > gpurun_out/bench_ncu.log 2>&1; echo "ncu list $?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tc_mma -s 3 -c 1 -o gpurun_out/prof_tcm_r01g -f python bench.py --steps 3 --warmup 3 --e2e-steps 1 --no-cpu-baseline --no-secondary --no-configs > /dev/null 2>&1; echo "ncu tcm $?"
tail -3 gpurun_out/pytest_gpu.log; tail -2 gpurun_out/smoke.log; tail -c 400 gpurun_out/bench.log
timeout 120 python scripts/time_kernel.py mttkrp 512,32,512,512 1,32,128,32 --engine 2 --iters 20 > gpurun_out/mtc_final.txt 2>&1; cat gpurun_out/mtc_final.txt
