cd $GRAFT_REPO_ROOT
timeout 1200 python -m pytest tests -m gpu -q --timeout 600 -p no:cacheprovider 2>&1 | tail -3
timeout 600 python bench.py > gpurun_out/bench_r01c.json 2> gpurun_out/bench_r01c.err; echo "bench exit $?"; cat gpurun_out/bench_r01c.json; tail -3 gpurun_out/bench_r01c.err
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 80 --csv --log-file gpurun_out/launches_r01c.csv python bench.py --steps 10 --warmup 3 --e2e-steps 2 --no-cpu-baseline --no-secondary > /dev/null 2>&1; echo "ncu1 $?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tc_mma -s 3 -c 1 -o gpurun_out/prof_tcm_r01 python bench.py --steps 3 --warmup 3 --e2e-steps 1 --no-cpu-baseline --no-secondary > /dev/null 2>&1; echo "ncu2 $?"
