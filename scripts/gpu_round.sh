cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
#timeout 1500 python -m pytest tests -m gpu -q --timeout 600 -p no:cacheprovider 2>&1 | tail -4
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench exit $?"; cat gpurun_out/bench.json; tail -3 gpurun_out/bench.err
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:'split_kernel|tail_prepass|tc_mma|contract' --csv --log-file gpurun_out/launches.csv python bench.py --steps 5 --warmup 3 --e2e-steps 1 --no-cpu-baseline --no-secondary > /dev/null 2>&1; echo "ncu1 $?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tc_mma -s 3 -c 1 -o gpurun_out/prof_tcm python bench.py --steps 3 --warmup 3 --e2e-steps 1 --no-cpu-baseline --no-secondary > /dev/null 2>&1; echo "ncu2 $?"
