# A/B of the fused prep launch (operand splits + tail pre-pass) against separate launches:
# abtmp/{old,new}.so are the two library builds, interleaved bench runs of the headline step.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out; L=paper_conf_cgo_jayaweerakwk24_b200/libeatss.so
for rep in 1 2 3; do for v in old new; do cp abtmp/$v.so $L; echo -n "$v "; timeout 200 python bench.py --no-cpu-baseline --no-secondary --no-configs --steps 300 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value'],2),round(d['ms_per_step'],4),round(d['roofline']['achieved'],1),d['clocks']['sm_mhz'],d['gpu_launches'])"; done; done > gpurun_out/prep_ab.txt 2>&1
cp abtmp/new.so $L
timeout 1000 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/gpu_tests_prep.log 2>&1; echo "pytest rc=$?" >> gpurun_out/gpu_tests_prep.log
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches_prep.csv python bench.py --no-cpu-baseline --no-secondary --no-configs --steps 10 --warmup 3 --e2e-steps 1 > /dev/null 2>&1
cat gpurun_out/prep_ab.txt; tail -3 gpurun_out/gpu_tests_prep.log
