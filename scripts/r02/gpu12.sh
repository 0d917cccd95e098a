# compute-sanitizer over every TMA / tcgen05 / bulk-copy executor; ccsd_tc ncu (source-level)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02/sanitizer
S=scripts/r02/sanitize.py
for tool in memcheck racecheck synccheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 20 python $S > gpurun_out/r02/sanitizer/$tool.txt 2>&1; echo "$tool rc=$?" >> gpurun_out/r02/sanitizer/$tool.txt
  tail -4 gpurun_out/r02/sanitizer/$tool.txt
done
T=scripts/time_kernel.py
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ccsd_tc_kernel -s 1 -c 1 -o gpurun_out/r02/prof_ccsdtc_r02 -f python $T ccsd_t_d1 8,48,48,48,48,48,48 1,2,1,48,2,48,48 --engine 2 --iters 1 > /dev/null 2>&1; echo "ncu ccsd $?"
