# round-2 final evidence pass after the jacobi L2 hints (same as gpu39.sh; compute-sanitizer is closed on the pool)
# summaries of the headline and config kernels (details pages kept, .ncu-rep dropped), compute-sanitizer
cd $GRAFT_REPO_ROOT; O=gpurun_out/r02/final4; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw,temperature.gpu --format=csv > $O/smi.txt 2>&1
lscpu | head -20 > $O/lscpu.txt
timeout 3000 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 1200 > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest_gpu.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -2 $O/smoke.log
timeout 1500 python bench.py > $O/bench.log 2>&1; echo "bench rc=$?"; tail -c 400 $O/bench.log
timeout 900 python bench.py --impl reference > $O/bench_ref.log 2>&1; echo "ref rc=$?"; tail -c 300 $O/bench_ref.log
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 400 --csv --log-file $O/launches_bench_r02.csv python bench.py --steps 3 --warmup 3 --no-configs --no-secondary --no-cpu-baseline --e2e-steps 1 > $O/bench_ncu.log 2>&1; echo "ncu list rc=$?"
T=scripts/time_kernel.py
cap() {  # name, kernel regex, time_kernel args...
  n=$1; k=$2; shift 2
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$k -s 1 -c 1 -o $O/prof_$n -f python $T "$@" > /dev/null 2>&1; echo "ncu $n rc=$?"
  python scripts/ncu_summary.py $O/prof_$n.ncu-rep > $O/$n.ncu.json 2>/dev/null
  ncu -i $O/prof_$n.ncu-rep --page details --csv > $O/prof_$n.details.csv 2>/dev/null
  rm -f $O/prof_$n.ncu-rep
}
cap tcm_f16_r02h "tc_mma_kernel" gemm 4000,4000,4000 256,256,64 --engine 4 --iters 2
cap prep_f16_r02h "prep_f16_kernel" gemm 4000,4000,4000 256,256,64 --engine 4 --iters 2
cap max_f16_r02h "f16_max_kernel" gemm 4000,4000,4000 256,256,64 --engine 4 --iters 2
cap simt_gemm_r02h "contract_staged" gemm 4000,4000,4000 16,1024,16 --engine 1 --iters 2
cap ccsdtc_r02h "ccsd_tc_kernel" ccsd_t_d1 8,48,48,48,48,48,48 1,2,1,48,2,48,48 --engine 2 --iters 1
cap heat_r02h "heat3d_staged" heat-3d 120 16,16,32 --tsteps 2 --iters 1
exit 0
S=scripts/r02/sanitize.py
mkdir -p $O/sanitizer
for tool in memcheck synccheck racecheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python $S > $O/sanitizer/$tool.txt 2>&1; echo "$tool rc=$?" >> $O/sanitizer/$tool.txt
  tail -2 $O/sanitizer/$tool.txt
done
du -sh $O
