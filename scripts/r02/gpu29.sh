# round-2 evidence pass (gpu26 + details pages, large .ncu-rep files dropped so gpurun_out stays under 64 MiB)
# captures of the headline kernels (summarised by scripts/ncu_summary.py)
cd $GRAFT_REPO_ROOT; O=gpurun_out/r02/final; mkdir -p $O
timeout 3000 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 1200 > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest_gpu.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -2 $O/smoke.log
timeout 1500 python bench.py > $O/bench.log 2>&1; echo "bench rc=$?"; tail -c 600 $O/bench.log
timeout 900 python bench.py --impl reference > $O/bench_ref.log 2>&1; echo "ref rc=$?"; tail -c 400 $O/bench_ref.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches_bench_r02.csv python bench.py --steps 3 --warmup 3 --no-configs --no-secondary --no-cpu-baseline --e2e-steps 1 > $O/bench_ncu.log 2>&1; echo "ncu list rc=$?"
T=scripts/time_kernel.py
cap() {  # name, kernel regex, time_kernel args...
  n=$1; k=$2; shift 2
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$k -s 1 -c 1 -o $O/prof_$n -f python $T "$@" > /dev/null 2>&1; echo "ncu $n rc=$?"
  python scripts/ncu_summary.py $O/prof_$n.ncu-rep > $O/$n.ncu.json 2>/dev/null
}
cap tcm_f16_r02 "tc_mma_kernel" gemm 4000,4000,4000 256,256,64 --engine 4 --iters 2
cap prep_f16_r02 "prep_f16_kernel" gemm 4000,4000,4000 256,256,64 --engine 4 --iters 2
cap max_f16_r02 "f16_max_kernel" gemm 4000,4000,4000 256,256,64 --engine 4 --iters 2
cap tcm_tf32_r02 "tc_mma_kernel" gemm 4000,4000,4000 256,256,32 --engine 2 --iters 2
cap prep_tf32_r02 "prep_kernel" gemm 4000,4000,4000 256,256,32 --engine 2 --iters 2
cap simt_gemm_r02 "contract_staged" gemm 4000,4000,4000 16,1024,16 --engine 1 --iters 2
cap ccsdtc_r02 "ccsd_tc_kernel" ccsd_t_d1 8,48,48,48,48,48,48 1,2,1,48,2,48,48 --engine 2 --iters 1
for f in $O/prof_*.ncu-rep; do n=$(basename $f .ncu-rep); ncu -i $f --page details --csv > $O/${n}.details.csv 2>/dev/null; done
rm -f $O/prof_tcm_tf32_r02.ncu-rep $O/prof_prep_*.ncu-rep $O/prof_max_*.ncu-rep
for f in $O/prof_*.ncu-rep; do s=$(stat -c %s $f); [ $s -gt 15000000 ] && rm -f $f; done
ls -la $O; du -sh $O
