# 3xFP16 row operands read once (bulk-staged rows, max + split fused in the first launch): parity, A/B, ncu
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
timeout 900 python -m pytest tests/test_gpu_f16.py tests/test_gpu_fullsize.py -k "f16" -q -x --timeout 600 -p no:cacheprovider 2>&1 | tail -2
T=scripts/time_kernel.py
for f in 1 0; do for i in 1 2; do
  r=$(EATSS_TCF_STAGED_ROWS=$f timeout 120 python $T gemm 4000,4000,4000 256,256,64 --engine 4 --iters 50 2>&1 | tail -1); echo "staged $f: $r"
  r=$(EATSS_TCF_STAGED_ROWS=$f timeout 120 python $T syrk 4000,4000 256,256,64 --engine 4 --iters 50 2>&1 | tail -1); echo "staged $f: $r"
done; done
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 12 --csv --log-file gpurun_out/r02/launch_f16c.csv python $T gemm 4000,4000,4000 256,256,64 --engine 4 --iters 3 > /dev/null 2>&1
python - <<'PY'
import csv
rows=[r for r in csv.reader(open('gpurun_out/r02/launch_f16c.csv')) if len(r)>10]
h=rows[0]; ki=h.index('Kernel Name'); mi=h.index('Metric Name'); vi=h.index('Metric Value')
for r in rows[1:10]:
    if 'eatss' in r[ki]: print(r[ki][:40], r[mi], r[vi])
PY
