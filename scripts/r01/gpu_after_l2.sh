cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out; T=scripts/time_kernel.py
timeout 300 python harness/nvml_check.py --out gpurun_out/nvml_check_r01.json > gpurun_out/nvml_check.log 2>&1; echo "nvml $?"
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/gemver_launches.csv python $T gemver 16384 16,1024 --engine 1 --iters 1 > /dev/null 2>&1; echo "ncu gemver $?"
cat gpurun_out/nvml_check.log; python - <<'PY'
import csv
rows=list(csv.reader(open('gpurun_out/gemver_launches.csv')))
hdr=[r for r in rows if r and r[0]=='ID'][0]; i=rows.index(hdr)
for r in rows[i+1:]:
    d=dict(zip(hdr,r)); print(d.get('Kernel Name','')[:60], d.get('Metric Name'), d.get('Metric Value'))
PY
