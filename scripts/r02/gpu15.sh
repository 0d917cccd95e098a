cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
T=scripts/time_kernel.py
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 12 --csv --log-file gpurun_out/r02/launch_f16.csv python $T gemm 4000,4000,4000 256,256,64 --engine 4 --iters 3 > /dev/null 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 12 --csv --log-file gpurun_out/r02/launch_tf32.csv python $T gemm 4000,4000,4000 256,256,32 --engine 2 --iters 3 > /dev/null 2>&1
python - <<'PY'
import csv
for f in ('gpurun_out/r02/launch_f16.csv','gpurun_out/r02/launch_tf32.csv'):
    rows=[r for r in csv.reader(open(f)) if len(r)>10]
    h=rows[0]; ki=h.index('Kernel Name'); mi=h.index('Metric Name'); vi=h.index('Metric Value')
    for r in rows[1:]:
        print(f.split('/')[-1], r[ki][:40], r[mi], r[vi])
PY
