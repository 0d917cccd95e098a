cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
timeout 900 python -m pytest tests/test_gpu_f16.py -q -x --timeout 600 -p no:cacheprovider 2>&1 | tail -2
ENGINE=4 TILE=256,256,64 timeout 600 python scripts/r02/chunk_ab.py > gpurun_out/r02/chunk_ab_f16.jsonl 2>&1; cat gpurun_out/r02/chunk_ab_f16.jsonl
T=scripts/time_kernel.py
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 12 --csv --log-file gpurun_out/r02/launch_f16b.csv python $T gemm 4000,4000,4000 256,256,64 --engine 4 --iters 3 > /dev/null 2>&1
python - <<'PY'
import csv
rows=[r for r in csv.reader(open('gpurun_out/r02/launch_f16b.csv')) if len(r)>10]
h=rows[0]; ki=h.index('Kernel Name'); mi=h.index('Metric Name'); vi=h.index('Metric Value')
for r in rows[1:]:
    if 'eatss' in r[ki]: print(r[ki][:40], r[mi], r[vi])
PY
timeout 120 python $T gemm 4000,4000,4000 256,256,64 --engine 4 --iters 50 2>&1 | tail -1
