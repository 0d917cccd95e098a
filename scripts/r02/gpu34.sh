# 3xFP16 B split through shared memory (parked tile, contiguous K-major column stores) vs direct: parity, A/B, launch times
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
timeout 900 python -m pytest tests/test_gpu_f16.py tests/test_gpu_fullsize.py -k "f16" -q -x -p no:cacheprovider 2>&1 | tail -2
T="scripts/time_kernel.py gemm 4000,4000,4000 256,256,64 --engine 4 --iters 50"
for rep in 1 2 3; do for v in 1 0; do echo "== parked=$v"; EATSS_TCF_PARKED=$v timeout 120 python $T 2>&1 | tail -1; done; done
for v in 1 0; do
EATSS_TCF_PARKED=$v timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:prep_f16 -c 3 --csv python $T > gpurun_out/r02/parked_$v.csv 2>/dev/null
python - $v <<'PY'
import csv,sys
rows=[r for r in csv.reader(open(f'gpurun_out/r02/parked_{sys.argv[1]}.csv')) if len(r)>10]
h=rows[0]; mi=h.index('Metric Name'); vi=h.index('Metric Value')
print('parked', sys.argv[1], [(r[mi], r[vi]) for r in rows[1:]])
PY
done
