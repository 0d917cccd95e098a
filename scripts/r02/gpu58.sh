# conv-2d: evict-last TMA windows + streamed outputs vs none -- parity, same-box A/B, DRAM bytes
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
timeout 900 python -m pytest tests/test_gpu_fourd.py -q -p no:cacheprovider -k "conv" 2>&1 | tail -1
for rep in 1 2 3; do for v in 1 0; do echo "== conv l2hint=$v"; EATSS_CONV_L2HINT=$v timeout 120 python scripts/time_kernel.py conv-2d 8192,5 16,64,5,5 --iters 100 2>&1 | tail -1 | cut -c1-100; done; done
for v in 1 0; do EATSS_CONV_L2HINT=$v timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:conv2d_kernel -c 1 --csv python scripts/time_kernel.py conv-2d 8192,5 16,64,5,5 --iters 1 > gpurun_out/r02/cv_$v.csv 2>/dev/null; echo "ncu conv l2hint=$v"; python - $v <<'PY'
import csv,sys
rows=[r for r in csv.reader(open(f'gpurun_out/r02/cv_{sys.argv[1]}.csv')) if len(r)>10]
h=rows[0]; mi=h.index('Metric Name'); vi=h.index('Metric Value')
print([(r[mi].split('.')[0], r[vi]) for r in rows[-3:]])
PY
done
