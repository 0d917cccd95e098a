# 3xTF32 with the lo halves formed on chip: parity, timing A/B against the materialised split, ncu bytes
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
timeout 900 python -m pytest tests/test_gpu_tensor.py tests/test_gpu_fullsize.py -q -x --timeout 600 -p no:cacheprovider 2>&1 | tail -3
T=scripts/time_kernel.py
for f in 1 0; do for t in 256,256,32 128,256,32 256,256,16; do
  r=$(EATSS_TCM_FUSE=$f timeout 120 python $T gemm 4000,4000,4000 $t --engine 2 --iters 50 2>&1 | tail -1); echo "fuse $f $t: $r"
done; done
for st in 3 4; do r=$(EATSS_TCM_STAGES=$st timeout 120 python $T gemm 4000,4000,4000 256,256,32 --engine 2 --iters 50 2>&1 | tail -1); echo "fuse 1 stages $st: $r"; done
EATSS_TCM_PROF=1 timeout 120 python $T gemm 4000,4000,4000 256,256,32 --engine 2 --iters 2 2>&1 | grep prof | tail -1
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 8 --csv --log-file gpurun_out/r02/launch_tf32_fused.csv python $T gemm 4000,4000,4000 256,256,32 --engine 2 --iters 3 > /dev/null 2>&1
python - <<'PY'
import csv
rows=[r for r in csv.reader(open('gpurun_out/r02/launch_tf32_fused.csv')) if len(r)>10]
h=rows[0]; ki=h.index('Kernel Name'); mi=h.index('Metric Name'); vi=h.index('Metric Value')
for r in rows[1:]:
    if 'eatss' in r[ki]: print(r[ki][:40], r[mi], r[vi])
PY
