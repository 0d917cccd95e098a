# tensor engines: evict-last L2 hints on the split operands (prep stores, GEMM TMA loads) vs none
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
timeout 1500 python -m pytest tests/test_gpu_f16.py tests/test_gpu_tensor.py tests/test_gpu_fullsize.py tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "f16 or tensor or fullsize or jacobi" 2>&1 | tail -1
T="scripts/time_kernel.py gemm 4000,4000,4000 256,256,64 --engine 4 --iters 100"
T2="scripts/time_kernel.py gemm 4000,4000,4000 256,256,32 --engine 2 --iters 100"
for rep in 1 2 3; do for v in 1 0; do echo "== l2hint=$v"; EATSS_TCM_L2HINT=$v timeout 120 python $T 2>&1 | tail -1; EATSS_TCM_L2HINT=$v timeout 120 python $T2 2>&1 | tail -1; done; done
for v in 1 0; do EATSS_TCM_L2HINT=$v timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"tc_mma|prep_f16|f16_max" -c 6 --csv python $T > gpurun_out/r02/tl2_$v.csv 2>/dev/null; echo "ncu l2hint=$v"; python - $v <<'PY'
import csv,sys
rows=[r for r in csv.reader(open(f'gpurun_out/r02/tl2_{sys.argv[1]}.csv')) if len(r)>10]
h=rows[0]; ki=h.index('Kernel Name'); mi=h.index('Metric Name'); vi=h.index('Metric Value')
for r in rows[-9:]: print(r[ki][:22], r[mi].split('.')[0], r[vi])
PY
done
for rep in 1 2; do for v in 1 0; do echo "== bench l2hint=$v"; EATSS_TCM_L2HINT=$v timeout 300 python bench.py --steps 100 --warmup 5 --no-configs --no-secondary --no-cpu-baseline --e2e-steps 2 2>&1 | grep '^{' | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print(round(d['ms_per_step'],4), round(d['value'],1), round(r['frac'],3))"; done; done
