# jacobi-2d at L2-sized grids: evict-first source windows + evict-last destination stores vs no hints
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_waf.py -q -p no:cacheprovider -k "jacobi" 2>&1 | tail -1
for rep in 1 2 3; do for v in 1 0; do
  echo "== l2hint=$v"; EATSS_JACOBI_L2HINT=$v timeout 120 python scripts/time_kernel.py jacobi-2d 4000 16,1024 --tsteps 500 --iters 3 2>&1 | tail -1 | cut -c1-100
done; done
for v in 1 0; do EATSS_JACOBI_L2HINT=$v timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:jacobi2d_staged -s 20 -c 2 --csv python scripts/time_kernel.py jacobi-2d 4000 16,1024 --tsteps 20 --iters 1 > gpurun_out/r02/jl2_$v.csv 2>/dev/null; echo "ncu l2hint=$v"; python - $v <<'PY'
import csv,sys
rows=[r for r in csv.reader(open(f'gpurun_out/r02/jl2_{sys.argv[1]}.csv')) if len(r)>10]
h=rows[0]; mi=h.index('Metric Name'); vi=h.index('Metric Value')
print([(r[mi].split('.')[0], r[vi]) for r in rows[-4:]])
PY
done
