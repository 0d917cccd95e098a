# raster group of the 3xFP16 GEMM: DRAM bytes per launch (ncu) and time, groups 8 / 16 / 32
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
T="scripts/time_kernel.py gemm 4000,4000,4000 256,256,64 --engine 4 --iters 3"
for g in 8 16 32 4; do
  EATSS_TCM_GROUP=$g timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum --clock-control none -k regex:tc_mma -c 2 --csv python $T > gpurun_out/r02/group_$g.csv 2>/dev/null
  python - $g <<'PY'
import csv,sys
rows=[r for r in csv.reader(open(f'gpurun_out/r02/group_{sys.argv[1]}.csv')) if len(r)>10]
h=rows[0]; mi=h.index('Metric Name'); vi=h.index('Metric Value')
print('group', sys.argv[1], [(r[mi].split('.')[0], r[vi]) for r in rows[-4:]])
PY
done
for rep in 1 2; do for g in 8 16; do echo "== group $g"; EATSS_TCM_GROUP=$g timeout 120 python scripts/time_kernel.py gemm 4000,4000,4000 256,256,64 --engine 4 --iters 100 2>&1 | tail -1; done; done
