cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out; T=scripts/time_kernel.py
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "jacobi or heat or stencil" --timeout 600 -p no:cacheprovider > gpurun_out/pytest_pdl.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_pdl.log
{ for pdl in 1 0; do
  EATSS_STENCIL_PDL=$pdl timeout 120 python $T heat-3d 120 16,16,32 --tsteps 500 --iters 5 2>&1 | tail -1 | sed "s/^/pdl$pdl /"
  EATSS_STENCIL_PDL=$pdl timeout 120 python $T jacobi-2d 4000 16,1024 --tsteps 500 --iters 5 2>&1 | tail -1 | sed "s/^/pdl$pdl /"
  EATSS_STENCIL_PDL=$pdl timeout 120 python $T heat-3d 512 16,16,32 --tsteps 5 --iters 5 2>&1 | tail -1 | sed "s/^/pdl$pdl /"
  EATSS_STENCIL_PDL=$pdl timeout 120 python $T jacobi-2d 16384 16,1024 --tsteps 10 --iters 3 2>&1 | tail -1 | sed "s/^/pdl$pdl /"
done; } > gpurun_out/pdl_times.txt 2>&1
tail -3 gpurun_out/pytest_pdl.log; cat gpurun_out/pdl_times.txt
