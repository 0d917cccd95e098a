# jacobi-2d N=4000 T=500, L2 hints on/off, same box, interleaved (time_kernel: graph of 1000 sweeps per call)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
for rep in 1 2 3 4; do for v in 1 0; do
  echo "== l2hint=$v"; EATSS_JACOBI_L2HINT=$v timeout 120 python scripts/time_kernel.py jacobi-2d 4000 16,1024 --tsteps 500 --iters 5 2>&1 | tail -1 | cut -c1-100
done; done
