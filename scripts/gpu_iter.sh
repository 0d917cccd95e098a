cd $GRAFT_REPO_ROOT
T=scripts/time_kernel.py
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_host.py -q --timeout 600 -p no:cacheprovider -k "heat or gemm or syrk or 2mm or 3mm or host" 2>&1 | tail -3
timeout 120 python $T heat-3d 120 16,16,32 --tsteps 500 --iters 3 2>&1 | tail -1
EATSS_HEAT_PERSISTENT=0 timeout 120 python $T heat-3d 120 16,16,32 --tsteps 500 --iters 3 2>&1 | tail -1
timeout 120 python $T heat-3d 120 8,16,80 --tsteps 500 --iters 3 2>&1 | tail -1
timeout 120 python $T heat-3d 256 16,16,32 --tsteps 50 --iters 3 2>&1 | tail -1
EATSS_HEAT_PERSISTENT=0 timeout 120 python $T heat-3d 256 16,16,32 --tsteps 50 --iters 3 2>&1 | tail -1
for t in 16,1024,16 32,512,32 32,32,32; do timeout 120 python $T gemm 4000,4000,4000 $t --engine 1 --iters 10 2>&1 | tail -1; done
