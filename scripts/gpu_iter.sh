cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_tensor.py -q --timeout 600 -p no:cacheprovider -k "heat or stencil or ccsd or tcm" 2>&1 | tail -3
T=scripts/time_kernel.py
timeout 300 python $T ccsd_t_d1 48 1,1,1,48,2,48,48 --engine 2 --iters 5 2>&1 | tail -1
EATSS_CCSD_TC_DBG=7 timeout 300 python $T ccsd_t_d1 48 1,1,1,48,2,48,48 --engine 2 --iters 5 2>&1 | tail -1
EATSS_CCSD_TC_DBG=2 timeout 300 python $T ccsd_t_d1 48 1,1,1,48,2,48,48 --engine 2 --iters 5 2>&1 | tail -1
timeout 120 python $T heat-3d 512 16,16,32 --tsteps 5 --iters 5 2>&1 | tail -1
timeout 120 python $T gemm 4000,4000,4000 128,256,32 --engine 2 --iters 20 2>&1 | tail -1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:ccsd_tc -c 1 -o gpurun_out/prof_ccsd_r01d -f python $T ccsd_t_d1 4,48,48,48,48,48,48 1,1,1,48,2,48,48 --engine 2 --iters 1 > /dev/null 2>&1; echo "ncu $?"
timeout 1500 python harness/candidates.py --out gpurun_out/candidates_r01.jsonl 2>&1 | tail -8
