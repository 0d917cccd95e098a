# tc_mma: L2 prefetch of each unit's C rows EATSS_TCM_CPF chunks before its epilogue (0 = off): parity, A/B
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
timeout 1500 python -m pytest tests/test_gpu_f16.py tests/test_gpu_tensor.py tests/test_gpu_fullsize.py -q -x -p no:cacheprovider 2>&1 | tail -2
T="scripts/time_kernel.py gemm 4000,4000,4000 256,256,64 --engine 4 --iters 100"
T2="scripts/time_kernel.py gemm 4000,4000,4000 256,256,32 --engine 2 --iters 100"
for rep in 1 2 3; do for v in 2 0 4; do echo "== cpf=$v"; EATSS_TCM_CPF=$v timeout 120 python $T 2>&1 | tail -1; EATSS_TCM_CPF=$v timeout 120 python $T2 2>&1 | tail -1; done; done
for v in 2 0; do EATSS_TCM_CPF=$v timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum --clock-control none -k regex:tc_mma -c 2 --csv python $T > gpurun_out/r02/cpf_$v.csv 2>/dev/null; echo "cpf $v"; grep -o '"gpu__time_duration.sum","[^"]*","[0-9.]*"' gpurun_out/r02/cpf_$v.csv | tail -1; done
