# Round-2 pass 4: full GPU suite after the tcgen05 rework, bench, ncu of the headline GEMM at chunk 128 / 512.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
timeout 1800 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/r02/pytest_gpu4.log 2>&1; echo "rc=$?" >> gpurun_out/r02/pytest_gpu4.log
timeout 900 python bench.py > gpurun_out/r02/bench4.log 2>&1; echo "bench rc=$?" >> gpurun_out/r02/bench4.log
T=scripts/time_kernel.py
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tc_mma -s 2 -c 1 -o gpurun_out/r02/prof_tcm_c128 -f python $T gemm 4000,4000,4000 256,256,32 --engine 2 --iters 1 > /dev/null 2>&1; echo "ncu c128 $?"
EATSS_TCM_CHUNK_K=512 timeout 600 ncu --set full --clock-control none --import-source on -k regex:tc_mma -s 2 -c 1 -o gpurun_out/r02/prof_tcm_c512 -f python $T gemm 4000,4000,4000 256,256,32 --engine 2 --iters 1 > /dev/null 2>&1; echo "ncu c512 $?"
tail -3 gpurun_out/r02/pytest_gpu4.log; grep -E "FAILED|Error" gpurun_out/r02/pytest_gpu4.log | head -20; tail -c 300 gpurun_out/r02/bench4.log
