cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out; T=scripts/time_kernel.py
timeout 600 python -m pytest tests/test_gpu_fourd.py -x -q -k "tensor" --timeout 300 -p no:cacheprovider > gpurun_out/pytest_mtc.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_mtc.log
timeout 120 python $T mttkrp 512,32,512,512 1,32,128,32 --engine 2 --iters 20 > gpurun_out/mtc_times.txt 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:mttkrp_tc_kernel -s 2 -c 1 -o gpurun_out/prof_mttkrp_tc_r01 -f python $T mttkrp 512,32,512,512 1,32,128,32 --engine 2 --iters 1 > /dev/null 2>&1; echo "ncu $?"
tail -3 gpurun_out/pytest_mtc.log; cat gpurun_out/mtc_times.txt
