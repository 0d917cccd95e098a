cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 12 --csv --log-file gpurun_out/tcm2_launches.csv python scripts/time_kernel.py gemm 4000,4000,4000 128,256,32 --engine 2 --iters 2 > /dev/null 2>&1; echo "ncu1 $?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tc_mma -s 2 -c 1 -o gpurun_out/prof_tcm2 python scripts/time_kernel.py gemm 4000,4000,4000 128,256,32 --engine 2 --iters 2 > /dev/null 2>&1; echo "ncu2 $?"
