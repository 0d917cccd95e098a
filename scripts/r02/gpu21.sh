cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
timeout 300 ncu --set full --clock-control none --import-source on -k regex:prep_f16_kernel -c 1 -o gpurun_out/r02/prof_prep_f16 python scripts/time_kernel.py gemm 4000,4000,4000 256,256,64 --engine 4 --iters 1 > gpurun_out/r02/prof_prep_f16.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:f16_max_kernel -c 1 -o gpurun_out/r02/prof_max_f16 python scripts/time_kernel.py gemm 4000,4000,4000 256,256,64 --engine 4 --iters 1 >> gpurun_out/r02/prof_prep_f16.log 2>&1
tail -3 gpurun_out/r02/prof_prep_f16.log
