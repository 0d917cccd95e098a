# End-of-round evidence: all GPU tests, smoke, bench + reference arm, launch list, ncu captures of the
# headline GEMM and of the kernels changed late in the round (conv-2d TMA window, mvt column walk).
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out; T=scripts/time_kernel.py
bash scripts/gpu_final.sh
timeout 600 ncu --set full --clock-control none --import-source on -k regex:conv2d_kernel -s 3 -c 1 -o gpurun_out/prof_conv2d_r01g -f python $T conv-2d 8192,5 16,64,5,5 --iters 1 > /dev/null 2>&1; echo "ncu conv $?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:lowdim_kernel -s 1 -c 1 -o gpurun_out/prof_mvt_r01g -f python $T mvt 16384 16,1024 --engine 1 --iters 1 > /dev/null 2>&1; echo "ncu mvt $?"
