# mttkrp / conv-2d: GPU parity tests, tile timings, ncu captures of the EATSS-tile kernels.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
T=scripts/time_kernel.py
timeout 900 python -m pytest tests/test_gpu_fourd.py -x -q --timeout 600 -p no:cacheprovider > gpurun_out/pytest_fourd.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_fourd.log
{
for t in 128,32,16,16 512,32,4,4 512,32,8,8 32,32,32,32 64,32,16,16 32,32,16,16 16,32,16,16 64,32,32,32 128,32,32,32; do timeout 120 python $T mttkrp 512,32,512,512 $t --iters 20 2>&1 | tail -1; done
for t in 16,64,5,5 8,152,5,5 4,480,4,4 32,32,5,5 16,1024,5,5 32,256,5,5 64,128,5,5 8,512,5,5; do timeout 120 python $T conv-2d 8192,5 $t --iters 20 2>&1 | tail -1; done
} > gpurun_out/fourd_times.txt 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:mttkrp_kernel -s 3 -c 1 -o gpurun_out/prof_mttkrp_r01 -f python $T mttkrp 512,32,512,512 128,32,16,16 --iters 1 > /dev/null 2>&1; echo "ncu mttkrp $?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:conv2d_kernel -s 3 -c 1 -o gpurun_out/prof_conv2d_r01 -f python $T conv-2d 8192,5 16,64,5,5 --iters 1 > /dev/null 2>&1; echo "ncu conv $?"
tail -3 gpurun_out/pytest_fourd.log; cat gpurun_out/fourd_times.txt
