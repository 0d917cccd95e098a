cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out; T=scripts/time_kernel.py
{ timeout 120 python $T mttkrp 512,32,512,512 1,32,128,32 --engine 2 --iters 20 2>&1 | tail -1
  timeout 120 python $T mttkrp 512,32,8192,32 1,32,128,32 --engine 2 --iters 20 2>&1 | tail -1
  timeout 120 python $T mttkrp 512,32,2048,128 1,32,128,32 --engine 2 --iters 20 2>&1 | tail -1
  for k in "mvt 16384" "atax 16384,16384" "bicg 16384,16384" "gemver 16384"; do set -- $k; timeout 120 python $T $1 $2 16,1024 --engine 1 --iters 10 2>&1 | tail -1; done
  timeout 120 python $T gemver 16384 816,16 --engine 1 --iters 5 2>&1 | tail -1
} > gpurun_out/misc_times.txt 2>&1
cat gpurun_out/misc_times.txt
