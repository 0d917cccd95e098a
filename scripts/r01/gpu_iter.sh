cd $GRAFT_REPO_ROOT
T=scripts/time_kernel.py
timeout 900 python -m pytest tests/test_gpu_lowdim.py -q --timeout 600 -p no:cacheprovider 2>&1 | tail -3
for k in "mvt 16384" "atax 16384,16384" "bicg 16384,16384" "gemver 16384"; do set -- $k; for t in 16,1024 128,512; do timeout 120 python $T $1 $2 $t --engine 1 --iters 10 2>&1 | tail -1; done; done
timeout 120 python $T gemver 16384 816,16 --engine 1 --iters 5 2>&1 | tail -1
