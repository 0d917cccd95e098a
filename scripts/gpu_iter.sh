cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_lowdim.py tests/test_gpu_host.py -q --timeout 600 -p no:cacheprovider 2>&1 | tail -5
T=scripts/time_kernel.py
for k in "mvt 4000" "atax 4000,4000" "bicg 4000,4000" "gemver 4000"; do set -- $k; for t in 16,1024 64,512 256,256; do timeout 120 python $T $1 $2 $t --engine 1 --iters 20 2>&1 | tail -1; done; done
timeout 120 python $T gemver 4000 816,16 --engine 1 --iters 20 2>&1 | tail -1
