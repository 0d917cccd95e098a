cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out; T=scripts/time_kernel.py
timeout 600 python -m pytest tests/test_gpu_fourd.py -x -q -k "conv2d" --timeout 600 -p no:cacheprovider > gpurun_out/pytest_conv.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_conv.log
{ for tma in 1 0; do for t in 16,64,5,5 32,32,5,5 8,152,5,5 8,512,5,5 16,1024,5,5; do EATSS_CONV_TMA=$tma timeout 120 python $T conv-2d 8192,5 $t --iters 20 2>&1 | tail -1 | sed "s/^/tma$tma /"; done; done; } > gpurun_out/conv_tma.txt 2>&1
tail -2 gpurun_out/pytest_conv.log; cat gpurun_out/conv_tma.txt
timeout 2400 python harness/candidates.py --confirm 7 --out gpurun_out/candidates_r01g.jsonl > gpurun_out/candidates_r01g.log 2>&1; echo "cand $?"
tail -15 gpurun_out/candidates_r01g.log | cut -c1-300
T=scripts/time_kernel.py
{ for at in 0 1; do EATSS_MTC_ATMEM=$at timeout 120 python $T mttkrp 512,32,512,512 1,32,128,32 --engine 2 --iters 20 2>&1 | tail -1 | sed "s/^/atmem$at /"; done; } > gpurun_out/mtc_atmem.txt 2>&1
EATSS_MTC_ATMEM=1 timeout 600 python -m pytest tests/test_gpu_fourd.py -x -q -k "tensor" --timeout 300 -p no:cacheprovider > gpurun_out/pytest_atmem.log 2>&1; echo "pytest atmem rc=$?" >> gpurun_out/pytest_atmem.log
cat gpurun_out/mtc_atmem.txt; tail -2 gpurun_out/pytest_atmem.log
{ for w in 1 0; do for k in "mvt 16384" "atax 16384,16384" "bicg 16384,16384" "gemver 16384"; do set -- $k; EATSS_LOWDIM_WALK=$w timeout 120 python $T $1 $2 16,1024 --engine 1 --iters 10 2>&1 | tail -1 | sed "s/^/walk$w /"; done; done; } > gpurun_out/lowdim_walk.txt 2>&1
timeout 600 python -m pytest tests/test_gpu_lowdim.py -x -q --timeout 300 -p no:cacheprovider > gpurun_out/pytest_lowdim.log 2>&1; echo "pytest lowdim rc=$?" >> gpurun_out/pytest_lowdim.log
cat gpurun_out/lowdim_walk.txt; tail -2 gpurun_out/pytest_lowdim.log
