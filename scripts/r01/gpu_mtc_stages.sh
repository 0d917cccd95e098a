cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out; T=scripts/time_kernel.py
{ for st in 3 4 5 6; do for dbg in 0 2; do EATSS_MTC_STAGES=$st EATSS_MTC_DBG=$dbg timeout 120 python $T mttkrp 512,32,512,512 1,32,128,32 --engine 2 --iters 20 2>&1 | tail -1 | sed "s/^/st$st dbg$dbg /"; done; done; } > gpurun_out/mtc_stages.txt 2>&1
cat gpurun_out/mtc_stages.txt
