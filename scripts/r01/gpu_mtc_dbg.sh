cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out; T=scripts/time_kernel.py
{ for dbg in 0 1 2 3; do EATSS_MTC_DBG=$dbg timeout 120 python $T mttkrp 512,32,512,512 1,32,128,32 --engine 2 --iters 20 2>&1 | tail -1 | sed "s/^/dbg$dbg /"; done; } > gpurun_out/mtc_dbg.txt 2>&1
cat gpurun_out/mtc_dbg.txt
