cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1500 python harness/candidates.py --kinds mttkrp,conv-2d --out gpurun_out/candidates_fourd_r01.jsonl > gpurun_out/candidates_fourd.log 2>&1; echo "cand $?"
tail -30 gpurun_out/candidates_fourd.log
