# SURVEY 8(f) row 1 (split x warp-fraction candidate protocol) re-run on the final round-2 executors
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
timeout 3000 python harness/candidates.py --out gpurun_out/r02/candidates_r02_final.jsonl > gpurun_out/r02/candidates_final.log 2>&1; echo "cand rc=$?"
tail -20 gpurun_out/r02/candidates_final.log | cut -c1-300
