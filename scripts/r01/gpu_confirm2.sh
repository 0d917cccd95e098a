cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
TILES="32,512,48;32,512,192;64,256,48;32,512,32;32,512,24;48,192,48;16,1024,24;64,256,16;16,1024,16;64,256,64;32,384,24;32,512,16"
timeout 1500 python harness/sweep.py --tiles "$TILES" --repeats 7 --window 1.0 --out gpurun_out/sweep_confirm_r01b.jsonl > gpurun_out/sweep_confirm_r01b.log 2>&1; echo "confirm $?"
python harness/report.py gpurun_out/sweep_confirm_r01b.jsonl --confirm --json gpurun_out/sweep_confirm_r01b.summary.json | head -40
