cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 600 python harness/sizes.py --kind conv-2d --window 0.6 --out gpurun_out/sizes4d_r01.jsonl > gpurun_out/sizes4d.log 2>&1; echo "conv $?"
timeout 600 python harness/sizes.py --kind mttkrp --window 0.6 --out gpurun_out/sizes4d_r01.jsonl >> gpurun_out/sizes4d.log 2>&1; echo "mttkrp $?"
cat gpurun_out/sizes4d_r01.jsonl | python -c "
import sys,json
for l in sys.stdin:
    r=json.loads(l); print(r['kind'], r['n'], r['arm'], r['tiles'], round(r['ms'],3), round(r['tflops'],1), round(r['watts']), round(r['ppw'],1))"
