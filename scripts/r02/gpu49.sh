# the fp32 3,375-variant sweep (config 2) re-run on the round-2 SIMT executor (bulk copies spread over
# the warps, two CTAs per SM pinned), then a 7-repeat confirmation of its leaders
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
timeout 3000 python harness/sweep.py --kind gemm --n 4000 --out gpurun_out/r02/sweep_gemm4000_f32_r02.jsonl > gpurun_out/r02/sweep_f32_r02.log 2>&1; echo "sweep rc=$?"
tail -2 gpurun_out/r02/sweep_f32_r02.log
python harness/report.py gpurun_out/r02/sweep_gemm4000_f32_r02.jsonl --json gpurun_out/r02/sweep_gemm4000_f32_r02.summary.json > /dev/null 2>&1
TILES=$(python - <<'PY'
import json
s=json.load(open('gpurun_out/r02/sweep_gemm4000_f32_r02.summary.json'))
d=s.get('drift_corrected',s)
t=[tuple(x['tile']) for x in s['top5_ppw'][:4]]+[tuple(x) for x in d['top10_ppw'][:3]]+[tuple(x['tile']) for x in s['top5_perf'][:3]]+[tuple(s['eatss_tile']),(32,32,32)]
seen=[];[seen.append(x) for x in t if x not in seen]
print(";".join(",".join(map(str,x)) for x in seen))
PY
)
echo "confirm: $TILES"
timeout 1500 python harness/sweep.py --kind gemm --n 4000 --tiles "$TILES" --repeats 7 --out gpurun_out/r02/confirm_gemm4000_f32_r02.jsonl > gpurun_out/r02/confirm_f32_r02.log 2>&1; echo "confirm rc=$?"
python harness/report.py gpurun_out/r02/confirm_gemm4000_f32_r02.jsonl --confirm --json gpurun_out/r02/confirm_gemm4000_f32_r02.summary.json > /dev/null 2>&1; echo done
