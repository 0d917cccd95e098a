# fp64 sweep: re-measure the 19 records of the window bug, regenerate the report, interleaved confirmation of
# the top tiles (7 repeats); then compute-sanitizer over every TMA/tcgen05 executor and the ccsd_tc ncu capture
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
F=gpurun_out/r02/sweep_gemm4000_f64_r02.jsonl
ONLY=$(python - <<'PY'
import json
recs=[json.loads(l) for l in open('gpurun_out/r02/sweep_gemm4000_f64_r02.jsonl') if l.strip().startswith('{')]
bad=[r for r in recs if r.get('kind')=='variant' and r['ms']<0.01]
print(";".join(",".join(map(str,r['tile'])) for r in bad))
PY
)
echo "re-measure: $ONLY"
timeout 1200 python harness/sweep.py --kind gemm --n 4000 --dtype f64 --only "$ONLY" --out $F > gpurun_out/r02/sweep_f64_only.log 2>&1; echo "only rc=$?"
python harness/report.py $F --json gpurun_out/r02/sweep_gemm4000_f64_r02.summary.json > gpurun_out/r02/sweep_f64_report.txt 2>&1
TILES=$(python - <<'PY'
import json
s=json.load(open('gpurun_out/r02/sweep_gemm4000_f64_r02.summary.json'))
d=s.get('drift_corrected',s)
t=[tuple(x) for x in d['top10_ppw'][:3]]+[tuple(x) for x in d['top10_perf'][:3]]+[tuple(s['eatss_tile']),(32,32,32)]
seen=[];[seen.append(x) for x in t if x not in seen]
print(";".join(",".join(map(str,x)) for x in seen))
PY
)
echo "confirm: $TILES"
timeout 1800 python harness/sweep.py --kind gemm --n 4000 --dtype f64 --tiles "$TILES" --repeats 7 --out gpurun_out/r02/confirm_gemm4000_f64_r02.jsonl > gpurun_out/r02/confirm_f64.log 2>&1; echo "confirm rc=$?"
python harness/report.py gpurun_out/r02/confirm_gemm4000_f64_r02.jsonl --confirm --json gpurun_out/r02/confirm_gemm4000_f64_r02.summary.json > /dev/null 2>&1
bash scripts/r02/gpu12.sh
