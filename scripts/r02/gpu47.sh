# bench configs after the per-config 50 ms warm-up (conv-2d / mttkrp measured ~20% slow right after the GEMMs)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --e2e-steps 2 > gpurun_out/r02/bench_cfgwarm.log 2>&1; echo rc=$?
python - <<'PY'
import json
d=json.loads([x for x in open('gpurun_out/r02/bench_cfgwarm.log') if x.startswith('{')][-1])
print('value', round(d['value'],1), 'frac', round(d['roofline']['frac'],3))
for k,v in d['configs'].items():
    print(k, json.dumps(v)[:300])
PY
