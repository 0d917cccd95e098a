# sharded check, then the fp64 3,375-variant sweep (the paper's precision, P:117 / P:202)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 1 --steps 20 --warmup 3 --no-configs --no-secondary --no-cpu-baseline --e2e-steps 2 --sharded on > gpurun_out/r02/bench_sharded11.log 2>&1; echo "bench rc=$?"
python - <<'PY'
import json
l=[x for x in open('gpurun_out/r02/bench_sharded11.log') if x.startswith('{')]
d=json.loads(l[-1]) if l else {}
for k,v in d.get('configs',{}).get('sharded',{}).items(): print(k, {x: v[x] for x in ('ms','ms_1gpu','speedup','bit_equal','rel_err_vs_1gpu')})
PY
timeout 5000 python harness/sweep.py --kind gemm --n 4000 --dtype f64 --out gpurun_out/r02/sweep_gemm4000_f64_r02.jsonl > gpurun_out/r02/sweep_f64.log 2>&1; echo "sweep rc=$?"
python harness/report.py gpurun_out/r02/sweep_gemm4000_f64_r02.jsonl --json gpurun_out/r02/sweep_gemm4000_f64_r02.summary.json > /dev/null 2>&1
tail -3 gpurun_out/r02/sweep_f64.log
