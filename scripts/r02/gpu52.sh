# third confirmation (2 s windows) of the fp32 sweep's close pair: the PPW-optimal (32,512,48) vs the fastest
# (16,1024,24), with the EATSS pick and (32,512,24): 15 interleaved repeats of >= 1 s a9 windows
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
timeout 1500 python harness/sweep.py --kind gemm --n 4000 --tiles "32,512,48;16,1024,24;16,1024,16;32,512,24" --repeats 10 --window 2.0 --out gpurun_out/r02/confirm3_gemm4000_f32_r02.jsonl > gpurun_out/r02/confirm3_f32_r02.log 2>&1; echo "confirm2 rc=$?"
python harness/report.py gpurun_out/r02/confirm3_gemm4000_f32_r02.jsonl --confirm --json gpurun_out/r02/confirm3_gemm4000_f32_r02.summary.json > /dev/null 2>&1
python - <<'PY'
import json
c=json.load(open('gpurun_out/r02/confirm3_gemm4000_f32_r02.summary.json'))
for t in c['tiles']:
    print(t['tile'], t['n'], 'ppw', round(t['gflops_per_watt']['mean'],2), [round(x,2) for x in t['gflops_per_watt']['ci95']], 'tf', round(t['tflops']['mean'],3), [round(x,3) for x in t['tflops']['ci95']], 'W', round(t['watts']['mean']))
print('separated', c['finding_energy_beats_perf_on_ppw_ci_separated'], c['energy_optimal'], c['perf_optimal'])
PY
