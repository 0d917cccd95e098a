cd $GRAFT_REPO_ROOT
timeout 900 python harness/sweep.py --limit 60 --window 0.5 --out gpurun_out/sweep_cal2.jsonl 2>&1 | tail -2
python harness/report.py gpurun_out/sweep_cal2.jsonl | python -c "import json,sys; d=json.load(sys.stdin); [print(k, d.get(k)) for k in ['measured_ok','perf_optimal','energy_optimal','anchor_default','anchor_eatss','ppw_noise_rel','finding_energy_beats_perf_on_ppw','eatss_rank_ppw','eatss_rank_perf']]"
