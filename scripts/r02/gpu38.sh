# SIMT: deeper rings of whole k-tiles (one CTA per SM) vs S = 1 (two CTAs per SM)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
b() { echo "== $*"; env "$@" timeout 300 python bench.py --engine simt --steps 20 --warmup 3 --no-configs --no-secondary --no-cpu-baseline --e2e-steps 1 2>&1 | grep '^{' | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['value'], d['roofline']['frac'])"; }
for rep in 1 2; do b EATSS_STAGES=1; b EATSS_STAGES=2; b EATSS_STAGES=3; done
