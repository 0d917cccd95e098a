# SIMT staging variants on the bench plan (after the spread copies): ring stages x k-rows per stage x threads
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
b() { echo "== $*"; env "$@" timeout 300 python bench.py --engine simt --steps 20 --warmup 3 --no-configs --no-secondary --no-cpu-baseline --e2e-steps 1 2>&1 | grep '^{' | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['value'], d['roofline']['frac'])"; }
for rep in 1 2; do
b EATSS_STAGES=1
b EATSS_STAGES=3 EATSS_KSUB=2
b EATSS_STAGES=2 EATSS_KSUB=2
b EATSS_STAGES=4 EATSS_KSUB=4
b EATSS_STAGES=2 EATSS_THREADS=512
b EATSS_STAGES=3 EATSS_KSUB=2 EATSS_THREADS=512
done
T="scripts/time_kernel.py gemm 4000,4000,4000 32,512,48 --engine 1 --iters 20"
for v in "EATSS_STAGES=1" "EATSS_STAGES=3 EATSS_KSUB=3" "EATSS_STAGES=2 EATSS_KSUB=2"; do echo "== (32,512,48) $v"; env $v timeout 120 python $T 2>&1 | tail -1; done
