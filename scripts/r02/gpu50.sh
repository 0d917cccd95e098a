# SIMT staged executor: suspended stage wait (time-hinted try_wait) vs re-polling -- parity, bench-plan A/B
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_waf.py -q -p no:cacheprovider -k "gemm or 2mm or syrk or 3mm" 2>&1 | tail -1
b() { echo "== $*"; env "$@" timeout 300 python bench.py --engine simt --steps 20 --warmup 3 --no-configs --no-secondary --no-cpu-baseline --e2e-steps 1 2>&1 | grep '^{' | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['value'], d['roofline']['frac'])"; }
for rep in 1 2 3; do b EATSS_SIMT_WAIT_SUSPEND=1; b EATSS_SIMT_WAIT_SUSPEND=0; done
T="scripts/time_kernel.py gemm 4000,4000,4000 32,512,48 --engine 1 --iters 20"
for v in 1 0; do echo "== (32,512,48) suspend=$v"; EATSS_SIMT_WAIT_SUSPEND=$v timeout 120 python $T 2>&1 | tail -1; done
# stencils / conv-2d: suspended window wait (default build) vs re-polling (-DEATSS_SPIN_WAIT)
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fourd.py -q -p no:cacheprovider -k "jacobi or heat or conv" 2>&1 | tail -1
S() { for a in "jacobi-2d 4000 16,1024 --tsteps 500 --iters 3" "jacobi-2d 16384 16,1024 --tsteps 10 --iters 3" "heat-3d 120 16,16,32 --tsteps 500 --iters 3" "heat-3d 512 16,16,32 --tsteps 5 --iters 3" "conv-2d 8192,5 16,64,5,5 --iters 50"; do timeout 120 python scripts/time_kernel.py $a 2>&1 | tail -1 | cut -c1-90; done; }
for rep in 1 2; do echo "== suspended"; S; done
EATSS_DEV_NVCC_FLAGS=-DEATSS_SPIN_WAIT python paper_conf_cgo_jayaweerakwk24_b200/build.py --force -j 32 > /dev/null 2>&1
for rep in 1 2; do echo "== spin"; S; done
