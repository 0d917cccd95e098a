# tc_mma with 12 epilogue warps (16 warps in all: 128 registers, 88 accumulators) vs 16 (96 registers)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
timeout 1500 python -m pytest tests/test_gpu_f16.py tests/test_gpu_tensor.py tests/test_gpu_fullsize.py -q -x -p no:cacheprovider 2>&1 | tail -2
T="scripts/time_kernel.py gemm 4000,4000,4000 256,256,64 --engine 4 --iters 100 --kernel-ms"
T2="scripts/time_kernel.py gemm 4000,4000,4000 256,256,32 --engine 2 --iters 100 --kernel-ms"
b() { timeout 300 python bench.py --steps 100 --warmup 5 --no-configs --no-secondary --no-cpu-baseline --e2e-steps 2 2>&1 | grep '^{' | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('bench', round(d['ms_per_step'],4), round(d['value'],1), round(r['frac'],3))"; }
for rep in 1 2; do echo "== NEPI 12"; timeout 120 python $T 2>&1 | tail -2; timeout 120 python $T2 2>&1 | tail -2; b; done
EATSS_DEV_NVCC_FLAGS=-DEATSS_TCM_NEPI=16 python paper_conf_cgo_jayaweerakwk24_b200/build.py --force -j 32 > /dev/null 2>&1
for rep in 1 2; do echo "== NEPI 16"; timeout 120 python $T 2>&1 | tail -2; timeout 120 python $T2 2>&1 | tail -2; b; done
