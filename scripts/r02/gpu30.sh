# headline GEMM cost isolation (development build, -DEATSS_DEVTOOLS; not bench values):
# split order A/B (0: rows+colmax then B split; 1: colmax, then B split + rows), dbg 16 = no MMAs (operand delivery only), 32 = no operand TMA (MMA only), raster group and chunk
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
EATSS_DEV_NVCC_FLAGS=-DEATSS_DEVTOOLS python paper_conf_cgo_jayaweerakwk24_b200/build.py --force -j 32 > /dev/null 2>&1 || echo BUILD FAILED

T="scripts/time_kernel.py gemm 4000,4000,4000 256,256,64 --engine 4 --iters 50 --kernel-ms"
run() { echo "== $*"; env "$@" timeout 120 python $T 2>&1 | tail -2; }

for rep in 1 2; do
run EATSS_TCM_DBG=0
run EATSS_TCM_DBG=16
run EATSS_TCM_DBG=32
run EATSS_TCM_DBG=48
run EATSS_TCM_DBG=1
done
for g in 2 4 16 32; do run EATSS_TCM_GROUP=$g; done
run EATSS_TCM_CHUNK_K=512
run EATSS_TCM_CHUNK_K=4000
run EATSS_TCM_STAGES=2
T="scripts/time_kernel.py gemm 4000,4000,4000 256,256,32 --engine 4 --iters 50 --kernel-ms"
run EATSS_TCM_DBG=0
run EATSS_TCM_DBG=16
T="scripts/time_kernel.py gemm 4000,4000,4000 256,128,64 --engine 4 --iters 50 --kernel-ms"
run EATSS_TCM_DBG=0
run EATSS_TCM_DBG=16
# SIMT staged executor: B row copies issued by every warp's lane 0 (1) vs thread 0 alone (0)
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_waf.py -q -x -p no:cacheprovider -k "gemm or 2mm or syrk" 2>&1 | tail -2
for rep in 1 2 3; do for v in 1 0; do
  echo "== simt spread=$v"; EATSS_SIMT_BULK_SPREAD=$v timeout 120 python scripts/time_kernel.py gemm 4000,4000,4000 16,1024,16 --engine 1 --iters 20 2>&1 | tail -1
  EATSS_SIMT_BULK_SPREAD=$v timeout 120 python scripts/time_kernel.py gemm 4000,4000,4000 32,512,48 --engine 1 --iters 20 2>&1 | tail -1
done; done
for t in 512 128; do echo "== simt threads=$t"; EATSS_THREADS=$t timeout 120 python scripts/time_kernel.py gemm 4000,4000,4000 16,1024,16 --engine 1 --iters 20 2>&1 | tail -1; done
