# accumulator-chunk cost vs Tk (stages) on the 3xFP16 engine (development build; not bench values)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
EATSS_DEV_NVCC_FLAGS=-DEATSS_DEVTOOLS python paper_conf_cgo_jayaweerakwk24_b200/build.py --force -j 32 > /dev/null 2>&1 || echo BUILD FAILED
T=scripts/time_kernel.py
for spec in "4 256,256,32 256" "4 256,256,32 4000" "4 256,256,16 256" "4 256,256,64 512" "4 128,256,64 256" "4 128,256,64 4000"; do
  set -- $spec
  for dbg in 0 1; do
    r=$(EATSS_TCM_CHUNK_K=$3 EATSS_TCM_DBG=$dbg timeout 120 python $T gemm 4000,4000,4000 $2 --engine $1 --iters 50 2>&1 | tail -1)
    echo "engine $1 tile $2 chunk $3 dbg $dbg: $r"
  done
  EATSS_TCM_CHUNK_K=$3 EATSS_TCM_PROF=1 timeout 120 python $T gemm 4000,4000,4000 $2 --engine $1 --iters 2 2>&1 | grep "prof" | tail -1
done 2>&1 | tee gpurun_out/r02/chunk_cost2.log
