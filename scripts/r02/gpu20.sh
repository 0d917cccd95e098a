# which part of the accumulator hand-off costs time (development build; not bench values)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
EATSS_DEV_NVCC_FLAGS=-DEATSS_DEVTOOLS python paper_conf_cgo_jayaweerakwk24_b200/build.py --force -j 32 > /dev/null 2>&1 || echo BUILD FAILED
T=scripts/time_kernel.py
for ck in 256 4000; do for dbg in 0 1 8 9; do
  r=$(EATSS_TCM_CHUNK_K=$ck EATSS_TCM_DBG=$dbg timeout 60 python $T gemm 4000,4000,4000 256,256,64 --engine 4 --iters 50 2>&1 | tail -1)
  echo "chunk $ck dbg $dbg: $r"
done; done 2>&1 | tee gpurun_out/r02/chunk_cost3.log
