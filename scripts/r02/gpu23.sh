# fused 3xTF32 converter cost isolation (development build; not bench values)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
T=scripts/time_kernel.py
for t in 256,256,32 128,256,32; do
  r=$(timeout 120 python $T gemm 4000,4000,4000 $t --engine 2 --iters 50 2>&1 | tail -1); echo "release $t: $r"
done
EATSS_DEV_NVCC_FLAGS=-DEATSS_DEVTOOLS python paper_conf_cgo_jayaweerakwk24_b200/build.py --force -j 32 > /dev/null 2>&1 || echo BUILD FAILED
for t in 256,256,32 128,256,32; do for dbg in 16; do
  r=$(EATSS_TCM_DBG=$dbg timeout 120 python $T gemm 4000,4000,4000 $t --engine 2 --iters 50 2>&1 | tail -1); echo "dbg $dbg $t: $r"
done; done
timeout 300 ncu --set full --import-source on --clock-control none -k regex:tc_mma_kernel -c 1 -o gpurun_out/r02/prof_tcm_fused python $T gemm 4000,4000,4000 256,256,32 --engine 2 --iters 1 > /dev/null 2>&1
