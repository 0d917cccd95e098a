cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
T=scripts/time_kernel.py
for c in 128 512; do EATSS_TCM_PROF=1 EATSS_TCM_CHUNK_K=$c python $T gemm 4000,4000,4000 256,256,32 --engine 2 --iters 3 2>&1 | tail -2; done
for c in 128 512; do EATSS_TCM_CHUNK_K=$c python $T gemm 4000,4000,4000 256,256,32 --engine 2 --iters 50 2>&1 | tail -1; done
for g in 2 4 16 32; do EATSS_TCM_GROUP=$g python $T gemm 4000,4000,4000 256,256,32 --engine 2 --iters 50 2>&1 | tail -1; done
