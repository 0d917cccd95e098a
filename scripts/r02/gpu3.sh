# Round-2 pass 3: the reworked tcgen05 GEMM (Ti/Tj/Tk honoured, 16 epilogue warps): tile-space
# exactness + timing, chunk A/B, the tensor tests.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
timeout 900 python scripts/r02/tcm_space_check.py > gpurun_out/r02/tcm_space.jsonl 2>&1; echo "rc=$?" >> gpurun_out/r02/tcm_space.jsonl
timeout 600 python scripts/r02/chunk_ab.py > gpurun_out/r02/chunk_ab2.jsonl 2>&1
timeout 600 python -m pytest tests/test_gpu_tensor.py -q -x --timeout 300 -p no:cacheprovider > gpurun_out/r02/pytest_tensor3.log 2>&1; echo "rc=$?" >> gpurun_out/r02/pytest_tensor3.log
head -c 3000 gpurun_out/r02/tcm_space.jsonl; cat gpurun_out/r02/chunk_ab2.jsonl; tail -5 gpurun_out/r02/pytest_tensor3.log
