cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests/test_gpu_tensor.py -q --timeout 300 -p no:cacheprovider 2>&1 | tail -8
echo "== rna mode tests"; EATSS_TCM_SPLIT=rna timeout 600 python -m pytest tests/test_gpu_tensor.py -q --timeout 300 -p no:cacheprovider -k "tcm" 2>&1 | tail -3
for cfg in "gemm 4000,4000,4000" "syrk 4000,4000" "2mm 4000,4000,4000,4000" "3mm 4000,4000,4000,4000,4000"; do
  echo "== $cfg"; timeout 120 python scripts/time_kernel.py $cfg 128,256,32 --engine 2 --iters 20 2>&1 | tail -1
done
echo "== gemm rna"; EATSS_TCM_SPLIT=rna timeout 120 python scripts/time_kernel.py gemm 4000,4000,4000 128,256,32 --engine 2 2>&1 | tail -1
