cd $GRAFT_REPO_ROOT
timeout 120 python scripts/debug_tcm.py 2>&1 | grep -v -i "warning\|Exception\|Traceback\|File\|AttributeError" | head -4
timeout 600 python -m pytest tests/test_gpu_tensor.py -q -k tcm --timeout 120 -p no:cacheprovider 2>&1 | tail -4
T="timeout 120 python scripts/time_kernel.py gemm 4000,4000,4000"
$T 128,256,32 --engine 2; $T 128,128,32 --engine 2; $T 128,192,32 --engine 2; $T 128,64,32 --engine 2
timeout 120 python scripts/debug_tc.py 4000 128,256,32
