# 3xFP16 engine: tests, timing, chunk A/B, quick bench
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
timeout 900 python -m pytest tests/test_gpu_f16.py -q -x --timeout 600 -p no:cacheprovider > gpurun_out/r02/pytest_f16.log 2>&1; echo "rc=$?" >> gpurun_out/r02/pytest_f16.log; tail -15 gpurun_out/r02/pytest_f16.log
T=scripts/time_kernel.py
for t in 256,256,64 256,256,32 128,256,64 256,192,128 256,256,16; do timeout 120 python $T gemm 4000,4000,4000 $t --engine 4 --iters 30 2>&1 | tail -1; done
for c in 128 256 512; do EATSS_TCM_CHUNK_K=$c timeout 120 python $T gemm 4000,4000,4000 256,256,64 --engine 4 --iters 30 2>&1 | tail -1; done
timeout 600 python bench.py --no-configs --steps 100 > gpurun_out/r02/bench13.log 2>&1; echo "bench rc=$?"; tail -c 2500 gpurun_out/r02/bench13.log
# ccsd_tc: sliced t3 pipeline A/B at the model tile, then its parity tests
for xs in 1 0; do EATSS_CCSD_TC_SLICES=$xs timeout 300 python $T ccsd_t_d1 48 1,2,1,48,2,48,48 --engine 2 --iters 5 2>&1 | tail -1; done
timeout 600 python -m pytest tests/test_gpu_tensor.py -q -x --timeout 600 -p no:cacheprovider -k ccsd 2>&1 | tail -2
