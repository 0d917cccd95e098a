# SURVEY 8(f) row 3 on the headline engine: the 3xFP16 tcgen05 tile space of gemm N=4000 (every executable
# (Ti, Tj, Tk) with Tk in fp16 elements), exactness first, then 4 interleaved rounds of >= 1 s a9 windows
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
timeout 2400 python harness/tensor_sweep.py --engine 4 --repeats 4 --window 1.0 --out gpurun_out/r02/tensor16_sweep_r02.jsonl > gpurun_out/r02/tensor16_sweep.log 2>&1; echo "rc=$?"
tail -3 gpurun_out/r02/tensor16_sweep.log | cut -c1-1500
