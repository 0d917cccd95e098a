# fp64 confirmation on the leaders of the WHOLE 3,375-variant fp64 sweep (part 1 + part 2): the single-window
# PPW top 5, the drift-corrected PPW top 4, the TFLOP/s top 4, EATSS and default; 7 interleaved repeats
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
TILES="64,256,48;128,128,48;64,256,768;64,256,384;128,128,512;64,256,512;64,256,192;64,256,128;64,256,256;64,256,64;16,512,16;32,32,32"
timeout 1800 python harness/sweep.py --kind gemm --n 4000 --dtype f64 --tiles "$TILES" --repeats 7 --out gpurun_out/r02/confirm_gemm4000_f64_full_r02.jsonl > gpurun_out/r02/confirm_f64_full.log 2>&1; echo "confirm rc=$?"
python harness/report.py gpurun_out/r02/confirm_gemm4000_f64_full_r02.jsonl --confirm --json gpurun_out/r02/confirm_gemm4000_f64_full_r02.summary.json | tail -30
