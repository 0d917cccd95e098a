# the rest of the fp64 3,375-variant sweep (part 1 = the variants measured before the 1200 s limit)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
timeout 3300 python harness/sweep.py --kind gemm --n 4000 --dtype f64 --resume profiles/r02/sweep_gemm4000_f64_r02.part1.jsonl --out gpurun_out/r02/sweep_gemm4000_f64_r02.part2.jsonl > gpurun_out/r02/sweep_f64_part2.log 2>&1; echo "sweep rc=$?"
tail -2 gpurun_out/r02/sweep_f64_part2.log
