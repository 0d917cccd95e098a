cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out; T=scripts/time_kernel.py
{ for t in 16,1024,16 32,512,48 32,512,32; do
  timeout 120 python $T gemm 4000,4000,4000 $t --engine 1 --iters 5 2>&1 | tail -1 | sed "s/^/default /"
  for sk in "2 2" "3 4" "4 4" "2 4" "3 2"; do set -- $sk; EATSS_STAGES=$1 EATSS_KSUB=$2 timeout 120 python $T gemm 4000,4000,4000 $t --engine 1 --iters 5 2>&1 | tail -1 | sed "s/^/S$1 ksub$2 /"; done
done; } > gpurun_out/simt_stages.txt 2>&1
cat gpurun_out/simt_stages.txt
