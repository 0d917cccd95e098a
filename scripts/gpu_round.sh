cd $GRAFT_REPO_ROOT
T="timeout 120 python scripts/time_kernel.py gemm 4000,4000,4000"
$T 16,1024,16 --engine 2; EATSS_TC_ABULK=1 $T 16,1024,16 --engine 2; EATSS_TC_STAGES=8 $T 16,1024,16 --engine 2
$T 32,512,16 --engine 2; $T 64,256,16 --engine 2; $T 16,512,16 --engine 2
