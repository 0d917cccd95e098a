cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out; T=scripts/time_kernel.py
{ for rm in 8; do for t in 128,32,16,16 64,32,16,16 128,32,32,32 256,32,16,16; do EATSS_MT_MAXRM=$rm timeout 120 python $T mttkrp 512,32,512,512 $t --iters 20 2>&1 | tail -1 | sed "s/^/rm$rm /"; done; done
  for t in 16,64,5,5 8,512,5,5 16,1024,5,5; do timeout 120 python $T conv-2d 8192,5 $t --iters 20 2>&1 | tail -1; done; } > gpurun_out/mt_times.txt 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:mttkrp_kernel -s 3 -c 1 -o gpurun_out/prof_mttkrp_r01 -f python $T mttkrp 512,32,512,512 128,32,16,16 --iters 1 > /dev/null 2>&1; echo "ncu mttkrp $?"
cat gpurun_out/mt_times.txt
