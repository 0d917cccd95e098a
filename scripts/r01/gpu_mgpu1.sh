# The multi-GPU runner's NCCL path at world size 1 (this environment exposes one GPU per call).
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for k in 3mm syrk ccsd_t_d1; do
  timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29511 harness/multigpu.py --kind $k --steps 3 --warmup 2 > gpurun_out/mgpu1_$k.log 2>&1; echo "$k rc=$?"; tail -1 gpurun_out/mgpu1_$k.log | cut -c1-400
done
