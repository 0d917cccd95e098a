# sharded configs through bench (N=1 and torchrun N=1 over NCCL), ccsd model-tile tests, ccsd timing
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
timeout 900 python -m pytest tests/test_gpu_tensor.py -q -x --timeout 600 -p no:cacheprovider -k ccsd > gpurun_out/r02/pytest_ccsd9.log 2>&1; echo "rc=$?" >> gpurun_out/r02/pytest_ccsd9.log; tail -2 gpurun_out/r02/pytest_ccsd9.log
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 1 --steps 20 --warmup 3 --no-configs --no-secondary --no-cpu-baseline --e2e-steps 2 --sharded on > gpurun_out/r02/bench_sharded9.log 2>&1; echo "bench rc=$?"
tail -c 2500 gpurun_out/r02/bench_sharded9.log
T=scripts/time_kernel.py
timeout 300 python $T ccsd_t_d1 48 1,2,2,48,1,48,48 --engine 2 --iters 5 2>&1 | tail -1
timeout 300 python $T ccsd_t_d1 48 1,2,1,48,2,48,48 --engine 2 --iters 5 2>&1 | tail -1
