cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 1 --steps 20 --warmup 3 --no-configs --no-secondary --no-cpu-baseline --e2e-steps 2 --sharded on > gpurun_out/r02/bench_sharded10.log 2>&1; echo "bench rc=$?"
tail -c 3000 gpurun_out/r02/bench_sharded10.log
timeout 600 python -m pytest tests/test_gpu_tensor.py -q -x --timeout 600 -p no:cacheprovider -k ccsd 2>&1 | tail -2
