# End-of-session evidence on the fused prep launch: the full evidence pass plus an ncu capture of prep_kernel.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
bash scripts/gpu_final.sh
timeout 600 ncu --set full --clock-control none --import-source on -k regex:prep_kernel -s 3 -c 1 -o gpurun_out/prof_prep_r01h -f python bench.py --steps 3 --warmup 3 --e2e-steps 1 --no-cpu-baseline --no-secondary --no-configs > /dev/null 2>&1; echo "ncu prep $?"
