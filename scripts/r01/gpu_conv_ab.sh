cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out; T=scripts/time_kernel.py; L=paper_conf_cgo_jayaweerakwk24_b200/libeatss.so
for rep in 1 2; do for v in old new; do cp abtmp/$v.so $L; for t in 16,64,5,5 32,32,5,5 8,512,5,5 16,1024,5,5; do echo -n "$v "; timeout 120 python $T conv-2d 8192,5 $t --iters 50 2>&1 | tail -1; done; done; done > gpurun_out/conv_ab.txt 2>&1
cp abtmp/new.so $L
timeout 600 python -m pytest tests/test_gpu_fourd.py -x -q -k "conv2d" -p no:cacheprovider > gpurun_out/pytest_conv.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_conv.log
cat gpurun_out/conv_ab.txt; tail -2 gpurun_out/pytest_conv.log
