# §8(f) row 2 at the paper's sample size ("700+ variants"): 350 gemm + 350 2mm variants.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
P=gpurun_out/l2power700_power.jsonl; L=gpurun_out/l2power700_l2.csv
timeout 2400 python harness/l2power.py --phase power --kinds gemm,2mm --count 350 --seed 1 --power $P > gpurun_out/l2power700.log 2>&1; echo "power $?"
timeout 2400 ncu --metrics lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_op_read.sum,gpu__time_duration.sum --clock-control none -k regex:'contract' --csv --log-file $L python harness/l2power.py --phase l2 --kinds gemm,2mm --power $P > /dev/null 2>&1; echo "ncu $?"
python harness/l2power.py --phase report --kinds gemm,2mm --power $P --l2csv $L --out gpurun_out/l2power700_summary.json >> gpurun_out/l2power700.log 2>&1; echo "report $?"
tail -20 gpurun_out/l2power700.log
