# Round-2 pass 2: new tests (WAF, carve-out, full-size 2mm/3mm), the whole GPU suite, bench, chunk A/B.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
timeout 600 python -m pytest tests/test_gpu_waf.py -q -x --timeout 300 -p no:cacheprovider > gpurun_out/r02/pytest_waf.log 2>&1; echo "rc=$?" >> gpurun_out/r02/pytest_waf.log
timeout 1200 python -m pytest tests/test_gpu_fullsize.py -q --timeout 900 -p no:cacheprovider > gpurun_out/r02/pytest_full.log 2>&1; echo "rc=$?" >> gpurun_out/r02/pytest_full.log
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider --deselect tests/test_gpu_fullsize.py > gpurun_out/r02/pytest_gpu2.log 2>&1; echo "rc=$?" >> gpurun_out/r02/pytest_gpu2.log
timeout 900 python bench.py > gpurun_out/r02/bench2.log 2>&1; echo "bench rc=$?" >> gpurun_out/r02/bench2.log
timeout 600 python scripts/r02/chunk_ab.py > gpurun_out/r02/chunk_ab.jsonl 2>&1
tail -3 gpurun_out/r02/pytest_waf.log gpurun_out/r02/pytest_full.log gpurun_out/r02/pytest_gpu2.log; cat gpurun_out/r02/chunk_ab.jsonl | tail -8
