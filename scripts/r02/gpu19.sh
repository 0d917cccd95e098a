cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02
python scripts/r02/precision_chunks.py 4 256,256,64 256 512 1024 4000 2>&1 | tee gpurun_out/r02/precision_chunks.jsonl
python scripts/r02/precision_chunks.py 2 256,256,32 128 256 2>&1 | tee -a gpurun_out/r02/precision_chunks.jsonl
