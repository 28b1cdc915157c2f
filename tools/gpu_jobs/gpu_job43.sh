cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python tools/chunk_sweep.py jacobi7 8 10 12 16 20 31 62 > gpurun_out/chunk_j7b.jsonl 2>&1
