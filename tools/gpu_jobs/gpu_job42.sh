cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python tools/chunk_sweep.py jacobi7 auto 1 2 3 4 5 6 8 > gpurun_out/chunk_j7.jsonl 2>&1
timeout 900 python tools/chunk_sweep.py lap25 auto 1 2 3 4 6 8 > gpurun_out/chunk_l25.jsonl 2>&1
timeout 900 python tools/chunk_sweep.py hypterm auto 1 2 3 4 6 > gpurun_out/chunk_hyp.jsonl 2>&1
timeout 900 python tools/chunk_sweep.py rhs4center auto 1 2 3 4 6 > gpurun_out/chunk_r4.jsonl 2>&1
