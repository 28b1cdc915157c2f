cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python tools/chunk_sweep.py lap25 12 16 24 32 > gpurun_out/chunk_l25b.jsonl 2>&1
timeout 900 python tools/chunk_sweep.py hypterm 8 12 16 > gpurun_out/chunk_hypb.jsonl 2>&1
timeout 900 python tools/chunk_sweep.py rhs4center 8 12 16 > gpurun_out/chunk_r4b.jsonl 2>&1
timeout 900 python tools/chunk_sweep.py smooth27 auto 2 4 8 16 32 > gpurun_out/chunk_s27.jsonl 2>&1
