cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1500 python tools/ablation.py lap25 smooth27 jacobi7 > gpurun_out/ablation2.jsonl 2> gpurun_out/ablation2.err
