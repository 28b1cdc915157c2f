cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1500 python tools/ablation.py > gpurun_out/ablation.jsonl 2> gpurun_out/ablation.err
