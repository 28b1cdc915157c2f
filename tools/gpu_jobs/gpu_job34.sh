cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python tools/fusion_sweep.py --reps 2 > gpurun_out/fus_head.jsonl 2>&1
cd _prev && timeout 600 python tools/fusion_sweep.py --reps 2 > ../gpurun_out/fus_prev.jsonl 2>&1
