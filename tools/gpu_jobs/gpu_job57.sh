cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python tools/jit_perf.py > gpurun_out/jit_perf.jsonl 2> gpurun_out/jit_perf.err
