cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 python tools/e2e_probe.py 4 8 16 32 48 63 > gpurun_out/e2e.jsonl 2> gpurun_out/e2e.err
