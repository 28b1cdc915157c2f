cd $GRAFT_REPO_ROOT
timeout 900 python tools/perf_sweep.py rhs4center > gpurun_out/perf_sweep.jsonl 2> gpurun_out/perf_sweep.err
