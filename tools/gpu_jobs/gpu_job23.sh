cd $GRAFT_REPO_ROOT
timeout 900 python tools/perf_sweep.py lap25 --only star > gpurun_out/perf_lap25.jsonl 2> gpurun_out/perf_lap25.err
