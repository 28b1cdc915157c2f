cd $GRAFT_REPO_ROOT
timeout 900 python tools/debug_variants.py 20,34,70 lap25,jacobi7 > gpurun_out/debug_variants.jsonl 2>&1
timeout 900 python tools/perf_sweep.py lap25 jacobi7 > gpurun_out/perf_sweep.jsonl 2> gpurun_out/perf_sweep.err
