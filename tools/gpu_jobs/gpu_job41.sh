cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python tools/perf_sweep.py rhs4center --only r4_tma > gpurun_out/perf_rhs4f.jsonl 2> gpurun_out/perf_rhs4f.err
timeout 600 python tools/perf_sweep.py hypterm > gpurun_out/perf_hyp.jsonl 2> gpurun_out/perf_hyp.err
timeout 600 python tools/perf_sweep.py jacobi7 > gpurun_out/perf_j7.jsonl 2> gpurun_out/perf_j7.err
