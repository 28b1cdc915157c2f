cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python tools/perf_sweep.py rhs4center --only r4_ > gpurun_out/perf_rhs4b.jsonl 2> gpurun_out/perf_rhs4b.err
timeout 600 python -m pytest tests/test_gpu_parity.py -q -m gpu --timeout 600 -x -k "rhs4" > gpurun_out/pt_rhs4.log 2>&1; echo "exit $?" >> gpurun_out/pt_rhs4.log
