cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu --timeout 600 -x > gpurun_out/pytest_var.log 2>&1
echo "exit $?" >> gpurun_out/pytest_var.log
timeout 900 python tools/perf_sweep.py lap25 jacobi7 --only tma > gpurun_out/perf_p.jsonl 2> gpurun_out/perf_p.err
