cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu --timeout 600 -k "every_variant" > gpurun_out/pytest_var.log 2>&1
echo "exit $?" >> gpurun_out/pytest_var.log
timeout 900 python tools/perf_sweep.py lap25 --only tma > gpurun_out/perf_lap25.jsonl 2> gpurun_out/perf_lap25.err
