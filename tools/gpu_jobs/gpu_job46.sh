cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -m gpu --timeout 600 -k "apply_host" > gpurun_out/pt_host.log 2>&1; echo "exit $?" >> gpurun_out/pt_host.log
timeout 600 python bench.py --no-cpu > gpurun_out/bench_e2e.json 2> gpurun_out/bench_e2e.err
