cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 python tools/e2e_probe.py 64 > gpurun_out/e2e2.jsonl 2> gpurun_out/e2e2.err
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -k "host" --timeout 800 > gpurun_out/pt_host.log 2>&1; echo "exit $?" >> gpurun_out/pt_host.log
timeout 600 python bench.py > gpurun_out/bench_lap25_e2e.json 2> gpurun_out/bench_lap25_e2e.err
