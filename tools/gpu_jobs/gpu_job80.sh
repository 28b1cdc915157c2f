cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -k "graph or iterated or fusion or loopback" --timeout 800 > gpurun_out/pt_graph.log 2>&1; echo "exit $?" >> gpurun_out/pt_graph.log
timeout 300 python tools/perf_graphs.py > gpurun_out/graphs.jsonl 2> gpurun_out/graphs.err
