cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export SDAG_P2P_TIMEOUT_S=20
timeout 900 python -m pytest tests/test_gpu_p2p.py -x -q -m gpu --timeout 600 > gpurun_out/pt_p2p.log 2>&1; echo "exit $?" >> gpurun_out/pt_p2p.log
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -k "loopback or smooth27 or jacobi7 or fusion" --timeout 800 > gpurun_out/pt_p2p2.log 2>&1; echo "exit $?" >> gpurun_out/pt_p2p2.log
timeout 300 python bench.py --config smooth27 --no-cpu > gpurun_out/bench_s27.json 2> gpurun_out/bench_s27.err
