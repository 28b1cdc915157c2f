cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export SDAG_P2P_TIMEOUT_S=30
timeout 900 python -m pytest tests/test_gpu_p2p.py tests/test_gpu_parity.py -q -m gpu -k "p2p or every_variant or loopback or smoke" --timeout 800 > gpurun_out/pt_starmir.log 2>&1; echo "exit $?" >> gpurun_out/pt_starmir.log
timeout 300 python bench.py --no-cpu --no-e2e > gpurun_out/b83.json 2>/dev/null
