cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export SDAG_P2P_TIMEOUT_S=20
timeout 900 python -m pytest tests/test_gpu_p2p.py -q -m gpu --timeout 600 -x > gpurun_out/pt_p2p.log 2>&1; echo "exit $?" >> gpurun_out/pt_p2p.log
