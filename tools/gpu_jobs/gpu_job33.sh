cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu --timeout 600 -k "loopback or fusion" > gpurun_out/pytest_dist.log 2>&1
echo "exit $?" >> gpurun_out/pytest_dist.log
