cd $GRAFT_REPO_ROOT
timeout 1500 python -m pytest tests/test_gpu_jit.py -q -m gpu --timeout 900 -x > gpurun_out/pytest_jit.log 2>&1
echo "exit $?" >> gpurun_out/pytest_jit.log
