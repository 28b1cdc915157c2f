cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_jit.py -q -m gpu --timeout 800 > gpurun_out/pt_r1.log 2>&1; echo "exit $?" >> gpurun_out/pt_r1.log
