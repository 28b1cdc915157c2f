cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_jit.py -q -m gpu -k "random_star or star or box" --timeout 800 > gpurun_out/pt_rform.log 2>&1; echo "exit $?" >> gpurun_out/pt_rform.log
