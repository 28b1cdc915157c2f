cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -k "batched" --timeout 800 > gpurun_out/pt_batched.log 2>&1; echo "exit $?" >> gpurun_out/pt_batched.log
