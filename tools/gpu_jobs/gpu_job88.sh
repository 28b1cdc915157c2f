cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -m gpu -k "full_size" --timeout 1400 > gpurun_out/pt_full.log 2>&1; echo "exit $?" >> gpurun_out/pt_full.log
