cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_jit.py tests/test_gpu_p2p.py -q -m gpu -k "box or smooth27 or fusion or loopback or p2p" --timeout 800 > gpurun_out/pt_boxfuse.log 2>&1; echo "exit $?" >> gpurun_out/pt_boxfuse.log
