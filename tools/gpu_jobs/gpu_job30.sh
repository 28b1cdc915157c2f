cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu --timeout 600 -k fusion -x > gpurun_out/pytest_fuse.log 2>&1
echo "exit $?" >> gpurun_out/pytest_fuse.log
timeout 900 python tools/fusion_sweep.py > gpurun_out/fuse_sweep.jsonl 2>&1
