cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu --timeout 600 -k "fusion or loopback" > gpurun_out/pt_fuse.log 2>&1; echo "exit $?" >> gpurun_out/pt_fuse.log
timeout 600 python tools/fusion_sweep.py --reps 2 > gpurun_out/fus_odd.jsonl 2>&1
