cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -m gpu --timeout 600 -x -k "rhs4" > gpurun_out/pt_rhs4.log 2>&1; echo "exit $?" >> gpurun_out/pt_rhs4.log
timeout 600 python tools/perf_sweep.py rhs4center > gpurun_out/perf_rhs4.jsonl 2> gpurun_out/perf_rhs4.err
timeout 600 python tools/fusion_sweep.py --reps 2 > gpurun_out/fus_head2.jsonl 2>&1
