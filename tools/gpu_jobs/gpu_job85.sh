cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for i in 1 2; do timeout 600 python tools/perf_sweep.py rhs4center --reps 20 --only r4_tma > gpurun_out/perf_r4_$i.jsonl 2>/dev/null; done
timeout 600 python -m pytest tests/test_gpu_parity.py -q -m gpu -k "rhs4" --timeout 500 > gpurun_out/pt_r4.log 2>&1; echo "exit $?" >> gpurun_out/pt_r4.log
