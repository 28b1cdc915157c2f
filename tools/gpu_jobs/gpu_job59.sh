cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python -m pytest tests -q -m gpu -k "hypterm or jit" --timeout 500 > gpurun_out/pt_hyp.log 2>&1; echo "exit $?" >> gpurun_out/pt_hyp.log
timeout 600 python tools/perf_sweep.py hypterm --reps 20 > gpurun_out/perf_hyp.jsonl 2> gpurun_out/perf_hyp.err
