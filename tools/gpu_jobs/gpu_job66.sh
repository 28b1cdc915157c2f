cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_fission.py tests/test_program.py -q -m gpu --timeout 600 > gpurun_out/pt_fis.log 2>&1; echo "exit $?" >> gpurun_out/pt_fis.log
timeout 600 python tools/perf_sweep.py jacobi7 --reps 20 > gpurun_out/perf_j7.jsonl 2> gpurun_out/perf_j7.err
