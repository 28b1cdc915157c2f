cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_jit.py tests/test_program.py -q -m gpu --timeout 600 > gpurun_out/pt_jit.log 2>&1; echo "exit $?" >> gpurun_out/pt_jit.log
timeout 900 python tools/jit_perf.py > gpurun_out/jit_perf2.jsonl 2> gpurun_out/jit_perf2.err
