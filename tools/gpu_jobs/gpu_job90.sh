cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_jit.py tests/test_gpu_parity.py -q -m gpu -k "box or star or forced or every_variant or smooth27" --timeout 800 > gpurun_out/pt_box.log 2>&1; echo "exit $?" >> gpurun_out/pt_box.log
timeout 600 python tools/jit_perf.py > gpurun_out/jit_perf4.jsonl 2> gpurun_out/jit_perf4.err
