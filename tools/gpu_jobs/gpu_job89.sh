cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_jit.py -q -m gpu --timeout 800 > gpurun_out/pt_jitstar.log 2>&1; echo "exit $?" >> gpurun_out/pt_jitstar.log
timeout 900 python tools/ablation.py lap25 > gpurun_out/ablation_star.jsonl 2> gpurun_out/ablation_star.err
timeout 600 python tools/jit_perf.py > gpurun_out/jit_perf3.jsonl 2> gpurun_out/jit_perf3.err
