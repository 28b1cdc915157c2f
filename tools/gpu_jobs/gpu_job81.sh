cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_jit.py tests/test_fission.py tests/test_program.py -q -m gpu --timeout 800 > gpurun_out/pt_jitq.log 2>&1; echo "exit $?" >> gpurun_out/pt_jitq.log
timeout 1500 python tools/ablation.py lap25 smooth27 jacobi7 hypterm rhs4center > gpurun_out/ablation3.jsonl 2> gpurun_out/ablation3.err
