cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -k "tune" --timeout 600 > gpurun_out/pt_tune.log 2>&1; echo "exit $?" >> gpurun_out/pt_tune.log
for c in lap25 jacobi7 hypterm rhs4center; do timeout 600 python tools/perf_tuned.py $c >> gpurun_out/tuned.jsonl 2>>gpurun_out/tuned.err; done
