cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/meas2
for c in jacobi7 hypterm rhs4center smooth27; do
  timeout 600 python bench.py --config $c > gpurun_out/meas2/bench_$c.json 2> gpurun_out/meas2/bench_$c.err
done
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -k "tune or iterated or fusion" --timeout 800 > gpurun_out/meas2/pt.log 2>&1; echo "exit $?" >> gpurun_out/meas2/pt.log
