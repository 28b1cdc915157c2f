cd $GRAFT_REPO_ROOT
for args in "-2 0 0 68 34" "-4 -4 0 72 40" "0 -3 0 68 34" "0 0 -2 68 34" "-4 -3 -1 72 40" "2 3 5 68 34"; do
  timeout 60 ./tools/tma_probe $args >> gpurun_out/tma_probe2.txt 2>&1
done
timeout 900 python tools/debug_variants.py 20,34,70 > gpurun_out/debug_variants.jsonl 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -m gpu --timeout 300 > gpurun_out/pytest_gpu.log 2>&1
echo "pytest exit $?" >> gpurun_out/pytest_gpu.log
