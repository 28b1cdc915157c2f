cd $GRAFT_REPO_ROOT
for args in "0 0 0 68 34" "-1 0 0 68 34" "63 0 0 68 34" "64 0 0 68 34" "1 0 0 68 34" "2 0 0 68 34" "0 0 3 68 34" "0 0 0 66 18" "1 0 0 66 18" "0 0 0 72 40" "-1 0 0 72 40" "1 0 0 72 40" "0 0 0 68 32" "0 0 0 64 34" "0 0 0 70 34" "0 0 0 68 8" "0 0 0 2 34" "0 0 0 4 34" "0 0 0 34 34" "0 0 0 36 34" "0 0 0 66 34" "0 0 0 132 34" "0 0 0 136 34"; do
  timeout 60 ./tools/tma_probe $args >> gpurun_out/tma_probe.txt 2>&1
done
timeout 900 python tools/debug_variants.py 20,34,70 jacobi7,smooth27 > gpurun_out/debug_variants.jsonl 2>&1
