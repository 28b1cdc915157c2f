cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python tools/perf_sweep.py rhs4center --only u2x1 > gpurun_out/perf_rhs4d.jsonl 2> gpurun_out/perf_rhs4d.err
timeout 600 python -m pytest tests/test_gpu_parity.py -q -m gpu --timeout 600 -x -k "rhs4" > gpurun_out/pt_rhs4.log 2>&1; echo "exit $?" >> gpurun_out/pt_rhs4.log
timeout 600 ncu --set full --import-source on --clock-control none -k regex:sdag_rhs4 -c 1 -o gpurun_out/r4_16x16c python tools/prof_one.py rhs4center r4_tma_16x16_u2x1_pf1 2 > gpurun_out/ncu_r4.log 2>&1
