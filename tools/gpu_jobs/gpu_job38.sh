cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python tools/perf_sweep.py rhs4center --only r4_tma > gpurun_out/perf_rhs4c.jsonl 2> gpurun_out/perf_rhs4c.err
timeout 600 ncu --set full --import-source on --clock-control none -k regex:sdag_rhs4 -c 1 -o gpurun_out/r4_16x16b python tools/prof_one.py rhs4center r4_tma_16x16_u2x1_pf1 2 > gpurun_out/ncu_r4.log 2>&1
