cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 ncu --set full --import-source on --clock-control none -k regex:sdag_rhs4 -c 1 -o gpurun_out/r4_16x16 python tools/prof_one.py rhs4center r4_tma_16x16_u2x1_pf1 2 > gpurun_out/ncu_r4.log 2>&1
timeout 600 ncu --set full --clock-control none -k regex:sdag_sweep -c 1 -o gpurun_out/r4_generic python tools/prof_one.py rhs4center tma_16x16_u1x1_pf1 2 > gpurun_out/ncu_r4g.log 2>&1
