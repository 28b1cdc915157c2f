cd $GRAFT_REPO_ROOT
timeout 600 ncu --set full --import-source on --clock-control none -k regex:sdag_star -s 1 -c 1 -o gpurun_out/prof_lap25_z2 python tools/prof_one.py lap25 star_tma_32x32_u2x4_pf3_z2 3 > gpurun_out/ncu_z2.log 2>&1
