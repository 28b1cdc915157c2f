cd $GRAFT_REPO_ROOT
timeout 600 ncu --set full --import-source on --clock-control none -k regex:box27x2 -s 1 -c 1 -o gpurun_out/prof_fuse2 python tools/prof_fuse.py fuse2_tma_62x14_u2x2_pf2 > gpurun_out/ncu_fuse.log 2>&1
