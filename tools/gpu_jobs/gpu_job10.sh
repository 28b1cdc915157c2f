cd $GRAFT_REPO_ROOT
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sdag_sweep -s 2 -c 1 -o gpurun_out/prof_hypterm python tools/prof_one.py hypterm - 3 > gpurun_out/ncu_h.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sdag_sweep -s 2 -c 1 -o gpurun_out/prof_rhs4 python tools/prof_one.py rhs4center - 3 > gpurun_out/ncu_r.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sdag_box27 -s 2 -c 1 -o gpurun_out/prof_smooth27 python tools/prof_one.py smooth27 box_tma_128x16_u2x4_pf2 3 > gpurun_out/ncu_s.log 2>&1
python -c "
import sys; sys.path.insert(0,'.')
import paper_conf_ipps_rawatvsrps19_b200 as s, torch
print('fp64 peak', s.fp64_peak()/1e12, 'TF')
print('fp64 peak', s.fp64_peak()/1e12, 'TF')
" > gpurun_out/fp64_peak.txt 2>&1
