cd $GRAFT_REPO_ROOT
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -m gpu --timeout 600 -k "fusion" -x > gpurun_out/pytest_fuse.log 2>&1
echo "exit $?" >> gpurun_out/pytest_fuse.log
cat > /tmp/fz.py <<'PY'
import sys, json, torch; sys.path.insert(0, ".")
import paper_conf_ipps_rawatvsrps19_b200 as sdag
dims=(1024,1024,1024); T=12; s=[-128/30,14/30,3/30,1/30,0.125]
b0=torch.rand(dims,dtype=torch.float64,device="cuda"); b1=b0.clone()
for name, kw in [("fused", {}), ("plain", {"fusion": False})] + [(v, {"variant": v}) for v in ["fuse2_tma_126x14_u2x2_pf2","fuse2_tma_62x14_u2x2_pf2","fuse2_tma_126x14_u2x4_pf2"]]:
    p=sdag.Plan(sdag.spec_text("smooth27"), dims, **kw)
    p.apply_iterated(b0,b1,T,s); torch.cuda.synchronize()
    e0,e1=torch.cuda.Event(enable_timing=True),torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(3): p.apply_iterated(b0,b1,T,s)
    e1.record(); torch.cuda.synchronize()
    ms=e0.elapsed_time(e1)/3/T
    i=p.info; byts=i["bytes_per_point"]*i["points"]
    print(json.dumps({"cfg":name,"ms_per_sweep":ms,"GBps_per_sweep_equiv":byts/ms/1e6,"frac_single_sweep_roofline":byts/ms/1e6/6456.2}))
PY
timeout 600 python /tmp/fz.py > gpurun_out/fuse_perf.jsonl 2>&1
