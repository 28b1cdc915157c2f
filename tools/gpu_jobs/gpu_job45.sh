cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for d in jacobi7 lap25 smooth27 hypterm rhs4center; do timeout 300 python tools/chunk_sweep.py $d auto; done > gpurun_out/chunk_auto.jsonl 2>&1
timeout 600 python tools/fusion_sweep.py --reps 2 > gpurun_out/fus_head3.jsonl 2>&1
