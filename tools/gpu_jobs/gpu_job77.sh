cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for i in 1 2 3; do timeout 300 python bench.py --no-cpu --no-e2e > gpurun_out/b77_$i.json 2>/dev/null; done
