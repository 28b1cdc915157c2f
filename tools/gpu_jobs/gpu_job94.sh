cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python tools/gen_jacobi_probe.py > gpurun_out/j7gen.jsonl 2> gpurun_out/j7gen.err
