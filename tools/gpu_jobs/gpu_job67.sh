cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 python bench.py --force-dist --steps 5 --no-cpu > gpurun_out/b67_fd.json 2> gpurun_out/b67_fd.err
