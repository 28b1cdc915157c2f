cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_fission.py tests/test_program.py -q -m gpu --timeout 600 > gpurun_out/pt_fuse.log 2>&1; echo "exit $?" >> gpurun_out/pt_fuse.log
timeout 600 python tools/perf_fuse_program.py > gpurun_out/fuse_prog.json 2> gpurun_out/fuse_prog.err
