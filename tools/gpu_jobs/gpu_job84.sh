cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1500 python tools/jit_fuzz.py 40 > gpurun_out/jit_fuzz.log 2>&1; echo "exit $?" >> gpurun_out/jit_fuzz.log
