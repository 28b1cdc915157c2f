cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1200 python tools/form_fuzz.py 40 > gpurun_out/form_fuzz.log 2>&1; echo "exit $?" >> gpurun_out/form_fuzz.log
