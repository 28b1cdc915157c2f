cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export SDAG_P2P_TIMEOUT_S=30
timeout 1500 python -m pytest tests -q -m gpu --timeout 900 > gpurun_out/pt_all.log 2>&1; echo "exit $?" >> gpurun_out/pt_all.log
timeout 600 python tools/classify.py > gpurun_out/classify.jsonl 2> gpurun_out/classify.err
