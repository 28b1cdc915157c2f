cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export SDAG_P2P_TIMEOUT_S=30
timeout 1500 python -m pytest tests -q -m gpu --timeout 1400 > gpurun_out/pt_all2.log 2>&1; echo "exit $?" >> gpurun_out/pt_all2.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke2.log 2>&1
timeout 1200 python tools/ablation.py > gpurun_out/ablation4.jsonl 2> gpurun_out/ablation4.err
