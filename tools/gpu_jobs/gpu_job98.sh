cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export SDAG_P2P_TIMEOUT_S=30
timeout 1500 python -m pytest tests -q -m gpu --timeout 1400 > gpurun_out/pt_final.log 2>&1; echo "exit $?" >> gpurun_out/pt_final.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke_final.log 2>&1
timeout 600 python bench.py > gpurun_out/bench_final.json 2> gpurun_out/bench_final.err
