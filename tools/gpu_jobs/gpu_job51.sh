cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu --timeout 600 -k "fusion" > gpurun_out/pt_fj7.log 2>&1; echo "exit $?" >> gpurun_out/pt_fj7.log
timeout 600 python tools/table2_sweep.py > gpurun_out/table2.jsonl 2>&1
timeout 600 python tools/table2_sweep.py --n 1024 > gpurun_out/table2_1024.jsonl 2>&1
