cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu --timeout 600 -k "fusion" > gpurun_out/pt_fN.log 2>&1; echo "exit $?" >> gpurun_out/pt_fN.log
timeout 900 python tools/table2_sweep.py --all > gpurun_out/table2_all512.jsonl 2>&1
timeout 900 python tools/table2_sweep.py --all --n 1024 --reps 2 > gpurun_out/table2_all1024.jsonl 2>&1
