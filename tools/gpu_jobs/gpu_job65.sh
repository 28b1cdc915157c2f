cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -k "jacobi7 or batched" --timeout 600 > gpurun_out/pt_j7.log 2>&1; echo "exit $?" >> gpurun_out/pt_j7.log
for i in 1 2; do
SDAG_STACKED=0 timeout 300 python bench.py --config jacobi7 --no-cpu > gpurun_out/bj7_0_$i.json 2>/dev/null
timeout 300 python bench.py --config jacobi7 --no-cpu > gpurun_out/bj7_1_$i.json 2>/dev/null
done
for n in 37 74 111 148 222; do SDAG_NCHUNK=$n timeout 300 python bench.py --config jacobi7 --no-cpu > gpurun_out/bj7_n$n.json 2>/dev/null; done
