cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r01
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/r01/bench_lap25.json 2> gpurun_out/r01/bench_lap25.err
for c in jacobi7 hypterm rhs4center smooth27; do
  timeout 600 python bench.py --config $c --steps 10 --warmup 3 > gpurun_out/r01/bench_$c.json 2> gpurun_out/r01/bench_$c.err
done
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/r01/bench_reference.json 2> gpurun_out/r01/bench_reference.err
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sdag_hyp -s 2 -c 1 -o gpurun_out/r01/prof_hypterm python tools/prof_one.py hypterm - 3 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sdag_box27 -s 2 -c 1 -o gpurun_out/r01/prof_smooth27 python tools/prof_one.py smooth27 - 3 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sdag_star -s 2 -c 1 -o gpurun_out/r01/prof_jacobi7 python tools/prof_one.py jacobi7 - 3 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sdag_sweep -s 2 -c 1 -o gpurun_out/r01/prof_rhs4 python tools/prof_one.py rhs4center - 3 > /dev/null 2>&1
timeout 300 python tools/perf_sweep.py hypterm smooth27 > gpurun_out/r01/perf_sweep.jsonl 2>&1
echo done > gpurun_out/r01/done.txt
