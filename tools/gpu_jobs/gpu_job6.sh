cd $GRAFT_REPO_ROOT
timeout 900 python tools/perf_sweep.py > gpurun_out/perf_sweep.jsonl 2> gpurun_out/perf_sweep.err
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e > /dev/null 2> gpurun_out/ncu1.err
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sdag_star -s 3 -c 1 -o gpurun_out/prof_lap25 python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e > /dev/null 2> gpurun_out/ncu2.err
echo done > gpurun_out/done.txt
