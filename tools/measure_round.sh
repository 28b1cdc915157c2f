# Full measurement pass on one B200 (run through gpurun): GPU tests, smoke,
# the bench line of every config, the reference arm, the ncu launch list of the
# headline command and one ncu --set full capture per hot kernel.
# Outputs under gpurun_out/meas/ (copied to profiles/ by hand).
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/meas
M=gpurun_out/meas
timeout 1500 python -m pytest tests -q -m gpu --timeout 900 > $M/pytest_gpu.log 2>&1; echo "exit $?" >> $M/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $M/smoke.log 2>&1
timeout 600 python bench.py > $M/bench_lap25.json 2> $M/bench_lap25.err   # headline: heuristic plan
for c in jacobi7 hypterm rhs4center smooth27; do
  timeout 600 python bench.py --config $c > $M/bench_$c.json 2> $M/bench_$c.err
done
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > $M/bench_reference.json 2> $M/bench_reference.err
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $M/lap25_bench_launches.csv python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e > /dev/null 2> $M/ncu_launches.err
# one full capture per hot kernel (default variant at the BASELINE size)
for d in lap25 jacobi7 hypterm rhs4center smooth27; do
  timeout 600 ncu --set full --import-source on --clock-control none -k regex:sdag_ -c 1 -o $M/prof_$d python tools/prof_one.py $d - 2 > $M/ncu_$d.log 2>&1
done
timeout 600 ncu --set full --import-source on --clock-control none -k regex:sdag_box27x2 -c 1 -o $M/prof_fuse2 python tools/prof_fuse.py fuse2_tma_62x14_u2x2_pf2_mb2 1024 > $M/ncu_fuse2.log 2>&1
echo done > $M/done.txt
