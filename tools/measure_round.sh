# Full measurement pass on one B200 (run through gpurun): GPU tests (worst e_p
# per parity check to parity_worst.json), smoke, the bench line (headline +
# per_config of every BASELINE config), the reference arm, the ncu launch list
# of the headline command and one ncu --set full capture per hot kernel (with
# the FP64 instruction counters).  Outputs under gpurun_out/meas/ (summarised
# into profiles/ by tools/ncu_summary.py).
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/meas
M=gpurun_out/meas
SDAG_PARITY_LOG=$M/parity_worst.json timeout 2400 python -m pytest tests -q -m gpu --timeout 1200 > $M/pytest_gpu.log 2>&1; echo "exit $?" >> $M/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $M/smoke.log 2>&1
timeout 900 python bench.py > $M/bench.json 2> $M/bench.err
timeout 900 python bench.py --impl reference --steps 5 --warmup 3 > $M/bench_reference.json 2> $M/bench_reference.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $M/bench_launches.csv python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e > /dev/null 2> $M/ncu_launches.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $M/bench_launches_headline.csv python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e --no-per-config > /dev/null 2> $M/ncu_launches_headline.err
FP64=smsp__sass_thread_inst_executed_op_dfma_pred_on.sum,smsp__sass_thread_inst_executed_op_dadd_pred_on.sum,smsp__sass_thread_inst_executed_op_dmul_pred_on.sum
for d in lap25 jacobi7 hypterm rhs4center smooth27; do
  timeout 900 ncu --set full --metrics $FP64 --import-source on --clock-control none -k regex:sdag_ -c 1 -o $M/prof_$d python tools/prof_one.py $d - 2 > $M/ncu_$d.log 2>&1
done
timeout 900 ncu --set full --metrics $FP64 --import-source on --clock-control none -k regex:sdag_box27x2 -c 1 -o $M/prof_fuse2 python tools/prof_fuse.py fuse2o_tma_62x14_u2x2_pf2_mb2 1024 > $M/ncu_fuse2.log 2>&1
echo done > $M/done.txt
