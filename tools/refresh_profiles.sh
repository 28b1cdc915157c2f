# Copy one tools/measure_round.sh session (gpurun_out/meas/) into profiles/<round>/:
# the bench lines, GPU test log + worst parity errors, smoke log, launch lists,
# one ncu summary per hot kernel (profiles/ncu_counters.json refreshed: the
# per-launch DRAM bytes and executed FP64 flops bench.py's roofline reads) and
# the static SASS evidence.  usage: tools/refresh_profiles.sh r02
set -e
R=${1:?round, e.g. r02}
M=gpurun_out/meas
P=profiles/$R
mkdir -p $P/ncu
for f in bench.json bench_reference.json pytest_gpu.log parity_worst.json smoke.log bench_launches.csv bench_launches_headline.csv; do
  [ -f $M/$f ] && cp $M/$f $P/$f
done
# name -> ncu_counters key (variant@dims) of the kernel the plan picks
declare -A KEY=(
  [lap25]="star_tma_32x32_u2x4_pf3_z2@512x512x512"
  [jacobi7]="star_tma_64x16_u2x2_pf6@128x64x64x64"
  [hypterm]="hyp_tma_64x8_u2x1_pf2@320x320x320"
  [rhs4center]="r4_tma_32x16_u2x1_pf1@320x320x320"
  [smooth27]="box_tma_128x16_u2x4_pf2@512x512x512"
  [fuse2]="fuse2o_tma_62x14_u2x2_pf2_mb2@1024x1024x1024"
)
for d in lap25 jacobi7 hypterm rhs4center smooth27 fuse2; do
  [ -f $M/prof_$d.ncu-rep ] || continue
  python3 tools/ncu_summary.py $M/prof_$d.ncu-rep $P/ncu/${d}_ncu --variant "${KEY[$d]}" > /dev/null
done
python3 tools/sass_evidence.py $P/sass_evidence.md
python3 tools/floors.py $M $P/floors > /dev/null
echo "refreshed $P"
