# compute-sanitizer memcheck + synccheck on every kernel family and the P2P
# flag protocol, racecheck on the shared-memory rings (tools/sanitize_run.py
# launches one small problem per family).  Run through gpurun; logs under
# gpurun_out/san/ (copied to profiles/<round>/sanitizer/).
cd $GRAFT_REPO_ROOT
M=gpurun_out/san; mkdir -p $M
export SDAG_P2P_TIMEOUT_S=60
for f in star box27 fuse2 fuseN hyp hypc rhs4 rhs4f sweep lsu jit p2p; do
  timeout 900 compute-sanitizer --tool memcheck --print-limit 20 python tools/sanitize_run.py $f > $M/san_memcheck_$f.log 2>&1; echo "rc $?" >> $M/san_memcheck_$f.log
  timeout 900 compute-sanitizer --tool synccheck --print-limit 20 python tools/sanitize_run.py $f > $M/san_synccheck_$f.log 2>&1; echo "rc $?" >> $M/san_synccheck_$f.log
done
for f in star box27 fuse2 fuseN hyp hypc rhs4 rhs4f sweep lsu; do
  timeout 900 compute-sanitizer --tool racecheck --racecheck-report analysis --print-limit 20 python tools/sanitize_run.py $f > $M/san_racecheck_$f.log 2>&1; echo "rc $?" >> $M/san_racecheck_$f.log
done
echo done > $M/done.txt
