cd $GRAFT_REPO_ROOT
timeout 1800 python -m pytest tests/ -q -m gpu --timeout 900 -k "full_size or synth" > gpurun_out/pytest_full.log 2>&1
echo "pytest exit $?" >> gpurun_out/pytest_full.log
