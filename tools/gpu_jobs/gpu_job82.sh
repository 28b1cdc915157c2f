cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -k "apply_host or host" --timeout 800 > gpurun_out/pt_dhost.log 2>&1; echo "exit $?" >> gpurun_out/pt_dhost.log
timeout 300 python bench.py --force-dist --steps 5 --no-cpu > gpurun_out/b82_fd.json 2> gpurun_out/b82_fd.err
timeout 300 python bench.py --halo p2p --steps 5 --no-cpu > gpurun_out/b82_p2p.json 2> gpurun_out/b82_p2p.err
