cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python bench.py --force-dist --steps 5 --warmup 3 > gpurun_out/bench_fdist.json 2> gpurun_out/bench_fdist.err
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 1 --steps 5 --warmup 3 --no-cpu > gpurun_out/bench_trun.json 2> gpurun_out/bench_trun.err
