cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export SDAG_P2P_TIMEOUT_S=30
timeout 300 python bench.py --halo p2p --steps 5 --no-cpu > gpurun_out/b76_p2p1.json 2> gpurun_out/b76_p2p1.err
SDAG_BENCH_SAME_DEVICE=1 timeout 400 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29631 bench.py --halo p2p --gpus 2 --steps 5 --no-cpu > gpurun_out/b76_p2p2.json 2> gpurun_out/b76_p2p2.err
timeout 300 python bench.py --steps 5 --no-cpu > gpurun_out/b76_default.json 2> gpurun_out/b76_default.err
