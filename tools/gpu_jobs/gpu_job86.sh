cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 python bench.py --force-dist --steps 5 --no-cpu > gpurun_out/b86_fd.json 2> gpurun_out/b86_fd.err
timeout 300 python bench.py --halo p2p --steps 5 --no-cpu > gpurun_out/b86_p2p.json 2> gpurun_out/b86_p2p.err
SDAG_BENCH_SAME_DEVICE=1 timeout 400 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29641 bench.py --halo p2p --gpus 2 --steps 5 --no-cpu > gpurun_out/b86_p2p2.json 2> gpurun_out/b86_p2p2.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/b86_ref.json 2> gpurun_out/b86_ref.err
