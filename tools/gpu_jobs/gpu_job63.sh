cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export SDAG_P2P_TIMEOUT_S=30
timeout 300 python bench.py --config smooth27 --halo p2p --steps 5 > gpurun_out/b63_p2p1.json 2> gpurun_out/b63_p2p1.err
timeout 300 python bench.py --config smooth27 --halo nccl --steps 5 > gpurun_out/b63_nccl1.json 2> gpurun_out/b63_nccl1.err
SDAG_BENCH_SAME_DEVICE=1 SDAG_BENCH_SLAB_N=512 timeout 400 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29611 bench.py --config smooth27 --halo p2p --gpus 2 --steps 5 > gpurun_out/b63_p2p2.json 2> gpurun_out/b63_p2p2.err
echo done
