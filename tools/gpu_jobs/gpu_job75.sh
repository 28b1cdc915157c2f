cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/tmem_probe tools/tmem_probe.cu && timeout 120 /tmp/tmem_probe > gpurun_out/tmem.jsonl 2> gpurun_out/tmem.err
