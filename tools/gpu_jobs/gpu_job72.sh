cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 python tools/pcie_probe.py > gpurun_out/pcie.json 2> gpurun_out/pcie.err
nvidia-smi -q | grep -i -A3 "PCIe Generation\|Link Width" >> gpurun_out/pcie.err
