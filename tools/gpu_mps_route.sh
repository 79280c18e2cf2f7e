#!/bin/bash
# NEXT-2 host route (P->C->D, two processes on one GPU) with and without MPS: without MPS the two
# CUDA contexts time-slice the GPU; under MPS they run concurrently, as P and D would on two GPUs.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
run() {
  timeout 600 python -c "
import json, torch, bench
import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg
torch.cuda.init()
print(json.dumps(bench.host_route_leg(aeg, torch, aeg.KERNEL_AUTO)))" > gpurun_out/host_route_$1.json 2> gpurun_out/host_route_$1.err
}
run nomps
export CUDA_MPS_PIPE_DIRECTORY=/tmp/aeg_mps_pipe CUDA_MPS_LOG_DIRECTORY=/tmp/aeg_mps_log
mkdir -p $CUDA_MPS_PIPE_DIRECTORY $CUDA_MPS_LOG_DIRECTORY
nvidia-cuda-mps-control -d && echo "mps started" >> gpurun_out/host_route_mps.err
run mps
echo quit | nvidia-cuda-mps-control
sleep 2
