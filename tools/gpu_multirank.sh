#!/bin/bash
# the N>1 bench path with ranks sharing the one GPU (gloo control plane): 2 and 4 ranks
mkdir -p gpurun_out
for n in 2 4; do
  AEG_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node $n --master-addr 127.0.0.1 \
     --master-port 2953$n bench.py --gpus $n --requests 4 --no-switch --no-cpu --steps 2 --warmup 1 \
     > gpurun_out/bench_${n}rank.json 2> gpurun_out/bench_${n}rank.err; echo "rc=$?" >> gpurun_out/bench_${n}rank.err
done
