#!/bin/bash
# Exercise the N = 8 bench path (replicas + pairs + all-to-all hand-off + the configs[4] TP=4 leg)
# with 8 ranks sharing the one GPU (gloo control plane, small sizes via the hidden exercise knobs).
mkdir -p gpurun_out
AEG_DIST_BACKEND=gloo timeout 1200 python -m torch.distributed.run --nnodes=1 --nproc-per-node 8 --master-addr 127.0.0.1 \
   --master-port 29538 bench.py --gpus 8 --requests 2 --no-switch --no-cpu --steps 2 --warmup 1 \
   --slot-mib 256 --slots 2 --churn-slabs 2 --c5-model qwen-7b --migrate-requests 2 \
   > gpurun_out/bench_8rank.json 2> gpurun_out/bench_8rank.err; echo "rc=$?" >> gpurun_out/bench_8rank.err
nvidia-smi --query-gpu=memory.used --format=csv >> gpurun_out/bench_8rank.err
