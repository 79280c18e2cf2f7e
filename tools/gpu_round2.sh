#!/bin/bash
# GPU tests + a 2-rank bench run sharing the one GPU (gloo control plane) + the default bench
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 300 --timeout-method thread -rA > gpurun_out/gpu_tests.log 2>&1
echo "pytest rc=$?" >> gpurun_out/gpu_tests.log
timeout 180 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
AEG_DIST_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
   --master-port 29533 bench.py --gpus 2 --requests 8 --no-switch --no-cpu --steps 3 --warmup 1 \
   > gpurun_out/bench_2rank.json 2> gpurun_out/bench_2rank.err; echo "2rank rc=$?" >> gpurun_out/bench_2rank.err
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?" >> gpurun_out/bench.err
