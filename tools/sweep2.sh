#!/bin/bash
# weight-stage chunk size sweep (switch leg only) + default bench
mkdir -p gpurun_out/sweep2
for c in 8 16 32 64; do
  AEG_STAGE_CHUNK_MIB=$c timeout 600 python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu --no-migrate --switches 15 \
     > gpurun_out/sweep2/chunk$c.json 2> gpurun_out/sweep2/chunk$c.err
done
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?" >> gpurun_out/bench.err
