#!/bin/bash
# host fill piece size for the staged weight path (switch leg, staged mode matters)
mkdir -p gpurun_out/sweep3
for p in 0 16384 65536 262144 1048576; do
  AEG_FILL_PIECE=$p timeout 600 python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu --no-migrate --switches 12 \
     > gpurun_out/sweep3/piece$p.json 2> gpurun_out/sweep3/piece$p.err
done
