#!/bin/bash
# slot size / kernel sweep of the C2 leg + pin probe + one full default bench
mkdir -p gpurun_out/sweep1
./build/pin_probe 16 16 > gpurun_out/sweep1/pin_probe.txt 2>&1
for cfg in "--kernel lsu" "--kernel bulk" "--kernel lsu --slot-mib 1024 --slots 3" "--kernel bulk --slot-mib 1024 --slots 3" "--kernel lsu --slot-mib 512 --slots 3"; do
  tag=$(echo $cfg | tr -d ' -')
  timeout 300 python bench.py $cfg --no-switch --no-migrate --no-cpu --no-e2e > gpurun_out/sweep1/$tag.json 2> gpurun_out/sweep1/$tag.err
done
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?" >> gpurun_out/bench.err
