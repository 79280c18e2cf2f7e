#!/bin/bash
# One gpurun call: GPU tests + smoke, default bench, and the ncu launch list of the bench's own
# full-size step (per-launch duration + DRAM bytes of every copy kernel, single pass, no replay).
# Usage (under gpurun): bash tools/gpu_check.sh [tests] [bench] [ncu]
mkdir -p gpurun_out
what="${*:-tests bench ncu}"
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > gpurun_out/gpu_info.csv 2>&1
if [[ $what == *tests* ]]; then
  timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 400 --timeout-method thread -rA > gpurun_out/gpu_tests.log 2>&1
  echo "pytest rc=$?" >> gpurun_out/gpu_tests.log
  timeout 180 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
fi
if [[ $what == *bench* ]]; then
  timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?" >> gpurun_out/bench.err
fi
if [[ $what == *ncu* ]]; then
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
      -k regex:"copy_|fetch_table" -c 400 --csv --log-file gpurun_out/ncu_fullsize_launches.csv \
      python bench.py --profile --steps 1 --warmup 1 > gpurun_out/ncu_fullsize.log 2>&1
  echo "ncu rc=$?" >> gpurun_out/ncu_fullsize.log
fi
