#!/bin/bash
# One gpurun call: GPU tests, bench, ncu launch list, ncu --set full of the top kernel.
# Usage (under gpurun): bash tools/gpu_round.sh [tests] [bench] [ncu]
mkdir -p gpurun_out
what="${*:-tests bench ncu}"
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm --format=csv > gpurun_out/clocks_start.csv 2>&1
if [[ $what == *tests* ]]; then
  timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 300 --timeout-method thread -rA > gpurun_out/gpu_tests.log 2>&1
  echo "pytest rc=$?" >> gpurun_out/gpu_tests.log
  timeout 180 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
fi
if [[ $what == *bench* ]]; then
  timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?" >> gpurun_out/bench.err
fi
if [[ $what == *ncu* ]]; then
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv --log-file gpurun_out/launches.csv \
      python bench.py --profile --requests 16 --steps 1 --warmup 1 > gpurun_out/ncu_launch_bench.log 2>&1
  echo "ncu launches rc=$?" >> gpurun_out/ncu_launch_bench.log
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:copy_ -s 8 -c 4 -o gpurun_out/prof_copy -f \
      python bench.py --profile --requests 16 --steps 1 --warmup 1 > gpurun_out/ncu_full.log 2>&1
  echo "ncu full rc=$?" >> gpurun_out/ncu_full.log
fi
