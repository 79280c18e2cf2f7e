#!/bin/bash
# --set full captures of the other hot kernels at the bench's sizes: the LSU migrate kernel of the
# configs[2] leg (16 requests, one launch per layer) and one full-size scatter launch of the C2 step.
# Usage: bash tools/gpu_ncu_more.sh [migrate] [scatter]
mkdir -p gpurun_out
what="${*:-migrate scatter}"
if [[ $what == *migrate* ]]; then
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:copy_lsu -s 2 -c 1 -o gpurun_out/prof_migrate -f \
      python tools/run_leg.py migrate > gpurun_out/ncu_migrate.log 2>&1
  echo "rc=$?" >> gpurun_out/ncu_migrate.log
fi
if [[ $what == *scatter* ]]; then
  timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base mangled \
      -k regex:copy_bulkILb0ELb1E -s 4 -c 1 -o gpurun_out/prof_scatter -f \
      python bench.py --profile --steps 1 --warmup 1 > gpurun_out/ncu_scatter.log 2>&1
  echo "rc=$?" >> gpurun_out/ncu_scatter.log
fi
