#!/bin/bash
# configs[4] leg alone, then an ncu --set full attempt on one full-size gather launch of the bench step
mkdir -p gpurun_out
free -g > gpurun_out/free.txt
timeout 600 python tools/run_leg.py c5 > gpurun_out/c5.json 2> gpurun_out/c5.err; echo "c5 rc=$?" >> gpurun_out/c5.err
free -g >> gpurun_out/free.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:copy_bulk -s 4 -c 1 -o gpurun_out/prof_full_gather -f \
    python bench.py --profile --steps 1 --warmup 1 > gpurun_out/ncu_full_gather.log 2>&1
echo "ncu rc=$?" >> gpurun_out/ncu_full_gather.log
