#!/bin/bash
# final ncu evidence: gather + scatter launches of the profiled bench step, and the migrate kernel
mkdir -p gpurun_out/ncu_final
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file gpurun_out/ncu_final/launches_bench.csv \
   python bench.py --profile --requests 16 --steps 1 --warmup 1 > gpurun_out/ncu_final/launch_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:copy_ -c 70 -o gpurun_out/ncu_final/swap -f \
   python bench.py --profile --requests 16 --steps 1 --warmup 1 > gpurun_out/ncu_final/swap.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:copy_ -s 20 -c 6 -o gpurun_out/ncu_final/migrate -f \
   python tools/profile_migrate.py > gpurun_out/ncu_final/migrate.log 2>&1
echo done > gpurun_out/ncu_final/done
