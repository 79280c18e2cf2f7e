#!/bin/bash
# Round-2 ncu evidence for the FINAL kernels (BULKW under AUTO): launch list of the bench's timed step
# (duration + DRAM bytes per launch) and --set full of four consecutive copy launches of the step.
O=gpurun_out/ncu_r02b
mkdir -p $O
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 4000 --csv \
   --log-file $O/launches_bench.csv python bench.py --profile --steps 2 --warmup 1 > $O/launch_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:copy_ -s 72 -c 4 -o $O/step_full -f \
   python bench.py --profile --steps 1 --warmup 1 > $O/step_full.log 2>&1
for f in $O/*.ncu-rep; do ncu -i $f --page raw --csv > ${f%.ncu-rep}_raw.csv 2>/dev/null; ncu -i $f --page details --csv > ${f%.ncu-rep}_details.csv 2>/dev/null; done
ls -la $O
