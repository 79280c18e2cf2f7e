#!/bin/bash
# Round-2 ncu evidence (B200_PROFILING.md recipe): the launch list of the bench's timed step, one
# --set full capture of the dominant gather launch and of a scatter launch at the bench's size, and
# the BULKW small-chunk kernel (8 KiB chunks, tools/small_chunk_probe.cu) under --set full.
set -x
O=gpurun_out/ncu_r02
mkdir -p $O
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 4000 --csv \
   --log-file $O/launches_bench.csv python bench.py --profile --steps 2 --warmup 1 > $O/launch_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:copy_bulk -s 40 -c 1 -o $O/gather_full -f \
   python bench.py --profile --steps 1 --warmup 1 > $O/gather_full.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:copy_ -s 72 -c 2 -o $O/step_full -f \
   python bench.py --profile --steps 1 --warmup 1 > $O/step_full.log 2>&1
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -o /tmp/scp tools/small_chunk_probe.cu
timeout 600 ncu --set full --clock-control none --import-source on -k regex:copy_bulkw -s 0 -c 1 -o $O/bulkw_2k_full -f /tmp/scp > $O/bulkw_full.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:copy_bulkw -s 48 -c 1 -o $O/bulkw_8k_full -f /tmp/scp > $O/bulkw8_full.log 2>&1
for f in $O/*.ncu-rep; do ncu -i $f --page raw --csv > ${f%.ncu-rep}_raw.csv 2>/dev/null; ncu -i $f --page details --csv > ${f%.ncu-rep}_details.csv 2>/dev/null; done
ls -la $O
