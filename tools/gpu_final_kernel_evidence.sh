#!/bin/bash
# Final-kernel evidence for VERDICT r1 #7: launch_probe.cu (event and %globaltimer spans, back to
# back and after a cross-stream wait) with BULKW, and ncu --set full of an 8 KiB-chunk BULKW gather.
O=gpurun_out/final_kernel
mkdir -p $O
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I include -o /tmp/lp tools/launch_probe.cu && \
  timeout 300 /tmp/lp > $O/launch_probe.txt 2>&1
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -o /tmp/scp tools/small_chunk_probe.cu
# 8 KiB chunks: the 5th BULKW gather launch of the 8 KiB case (CHUNKS=8192 -> 12 gathers then 12 scatters)
CHUNKS=8192 SPREAD=30 timeout 300 ncu --set full --clock-control none --import-source on -k regex:copy_bulkw -s 4 -c 1 \
  -o $O/bulkw_8k_final -f /tmp/scp > $O/bulkw_8k_final.log 2>&1
ncu -i $O/bulkw_8k_final.ncu-rep --page raw --csv > $O/bulkw_8k_final_raw.csv 2>/dev/null
ncu -i $O/bulkw_8k_final.ncu-rep --page details --csv > $O/bulkw_8k_final_details.csv 2>/dev/null
grep -E "BLKW|LSU |WARP|BULK" $O/launch_probe.txt | grep "n= 65536\|n=16384" | head -30
