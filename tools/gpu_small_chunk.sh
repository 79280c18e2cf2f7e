#!/bin/bash
# Build and run tools/small_chunk_probe.cu (SWEEP=1: BULKW piece sweep) for several BULKW geometries
# (warps per CTA, dynamic smem KiB per CTA, max stages per warp).
mkdir -p gpurun_out/scp
for w in "4 192 16" "8 192 16" "16 192 16" "4 96 16" "8 96 16" "4 64 16" "8 64 8"; do
  set -- $w
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -DAEG_BW_WARPS=$1 -DAEG_BW_SMEM_KIB=$2 \
    -DAEG_BW_MAX_STAGES=$3 -o /tmp/scp_$1_$2_$3 tools/small_chunk_probe.cu && \
    SWEEP=1 timeout 60 stdbuf -oL /tmp/scp_$1_$2_$3 > gpurun_out/scp/sweep_w$1_s$2_m$3.txt 2>&1
done
cat gpurun_out/scp/sweep_*.txt | sort -t= -k2,2n -k8 | awk '{print}' | sort -k1,1 -k2,2 -k10,10nr | head -0
