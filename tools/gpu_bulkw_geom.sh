#!/bin/bash
# BULKW geometry x piece size sweep at one CTA per SM (96 KiB-class shared memory), gather / scatter /
# migrate over 30 GB-spread tables: picks the product geometry and the piece size per chunk size.
mkdir -p gpurun_out/bwgeom4
for w in "4 96" "8 96" "6 96" "4 80" "8 112" "4 128"; do
  set -- $w
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -DAEG_BW_WARPS=$1 -DAEG_BW_SMEM_KIB=$2 \
    -o /tmp/bw_$1_$2 tools/small_chunk_probe.cu || continue
  SWEEP=1 SPREAD=30 CTAS_PER_SM=1 CHUNKS=2048,4096,8192,16384,32768,262144,327680 timeout 200 /tmp/bw_$1_$2 > gpurun_out/bwgeom4/gs_w$1_s$2.txt 2>&1
  SWEEP=1 SPREAD=30 CTAS_PER_SM=1 MIGRATE=1 CHUNKS=32768,327680 timeout 100 /tmp/bw_$1_$2 > gpurun_out/bwgeom4/mig_w$1_s$2.txt 2>&1
done
echo done
