#!/bin/bash
# paged -> paged (migrate) kernels over pools spread like the C3 leg's (SPREAD x 1 GiB), for BULKW
# geometries (warps per CTA x smem KiB)
mkdir -p gpurun_out/mgeom
for w in "4 192" "8 192" "16 192" "8 96"; do
  set -- $w
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -DAEG_BW_WARPS=$1 -DAEG_BW_SMEM_KIB=$2 \
    -o /tmp/mg_$1_$2 tools/small_chunk_probe.cu || continue
  for sp in 2 30; do
    MIGRATE=1 SPREAD=$sp timeout 120 /tmp/mg_$1_$2 > gpurun_out/mgeom/w$1_s$2_sp$sp.txt 2>&1
  done
done
for f in gpurun_out/mgeom/*.txt; do echo "== $f"; grep -E "LSU|BULK" $f; done
