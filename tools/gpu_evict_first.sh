#!/bin/bash
# A/B: BULKW bulk copies with an L2 evict_first policy vs the default, in the C2 step (in-step
# gather / scatter next to the PCIe DMA) and alone.  Interleaved repeats against box drift.
mkdir -p gpurun_out/ef
for rep in 1 2; do
for v in "" "-DAEG_BW_EVICT_FIRST"; do
  AEG_NVCC_EXTRA="$v" python -m paper_conf_sosp_xiang0qyzyzl0025_b200.build --force > /dev/null 2>&1
  AEG_BENCH_NO_REBUILD=1 timeout 400 python bench.py --no-switch --no-c5 --no-cpu --no-migrate --steps 8 --warmup 3 \
      --leg-budget-s 300 > gpurun_out/ef/b.json 2> /dev/null
  python -c "
import json; d=json.loads(open('gpurun_out/ef/b.json').read().strip().splitlines()[-1]); r=d['roofline']
od=d.get('one_direction') or {}; ka=d.get('kernel_alone') or {}
print('variant=[$v]', 'value', d['value'], 'gather', r['achieved'], r['frac'], 'scatter', r['scatter_achieved'], 'out_alone_kernel', (od.get('swap_out') or {}).get('kernel_GBps'), 'in_alone_kernel', (od.get('swap_in') or {}).get('kernel_GBps'), 'alone', ka.get('gather'), ka.get('scatter'))"
done
done
python -m paper_conf_sosp_xiang0qyzyzl0025_b200.build --force > /dev/null 2>&1
