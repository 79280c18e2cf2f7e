#!/bin/bash
# In-step gather / scatter of the C2 step vs the BULKW grid size (CTAs; one per SM at 148) and
# geometry, rebuilt per variant (AEG_NVCC_EXTRA).  Side legs off; 8 timed steps.
mkdir -p gpurun_out/grid
for v in "-DAEG_BW_GRID=148" "-DAEG_BW_GRID=132" "-DAEG_BW_GRID=120" "-DAEG_BW_GRID=100" "-DAEG_BW_GRID=296" \
         "-DAEG_BW_WARPS=4 -DAEG_BW_SMEM_KIB=80" "-DAEG_BW_WARPS=8 -DAEG_BW_SMEM_KIB=128"; do
  AEG_NVCC_EXTRA="$v" python -m paper_conf_sosp_xiang0qyzyzl0025_b200.build --force > /dev/null 2>&1
  timeout 400 python bench.py --no-switch --no-c5 --no-cpu --no-migrate --steps 8 --warmup 3 --leg-budget-s 200 \
      > gpurun_out/grid/b.json 2> /dev/null
  python -c "
import json; d=json.loads(open('gpurun_out/grid/b.json').read().strip().splitlines()[-1]); r=d['roofline']
od=d.get('one_direction') or {}
print('$v', d['value'], r['achieved'], r['frac'], r['scatter_achieved'], (od.get('swap_out') or {}).get('kernel_GBps'), (od.get('swap_in') or {}).get('kernel_GBps'))"
done
python -m paper_conf_sosp_xiang0qyzyzl0025_b200.build --force > /dev/null 2>&1
