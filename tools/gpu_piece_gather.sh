#!/bin/bash
# In-step gather / scatter rate and round-trip value vs the swap-out D2H piece size (sub-layer rule ❷).
mkdir -p gpurun_out/piece
for p in 32 128 512 1024; do
  timeout 400 python bench.py --no-switch --no-c5 --no-cpu --no-migrate --steps 8 --warmup 3 --leg-budget-s 200 \
      --dma-piece-mib $p > gpurun_out/piece/b$p.json 2> /dev/null
  python -c "
import json; d=json.loads(open('gpurun_out/piece/b$p.json').read().strip().splitlines()[-1]); r=d['roofline']
od=d.get('one_direction') or {}
print('piece_mib=$p', 'value', d['value'], 'gather', r['achieved'], r['frac'], 'scatter', r['scatter_achieved'], 'out_alone_kernel', (od.get('swap_out') or {}).get('kernel_GBps'), 'out_alone', (od.get('swap_out') or {}).get('GBps'), 'e2e_l0', d['e2e']['round_trip_layer0_ready_ms_p50'])"
done
