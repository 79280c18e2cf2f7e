"""Host enqueue cost of aeg_kv_swap_out / aeg_kv_swap_in for small transfers (configs[0] shape):
how much is fixed per call and how much per host run (one copy-engine command per run and layer
group).  Host blocks are either one contiguous run or spread one run per slab."""
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import aeg_inputs as gi  # noqa: E402
import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg  # noqa: E402

sht = gi.KV_SHAPES["tiny"]
KIB = 1024
for slab_kib, slot_mib in ((256, 1), (4096, 1), (256, 8)):
    ctx = aeg.Context(0, aeg.default_config(device_kv_bytes=64 * 256 * KIB, host_kv_bytes=64 * slab_kib * KIB,
                                            dev_slab_bytes=256 * KIB, host_slab_bytes=slab_kib * KIB,
                                            staging_slot_bytes=slot_mib << 20, staging_slots=2, stage_ring_bytes=2 << 20,
                                            stage_chunk_bytes=1 << 20, device_weight_bytes=2 << 20,
                                            table_arena_bytes=2 << 20, host_threads=1))
    for nb in (1, 8, 75):
        src = ctx.kv_alloc(0, sht, nb)
        out, inn = [], []
        for it in range(60):
            torch.cuda.synchronize()
            hc = ctx.kv_alloc(1, sht, nb)
            nd = ctx.kv_alloc(0, sht, nb)
            t0 = time.perf_counter()
            x = ctx.kv_swap_out(sht, src, hc, flags=aeg.FREE_SRC)
            t1 = time.perf_counter()
            y = ctx.kv_swap_in(sht, hc, nd, flags=aeg.FREE_SRC)
            t2 = time.perf_counter()
            ctx.layer_ready(y, -1, aeg.READY_BLOCK)
            ctx.layer_ready(x, -1, aeg.READY_BLOCK)
            ctx.xfer_release(x)
            ctx.xfer_release(y)
            src = nd
            if it >= 10:
                out.append((t1 - t0) * 1e6)
                inn.append((t2 - t1) * 1e6)
        runs = -(-nb // ((slab_kib * KIB) // (2 * 32 * KIB)))
        print(f"slot {slot_mib} MiB host slab {slab_kib:5d} KiB  blocks {nb:3d} (host runs ~{runs:2d}): enqueue swap_out "
              f"{statistics.median(out):6.1f} us, swap_in {statistics.median(inn):6.1f} us", flush=True)
    ctx.shutdown()
# the CUDA calls themselves, for scale
s = torch.cuda.Stream()
h = torch.empty(64 << 10, dtype=torch.uint8, pin_memory=True)
d = torch.empty(64 << 10, dtype=torch.uint8, device="cuda")
ev = torch.cuda.Event()
for name, fn in (("record", lambda: ev.record(s)), ("wait", lambda: s.wait_event(ev)),
                 ("h2d 64K", lambda: d.copy_(h, non_blocking=True))):
    ts = []
    for _ in range(200):
        t0 = time.perf_counter()
        with torch.cuda.stream(s):
            fn()
        ts.append((time.perf_counter() - t0) * 1e6)
    torch.cuda.synchronize()
    print(f"torch {name}: {statistics.median(ts):.1f} us per call (incl. Python)")
