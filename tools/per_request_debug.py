"""Debug: per-request swap-ins issued back to back — when does each request (and request 0's layers)
become ready, and in what order does the library enqueue its ops (trace)?"""
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import aeg_inputs as gi  # noqa: E402
import bench  # noqa: E402
import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg  # noqa: E402

sh = bench.QWEN7B
bb = aeg.KVShape.of(sh).block_bytes()
g = gi.rng(31)
lens = [int(g.lognormal(np.log(600), 0.8)) + int(g.lognormal(np.log(300), 0.8)) for _ in range(32)]
nblk = [-(-max(1, t) // 16) for t in lens]
GIB = 1 << 30
nreq = int(os.environ.get("NREQ", "12"))
KERN = {"auto": aeg.KERNEL_AUTO, "lsu": aeg.KERNEL_LSU, "bulk": aeg.KERNEL_BULK}[os.environ.get("KERNEL", "auto")]
SLOTS = int(os.environ.get("SLOTS", "3"))
SLOT_MIB = int(os.environ.get("SLOT_MIB", "1024"))
ctx = aeg.Context(0, aeg.default_config(device_kv_bytes=(sum(nblk) * bb // GIB + 4) * GIB,
                                        host_kv_bytes=(sum(nblk) * bb // GIB + 4) * GIB, kernel=KERN,
                                        staging_slots=SLOTS, staging_slot_bytes=SLOT_MIB << 20))
host = [ctx.kv_alloc(aeg.POOL_HOST, sh, n) for n in nblk[:nreq]]
cons = bench.new_stream(torch)
REPS = int(os.environ.get('REPS', '2'))
for rep in range(REPS):
    dev = [ctx.kv_alloc(aeg.POOL_DEVICE, sh, n) for n in nblk[:nreq]]
    torch.cuda.synchronize()
    if rep == REPS - 1:
        ctx.trace_enable(True)
    e0 = torch.cuda.Event(enable_timing=True)
    e0.record(cons)
    ctx.stream_fence(cons.cuda_stream)
    xs = [ctx.kv_swap_in(sh, h, d) for h, d in zip(host, dev)]
    lay = []
    for l in range(32):
        s = bench.new_stream(torch)
        ctx.layer_ready(xs[0], l, aeg.READY_WAIT_STREAM, s.cuda_stream)
        e = torch.cuda.Event(enable_timing=True)
        e.record(s)
        lay.append(e)
    evs = []
    for x in xs:
        s = bench.new_stream(torch)
        ctx.layer_ready(x, -1, aeg.READY_WAIT_STREAM, s.cuda_stream)
        e = torch.cuda.Event(enable_timing=True)
        e.record(s)
        evs.append(e)
    torch.cuda.synchronize()
    ready = [e0.elapsed_time(e) for e in evs]
    cum = np.cumsum([n * bb for n in nblk[:nreq]]) / 55.6e6
    if rep == REPS - 1:
        print("request 0 layers ready (ms):", [round(e0.elapsed_time(e), 1) for e in lay])
        for i in range(nreq):
            print(i, nblk[i], f"ready {ready[i]:.1f} ideal {cum[i]:.1f}")
        tr = ctx.trace_read().splitlines()
        ctx.trace_enable(False)
        # first lines per stream kind, abbreviated
        print(len(tr), "trace lines; first 40, abbreviated:")
        for line in tr[:40]:
            print(line[:140])
    for x in xs:
        ctx.xfer_release(x)
    for d in dev:
        ctx.kv_free(aeg.POOL_DEVICE, d)
ctx.shutdown()
