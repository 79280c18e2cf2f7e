"""Per-layer completion timeline of a chained C2 round trip (swap-out then swap-in of the same
64-request Qwen-7B batch, as in bench.py's step): the host polls aeg_layer_ready(QUERY) of every
layer of both transfers and stamps when each first reports ready.  Prints one JSON line.
Usage: python tools/roundtrip_timeline.py [--dma-piece-mib P] [--requests N]"""
import argparse
import json
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--dma-piece-mib", type=int, default=0)
    ap.add_argument("--requests", type=int, default=64)
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--kernel", default="auto", choices=["auto", "lsu", "bulk"])
    ap.add_argument("--slots", type=int, default=0)
    ap.add_argument("--no-timing", action="store_true")
    a = ap.parse_args()
    import torch
    import bench
    import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg
    torch.cuda.init()
    kern = {"auto": aeg.KERNEL_AUTO, "lsu": aeg.KERNEL_LSU, "bulk": aeg.KERNEL_BULK}[a.kernel]
    sb = bench.SwapBench(aeg, bench.QWEN7B, a.requests, kern, dma_piece_mib=a.dma_piece_mib, slots=a.slots,
                         timing=not a.no_timing).setup()
    ctx, sht, n, L = sb.ctx, sb.sht, sb.n, sb.L
    out = []
    for rep in range(a.reps):
        hc = ctx.kv_alloc(aeg.POOL_HOST, sht, n)
        nd = ctx.kv_alloc(aeg.POOL_DEVICE, sht, n)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        x = ctx.kv_swap_out(sht, sb.src_c, hc, flags=aeg.FREE_SRC)
        t1 = time.perf_counter()
        y = ctx.kv_swap_in(sht, hc, nd, flags=aeg.FREE_SRC)
        t2 = time.perf_counter()
        pend = [(x, l) for l in range(L)] + [(y, l) for l in range(L)]
        seen = {}
        while pend:
            rest = []
            for (t, l) in pend:
                if ctx.layer_ready(t, l, aeg.READY_QUERY):
                    seen[(t, l)] = (time.perf_counter() - t0) * 1e3
                else:
                    rest.append((t, l))
            pend = rest
        ctx.layer_ready(y, -1, aeg.READY_BLOCK)
        ctx.xfer_release(x)
        ctx.xfer_release(y)
        sb.src_c = nd
        out.append({"enqueue_ms": [round((t1 - t0) * 1e3, 2), round((t2 - t1) * 1e3, 2)],
                    "swap_out_layer_ready_ms": [round(seen[(x, l)], 1) for l in range(L)],
                    "swap_in_layer_ready_ms": [round(seen[(y, l)], 1) for l in range(L)]})
    print(json.dumps({"dma_piece_mib": sb.cfg.dma_piece_mib, "kernel": a.kernel, "slots": sb.cfg.staging_slots,
                      "timing": not a.no_timing, "blocks": n, "runs": out}))
    ctx.shutdown()


if __name__ == "__main__":
    main()
