"""Per-layer timeline of configs[1] round trips issued back to back (bench.py back_to_back): a
polling thread stamps when each layer of every swap-out / swap-in first reports ready.
Usage: python tools/b2b_timeline.py [--k 4] [--requests 64] [--dma-piece-mib P]"""
import argparse
import json
import os
import sys
import threading
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--k", type=int, default=4)
    ap.add_argument("--requests", type=int, default=64)
    ap.add_argument("--dma-piece-mib", type=int, default=0)
    ap.add_argument("--inflight", type=int, default=2)
    a = ap.parse_args()
    import torch
    import bench
    import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg
    torch.cuda.init()
    sb = bench.SwapBench(aeg, bench.QWEN7B, a.requests, aeg.KERNEL_AUTO, dma_piece_mib=a.dma_piece_mib,
                         dev_batches=a.inflight + 1, host_batches=a.inflight, timing=False).setup()
    ctx, sht, n, L = sb.ctx, sb.sht, sb.n, sb.L
    seen, watch, lock, stop = {}, [], threading.Lock(), [False]

    def poller():
        while not stop[0]:
            with lock:
                items = list(watch)
            for key in items:
                (kind, j, x, l) = key
                if key not in seen and ctx.layer_ready(x, l, aeg.READY_QUERY):
                    seen[key] = (time.perf_counter() - t0) * 1e3
    th = threading.Thread(target=poller, daemon=True)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    th.start()
    inflight, enq = [], []
    for j in range(a.k):
        if len(inflight) == a.inflight:
            for t in inflight.pop(0):
                ctx.layer_ready(t, -1, aeg.READY_BLOCK)
        tj = (time.perf_counter() - t0) * 1e3
        hc = ctx.kv_alloc(aeg.POOL_HOST, sht, n)
        nd = ctx.kv_alloc(aeg.POOL_DEVICE, sht, n)
        x = ctx.kv_swap_out(sht, sb.src_c, hc, flags=aeg.FREE_SRC)
        y = ctx.kv_swap_in(sht, hc, nd, flags=aeg.FREE_SRC)
        enq.append((round(tj, 1), round((time.perf_counter() - t0) * 1e3, 1)))
        with lock:
            watch.extend([("out", j, x, l) for l in range(L)] + [("in", j, y, l) for l in range(L)])
        inflight.append((x, y))
        sb.src_c = nd
    for xs in inflight:
        for t in xs:
            ctx.layer_ready(t, -1, aeg.READY_BLOCK)
    time.sleep(0.05)
    stop[0] = True
    th.join()
    out = {"k": a.k, "enqueue_ms": enq, "rt": []}
    for j in range(a.k):
        o = [round(v, 1) for (kd, jj, x, l), v in sorted(seen.items(), key=lambda kv: (kv[0][0], kv[0][1], kv[0][3]))
             if kd == "out" and jj == j]
        i = [round(v, 1) for (kd, jj, x, l), v in sorted(seen.items(), key=lambda kv: (kv[0][0], kv[0][1], kv[0][3]))
             if kd == "in" and jj == j]
        out["rt"].append({"out": o, "in": i})
    print(json.dumps(out))
    ctx.shutdown()


if __name__ == "__main__":
    main()
