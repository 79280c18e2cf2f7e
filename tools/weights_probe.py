"""Weight staging alone (H7): Llama-7B shapes (13.5 GB) staged from a pageable Model Cache through
the pinned Stage Buffer, for several host-thread counts and chunk sizes; GB/s and pipeline stall
counters (aeg_weights_stats).  Run on the GPU box:  python tools/weights_probe.py"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402
import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg  # noqa: E402

GIB, MIB = 1 << 30, 1 << 20


def main():
    descs, caches = bench.model_caches(["llama-7b"])
    d = descs["llama-7b"]
    total = sum(x["rows"] * x["cols"] * 2 for x in d)
    out = []
    for threads, chunk_mib in [(4, 64), (8, 64), (12, 64), (16, 64), (12, 16), (12, 128), (16, 32)]:
        cfg = aeg.default_config(device_kv_bytes=GIB, host_kv_bytes=GIB, device_weight_bytes=16 * GIB,
                                 host_threads=threads, stage_chunk_bytes=chunk_mib * MIB)
        ctx = aeg.Context(0, cfg)
        ts = []
        for _ in range(3):
            ctx.weights_reset(0)
            t0 = time.perf_counter()
            _, x = ctx.weights_stage(d)
            ctx.layer_ready(x, -1, aeg.READY_BLOCK)
            ts.append(time.perf_counter() - t0)
            ctx.xfer_release(x)
        n, wf, ws = ctx.weights_stats()
        ctx.shutdown()
        best = min(ts)
        r = {"threads": threads, "chunk_MiB": chunk_mib, "best_ms": round(best * 1e3, 1),
             "GBps": round(total / best / 1e9, 1), "chunks": n, "issuer_wait_fill_ms": round(wf, 1),
             "fill_wait_slot_ms": round(ws, 1)}
        print(json.dumps(r), flush=True)
        out.append(r)
    json.dump(out, open(os.path.join(ROOT, "gpurun_out", "weights_probe.json"), "w"), indent=1)


if __name__ == "__main__":
    main()
