"""N3 — fragmentation of the unified CPU KV cache on synthetic alloc/free traces (CPU only).

PAPER.md:2030-2033 (§7.3, Fig. 16): fragmentation is "the ratio of unused memory to peak allocated
memory"; "Aegaeon achieves proportional memory utilization across different block shapes, keeping
overall fragmentation below 20%".  The slab size is "customizable"
(PAPER.md:1468-1471).  This replays seeded traces of six KV shapes (S0-S5) through libaegkv's slab
allocator (host-only context: the same C++ code as the GPU build, no CUDA) for several slab sizes.

Trace recipe: per model a Poisson request stream (popularity skewed 1/rank), prompt +
output lengths lognormal (ShareGPT-like means ~ 600 / 300 tokens), a request holds ceil(T/16) blocks
for an exponential residence time; load set (Little's law) for a target mean occupancy of the pool (default 50% and 70%); the
achieved occupancy and any OOMs are reported next to each fragmentation value.

    python tools/fragmentation.py [--events N] [--out profiles/fragmentation.json]
"""
from __future__ import annotations

import argparse
import heapq
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

GIB = 1 << 30
# S0-S5: (name, L, H, D) at 16-bit, 16-token blocks
SHAPES = [("S0 Qwen-7B", 32, 32, 128), ("S1 InternLM2.5-7B", 32, 8, 128), ("S2 LLaMA-13B", 40, 40, 128),
          ("S3 Qwen-72B/TP4", 80, 16, 128), ("S4 Qwen-1.8B", 24, 16, 128), ("S5 Yi-9B", 48, 4, 128)]


def trace(n_events: int, pool_bytes: int, seed: int = 3000, occupancy: float = 0.5):
    """Seeded list of (time, kind, model, blocks) events; kind 'a' alloc, 'f' free of that request."""
    g = np.random.Generator(np.random.PCG64(seed))
    pop = 1.0 / np.arange(1, len(SHAPES) + 1)
    pop /= pop.sum()
    block = [L * 2 * H * D * 2 * 16 for _, L, H, D in SHAPES]
    mean_tokens = np.exp(np.log(600) + 0.32) + np.exp(np.log(300) + 0.32)   # E[lognormal] = e^(mu + s^2/2)
    mean_bytes = sum(p * b * mean_tokens / 16 for p, b in zip(pop, block))
    hold = 30.0                                       # mean residence (s)
    rate = occupancy * pool_bytes / (mean_bytes * hold)   # Little's law: mean used bytes
    t, ev, heap, rid = 0.0, [], [], 0
    while len(ev) < n_events:
        t += g.exponential(1.0 / rate)
        while heap and heap[0][0] <= t:
            ft, r, m, nb = heapq.heappop(heap)
            ev.append((ft, "f", m, r))
        m = int(g.choice(len(SHAPES), p=pop))
        tokens = int(g.lognormal(np.log(600), 0.8)) + int(g.lognormal(np.log(300), 0.8))
        nb = -(-max(1, tokens) // 16)
        ev.append((t, "a", m, rid))
        heapq.heappush(heap, (t + g.exponential(hold), rid, m, nb))
        ev[-1] = (t, "a", m, rid, nb)
        rid += 1
    return ev


def run(ev, pool_bytes: int, slab_bytes: int):
    import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg
    cfg = aeg.default_config(device_kv_bytes=slab_bytes, host_kv_bytes=pool_bytes, dev_slab_bytes=slab_bytes,
                             host_slab_bytes=slab_bytes, flags=aeg.CFG_HOST_ONLY | aeg.CFG_NO_DAEMON)
    ctx = aeg.Context(0, cfg)
    shapes = [(L, H, D, 2, 16) for _, L, H, D in SHAPES]
    live, oom = {}, 0
    samples = []
    peak = (0, 0, None)
    names = [n for n, _, _, _ in SHAPES]
    block = {n: L * 2 * H * D * 2 * 16 for n, L, H, D in SHAPES}
    shape_peak = {n: 0 for n in names}        # per-shape peak allocated (assigned slab) bytes
    shape_frag = {n: [] for n in names}       # per-shape unused / peak allocated, at every event
    for e in ev:
        if e[1] == "a":
            _, _, m, r, nb = e
            try:
                live[r] = ctx.kv_alloc(aeg.POOL_HOST, shapes[m], nb)
            except aeg.AegError:
                oom += 1
                continue
        else:
            r = e[3]
            if r in live:
                ctx.kv_free(aeg.POOL_HOST, live.pop(r))
        s = ctx.stats(aeg.POOL_HOST)
        samples.append((s.assigned_bytes, s.used_bytes, s.peak_assigned_bytes))
        cur = {}
        for i in range(s.n_shapes):
            p = s.per_shape[i]
            nm = [n for n, L_, H, D in SHAPES if L_ == p.shape.num_layers and H == p.shape.num_kv_heads][0]
            cur[nm] = (p.slabs * slab_bytes, p.owned_blocks * block[nm])
        for nm in names:
            asg, used = cur.get(nm, (0, 0))
            shape_peak[nm] = max(shape_peak[nm], asg)
            if shape_peak[nm]:
                shape_frag[nm].append((asg - used) / shape_peak[nm])
        if s.assigned_bytes > peak[0]:
            per = {}
            for i in range(s.n_shapes):
                p = s.per_shape[i]
                L = p.shape.num_layers
                name = [n for n, L_, H, D in SHAPES if L_ == L and H == p.shape.num_kv_heads][0]
                bb = L * 2 * p.shape.num_kv_heads * p.shape.head_dim * 2 * 16
                per[name] = 1 - p.owned_blocks * bb / (p.slabs * slab_bytes)
            peak = (s.assigned_bytes, s.used_bytes, per)
    ctx.shutdown()
    a = np.array(samples, dtype=np.float64)
    a = a[len(a) // 10:]                       # drop the fill-up transient (first 10% of events)
    frag = (a[:, 0] - a[:, 1]) / a[:, 2]       # Fig. 16: unused / peak allocated, at every event
    occ = a[:, 1] / pool_bytes
    return {"slab_GiB": slab_bytes / GIB, "events": len(ev), "oom_allocs": oom,
            "per_shape_frag_unused_over_peak_allocated_mean": {
                n: round(float(np.mean(v[len(v) // 10:])), 4) for n, v in shape_frag.items() if v},
            "occupancy_used_over_pool_mean": round(float(occ.mean()), 4),
            "occupancy_used_over_pool_max": round(float(occ.max()), 4),
            "frag_unused_over_peak_allocated_mean": round(float(frag.mean()), 4),
            "frag_unused_over_peak_allocated_p90": round(float(np.quantile(frag, 0.9)), 4),
            "frag_at_peak_allocated": round(1 - peak[1] / peak[0], 4) if peak[0] else None,
            "peak_allocated_GiB": round(peak[0] / GIB, 1),
            "per_shape_unused_over_assigned_at_peak": {k: round(v, 4) for k, v in (peak[2] or {}).items()}}


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--events", type=int, default=60000)
    p.add_argument("--pool-gib", type=int, default=320)     # "Unified CPU KV Cache (320 GB)", Fig. 9
    p.add_argument("--occupancy", default="0.5,0.7")
    p.add_argument("--slabs", default="0.25,0.5,1,2,4")
    p.add_argument("--out", default=os.path.join(ROOT, "profiles", "fragmentation.json"))
    a = p.parse_args()
    from paper_conf_sosp_xiang0qyzyzl0025_b200 import build
    build.build()
    pool = a.pool_gib * GIB
    res = []
    for occ in (float(x) for x in a.occupancy.split(",")):
        ev = trace(a.events, pool, occupancy=occ)
        for s in a.slabs.split(","):
            r = run(ev, pool, int(float(s) * GIB))
            r["target_mean_occupancy"] = occ
            res.append(r)
    out = {"what": "N3 fragmentation of the unified CPU KV cache (slab allocator of libaegkv, host-only)",
           "paper": "overall < 20% (PAPER.md:2068-2070, Fig. 16)", "pool_GiB": a.pool_gib, "results": res}
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    json.dump(out, open(a.out, "w"), indent=1)
    for r in res:
        print(json.dumps(r))


if __name__ == "__main__":
    main()
