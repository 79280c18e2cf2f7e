"""GPU parity for H1-H4 + H6 on C1 (BASELINE.json configs[0]): every byte of the device and host
pool images after swap-out and swap-in equals the oracle's (O5/O6 applied to the same generated
inputs), for every combination of slab layouts and both kernel implementations, with staging slots
small enough to split layers into several segments and large enough to pack layers together."""
import numpy as np
import pytest

import aeg_inputs as gi
import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg
from aeg_inputs import dev as D
from oracle import kv as OK
from oracle.rules import check
from oracle.shape import KVShape

from .gpu_harness import SEED, Side, fill_blocks, first_diff, poison_blocks, require_gpu

pytestmark = pytest.mark.gpu

SH = KVShape(2, 4, 64, 2, 16)            # configs[0]: 2 layers, 4 KV heads, d=64, fp16, 16-token blocks
KIB = 1024


def make(dev_layout, host_layout, kernel, slot, host_slab=256 * KIB, timing=False):
    cfg = aeg.default_config(device_kv_bytes=32 * 256 * KIB, host_kv_bytes=64 * host_slab,
                             dev_slab_bytes=256 * KIB, host_slab_bytes=host_slab,
                             dev_slab_layout=dev_layout, host_slab_layout=host_layout,
                             staging_slot_bytes=slot, staging_slots=3, stage_ring_bytes=4 << 20,
                             stage_chunk_bytes=1 << 20, device_weight_bytes=8 << 20, table_arena_bytes=4 << 20,
                             host_threads=2, kernel=kernel, flags=aeg.CFG_TIMING if timing else 0)
    ctx = aeg.Context(0, cfg)
    dev = Side(ctx, aeg.POOL_DEVICE, cfg.device_kv_bytes, cfg.dev_slab_bytes, dev_layout)
    host = Side(ctx, aeg.POOL_HOST, cfg.host_kv_bytes, cfg.host_slab_bytes, host_layout)
    return ctx, dev, host


def age(side: Side, sh, cfg_id=1):
    """Seeded churn so block tables are fragmented across slabs (SURVEY §8(d) placement realism)."""
    live = []
    k = side.geom.slab_bytes // sh.block_bytes()
    for op, v in gi.churn_ops(cfg_id, capacity_blocks=(side.geom.nbytes // side.geom.slab_bytes) * k // 2,
                              hi_blocks=6):
        if op == "alloc":
            live.append(side.alloc(sh, v))
        else:
            c, o = live[v]
            if c is not None:
                side.free(c, o)
                live[v] = (None, None)
    return [x for x in live if x[0] is not None]


def requests(dev: Side, dimg, sh):
    lens = gi.request_lengths(1, 8, 1, 256, forced=(1, 16, 17, 255, 256))
    c_all, o_all = [], []
    for r, T in enumerate(lens):
        c, o = dev.alloc(sh, sh.blocks_for(T))
        fill_blocks(dev, dimg, sh, o, [(r, j) for j in range(len(o))])
        c_all += list(c)
        o_all += list(o)
    return np.array(c_all, dtype=np.uint64), o_all


LAYOUTS = [(aeg.LAYER_MAJOR, aeg.LAYER_MAJOR), (aeg.BLOCK_MAJOR, aeg.LAYER_MAJOR),
           (aeg.LAYER_MAJOR, aeg.BLOCK_MAJOR), (aeg.BLOCK_MAJOR, aeg.BLOCK_MAJOR)]


@pytest.mark.parametrize("kernel", [aeg.KERNEL_LSU, aeg.KERNEL_BULK, aeg.KERNEL_WARP, aeg.KERNEL_BULKW])
@pytest.mark.parametrize("layouts", LAYOUTS)
@pytest.mark.parametrize("slot", [1 << 20, 8 << 20])
def test_c1_round_trip_full_images(layouts, kernel, slot):
    require_gpu()
    ctx, dev, host = make(*layouts, kernel, slot, host_slab=320 * KIB)
    try:
        dev.poison(gi.TAG_NEVER)
        host.poison(gi.TAG_NEVER)
        dimg, himg = dev.poison_img(gi.TAG_NEVER), host.poison_img(gi.TAG_NEVER)
        age(dev, SH)
        dc, do = requests(dev, dimg, SH)
        # the CUDA and NumPy generators agree on the whole input image
        assert first_diff(dev.read(), dimg) is None
        hc, ho = host.alloc(SH, len(do))
        x = ctx.kv_swap_out(SH.as_tuple(), dc, hc, flags=aeg.FREE_SRC)
        xo = dev.oracle.begin(do)
        dev.oracle.free(do)
        himg = OK.swap_out(dimg, dev.geom, himg, host.geom, SH, do, ho)
        ctx.layer_ready(x, -1, aeg.READY_BLOCK)
        assert first_diff(host.read(), himg) is None
        assert first_diff(dev.read(), dimg) is None          # swap-out leaves the device as it was
        dev.oracle.complete(xo)
        # swap back in, into fresh blocks (the quarantined sources are reclaimed first)
        nc, no = dev.alloc(SH, len(do))
        poison_blocks(dev, dimg, SH, no)
        y = ctx.kv_swap_in(SH.as_tuple(), hc, nc)
        dimg = OK.swap_in(himg, host.geom, dimg, dev.geom, SH, ho, no)
        for l in range(SH.L):
            ctx.layer_ready(y, l, aeg.READY_BLOCK)
        ctx.layer_ready(y, -1, aeg.READY_BLOCK)
        assert first_diff(dev.read(), dimg) is None
        assert first_diff(host.read(), himg) is None
        ctx.xfer_release(x)
        ctx.xfer_release(y)
    finally:
        ctx.shutdown()


def test_c1_swap_in_chained_on_swap_out_without_host_sync():
    """Fig. 10 ③: the swap-in is issued right after the swap-out, with no host synchronisation;
    a long delay kernel holds the swap-out back, so only the per-layer event waits (rule ❷) keep
    the H2D of layer l behind the D2H of layer l.  The consumer waits per layer (rule ❶)."""
    require_gpu()
    import torch
    ctx, dev, host = make(aeg.LAYER_MAJOR, aeg.BLOCK_MAJOR, aeg.KERNEL_LSU, 1 << 20)
    try:
        dev.poison(gi.TAG_NEVER)
        host.poison(gi.TAG_NEVER)
        dimg, himg = dev.poison_img(gi.TAG_NEVER), host.poison_img(gi.TAG_NEVER)
        dc, do = requests(dev, dimg, SH)
        hc, ho = host.alloc(SH, len(do))
        s = torch.cuda.Stream()
        gate = D.Gate()
        gate.close_on(s.cuda_stream)                  # the "prefill" runs until gate.open()
        ctx.stream_fence(s.cuda_stream)               # swap-out ordered after the "prefill"
        ctx.trace_enable(True)
        x = ctx.kv_swap_out(SH.as_tuple(), dc, hc, flags=aeg.FREE_SRC)
        nc, no = dev.alloc(SH, len(do))               # sources are quarantined: fresh blocks
        assert not set(map(tuple, no)) & set(map(tuple, do))
        xo = dev.oracle.begin(do)
        dev.oracle.free(do)
        y = ctx.kv_swap_in(SH.as_tuple(), hc, nc)
        assert not ctx.layer_ready(x, 0, aeg.READY_QUERY)   # still held back by the gate
        assert not ctx.layer_ready(y, 0, aeg.READY_QUERY)   # rule ❷: the swap-in waits for it
        gate.open()
        himg = OK.swap_out(dimg, dev.geom, himg, host.geom, SH, do, ho)
        exp = OK.swap_in(himg, host.geom, dimg, dev.geom, SH, ho, no)
        cons = torch.cuda.Stream()
        for l in range(SH.L):
            ctx.layer_ready(y, l, aeg.READY_WAIT_STREAM, cons.cuda_stream)
        cons.synchronize()
        ctx.layer_ready(y, -1, aeg.READY_BLOCK)
        got = dev.read()
        for h in no:
            for l in range(SH.L):
                o = OK.addr(dev.geom, SH, h, l)
                assert np.array_equal(got[o:o + SH.chunk_bytes()], exp[o:o + SH.chunk_bytes()])
        dev.oracle.complete(xo)
        log = parse_trace(ctx.trace_read())
        # the consumer kernel of every layer, on the stream that waited per layer (rule ❶)
        log.append(("use", "u0x%x" % cons.cuda_stream,
                    [f"D:{s}:{j}:{l}" for (s, j) in no for l in range(SH.L)]))
        assert check(log)                             # ❶❷❸ hold on the library's own primitive log
    finally:
        ctx.shutdown()


SHP = KVShape(2, 16, 64, 2, 16)           # Cl = 64 KiB: a 75-block layer (4.7 MiB) is never packed


@pytest.mark.parametrize("host_layout", [aeg.LAYER_MAJOR, aeg.BLOCK_MAJOR])
@pytest.mark.parametrize("slot", [2 << 20, 8 << 20])
def test_swap_in_waits_per_d2h_piece(host_layout, slot):
    """Rule ❷ at sub-layer granularity: with 1 MiB D2H pieces a swap-out's layer is
    moved as several block-range pieces, each with its own event, and a chained swap-in waits for
    the pieces holding its blocks instead of the whole layer.  The swap-in is issued while a gate
    holds the swap-out back; the library's own primitive log must satisfy ❶❷❸ and the result must
    equal the oracle (O5, O6) on every chunk.  slot = 2 MiB also splits each layer into segments."""
    require_gpu()
    import torch
    MIB = 1 << 20
    cfg = aeg.default_config(device_kv_bytes=32 * MIB, host_kv_bytes=24 * 1280 * KIB,
                             dev_slab_bytes=MIB, host_slab_bytes=1280 * KIB,
                             dev_slab_layout=aeg.LAYER_MAJOR, host_slab_layout=host_layout,
                             staging_slot_bytes=slot, staging_slots=3, stage_ring_bytes=4 << 20,
                             stage_chunk_bytes=1 << 20, device_weight_bytes=8 << 20, table_arena_bytes=4 << 20,
                             host_threads=2, kernel=aeg.KERNEL_AUTO, dma_piece_mib=1, pack_layer_mib=1)
    ctx = aeg.Context(0, cfg)
    dev = Side(ctx, aeg.POOL_DEVICE, cfg.device_kv_bytes, cfg.dev_slab_bytes, aeg.LAYER_MAJOR)
    host = Side(ctx, aeg.POOL_HOST, cfg.host_kv_bytes, cfg.host_slab_bytes, host_layout)
    try:
        dev.poison(gi.TAG_NEVER)
        host.poison(gi.TAG_NEVER)
        dimg, himg = dev.poison_img(gi.TAG_NEVER), host.poison_img(gi.TAG_NEVER)
        dc, do = requests(dev, dimg, SHP)
        assert len(do) * SHP.chunk_bytes() > 4 * MIB
        hc, ho = host.alloc(SHP, len(do))
        s = torch.cuda.Stream()
        gate = D.Gate()
        gate.close_on(s.cuda_stream)
        ctx.stream_fence(s.cuda_stream)
        ctx.trace_enable(True)
        x = ctx.kv_swap_out(SHP.as_tuple(), dc, hc, flags=aeg.FREE_SRC)
        nc, no = dev.alloc(SHP, len(do))
        xo = dev.oracle.begin(do)
        dev.oracle.free(do)
        # read the host blocks in reverse: the swap-in's first piece needs the swap-out's last one
        y = ctx.kv_swap_in(SHP.as_tuple(), np.ascontiguousarray(hc[::-1]), nc)
        assert not ctx.layer_ready(y, 0, aeg.READY_QUERY)
        gate.open()
        himg = OK.swap_out(dimg, dev.geom, himg, host.geom, SHP, do, ho)
        exp = OK.swap_in(himg, host.geom, dimg, dev.geom, SHP, list(reversed(ho)), no)
        cons = torch.cuda.Stream()
        for l in range(SHP.L):
            ctx.layer_ready(y, l, aeg.READY_WAIT_STREAM, cons.cuda_stream)
        cons.synchronize()
        ctx.layer_ready(y, -1, aeg.READY_BLOCK)
        assert first_diff(dev.read(), exp) is None
        assert first_diff(host.read(), himg) is None
        dev.oracle.complete(xo)
        text = ctx.trace_read()
        log = parse_trace(text)
        # the D2H of a layer is several ops (pieces), and the H2D waits before several ops per layer
        d2h_ops = [e for e in log if e[0] == "op" and e[1] == "d2h"]
        h2d_ops = [e for e in log if e[0] == "op" and e[1] == "h2d"]
        assert len(d2h_ops) >= 5 * SHP.L and len(h2d_ops) >= 5 * SHP.L
        log.append(("use", "u0x%x" % cons.cuda_stream,
                    [f"D:{s}:{j}:{l}" for (s, j) in no for l in range(SHP.L)]))
        assert check(log)
        ctx.xfer_release(x)
        ctx.xfer_release(y)
    finally:
        ctx.shutdown()


def test_swap_in_from_two_piecewise_swap_outs():
    """One swap-in reads, in a shuffled order, half of the host blocks written by each of two
    in-flight swap-outs that both used D2H pieces: before each of its H2D pieces it must wait for
    the right piece of each writer (two piece dependencies, different highest pieces).  Gate-held,
    checked by the happens-before checker on the library's log and against the oracle."""
    require_gpu()
    import torch
    MIB = 1 << 20
    cfg = aeg.default_config(device_kv_bytes=48 * MIB, host_kv_bytes=40 * MIB,
                             dev_slab_bytes=MIB, host_slab_bytes=MIB,
                             dev_slab_layout=aeg.BLOCK_MAJOR, host_slab_layout=aeg.LAYER_MAJOR,
                             staging_slot_bytes=8 << 20, staging_slots=3, stage_ring_bytes=4 << 20,
                             stage_chunk_bytes=1 << 20, device_weight_bytes=8 << 20, table_arena_bytes=4 << 20,
                             host_threads=2, kernel=aeg.KERNEL_AUTO, dma_piece_mib=1, pack_layer_mib=1)
    ctx = aeg.Context(0, cfg)
    dev = Side(ctx, aeg.POOL_DEVICE, cfg.device_kv_bytes, cfg.dev_slab_bytes, aeg.BLOCK_MAJOR)
    host = Side(ctx, aeg.POOL_HOST, cfg.host_kv_bytes, cfg.host_slab_bytes, aeg.LAYER_MAJOR)
    try:
        dev.poison(gi.TAG_NEVER)
        host.poison(gi.TAG_NEVER)
        dimg, himg = dev.poison_img(gi.TAG_NEVER), host.poison_img(gi.TAG_NEVER)
        batches = []
        for m in (1, 2):
            c, o = dev.alloc(SHP, 96)
            fill_blocks(dev, dimg, SHP, o, [(0, j) for j in range(96)], m=m)
            batches.append((c, o))
        s = torch.cuda.Stream()
        gate = D.Gate()
        gate.close_on(s.cuda_stream)
        ctx.stream_fence(s.cuda_stream)
        ctx.trace_enable(True)
        xs, hosts = [], []
        for c, o in batches:
            hc, ho = host.alloc(SHP, len(o))
            xs.append(ctx.kv_swap_out(SHP.as_tuple(), c, hc))
            hosts.append((hc, ho))
        # half of each batch's host blocks, interleaved and shuffled
        rng = np.random.default_rng(11)
        pick = [(b, i) for b in (0, 1) for i in rng.choice(96, size=48, replace=False)]
        pick = [pick[k] for k in rng.permutation(len(pick))]
        hsel_c = np.array([hosts[b][0][i] for b, i in pick], dtype=np.uint64)
        hsel_o = [hosts[b][1][i] for b, i in pick]
        nc, no = dev.alloc(SHP, len(pick))
        y = ctx.kv_swap_in(SHP.as_tuple(), hsel_c, nc)
        assert not ctx.layer_ready(y, 0, aeg.READY_QUERY)
        gate.open()
        for (c, o), (hc, ho) in zip(batches, hosts):
            himg = OK.swap_out(dimg, dev.geom, himg, host.geom, SHP, o, ho)
        exp = OK.swap_in(himg, host.geom, dimg, dev.geom, SHP, hsel_o, no)
        ctx.layer_ready(y, -1, aeg.READY_BLOCK)
        for x in xs:
            ctx.layer_ready(x, -1, aeg.READY_BLOCK)
        assert first_diff(dev.read(), exp) is None
        assert first_diff(host.read(), himg) is None
        log = parse_trace(ctx.trace_read())
        assert sum(1 for e in log if e[0] == "op" and e[1] == "h2d") >= 6 * SHP.L
        assert check(log)
    finally:
        ctx.shutdown()


def parse_trace(text):
    """Library trace lines -> oracle.rules log tuples."""
    log = []
    for line in text.splitlines():
        f = line.split()
        if not f:
            continue
        if f[0] == "op":
            kv = dict(x.split("=", 1) for x in f[3:])
            cells = lambda s: [c for c in s.split(",") if c]  # noqa: E731
            log.append(("op", f[1], f[2], cells(kv.get("r", "")), cells(kv.get("w", ""))))
        elif f[0] in ("record", "wait"):
            log.append((f[0], f[1], f[2]))
        elif f[0] == "sync":
            log.append(("sync", f[1]))
    return log


def test_kernel_timing_counters():
    require_gpu()
    ctx, dev, host = make(aeg.LAYER_MAJOR, aeg.LAYER_MAJOR, aeg.KERNEL_LSU, 1 << 20, timing=True)
    try:
        dimg = dev.poison_img(gi.TAG_NEVER)
        dc, do = requests(dev, dimg, SH)
        hc, ho = host.alloc(SH, len(do))
        x = ctx.kv_swap_out(SH.as_tuple(), dc, hc)
        ctx.layer_ready(x, -1, aeg.READY_BLOCK)
        n, b, ms = ctx.kernel_stats(aeg.K_GATHER)
        assert n >= 1 and b == 2 * len(do) * SH.block_bytes() and ms > 0
    finally:
        ctx.shutdown()


def test_layer_readiness_is_monotone_and_live():
    """O9: every layer of a swap eventually becomes ready (liveness) and, once
    QUERY reports it ready, it stays ready (monotonicity); layer l never reports ready while its bytes
    differ from the oracle (safety: checked right after the first ready observation)."""
    require_gpu()
    ctx, dev, host = make(aeg.LAYER_MAJOR, aeg.LAYER_MAJOR, aeg.KERNEL_BULK, 1 << 20)
    try:
        dev.poison(gi.TAG_NEVER)
        host.poison(gi.TAG_NEVER)
        dimg, himg = dev.poison_img(gi.TAG_NEVER), host.poison_img(gi.TAG_NEVER)
        dc, do = requests(dev, dimg, SH)
        hc, ho = host.alloc(SH, len(do))
        x = ctx.kv_swap_out(SH.as_tuple(), dc, hc)
        himg = OK.swap_out(dimg, dev.geom, himg, host.geom, SH, do, ho)
        seen = [False] * SH.L
        for _ in range(1_000_000):
            for l in range(SH.L):
                r = ctx.layer_ready(x, l, aeg.READY_QUERY)
                assert r or not seen[l]
                if r and not seen[l]:
                    seen[l] = True
                    got = host.read()
                    for h in ho:
                        o = OK.addr(host.geom, SH, h, l)
                        assert np.array_equal(got[o:o + SH.chunk_bytes()], himg[o:o + SH.chunk_bytes()])
            if all(seen):
                break
        assert all(seen)
        assert ctx.layer_ready(x, -1, aeg.READY_QUERY) or ctx.layer_ready(x, -1, aeg.READY_BLOCK)
    finally:
        ctx.shutdown()
