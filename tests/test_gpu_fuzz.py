"""Seeded fuzz against the oracle.  Swap / hand-off: random KV shapes (chunks from 32 B to 128 KiB,
1-6 layers), slab sizes with ragged tails, both slab layouts on each side, every kernel, layer
packing and D2H piece sizes, aged pools; per case a swap-out, a swap-in into fresh blocks and a local
hand-off (fused kernel or copy-engine route), each compared with O5 / O6 / O7 on the whole device and
host pool images (every byte, including everything that must stay untouched); hand-offs between
contexts of different pool geometry (O7); and weight staging with random splits (O8)."""
import numpy as np
import pytest

import aeg_inputs as gi
import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg
from oracle import kv as OK
from oracle.shape import KVShape

from .gpu_harness import Side, fill_blocks, first_diff, poison_blocks, require_gpu

pytestmark = pytest.mark.gpu

MIB = 1 << 20
KERNELS = [aeg.KERNEL_AUTO, aeg.KERNEL_LSU, aeg.KERNEL_BULK, aeg.KERNEL_WARP, aeg.KERNEL_BULKW]


def draw(seed):
    """One case: a shape whose chunk is a multiple of 16 B, slab geometry for both pools, config."""
    r = np.random.default_rng(0xF022 + seed)
    while True:
        L, H = int(r.integers(1, 7)), int(r.choice([1, 2, 3, 5, 8]))
        D, B = int(r.choice([8, 16, 64, 128])), int(r.choice([1, 2, 16, 32]))
        sh = KVShape(L, H, D, 2, B)
        if sh.chunk_bytes() % 16 == 0 and sh.block_bytes() <= 2 * MIB:
            break

    def slab():
        k = int(r.integers(1, 10))
        while k > 1 and k * sh.block_bytes() > 6 * MIB:
            k -= 1
        tail = 16 * int(r.integers(0, max(1, sh.block_bytes() // 16)))   # ragged tail < one block
        s = k * sh.block_bytes() + tail
        return s, max(3, min(12, (16 * MIB) // s))
    (ds, dn), (hs, hn) = slab(), slab()
    return dict(sh=sh, dev_slab=ds, dev_slabs=dn, host_slab=hs, host_slabs=hn,
                dev_layout=int(r.integers(0, 2)), host_layout=int(r.integers(0, 2)),
                kernel=int(r.choice(KERNELS)), pack=int(r.choice([1, 32])), piece=int(r.choice([1, 128])),
                ce=bool(r.integers(0, 2)), rng=r)


@pytest.mark.parametrize("seed", range(64))
def test_fuzz_swap_and_hand_off_match_the_oracle(seed):
    require_gpu()
    c = draw(seed)
    sh, r = c["sh"], c["rng"]
    cfg = aeg.default_config(device_kv_bytes=c["dev_slabs"] * c["dev_slab"],
                             host_kv_bytes=c["host_slabs"] * c["host_slab"],
                             dev_slab_bytes=c["dev_slab"], host_slab_bytes=c["host_slab"],
                             dev_slab_layout=c["dev_layout"], host_slab_layout=c["host_layout"],
                             staging_slot_bytes=MIB, staging_slots=2, stage_ring_bytes=4 * MIB,
                             stage_chunk_bytes=MIB, device_weight_bytes=2 * MIB, table_arena_bytes=4 * MIB,
                             host_threads=1, kernel=c["kernel"], pack_layer_mib=c["pack"],
                             dma_piece_mib=c["piece"])
    ctx = aeg.Context(0, cfg)
    try:
        dev = Side(ctx, aeg.POOL_DEVICE, cfg.device_kv_bytes, cfg.dev_slab_bytes, c["dev_layout"])
        host = Side(ctx, aeg.POOL_HOST, cfg.host_kv_bytes, cfg.host_slab_bytes, c["host_layout"])
        dev.poison(gi.TAG_NEVER)
        host.poison(gi.TAG_NEVER)
        dimg, himg = dev.poison_img(gi.TAG_NEVER), host.poison_img(gi.TAG_NEVER)
        kd = cfg.dev_slab_bytes // sh.block_bytes()
        kh = cfg.host_slab_bytes // sh.block_bytes()
        cap_d, cap_h = c["dev_slabs"] * kd, c["host_slabs"] * kh
        # age the device pool: a few seeded allocations, some freed again
        live = []
        for _ in range(int(r.integers(0, 6))):
            m = int(r.integers(1, max(2, cap_d // 8)))
            if sum(len(o) for _, o in live) + m > cap_d // 4:
                break
            live.append(dev.alloc(sh, m))
        for i in sorted(r.permutation(len(live))[: len(live) // 2], reverse=True):
            dev.free(*live.pop(int(i)))
        used = sum(len(o) for _, o in live)
        n = int(r.integers(1, max(2, min(cap_h, (cap_d - used) // 3) + 1)))
        dc, do = dev.alloc(sh, n)
        fill_blocks(dev, dimg, sh, do, [(0, j) for j in range(n)], m=2)
        assert first_diff(dev.read(), dimg) is None
        # swap-out (FREE_SRC: the sources sit in the move list until it completes)
        hc, ho = host.alloc(sh, n)
        x = ctx.kv_swap_out(sh.as_tuple(), dc, hc, flags=aeg.FREE_SRC)
        xo = dev.oracle.begin(do)
        dev.oracle.free(do)
        himg = OK.swap_out(dimg, dev.geom, himg, host.geom, sh, do, ho)
        ctx.layer_ready(x, -1, aeg.READY_BLOCK)
        assert first_diff(host.read(), himg) is None, c
        assert first_diff(dev.read(), dimg) is None, c
        dev.oracle.complete(xo)
        # swap-in into fresh blocks
        nc, no = dev.alloc(sh, n)
        poison_blocks(dev, dimg, sh, no)
        y = ctx.kv_swap_in(sh.as_tuple(), hc, nc)
        dimg = OK.swap_in(himg, host.geom, dimg, dev.geom, sh, ho, no)
        ctx.layer_ready(y, -1, aeg.READY_BLOCK)
        assert first_diff(dev.read(), dimg) is None, c
        # local hand-off of the swapped-in blocks into fresh blocks of the same pool
        mc, mo = dev.alloc(sh, n)
        poison_blocks(dev, dimg, sh, mo)
        z = ctx.kv_migrate(sh.as_tuple(), nc, -1, mc, flags=aeg.MIGRATE_CE if c["ce"] else 0)
        dimg = OK.migrate(dimg, dev.geom, dimg, dev.geom, sh, no, mo)
        ctx.layer_ready(z, -1, aeg.READY_BLOCK)
        assert first_diff(dev.read(), dimg) is None, c
        assert first_diff(host.read(), himg) is None, c
        for t in (x, y, z):
            ctx.xfer_release(t)
    finally:
        ctx.shutdown()


@pytest.mark.parametrize("seed", range(32))
def test_fuzz_hand_off_between_contexts_of_different_geometry(seed):
    """Prefill context -> decode context of this process (peer mapped directly), each pool with its
    own random slab size, ragged tail and layout; fused kernel or copy-engine route; the whole
    destination pool vs O7 and the source pool unchanged."""
    require_gpu()
    c = draw(1000 + seed)
    sh, r = c["sh"], c["rng"]

    def mk(slab, slabs, layout):
        cfg = aeg.default_config(device_kv_bytes=slabs * slab, host_kv_bytes=MIB, dev_slab_bytes=slab,
                                 host_slab_bytes=MIB, dev_slab_layout=layout, staging_slot_bytes=MIB,
                                 staging_slots=2, stage_ring_bytes=4 * MIB, stage_chunk_bytes=MIB,
                                 device_weight_bytes=2 * MIB, table_arena_bytes=4 * MIB, host_threads=1,
                                 kernel=c["kernel"])
        ctx = aeg.Context(0, cfg)
        return ctx, Side(ctx, aeg.POOL_DEVICE, cfg.device_kv_bytes, slab, layout)
    a, src = mk(c["dev_slab"], c["dev_slabs"], c["dev_layout"])
    b, dst = mk(c["host_slab"], c["host_slabs"], c["host_layout"])    # the second geometry of the case
    try:
        for s in (src, dst):
            s.poison(gi.TAG_NEVER)
        simg, dimg = src.poison_img(gi.TAG_NEVER), dst.poison_img(gi.TAG_NEVER)
        cap_s = c["dev_slabs"] * (c["dev_slab"] // sh.block_bytes())
        cap_d = c["host_slabs"] * (c["host_slab"] // sh.block_bytes())
        if cap_d > 2:   # some resident blocks first, so the destination blocks are not the first ones
            dst.alloc(sh, int(r.integers(1, cap_d // 2)))
        n = int(r.integers(1, max(2, min(cap_s, cap_d - dst.oracle.owner_count()) + 1)))
        sc, so = src.alloc(sh, n)
        fill_blocks(src, simg, sh, so, [(1, j) for j in range(n)], m=3)
        dc, do = dst.alloc(sh, n)
        poison_blocks(dst, dimg, sh, do)
        a.import_peer(1, b.export_ipc())
        x = a.kv_migrate(sh.as_tuple(), sc, 1, dc, flags=aeg.MIGRATE_CE if c["ce"] else 0)
        exp = OK.migrate(simg, src.geom, dimg, dst.geom, sh, so, do)
        a.layer_ready(x, -1, aeg.READY_BLOCK)
        assert first_diff(dst.read(), exp) is None, c
        assert first_diff(src.read(), simg) is None, c
        a.xfer_release(x)
    finally:
        a.shutdown()
        b.shutdown()


@pytest.mark.parametrize("seed", range(24))
def test_fuzz_weight_staging_matches_the_oracle(seed):
    """Random tensor lists (REPLICATED / COL with 1 or 3 groups / ROW / VOCAB splits, odd sizes),
    TP size and rank, Stage Buffer chunk / ring / thread counts, staged or registered-direct path,
    two jobs back to back (the second bumps on from the first), over a region holding garbage: every
    shard vs oracle O8 and every padding byte zero (reading 17)."""
    require_gpu()
    from aeg_inputs import dev as D
    from oracle import weights as W
    r = np.random.default_rng(0x3E16 + seed)
    tp = int(r.choice([1, 2, 3, 4, 8]))
    rank = int(r.integers(0, tp))

    def tensors(m):
        descs = []
        for k in range(int(r.integers(1, 10))):
            split = int(r.choice([W.REPLICATED, W.COL, W.ROW, W.VOCAB]))
            groups = int(r.choice([1, 3])) if split == W.COL else 1
            rows = int(r.integers(1, 64)) * (groups * tp if split in (W.COL, W.VOCAB) else 1)
            cols = int(r.integers(1, 300)) * (tp if split == W.ROW else 1)
            descs.append(dict(rows=rows, cols=cols, split=split, groups=groups, layer=int(r.integers(0, 4))))
        sizes = [d["rows"] * d["cols"] * 2 for d in descs]
        buf = np.empty(sum(-(-n // 256) * 256 for n in sizes) + 256, np.uint8)
        tens, o = [], 0
        for k, (d, n) in enumerate(zip(descs, sizes)):
            v = buf[o:o + n]
            v[:] = gi.region_bytes(gi.w_seed(9), gi.weight_key(m, k), n)
            tens.append(v.reshape(d["rows"], d["cols"] * 2))
            o += -(-n // 256) * 256
        return descs, buf, tens
    direct = bool(r.integers(0, 2))
    chunk = int(r.choice([1, 2, 4])) << 20
    cfg = aeg.default_config(device_kv_bytes=4 * MIB, host_kv_bytes=4 * MIB, dev_slab_bytes=MIB,
                             host_slab_bytes=MIB, stage_ring_bytes=chunk * int(r.integers(2, 5)),
                             stage_chunk_bytes=chunk, staging_slot_bytes=MIB, staging_slots=2,
                             device_weight_bytes=48 * MIB, table_arena_bytes=2 * MIB,
                             host_threads=int(r.integers(1, 5)))
    ctx = aeg.Context(0, cfg)
    try:
        base, wbytes, _ = ctx.weights_region()
        D.fill_region(base, wbytes, gi.w_seed(9), gi.poison_key(gi.TAG_NEVER, 0))   # garbage in the region
        exp, end, shards = None, 0, []
        for m in (1, 2):
            descs, buf, tens = tensors(m)
            if direct:
                ctx.host_register(buf.ctypes.data, buf.nbytes)
            dl = [dict(host_src=t.ctypes.data, rows=d["rows"], cols=d["cols"], elem_bytes=2, layer=d["layer"],
                       split=d["split"], groups=d["groups"]) for t, d in zip(tens, descs)]
            offs, x = ctx.weights_stage(dl, tp_rank=rank, tp_size=tp)
            ctx.layer_ready(x, -1, aeg.READY_BLOCK)
            exp, eoffs, end = W.stage(tens, descs, rank, tp, region_bytes=wbytes, base=end, dst=exp)
            assert [int(o) for o in offs] == eoffs
            shards += [(o, W.shard(t.reshape(d["rows"], d["cols"], 2), d["split"], d["groups"], rank, tp).size)
                       for o, t, d in zip(eoffs, tens, descs)]
            got = D.read(base, end)
            for o, n in shards:   # every shard of both jobs
                assert first_diff(got[o:o + n], exp[o:o + n]) is None, (seed, m, tp, rank, direct, o)
            # reading 17: the 256-byte padding after every shard (up to the bump pointer) is zeros
            for (o, n), nxt in zip(shards, [o2 for o2, _ in shards[1:]] + [end]):
                assert not got[o + n:nxt].any(), (seed, m, tp, rank, direct, o + n, nxt)
            ctx.xfer_release(x)
            if direct:
                ctx.host_unregister(buf.ctypes.data)
    finally:
        ctx.shutdown()
