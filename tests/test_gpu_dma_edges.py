"""GPU edge cases of the host DMA planning (H3/H4) and of the cross-transfer dependency `after`.

1. Host runs whose 2-D merge would need a pitch above cudaDevAttrMaxPitch (2^31 - 1): runs of equal
   length at the same offset of 1 GiB slabs 0 and 2 are 2 GiB apart.  They must be copied as
   separate 1-D copies, and the swap round trip must still be the oracle's (O5/O6, checked at the
   oracle's addresses with the content-addressed generator).
2. `after` (aeg.h: "Layer l's H2D waits on layer l of transfer `after`") must hold even for host
   blocks `after` did not write itself: a swap-in with AEG_NO_DEPS that reads blocks written by an
   EARLIER swap-out X1 and names the later swap-out X2 (same D2H stream) as `after` reads landed
   data (rule ❷ across instances)."""
import numpy as np
import pytest

import aeg_inputs as gi
import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg
from aeg_inputs import dev as D
from oracle import kv as OK
from oracle.rules import check
from oracle.shape import KVShape

from .gpu_harness import SEED, Side, fill_blocks, first_diff, require_gpu
from .test_gpu_swap import parse_trace

pytestmark = pytest.mark.gpu
MIB, GIB = 1 << 20, 1 << 30


def _offs(side, sh, handles_o):
    return [OK.addr(side.geom, sh, h, l) for h in handles_o for l in range(sh.L)]


@pytest.mark.parametrize("kernel", [aeg.KERNEL_LSU, aeg.KERNEL_BULK, aeg.KERNEL_BULKW])
def test_host_runs_two_gib_apart_round_trip(kernel):
    require_gpu()
    sh = KVShape(2, 8, 128, 2, 16)          # chunk 64 KiB, block 128 KiB: 8192 blocks per 1 GiB slab
    cfg = aeg.default_config(device_kv_bytes=2 * GIB, host_kv_bytes=3 * GIB, dev_slab_bytes=GIB,
                             host_slab_bytes=GIB, dev_slab_layout=aeg.LAYER_MAJOR,
                             host_slab_layout=aeg.LAYER_MAJOR, staging_slot_bytes=64 * MIB, staging_slots=2,
                             stage_ring_bytes=4 * MIB, stage_chunk_bytes=MIB, device_weight_bytes=8 * MIB,
                             table_arena_bytes=4 * MIB, host_threads=2, kernel=kernel)
    ctx = aeg.Context(0, cfg)
    try:
        dev = Side(ctx, aeg.POOL_DEVICE, cfg.device_kv_bytes, cfg.dev_slab_bytes, aeg.LAYER_MAJOR)
        host = Side(ctx, aeg.POOL_HOST, cfg.host_kv_bytes, cfg.host_slab_bytes, aeg.LAYER_MAJOR)
        k = GIB // sh.block_bytes()
        # host: take slabs 0..2 whole, keep blocks 0..m-1 of slabs 0 and 2 (runs 2 GiB apart)
        m = 24
        hc, ho = host.alloc(sh, 3 * k)
        keep = [i for i in range(3 * k) if (i // k) in (0, 2) and i % k < m]
        drop = [i for i in range(3 * k) if i not in set(keep)]
        host.free(hc[drop], [ho[i] for i in drop])
        hc, ho = hc[keep], [ho[i] for i in keep]
        assert ho[m][0] - ho[0][0] == 2 and ho[m][1] == ho[0][1]
        n = len(ho)
        dc, do = dev.alloc(sh, n)
        fill_blocks(dev, _Sink(), sh, do, [(0, j) for j in range(n)])
        x = ctx.kv_swap_out(sh.as_tuple(), dc, hc)
        ctx.layer_ready(x, -1, aeg.READY_BLOCK)
        keys = [gi.kv_key(1, 0, j, l) for j in range(n) for l in range(sh.L)]
        bad, first = D.verify_chunks(host.base, _offs(host, sh, ho), keys, sh.chunk_bytes(), SEED)
        assert bad == 0, ("swap-out", first)
        nc, no = dev.alloc(sh, n)
        y = ctx.kv_swap_in(sh.as_tuple(), hc, nc)
        ctx.layer_ready(y, -1, aeg.READY_BLOCK)
        bad, first = D.verify_chunks(dev.base, _offs(dev, sh, no), keys, sh.chunk_bytes(), SEED)
        assert bad == 0, ("swap-in", first)
    finally:
        ctx.shutdown()


class _Sink:
    """Byte-image stand-in for fill_blocks when the test checks content-addressed chunks instead
    of a whole-pool image (a 3 GiB NumPy image per pool is not needed)."""

    def __setitem__(self, k, v):
        pass


def test_after_covers_blocks_it_did_not_write():
    require_gpu()
    import torch
    SHP = KVShape(4, 2, 64, 2, 16)          # chunk 8 KiB
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
        for mm in (1, 2):
            c, o = dev.alloc(SHP, 256)
            fill_blocks(dev, dimg, SHP, o, [(0, j) for j in range(256)], m=mm)
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
        # X2 really ran its D2H in pieces (its transfer blob carries the piece table and events)
        assert len(ctx.xfer_export(xs[1])) > 40 + (SHP.L + 1) * 64
        # read 64 of X1's host blocks only, ordered through `after` = X2 (X2 wrote none of them)
        rng = np.random.default_rng(5)
        pick = sorted(rng.choice(256, size=64, replace=False).tolist())
        hsel_c = np.array([hosts[0][0][i] for i in pick], dtype=np.uint64)
        hsel_o = [hosts[0][1][i] for i in pick]
        nc, no = dev.alloc(SHP, len(pick))
        y = ctx.kv_swap_in_from(SHP.as_tuple(), -1, hsel_c, nc, after=xs[1], flags=aeg.NO_DEPS)
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
        assert check(parse_trace(ctx.trace_read()))
    finally:
        ctx.shutdown()
