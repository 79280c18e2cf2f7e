"""GPU edge cases of the ABI: empty transfers, a one-layer shape, ragged single blocks, a block larger
than a staging slot, shapes whose chunk is not 16-byte aligned, OOM without state change, readiness
of released / unknown transfers — each against the oracle or the documented error code."""
import numpy as np
import pytest

import aeg_inputs as gi
import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg
from oracle import kv as OK
from oracle.shape import KVShape

from .gpu_harness import Side, fill_blocks, first_diff, require_gpu

pytestmark = pytest.mark.gpu
MIB = 1 << 20


def make(slot=MIB, dev_slabs=4, host_slabs=4, slab=MIB, kernel=aeg.KERNEL_AUTO):
    cfg = aeg.default_config(device_kv_bytes=dev_slabs * slab, host_kv_bytes=host_slabs * slab, dev_slab_bytes=slab,
                             host_slab_bytes=slab, staging_slot_bytes=slot, staging_slots=2,
                             stage_ring_bytes=4 * MIB, stage_chunk_bytes=MIB, table_arena_bytes=2 * MIB,
                             host_threads=1, kernel=kernel)
    ctx = aeg.Context(0, cfg)
    return ctx, Side(ctx, 0, dev_slabs * slab, slab, 0), Side(ctx, 1, host_slabs * slab, slab, 0)


def test_empty_transfers_are_ready():
    require_gpu()
    ctx, _, _ = make()
    try:
        sh = (2, 1, 64, 2, 16)
        for x in (ctx.kv_swap_out(sh, [], []), ctx.kv_swap_in(sh, [], []), ctx.kv_migrate(sh, [], -1, []),
                  ctx.kv_migrate(sh, [], -1, [], flags=aeg.MIGRATE_CE)):
            ctx.layer_ready(x, -1, aeg.READY_BLOCK)
            assert all(ctx.layer_ready(x, l, aeg.READY_QUERY) for l in range(2))
            ctx.xfer_release(x)
    finally:
        ctx.shutdown()


@pytest.mark.parametrize("kernel", [aeg.KERNEL_AUTO, aeg.KERNEL_BULKW, aeg.KERNEL_BULK, aeg.KERNEL_LSU])
@pytest.mark.parametrize("shape", [(1, 1, 8, 2, 1), (3, 1, 8, 2, 1), (1, 2, 64, 2, 16)])
def test_small_shapes_round_trip(shape, kernel):
    """One-layer shapes and 1-token blocks (chunk = 32 B): ragged, launch-bound, still bit-exact."""
    require_gpu()
    sh = KVShape(*shape)
    ctx, dev, host = make(kernel=kernel)
    try:
        dev.poison(gi.TAG_NEVER)
        host.poison(gi.TAG_NEVER)
        dimg, himg = dev.poison_img(gi.TAG_NEVER), host.poison_img(gi.TAG_NEVER)
        dc, do = dev.alloc(sh, 37)
        fill_blocks(dev, dimg, sh, do, [(0, j) for j in range(37)])
        hc, ho = host.alloc(sh, 37)
        x = ctx.kv_swap_out(sh.as_tuple(), dc, hc)
        ctx.layer_ready(x, -1, aeg.READY_BLOCK)
        himg = OK.swap_out(dimg, dev.geom, himg, host.geom, sh, do, ho)
        assert first_diff(host.read(), himg) is None
        nc, no = dev.alloc(sh, 37)
        y = ctx.kv_swap_in(sh.as_tuple(), hc, nc)
        ctx.layer_ready(y, -1, aeg.READY_BLOCK)
        dimg = OK.swap_in(himg, host.geom, dimg, dev.geom, sh, ho, no)
        assert first_diff(dev.read(), dimg) is None
    finally:
        ctx.shutdown()


def test_copy_engine_route_rejects_a_chunk_larger_than_a_slot():
    """AEG_MIGRATE_CE stages through the out ring: a chunk above staging_slot_bytes is INVALID and
    changes nothing (the fused kernel route has no such limit)."""
    require_gpu()
    ctx, dev, _ = make(slab=4 * MIB, dev_slabs=4)
    try:
        big = KVShape(1, 32, 128, 2, 128)        # chunk = 2 MiB > the 1 MiB slot
        sc, so = dev.alloc(big, 1)
        dc, do = dev.alloc(big, 1)
        with pytest.raises(aeg.AegError) as e:
            ctx.kv_migrate(big.as_tuple(), sc, -1, dc, flags=aeg.MIGRATE_CE)
        assert e.value.code == aeg.ERR_INVALID
        x = ctx.kv_migrate(big.as_tuple(), sc, -1, dc)   # the kernel route copies it
        ctx.layer_ready(x, -1, aeg.READY_BLOCK)
        ctx.xfer_release(x)
    finally:
        ctx.shutdown()


def test_invalid_shapes_and_sizes():
    require_gpu()
    ctx, dev, host = make(slot=MIB)
    try:
        with pytest.raises(aeg.AegError) as e:
            ctx.kv_alloc(0, (2, 1, 3, 2, 1), 1)          # chunk 12 B: not a multiple of 16
        assert e.value.code == aeg.ERR_INVALID
        big = (1, 9, 128, 2, 256)                         # chunk = 256*2*9*128*2 B = 1.125 MiB
        with pytest.raises(aeg.AegError) as e:
            ctx.kv_alloc(0, big, 1)                       # block larger than a 1 MiB slab
        assert e.value.code == aeg.ERR_INVALID
    finally:
        ctx.shutdown()
    ctx, dev, host = make(slot=MIB, slab=4 * MIB)
    try:
        big = (1, 9, 128, 2, 256)                         # 1.125 MiB chunk > 1 MiB staging slot
        d = ctx.kv_alloc(0, big, 1)
        h = ctx.kv_alloc(1, big, 1)
        with pytest.raises(aeg.AegError) as e:
            ctx.kv_swap_out(big, d, h)
        assert e.value.code == aeg.ERR_INVALID
        # the migrate kernel has no staging: it accepts the big chunk
        d2 = ctx.kv_alloc(0, big, 1)
        x = ctx.kv_migrate(big, d, -1, d2)
        ctx.layer_ready(x, -1, aeg.READY_BLOCK)
    finally:
        ctx.shutdown()


def test_oom_changes_nothing_and_release_semantics():
    require_gpu()
    ctx, dev, host = make()
    try:
        sh = (2, 2, 64, 2, 16)
        a = ctx.kv_alloc(0, sh, 10)
        before = ctx.stats(0)
        with pytest.raises(aeg.AegError) as e:
            ctx.kv_alloc(0, sh, 1000)
        assert e.value.code == aeg.ERR_OOM
        after = ctx.stats(0)
        assert (after.owned_blocks, after.free_slabs) == (before.owned_blocks, before.free_slabs)
        h = ctx.kv_alloc(1, sh, 10)
        x = ctx.kv_swap_out(sh, a, h)
        ctx.layer_ready(x, -1, aeg.READY_BLOCK)
        ctx.xfer_release(x)
        with pytest.raises(aeg.AegError) as e:
            ctx.layer_ready(x, 0, aeg.READY_QUERY)       # released
        assert e.value.code == aeg.ERR_STATE
        with pytest.raises(aeg.AegError) as e:
            ctx.layer_ready(987654, 0, aeg.READY_QUERY)  # unknown
        assert e.value.code == aeg.ERR_STATE
        y = ctx.kv_swap_in(sh, h, a)
        with pytest.raises(aeg.AegError) as e:
            ctx.layer_ready(y, 2, aeg.READY_QUERY)       # layer out of range
        assert e.value.code == aeg.ERR_INVALID
        ctx.layer_ready(y, -1, aeg.READY_BLOCK)
    finally:
        ctx.shutdown()


def test_swap_sources_must_be_owned_and_distinct():
    require_gpu()
    ctx, dev, host = make()
    try:
        sh = (2, 2, 64, 2, 16)
        a = ctx.kv_alloc(0, sh, 4)
        h = ctx.kv_alloc(1, sh, 4)
        with pytest.raises(aeg.AegError) as e:
            ctx.kv_swap_out(sh, np.array([a[0], a[0], a[1], a[2]], np.uint64), h)
        assert e.value.code == aeg.ERR_STATE
        with pytest.raises(aeg.AegError) as e:
            ctx.kv_swap_out(sh, h, a)                    # pools swapped
        assert e.value.code == aeg.ERR_INVALID
        ctx.kv_free(0, a)
        with pytest.raises(aeg.AegError) as e:
            ctx.kv_swap_out(sh, a, h)                    # freed sources
        assert e.value.code in (aeg.ERR_STATE, aeg.ERR_INVALID)
    finally:
        ctx.shutdown()


def test_default_device_kv_takes_90pct_of_free_vram():
    """Reading 22: device_kv_bytes = 0 sizes the one device allocation to ~90% of
    free VRAM ("leaving around 10% free memory for tensor libraries"), the KV region in whole slabs."""
    require_gpu()
    import torch
    free0, _ = torch.cuda.mem_get_info()
    cfg = aeg.default_config(device_kv_bytes=0, host_kv_bytes=4 * MIB, dev_slab_bytes=64 * MIB,
                             host_slab_bytes=MIB, staging_slot_bytes=MIB, staging_slots=2,
                             stage_ring_bytes=4 * MIB, stage_chunk_bytes=MIB, device_weight_bytes=256 * MIB,
                             table_arena_bytes=2 * MIB, host_threads=1)
    ctx = aeg.Context(0, cfg)
    try:
        _, kv = ctx.pool_region(aeg.POOL_DEVICE)
        others = 256 * MIB + 2 * 2 * MIB + 2 * MIB
        assert kv % (64 * MIB) == 0 and kv > 0
        assert 0.9 * free0 - others - 64 * MIB - 256 * MIB <= kv <= 0.9 * free0 - others
        free1, _ = torch.cuda.mem_get_info()
        assert free1 >= 0.09 * free0            # ~10% left to the caller
        b = ctx.kv_alloc(aeg.POOL_DEVICE, (2, 4, 64, 2, 16), 8)
        ctx.kv_free(aeg.POOL_DEVICE, b)
    finally:
        ctx.shutdown()


def test_readme_example_round_trip():
    """The README's minimal use of the binding (default 90 %-of-free-VRAM device pool, Qwen-7B shape,
    128 blocks out and back with per-layer stream waits) moves every chunk back intact."""
    require_gpu()
    import torch
    from aeg_inputs import dev as Dv
    ctx = aeg.Context(0, aeg.default_config(host_kv_bytes=2 << 30))
    try:
        qwen7b = (32, 32, 128, 2, 16)
        sh = KVShape(*qwen7b)
        dev = ctx.kv_alloc(aeg.POOL_DEVICE, qwen7b, 128)
        host = ctx.kv_alloc(aeg.POOL_HOST, qwen7b, 128)
        base, _ = ctx.pool_region(aeg.POOL_DEVICE)

        def offs(blocks):
            o0, ls = ctx.block_offsets(aeg.POOL_DEVICE, qwen7b, blocks)
            return [int(o) + l * int(ls) for o in o0 for l in range(sh.L)]
        keys = [gi.kv_key(9, 0, i, l) for i in range(128) for l in range(sh.L)]
        seed = gi.kv_seed(1)
        Dv.fill_chunks(base, offs(dev), keys, sh.chunk_bytes(), seed)
        x = ctx.kv_swap_out(qwen7b, dev, host, flags=aeg.FREE_SRC)
        back = ctx.kv_alloc(aeg.POOL_DEVICE, qwen7b, 128)
        y = ctx.kv_swap_in(qwen7b, host, back, flags=aeg.FREE_SRC)
        decode_stream = torch.cuda.Stream()
        for l in range(32):
            ctx.layer_ready(y, l, aeg.READY_WAIT_STREAM, decode_stream.cuda_stream)
        decode_stream.synchronize()
        bad, first = Dv.verify_chunks(base, offs(back), keys, sh.chunk_bytes(), seed)
        assert bad == 0, first
        ctx.xfer_release(x)
        ctx.xfer_release(y)
    finally:
        ctx.shutdown()
