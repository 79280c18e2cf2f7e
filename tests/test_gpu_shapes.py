"""Every KV shape of the paper's workloads (Table 1, and the configs' models)
through a swap round trip with the default (AUTO) kernel choice, whose chunk sizes span 32 KiB
(Yi-9B: LSU), 64-320 KiB (BULK) and 512 KiB (Qwen-72B full width): source and destination pools of
different slab sizes and layouts, a ragged block count that crosses slab boundaries, destinations
interleaved with live blocks; both whole pool images compared with the oracle (O5/O6)."""
import pytest

import aeg_inputs as gi
import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg
from oracle import kv as OK
from oracle.shape import KVShape

from .gpu_harness import Side, fill_blocks, first_diff, poison_blocks, require_gpu

pytestmark = pytest.mark.gpu
SHAPES = [k for k in gi.KV_SHAPES if k != "tiny"]


@pytest.mark.parametrize("name", SHAPES)
def test_paper_shape_round_trip_auto_kernel(name):
    require_gpu()
    sh = KVShape(*gi.KV_SHAPES[name])
    bb = sh.block_bytes()
    dslab, hslab = 3 * bb, 5 * bb
    cfg = aeg.default_config(device_kv_bytes=4 * dslab, host_kv_bytes=2 * hslab, dev_slab_bytes=dslab,
                             host_slab_bytes=hslab, dev_slab_layout=aeg.LAYER_MAJOR,
                             host_slab_layout=aeg.BLOCK_MAJOR, staging_slot_bytes=64 << 20, staging_slots=2,
                             host_threads=1)
    ctx = aeg.Context(0, cfg)
    try:
        dev = Side(ctx, 0, 4 * dslab, dslab, aeg.LAYER_MAJOR)
        host = Side(ctx, 1, 2 * hslab, hslab, aeg.BLOCK_MAJOR)
        dev.poison(gi.TAG_NEVER)
        host.poison(gi.TAG_NEVER)
        dimg, himg = dev.poison_img(gi.TAG_NEVER), host.poison_img(gi.TAG_NEVER)
        keep_c, keep_o = dev.alloc(sh, 2)                     # a live request
        fill_blocks(dev, dimg, sh, keep_o, [(9, j) for j in range(2)], m=2)
        dc, do = dev.alloc(sh, 7)                             # the batch: crosses two slab boundaries
        fill_blocks(dev, dimg, sh, do, [(0, j) for j in range(7)])
        hc, ho = host.alloc(sh, 7)
        x = ctx.kv_swap_out(sh.as_tuple(), dc, hc, flags=aeg.FREE_SRC)
        ctx.layer_ready(x, -1, aeg.READY_BLOCK)
        ctx.xfer_release(x)
        himg = OK.swap_out(dimg, dev.geom, himg, host.geom, sh, do, ho)
        assert first_diff(host.read(), himg) is None
        ctx.reclaim(True)
        xo = dev.oracle.begin(do)
        dev.oracle.free(do)
        dev.oracle.complete(xo)
        nc, no = dev.alloc(sh, 7)                             # reuses the freed blocks around the live ones
        poison_blocks(dev, dimg, sh, no)
        y = ctx.kv_swap_in(sh.as_tuple(), hc, nc)
        for l in range(sh.L):
            ctx.layer_ready(y, l, aeg.READY_BLOCK)
        dimg = OK.swap_in(himg, host.geom, dimg, dev.geom, sh, ho, no)
        assert first_diff(dev.read(), dimg) is None
        assert first_diff(host.read(), himg) is None
    finally:
        ctx.shutdown()
