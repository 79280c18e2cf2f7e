"""GPU parity for H5 (prefill->decode KV hand-off): the fused migrate kernel's destination image
equals oracle.kv.migrate (O7) — within one pool (peer -1), between two contexts of this process
with different slab sizes/layouts (peer mapped directly), and between two processes through CUDA
IPC memory and IPC events (the multi-process path of §8(e), exercised on one GPU)."""
import multiprocessing as mp
import os

import numpy as np
import pytest

import aeg_inputs as gi
import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg
from oracle import kv as OK
from oracle.shape import KVShape

from .gpu_harness import Side, fill_blocks, first_diff, poison_blocks, require_gpu

pytestmark = pytest.mark.gpu
SH = KVShape(3, 2, 64, 2, 16)   # Cl = 8 KiB
MIB = 1 << 20


def make(layout, slab=MIB, nslabs=8, kernel=aeg.KERNEL_LSU):
    cfg = aeg.default_config(device_kv_bytes=nslabs * slab, host_kv_bytes=MIB, dev_slab_bytes=slab,
                             host_slab_bytes=MIB, dev_slab_layout=layout, staging_slot_bytes=MIB,
                             staging_slots=2, stage_ring_bytes=4 * MIB, stage_chunk_bytes=MIB,
                             table_arena_bytes=2 * MIB, host_threads=1, kernel=kernel)
    ctx = aeg.Context(0, cfg)
    return ctx, Side(ctx, aeg.POOL_DEVICE, cfg.device_kv_bytes, slab, layout)


@pytest.mark.parametrize("ce", [False, True], ids=["kernel", "ce"])
@pytest.mark.parametrize("kernel", [aeg.KERNEL_LSU, aeg.KERNEL_BULK, aeg.KERNEL_BULKW])
def test_local_migrate(kernel, ce):
    """Local relocation (peer -1) through the fused kernel or the copy-engine route (AEG_MIGRATE_CE:
    gather kernel `kernel` into staging, then copy-engine commands into the destination blocks)."""
    require_gpu()
    ctx, dev = make(aeg.BLOCK_MAJOR, kernel=kernel)
    try:
        dev.poison(gi.TAG_NEVER)
        img = dev.poison_img(gi.TAG_NEVER)
        sc, so = dev.alloc(SH, 37)
        fill_blocks(dev, img, SH, so, [(0, j) for j in range(37)])
        dc, do = dev.alloc(SH, 37)
        poison_blocks(dev, img, SH, do)
        x = ctx.kv_migrate(SH.as_tuple(), sc, -1, dc, flags=aeg.MIGRATE_CE if ce else 0)
        exp = OK.migrate(img, dev.geom, img, dev.geom, SH, so, do)
        ctx.layer_ready(x, -1, aeg.READY_BLOCK)
        assert first_diff(dev.read(), exp) is None
    finally:
        ctx.shutdown()


@pytest.mark.parametrize("ctas", [1, 3])
def test_local_migrate_under_an_sm_budget(ctas):
    """aeg_set_migrate_ctas: a grid of 1 or 3 CTAs strides over every (block, layer) piece."""
    require_gpu()
    ctx, dev = make(aeg.LAYER_MAJOR, kernel=aeg.KERNEL_AUTO)
    try:
        with pytest.raises(aeg.AegError):
            ctx.set_migrate_ctas(-1)
        ctx.set_migrate_ctas(ctas)
        dev.poison(gi.TAG_NEVER)
        img = dev.poison_img(gi.TAG_NEVER)
        sc, so = dev.alloc(SH, 29)
        fill_blocks(dev, img, SH, so, [(0, j) for j in range(29)])
        dc, do = dev.alloc(SH, 29)
        poison_blocks(dev, img, SH, do)
        x = ctx.kv_migrate(SH.as_tuple(), sc, -1, dc)
        exp = OK.migrate(img, dev.geom, img, dev.geom, SH, so, do)
        ctx.layer_ready(x, -1, aeg.READY_BLOCK)
        assert first_diff(dev.read(), exp) is None
    finally:
        ctx.shutdown()


@pytest.mark.parametrize("ce", [False, True], ids=["kernel", "ce"])
def test_same_process_peer_migrate_and_imported_events(ce):
    require_gpu()
    a, A = make(aeg.LAYER_MAJOR, slab=MIB)
    b, B = make(aeg.BLOCK_MAJOR, slab=MIB + 64 * 1024, nslabs=6)
    try:
        A.poison(gi.TAG_NEVER)
        B.poison(gi.TAG_NEVER)
        aimg, bimg = A.poison_img(gi.TAG_NEVER), B.poison_img(gi.TAG_NEVER)
        sc, so = A.alloc(SH, 50)
        fill_blocks(A, aimg, SH, so, [(3, j) for j in range(50)])
        dc, do = B.alloc(SH, 50)
        poison_blocks(B, bimg, SH, do)
        a.import_peer(5, b.export_ipc())
        b.import_peer(0, a.export_ipc())
        x = a.kv_migrate(SH.as_tuple(), sc, 5, dc, flags=aeg.MIGRATE_CE if ce else 0)
        xi = b.xfer_import(0, a.xfer_export(x))
        for l in range(SH.L):
            b.layer_ready(xi, l, aeg.READY_BLOCK)
        exp = OK.migrate(aimg, A.geom, bimg, B.geom, SH, so, do)
        assert first_diff(B.read(), exp) is None
        assert first_diff(A.read(), aimg) is None
    finally:
        a.shutdown()
        b.shutdown()


def test_same_process_import_pins_the_exporters_events():
    """a same-process import borrows the exporter's raw events.  After the exporter
    releases and reaps its transfer, a new gate-held transfer of the exporter must NOT re-record
    those events (they stay pinned until the import is reaped): the importer still sees every
    layer complete."""
    require_gpu()
    import torch
    from aeg_inputs import dev as D
    a, A = make(aeg.LAYER_MAJOR)
    b, B = make(aeg.BLOCK_MAJOR)
    try:
        sc, so = A.alloc(SH, 20)
        dc, do = A.alloc(SH, 20)
        x = a.kv_migrate(SH.as_tuple(), sc, -1, dc)
        a.layer_ready(x, -1, aeg.READY_BLOCK)
        xi = b.xfer_import(0, a.xfer_export(x))
        a.xfer_release(x)
        with pytest.raises(aeg.AegError):
            a.xfer_export(x)                    # released: no more exports
        a.reclaim(True)                         # the exporter reaps what it may
        s = torch.cuda.Stream()
        gate = D.Gate()
        gate.close_on(s.cuda_stream)
        a.stream_fence(s.cuda_stream)
        ys = [a.kv_migrate(SH.as_tuple(), dc, -1, sc) for _ in range(2)]   # would take recycled events
        assert not a.layer_ready(ys[0], 0, aeg.READY_QUERY)
        for l in range(SH.L):
            assert b.layer_ready(xi, l, aeg.READY_QUERY), f"imported layer {l} re-armed by the exporter"
        assert b.layer_ready(xi, -1, aeg.READY_QUERY)
        gate.open()
        for y in ys:
            a.layer_ready(y, -1, aeg.READY_BLOCK)
        b.xfer_release(xi)
        b.reclaim(True)                         # import reaped: the pin is dropped
        a.reclaim(True)
    finally:
        b.shutdown()
        a.shutdown()


def _decode_side(conn):
    """Child process: the decode instance.  Allocates destination blocks, exports its pool, waits on
    the imported per-layer events, then reports its image."""
    try:
        _decode_body(conn)
    except BaseException:
        import traceback
        conn.send(("error", traceback.format_exc()))
        raise


def _decode_body(conn):
    ctx, dev = make(aeg.BLOCK_MAJOR, slab=MIB, nslabs=4)
    dev.poison(gi.TAG_NEVER)
    dc, do = dev.alloc(SH, 20)
    img = dev.poison_img(gi.TAG_NEVER)
    poison_blocks(dev, img, SH, do)
    conn.send((ctx.export_ipc(), [int(b) for b in dc], do))
    blob = conn.recv()
    x = ctx.xfer_import(0, blob)
    for l in range(SH.L):
        ctx.layer_ready(x, l, aeg.READY_BLOCK)
    conn.send(dev.read().tobytes())
    conn.recv()
    ctx.shutdown()


@pytest.mark.parametrize("ce", [False, True], ids=["kernel", "ce"])
def test_two_process_ipc_migrate(ce):
    require_gpu()
    ctxm = mp.get_context("spawn")
    parent, child = ctxm.Pipe()
    p = ctxm.Process(target=_decode_side, args=(child,))
    p.start()
    child.close()

    def recv():
        assert parent.poll(120), "decode process did not answer"
        m = parent.recv()
        if isinstance(m, tuple) and len(m) == 2 and m[0] == "error":
            raise AssertionError("decode process failed:\n" + m[1])
        return m

    try:
        a, A = make(aeg.LAYER_MAJOR, slab=MIB, nslabs=4)
        A.poison(gi.TAG_NEVER)
        aimg = A.poison_img(gi.TAG_NEVER)
        sc, so = A.alloc(SH, 20)
        fill_blocks(A, aimg, SH, so, [(7, j) for j in range(20)])
        blob, dc, do = recv()
        a.import_peer(0, blob)
        x = a.kv_migrate(SH.as_tuple(), sc, 0, np.array(dc, dtype=np.uint64),
                         flags=aeg.FREE_SRC | (aeg.MIGRATE_CE if ce else 0))
        parent.send(a.xfer_export(x))
        got = np.frombuffer(recv(), dtype=np.uint8)
        geom = OK.PoolGeom(4 * MIB, MIB, aeg.BLOCK_MAJOR)
        bimg = gi.region_bytes(gi.kv_seed(1), gi.poison_key(gi.TAG_NEVER, 0), geom.nbytes)
        for h in do:
            for l in range(SH.L):
                o = OK.addr(geom, SH, h, l)
                bimg[o:o + SH.chunk_bytes()] = gi.region_bytes(gi.kv_seed(1), gi.poison_key(gi.TAG_DST, o), SH.chunk_bytes())
        exp = OK.migrate(aimg, A.geom, bimg, geom, SH, so, do)
        assert first_diff(got, exp) is None
        parent.send("bye")
        a.shutdown()
    finally:
        p.join(timeout=30)
        if p.is_alive():
            p.kill()
    assert p.exitcode == 0


# ------------------------------------------------------------------------------------ NEXT-2
def _decode_side_host_route(conn, nslabs=4):
    try:
        _decode_host_route_body(conn, nslabs)
    except BaseException:
        import traceback
        conn.send(("error", traceback.format_exc()))
        raise


def _decode_host_route_body(conn, nslabs=4):
    """Decode instance of Fig. 10: imports the prefill instance's shared CPU cache and its swap-out
    events, swaps R1 in from there (C->D) without any host synchronisation on the prefill side's
    progress, and exports its swap-in so the prefill side can release the CPU blocks."""
    import sys
    ctx, dev = make(aeg.LAYER_MAJOR, slab=MIB, nslabs=nslabs)
    dev.poison(gi.TAG_NEVER)
    # connect once at start-up (mapping a peer's pool / registering its shared host region may wait
    # for the GPU to drain, so it must not sit on the critical path of a hand-off)
    ctx.import_peer(0, conn.recv())
    conn.send("ready")
    hb, xblob = conn.recv()
    print("decode: got hand-off", file=sys.stderr, flush=True)
    xo = ctx.xfer_import(0, xblob)
    print("decode: imported events", file=sys.stderr, flush=True)
    dc, do = dev.alloc(SH, len(hb))
    print("decode: allocated", file=sys.stderr, flush=True)
    xi = ctx.kv_swap_in_from(SH.as_tuple(), 0, np.array(hb, dtype=np.uint64), dc, after=xo)   # ③④⑤
    print("decode: swap-in enqueued", file=sys.stderr, flush=True)
    blob = ctx.xfer_export(xi)
    print("decode: exported", file=sys.stderr, flush=True)
    conn.send((blob, do))
    for l in range(SH.L):
        ctx.layer_ready(xi, l, aeg.READY_BLOCK)                                                  # ⑥
    conn.send(dev.read().tobytes())
    conn.recv()
    ctx.shutdown()


@pytest.mark.parametrize("nblocks", [20, 600])
def test_two_process_host_route_p_c_d(nblocks):
    """NEXT-2: prefill P swaps R1 out to its part of the node-shared
    CPU KV cache (P->C) behind a 0.2 s delay kernel; decode D swaps it in (C->D) waiting only on P's
    per-layer IPC events (rule ❷); P frees the CPU blocks after importing D's swap-in, so they stay
    in P's move list until D is done (rule ❸).  D's device image = oracle swap_in∘swap_out.
    nblocks = 600: 4.7 MiB layers, so P's D2H runs in pieces whose IPC events travel in the
    transfer blob and D's H2D waits per piece."""
    require_gpu()
    import torch
    nslabs = 4 if nblocks <= 160 else 16
    ctxm = mp.get_context("spawn")
    parent, child = ctxm.Pipe()
    p = ctxm.Process(target=_decode_side_host_route, args=(child, nslabs))
    p.start()
    child.close()

    def recv():
        assert parent.poll(120), "decode process did not answer"
        m = parent.recv()
        if isinstance(m, tuple) and len(m) == 2 and m[0] == "error":
            raise AssertionError("decode process failed:\n" + m[1])
        return m

    try:
        cfg = aeg.default_config(device_kv_bytes=nslabs * MIB, host_kv_bytes=nslabs * MIB, dev_slab_bytes=MIB,
                                 host_slab_bytes=MIB, host_slab_layout=aeg.BLOCK_MAJOR, staging_slot_bytes=MIB,
                                 staging_slots=2, stage_ring_bytes=4 * MIB, stage_chunk_bytes=MIB,
                                 table_arena_bytes=2 * MIB, host_threads=1, flags=aeg.CFG_SHARED_HOST,
                                 dma_piece_mib=1, pack_layer_mib=1)
        a = aeg.Context(0, cfg)
        A = Side(a, aeg.POOL_DEVICE, nslabs * MIB, MIB, aeg.LAYER_MAJOR)
        H = Side(a, aeg.POOL_HOST, nslabs * MIB, MIB, aeg.BLOCK_MAJOR)
        A.poison(gi.TAG_NEVER)
        H.poison(gi.TAG_NEVER)
        aimg, himg = A.poison_img(gi.TAG_NEVER), H.poison_img(gi.TAG_NEVER)
        sc, so = A.alloc(SH, nblocks)
        fill_blocks(A, aimg, SH, so, [(1, j) for j in range(nblocks)])
        hc, ho = H.alloc(SH, nblocks)
        parent.send(a.export_ipc())                   # instances connect at start-up
        assert recv() == "ready"                      # the decode instance is up and connected
        s = torch.cuda.Stream()
        from aeg_inputs import dev as Dv
        gate = Dv.Gate()
        gate.close_on(s.cuda_stream)                  # the prefill is still running until gate.open()
        a.stream_fence(s.cuda_stream)
        xo = a.kv_swap_out(SH.as_tuple(), sc, hc, flags=aeg.FREE_SRC)                            # ①②
        xob = a.xfer_export(xo)
        # 40-byte head + (L + 1) 64-byte IPC event handles; pieces add their table and events
        assert (len(xob) > 40 + (SH.L + 1) * 64) == (nblocks * SH.chunk_bytes() > 4 * MIB)
        parent.send(([int(b) for b in hc], xob))
        xblob, do = recv()
        xd = a.xfer_import(1, xblob)
        out_done = a.layer_ready(xo, -1, aeg.READY_QUERY)
        in_done = a.layer_ready(xd, -1, aeg.READY_QUERY)
        a.kv_free_after(aeg.POOL_HOST, hc, xd)        # Ry-style: CPU blocks wait in the move list
        q = a.stats(aeg.POOL_HOST).quarantined_blocks
        fresh = a.kv_alloc(aeg.POOL_HOST, SH.as_tuple(), 4)      # allocation skips them (❸)
        assert (out_done, in_done, q) == (False, False, nblocks)
        assert not {aeg.decode_block(b)[1:] for b in fresh} & set(map(tuple, ho))
        gate.open()                                   # prefill done: P->C runs, then C->D on D's side
        got = np.frombuffer(recv(), dtype=np.uint8)
        himg2 = OK.swap_out(aimg, A.geom, himg, H.geom, SH, so, ho)
        geom = OK.PoolGeom(nslabs * MIB, MIB, aeg.LAYER_MAJOR)
        dimg = gi.region_bytes(gi.kv_seed(1), gi.poison_key(gi.TAG_NEVER, 0), geom.nbytes)
        exp = OK.swap_in(himg2, H.geom, dimg, geom, SH, ho, do)
        assert first_diff(got, exp) is None
        for _ in range(2000):                         # step ⑧: reclaimed once D's swap-in completed
            a.reclaim()
            if a.stats(aeg.POOL_HOST).quarantined_blocks == 0:
                break
        assert a.stats(aeg.POOL_HOST).quarantined_blocks == 0
        parent.send("bye")
        a.shutdown()
    finally:
        p.join(timeout=30)
        if p.is_alive():
            p.kill()
    assert p.exitcode == 0


@pytest.mark.parametrize("ce", [False, True], ids=["kernel", "ce"])
def test_two_device_same_process_migrate(ce):
    """H5 across two GPUs of one process (aeg_import_peer's same-process cross-device branch: peer
    access enabled, the migrate kernel on cuda:0 stores into cuda:1's pool over NVLink): the
    destination image equals oracle.kv.migrate (O7).  Needs two visible GPUs."""
    require_gpu()
    import torch
    if torch.cuda.device_count() < 2:
        pytest.skip("needs two visible GPUs")
    cfg = lambda lay, slab: aeg.default_config(  # noqa: E731
        device_kv_bytes=6 * slab, host_kv_bytes=MIB, dev_slab_bytes=slab, host_slab_bytes=MIB,
        dev_slab_layout=lay, staging_slot_bytes=MIB, staging_slots=2, stage_ring_bytes=4 * MIB,
        stage_chunk_bytes=MIB, table_arena_bytes=2 * MIB, host_threads=1, kernel=aeg.KERNEL_LSU)
    a = aeg.Context(0, cfg(aeg.LAYER_MAJOR, MIB))
    b = aeg.Context(1, cfg(aeg.BLOCK_MAJOR, MIB + 64 * 1024))
    try:
        A = Side(a, aeg.POOL_DEVICE, 6 * MIB, MIB, aeg.LAYER_MAJOR)
        torch.cuda.set_device(1)
        B = Side(b, aeg.POOL_DEVICE, 6 * (MIB + 64 * 1024), MIB + 64 * 1024, aeg.BLOCK_MAJOR)
        B.poison(gi.TAG_NEVER)
        bimg = B.poison_img(gi.TAG_NEVER)
        dc, do = B.alloc(SH, 50)
        poison_blocks(B, bimg, SH, do)
        torch.cuda.set_device(0)
        A.poison(gi.TAG_NEVER)
        aimg = A.poison_img(gi.TAG_NEVER)
        sc, so = A.alloc(SH, 50)
        fill_blocks(A, aimg, SH, so, [(4, j) for j in range(50)])
        a.import_peer(1, b.export_ipc())
        x = a.kv_migrate(SH.as_tuple(), sc, 1, dc, flags=aeg.MIGRATE_CE if ce else 0)
        a.layer_ready(x, -1, aeg.READY_BLOCK)
        exp = OK.migrate(aimg, A.geom, bimg, B.geom, SH, so, do)
        torch.cuda.set_device(1)
        assert first_diff(B.read(), exp) is None
        torch.cuda.set_device(0)
        assert first_diff(A.read(), aimg) is None
    finally:
        torch.cuda.set_device(0)
        a.shutdown()
        b.shutdown()
