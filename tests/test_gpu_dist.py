"""The multi-rank hand-off path with REAL contexts: world-size-2 torch.distributed
(gloo control plane) with both ranks on the one GPU — rank 0 the prefill instance, rank 1 the
decode instance (PAPER.md:2096-2098 layout, dist.handoff_pairs).  Pools and per-layer events travel
through dist.connect / dist.exchange (CUDA IPC memory + IPC events), the bytes through aeg_kv_migrate
(fused kernel, then the copy-engine route), and the decode rank checks every chunk of its destination
blocks against the generator (O7: a hand-off is the identity under relabelling)."""
import multiprocessing as mp
import os
import socket

import pytest

pytestmark = pytest.mark.gpu


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _rank(rank, world, port, q):
    import torch.distributed as td
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    td.init_process_group("gloo", rank=rank, world_size=world)
    ctx = None
    try:
        import aeg_inputs as gi
        import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg
        from aeg_inputs import dev as D
        from paper_conf_sosp_xiang0qyzyzl0025_b200 import dist as PD
        MIB = 1 << 20
        sht = (40, 2, 128, 2, 16)                      # Llama-2-13B layers, 2 KV heads: 16 KiB chunks
        ch = aeg.KVShape.of(sht).chunk_bytes()
        n = 150
        layout = aeg.LAYER_MAJOR if PD.role(rank, world) == "prefill" else aeg.BLOCK_MAJOR
        ctx = aeg.Context(0, aeg.default_config(device_kv_bytes=192 * MIB, host_kv_bytes=4 * MIB,
                                                dev_slab_bytes=4 * MIB, host_slab_bytes=MIB, dev_slab_layout=layout,
                                                staging_slot_bytes=8 * MIB, staging_slots=2,
                                                stage_ring_bytes=4 * MIB, stage_chunk_bytes=MIB,
                                                table_arena_bytes=2 * MIB, host_threads=1))
        base, _ = ctx.pool_region(aeg.POOL_DEVICE)
        seed = gi.kv_seed(5)
        PD.connect(ctx, rank)
        pairs = PD.handoff_pairs(world)
        prefill = PD.role(rank, world) == "prefill"

        def offs(blocks):
            o0, ls = ctx.block_offsets(aeg.POOL_DEVICE, sht, blocks)
            return [int(o) + l * int(ls) for o in o0 for l in range(sht[0])]
        results = []
        for route, flags in (("kernel", 0), ("copy engines", aeg.MIGRATE_CE)):
            dst = None if prefill else [int(b) for b in ctx.kv_alloc(aeg.POOL_DEVICE, sht, n)]
            if not prefill:    # poison the destination so a missed chunk cannot pass
                D.fill_chunks(base, offs(dst), [gi.poison_key(gi.TAG_DST, 8 * i) for i in range(n * sht[0])], ch,
                              seed)
            handles = PD.exchange(dst)
            dst_by_rank = {d: h for d, h in enumerate(handles) if h}
            xs = {}
            if prefill:
                src = ctx.kv_alloc(aeg.POOL_DEVICE, sht, n)
                keys = [gi.kv_key(3, rank, i, l) for i in range(n) for l in range(sht[0])]
                D.fill_chunks(base, offs(src), keys, ch, seed)
                xs = PD.handoff(ctx, sht, src, pairs, rank, dst_by_rank, flags=flags | aeg.FREE_SRC)
            blobs = PD.exchange({d: ctx.xfer_export(x) for d, x in xs.items()})
            if not prefill:
                sender = [s for s, d in pairs if d == rank][0]
                xi = ctx.xfer_import(sender, blobs[sender][rank])
                for l in range(sht[0]):                     # per-layer readiness through IPC events
                    ctx.layer_ready(xi, l, aeg.READY_BLOCK)
                keys = [gi.kv_key(3, sender, i, l) for i in range(n) for l in range(sht[0])]
                bad, first = D.verify_chunks(base, offs(dst), keys, ch, seed)
                results.append((route, bad, first))
                ctx.xfer_release(xi)
                ctx.kv_free(aeg.POOL_DEVICE, dst)
            PD.exchange("done")                             # the importer finished before release
            for x in xs.values():
                ctx.layer_ready(x, -1, aeg.READY_BLOCK)
                ctx.xfer_release(x)
        q.put((rank, results))
    except Exception:  # pragma: no cover - reported to the parent
        import traceback
        q.put((rank, traceback.format_exc()))
    finally:
        if ctx is not None:
            ctx.shutdown()
        td.destroy_process_group()


def test_two_rank_handoff_with_real_contexts():
    from .gpu_harness import require_gpu
    require_gpu()
    world = 2
    c = mp.get_context("spawn")
    q = c.Queue()
    port = _free_port()
    ps = [c.Process(target=_rank, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = dict(q.get(timeout=300) for _ in range(world))
    for p in ps:
        p.join(timeout=60)
        if p.is_alive():
            p.kill()
    assert isinstance(res[0], list), res[0]
    assert isinstance(res[1], list), res[1]
    assert [r for r, _, _ in res[1]] == ["kernel", "copy engines"]
    for route, bad, first in res[1]:
        assert bad == 0, (route, first)
