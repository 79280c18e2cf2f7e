"""World-size-2 `gloo` tests (CPU) of the multi-GPU host logic: rank roles, hand-off pairing, the
control-data exchange (pool blobs, destination handles, transfer blobs) and that exchanged handles
decode to blocks the destination's allocator really owns.  The GPU data path itself needs >= 2 GPUs
(not available to this build) and is covered on one GPU by tests/test_gpu_migrate.py."""
import os
import socket

import pytest
import torch.distributed as td
import torch.multiprocessing as mp

from paper_conf_sosp_xiang0qyzyzl0025_b200 import dist as D


def test_pairs_layout():
    assert D.handoff_pairs(1) == []
    assert D.handoff_pairs(2) == [(0, 1)]
    assert D.handoff_pairs(8) == [(0, 4), (1, 5), (2, 6), (3, 7)]
    for w in (2, 4, 8):
        h = w // 2
        seen = set()
        for r in range(h):
            p = D.handoff_pairs(w, "all2all", r)
            assert sorted(s for s, _ in p) == list(range(h))          # every prefill rank sends once
            assert sorted(d for _, d in p) == list(range(h, w))       # every decode rank receives once
            seen |= set(p)
        assert seen == {(i, j) for i in range(h) for j in range(h, w)}
    assert [D.role(r, 8) for r in range(8)] == ["prefill"] * 4 + ["decode"] * 4


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


class FakeCtx:
    """Stands in for aeg.Context on CPU: a host-only library context for the allocator plus a fixed
    export blob (no CUDA IPC without a GPU)."""

    def __init__(self, rank):
        import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg
        self.aeg = aeg
        self.rank = rank
        self.c = aeg.Context(0, aeg.default_config(device_kv_bytes=8 << 20, host_kv_bytes=1 << 20,
                                                   dev_slab_bytes=1 << 20, host_slab_bytes=1 << 20,
                                                   flags=aeg.CFG_HOST_ONLY | aeg.CFG_NO_DAEMON))
        self.imported = {}
        self.migrated = []

    def export_ipc(self):
        return b"blob-of-rank-%d" % self.rank

    def import_peer(self, peer, blob):
        self.imported[peer] = blob

    def kv_migrate(self, shape, src, peer, dst, flags):
        self.migrated.append((peer, list(map(int, dst))))
        return 100 + peer


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    td.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg
        ctx = FakeCtx(rank)
        blobs = D.connect(ctx, rank)
        assert blobs == [b"blob-of-rank-%d" % r for r in range(world)]
        assert set(ctx.imported) == set(range(world)) - {rank}
        shape = (2, 1, 2, 2, 16)
        # decode ranks allocate destinations and publish their handles
        mine = [int(b) for b in ctx.c.kv_alloc(aeg.POOL_DEVICE, shape, 5)] if D.role(rank, world) == "decode" else None
        handles = D.exchange(mine)
        pairs = D.handoff_pairs(world)
        src = [int(b) for b in ctx.c.kv_alloc(aeg.POOL_DEVICE, shape, 5)] if D.role(rank, world) == "prefill" else []
        xs = D.handoff(ctx, shape, src, pairs, rank, handles)
        # transfer blobs travel back to the decode side
        got = D.exchange({d: x for d, x in xs.items()})
        if D.role(rank, world) == "decode":
            senders = [r for r, m in enumerate(got) if m and rank in m]
            assert senders == [s for s, d in pairs if d == rank]
            # the handles the prefill rank used are blocks this rank owns (geometry + ownership)
            ctx.c.kv_free(aeg.POOL_DEVICE, mine)
        else:
            assert ctx.migrated == [(d, handles[d]) for s, d in pairs if s == rank]
        q.put((rank, "ok"))
    except Exception as e:  # pragma: no cover - reported to the parent
        import traceback
        q.put((rank, traceback.format_exc()))
        raise
    finally:
        td.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_gloo_handoff_exchange(world):
    from paper_conf_sosp_xiang0qyzyzl0025_b200 import build
    build.build()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = dict(q.get(timeout=120) for _ in range(world))
    for p in ps:
        p.join(timeout=60)
    assert res == {r: "ok" for r in range(world)}, res
