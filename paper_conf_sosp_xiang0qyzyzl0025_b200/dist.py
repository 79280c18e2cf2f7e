"""Multi-GPU plumbing of the hand-off path (H5) and the per-rank replicas.

One process per GPU.  `torch.distributed` carries only control data: the aeg_export_ipc blobs (pool
IPC handle + geometry), destination block handles and aeg_xfer_export blobs (per-layer IPC events).
The bytes themselves move GPU->GPU through aeg_kv_migrate (fused gather -> NVLink stores); there is
no collective on the data path.

Layout (§7.4: "one prefill and one decode instance" per TP group on 8 GPUs):
ranks [0, N/2) are prefill instances, [N/2, N) decode instances.
"""
from __future__ import annotations


def handoff_pairs(world: int, mode: str = "pairs", round_: int = 0):
    """(src, dst) rank pairs of one hand-off round.
    pairs  : prefill i -> decode i + N/2 (the §7.4 layout).
    all2all: round r sends prefill i -> decode (i + r) mod N/2 + N/2, so N/2 rounds cover every
             (prefill, decode) pair exactly once and every rank has one partner per round."""
    if world < 2:
        return []
    h = world // 2
    if mode == "pairs":
        return [(i, i + h) for i in range(h)]
    if mode == "all2all":
        return [(i, (i + round_) % h + h) for i in range(h)]
    raise ValueError(mode)


def role(rank: int, world: int) -> str:
    return "prefill" if rank < world // 2 else "decode"


def exchange(obj, group=None):
    """all_gather_object of a small control object (bytes, lists of ints)."""
    import torch.distributed as td
    out = [None] * td.get_world_size(group)
    td.all_gather_object(out, obj, group=group)
    return out


def connect(ctx, rank: int, group=None):
    """Exchange pool IPC blobs and import every other rank as peer index = its rank."""
    blobs = exchange(ctx.export_ipc(), group)
    for peer, b in enumerate(blobs):
        if peer != rank:
            ctx.import_peer(peer, b)
    return blobs


def handoff(ctx, shape, src_blocks, pairs, rank: int, dst_handles_by_rank, flags: int = 0):
    """Enqueue this rank's migrates of one round.  Returns {dst_rank: xfer_id}."""
    out = {}
    for s, d in pairs:
        if s == rank:
            out[d] = ctx.kv_migrate(shape, src_blocks, d, dst_handles_by_rank[d], flags)
    return out
