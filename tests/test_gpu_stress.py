"""Race stress (SURVEY.md §4 race tests; rules ❶❷❸): seeded random sequences of
swap-out / swap-in / local migrate (fused kernel or copy-engine route) / free (with FREE_SRC move lists) over small pools, while gate
kernels hold some transfers back and open at random later points, so transfers overlap in every
order the rules allow.  Checks: (1) the library's own primitive log passes the oracle's
happens-before checker (oracle/rules.py), including consumer reads after per-layer waits (❶);
(2) the final device and host images equal the oracle's sequential replay (oracle/kv.py) of the same
operations in host order, at the placements the library chose."""
import random

import numpy as np
import pytest

import aeg_inputs as gi
import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg
from aeg_inputs import dev as D
from oracle import kv as OK
from oracle.rules import check
from oracle.shape import KVShape

from .gpu_harness import SEED, Side, first_diff, require_gpu
from .test_gpu_swap import parse_trace

pytestmark = pytest.mark.gpu
KIB = 1024
SH = KVShape(2, 4, 64, 2, 16)            # 16 KiB chunks, 32 KiB blocks


def dec(bs):
    return [aeg.decode_block(b)[1:] for b in bs]


@pytest.mark.parametrize("seed", range(6))
def test_random_overlapping_transfers(seed):
    cfg = aeg.default_config(device_kv_bytes=24 * 256 * KIB, host_kv_bytes=24 * 256 * KIB, dev_slab_bytes=256 * KIB,
                             host_slab_bytes=256 * KIB, dev_slab_layout=seed % 2, host_slab_layout=(seed // 2) % 2,
                             staging_slot_bytes=1 << 20, staging_slots=2, stage_ring_bytes=4 << 20,
                             stage_chunk_bytes=1 << 20, device_weight_bytes=2 << 20, table_arena_bytes=2 << 20,
                             host_threads=1, kernel=[aeg.KERNEL_LSU, aeg.KERNEL_BULK, aeg.KERNEL_BULKW][seed % 3])
    _stress(seed, cfg, SH, 12)


SHB = KVShape(2, 32, 128, 2, 16)         # 256 KiB chunks: layers of >= 16 blocks are >= 4 MiB (pieces)


@pytest.mark.parametrize("seed", range(4))
def test_random_overlapping_transfers_with_d2h_pieces(seed):
    """The same stress with 1 MiB D2H pieces and layers big enough to use them: swap-ins (and
    migrates) of host blocks written by in-flight piecewise swap-outs wait per piece."""
    cfg = aeg.default_config(device_kv_bytes=40 * 2048 * KIB, host_kv_bytes=40 * 2048 * KIB,
                             dev_slab_bytes=2048 * KIB, host_slab_bytes=2048 * KIB, dev_slab_layout=seed % 2,
                             host_slab_layout=(seed // 2) % 2, staging_slot_bytes=(4 << 20) if seed % 2 else (8 << 20),
                             staging_slots=2, stage_ring_bytes=4 << 20, stage_chunk_bytes=1 << 20,
                             device_weight_bytes=2 << 20, table_arena_bytes=2 << 20, host_threads=1,
                             kernel=aeg.KERNEL_AUTO, dma_piece_mib=1, pack_layer_mib=1)
    log, n_out = _stress(100 + seed, cfg, SHB, 28, lo=14)
    # the swap-outs really ran in pieces: more D2H ops than (swap-out, layer) pairs
    assert n_out > 0 and sum(1 for e in log if e[0] == "op" and e[1] == "d2h") > n_out * SHB.L


SHP = KVShape(8, 2, 64, 2, 16)           # 8 KiB chunks, 8 layers: small layers are packed 2 per segment


@pytest.mark.parametrize("seed", range(4))
def test_random_overlapping_transfers_with_packed_layers(seed):
    """The same stress with layers small enough to be packed (default pack_layer_mib; the planner
    keeps >= 4 segments, so 2 of the 8 layers share each segment): per-layer events recorded after a
    multi-layer segment, waited for per layer by later transfers."""
    cfg = aeg.default_config(device_kv_bytes=24 * 512 * KIB, host_kv_bytes=24 * 512 * KIB, dev_slab_bytes=512 * KIB,
                             host_slab_bytes=512 * KIB, dev_slab_layout=seed % 2, host_slab_layout=(seed // 2) % 2,
                             staging_slot_bytes=1 << 20, staging_slots=2, stage_ring_bytes=4 << 20,
                             stage_chunk_bytes=1 << 20, device_weight_bytes=2 << 20, table_arena_bytes=2 << 20,
                             host_threads=1, kernel=aeg.KERNEL_AUTO)
    log, _ = _stress(200 + seed, cfg, SHP, 12)
    # packing really happened: some gather read two layers in one segment
    assert any(e[0] == "op" and e[1] == "gather" and len({c.rsplit(":", 1)[1] for c in e[3]}) == 2 for e in log)


def _stress(seed, cfg, SH, nmax, lo=1):
    require_gpu()
    import torch
    r = random.Random(seed)
    ctx = aeg.Context(0, cfg)
    try:
        dev = Side(ctx, 0, cfg.device_kv_bytes, cfg.dev_slab_bytes, cfg.dev_slab_layout)
        host = Side(ctx, 1, cfg.host_kv_bytes, cfg.host_slab_bytes, cfg.host_slab_layout)
        dev.poison(gi.TAG_NEVER)
        host.poison(gi.TAG_NEVER)
        dimg, himg = dev.poison_img(gi.TAG_NEVER), host.poison_img(gi.TAG_NEVER)
        log = []
        ctx.trace_enable(True)

        def flush():
            log.extend(parse_trace(ctx.trace_read()))

        objs = []        # [where, handles]
        n_out = 0
        gates = []       # open gates
        used = [False]   # a consumer read since the consumer stream was last drained
        cons = torch.cuda.Stream()
        for step in range(45):
            op = r.choice(["new", "new", "out", "out", "in", "in", "mig", "free", "gate", "open", "use"])
            if op == "new" or not objs:
                n = r.randint(lo, nmax)
                try:
                    c = ctx.kv_alloc(0, SH.as_tuple(), n)
                except aeg.AegError:
                    continue
                offs, keys = [], []
                for j, h in enumerate(dec(c)):
                    for l in range(SH.L):
                        o = OK.addr(dev.geom, SH, h, l)
                        offs.append(o)
                        keys.append(gi.kv_key(2, step, j, l))
                        dimg[o:o + SH.chunk_bytes()] = gi.region_bytes(SEED, keys[-1], SH.chunk_bytes())
                if used[0]:
                    # the test's own consumer may still be reading blocks freed since (the library
                    # cannot see reads outside it): like an engine that reuses memory only after its
                    # decode step, drain the consumer before the host writes fresh blocks — opening
                    # the gates first, since the consumer may wait on transfers they hold back
                    for g in gates:
                        g.open()
                    gates.clear()
                    cons.synchronize()
                    flush()
                    log.append(("record", "u0x%x" % cons.cuda_stream, f"cons{step}"))
                    log.append(("sync", f"cons{step}"))
                    used[0] = False
                D.fill_chunks(dev.base, offs, keys, SH.chunk_bytes(), SEED)
                # fresh blocks are touched by no incomplete transfer (❸); log the fill as a write
                flush()
                # the fill is synchronous: the host saw it complete before issuing anything later
                log.append(("op", "fill", "fill", [], [f"D:{s}:{j}:{l}" for s, j in dec(c) for l in range(SH.L)]))
                log.append(("record", "fill", f"fill{step}"))
                log.append(("sync", f"fill{step}"))
                objs.append(["dev", c])
                continue
            oi = r.randrange(len(objs))
            o = objs[oi]
            try:
                if op == "out" and o[0] == "dev":
                    hc = ctx.kv_alloc(1, SH.as_tuple(), len(o[1]))
                    ctx.kv_swap_out(SH.as_tuple(), o[1], hc, flags=aeg.FREE_SRC)
                    n_out += 1
                    himg = OK.swap_out(dimg, dev.geom, himg, host.geom, SH, dec(o[1]), dec(hc))
                    o[:] = ["host", hc]
                elif op == "in" and o[0] == "host":
                    dc = ctx.kv_alloc(0, SH.as_tuple(), len(o[1]))
                    x = ctx.kv_swap_in(SH.as_tuple(), o[1], dc, flags=aeg.FREE_SRC)
                    dimg = OK.swap_in(himg, host.geom, dimg, dev.geom, SH, dec(o[1]), dec(dc))
                    o[:] = ["dev", dc, x]
                elif op == "mig" and o[0] == "dev":
                    dc = ctx.kv_alloc(0, SH.as_tuple(), len(o[1]))
                    # the fused kernel or the copy-engine route (AEG_MIGRATE_CE), at random
                    ce = aeg.MIGRATE_CE if r.random() < 0.5 else 0
                    x = ctx.kv_migrate(SH.as_tuple(), o[1], -1, dc, flags=aeg.FREE_SRC | ce)
                    dimg = OK.migrate(dimg, dev.geom, dimg, dev.geom, SH, dec(o[1]), dec(dc))
                    o[:] = ["dev", dc, x]
                elif op == "free":
                    ctx.kv_free(0 if o[0] == "dev" else 1, o[1])
                    del objs[oi]
                elif op == "gate":
                    s = torch.cuda.Stream()
                    g = D.Gate()
                    g.close_on(s.cuda_stream)
                    ctx.stream_fence(s.cuda_stream)     # later transfers wait until it opens
                    gates.append(g)
                elif op == "open" and gates:
                    gates.pop(r.randrange(len(gates))).open()
                elif op == "use" and o[0] == "dev" and len(o) > 2:
                    # rule ❶: a decode consumer waits per layer on the transfer that produced o, then reads
                    for l in range(SH.L):
                        ctx.layer_ready(o[2], l, aeg.READY_WAIT_STREAM, cons.cuda_stream)
                    flush()
                    log.append(("use", "u0x%x" % cons.cuda_stream,
                                [f"D:{s}:{j}:{l}" for s, j in dec(o[1]) for l in range(SH.L)]))
                    used[0] = True
            except aeg.AegError as e:
                assert e.code == aeg.ERR_OOM, e       # pools are small: OOM is the only legal refusal
            flush()
        for g in gates:
            g.open()
        ctx.reclaim(blocking=True)
        torch.cuda.synchronize()
        flush()
        assert check(log)
        assert first_diff(dev.read(), dimg) is None
        assert first_diff(host.read(), himg) is None
        return log, n_out
    finally:
        for g in locals().get("gates", []):
            g.open()
        ctx.shutdown()
