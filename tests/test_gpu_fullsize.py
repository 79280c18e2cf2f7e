"""Full-size parity (BASELINE.json configs[1] and configs[3] sizes) in the launch configuration
bench.py times: the 64-request Qwen-7B batch (3,970 blocks, 31 GiB per direction) on an aged pool,
one swap round trip through the default staging slots and kernels; then every chunk of the 82 GiB
device pool and every written host chunk is checked against the oracle's label image (oracle/kv.py at
chunk granularity, O5/O6), plus chunks compared byte-for-byte with the NumPy generator.
Weights: Qwen-1.8B shapes staged at TP=2, rank 1, sampled tensors compared with oracle O8."""
import numpy as np
import pytest

import aeg_inputs as gi
import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg
from aeg_inputs import dev as D
from oracle import weights as W

from .gpu_harness import require_gpu

pytestmark = pytest.mark.gpu


def test_c2_full_size_round_trip():
    require_gpu()
    import torch
    import bench
    from .oracle_swapbench import OracleSwapBench
    sb = OracleSwapBench(aeg, bench.QWEN7B, 64, aeg.KERNEL_AUTO).setup()
    try:
        sb.sink = torch.zeros(1, dtype=torch.int64, device="cuda")
        cons = torch.cuda.Stream()
        sb.step(torch, cons)
        sb.step(torch, cons, with_consumer=False, keep_host_offsets=True)
        v = sb.replay_and_verify()
        assert v["device_chunks_checked"] > 300_000 and v["host_chunks_checked"] >= sb.n * 32
        assert v["ok"], v
        w = sb.verify()   # bench.py's own (oracle-free) invariant check agrees
        assert w["ok"] and w["batch_host_chunks_checked"] == sb.n * 32, w
    finally:
        sb.ctx.shutdown()


def test_c2_full_size_back_to_back():
    """The bench's back_to_back leg at full size: six 31 GiB round trips issued with no host sync
    between them (two in flight, no timing events), each swap-out reading blocks the previous
    swap-in is still writing (rule ❷ per layer / piece) into host blocks the previous swap-in may
    still read (❸).  The oracle replays the same placements sequentially; every chunk of the
    device pool (~450k) and every written host chunk must match."""
    require_gpu()
    import torch
    import bench
    from .oracle_swapbench import OracleSwapBench
    sb = OracleSwapBench(aeg, bench.QWEN7B, 64, aeg.KERNEL_AUTO, dev_batches=3, host_batches=2,
                         timing=False).setup()
    try:
        ops, inflight = [], []
        for j in range(6):
            if len(inflight) == 2:
                for t in inflight.pop(0):
                    sb.ctx.layer_ready(t, -1, aeg.READY_BLOCK)
                    sb.ctx.xfer_release(t)
            hc = sb.ctx.kv_alloc(aeg.POOL_HOST, sb.sht, sb.n)
            nd = sb.ctx.kv_alloc(aeg.POOL_DEVICE, sb.sht, sb.n)
            x = sb.ctx.kv_swap_out(sb.sht, sb.src_c, hc, flags=aeg.FREE_SRC)
            y = sb.ctx.kv_swap_in(sb.sht, hc, nd, flags=aeg.FREE_SRC)
            inflight.append((x, y))
            ops.append((sb.src_c, hc, nd))
            sb.src_c = nd
        for xs in inflight:
            for t in xs:
                sb.ctx.layer_ready(t, -1, aeg.READY_BLOCK)
                sb.ctx.xfer_release(t)
        torch.cuda.synchronize()
        v = sb.replay_given_and_verify(ops)
        assert v["device_chunks_checked"] > 400_000 and v["host_chunks_checked"] >= 2 * sb.n * 32, v
        assert v["ok"], v
    finally:
        sb.ctx.shutdown()


def test_qwen18b_tp2_weights_full_size_sampled():
    require_gpu()
    descs_all = gi.model_tensors("qwen-1.8b")
    sizes = [d["rows"] * d["cols"] * 2 for d in descs_all]
    offs = np.cumsum([0] + [-(-s // 256) * 256 for s in sizes])
    buf = np.empty(int(offs[-1]), dtype=np.uint8)
    for k, (o, s) in enumerate(zip(offs, sizes)):
        D.host_fill(buf[o:o + s], gi.w_seed(5), gi.weight_key(2, k), threads=16)
    descs = [dict(host_src=buf.ctypes.data + int(o), rows=t["rows"], cols=t["cols"], elem_bytes=2, layer=t["layer"],
                  split=t["split"], groups=t["groups"]) for t, o in zip(descs_all, offs)]
    ctx = aeg.Context(0, aeg.default_config(device_kv_bytes=1 << 30, host_kv_bytes=1 << 30,
                                            device_weight_bytes=2 << 30))
    try:
        got_offs, x = ctx.weights_stage(descs, tp_rank=1, tp_size=2)
        ctx.layer_ready(x, -1, aeg.READY_BLOCK)
        shard_sizes = [d["rows"] * d["cols"] * 2 // (1 if d["split"] == W.REPLICATED else 2) for d in descs_all]
        exp_offs, _ = W.bump_offsets(shard_sizes, 0)
        assert [int(o) for o in got_offs] == exp_offs
        base, _, _ = ctx.weights_region()
        rng = np.random.default_rng(0)
        for k in sorted(set([0, len(descs_all) - 1] + rng.choice(len(descs_all), 12, replace=False).tolist())):
            d = descs_all[k]
            full = buf[offs[k]:offs[k] + sizes[k]].reshape(d["rows"], d["cols"], 2)
            sh = np.ascontiguousarray(W.shard(full, d["split"], d["groups"], 1, 2)).reshape(-1)
            got = D.read(base + exp_offs[k], sh.size)
            assert np.array_equal(got, sh), (k, d["name"])
    finally:
        ctx.shutdown()


def test_c3_full_size_handoff():
    """configs[2] at the size bench.py times on one GPU: 16 Llama-2-13B requests (2,346 blocks,
    30.7 GB) from a layer-major pool into a block-major pool of another context (peer-mapped), AUTO
    kernel (LSU).  Expected image: oracle O7 on chunk labels over the whole destination pool
    (every chunk, including the untouched poison around the destination blocks)."""
    require_gpu()
    from oracle import kv as OK
    from oracle.shape import KVShape
    from oracle.slab import SlabPool
    sht = gi.KV_SHAPES["llama-2-13b"]
    sh = KVShape(*sht)
    cl = sh.chunk_bytes()
    lens = gi.request_lengths(3, 16, 512, 4096)
    blocks = [-(-t // 16) for t in lens]
    n = sum(blocks)
    slab = (1 << 30) + (256 << 20)
    nslab = -(-n // (slab // sh.block_bytes())) + 1
    seed = gi.kv_seed(3)
    mk = lambda lay: aeg.Context(0, aeg.default_config(device_kv_bytes=nslab * slab, host_kv_bytes=1 << 30,  # noqa: E731
                                                       dev_slab_bytes=slab, dev_slab_layout=lay))
    a, b = mk(aeg.LAYER_MAJOR), mk(aeg.BLOCK_MAJOR)
    try:
        ga = OK.PoolGeom(nslab * slab, slab, aeg.LAYER_MAJOR)
        gb = OK.PoolGeom(nslab * slab, slab, aeg.BLOCK_MAJOR)
        oa, ob = SlabPool(ga.nbytes, slab), SlabPool(gb.nbytes, slab)
        abase, _ = a.pool_region(0)
        bbase, _ = b.pool_region(0)
        D.fill_region(bbase, gb.nbytes, seed, gi.poison_key(gi.TAG_NEVER, 0))
        cells = gb.nbytes // cl
        blab = np.uint64(gi.poison_key(gi.TAG_NEVER, 0)) + np.arange(cells, dtype=np.uint64) * np.uint64(cl // 8)
        alab = np.zeros(ga.nbytes // cl, dtype=np.uint64)
        sc, so = a.kv_alloc(0, sht, n), oa.alloc(sh, n)
        dc, do = b.kv_alloc(0, sht, n), ob.alloc(sh, n)
        assert [aeg.decode_block(x)[1:] for x in sc] == list(so)
        assert [aeg.decode_block(x)[1:] for x in dc] == list(do)
        labels = [(r, j) for r, k in enumerate(blocks) for j in range(k)]
        offs = np.array([OK.addr(ga, sh, h, l) for h in so for l in range(sh.L)], np.uint64)
        keys = np.array([gi.kv_key(1, r, j, l) for (r, j) in labels for l in range(sh.L)], np.uint64)
        for i in range(0, offs.size, 1 << 16):
            D.fill_chunks(abase, offs[i:i + (1 << 16)], keys[i:i + (1 << 16)], cl, seed)
        alab[(offs // np.uint64(cl)).astype(np.int64)] = keys
        a.import_peer(1, b.export_ipc())
        x = a.kv_migrate(sht, sc, 1, dc)
        a.layer_ready(x, -1, aeg.READY_BLOCK)
        a.xfer_release(x)
        exp = OK.migrate(alab, ga, blab, gb, sh, so, do, unit=cl)
        bad = 0
        allo = np.arange(cells, dtype=np.uint64) * np.uint64(cl)
        for i in range(0, cells, 1 << 16):
            bd, _ = D.verify_chunks(bbase, allo[i:i + (1 << 16)], exp[i:i + (1 << 16)], cl, seed)
            bad += bd
        assert bad == 0
        # two chunks byte-for-byte against the NumPy generator
        for h, l in ((do[0], 0), (do[-1], sh.L - 1)):
            o = OK.addr(gb, sh, h, l)
            assert np.array_equal(D.read(bbase + o, cl), gi.region_bytes(seed, int(exp[o // cl]), cl))
    finally:
        a.shutdown()
        b.shutdown()


def test_packed_local_migrate_with_a_short_last_launch():
    """Local hand-off launches pack consecutive layers up to 4 GiB (swap.cc): with 1.5 GiB layers
    and L = 3 the layers go as [0, 2) + [2, 3) — a multi-layer launch and a short last one.  Every
    chunk of the destination pool equals oracle O7 on chunk labels, and each layer is ready (its
    event recorded when the launch holding it completes) with its bytes in place."""
    require_gpu()
    from oracle import kv as OK
    from oracle.shape import KVShape
    from oracle.slab import SlabPool
    sht = (3, 8, 128, 2, 16)                 # Cl = 64 KiB, block = 192 KiB
    sh = KVShape(*sht)
    cl = sh.chunk_bytes()
    n = (3 << 29) // cl                      # 1.5 GiB per layer
    slab = 1 << 30
    nslab = -(-n // (slab // sh.block_bytes())) + 1
    seed = gi.kv_seed(7)
    mk = lambda lay: aeg.Context(0, aeg.default_config(device_kv_bytes=nslab * slab, host_kv_bytes=1 << 30,  # noqa: E731
                                                       dev_slab_bytes=slab, dev_slab_layout=lay,
                                                       flags=aeg.CFG_TIMING))
    a, b = mk(aeg.LAYER_MAJOR), mk(aeg.BLOCK_MAJOR)
    try:
        ga = OK.PoolGeom(nslab * slab, slab, aeg.LAYER_MAJOR)
        gb = OK.PoolGeom(nslab * slab, slab, aeg.BLOCK_MAJOR)
        oa, ob = SlabPool(ga.nbytes, slab), SlabPool(gb.nbytes, slab)
        abase, _ = a.pool_region(0)
        bbase, _ = b.pool_region(0)
        D.fill_region(bbase, gb.nbytes, seed, gi.poison_key(gi.TAG_NEVER, 0))
        cells = gb.nbytes // cl
        blab = np.uint64(gi.poison_key(gi.TAG_NEVER, 0)) + np.arange(cells, dtype=np.uint64) * np.uint64(cl // 8)
        alab = np.zeros(ga.nbytes // cl, dtype=np.uint64)
        sc, so = a.kv_alloc(0, sht, n), oa.alloc(sh, n)
        dc, do = b.kv_alloc(0, sht, n), ob.alloc(sh, n)
        assert [aeg.decode_block(x)[1:] for x in sc] == list(so)
        assert [aeg.decode_block(x)[1:] for x in dc] == list(do)
        offs = np.array([OK.addr(ga, sh, h, l) for h in so for l in range(sh.L)], np.uint64)
        keys = np.array([gi.kv_key(9, 0, j, l) for j in range(n) for l in range(sh.L)], np.uint64)
        for i in range(0, offs.size, 1 << 16):
            D.fill_chunks(abase, offs[i:i + (1 << 16)], keys[i:i + (1 << 16)], cl, seed)
        alab[(offs // np.uint64(cl)).astype(np.int64)] = keys
        a.import_peer(1, b.export_ipc())
        a.kernel_stats_reset()
        x = a.kv_migrate(sht, sc, 1, dc)
        exp = OK.migrate(alab, ga, blab, gb, sh, so, do, unit=cl)
        for l in range(sh.L):                # per-layer readiness: that layer's chunks are in place
            a.layer_ready(x, l, aeg.READY_BLOCK)
            lo = np.array([OK.addr(gb, sh, h, l) for h in do], np.uint64)
            bad, _ = D.verify_chunks(bbase, lo, exp[(lo // np.uint64(cl)).astype(np.int64)], cl, seed)
            assert bad == 0, (l, bad)
        a.layer_ready(x, -1, aeg.READY_BLOCK)
        a.xfer_release(x)
        assert a.kernel_stats(aeg.K_MIGRATE)[0] == 2     # [0, 2) and [2, 3)
        bad = 0
        allo = np.arange(cells, dtype=np.uint64) * np.uint64(cl)
        for i in range(0, cells, 1 << 16):
            bd, _ = D.verify_chunks(bbase, allo[i:i + (1 << 16)], exp[i:i + (1 << 16)], cl, seed)
            bad += bd
        assert bad == 0
    finally:
        a.shutdown()
        b.shutdown()


def test_c4_full_size_three_model_switch():
    """configs[3] at full size: Qwen-1.8B / Llama-7B / Yi-9B weights (3.7 / 13.5 / 17.7 GB, generated
    pageable Model Caches) with 1 GiB of KV each, switched A -> B -> C -> A in the production order
    (B's KV in, B's weights staged through the Stage Buffer, a per-layer consumer wait, A's KV out
    fenced after it).  After every switch: every KV chunk of every
    model — on the device or in the host pool — equals the generator's content at the library's
    block table (O5/O6: a swap is the identity under relabelling), and the running model's weights
    equal oracle O8 (TP = 1: the tensors at the bump offsets) on 14 sampled tensors."""
    require_gpu()
    import torch
    GIB = 1 << 30
    names = ["qwen-1.8b", "llama-7b", "yi-9b"]
    seed = gi.kv_seed(4)
    models = []
    wmax = 0
    for m, nm in enumerate(names):
        ts = gi.model_tensors(nm)
        sizes = [t["rows"] * t["cols"] * 2 for t in ts]
        offs = np.cumsum([0] + [-(-s // 256) * 256 for s in sizes])
        buf = np.empty(int(offs[-1]), dtype=np.uint8)
        for k, (o, s) in enumerate(zip(offs, sizes)):
            D.host_fill(buf[o:o + s], gi.w_seed(6), gi.weight_key(10 + m, k), threads=16)
        descs = [dict(host_src=buf.ctypes.data + int(o), rows=t["rows"], cols=t["cols"], elem_bytes=2,
                      layer=t["layer"], split=t["split"], groups=t["groups"]) for t, o in zip(ts, offs)]
        sht = gi.KV_SHAPES[nm]
        L, H, Dh, s_, B = sht
        n = GIB // (L * 2 * H * Dh * s_ * B)
        models.append(dict(name=nm, ts=ts, sizes=sizes, offs=offs, buf=buf, descs=descs, sht=sht, n=n,
                           keys=[gi.kv_key(11 + m, 0, i, l) for i in range(n) for l in range(L)]))
        wmax = max(wmax, int(offs[-1]))
    ctx = aeg.Context(0, aeg.default_config(device_kv_bytes=8 * GIB, host_kv_bytes=8 * GIB,
                                            device_weight_bytes=wmax + (64 << 20), host_threads=12))
    try:
        dbase, _ = ctx.pool_region(aeg.POOL_DEVICE)
        hbase, _ = ctx.pool_region(aeg.POOL_HOST)
        wbase, _, _ = ctx.weights_region()

        def chunk_offs(pool, M, blocks):
            o0, ls = ctx.block_offsets(pool, M["sht"], blocks)
            return [int(o) + l * int(ls) for o in o0 for l in range(M["sht"][0])]

        def check_kv():
            for M in models:
                pool, base = (aeg.POOL_DEVICE, dbase) if M["where"] == "dev" else (aeg.POOL_HOST, hbase)
                bad, first = D.verify_chunks(base, chunk_offs(pool, M, M["blocks"]), M["keys"],
                                             aeg.KVShape.of(M["sht"]).chunk_bytes(), seed)
                assert bad == 0, (M["name"], M["where"], first)

        for M in models:   # every model's decode KV starts in the host pool
            M["blocks"] = ctx.kv_alloc(aeg.POOL_HOST, M["sht"], M["n"])
            M["where"] = "host"
            D.fill_chunks(hbase, chunk_offs(aeg.POOL_HOST, M, M["blocks"]), M["keys"],
                          aeg.KVShape.of(M["sht"]).chunk_bytes(), seed)
        cons = torch.cuda.Stream()
        rng = np.random.default_rng(4)
        cur = None
        for b in [0, 1, 2, 0]:
            B_, A_ = models[b], (models[cur] if cur is not None else None)
            db = ctx.kv_alloc(aeg.POOL_DEVICE, B_["sht"], B_["n"])
            ctx.stream_fence(cons.cuda_stream)
            xi = ctx.kv_swap_in(B_["sht"], B_["blocks"], db, flags=aeg.FREE_SRC)
            ctx.weights_reset(0)
            woffs, xw = ctx.weights_stage(B_["descs"])
            for l in range(B_["sht"][0]):
                ctx.layer_ready(xi, l, aeg.READY_WAIT_STREAM, cons.cuda_stream)
            ctx.layer_ready(xw, -1, aeg.READY_WAIT_STREAM, cons.cuda_stream)
            xo = None
            if A_ is not None:
                ctx.stream_fence(cons.cuda_stream)
                hb = ctx.kv_alloc(aeg.POOL_HOST, A_["sht"], A_["n"])
                xo = ctx.kv_swap_out(A_["sht"], A_["blocks"], hb, flags=aeg.FREE_SRC)
            for x in (xi, xw, xo):
                if x is not None:
                    ctx.layer_ready(x, -1, aeg.READY_BLOCK)
                    ctx.xfer_release(x)
            B_.update(blocks=db, where="dev")
            if A_ is not None:
                A_.update(blocks=hb, where="host")
            check_kv()
            exp_offs, _ = W.bump_offsets(B_["sizes"], 0)
            assert [int(o) for o in woffs] == exp_offs
            nt = len(B_["ts"])
            for k in sorted(set([0, nt - 1] + rng.choice(nt, 12, replace=False).tolist())):
                nbytes = min(B_["sizes"][k], 1 << 24)
                got = D.read(wbase + exp_offs[k], nbytes)
                assert np.array_equal(got, B_["buf"][B_["offs"][k]:B_["offs"][k] + nbytes]), (B_["name"], k)
            cur = b
    finally:
        ctx.shutdown()
