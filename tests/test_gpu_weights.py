"""GPU parity for H7 (weight staging) and N1 (relocation): the weights region after
aeg_weights_stage equals oracle/weights.stage on the same generated Model Cache, for TP ranks of
1/2/4, through the staged pipeline (small chunks and a small Stage Buffer ring so slots are reused
many times) and through the registered direct path; per-layer readiness; relocation = memmove."""
import numpy as np
import pytest

import aeg_inputs as gi
import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg
from aeg_inputs import dev as D
from oracle import weights as W

from .gpu_harness import first_diff, require_gpu

pytestmark = pytest.mark.gpu
SEEDW = gi.w_seed(4)


def model_cache(descs, m=1):
    """Host Model Cache: tensors at 256-aligned offsets of one pageable buffer (generated content)."""
    sizes = [d["rows"] * d["cols"] * 2 for d in descs]
    offs, p = [], 0
    for n in sizes:
        offs.append(p)
        p += -(-n // 256) * 256
    buf = np.empty(p + 256, dtype=np.uint8)
    tens = []
    for k, (o, n) in enumerate(zip(offs, sizes)):
        view = buf[o:o + n]
        view[:] = gi.region_bytes(SEEDW, gi.weight_key(m, k), n)
        tens.append(view.reshape(descs[k]["rows"], descs[k]["cols"] * 2))
    return buf, tens


def synth_model(h=512, L=4, ff=1536, V=4096, arch="llama"):
    gi.MODELS["_test"] = (h, L, ff, V, h // 4, arch)
    d = gi.model_tensors("_test")
    del gi.MODELS["_test"]
    return d


def make(chunk=1 << 20, ring=4 << 20, wbytes=64 << 20, threads=4):
    cfg = aeg.default_config(device_kv_bytes=4 << 20, host_kv_bytes=4 << 20, dev_slab_bytes=1 << 20,
                             host_slab_bytes=1 << 20, stage_ring_bytes=ring, stage_chunk_bytes=chunk,
                             staging_slot_bytes=1 << 20, staging_slots=2, device_weight_bytes=wbytes,
                             table_arena_bytes=2 << 20, host_threads=threads)
    return aeg.Context(0, cfg)


def descs_for(buf_tens, descs):
    return [dict(host_src=t.ctypes.data, rows=d["rows"], cols=d["cols"], elem_bytes=2, layer=d["layer"],
                 split=d["split"], groups=d["groups"]) for t, d in zip(buf_tens, descs)]


@pytest.mark.parametrize("tp", [1, 2, 4, 8])
@pytest.mark.parametrize("direct", [False, True])
@pytest.mark.parametrize("arch", ["llama", "qwen1"])      # qwen1: fused QKV, COL split per group of 3
def test_stage_matches_oracle(tp, direct, arch):
    require_gpu()
    descs = synth_model(arch=arch)
    buf, tens = model_cache(descs)
    ctx = make()
    try:
        if direct:
            ctx.host_register(buf.ctypes.data, buf.nbytes)
        base, wbytes, _ = ctx.weights_region()
        for r in range(tp):
            ctx.weights_reset(0)
            offs, x = ctx.weights_stage(descs_for(tens, descs), tp_rank=r, tp_size=tp)
            n_layers = ctx.xfer_layers(x)
            assert n_layers == max(d["layer"] for d in descs) + 1
            for l in range(n_layers):
                ctx.layer_ready(x, l, aeg.READY_BLOCK)
            ctx.layer_ready(x, -1, aeg.READY_BLOCK)
            exp, eoffs, end = W.stage(tens, descs, r, tp, region_bytes=wbytes)
            assert [int(o) for o in offs] == eoffs
            got = D.read(base, end)
            assert first_diff(got, exp[:end]) is None
            _, _, bump = ctx.weights_region()
            assert bump == end
            ctx.xfer_release(x)
        if direct:
            ctx.host_unregister(buf.ctypes.data)
    finally:
        ctx.shutdown()


def test_layer_events_fire_in_order_and_queries_are_monotone():
    require_gpu()
    descs = synth_model(L=6)
    buf, tens = model_cache(descs)
    ctx = make(chunk=1 << 20, ring=2 << 20, threads=2)
    try:
        offs, x = ctx.weights_stage(descs_for(tens, descs))
        L = ctx.xfer_layers(x)
        seen = [False] * L
        for _ in range(100000):
            for l in range(L):
                r = ctx.layer_ready(x, l, aeg.READY_QUERY)
                assert r or not seen[l]                # once ready, stays ready
                seen[l] = seen[l] or r
            if all(seen):
                break
        ctx.layer_ready(x, -1, aeg.READY_BLOCK)
        assert all(ctx.layer_ready(x, l, aeg.READY_QUERY) for l in range(L))
    finally:
        ctx.shutdown()


def test_relocate_is_memmove():
    """N1: a model prefetched after the running one moves to the buffer start."""
    require_gpu()
    descs = synth_model()
    buf, tens = model_cache(descs)
    ctx = make(wbytes=64 << 20)
    try:
        base, wbytes, _ = ctx.weights_region()
        running = 3 << 20                                   # pretend a 3 MiB model occupies [0, 3 MiB)
        ctx.weights_reset(running)
        offs, x = ctx.weights_stage(descs_for(tens, descs))
        ctx.layer_ready(x, -1, aeg.READY_BLOCK)            # the prefetch has landed
        _, _, end = ctx.weights_region()
        size = end - running
        assert size > running                                 # overlapping move (size > gap)
        y = ctx.weights_relocate(running, 0, size)
        ctx.layer_ready(y, -1, aeg.READY_BLOCK)
        # expected: oracle O8 staging at base `running`, then oracle N1 memmove to 0
        img, offs_o, end_o = W.stage(tens, descs, 0, 1, region_bytes=wbytes, base=running)
        assert end_o == end and [int(o) for o in offs] == offs_o
        from oracle.memmove import memmove
        exp = memmove(img, running, 0, size)
        got = D.read(base, size)
        assert first_diff(got, exp[:size]) is None
        ctx.xfer_release(x)
        ctx.xfer_release(y)
    finally:
        ctx.shutdown()


def test_invalid_and_oom():
    require_gpu()
    ctx = make(wbytes=1 << 20)
    try:
        a = np.zeros(6 * 5 * 2, np.uint8)
        with pytest.raises(aeg.AegError) as e:
            ctx.weights_stage([dict(host_src=a.ctypes.data, rows=6, cols=5, layer=0, split=aeg.SPLIT_COL)], 0, 4)
        assert e.value.code == aeg.ERR_INVALID
        big = np.zeros(2 << 20, np.uint8)
        with pytest.raises(aeg.AegError) as e:
            ctx.weights_stage([dict(host_src=big.ctypes.data, rows=1024, cols=1024, layer=0)])
        assert e.value.code == aeg.ERR_OOM
    finally:
        ctx.shutdown()


@pytest.mark.parametrize("direct", [False, True])
def test_region_boundary_matches_the_oracle(direct):
    """The region must hold the shards, [0, off_last + size_last) (oracle O8, reading 17): with a
    region size that is not a multiple of the 256-byte bump alignment, an exact fit stages (padding
    written only up to the region's end), one byte short is ERR_OOM — as in oracle/weights.stage."""
    require_gpu()
    descs = [dict(rows=3, cols=100, split=W.REPLICATED, groups=1, layer=0),
             dict(rows=1, cols=50, split=W.REPLICATED, groups=1, layer=1)]
    buf, tens = model_cache(descs, m=3)
    need = 768 + 100                       # 600 B at 0, 100 B at 768 (bump alignment 256)
    for wbytes, ok in ((need, True), (need - 1, False)):
        ctx = make(wbytes=wbytes)
        try:
            if direct:
                ctx.host_register(buf.ctypes.data, buf.nbytes)
            dl = descs_for(tens, descs)
            if not ok:
                with pytest.raises(aeg.AegError) as e:
                    ctx.weights_stage(dl)
                assert e.value.code == aeg.ERR_OOM
                with pytest.raises(W.WeightError):
                    W.stage(tens, descs, 0, 1, region_bytes=wbytes)
                continue
            base, _, _ = ctx.weights_region()
            offs, x = ctx.weights_stage(dl)
            ctx.layer_ready(x, -1, aeg.READY_BLOCK)
            exp, eoffs, _ = W.stage(tens, descs, 0, 1, region_bytes=wbytes)
            assert [int(o) for o in offs] == eoffs == [0, 768]
            assert first_diff(D.read(base, wbytes), exp[:wbytes]) is None
            ctx.xfer_release(x)
            if direct:
                ctx.host_unregister(buf.ctypes.data)
        finally:
            ctx.shutdown()
