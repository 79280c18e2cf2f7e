"""GPU parity for H8 (model-switch composition, BASELINE.json configs[3]): a token-level switch
A -> B on one GPU is B's KV swap-in (host -> fresh device blocks) enqueued first, then B's weights
(staged through the Stage Buffer, or relocated on the device after a prefetch, N1), a per-layer
consumer that waits on weights layer l and KV layer l, and A's KV swap-out fenced after that
consumer (§5, 2510-2513 A.2; Fig. 9 3.a/3.b).

Three models shaped like Qwen-1.8B / Llama-7B / Yi-9B (their layer counts; fewer KV heads and a
narrow hidden size so whole-pool images stay small) rotate through five switches.  After every
switch the whole device KV pool, the whole host KV pool and the whole weights region are compared
byte for byte with the oracle: O6 swap-in, O5 swap-out, O8 weight staging and N1 memmove applied
to the same generated inputs in the same order; the library trace passes the happens-before
checker of rules ❶❷❸."""
import numpy as np
import pytest

import aeg_inputs as gi
import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg
from aeg_inputs import dev as D
from oracle import kv as OK
from oracle import weights as W
from oracle.memmove import memmove
from oracle.rules import check
from oracle.shape import KVShape

from .gpu_harness import SEED, Side, fill_blocks, first_diff, require_gpu
from .test_gpu_swap import parse_trace
from .test_gpu_weights import descs_for, model_cache, synth_model

pytestmark = pytest.mark.gpu
MIB = 1 << 20

# (name, reduced KV shape keeping the model's layer count, weights (h, L, ff, V, arch), KV blocks)
MODELS3 = [
    ("qwen-1.8b", KVShape(24, 2, 64, 2, 16), dict(h=128, L=24, ff=256, V=2048, arch="qwen1"), 17),
    ("llama-7b", KVShape(32, 4, 64, 2, 16), dict(h=128, L=32, ff=384, V=2048, arch="llama"), 11),
    ("yi-9b", KVShape(48, 1, 128, 2, 16), dict(h=128, L=48, ff=256, V=3072, arch="llama"), 15),
]
WPOISON = gi.poison_key(gi.TAG_NEVER, 8 * 7)


def _align(x):
    return -(-x // 256) * 256


@pytest.mark.parametrize("mode", ["staged", "prefetch"])
def test_three_model_switch_matches_oracle(mode):
    require_gpu()
    import torch
    cfg = aeg.default_config(device_kv_bytes=40 * MIB, host_kv_bytes=40 * MIB, dev_slab_bytes=MIB,
                             host_slab_bytes=MIB, dev_slab_layout=aeg.LAYER_MAJOR,
                             host_slab_layout=aeg.BLOCK_MAJOR, staging_slot_bytes=MIB, staging_slots=3,
                             stage_ring_bytes=4 * MIB, stage_chunk_bytes=MIB, device_weight_bytes=64 * MIB,
                             table_arena_bytes=4 * MIB, host_threads=4, kernel=aeg.KERNEL_AUTO)
    ctx = aeg.Context(0, cfg)
    dev = Side(ctx, aeg.POOL_DEVICE, cfg.device_kv_bytes, cfg.dev_slab_bytes, aeg.LAYER_MAJOR)
    host = Side(ctx, aeg.POOL_HOST, cfg.host_kv_bytes, cfg.host_slab_bytes, aeg.BLOCK_MAJOR)
    try:
        dev.poison(gi.TAG_NEVER)
        host.poison(gi.TAG_NEVER)
        dimg, himg = dev.poison_img(gi.TAG_NEVER), host.poison_img(gi.TAG_NEVER)
        wbase, wbytes, _ = ctx.weights_region()
        D.fill_region(wbase, wbytes, SEED, WPOISON)
        wimg = gi.region_bytes(SEED, WPOISON, wbytes)
        # Model Caches (pageable host memory, generated content) and each model's decode KV, resident
        # in the host pool before the first switch
        models = []
        for m, (name, sh, wk, nb) in enumerate(MODELS3):
            descs = synth_model(**wk)
            buf, tens = model_cache(descs, m=20 + m)
            hc, ho = host.alloc(sh, nb)
            fill_blocks(host, himg, sh, ho, [(m, j) for j in range(nb)], m=m + 1)
            models.append(dict(name=name, sh=sh, descs=descs, buf=buf, tens=tens, n=nb, where="host",
                               c=hc, o=ho, size=None))
        ctx.trace_enable(True)
        cons = torch.cuda.Stream()
        pre = None                            # prefetch mode: (model index, xfer, its offset, offsets)

        def stage_oracle(img, k, base):
            M = models[k]
            return W.stage(M["tens"], M["descs"], 0, 1, region_bytes=wbytes, base=base, dst=img)

        def bring_in(b, a):
            """Switch a -> b (a None: cold start).  Returns the oracle's expectations updated."""
            nonlocal dimg, himg, wimg, pre
            B = models[b]
            A = models[a] if a is not None else None
            if A is not None:                 # A's KV-out destination, allocated before anything is enqueued
                ha_c, ha_o = host.alloc(A["sh"], A["n"])
            db_c, db_o = dev.alloc(B["sh"], B["n"])
            ctx.stream_fence(cons.cuda_stream)
            xi = ctx.kv_swap_in(B["sh"].as_tuple(), B["c"], db_c, flags=aeg.FREE_SRC)      # B's KV first
            if mode == "staged" or pre is None:
                ctx.weights_reset(0)
                offs, xw = ctx.weights_stage(descs_for(B["tens"], B["descs"]))
                wimg, eoffs, end = stage_oracle(wimg, b, 0)
                assert [int(o) for o in offs] == eoffs
                B["size"] = end
            else:
                k, xp, poff, poffs = pre
                assert k == b
                ctx.layer_ready(xp, -1, aeg.READY_BLOCK)        # the prefetch landed during A's turn
                xw = ctx.weights_relocate(poff, 0, B["size"])
                ctx.xfer_release(xp)
                wimg = memmove(wimg, poff, 0, B["size"])
            nl = B["sh"].L
            wl = ctx.xfer_layers(xw)
            for l in range(nl):                # the decode consumer of B, layer by layer (rule ❶)
                ctx.layer_ready(xw, min(l, wl - 1), aeg.READY_WAIT_STREAM, cons.cuda_stream)
                ctx.layer_ready(xi, l, aeg.READY_WAIT_STREAM, cons.cuda_stream)
            ctx.layer_ready(xw, -1, aeg.READY_WAIT_STREAM, cons.cuda_stream)
            xo = None
            if A is not None:                  # A's KV out, fenced after B's consumer
                ctx.stream_fence(cons.cuda_stream)
                xo = ctx.kv_swap_out(A["sh"].as_tuple(), A["c"], ha_c, flags=aeg.FREE_SRC)
            # oracle, in the same order
            dimg = OK.swap_in(himg, host.geom, dimg, dev.geom, B["sh"], B["o"], db_o)
            xb = host.oracle.begin(B["o"])
            host.oracle.free(B["o"])
            if A is not None:
                himg = OK.swap_out(dimg, dev.geom, himg, host.geom, A["sh"], A["o"], ha_o)
                xa = dev.oracle.begin(A["o"])
                dev.oracle.free(A["o"])
            for x in (xi, xw, xo):
                if x is not None:
                    ctx.layer_ready(x, -1, aeg.READY_BLOCK)
                    ctx.xfer_release(x)
            host.oracle.complete(xb)
            if A is not None:
                dev.oracle.complete(xa)
                A.update(where="host", c=ha_c, o=ha_o)
            B.update(where="dev", c=db_c, o=db_o)
            if mode == "prefetch":             # prefetch the next model behind B during B's turn
                nxt = (b + 1) % len(models)
                poff = _align(B["size"])
                ctx.weights_reset(poff)
                offs, xp = ctx.weights_stage(descs_for(models[nxt]["tens"], models[nxt]["descs"]))
                wimg, eoffs, end = stage_oracle(wimg, nxt, poff)
                assert [int(o) for o in offs] == eoffs
                models[nxt]["size"] = end - poff
                pre = (nxt, xp, poff, offs)

        order = [0, 1, 2, 0, 1, 2]
        for i, b in enumerate(order):
            bring_in(b, order[i - 1] if i else None)
            if pre is not None:
                ctx.layer_ready(pre[1], -1, aeg.READY_BLOCK)
            assert first_diff(dev.read(), dimg) is None, f"device KV after switch {i}"
            assert first_diff(host.read(), himg) is None, f"host KV after switch {i}"
            assert first_diff(D.read(wbase, wbytes), wimg) is None, f"weights after switch {i}"
        if pre is not None:
            ctx.xfer_release(pre[1])
        assert check(parse_trace(ctx.trace_read()))
    finally:
        ctx.shutdown()
