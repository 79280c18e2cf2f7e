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
