"""configs[4] at full size on one GPU (the launch configuration bench.py times): one decode rank of
the Qwen-72B TP=4 scale-up stages its 36.1 GB weight shard from a 144.6 GB (sparse) host Model Cache
while its prefill partner's 2 GiB of KV is migrated into its pool.  Sampled tensors are compared with
the oracle's shard of the densely generated tensor (O8); every KV chunk is checked (O7)."""
import pytest

import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg

from .gpu_harness import require_gpu

pytestmark = pytest.mark.gpu


def _oracle_check(aeg_, ctx, name, m, seed, tp_rank, tp_size, got_offs, picks):
    """O8: bump offsets from the shard sizes, shard bytes = oracle shard of the dense tensor."""
    import numpy as np

    import aeg_inputs as gi
    from aeg_inputs import dev as D
    from oracle import weights as W
    ts = gi.model_tensors(name)
    sizes = [t["rows"] * t["cols"] * 2 // (1 if t["split"] == W.REPLICATED else tp_size) for t in ts]
    exp_offs, _ = W.bump_offsets(sizes, 0)
    assert [int(o) for o in got_offs] == exp_offs
    base, _, _ = ctx.weights_region()
    bad = 0
    for k in picks:
        t = ts[k]
        full = gi.region_bytes(seed, gi.weight_key(m, k), t["rows"] * t["cols"] * 2).reshape(t["rows"], t["cols"], 2)
        exp = np.ascontiguousarray(W.shard(full, t["split"], t["groups"], tp_rank, tp_size)).reshape(-1)
        bad += int((D.read(base + exp_offs[k], exp.size) != exp).sum())
    return bad == 0, len(picks)


def test_c5_one_rank_pair_full_size():
    require_gpu()
    import torch
    import bench
    r = bench.c5_leg(aeg, torch, aeg.KERNEL_AUTO, reps=1, check=_oracle_check)
    assert r["shard_bytes_per_rank"] > 36_000_000_000
    assert r["weights_bit_exact_sample"] and r["weights_tensors_checked"] >= 10, r
    assert r["kv_bit_exact"], r
