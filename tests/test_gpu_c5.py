"""configs[4] at full size on one GPU (the launch configuration bench.py times): one decode rank of
the Qwen-72B TP=4 scale-up stages its 36.1 GB weight shard from a 144.6 GB (sparse) host Model Cache
while its prefill partner's 2 GiB of KV is migrated into its pool.  Sampled tensors are compared with
the oracle's shard of the densely generated tensor (O8); every KV chunk is checked (O7)."""
import pytest

import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg

from .gpu_harness import require_gpu

pytestmark = pytest.mark.gpu


def test_c5_one_rank_pair_full_size():
    require_gpu()
    import torch
    import bench
    r = bench.c5_leg(aeg, torch, aeg.KERNEL_AUTO, reps=1)
    assert r["shard_bytes_per_rank"] > 36_000_000_000
    assert r["weights_bit_exact_sample"] and r["weights_tensors_checked"] >= 10, r
    assert r["kv_bit_exact"], r
