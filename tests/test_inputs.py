"""The seeded input generator (aeg_inputs): published splitmix64 outputs, determinism, recipe sizes."""
import numpy as np

import aeg_inputs as gi


def test_splitmix64_published_sequence():
    # splitmix64 seeded with 0 (Vigna's reference generator): state += golden; out = mix(state).
    # Our words(seed=0, key=k) = mix(k + golden) are those outputs for k = 0, golden, 2*golden.
    gold = 0x9E3779B97F4A7C15
    keys = np.array([0, gold, (2 * gold) & gi.M64], dtype=np.uint64)
    out = gi.splitmix64(keys)
    assert int(out[0]) == 0xE220A8397B1DCDAF
    assert int(out[1]) == 0x6E789E6AA1B965F4
    assert int(out[2]) == 0x06C45D188009454F


def test_words_are_keyed_and_deterministic():
    a = gi.words(5, gi.kv_key(1, 2, 3, 4), 100)
    b = gi.words(5, gi.kv_key(1, 2, 3, 4), 100)
    c = gi.words(5, gi.kv_key(1, 2, 3, 5), 100)
    assert np.array_equal(a, b) and not np.array_equal(a, c)
    assert np.array_equal(gi.words(5, gi.kv_key(1, 2, 3, 4), 10, first=90), a[90:])
    assert len(set(a.tolist())) == 100


def test_request_lengths_recipes():
    c1 = gi.request_lengths(1, 8, 1, 256, forced=(1, 16, 17, 255, 256))
    assert c1[:5] == [1, 16, 17, 255, 256] and all(1 <= x <= 256 for x in c1)
    c2 = gi.request_lengths(2, 64, 256, 1792)
    assert all(256 <= x <= 1792 for x in c2)
    assert 50_000 < sum(c2) < 80_000          # E = 65,536 tokens
    assert c2 == gi.request_lengths(2, 64, 256, 1792)


def test_model_recipe_sizes():
    # SURVEY §8 H7 sizes (bf16, public HF configs)
    exp = {"qwen-1.8b": 3.67e9, "llama-7b": 13.48e9, "yi-9b": 17.66e9, "qwen-7b": 15.44e9,
           "llama-2-13b": 26.03e9, "qwen-72b": 144.57e9}
    for name, b in exp.items():
        assert abs(gi.model_bytes(name) - b) / b < 0.003, name


def test_churn_ops_shape():
    ops = gi.churn_ops(2, 1000)
    allocs = [o for o in ops if o[0] == "alloc"]
    frees = [o for o in ops if o[0] == "free"]
    assert sum(n for _, n in allocs) <= 900
    assert len(frees) == len(allocs) // 2


def test_host_fill_matches_numpy_and_2d_matches_dense():
    from aeg_inputs import dev as D
    dense = np.zeros(64 * 48, dtype=np.uint8)
    D.host_fill(dense, 9, 1234, threads=3)
    assert np.array_equal(dense, gi.region_bytes(9, 1234, dense.size))
    part = np.zeros_like(dense)
    D.host_fill_2d(part.ctypes.data + 16, 64, 48, 24, 9, 1234 + 2, threads=4)
    m = np.zeros((64, 48), bool)
    m[:, 16:40] = True
    assert np.array_equal(part.reshape(64, 48)[m], dense.reshape(64, 48)[m])
    assert not part.reshape(64, 48)[~m].any()


def test_sparse_model_cache_materialises_exactly_one_shard():
    """bench.sparse_model_cache (configs[4] host cache): rank r's shard bytes equal the dense cache's,
    every other byte is untouched (zero), checked through the oracle's shard rule (O8)."""
    import bench
    from oracle import weights as W
    dense_descs, dense_caches = bench.model_caches(["tiny"])
    dense = dense_caches["tiny"]
    for r in range(2):
        descs, keep, touched = bench.sparse_model_cache("tiny", 0, r, 2, gi.w_seed(3), min_sparse=0)
        buf = keep[1]
        assert buf.size == dense.size
        tot = 0
        for d, dd in zip(descs, dense_descs["tiny"]):
            o = d["host_src"] - buf.ctypes.data
            n = d["rows"] * d["cols"] * 2
            got = buf[o:o + n].reshape(d["rows"], d["cols"], 2)
            exp = dense[o:o + n].reshape(d["rows"], d["cols"], 2)
            gs = W.shard(got, d["split"], d["groups"], r, 2)
            assert np.array_equal(gs, W.shard(exp, d["split"], d["groups"], r, 2))
            tot += gs.size
        assert int(np.count_nonzero(buf)) <= tot == touched
