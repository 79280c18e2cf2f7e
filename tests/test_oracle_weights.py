"""Pins for O8 (oracle/weights.py): shards reassemble the tensor, TP=1 is the identity, shards of
different ranks are disjoint, bump offsets satisfy the bump-allocator properties
and the staged image reads back every (sharded) tensor at its offset."""
import numpy as np
import pytest

import aeg_inputs as gi
from oracle import weights as W


def tensor(rows, cols, seed, eb=2):
    return gi.region_bytes(seed, gi.weight_key(1, seed), rows * cols * eb).reshape(rows, cols * eb)


@pytest.mark.parametrize("tp", [1, 2, 4, 8])
@pytest.mark.parametrize("groups", [1, 3])
def test_col_shards_reassemble(tp, groups):
    rows, cols = 24 * groups, 5
    w = tensor(rows, cols, 3).reshape(rows, cols, 2)
    parts = [W.shard(w, W.COL, groups, r, tp) for r in range(tp)]
    # each group of rows is the concatenation of the ranks' group-slices, in rank order
    g_rows, per = rows // groups, rows // groups // tp
    for gi_ in range(groups):
        rebuilt = np.concatenate([p[gi_ * per:(gi_ + 1) * per] for p in parts], axis=0)
        assert np.array_equal(rebuilt, w[gi_ * g_rows:(gi_ + 1) * g_rows])
    assert sum(p.size for p in parts) == w.size


@pytest.mark.parametrize("tp", [1, 2, 4])
def test_row_and_vocab_and_replicated(tp):
    w = tensor(8, 16, 4).reshape(8, 16, 2)
    rows = [W.shard(w, W.ROW, 1, r, tp) for r in range(tp)]
    assert np.array_equal(np.concatenate(rows, axis=1), w)
    voc = [W.shard(w, W.VOCAB, 1, r, tp) for r in range(tp)]
    assert np.array_equal(np.concatenate(voc, axis=0), w)
    for r in range(tp):
        assert np.array_equal(W.shard(w, W.REPLICATED, 1, r, tp), w)
    if tp == 1:
        for split in (W.COL, W.ROW, W.VOCAB, W.REPLICATED):
            assert np.array_equal(W.shard(w, split, 1, 0, 1), w)


def test_non_divisible_is_invalid():
    w = np.zeros((6, 5, 2), np.uint8)
    with pytest.raises(W.WeightError):
        W.shard(w, W.COL, 1, 0, 4)
    with pytest.raises(W.WeightError):
        W.shard(w, W.ROW, 1, 0, 2)
    with pytest.raises(W.WeightError):
        W.shard(w, W.COL, 4, 0, 1)


def test_bump_offsets_properties():
    r = np.random.default_rng(5)
    sizes = [int(x) for x in r.integers(1, 5000, size=200)] + [256, 512, 1]
    base = 1024
    offs, end = W.bump_offsets(sizes, base)
    assert offs[0] == base
    for k, (o, n) in enumerate(zip(offs, sizes)):
        assert o % 256 == 0                                   # reading 17
        if k + 1 < len(offs):
            gap = offs[k + 1] - (o + n)
            assert 0 <= gap < 256                             # consecutive, no overlap, minimal pad
    assert end % 256 == 0 and 0 <= end - (offs[-1] + sizes[-1]) < 256
    # reset = pointer back to base: staging again reproduces the same offsets
    assert W.bump_offsets(sizes, base)[0] == offs


@pytest.mark.parametrize("tp", [1, 2, 4])
def test_stage_reads_back_and_ranks_cover_model(tp):
    descs = gi.model_tensors("tiny")
    tens = [tensor(d["rows"], d["cols"], k) for k, d in enumerate(descs)]
    total = sum(t.size for t in tens)
    got_bytes = 0
    for r in range(tp):
        img, offs, end = W.stage(tens, descs, r, tp, region_bytes=total + 256 * len(descs) + 4096, base=256)
        for t, d, o in zip(tens, descs, offs):
            sh = W.shard(t.reshape(d["rows"], d["cols"], 2), d["split"], d["groups"], r, tp)
            assert np.array_equal(img[o:o + sh.size], sh.reshape(-1))
            got_bytes += sh.size if d["split"] != W.REPLICATED or r == 0 else 0
        assert img[:256].sum() == 0                           # nothing below base
    assert got_bytes == total                                 # shards over ranks = the model


def test_region_exhausted():
    descs = gi.model_tensors("tiny")
    tens = [tensor(d["rows"], d["cols"], k) for k, d in enumerate(descs)]
    with pytest.raises(W.WeightError):
        W.stage(tens, descs, 0, 1, region_bytes=1 << 16)


def test_region_exact_fit_and_one_byte_over():
    """Reading 17's bump layout: the region must hold [base, off_last + size_last); an exact fit
    stages, one byte less raises (pins the boundary of the exhaustion check)."""
    descs = gi.model_tensors("tiny")
    tens = [tensor(d["rows"], d["cols"], k) for k, d in enumerate(descs)]
    sizes = [W.shard(t.reshape(d["rows"], d["cols"], 2), d["split"], d["groups"], 0, 1).size
             for t, d in zip(tens, descs)]
    base = 512
    p, last = base, base
    for n in sizes:                  # worked out independently of bump_offsets: align each start
        last = p
        p = (p + n + 255) // 256 * 256
    need = last + sizes[-1]
    img, offs, _ = W.stage(tens, descs, 0, 1, region_bytes=need, base=base)
    assert img.size == need and offs[-1] == last
    with pytest.raises(W.WeightError):
        W.stage(tens, descs, 0, 1, region_bytes=need - 1, base=base)


def test_row_split_has_no_groups():
    """Reading 18: `groups` cuts fused QKV-style tensors into row groups, so it applies to COL/VOCAB
    only; a ROW (strided column) split with groups > 1 is undefined and rejected."""
    w = np.zeros((6, 4, 2), np.uint8)
    with pytest.raises(W.WeightError):
        W.shard(w, W.ROW, 2, 0, 2)
    with pytest.raises(W.WeightError):
        W.shard(w, W.ROW, 3, 0, 1)


def test_stage_leaves_the_given_image_untouched():
    """stage() returns the new region image; the `dst` passed in (the previous image) is not written."""
    descs = [dict(rows=4, cols=8, split=W.REPLICATED, groups=1)]
    ts = [tensor(4, 8, 9)]
    before = np.full(4096, 0xAB, np.uint8)
    keep = before.copy()
    out, offs, _ = W.stage(ts, descs, 0, 1, 4096, dst=before)
    assert np.array_equal(before, keep)
    assert np.array_equal(out[:64], ts[0].reshape(-1)) and not out[64:256].any() and np.all(out[256:] == 0xAB)


def test_padding_after_every_shard_is_zero():
    """Reading 17: shards sit at 256-byte bump offsets and the padding up to the next
    offset (and after the last shard, up to the bump pointer) is written as zeros, whatever the
    region held before; bytes beyond the bump pointer are untouched."""
    descs = [dict(rows=3, cols=5, split=W.REPLICATED, groups=1), dict(rows=1, cols=7, split=W.REPLICATED, groups=1)]
    ts = [tensor(3, 5, 11), tensor(1, 7, 12)]
    before = np.full(2048, 0xCD, np.uint8)
    out, offs, end = W.stage(ts, descs, 0, 1, 2048, base=256, dst=before)
    assert offs == [256, 512] and end == 768                   # 30 B -> next at 512; 14 B -> bump 768
    assert np.array_equal(out[256:286], ts[0].reshape(-1)) and not out[286:512].any()
    assert np.array_equal(out[512:526], ts[1].reshape(-1)) and not out[526:768].any()
    assert np.all(out[:256] == 0xCD) and np.all(out[768:] == 0xCD)
