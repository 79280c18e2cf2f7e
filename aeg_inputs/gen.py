"""Seeded synthetic inputs (see package docstring).  No method arithmetic lives here.

Recipe (DESIGN.md §"Input recipe"):
* lengths / churn / placement: ``numpy.random.Generator(PCG64(1000 + cfg))``;
* content: word ``w`` of a region whose key base is ``K`` is ``splitmix64(seed ^ (K + w))``
  (little-endian uint64 words; a region of ``nbytes`` is the first ``nbytes`` bytes of that
  word stream).  KV seed = ``0xAE6A0000 + cfg``, weight seed = ``0xAE6A1000 + cfg``.
* KV chunk keys: ``kv_key(m, r, j, l)`` packs model / request / logical block / layer into the
  high 44 bits; the low 20 bits count words inside the chunk.  Poison keys tag a byte region by
  its absolute offset: ``poison_key(tag, off) = (tag << 60) + off // 8`` with tag 14 for
  never-allocated bytes and 15 for pre-poisoned destination blocks.
"""
from __future__ import annotations

import numpy as np

M64 = (1 << 64) - 1
GOLDEN = 0x9E3779B97F4A7C15

KV_SEED_BASE = 0xAE6A0000
W_SEED_BASE = 0xAE6A1000
TAG_NEVER = 14
TAG_DST = 15


def kv_seed(cfg: int) -> int:
    return KV_SEED_BASE + cfg


def w_seed(cfg: int) -> int:
    return W_SEED_BASE + cfg


def rng(cfg: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(1000 + cfg))


# ----------------------------------------------------------------------------- content generator

def splitmix64(x):
    """splitmix64 finaliser applied to (x + golden); vectorised over uint64 arrays."""
    x = np.asarray(x, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = x + np.uint64(GOLDEN)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        return z ^ (z >> np.uint64(31))


def words(seed: int, key_base: int, nwords: int, first: int = 0) -> np.ndarray:
    """Words [first, first+nwords) of the stream with key base ``key_base``."""
    with np.errstate(over="ignore"):
        k = np.uint64(key_base & M64) + np.arange(first, first + nwords, dtype=np.uint64)
    return splitmix64(np.uint64(seed & M64) ^ k)


def region_bytes(seed: int, key_base: int, nbytes: int) -> np.ndarray:
    """First ``nbytes`` bytes of the stream with key base ``key_base`` as uint8."""
    nw = (nbytes + 7) // 8
    return words(seed, key_base, nw).view(np.uint8)[:nbytes].copy()


def kv_key(m: int, r: int, j: int, l: int) -> int:
    """Key base of KV chunk (model m, request r, logical block j, layer l)."""
    assert 0 <= m < 16 and 0 <= r < (1 << 16) and 0 <= j < (1 << 16) and 0 <= l < 256
    return (m << 60) | (r << 44) | (j << 28) | (l << 20)


def poison_key(tag: int, offset: int) -> int:
    assert offset % 8 == 0 and offset < (1 << 59)
    return (tag << 60) + offset // 8


def weight_key(m: int, k: int) -> int:
    """Key base of tensor k of model m (word index in the low 40 bits)."""
    assert 0 <= m < 256 and 0 <= k < (1 << 16)
    return (m << 56) | (k << 40)


# ----------------------------------------------------------------------------- workloads

def request_lengths(cfg: int, n: int, lo: int, hi: int, forced=()) -> list[int]:
    """n prompt/context lengths from U[lo, hi]; ``forced`` values come first."""
    g = rng(cfg)
    rest = g.integers(lo, hi + 1, size=n - len(forced)).tolist()
    return [int(x) for x in forced] + [int(x) for x in rest]


def churn_ops(cfg: int, capacity_blocks: int, fill: float = 0.9, free_frac: float = 0.5,
              lo_blocks: int = 1, hi_blocks: int = 64):
    """Aging sequence: ('alloc', n) until ~fill*capacity, then ('free', idx) for a random
    ``free_frac`` of the allocations (idx = allocation ordinal)."""
    g = np.random.Generator(np.random.PCG64(2000 + cfg))
    ops, used, sizes = [], 0, []
    while True:
        n = int(g.integers(lo_blocks, hi_blocks + 1))
        if used + n > fill * capacity_blocks:
            break
        ops.append(("alloc", n))
        sizes.append(n)
        used += n
    order = g.permutation(len(sizes))[: int(len(sizes) * free_frac)]
    ops += [("free", int(i)) for i in sorted(order.tolist())]
    return ops


# KV shapes (L layers, H kv heads per rank, D head dim, s bytes, B tokens/block).  Table 1 of
# PAPER.md:1120-1128 fixes Qwen-7B / LLaMA-13B / Qwen-72B / InternLM2.5-7B; the rest are public
# HF configs (sizes only, content is synthetic).
KV_SHAPES = {
    "tiny": (2, 4, 64, 2, 16),
    "qwen-7b": (32, 32, 128, 2, 16),
    "internlm2.5-7b": (32, 8, 128, 2, 16),
    "llama-7b": (32, 32, 128, 2, 16),
    "llama-2-13b": (40, 40, 128, 2, 16),
    "qwen-1.8b": (24, 16, 128, 2, 16),
    "yi-9b": (48, 4, 128, 2, 16),
    "yi-9b-tp4": (48, 1, 128, 2, 16),       # one KV head per rank: 8 KiB chunks
    "qwen-72b": (80, 64, 128, 2, 16),
    "qwen-72b-tp4": (80, 16, 128, 2, 16),
}

REPLICATED, COL, ROW, VOCAB = 0, 1, 2, 3

# (hidden, layers, ffn, vocab, kv_dim, arch) from public HF configs.  arch "qwen1": fused
# c_attn [3h, h] + bias, w1/w2 [ffn, h], mlp c_proj [h, ffn], untied lm_head.  arch "llama":
# q [h,h], k/v [kv_dim, h], o [h,h], gate/up [ffn, h], down [h, ffn], untied lm_head.
MODELS = {
    "qwen-1.8b": (2048, 24, 5504, 151936, 2048, "qwen1"),
    "qwen-7b": (4096, 32, 11008, 151936, 4096, "qwen1"),
    "qwen-72b": (8192, 80, 24576, 152064, 8192, "qwen1"),
    "llama-7b": (4096, 32, 11008, 32000, 4096, "llama"),
    "llama-2-13b": (5120, 40, 13824, 32000, 5120, "llama"),
    "yi-9b": (4096, 48, 11008, 64000, 512, "llama"),
    "tiny": (256, 2, 512, 1024, 256, "qwen1"),
}


def model_tensors(name: str):
    """Checkpoint tensor list: dicts(name, rows, cols, layer, split, groups).  ``layer`` is the
    weight-stage index: 0 = embedding, 1..L = decoder layers, L+1 = final norm + lm_head."""
    h, L, ff, V, kv, arch = MODELS[name]
    t = [dict(name="embed", rows=V, cols=h, layer=0, split=VOCAB, groups=1)]
    for i in range(L):
        p, li = f"layers.{i}.", i + 1
        t.append(dict(name=p + "ln1", rows=1, cols=h, layer=li, split=REPLICATED, groups=1))
        if arch == "qwen1":
            t.append(dict(name=p + "c_attn.w", rows=3 * h, cols=h, layer=li, split=COL, groups=3))
            t.append(dict(name=p + "c_attn.b", rows=3 * h, cols=1, layer=li, split=COL, groups=3))
            t.append(dict(name=p + "attn.c_proj", rows=h, cols=h, layer=li, split=ROW, groups=1))
            t.append(dict(name=p + "ln2", rows=1, cols=h, layer=li, split=REPLICATED, groups=1))
            t.append(dict(name=p + "w1", rows=ff, cols=h, layer=li, split=COL, groups=1))
            t.append(dict(name=p + "w2", rows=ff, cols=h, layer=li, split=COL, groups=1))
            t.append(dict(name=p + "mlp.c_proj", rows=h, cols=ff, layer=li, split=ROW, groups=1))
        else:
            t.append(dict(name=p + "q", rows=h, cols=h, layer=li, split=COL, groups=1))
            t.append(dict(name=p + "k", rows=kv, cols=h, layer=li, split=COL, groups=1))
            t.append(dict(name=p + "v", rows=kv, cols=h, layer=li, split=COL, groups=1))
            t.append(dict(name=p + "o", rows=h, cols=h, layer=li, split=ROW, groups=1))
            t.append(dict(name=p + "ln2", rows=1, cols=h, layer=li, split=REPLICATED, groups=1))
            t.append(dict(name=p + "gate", rows=ff, cols=h, layer=li, split=COL, groups=1))
            t.append(dict(name=p + "up", rows=ff, cols=h, layer=li, split=COL, groups=1))
            t.append(dict(name=p + "down", rows=h, cols=ff, layer=li, split=ROW, groups=1))
    t.append(dict(name="norm", rows=1, cols=h, layer=L + 1, split=REPLICATED, groups=1))
    t.append(dict(name="lm_head", rows=V, cols=h, layer=L + 1, split=VOCAB, groups=1))
    return t


def model_bytes(name: str, elem_bytes: int = 2) -> int:
    return sum(x["rows"] * x["cols"] * elem_bytes for x in model_tensors(name))
