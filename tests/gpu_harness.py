"""Helpers shared by the GPU parity tests.

Division of labour (task rule ③): the CUDA library under test (libaegkv via the binding) only
executes the calls; every expected byte comes from the oracle (oracle/*) applied to inputs made by
the seeded generator (aeg_inputs).  Placement of input content and of expected content uses the
oracle's own address function (oracle.kv.addr) on the oracle allocator's handles, which are first
checked to equal the library's handles.  The library's pool base pointers are the only thing read
from it besides the results.
"""
from __future__ import annotations

import numpy as np

import aeg_inputs as gi
import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg
from aeg_inputs import dev as D
from oracle import kv as OK
from oracle.shape import KVShape
from oracle.slab import SlabPool

SEED = gi.kv_seed(1)


def require_gpu():
    import pytest
    try:
        import torch
    except Exception:  # pragma: no cover
        pytest.fail("torch missing")
    if not torch.cuda.is_available():
        pytest.fail("GPU test selected but no CUDA device is visible (no CPU fallback exists)")


class Side:
    """One pool seen by both the library and the oracle."""

    def __init__(self, ctx, pool, nbytes, slab, layout):
        self.ctx, self.pool = ctx, pool
        self.geom = OK.PoolGeom(nbytes, slab, layout)
        self.oracle = SlabPool(nbytes, slab)
        self.base, n = ctx.pool_region(pool)
        assert n == nbytes

    def alloc(self, sh: KVShape, n: int):
        c = self.ctx.kv_alloc(self.pool, sh.as_tuple(), n)
        o = self.oracle.alloc(sh, n)
        assert [(s, j) for _, s, j in map(aeg.decode_block, c)] == list(o), "allocator diverged from oracle"
        return c, o

    def free(self, c, o):
        self.ctx.kv_free(self.pool, c)
        self.oracle.free(o)

    def offsets(self, sh, handles, layers=None):
        layers = range(sh.L) if layers is None else layers
        return [OK.addr(self.geom, sh, h, l) for h in handles for l in layers]

    def poison(self, tag):
        D.fill_region(self.base, self.geom.nbytes, SEED, gi.poison_key(tag, 0))

    def poison_img(self, tag):
        return gi.region_bytes(SEED, gi.poison_key(tag, 0), self.geom.nbytes)

    def read(self):
        return D.read(self.base, self.geom.nbytes)


def fill_blocks(side: Side, img: np.ndarray, sh: KVShape, handles, labels, m=1):
    """Write KV content key kv_key(m, r, j, l) into every layer chunk of each block — on the device
    (CUDA generator) and into the oracle's byte image (NumPy generator)."""
    offs, keys = [], []
    for h, (r, j) in zip(handles, labels):
        for l in range(sh.L):
            o = OK.addr(side.geom, sh, h, l)
            k = gi.kv_key(m, r, j, l)
            offs.append(o)
            keys.append(k)
            img[o:o + sh.chunk_bytes()] = gi.region_bytes(SEED, k, sh.chunk_bytes())
    D.fill_chunks(side.base, offs, keys, sh.chunk_bytes(), SEED)


def poison_blocks(side: Side, img: np.ndarray, sh: KVShape, handles, tag=gi.TAG_DST):
    offs, keys = [], []
    for h in handles:
        for l in range(sh.L):
            o = OK.addr(side.geom, sh, h, l)
            offs.append(o)
            keys.append(gi.poison_key(tag, o))
            img[o:o + sh.chunk_bytes()] = gi.region_bytes(SEED, gi.poison_key(tag, o), sh.chunk_bytes())
    D.fill_chunks(side.base, offs, keys, sh.chunk_bytes(), SEED)


def first_diff(a: np.ndarray, b: np.ndarray):
    d = np.nonzero(a != b)[0]
    return None if d.size == 0 else (int(d[0]), int(d.size))
