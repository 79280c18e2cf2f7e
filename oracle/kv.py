"""O3–O7 — KV block copies as plain byte definitions.  TEST INFRASTRUCTURE ONLY.

What the hot path computes (BASELINE.json north_star; §5.2-§5.3, Fig. 10 "memcpy(async)"
steps ② ⑤): the non-contiguous KV blocks named by a block table are gathered into a contiguous
staging image (O3), scattered from one into freshly allocated blocks (O4), swapped out to the
unified CPU cache (O5, P->C), swapped in (O6, C->D) and handed prefill->decode (O7).  Every
operation is a byte copy, so the oracle is that copy written out chunk by chunk.

Geometry (SURVEY.md §8 "Shared definitions"; readings 2, 4, 5): a pool is cut into slabs of S
bytes; a slab assigned shape σ holds k = floor(S / block_bytes) blocks.
  layer-major  addr(s, j, l) = s*S + l*k*Cl + j*Cl
  block-major  addr(s, j, l) = s*S + j*L*Cl + l*Cl
Staging image of n blocks over layers [l0, l1): stage[((l - l0)*n + i)*Cl + b].

``unit``: every function works on an array whose elements stand for ``unit`` bytes (1 for a
byte image; Cl for an image of per-chunk labels).  All offsets are multiples of ``unit``.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

from .shape import KVShape

LAYER_MAJOR, BLOCK_MAJOR = 0, 1


@dataclass(frozen=True)
class PoolGeom:
    nbytes: int
    slab_bytes: int
    layout: int = LAYER_MAJOR


def addr(g: PoolGeom, sh: KVShape, h, l: int) -> int:
    """Byte offset of layer l of block h = (slab s, index j) in pool g."""
    s, j = h
    Cl, L = sh.chunk_bytes(), sh.L
    k = g.slab_bytes // sh.block_bytes()
    assert 0 <= j < k and 0 <= l < L
    if g.layout == LAYER_MAJOR:
        return s * g.slab_bytes + l * k * Cl + j * Cl
    return s * g.slab_bytes + j * L * Cl + l * Cl


def _c(sh: KVShape, unit: int) -> int:
    assert sh.chunk_bytes() % unit == 0
    return sh.chunk_bytes() // unit


def gather(pool, g: PoolGeom, sh: KVShape, handles, l0: int, l1: int, unit: int = 1):
    """O3: stage[((l-l0)*n+i)*Cl + b] = pool[addr(h_i, l) + b]."""
    n, c = len(handles), _c(sh, unit)
    stage = np.empty((l1 - l0) * n * c, dtype=pool.dtype)
    for l in range(l0, l1):
        for i, h in enumerate(handles):
            a = addr(g, sh, h, l) // unit
            d = ((l - l0) * n + i) * c
            stage[d:d + c] = pool[a:a + c]
    return stage


def scatter(pool, g: PoolGeom, sh: KVShape, handles, l0: int, l1: int, stage, unit: int = 1):
    """O4: pool'[addr(h'_i, l) + b] = stage[((l-l0)*n+i)*Cl + b]; every other byte unchanged."""
    out = pool.copy()
    n, c = len(handles), _c(sh, unit)
    for l in range(l0, l1):
        for i, h in enumerate(handles):
            a = addr(g, sh, h, l) // unit
            d = ((l - l0) * n + i) * c
            out[a:a + c] = stage[d:d + c]
    return out


def copy_blocks(src, sg: PoolGeom, dst, dg: PoolGeom, sh: KVShape, src_handles, dst_handles,
                l0: int = 0, l1: int | None = None, unit: int = 1):
    """dst'[addr_d(h'_i, l) + b] = src[addr_s(h_i, l) + b] for all i, l in [l0, l1), b < Cl."""
    assert len(src_handles) == len(dst_handles)
    l1 = sh.L if l1 is None else l1
    out = dst.copy()
    c = _c(sh, unit)
    for l in range(l0, l1):
        for hs, hd in zip(src_handles, dst_handles):
            a, b = addr(sg, sh, hs, l) // unit, addr(dg, sh, hd, l) // unit
            out[b:b + c] = src[a:a + c]
    return out


def swap_out(dev, dg, host, hg, sh, dev_handles, host_handles, unit=1):
    """O5 (P->C, Fig. 10 step ②): host[addr_H(g_i, l) + b] = dev[addr_D(h_i, l) + b]; the
    device image is unchanged."""
    return copy_blocks(dev, dg, host, hg, sh, dev_handles, host_handles, unit=unit)


def swap_in(host, hg, dev, dg, sh, host_handles, dev_handles, unit=1):
    """O6 (C->D, Fig. 10 step ⑤): dev'[addr_D'(h'_i, l) + b] = host[addr_H(g_i, l) + b]."""
    return copy_blocks(host, hg, dev, dg, sh, host_handles, dev_handles, unit=unit)


def migrate(src, sg, dst, dg, sh, src_handles, dst_handles, unit=1):
    """O7 (prefill->decode hand-off; the paper's P->C->D route composed, reading 15)."""
    return copy_blocks(src, sg, dst, dg, sh, src_handles, dst_handles, unit=unit)
