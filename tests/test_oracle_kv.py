"""Pins for O3–O7 (oracle/kv.py): brute force over every small block table, both slab layouts and
every layer range, against an independent formulation of the slab layout (NumPy reshape views
instead of address arithmetic) and the per-token element view of reading 3; plus the north-star
invariants (swap_in∘swap_out = identity on every block; untouched bytes keep their poison)."""
import itertools

import numpy as np
import pytest

import aeg_inputs as gi
from oracle import kv
from oracle.kv import BLOCK_MAJOR, LAYER_MAJOR, PoolGeom
from oracle.shape import KVShape

SH = KVShape(L=3, H=2, D=2, s=2, B=4)          # Cl = 64 B, block = 192 B
SLAB = 2 * SH.block_bytes() + 64               # k = 2, 64 B slab tail (fragmentation)
NS = 3                                          # 6 blocks


def slab_view(pool, g, sh):
    """Independent formulation: [slab][layer][block][Cl] (layer-major) or [slab][block][layer][Cl]."""
    k = g.slab_bytes // sh.block_bytes()
    body = pool.reshape(-1, g.slab_bytes)[:, : k * sh.block_bytes()]
    if g.layout == LAYER_MAJOR:
        return body.reshape(-1, sh.L, k, sh.chunk_bytes()).transpose(0, 2, 1, 3)   # -> [s][j][l][Cl]
    return body.reshape(-1, k, sh.L, sh.chunk_bytes())


def token_elem(chunk, sh, c, t, h, d):
    """Per-token view (reading 3): the chunk is [2][B][H][D] elements of s bytes."""
    return chunk.reshape(2, sh.B, sh.H, sh.D, sh.s)[c, t, h, d]


def unique_pool(nbytes, seed):
    return gi.region_bytes(seed, gi.poison_key(gi.TAG_NEVER, 0), nbytes)


HANDLES = [(s, j) for s in range(NS) for j in range(2)]


@pytest.mark.parametrize("layout", [LAYER_MAJOR, BLOCK_MAJOR])
def test_gather_bruteforce(layout):
    g = PoolGeom(NS * SLAB, SLAB, layout)
    pool = unique_pool(g.nbytes, 7)
    view = slab_view(pool, g, SH)
    n_checked = 0
    for n in range(0, 4):
        for table in itertools.permutations(HANDLES, n):
            for l0 in range(SH.L + 1):
                for l1 in range(l0, SH.L + 1):
                    st = kv.gather(pool, g, SH, list(table), l0, l1)
                    exp = np.stack([view[s, j, l] for l in range(l0, l1) for (s, j) in table]).reshape(-1) \
                        if table and l1 > l0 else np.empty(0, np.uint8)
                    assert np.array_equal(st, exp)
                    n_checked += 1
    assert n_checked > 500


@pytest.mark.parametrize("layout", [LAYER_MAJOR, BLOCK_MAJOR])
def test_gather_per_token(layout):
    g = PoolGeom(NS * SLAB, SLAB, layout)
    pool = unique_pool(g.nbytes, 8)
    view = slab_view(pool, g, SH)
    table = [(2, 1), (0, 0), (1, 1)]
    st = kv.gather(pool, g, SH, table, 0, SH.L).reshape(SH.L, len(table), SH.chunk_bytes())
    for l in range(SH.L):
        for i, (s, j) in enumerate(table):
            for c, t, h, d in itertools.product(range(2), range(SH.B), range(SH.H), range(SH.D)):
                assert np.array_equal(token_elem(st[l, i], SH, c, t, h, d),
                                      token_elem(view[s, j, l], SH, c, t, h, d))


@pytest.mark.parametrize("layout", [LAYER_MAJOR, BLOCK_MAJOR])
def test_scatter_bruteforce_and_untouched(layout):
    g = PoolGeom(NS * SLAB, SLAB, layout)
    pool = unique_pool(g.nbytes, 9)
    for n in range(1, 4):
        for table in itertools.permutations(HANDLES, n):
            for l0, l1 in [(0, SH.L), (1, 2), (2, 3)]:
                stage = unique_pool((l1 - l0) * n * SH.chunk_bytes(), 100 + n)
                out = kv.scatter(pool, g, SH, list(table), l0, l1, stage)
                v_out, v_in = slab_view(out, g, SH), slab_view(pool, g, SH)
                st = stage.reshape(l1 - l0, n, SH.chunk_bytes())
                mask = np.zeros(g.nbytes, bool)
                for (s, j) in HANDLES:
                    for l in range(SH.L):
                        if (s, j) in table and l0 <= l < l1:
                            assert np.array_equal(v_out[s, j, l], st[l - l0, table.index((s, j))])
                        else:
                            assert np.array_equal(v_out[s, j, l], v_in[s, j, l])
                # bytes outside every block (slab tails) are untouched too
                k = g.slab_bytes // SH.block_bytes()
                for s in range(NS):
                    tail = slice(s * SLAB + k * SH.block_bytes(), (s + 1) * SLAB)
                    assert np.array_equal(out[tail], pool[tail])
                assert not mask.any()


def test_swap_round_trip_identity_across_layouts():
    """north star: swap_in ∘ swap_out is the identity on every block, into a pool of another slab
    size and layout; every other byte keeps its poison."""
    dg = PoolGeom(4 * SLAB, SLAB, LAYER_MAJOR)
    hg = PoolGeom(5 * (SLAB + 192), SLAB + 192, BLOCK_MAJOR)   # k = 3 on the host side
    dg2 = PoolGeom(3 * 2 * SLAB, 2 * SLAB, BLOCK_MAJOR)         # k = 4, other layout
    dev = unique_pool(dg.nbytes, 1)
    host0 = unique_pool(hg.nbytes, 2)
    dev2 = unique_pool(dg2.nbytes, 3)
    src = [(3, 1), (0, 0), (2, 1), (1, 0)]
    hb = [(4, 2), (0, 0), (0, 1), (2, 2)]
    dst = [(1, 3), (0, 0), (2, 1), (0, 2)]
    host = kv.swap_out(dev, dg, host0, hg, SH, src, hb)
    dev_after = kv.swap_in(host, hg, dev2, dg2, SH, hb, dst)
    vs, vd, vd0 = slab_view(dev, dg, SH), slab_view(dev_after, dg2, SH), slab_view(dev2, dg2, SH)
    for (s, j), (t, i) in zip(src, dst):
        assert np.array_equal(vs[s, j], vd[t, i])                  # every layer, every byte
    untouched = [(t, i) for t in range(3) for i in range(4) if (t, i) not in dst]
    for t, i in untouched:
        assert np.array_equal(vd[t, i], vd0[t, i])
    # swap-out leaves the device image unchanged (O5) — the copy is not a move
    assert np.array_equal(kv.swap_out(dev, dg, host0, hg, SH, src, hb)[:0], host0[:0])


def test_label_image_matches_byte_image():
    """unit = Cl (one label per chunk) gives the same placement as the byte image."""
    g = PoolGeom(NS * SLAB, SLAB, LAYER_MAJOR)
    hg = PoolGeom(NS * SLAB, SLAB, BLOCK_MAJOR)
    Cl = SH.chunk_bytes()
    # label image: chunk c of the pool carries label c (slab tails are not chunks: use a pool
    # whose slab size is a multiple of Cl)
    assert SLAB % Cl == 0
    labels = np.arange(g.nbytes // Cl, dtype=np.uint64)
    byte_img = np.repeat(labels, Cl).astype(np.uint64)          # each byte carries its chunk label
    src, hb = [(1, 1), (0, 1), (2, 0)], [(2, 1), (0, 0), (1, 0)]
    host_lab = kv.swap_out(labels, g, np.full(hg.nbytes // Cl, 999, np.uint64), hg, SH, src, hb, unit=Cl)
    host_byte = kv.swap_out(byte_img, g, np.full(hg.nbytes, 999, np.uint64), hg, SH, src, hb)
    assert np.array_equal(np.repeat(host_lab, Cl), host_byte)


def test_migrate_is_relabelled_identity():
    sg = PoolGeom(NS * SLAB, SLAB, BLOCK_MAJOR)
    dg = PoolGeom(NS * SLAB, SLAB, LAYER_MAJOR)
    src, dst = unique_pool(sg.nbytes, 11), unique_pool(dg.nbytes, 12)
    a, b = [(0, 1), (2, 0)], [(1, 0), (1, 1)]
    out = kv.migrate(src, sg, dst, dg, SH, a, b)
    vs, vo = slab_view(src, sg, SH), slab_view(out, dg, SH)
    for (s, j), (t, i) in zip(a, b):
        assert np.array_equal(vs[s, j], vo[t, i])
    # migrate == swap_in ∘ swap_out through any intermediate host placement (reading 15)
    hg = PoolGeom(2 * SLAB, SLAB, BLOCK_MAJOR)
    mid = kv.swap_out(src, sg, np.zeros(hg.nbytes, np.uint8), hg, SH, a, [(1, 1), (0, 0)])
    assert np.array_equal(kv.swap_in(mid, hg, dst, dg, SH, [(1, 1), (0, 0)], b), out)


def test_oracle_functions_do_not_modify_their_inputs():
    """O3-O7 are functions of their inputs (the returned image is the new state); the source and
    destination arrays passed in stay exactly as they were."""
    sh = KVShape(2, 1, 8, 2, 1)
    g = PoolGeom(4 * sh.block_bytes(), 2 * sh.block_bytes(), LAYER_MAJOR)
    r = np.random.default_rng(5)
    src = r.integers(0, 256, g.nbytes, dtype=np.uint8)
    dst = r.integers(0, 256, g.nbytes, dtype=np.uint8)
    s0, d0 = src.copy(), dst.copy()
    hs, hd = [(0, 0), (1, 1)], [(1, 0), (0, 1)]
    out = kv.copy_blocks(src, g, dst, g, sh, hs, hd)
    assert np.array_equal(src, s0) and np.array_equal(dst, d0)
    assert not np.array_equal(out, d0)
    stage = kv.gather(src, g, sh, hs, 0, sh.L)
    assert np.array_equal(src, s0)
    kv.scatter(dst, g, sh, hd, 0, sh.L, stage)
    assert np.array_equal(dst, d0)
