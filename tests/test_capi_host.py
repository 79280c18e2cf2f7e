"""CPU tests of the C-ABI library: it loads, exports every symbol include/aeg.h declares, and its
slab allocator (host-only context, no CUDA) takes the same decisions as the oracle (O2), call by
call, over exhaustive short and random long operation sequences on both pools."""
import itertools
import random
import subprocess

import numpy as np
import pytest

import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg
from oracle.shape import KVShape
from oracle.slab import AllocError, SlabPool


@pytest.fixture(scope="module", autouse=True)
def built():
    from paper_conf_sosp_xiang0qyzyzl0025_b200 import build
    build.build()


def test_library_exports_every_declared_symbol():
    declared = aeg.declared_symbols()
    assert len(declared) >= 30
    out = subprocess.run(["nm", "-D", "--defined-only", aeg.LIB_PATH], capture_output=True, text=True).stdout
    exported = {line.split()[-1] for line in out.splitlines() if line.strip()}
    missing = [s for s in declared if s not in exported]
    assert not missing, missing
    L = aeg.lib()
    for s in declared:
        assert hasattr(L, s)
    # the binding covers the whole ABI
    assert set(declared) == set(aeg._SIGS) | {"aeg_last_error"}


def test_no_torch_in_abi():
    src = open(aeg.HEADER).read()
    assert "torch" not in src.replace("torch.distributed", "")
    assert "at::" not in src and "Tensor" not in src


A = (2, 1, 2, 2, 8)      # chunk 64 B, block 128 B
Bs = (3, 1, 2, 2, 8)     # block 192 B
SLAB = 256


def host_ctx(n_slabs=3, layout=aeg.LAYER_MAJOR, **kw):
    cfg = aeg.default_config(device_kv_bytes=n_slabs * SLAB, host_kv_bytes=n_slabs * SLAB, dev_slab_bytes=SLAB,
                             host_slab_bytes=SLAB, dev_slab_layout=layout, host_slab_layout=layout,
                             flags=aeg.CFG_HOST_ONLY | aeg.CFG_NO_DAEMON, **kw)
    return aeg.Context(0, cfg)


class Pair:
    """Runs the same operations on the oracle pool and on the library (both pools)."""

    def __init__(self, n_slabs, pool):
        self.o = SlabPool(n_slabs * SLAB, SLAB)
        self.c = host_ctx(n_slabs)
        self.pool = pool
        self.live, self.order, self.xfers = {}, [], []
        self.tag = 0

    def alloc(self, shape, n):
        o_err = c_err = None
        try:
            o = self.o.alloc(KVShape(*shape), n)
        except AllocError as e:
            o, o_err = None, e.code
        try:
            c = self.c.kv_alloc(self.pool, shape, n)
        except aeg.AegError as e:
            c, c_err = None, e.code
        assert o_err == c_err
        if o is not None:
            dec = [aeg.decode_block(b) for b in c]
            assert all(p == self.pool for p, _, _ in dec)
            assert [(s, j) for _, s, j in dec] == list(o)
            self.live[self.tag] = (o, c)
            self.order.append(self.tag)
        self.tag += 1

    def free(self, k):
        if not self.order:
            return
        t = self.order.pop(k)
        o, c = self.live.pop(t)
        self.o.free(o)
        self.c.kv_free(self.pool, c)

    def xfer(self, k):
        if not self.order:
            return
        o, c = self.live[self.order[k]]
        self.xfers.append((self.o.begin(o), self.c.debug_xfer_begin(self.pool, c)))

    def complete(self):
        if self.xfers:
            xo, xc = self.xfers.pop(0)
            self.o.complete(xo)
            self.c.debug_xfer_complete(xc)

    def reclaim(self):
        self.o.reclaim()
        self.c.reclaim()

    def compare_stats(self):
        per, free = self.o.stats()
        s = self.c.stats(self.pool)
        assert s.free_slabs == free
        got = {}
        for i in range(s.n_shapes):
            p = s.per_shape[i]
            sh = KVShape(p.shape.num_layers, p.shape.num_kv_heads, p.shape.head_dim, p.shape.elem_bytes,
                         p.shape.block_tokens)
            got[sh] = (p.slabs, p.owned_blocks, p.quarantined_blocks)
        assert got == per
        used = sum(v[1] * sh.block_bytes() for sh, v in per.items())
        assert s.used_bytes == used
        # Fig. 16's fragmentation (unused / peak allocated) from the library's own fields
        assert s.peak_assigned_bytes == self.o.peak_assigned
        frag = 0.0 if s.peak_assigned_bytes == 0 else (s.assigned_bytes - s.used_bytes) / s.peak_assigned_bytes
        assert frag == pytest.approx(self.o.fragmentation())

    def run(self, ops):
        for op in ops:
            getattr(self, op[0])(*op[1:])
            self.compare_stats()


OPS = [("alloc", A, 1), ("alloc", A, 2), ("alloc", A, 3), ("alloc", Bs, 1), ("alloc", Bs, 2),
       ("free", 0), ("free", -1), ("xfer", 0), ("complete",), ("reclaim",)]


@pytest.mark.parametrize("pool", [aeg.POOL_DEVICE, aeg.POOL_HOST])
def test_allocator_matches_oracle_exhaustive(pool):
    for seq in itertools.product(OPS, repeat=4):
        p = Pair(3, pool)
        p.run(seq)
        p.c.shutdown()


@pytest.mark.parametrize("seed", range(40))
def test_allocator_matches_oracle_random(seed):
    r = random.Random(seed)
    p = Pair(5, seed % 2)
    p.run([r.choice(OPS) for _ in range(120)])
    p.c.shutdown()


def test_error_codes_and_validation():
    c = host_ctx(2)
    b = c.kv_alloc(aeg.POOL_DEVICE, A, 2)
    with pytest.raises(aeg.AegError) as e:
        c.kv_free(aeg.POOL_HOST, b)                    # wrong pool
    assert e.value.code == aeg.ERR_INVALID
    with pytest.raises(aeg.AegError) as e:
        c.kv_free(aeg.POOL_DEVICE, [b[0], b[0]])        # repeated
    assert e.value.code == aeg.ERR_STATE
    c.kv_free(aeg.POOL_DEVICE, b)
    with pytest.raises(aeg.AegError) as e:
        c.kv_free(aeg.POOL_DEVICE, b)                   # double free (slab reclaimed -> invalid)
    assert e.value.code in (aeg.ERR_STATE, aeg.ERR_INVALID)
    with pytest.raises(aeg.AegError) as e:
        c.kv_alloc(aeg.POOL_DEVICE, (3, 2, 2, 2, 8), 1)  # block larger than a slab
    assert e.value.code == aeg.ERR_INVALID
    with pytest.raises(aeg.AegError) as e:
        c.kv_alloc(aeg.POOL_DEVICE, A, 100)
    assert e.value.code == aeg.ERR_OOM
    with pytest.raises(aeg.AegError) as e:
        c.kv_alloc(aeg.POOL_DEVICE, (0, 1, 2, 2, 8), 1)  # invalid shape
    assert e.value.code == aeg.ERR_INVALID
    with pytest.raises(aeg.AegError) as e:
        c.kv_swap_out(A, [], [])                         # no data path in host-only mode
    assert e.value.code == aeg.ERR_STATE
    assert "host-only" in aeg.lib().aeg_last_error().decode()
    assert len(c.kv_alloc(aeg.POOL_DEVICE, A, 0)) == 0
    with pytest.raises(aeg.AegError) as e:
        c.peer_region(3)                                 # never imported
    assert e.value.code == aeg.ERR_INVALID
    with pytest.raises(aeg.AegError) as e:
        c.kernel_stats(5)                                # kinds 0..4 (4 = block-table fetch)
    assert e.value.code == aeg.ERR_INVALID
    assert c.kernel_stats(aeg.K_FETCH)[0] == 0
    cfg = aeg.default_config()
    assert cfg.dma_piece_mib == 128                      # sub-layer D2H pieces on by default
    assert cfg.pack_layer_mib == 32                      # layers < 32 MiB share a staging segment
    assert cfg.device_kv_bytes == 0                      # sized at init: 90 % of free VRAM (reading 22)
    c.shutdown()


@pytest.mark.parametrize("layout", [aeg.LAYER_MAJOR, aeg.BLOCK_MAJOR])
def test_block_offsets_match_oracle_addr(layout):
    """aeg_block_offsets (the consumer's block table) places every layer of every block exactly where
    the oracle's address function (O3 geometry) does, for both slab layouts."""
    from oracle import kv as OK
    slab = 1 << 20
    c = host_ctx(8, layout)
    c.shutdown()
    cfg = aeg.default_config(device_kv_bytes=8 * slab, host_kv_bytes=8 * slab, dev_slab_bytes=slab,
                             host_slab_bytes=slab, dev_slab_layout=layout, host_slab_layout=layout,
                             flags=aeg.CFG_HOST_ONLY | aeg.CFG_NO_DAEMON)
    c = aeg.Context(0, cfg)
    sh = KVShape(3, 2, 64, 2, 16)
    blocks = np.concatenate([c.kv_alloc(0, sh.as_tuple(), 37), c.kv_alloc(0, sh.as_tuple(), 5)])
    off0, stride = c.block_offsets(0, sh.as_tuple(), blocks)
    g = OK.PoolGeom(8 * slab, slab, layout)
    for b, o in zip(blocks, off0):
        h = aeg.decode_block(b)[1:]
        for l in range(sh.L):
            assert int(o) + l * stride == OK.addr(g, sh, h, l)
    c.shutdown()


def test_block_offsets_errors_stats_peaks_and_free_after():
    c = host_ctx(3)
    try:
        a = c.kv_alloc(0, A, 3)
        with pytest.raises(aeg.AegError) as e:
            c.block_offsets(0, Bs, a)                     # another shape
        assert e.value.code == aeg.ERR_INVALID
        b = c.kv_alloc(0, Bs, 1)
        c.kv_free(0, b)
        with pytest.raises(aeg.AegError) as e:
            c.block_offsets(0, A, [a[0], b[0]])           # b is no longer owned (slab reclaimed)
        assert e.value.code in (aeg.ERR_STATE, aeg.ERR_INVALID)
        s = c.stats(0)
        assert s.peak_used_bytes >= s.used_bytes and s.peak_assigned_bytes >= s.assigned_bytes
        assert s.peak_assigned_bytes == 3 * SLAB             # A used 2 slabs, Bs one more at the peak
        # aeg_kv_free_after: blocks stay in the move list until the named transfer completes (❸)
        x = c.debug_xfer_begin(0, a[:1])
        c.kv_free_after(0, a, x)
        assert c.stats(0).quarantined_blocks == 3
        c.reclaim()
        assert c.stats(0).quarantined_blocks == 3
        c.debug_xfer_complete(x)
        c.reclaim()
        s = c.stats(0)
        assert s.quarantined_blocks == 0 and s.free_slabs == 3
        assert aeg.default_config().numa_node == 0           # default: the GPU's NUMA node
    finally:
        c.shutdown()


def test_daemon_reclaims_move_list():
    """With the daemon running, a move-list block is reclaimed without an explicit aeg_reclaim."""
    import time
    cfg = aeg.default_config(device_kv_bytes=2 * SLAB, host_kv_bytes=SLAB, dev_slab_bytes=SLAB,
                             host_slab_bytes=SLAB, flags=aeg.CFG_HOST_ONLY)
    c = aeg.Context(0, cfg)
    b = c.kv_alloc(aeg.POOL_DEVICE, A, 2)
    x = c.debug_xfer_begin(aeg.POOL_DEVICE, b)
    c.kv_free(aeg.POOL_DEVICE, b)
    assert c.stats(aeg.POOL_DEVICE).quarantined_blocks == 2
    c.debug_xfer_complete(x)
    for _ in range(200):
        if c.stats(aeg.POOL_DEVICE).quarantined_blocks == 0:
            break
        time.sleep(0.005)
    s = c.stats(aeg.POOL_DEVICE)
    assert s.quarantined_blocks == 0 and s.free_slabs == 2
    c.shutdown()


def test_big_pool_alloc_is_fast():
    """H1 control overhead: µs-scale per call even for thousands of blocks."""
    import time
    cfg = aeg.default_config(device_kv_bytes=160 << 30, host_kv_bytes=64 << 30, flags=aeg.CFG_HOST_ONLY | aeg.CFG_NO_DAEMON)
    c = aeg.Context(0, cfg)
    sh = (32, 32, 128, 2, 16)
    t0 = time.perf_counter()
    blocks = [c.kv_alloc(aeg.POOL_DEVICE, sh, 64) for _ in range(64)]
    dt = time.perf_counter() - t0
    assert dt < 0.5
    for b in blocks[::2]:
        c.kv_free(aeg.POOL_DEVICE, b)
    got = c.kv_alloc(aeg.POOL_DEVICE, sh, 1024)
    assert len(set(got.tolist())) == 1024
    c.shutdown()


def test_bench_allocator_leg_runs_on_a_host_only_context():
    """bench.py's H1 control-overhead leg needs no GPU (host-only context, C2 geometry, aged pool)."""
    import bench
    r = bench.allocator_leg(aeg, reps=2)
    assert r["per_request_alloc_us_p50"] > 0 and r["batch_alloc_ns_per_block"] > 0
    assert r["batch_free_us"] > 0 and "3970" in r["workload"]


def test_slab_size_must_keep_16_byte_alignment():
    """Every copy is 16-byte vectors or bulk copies: slab bases must stay 16-byte aligned."""
    for bad in (SLAB + 8, 1000):
        with pytest.raises(aeg.AegError) as e:
            aeg.Context(0, aeg.default_config(device_kv_bytes=3 * bad, host_kv_bytes=3 * SLAB, dev_slab_bytes=bad,
                                              host_slab_bytes=SLAB, flags=aeg.CFG_HOST_ONLY | aeg.CFG_NO_DAEMON))
        assert e.value.code == aeg.ERR_INVALID


def test_malformed_transfer_blobs_are_rejected():
    """aeg_xfer_import bounds the header before sizing the blob (no overflow on hostile values)."""
    import os
    import struct
    ctx = aeg.Context(0, aeg.default_config(device_kv_bytes=1 << 30, host_kv_bytes=1 << 30,
                                            flags=aeg.CFG_HOST_ONLY | aeg.CFG_NO_DAEMON))
    try:
        def blob(L, npiece, n, tail=0):
            head = struct.pack("<IiiiQiiQ", 0xAE6A1BC2, os.getpid(), L, 0, 1, npiece, n, 1)
            return head + bytes(tail)
        for L, npiece, n in ((2 ** 31 - 1, 0, 0), (-1, 0, 0), (4097, 0, 0), (2, 5, 2), (2, 2 ** 31 - 1, 2 ** 31 - 1 - 1),
                             (1, -3, 0), (1, 0, -1)):
            with pytest.raises(aeg.AegError, match="malformed"):
                ctx.xfer_import(0, blob(L, npiece, n, 4096))
        with pytest.raises(aeg.AegError, match="truncated"):
            ctx.xfer_import(0, blob(2, 0, 0, 64))          # needs 3 event handles
        with pytest.raises(aeg.AegError, match="not an aegkv"):
            ctx.xfer_import(0, b"\0" * 256)
    finally:
        ctx.shutdown()
