"""aegkv — Python binding of libaegkv.so (include/aeg.h).

Argument marshalling only: every step of the data path runs inside the native library (C++ runtime
+ sm_100a kernels).  There is no CPU fallback: if the shared library is missing, importing the
binding raises ImportError-like AegError on first use.

Method names are the C-ABI names without the ``aeg_`` prefix (``Context.kv_swap_out`` ->
``aeg_kv_swap_out``).  Block handles are numpy uint64 arrays; streams are raw ``cudaStream_t``
integers (e.g. ``torch.cuda.current_stream().cuda_stream``).
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "lib", "libaegkv.so")
HEADER = os.path.join(os.path.dirname(_HERE), "include", "aeg.h")

POOL_DEVICE, POOL_HOST = 0, 1
LAYER_MAJOR, BLOCK_MAJOR = 0, 1
OK, NOT_READY, ERR_INVALID, ERR_OOM, ERR_CUDA, ERR_STATE = 0, 1, -1, -2, -3, -4
READY_QUERY, READY_WAIT_STREAM, READY_BLOCK = 0, 1, 2
FREE_SRC, NO_DEPS, IPC_EVENTS, MIGRATE_CE = 1, 2, 4, 8
SPLIT_REPLICATED, SPLIT_COL, SPLIT_ROW, SPLIT_VOCAB = 0, 1, 2, 3
CFG_HOST_ONLY, CFG_NO_DAEMON, CFG_TIMING, CFG_SHARED_HOST = 1, 2, 4, 8
KERNEL_AUTO, KERNEL_LSU, KERNEL_BULK, KERNEL_WARP, KERNEL_BULKW = 0, 1, 2, 3, 4
K_GATHER, K_SCATTER, K_MIGRATE, K_RELOCATE, K_FETCH = 0, 1, 2, 3, 4


class AegError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"aeg error {code}: {msg}")
        self.code = code


class KVShape(C.Structure):
    _fields_ = [("num_layers", C.c_int32), ("num_kv_heads", C.c_int32), ("head_dim", C.c_int32),
                ("elem_bytes", C.c_int32), ("block_tokens", C.c_int32)]

    @classmethod
    def of(cls, t):
        """From (L, H, D, s, B) or a KVShape."""
        if isinstance(t, KVShape):
            return t
        return cls(*[int(x) for x in t])

    def chunk_bytes(self):
        return self.block_tokens * 2 * self.num_kv_heads * self.head_dim * self.elem_bytes

    def block_bytes(self):
        return self.chunk_bytes() * self.num_layers


class Config(C.Structure):
    _fields_ = [("device_kv_bytes", C.c_uint64), ("device_weight_bytes", C.c_uint64),
                ("host_kv_bytes", C.c_uint64), ("dev_slab_bytes", C.c_uint64), ("host_slab_bytes", C.c_uint64),
                ("stage_ring_bytes", C.c_uint64), ("stage_chunk_bytes", C.c_uint64),
                ("staging_slot_bytes", C.c_uint64), ("table_arena_bytes", C.c_uint64),
                ("dev_slab_layout", C.c_int32), ("host_slab_layout", C.c_int32), ("staging_slots", C.c_int32),
                ("host_threads", C.c_int32), ("kernel", C.c_int32), ("migrate_ctas", C.c_int32),
                ("flags", C.c_uint32), ("numa_node", C.c_int32), ("dma_piece_mib", C.c_uint32),
                ("pack_layer_mib", C.c_uint32), ("reserved", C.c_uint32 * 4)]


class WeightDesc(C.Structure):
    _fields_ = [("host_src", C.c_void_p), ("rows", C.c_uint64), ("cols", C.c_uint64), ("elem_bytes", C.c_int32),
                ("layer", C.c_int32), ("split", C.c_int32), ("groups", C.c_int32)]


class ShapeStats(C.Structure):
    _fields_ = [("shape", KVShape), ("slabs", C.c_uint64), ("owned_blocks", C.c_uint64),
                ("quarantined_blocks", C.c_uint64)]


class PoolStats(C.Structure):
    _fields_ = [("pool_bytes", C.c_uint64), ("slab_bytes", C.c_uint64), ("n_slabs", C.c_uint64),
                ("free_slabs", C.c_uint64), ("owned_blocks", C.c_uint64), ("quarantined_blocks", C.c_uint64),
                ("used_bytes", C.c_uint64), ("assigned_bytes", C.c_uint64), ("peak_used_bytes", C.c_uint64),
                ("peak_assigned_bytes", C.c_uint64), ("n_shapes", C.c_int32), ("pad", C.c_int32),
                ("per_shape", ShapeStats * 16)]


_L = None
P, U64, I32, U32 = C.c_void_p, C.c_uint64, C.c_int32, C.c_uint32
PU64, PI32, PU32 = C.POINTER(C.c_uint64), C.POINTER(C.c_int32), C.POINTER(C.c_uint32)

_SIGS = {
    "aeg_config_default": [C.POINTER(Config)],
    "aeg_init": [C.c_int, C.POINTER(Config), C.POINTER(P)],
    "aeg_shutdown": [P],
    "aeg_kv_alloc": [P, I32, C.POINTER(KVShape), I32, PU64],
    "aeg_kv_free": [P, I32, PU64, I32],
    "aeg_reclaim": [P, C.c_int],
    "aeg_stats": [P, I32, C.POINTER(PoolStats)],
    "aeg_block_info": [P, U64, PI32, PU32, PU32],
    "aeg_block_ptr": [P, I32, C.POINTER(KVShape), U64, I32, C.POINTER(P)],
    "aeg_pool_region": [P, I32, C.POINTER(P), PU64],
    "aeg_peer_region": [P, I32, C.POINTER(P), PU64],
    "aeg_block_offsets": [P, I32, C.POINTER(KVShape), PU64, I32, PU64, PU64],
    "aeg_kv_swap_out": [P, C.POINTER(KVShape), PU64, PU64, I32, U32, PU64],
    "aeg_kv_swap_in": [P, C.POINTER(KVShape), PU64, PU64, I32, U32, PU64],
    "aeg_kv_migrate": [P, C.POINTER(KVShape), PU64, I32, PU64, I32, U32, PU64],
    "aeg_kv_swap_in_from": [P, C.POINTER(KVShape), I32, PU64, PU64, I32, U64, U32, PU64],
    "aeg_kv_free_after": [P, I32, PU64, I32, U64],
    "aeg_stream_fence": [P, P],
    "aeg_layer_ready": [P, U64, I32, I32, P],
    "aeg_xfer_layers": [P, U64, PI32],
    "aeg_xfer_release": [P, U64],
    "aeg_weights_stage": [P, C.POINTER(WeightDesc), I32, I32, I32, PU64, PU64],
    "aeg_weights_reset": [P, U64],
    "aeg_weights_region": [P, C.POINTER(P), PU64, PU64],
    "aeg_weights_relocate": [P, U64, U64, U64, PU64],
    "aeg_weights_stats": [P, PU64, C.POINTER(C.c_double), C.POINTER(C.c_double)],
    "aeg_host_register": [P, P, U64],
    "aeg_host_unregister": [P, P],
    "aeg_export_ipc": [P, P, PU64],
    "aeg_import_peer": [P, I32, P, U64],
    "aeg_xfer_export": [P, U64, P, PU64],
    "aeg_xfer_import": [P, I32, P, U64, PU64],
    "aeg_kernel_stats": [P, I32, PU64, PU64, C.POINTER(C.c_double)],
    "aeg_kernel_stats_reset": [P],
    "aeg_set_migrate_ctas": [P, C.c_int32],
    "aeg_trace_enable": [P, C.c_int],
    "aeg_trace_read": [P, C.c_char_p, PU64],
    "aeg_debug_xfer_begin": [P, I32, PU64, I32, PU64],
    "aeg_debug_xfer_complete": [P, U64],
}


def lib():
    """Load libaegkv.so (raises AegError if it has not been built — there is no fallback)."""
    global _L
    if _L is None:
        if not os.path.exists(LIB_PATH):
            raise AegError(ERR_STATE, f"{LIB_PATH} missing: run `python -m paper_conf_sosp_xiang0qyzyzl0025_b200.build`")
        L = C.CDLL(LIB_PATH)
        for name, args in _SIGS.items():
            f = getattr(L, name)
            f.argtypes = args
            f.restype = C.c_int
        L.aeg_last_error.restype = C.c_char_p
        L.aeg_last_error.argtypes = []
        _L = L
    return _L


def _chk(rc: int, allow_not_ready: bool = False) -> int:
    if rc < 0 or (rc == NOT_READY and not allow_not_ready):
        raise AegError(rc, lib().aeg_last_error().decode())
    return rc


def _blocks(a) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(a, dtype=np.uint64))


def _p64(a: np.ndarray):
    return a.ctypes.data_as(PU64)


def default_config(**kw) -> Config:
    c = Config()
    _chk(lib().aeg_config_default(C.byref(c)))
    for k, v in kw.items():
        setattr(c, k, v)
    return c


class Context:
    """One aeg_ctx (one process, one device)."""

    def __init__(self, device: int = 0, config: Config | None = None, **kw):
        self.cfg = config if config is not None else default_config(**kw)
        h = P()
        _chk(lib().aeg_init(int(device), C.byref(self.cfg), C.byref(h)))
        self.h = h

    # -- lifecycle
    def shutdown(self):
        if self.h:
            _chk(lib().aeg_shutdown(self.h))
            self.h = None

    close = shutdown

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.shutdown()

    def __del__(self):
        try:
            self.shutdown()
        except Exception:
            pass

    # -- H1
    def kv_alloc(self, pool: int, shape, n: int) -> np.ndarray:
        out = np.zeros(max(n, 1), dtype=np.uint64)
        sh = KVShape.of(shape)
        _chk(lib().aeg_kv_alloc(self.h, pool, C.byref(sh), int(n), _p64(out)))
        return out[:n]

    def kv_free(self, pool: int, blocks):
        b = _blocks(blocks)
        _chk(lib().aeg_kv_free(self.h, pool, _p64(b), int(b.size)))

    def reclaim(self, blocking: bool = False):
        _chk(lib().aeg_reclaim(self.h, int(blocking)))

    def stats(self, pool: int) -> PoolStats:
        s = PoolStats()
        _chk(lib().aeg_stats(self.h, pool, C.byref(s)))
        return s

    def block_info(self, b: int):
        pool, slab, idx = C.c_int32(), C.c_uint32(), C.c_uint32()
        _chk(lib().aeg_block_info(self.h, int(b), C.byref(pool), C.byref(slab), C.byref(idx)))
        return pool.value, slab.value, idx.value

    def block_ptr(self, pool: int, shape, b: int, layer: int) -> int:
        p = P()
        sh = KVShape.of(shape)
        _chk(lib().aeg_block_ptr(self.h, pool, C.byref(sh), int(b), int(layer), C.byref(p)))
        return p.value or 0

    def block_offsets(self, pool: int, shape, blocks):
        """(layer-0 byte offsets from the pool base [n], per-layer stride) for a consumer's block table."""
        b = _blocks(blocks)
        off = np.zeros(max(1, b.size), dtype=np.uint64)
        stride = C.c_uint64()
        sh = KVShape.of(shape)
        _chk(lib().aeg_block_offsets(self.h, pool, C.byref(sh), _p64(b), int(b.size), _p64(off), C.byref(stride)))
        return off[: b.size], stride.value

    def pool_region(self, pool: int):
        p, n = P(), C.c_uint64()
        _chk(lib().aeg_pool_region(self.h, pool, C.byref(p), C.byref(n)))
        return p.value or 0, n.value

    def peer_region(self, peer: int):
        p, n = P(), C.c_uint64()
        _chk(lib().aeg_peer_region(self.h, int(peer), C.byref(p), C.byref(n)))
        return p.value or 0, n.value

    # -- H2-H6
    def kv_swap_out(self, shape, dev, host, flags: int = 0) -> int:
        d, h = _blocks(dev), _blocks(host)
        assert d.size == h.size
        x = C.c_uint64()
        sh = KVShape.of(shape)
        _chk(lib().aeg_kv_swap_out(self.h, C.byref(sh), _p64(d), _p64(h), int(d.size), flags, C.byref(x)))
        return x.value

    def kv_swap_in(self, shape, host, dev, flags: int = 0) -> int:
        h, d = _blocks(host), _blocks(dev)
        assert d.size == h.size
        x = C.c_uint64()
        sh = KVShape.of(shape)
        _chk(lib().aeg_kv_swap_in(self.h, C.byref(sh), _p64(h), _p64(d), int(d.size), flags, C.byref(x)))
        return x.value

    def kv_migrate(self, shape, src, peer: int, dst, flags: int = 0) -> int:
        s, d = _blocks(src), _blocks(dst)
        assert s.size == d.size
        x = C.c_uint64()
        sh = KVShape.of(shape)
        _chk(lib().aeg_kv_migrate(self.h, C.byref(sh), _p64(s), int(peer), _p64(d), int(s.size), flags, C.byref(x)))
        return x.value

    def kv_swap_in_from(self, shape, peer: int, peer_host, dev, after: int = 0, flags: int = 0) -> int:
        h, d = _blocks(peer_host), _blocks(dev)
        assert d.size == h.size
        x = C.c_uint64()
        sh = KVShape.of(shape)
        _chk(lib().aeg_kv_swap_in_from(self.h, C.byref(sh), int(peer), _p64(h), _p64(d), int(d.size), int(after),
                                       flags, C.byref(x)))
        return x.value

    def kv_free_after(self, pool: int, blocks, after: int):
        b = _blocks(blocks)
        _chk(lib().aeg_kv_free_after(self.h, pool, _p64(b), int(b.size), int(after)))

    def stream_fence(self, stream: int = 0):
        _chk(lib().aeg_stream_fence(self.h, P(stream)))

    def layer_ready(self, x: int, layer: int = -1, mode: int = READY_QUERY, stream: int = 0) -> bool:
        rc = _chk(lib().aeg_layer_ready(self.h, int(x), int(layer), int(mode), P(stream)), allow_not_ready=True)
        return rc == OK

    def xfer_layers(self, x: int) -> int:
        n = C.c_int32()
        _chk(lib().aeg_xfer_layers(self.h, int(x), C.byref(n)))
        return n.value

    def xfer_release(self, x: int):
        _chk(lib().aeg_xfer_release(self.h, int(x)))

    # -- H7 / N1
    def weights_stage(self, descs, tp_rank: int = 0, tp_size: int = 1):
        """descs: list of dicts(host_src:int ptr, rows, cols, elem_bytes, layer, split, groups)."""
        arr = (WeightDesc * max(1, len(descs)))()
        for i, d in enumerate(descs):
            arr[i] = WeightDesc(d["host_src"], d["rows"], d["cols"], d.get("elem_bytes", 2), d["layer"],
                                d.get("split", SPLIT_REPLICATED), d.get("groups", 1))
        offs = np.zeros(max(1, len(descs)), dtype=np.uint64)
        x = C.c_uint64()
        _chk(lib().aeg_weights_stage(self.h, arr, len(descs), int(tp_rank), int(tp_size), _p64(offs), C.byref(x)))
        return offs[: len(descs)], x.value

    def weights_reset(self, offset: int = 0):
        _chk(lib().aeg_weights_reset(self.h, int(offset)))

    def weights_region(self):
        p, n, b = P(), C.c_uint64(), C.c_uint64()
        _chk(lib().aeg_weights_region(self.h, C.byref(p), C.byref(n), C.byref(b)))
        return p.value or 0, n.value, b.value

    def weights_relocate(self, src_off: int, dst_off: int, nbytes: int) -> int:
        x = C.c_uint64()
        _chk(lib().aeg_weights_relocate(self.h, int(src_off), int(dst_off), int(nbytes), C.byref(x)))
        return x.value

    def weights_stats(self):
        """(chunks issued, issuer ms waiting for host fills, fill ms waiting for Stage Buffer slots)."""
        n, a, b = C.c_uint64(), C.c_double(), C.c_double()
        _chk(lib().aeg_weights_stats(self.h, C.byref(n), C.byref(a), C.byref(b)))
        return n.value, a.value, b.value

    def host_register(self, ptr: int, nbytes: int):
        _chk(lib().aeg_host_register(self.h, P(ptr), int(nbytes)))

    def host_unregister(self, ptr: int):
        _chk(lib().aeg_host_unregister(self.h, P(ptr)))

    # -- multi-process
    def export_ipc(self) -> bytes:
        n = C.c_uint64(0)
        _chk(lib().aeg_export_ipc(self.h, None, C.byref(n)))
        buf = C.create_string_buffer(n.value)
        _chk(lib().aeg_export_ipc(self.h, buf, C.byref(n)))
        return buf.raw[: n.value]

    def import_peer(self, peer: int, blob: bytes):
        _chk(lib().aeg_import_peer(self.h, int(peer), blob, len(blob)))

    def xfer_export(self, x: int) -> bytes:
        n = C.c_uint64(0)
        _chk(lib().aeg_xfer_export(self.h, int(x), None, C.byref(n)))
        buf = C.create_string_buffer(n.value)
        _chk(lib().aeg_xfer_export(self.h, int(x), buf, C.byref(n)))
        return buf.raw[: n.value]

    def xfer_import(self, peer: int, blob: bytes) -> int:
        x = C.c_uint64()
        _chk(lib().aeg_xfer_import(self.h, int(peer), blob, len(blob), C.byref(x)))
        return x.value

    # -- instrumentation
    def kernel_stats(self, kind: int):
        n, b, ms = C.c_uint64(), C.c_uint64(), C.c_double()
        _chk(lib().aeg_kernel_stats(self.h, int(kind), C.byref(n), C.byref(b), C.byref(ms)))
        return n.value, b.value, ms.value

    def set_migrate_ctas(self, ctas: int):
        _chk(lib().aeg_set_migrate_ctas(self.h, int(ctas)))

    def kernel_stats_reset(self):
        _chk(lib().aeg_kernel_stats_reset(self.h))

    def trace_enable(self, on: bool = True):
        _chk(lib().aeg_trace_enable(self.h, int(on)))

    def trace_read(self) -> str:
        """Copy out and clear the primitive trace (the daemon may append between calls: retry)."""
        for _ in range(100):
            n = C.c_uint64(0)
            lib().aeg_trace_read(self.h, None, C.byref(n))      # INVALID by design: returns the size
            cap = 2 * n.value + 65536
            buf = C.create_string_buffer(cap)
            n2 = C.c_uint64(cap)
            if lib().aeg_trace_read(self.h, buf, C.byref(n2)) == OK:
                return buf.raw[: n2.value].decode()
        raise AegError(ERR_STATE, "trace kept growing")

    def debug_xfer_begin(self, pool: int, blocks) -> int:
        b = _blocks(blocks)
        x = C.c_uint64()
        _chk(lib().aeg_debug_xfer_begin(self.h, pool, _p64(b), int(b.size), C.byref(x)))
        return x.value

    def debug_xfer_complete(self, x: int):
        _chk(lib().aeg_debug_xfer_complete(self.h, int(x)))


def declared_symbols() -> list[str]:
    """Every function name include/aeg.h declares (for the export test)."""
    import re
    src = open(HEADER).read()
    return sorted(set(re.findall(r"^\s*(?:const\s+)?\w+\*?\s+\**(aeg_\w+)\s*\(", src, re.M)))


def decode_block(b: int):
    """(pool, slab, index) from the documented handle encoding (aeg.h)."""
    b = int(b)
    return b >> 62, (b >> 32) & 0x3FFFFFFF, b & 0xFFFFFFFF
