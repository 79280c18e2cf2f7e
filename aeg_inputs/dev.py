"""ctypes wrapper of libaeginputs.so: device/host evaluation of the aeg_inputs content generator at
caller-given places and keys, a synthetic per-layer consumer, a delay kernel and a plain copy.
Test/bench infrastructure; nothing here knows the method's layout or semantics."""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

PATH = os.path.join(os.path.dirname(os.path.abspath(__file__)), "libaeginputs.so")
_L = None
P, U64 = C.c_void_p, C.c_uint64
PU64 = C.POINTER(C.c_uint64)


def lib():
    global _L
    if _L is None:
        if not os.path.exists(PATH):
            raise RuntimeError(f"{PATH} missing: build with python -m paper_conf_sosp_xiang0qyzyzl0025_b200.build")
        L = C.CDLL(PATH)
        sig = {
            "aegin_fill_chunks": [P, PU64, PU64, U64, U64, U64, P],
            "aegin_verify_chunks": [P, PU64, PU64, U64, U64, U64, PU64, PU64, P],
            "aegin_fill_region": [P, U64, U64, U64, P],
            "aegin_verify_region": [P, U64, U64, U64, PU64, PU64, P],
            "aegin_consume": [P, P, U64, U64, P, P],
            "aegin_spin": [C.c_longlong, P],
            "aegin_gate": [P, P],
            "aegin_preload": [],
            "aegin_copy": [P, P, U64],
            "aegin_sync": [],
            "aegin_host_fill": [P, U64, U64, U64, C.c_int],
            "aegin_host_fill_2d": [P, U64, U64, U64, U64, U64, C.c_int],
            "aegin_copy_chunks": [P, PU64, P, PU64, U64, U64, P],
            "aegin_stamp": [P, P],
        }
        for k, a in sig.items():
            getattr(L, k).argtypes = a
            getattr(L, k).restype = C.c_int
        _L = L
        rc = L.aegin_preload()
        if rc not in (0, 35, 100):      # 35/100: no driver / no device (CPU-only box)
            _ck(rc)
    return _L


def _ck(rc):
    if rc != 0:
        raise RuntimeError(f"CUDA error {rc} in libaeginputs")


def _u64(a):
    return np.ascontiguousarray(np.asarray(a, dtype=np.uint64))


def fill_chunks(base: int, offsets, keys, chunk: int, seed: int, stream: int = 0):
    o, k = _u64(offsets), _u64(keys)
    _ck(lib().aegin_fill_chunks(P(base), o.ctypes.data_as(PU64), k.ctypes.data_as(PU64), o.size, chunk, seed, P(stream)))


def verify_chunks(base: int, offsets, keys, chunk: int, seed: int, stream: int = 0):
    """(number of mismatching words, index of the first one or None)."""
    o, k = _u64(offsets), _u64(keys)
    bad, first = C.c_uint64(), C.c_uint64()
    _ck(lib().aegin_verify_chunks(P(base), o.ctypes.data_as(PU64), k.ctypes.data_as(PU64), o.size, chunk, seed,
                                  C.byref(bad), C.byref(first), P(stream)))
    return bad.value, (None if bad.value == 0 else first.value)


def fill_region(ptr: int, nbytes: int, seed: int, key: int, stream: int = 0):
    _ck(lib().aegin_fill_region(P(ptr), nbytes, seed, key, P(stream)))


def verify_region(ptr: int, nbytes: int, seed: int, key: int, stream: int = 0):
    bad, first = C.c_uint64(), C.c_uint64()
    _ck(lib().aegin_verify_region(P(ptr), nbytes, seed, key, C.byref(bad), C.byref(first), P(stream)))
    return bad.value, (None if bad.value == 0 else first.value)


def consume(base: int, dev_offsets_ptr: int, n: int, chunk: int, out_ptr: int, stream: int):
    _ck(lib().aegin_consume(P(base), P(dev_offsets_ptr), n, chunk, P(out_ptr), P(stream)))


def spin(cycles: int, stream: int = 0):
    _ck(lib().aegin_spin(int(cycles), P(stream)))


class Gate:
    """Holds a stream until open(): a kernel polling a pinned host flag (deterministic race tests)."""

    def __init__(self):
        import torch
        self.flag = torch.zeros(1, dtype=torch.int32, pin_memory=True)

    def close_on(self, stream: int):
        self.flag[0] = 0
        _ck(lib().aegin_gate(P(self.flag.data_ptr()), P(stream)))

    def open(self):
        self.flag[0] = 1


def copy(dst: int, src: int, nbytes: int):
    _ck(lib().aegin_copy(P(dst), P(src), nbytes))


def sync():
    _ck(lib().aegin_sync())


def read(ptr: int, nbytes: int) -> np.ndarray:
    out = np.empty(nbytes, dtype=np.uint8)
    copy(out.ctypes.data, ptr, nbytes)
    return out


def write(ptr: int, arr: np.ndarray):
    a = np.ascontiguousarray(arr)
    copy(ptr, a.ctypes.data, a.nbytes)


def host_fill(arr: np.ndarray, seed: int, key: int, threads: int = 8):
    _ck(lib().aegin_host_fill(P(arr.ctypes.data), arr.nbytes, seed, key, threads))


def host_fill_2d(ptr: int, rows: int, pitch: int, width: int, seed: int, key: int, threads: int = 8):
    """Fill `rows` runs of `width` bytes at `pitch` from `ptr` with the bytes a dense host_fill of
    the [rows x pitch] region (key base `key`) would put there."""
    _ck(lib().aegin_host_fill_2d(P(ptr), rows, pitch, width, seed, key, threads))


def copy_chunks(dst_base: int, dst_offs, src_base: int, src_offs, chunk: int, stream: int = 0):
    """One cudaMemcpyAsync per chunk (the per-block memcpy baseline)."""
    d, s_ = _u64(dst_offs), _u64(src_offs)
    _ck(lib().aegin_copy_chunks(P(dst_base), d.ctypes.data_as(PU64), P(src_base), s_.ctypes.data_as(PU64), d.size,
                                chunk, P(stream)))


def stamp(dev_u64_ptr: int, stream: int = 0):
    """Enqueue a kernel writing %globaltimer (ns, GPU-wide) to the device word at dev_u64_ptr."""
    _ck(lib().aegin_stamp(P(dev_u64_ptr), P(stream)))
