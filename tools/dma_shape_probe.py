"""Copy-engine D2H / H2D GB/s by command shape, on the swap path's geometry (DESIGN.md §3 host DMAs):
8 GiB moved per case between a 1 GiB device staging buffer and 8 GiB of pinned host memory laid
out like 8 layer-major 1 GiB slabs (one Qwen-7B layer of a slab = 32 MiB at offset l * 32 MiB).
  1d_1g   : 8 x 1 GiB contiguous copies
  1d_32m  : 256 x 32 MiB copies, host contiguous
  2d_layer: per layer one cudaMemcpy2DAsync (8 rows x 32 MiB, host pitch 1 GiB)  <- what swap.cc issues
  1d_layer: per layer 8 separate 32 MiB copies (same addresses as 2d_layer)
  duplex share: a second direction started while an 8 GiB copy runs (GB/s it gets)
Usage: python tools/dma_shape_probe.py"""
import ctypes as C
import json
import sys
import time

import torch

GIB, MIB = 1 << 30, 1 << 20
rt = C.CDLL("libcudart.so.12")
D2H, H2D = 2, 1


def main():
    torch.cuda.init()
    dev = torch.empty(GIB, dtype=torch.uint8, device="cuda")
    host = torch.empty(8 * GIB, dtype=torch.uint8, pin_memory=True)
    s = torch.cuda.Stream()
    hs = C.c_void_p(s.cuda_stream)
    dp, hp = dev.data_ptr(), host.data_ptr()

    def cp(dst, src, n, kind):
        assert rt.cudaMemcpyAsync(C.c_void_p(dst), C.c_void_p(src), C.c_size_t(n), kind, hs) == 0

    def cp2(dst, dpitch, src, spitch, w, h, kind):
        assert rt.cudaMemcpy2DAsync(C.c_void_p(dst), C.c_size_t(dpitch), C.c_void_p(src), C.c_size_t(spitch),
                                    C.c_size_t(w), C.c_size_t(h), kind, hs) == 0

    def case(name, kind):
        d2h = kind == D2H
        def one(h, d, n):
            cp(h, d, n, kind) if d2h else cp(d, h, n, kind)
        if name == "1d_1g":
            for q in range(8):
                one(hp + q * GIB, dp, GIB)
        elif name == "1d_32m":
            for q in range(256):
                one(hp + q * 32 * MIB, dp + (q % 32) * 32 * MIB, 32 * MIB)
        elif name == "2d_layer":
            for l in range(32):
                if d2h:
                    cp2(hp + l * 32 * MIB, GIB, dp, 32 * MIB, 32 * MIB, 8, kind)
                else:
                    cp2(dp, 32 * MIB, hp + l * 32 * MIB, GIB, 32 * MIB, 8, kind)
        elif name == "1d_layer":
            for l in range(32):
                for r in range(8):
                    one(hp + r * GIB + l * 32 * MIB, dp + r * 32 * MIB, 32 * MIB)

    out = {}
    for kind, kn in ((D2H, "d2h"), (H2D, "h2d")):
        for name in ("1d_1g", "1d_32m", "2d_layer", "1d_layer"):
            best = 0.0
            for rep in range(3):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(s)
                case(name, kind)
                e1.record(s)
                e1.synchronize()
                best = max(best, 8 * GIB / (e0.elapsed_time(e1) * 1e6))
            out[f"{kn}_{name}"] = round(best, 2)
            print(kn, name, round(best, 2), flush=True)
    # duplex share: an 8 GiB D2H stream is running when a 1 GiB H2D starts on another stream (and
    # the reverse) -- GB/s each direction gets while both run (PCIe arbitration between posted
    # writes (D2H) and read requests (H2D))
    dev2 = torch.empty(GIB, dtype=torch.uint8, device="cuda")
    s2 = torch.cuda.Stream()
    hs2 = C.c_void_p(s2.cuda_stream)
    for first, second in ((D2H, H2D), (H2D, D2H)):
        torch.cuda.synchronize()
        a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        b0, b1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a0.record(s)
        for q in range(8):
            if first == D2H:
                cp(hp + q * GIB, dp, GIB, D2H)
            else:
                cp(dp, hp + q * GIB, GIB, H2D)
        a1.record(s)
        # start the other direction once ~1 GiB of the first has moved
        time.sleep(0.02)
        b0.record(s2)
        if second == H2D:
            assert rt.cudaMemcpyAsync(C.c_void_p(dev2.data_ptr()), C.c_void_p(hp), C.c_size_t(GIB), H2D, hs2) == 0
        else:
            assert rt.cudaMemcpyAsync(C.c_void_p(hp), C.c_void_p(dev2.data_ptr()), C.c_size_t(GIB), D2H, hs2) == 0
        b1.record(s2)
        torch.cuda.synchronize()
        kn = "d2h_running_then_h2d" if first == D2H else "h2d_running_then_d2h"
        out[kn] = {"second_GBps": round(GIB / (b0.elapsed_time(b1) * 1e6), 2),
                   "first_total_GBps": round(8 * GIB / (a0.elapsed_time(a1) * 1e6), 2),
                   "second_started_ms": round(a0.elapsed_time(b0), 1)}
        print(kn, out[kn], flush=True)
    json.dump(out, sys.stdout)
    print()


if __name__ == "__main__":
    main()
