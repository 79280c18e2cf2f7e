"""Copy-engine D2H / H2D GB/s by command shape, on the swap path's geometry (DESIGN.md §3 host DMAs):
8 GiB moved per case between a 1 GiB device staging buffer and 8 GiB of pinned host memory laid
out like 8 layer-major 1 GiB slabs (one Qwen-7B layer of a slab = 32 MiB at offset l * 32 MiB).
  1d_1g   : 8 x 1 GiB contiguous copies
  1d_32m  : 256 x 32 MiB copies, host contiguous
  2d_layer: per layer one cudaMemcpy2DAsync (8 rows x 32 MiB, host pitch 1 GiB)  <- what swap.cc issues
  1d_layer: per layer 8 separate 32 MiB copies (same addresses as 2d_layer)
Usage: python tools/dma_shape_probe.py"""
import ctypes as C
import json
import sys

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
    json.dump(out, sys.stdout)
    print()


if __name__ == "__main__":
    main()
