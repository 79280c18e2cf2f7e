"""Event-chain probe for the chained swap round trip (tools/roundtrip_timeline.py shows the
swap-in's first three layers becoming ready together): plain torch/cudart, no library.
  stream A (D2H)   : for i: 1 GiB D2H (from a device buffer to pinned host slot i) ; record a_i
  stream B (H2D)   : for i: wait a_i ; 1 GiB H2D (host slot i -> device) ; record b_i
  stream C (kernel): for i: wait b_i ; small kernel ; record c_i
The host polls cudaEventQuery on every event and stamps when each completes.  Variants: the
consumer stream C at high priority, and B's H2D split in 8 pieces.
Usage: python tools/chain_probe.py"""
import ctypes as C
import json
import time

import torch

GIB = 1 << 30
rt = C.CDLL("libcudart.so.12")


def run(n=6, prio=0, pieces=1, slots=3, timing=False, timing_b=False):
    dev = [torch.empty(GIB, dtype=torch.uint8, device="cuda") for _ in range(slots)]
    src = torch.empty(GIB, dtype=torch.uint8, device="cuda")
    host = torch.empty(n * GIB, dtype=torch.uint8, pin_memory=True)
    sA, sB = torch.cuda.Stream(), torch.cuda.Stream()
    sC = torch.cuda.Stream(priority=-1 if prio else 0)
    ev = {k: [torch.cuda.Event() for _ in range(n)] for k in "abc"}
    freed = [torch.cuda.Event() for _ in range(n)]
    tims = []
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for i in range(n):
        assert rt.cudaMemcpyAsync(C.c_void_p(host.data_ptr() + i * GIB), C.c_void_p(src.data_ptr()),
                                  C.c_size_t(GIB), 2, C.c_void_p(sA.cuda_stream)) == 0
        ev["a"][i].record(sA)
    for i in range(n):
        sB.wait_event(ev["a"][i])
        if i >= slots:
            sB.wait_event(freed[i - slots])
        d = dev[i % slots]
        step = GIB // pieces
        for p in range(pieces):
            assert rt.cudaMemcpyAsync(C.c_void_p(d.data_ptr() + p * step),
                                      C.c_void_p(host.data_ptr() + i * GIB + p * step),
                                      C.c_size_t(step), 1, C.c_void_p(sB.cuda_stream)) == 0
        ev["b"][i].record(sB)
        if timing_b:   # a timing event on the copy-engine stream too
            torch.cuda.Event(enable_timing=True).record(sB)
        sC.wait_event(ev["b"][i])
        if timing:     # CUDA timing events around the kernel, as AEG_CFG_TIMING does
            ta, tb = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            ta.record(sC)
        with torch.cuda.stream(sC):
            d[:1 << 20].add_(1)
        if timing:
            tb.record(sC)
            tims.append((ta, tb))
        ev["c"][i].record(sC)
        freed[i].record(sC)
    pend = [(k, i) for k in "abc" for i in range(n)]
    seen = {}
    while pend:
        rest = []
        for k, i in pend:
            if ev[k][i].query():
                seen[(k, i)] = round((time.perf_counter() - t0) * 1e3, 1)
            else:
                rest.append((k, i))
        pend = rest
    torch.cuda.synchronize()
    return {k: [seen[(k, i)] for i in range(n)] for k in "abc"}


def main():
    torch.cuda.init()
    out = {}
    for name, kw in (("warmup", {}), ("base", {}), ("timing", {"timing": True}),
                     ("timing_slots6", {"timing": True, "slots": 6}), ("timing_on_b_too", {"timing": True, "timing_b": True}),
                     ("c_high_prio_timing", {"prio": 1, "timing": True})):
        out[name] = run(**kw)
        print(name, out[name], flush=True)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
