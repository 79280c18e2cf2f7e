"""How many async operations can be queued on one stream before the enqueueing host call blocks?
A 2 s spin kernel (torch.cuda._sleep) holds the stream; then tiny D2H copies (pinned), event
records and cross-stream event waits are enqueued one by one and the first call that takes > 2 ms
is reported.  Usage: python tools/queue_depth_probe.py"""
import ctypes as C
import json
import time

import torch

rt = C.CDLL("libcudart.so.12")


def probe(kind, n=20000):
    s = torch.cuda.Stream()
    other = torch.cuda.Stream()
    d = torch.empty(1 << 20, dtype=torch.uint8, device="cuda")
    h = torch.empty(1 << 20, dtype=torch.uint8, pin_memory=True)
    ev = torch.cuda.Event()
    ev.record(other)
    torch.cuda.synchronize()
    with torch.cuda.stream(s):
        torch.cuda._sleep(4_000_000_000)   # ~2 s at 1.9 GHz
    hs = C.c_void_p(s.cuda_stream)
    evs = [torch.cuda.Event() for _ in range(64)]
    for i in range(n):
        t0 = time.perf_counter()
        if kind == "d2h":
            assert rt.cudaMemcpyAsync(C.c_void_p(h.data_ptr()), C.c_void_p(d.data_ptr()), C.c_size_t(4096), 2, hs) == 0
        elif kind == "record":
            evs[i % 64].record(s)
        elif kind == "wait":
            s.wait_event(ev)
        elif kind == "d2h+record":
            assert rt.cudaMemcpyAsync(C.c_void_p(h.data_ptr()), C.c_void_p(d.data_ptr()), C.c_size_t(4096), 2, hs) == 0
            evs[i % 64].record(s)
        dt = time.perf_counter() - t0
        if dt > 2e-3:
            torch.cuda.synchronize()
            return {"first_blocking_call": i, "blocked_ms": round(dt * 1e3, 1)}
    torch.cuda.synchronize()
    return {"first_blocking_call": None, "enqueued": n}


def main():
    torch.cuda.init()
    out = {k: probe(k) for k in ("d2h", "record", "wait", "d2h+record")}
    print(json.dumps(out))


if __name__ == "__main__":
    main()
