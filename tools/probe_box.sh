#!/bin/bash
# One-off host/GPU facts for DESIGN.md (host RAM, memlock, NUMA, PCIe/NVLink topology, pinned copy GB/s).
set -x
mkdir -p gpurun_out
{
nproc; lscpu | head -30; free -g; ulimit -l; cat /proc/meminfo | head -5
nvidia-smi; nvidia-smi topo -m; nvidia-smi -q | grep -iA3 'PCIe Generation\|Link Width' | head -30
numactl --hardware 2>/dev/null || ls /sys/devices/system/node/
cat /sys/bus/pci/devices/*/numa_node 2>/dev/null | sort | uniq -c
df -h /tmp /dev/shm
python - <<'PY'
import torch, time
d = torch.device('cuda:0')
for gib in (1, 4):
    n = gib << 30
    t0 = time.time(); h = torch.empty(n, dtype=torch.uint8, pin_memory=True); t1 = time.time()
    print(f"pin {gib} GiB: {t1-t0:.3f}s")
    g = torch.empty(n, dtype=torch.uint8, device=d)
    s = torch.cuda.Stream()
    for name, fn in (("H2D", lambda: g.copy_(h, non_blocking=True)), ("D2H", lambda: h.copy_(g, non_blocking=True))):
        with torch.cuda.stream(s):
            for _ in range(2): fn()
            e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
            e0.record(); 
            for _ in range(5): fn()
            e1.record()
        e1.synchronize()
        print(f"{name} {gib} GiB: {5*n/e0.elapsed_time(e1)/1e6:.1f} GB/s")
    # bidirectional
    h2 = torch.empty(n, dtype=torch.uint8, pin_memory=True); g2 = torch.empty(n, dtype=torch.uint8, device=d)
    s2 = torch.cuda.Stream()
    torch.cuda.synchronize(); t0 = time.time()
    with torch.cuda.stream(s):
        for _ in range(5): g.copy_(h, non_blocking=True)
    with torch.cuda.stream(s2):
        for _ in range(5): h2.copy_(g2, non_blocking=True)
    torch.cuda.synchronize(); t1 = time.time()
    print(f"bidir {gib} GiB each: {2*5*n/(t1-t0)/1e9:.1f} GB/s total")
    del h, g, h2, g2
t0 = time.time(); h = torch.empty(32 << 30, dtype=torch.uint8, pin_memory=True); print("pin 32 GiB:", time.time()-t0)
del h
print(torch.cuda.get_device_properties(0))
PY
} > gpurun_out/probe.txt 2>&1
