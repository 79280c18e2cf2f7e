"""Probe: do NVML's PCIe / NVLink byte counters see copy-engine traffic on this box?  Reads
NVML_FI_DEV_PCIE_COUNT_{TX,RX}_BYTES and nvmlDeviceGetPcieThroughput around known pinned copies."""
import time

import pynvml as N
import torch

N.nvmlInit()
h = N.nvmlDeviceGetHandleByIndex(0)
FIELDS = {"pcie_tx": N.NVML_FI_DEV_PCIE_COUNT_TX_BYTES, "pcie_rx": N.NVML_FI_DEV_PCIE_COUNT_RX_BYTES,
          "nvl_tx": N.NVML_FI_DEV_NVLINK_THROUGHPUT_DATA_TX, "nvl_rx": N.NVML_FI_DEV_NVLINK_THROUGHPUT_DATA_RX}


def read():
    out = {}
    vals = N.nvmlDeviceGetFieldValues(h, list(FIELDS.values()))
    for (k, _), v in zip(FIELDS.items(), vals):
        if v.nvmlReturn != 0:
            out[k] = f"err{v.nvmlReturn}"
            continue
        vt = v.valueType
        out[k] = {0: v.value.dVal, 1: v.value.uiVal, 2: v.value.ulVal, 3: v.value.ullVal, 4: v.value.sllVal}.get(vt, v.value.ullVal)
    return out


n = 4 << 30
hbuf = torch.empty(n, dtype=torch.uint8).pin_memory()
dbuf = torch.empty(n, dtype=torch.uint8, device="cuda")
for name, fn in (("h2d", lambda: dbuf.copy_(hbuf, non_blocking=True)), ("d2h", lambda: hbuf.copy_(dbuf, non_blocking=True))):
    torch.cuda.synchronize()
    a = read()
    thr = []
    t0 = time.perf_counter()
    fn()
    while not torch.cuda.current_stream().query():
        thr.append((N.nvmlDeviceGetPcieThroughput(h, N.NVML_PCIE_UTIL_TX_BYTES),
                    N.nvmlDeviceGetPcieThroughput(h, N.NVML_PCIE_UTIL_RX_BYTES)))
        time.sleep(0.01)
    torch.cuda.synchronize()
    dt = time.perf_counter() - t0
    b = read()
    d = {k: (b[k] - a[k]) if isinstance(a[k], (int, float)) and isinstance(b[k], (int, float)) else (a[k], b[k]) for k in a}
    print(name, f"{n / dt / 1e9:.1f} GB/s wall", "delta", d, "throughput samples KB/s (tx, rx):", thr[:3], thr[len(thr)//2:len(thr)//2+2])
