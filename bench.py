#!/usr/bin/env python
"""bench.py — Aegaeon KV/weight data-movement hot path on B200 (BASELINE.json metric).

Timed step (N=1: BASELINE.json configs[1], "Qwen-7B-shaped KV (32 layers, 32 heads, d=128, bf16):
preempt and swap out a 64-request decode batch, then swap back in, on 1 B200"):
    H1 alloc host blocks + fresh device blocks  ->  H2/H3 swap-out (gather kernel -> CE D2H, KV-Out
    stream, per-layer events)  ->  H4 swap-in (CE H2D -> scatter kernel into the fresh blocks, rule ❷
    per-layer waits on the swap-out, so the two directions overlap full duplex)  ->  H6 a synthetic
    decode consumer waits per layer (rule ❶) and reads each layer  ->  H1 free (move lists).
value = KV bytes moved over PCIe per step (out + in) / device time of the step, in GB/s.
After the timed region the north-star invariant is checked: swap_in o swap_out is the identity on
every chunk of the batch (generator content at the library's block table), resident blocks are
untouched.  bench.py runs the oracle (oracle/) only in its cpu_baseline leg and in --impl reference;
the oracle parity of the same workloads is in tests/ (test_gpu_fullsize.py, test_gpu_c5.py).

Also measured in the same run (not in `value`): H7+H8 model switch among Qwen-1.8B / Llama-7B /
Yi-9B shapes with 1 GiB KV each (configs[3]; staged, registered-cache and prefetch modes, Eq. 4 beta),
H5 hand-off (configs[2] shapes: fused kernel, copy-engine route, per-chunk memcpy baseline; across
GPUs at N >= 2), the P->C->D host route, configs[4] TP=4 scale-up, per-layer overlap, per-request
sync overhead (Fig. 15 right), small-chunk shapes, configs[0] latency, the allocator, NVML PCIe
counters, the oracle on host cores (cpu_baseline), and the whole step through the public Python
API with wall-clock timing (e2e).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
N > 1 runs under torchrun (one rank per GPU): every rank swaps its own batch (replicas, weak
scaling) and, for the migrate leg, rank i hands a batch to rank i + N/2 over NVLink.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "KV swap/migrate GB/s vs HBM/PCIe/NVLink roofline; model-switch latency (ms)"
GIB = 1 << 30
MIB = 1 << 20
PCIE_NOMINAL = 64.0   # GB/s per direction, PCIe Gen5 x16
NVLINK_NOMINAL = 900.0
NVLINK_PEER_COPY = 770.0   # GB/s per direction, measured peer copy (B200_PROFILING.md)
HBM_FALLBACK = 6650.0
BETA = 0.625          # PAPER.md:2515 (Eq. 4)


def log(*a):
    print(*a, file=sys.stderr, flush=True)


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=10)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--requests", type=int, default=64)
    p.add_argument("--kernel", default="auto", choices=["auto", "lsu", "bulk", "bulkw", "warp"])
    p.add_argument("--no-switch", action="store_true")
    p.add_argument("--no-migrate", action="store_true")
    p.add_argument("--no-c5", action="store_true", help="skip the configs[4] Qwen-72B TP=4 scale-up leg")
    # exercise knobs (several ranks sharing one GPU): not used for reported numbers
    p.add_argument("--c5-model", default="qwen-72b", help=argparse.SUPPRESS)
    p.add_argument("--churn-slabs", type=int, default=12, help=argparse.SUPPRESS)
    p.add_argument("--migrate-requests", type=int, default=16, help=argparse.SUPPRESS)
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--no-cpu", action="store_true")
    p.add_argument("--switches", type=int, default=30)
    p.add_argument("--slot-mib", type=int, default=0, help="staging slot size (0 = library default)")
    p.add_argument("--slots", type=int, default=0)
    p.add_argument("--dma-piece-mib", type=int, default=0, help="swap-out D2H piece (0 = library default)")
    p.add_argument("--profile", action="store_true", help="short run for ncu (no side legs)")
    p.add_argument("--two-device-probe", action="store_true", help=argparse.SUPPRESS)
    p.add_argument("--probe-peer-bulk", action="store_true",
                   help="N >= 2: also time cp.async.bulk stores into another GPU's memory (BULKW) in a throw-away "
                        "process; off by default — AUTO never uses them, and a fault there would be an Xid on the box")
    p.add_argument("--leg-budget-s", type=float, default=1500.0,
                   help="wall-clock budget of the side legs after the timed region")
    return p.parse_args()


_RAW_STREAMS = []


def new_stream(torch):
    """A dedicated CUDA stream.  torch.cuda.Stream() hands out pooled streams round-robin (32 per
    priority), so a "new" stream can be an earlier one with work still queued behind it, which
    silently corrupts event timings (the switch leg's landing probes read 270 ms for a layer that
    landed at 1 ms).  Created once per call through the CUDA runtime torch already loaded."""
    import ctypes as C
    rt = C.CDLL("libcudart.so.12")
    s = C.c_void_p()
    rc = rt.cudaStreamCreateWithFlags(C.byref(s), 1)   # cudaStreamNonBlocking
    if rc != 0:
        raise RuntimeError(f"cudaStreamCreateWithFlags failed: {rc}")
    _RAW_STREAMS.append(s)
    return torch.cuda.ExternalStream(s.value)


# ----------------------------------------------------------------------------------- plumbing
def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


class Dist:
    def __init__(self, world, rank, local):
        import torch
        self.world, self.rank, self.local = world, rank, local
        self.torch = torch
        # one process per GPU; AEG_DIST_BACKEND=gloo lets several ranks share one GPU to exercise the
        # multi-rank path on a 1-GPU box (control data only travels through torch.distributed)
        self.backend = os.environ.get("AEG_DIST_BACKEND", "nccl")
        self.device = local % max(1, torch.cuda.device_count())
        torch.cuda.set_device(self.device)
        self.pg = None
        if world > 1:
            import torch.distributed as td
            os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
            # NCCL's init lines (comm ... nRanks N) in the log let the driver count the ranks
            os.environ.setdefault("NCCL_DEBUG", "INFO")
            os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
            if self.backend == "nccl":
                td.init_process_group("nccl", device_id=torch.device("cuda", self.device))
            else:
                td.init_process_group(self.backend)
            self.td = td

    def _t(self, v):
        dev = "cuda" if self.backend == "nccl" else "cpu"
        return self.torch.tensor([v], dtype=self.torch.float64, device=dev)

    def barrier(self):
        self.torch.cuda.synchronize()
        if self.world > 1:
            self.td.barrier()

    def max(self, v: float) -> float:
        if self.world == 1:
            return v
        t = self._t(v)
        self.td.all_reduce(t, op=self.td.ReduceOp.MAX)
        return float(t.item())

    def sum(self, v: float) -> float:
        if self.world == 1:
            return v
        t = self._t(v)
        self.td.all_reduce(t, op=self.td.ReduceOp.SUM)
        return float(t.item())

    def gather_obj(self, o):
        if self.world == 1:
            return [o]
        out = [None] * self.world
        self.td.all_gather_object(out, o)
        return out

    def close(self):
        if self.world > 1:
            self.td.destroy_process_group()


class Clocks:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md clocks line)."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu: int):
        self.gpu = gpu
        self.proc = None

    def __enter__(self):
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                                          "-lms", "200", "-i", str(self.gpu)], stdout=self.f,
                                         stderr=subprocess.DEVNULL)
        except FileNotFoundError:
            self.proc = None
        return self

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            self.proc.wait()
        self.f.close()

    def summary(self):
        rows = []
        for line in open(self.f.name):
            f = [x.strip() for x in line.split(",")]
            if len(f) >= 9 and f[1].isdigit():
                rows.append(f)
        os.unlink(self.f.name)
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "samples": 0}
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in rows for i in range(4) if r[5 + i].lower() == "active"})
        return {"sm_mhz": statistics.median(int(r[1]) for r in rows), "sm_max_mhz": int(rows[0][2]),
                "reasons": reasons, "samples": len(rows),
                "power_w_max": max(float(r[3]) for r in rows if r[3].replace(".", "").isdigit())}


class PcieCounters:
    """NVML PCIe throughput counters of this GPU (nvmlDeviceGetPcieThroughput: bytes over the link in
    a 20 ms window, per direction) sampled by a thread while the block runs: hardware-counter
    evidence for the copy-engine traffic that ncu cannot see.  tx = device -> host (D2H), rx =
    host -> device (H2D); reported in GB/s (NVML's KB/s / 1e6)."""

    def __init__(self, gpu: int):
        self.gpu, self.rows, self.err = gpu, [], None

    def __enter__(self):
        import threading
        self.stop = threading.Event()
        try:
            import pynvml as N
            N.nvmlInit()
            self.N, self.h = N, N.nvmlDeviceGetHandleByIndex(self.gpu)
        except Exception as e:  # noqa: BLE001
            self.err = f"{type(e).__name__}: {e}"
            return self

        def run():
            N = self.N
            while not self.stop.is_set():
                try:
                    tx = N.nvmlDeviceGetPcieThroughput(self.h, N.NVML_PCIE_UTIL_TX_BYTES)
                    rx = N.nvmlDeviceGetPcieThroughput(self.h, N.NVML_PCIE_UTIL_RX_BYTES)
                except Exception as e:  # noqa: BLE001
                    self.err = f"{type(e).__name__}: {e}"
                    return
                self.rows.append((tx / 1e6, rx / 1e6))
        self.t = threading.Thread(target=run, daemon=True)
        self.t.start()
        return self

    def __exit__(self, *a):
        self.stop.set()
        if hasattr(self, "t"):
            self.t.join(timeout=5)

    def summary(self):
        if not self.rows:
            return {"error": self.err or "no samples"}
        r = self.rows[1:-1] or self.rows          # drop the windows straddling the region's edges
        tx = sorted(x[0] for x in r)
        rx = sorted(x[1] for x in r)
        med = lambda v: round(v[len(v) // 2], 1)  # noqa: E731
        return {"tx_d2h_GBps_median": med(tx), "rx_h2d_GBps_median": med(rx),
                "tx_d2h_GBps_mean": round(sum(tx) / len(tx), 1), "rx_h2d_GBps_mean": round(sum(rx) / len(rx), 1),
                "samples": len(r), "source": "NVML nvmlDeviceGetPcieThroughput (20 ms windows)"}


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d.get("hbm_gbs", HBM_FALLBACK)), "measured"
    return HBM_FALLBACK, "fallback"


def ncu_traffic(kind: str, alg_bytes_per_launch: int):
    """Per-launch DRAM bytes (read + write) of our kernel from the committed ncu capture of the same
    launch (profiles/ncu_summary.json), or None when that capture was of a different launch size."""
    p = os.path.join(ROOT, "profiles", "ncu_summary.json")
    if not os.path.exists(p):
        return None
    d = json.load(open(p)).get(kind, {})
    if int(d.get("algorithmic_bytes_per_launch", -1)) != int(alg_bytes_per_launch):
        return None
    return d.get("dram_bytes_per_launch")


# ----------------------------------------------------------------------------------- workload
QWEN7B = (32, 32, 128, 2, 16)


def c2_requests(n_req: int):
    import aeg_inputs as gi
    lens = gi.request_lengths(2, n_req, 256, 1792)
    blocks = [-(-t // 16) for t in lens]
    return lens, blocks


def chunk_offsets(ctx, pool, shape, blocks):
    """Byte offsets from the pool base of every (block, layer) chunk of `blocks`, block-major, from
    the library's block table (aeg_block_offsets)."""
    off0, stride = ctx.block_offsets(pool, shape, blocks)
    L = int(shape[0])
    return (off0[:, None] + np.arange(L, dtype=np.uint64)[None, :] * np.uint64(stride)).reshape(-1)


class SwapBench:
    """configs[1] on one GPU: aged device pool, a 64-request batch, swap round trips.  Library calls
    and the seeded generator only: input placement uses the library's own block table
    (aeg_block_offsets).  The oracle-mirrored variant with the whole-pool parity check is
    tests/oracle_swapbench.py (test infrastructure)."""

    def __init__(self, aeg, sh, n_req, kernel, extra_host_slabs=8, weight_bytes=0, seed_cfg=2, slot_mib=0, slots=0,
                 churn_slabs=12, dma_piece_mib=0, timing=True, dev_batches=2, host_batches=1):
        import aeg_inputs as gi
        self.aeg, self.gi = aeg, gi
        self.sht = sh
        self.sh = aeg.KVShape.of(sh)
        self.L = self.sh.num_layers
        self.Cl = self.sh.chunk_bytes()
        self.lens, blocks = c2_requests(n_req)
        self.labels = [(r, j) for r, b in enumerate(blocks) for j in range(b)]
        self.n = len(self.labels)
        self.k = GIB // self.sh.block_bytes()
        batch_slabs = -(-self.n // self.k)
        self.churn_slabs = churn_slabs
        dev_slabs = dev_batches * batch_slabs + self.churn_slabs + 4
        host_slabs = host_batches * batch_slabs + extra_host_slabs
        self.seed = gi.kv_seed(seed_cfg)
        cfg = aeg.default_config(device_kv_bytes=dev_slabs * GIB, host_kv_bytes=host_slabs * GIB,
                                 device_weight_bytes=weight_bytes, kernel=kernel,
                                 flags=aeg.CFG_TIMING if timing else 0)
        if slot_mib:
            cfg.staging_slot_bytes = slot_mib * MIB
        if slots:
            cfg.staging_slots = slots
        if dma_piece_mib:
            cfg.dma_piece_mib = dma_piece_mib
        self.cfg = cfg
        t0 = time.time()
        import torch
        self.ctx = aeg.Context(torch.cuda.current_device(), cfg)
        self.init_s = time.time() - t0
        self.dbase, _ = self.ctx.pool_region(aeg.POOL_DEVICE)
        self.hbase, _ = self.ctx.pool_region(aeg.POOL_HOST)
        self.ops = []   # (host blocks, device blocks) of every round trip, in order

    def chunk_offsets(self, pool, blocks):
        """Byte offsets (from the pool base) of every (block, layer) chunk, block-major, from the
        library's block table."""
        off0, stride = self.ctx.block_offsets(pool, self.sht, blocks)
        return (off0[:, None] + np.arange(self.L, dtype=np.uint64)[None, :] * np.uint64(stride)).reshape(-1)

    def batch_keys(self):
        gi = self.gi
        return np.array([gi.kv_key(1, r, j, l) for (r, j) in self.labels for l in range(self.L)], np.uint64)

    def setup(self):
        gi, aeg = self.gi, self.aeg
        # aging churn (SURVEY §8(d) placement realism): other requests' blocks stay resident
        live = []
        for op, v in gi.churn_ops(2, capacity_blocks=self.churn_slabs * self.k, hi_blocks=96):
            if op == "alloc":
                live.append(self.ctx.kv_alloc(aeg.POOL_DEVICE, self.sht, v))
            elif live[v] is not None:
                self.ctx.kv_free(aeg.POOL_DEVICE, live[v])
                live[v] = None
        self.churn = [x for x in live if x is not None]
        self.churn_offs = np.concatenate([self.chunk_offsets(0, c) for c in self.churn])
        self.churn_keys = np.array([gi.kv_key(2, q % 65536, j, l) for q, c in enumerate(self.churn)
                                    for j in range(len(c)) for l in range(self.L)], np.uint64)
        self._fill(self.churn_offs, self.churn_keys)
        self.src_c = self.ctx.kv_alloc(aeg.POOL_DEVICE, self.sht, self.n)
        self._fill(self.chunk_offsets(0, self.src_c), self.batch_keys())
        return self

    def _fill(self, offs, keys, base=None):
        from aeg_inputs import dev as D
        offs = np.asarray(offs, np.uint64)
        keys = np.asarray(keys, np.uint64)
        for a in range(0, offs.size, 1 << 16):
            D.fill_chunks(self.dbase if base is None else base, offs[a:a + (1 << 16)], keys[a:a + (1 << 16)],
                          self.Cl, self.seed)

    def _verify(self, base, offs, keys):
        from aeg_inputs import dev as D
        bad = 0
        for a in range(0, offs.size, 1 << 17):
            b, _ = D.verify_chunks(base, offs[a:a + (1 << 17)], keys[a:a + (1 << 17)], self.Cl, self.seed)
            bad += b
        return bad

    def verify(self):
        """The north-star invariant after all round trips: swap_in o swap_out is the identity on every
        chunk of the batch (its current device blocks and its last host copy hold the generator's
        bytes for each (request, block, layer) label), and the resident requests' blocks around it
        are untouched.  Chunks are located through the library's block table; expected bytes come
        from the seeded generator only (CUDA evaluation, plus a NumPy evaluation of sampled chunks)."""
        from aeg_inputs import dev as D
        keys = self.batch_keys()
        doffs = self.chunk_offsets(0, self.src_c)
        dbad = self._verify(self.dbase, doffs, keys)
        hbad, hn = 0, 0
        if getattr(self, "host_offs", None) is not None:   # the last swap-out's host copy
            hbad, hn = self._verify(self.hbase, self.host_offs, keys), self.host_offs.size
        cbad = self._verify(self.dbase, self.churn_offs, self.churn_keys)
        rng = np.random.default_rng(7)
        sample_bad = 0
        for c in rng.choice(doffs.size, size=8, replace=False):
            got = D.read(self.dbase + int(doffs[c]), self.Cl)
            sample_bad += int((got != self.gi.region_bytes(self.seed, int(keys[c]), self.Cl)).sum())
        return {"batch_device_chunks_checked": int(doffs.size), "batch_device_bad_words": int(dbad),
                "batch_host_chunks_checked": int(hn), "batch_host_bad_words": int(hbad),
                "resident_chunks_checked": int(self.churn_offs.size), "resident_bad_words": int(cbad),
                "numpy_sampled_chunks": 8, "numpy_sampled_bad_bytes": sample_bad,
                "ok": dbad == 0 and hbad == 0 and cbad == 0 and sample_bad == 0,
                "what": "swap_in o swap_out = identity on every chunk of the batch; resident blocks untouched "
                        "(whole-pool oracle parity: tests/test_gpu_fullsize.py)"}

    def consumer_tables(self, torch, blocks):
        """[L][n] byte offsets of each layer of `blocks` from the pool base (aeg_block_offsets: the
        block table a PagedAttention-style consumer would build)."""
        off0, stride = self.ctx.block_offsets(0, self.sht, blocks)
        t = off0[None, :] + np.arange(self.L, dtype=np.uint64)[:, None] * np.uint64(stride)
        return torch.from_numpy(t.astype(np.int64)).cuda()

    def step(self, torch, cons, with_consumer=True, record=True, keep_host_offsets=False, first_layer=None):
        """One timed step, library calls only (plus the synthetic consumer).  first_layer: a list
        that receives (start, layer-0-ready, last-layer-ready) events on the consumer stream."""
        aeg = self.aeg
        from aeg_inputs import dev as D
        if first_layer is not None:
            ev = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
            ev[0].record(cons)
            first_layer.extend(ev)
        hc = self.ctx.kv_alloc(aeg.POOL_HOST, self.sht, self.n)
        if keep_host_offsets:   # the host blocks are freed (and their slabs may be reclaimed) by the swap-in
            self.host_offs = self.chunk_offsets(1, hc)
        nd = self.ctx.kv_alloc(aeg.POOL_DEVICE, self.sht, self.n)
        # the consumer's block table is uploaded before the transfers are queued: a pageable H2D
        # copy queued behind the swap-in's DMAs would wait for all of them (one copy engine serves
        # H2D streams FIFO, profiles/r01/ce_probe.txt) and hold the host back from enqueueing the
        # per-layer waits
        tab = self.consumer_tables(torch, nd) if with_consumer else None
        self.ctx.stream_fence(cons.cuda_stream)
        t0 = time.perf_counter()
        x = self.ctx.kv_swap_out(self.sht, self.src_c, hc, flags=aeg.FREE_SRC)
        t1 = time.perf_counter()
        y = self.ctx.kv_swap_in(self.sht, hc, nd, flags=aeg.FREE_SRC)
        t2 = time.perf_counter()
        if first_layer is not None:   # diagnostics: host enqueue time of each call, swap-out layer 0 landed
            self.enqueue_ms = ((t1 - t0) * 1e3, (t2 - t1) * 1e3)
            if not hasattr(self, "diag_stream"):
                self.diag_stream = new_stream(torch)
            self.ctx.layer_ready(x, 0, aeg.READY_WAIT_STREAM, self.diag_stream.cuda_stream)
            ex = torch.cuda.Event(enable_timing=True)
            ex.record(self.diag_stream)
            first_layer.append(ex)
        if with_consumer:
            for l in range(self.L):
                self.ctx.layer_ready(y, l, aeg.READY_WAIT_STREAM, cons.cuda_stream)
                if first_layer is not None and l in (0, self.L - 1):
                    first_layer[1 if l == 0 else 2].record(cons)
                D.consume(self.dbase, tab[l].data_ptr(), self.n, self.Cl, self.sink.data_ptr(), cons.cuda_stream)
        else:
            self.ctx.layer_ready(y, -1, aeg.READY_WAIT_STREAM, cons.cuda_stream)
        self.ctx.layer_ready(x, -1, aeg.READY_BLOCK)
        self.ctx.layer_ready(y, -1, aeg.READY_BLOCK)
        self.ctx.xfer_release(x)
        self.ctx.xfer_release(y)
        if record:
            self.ops.append((hc, nd))
        self.src_c = nd

    def back_to_back(self, torch, cons, k=6):
        """Round trips issued back to back with no host synchronisation between them: round trip
        j+1's swap-out of the blocks round trip j swapped in waits per layer on j's events (rule ❷)
        and its fresh blocks come from the pools (rule ❸), so the D2H of j+1 overlaps the H2D of j.
        The host keeps at most two round trips in flight (pool capacity: 3 batches on the device,
        2 in host memory).  Returns GB/s over PCIe (out + in) on the consumer stream's clock."""
        aeg = self.aeg
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record(cons)
        self.ctx.stream_fence(cons.cuda_stream)
        inflight = []
        for j in range(k):
            if len(inflight) == 2:
                for t in inflight.pop(0):
                    self.ctx.layer_ready(t, -1, aeg.READY_BLOCK)
                    self.ctx.xfer_release(t)
            hc = self.ctx.kv_alloc(aeg.POOL_HOST, self.sht, self.n)
            nd = self.ctx.kv_alloc(aeg.POOL_DEVICE, self.sht, self.n)
            x = self.ctx.kv_swap_out(self.sht, self.src_c, hc, flags=aeg.FREE_SRC)
            y = self.ctx.kv_swap_in(self.sht, hc, nd, flags=aeg.FREE_SRC)
            inflight.append((x, y))
            self.src_c = nd
        for xs in inflight:
            for t in xs:
                self.ctx.layer_ready(t, -1, aeg.READY_WAIT_STREAM, cons.cuda_stream)
        e1.record(cons)
        e1.synchronize()
        for xs in inflight:
            for t in xs:
                self.ctx.layer_ready(t, -1, aeg.READY_BLOCK)
                self.ctx.xfer_release(t)
        ms = e0.elapsed_time(e1)
        return {"round_trips": k, "ms": round(ms, 1), "GBps": round(2 * k * self.n * self.sh.block_bytes() / (ms * 1e6), 2),
                "ms_per_round_trip": round(ms / k, 1)}

    def one_direction(self, torch, cons):
        """Diagnostic (not in `value`): swap-out alone, then swap-in alone, each to completion, with
        the kernel counters of each — per-direction PCIe GB/s and the kernels without the other
        direction's kernels competing for HBM."""
        aeg = self.aeg
        out = {}
        hc = self.ctx.kv_alloc(aeg.POOL_HOST, self.sht, self.n)
        nd = self.ctx.kv_alloc(aeg.POOL_DEVICE, self.sht, self.n)
        self.host_offs = self.chunk_offsets(1, hc)
        for name in ("swap_out", "swap_in"):
            self.ctx.kernel_stats_reset()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            with PcieCounters(torch.cuda.current_device()) as pc:
                e0.record(cons)
                self.ctx.stream_fence(cons.cuda_stream)
                if name == "swap_out":
                    x = self.ctx.kv_swap_out(self.sht, self.src_c, hc, flags=aeg.FREE_SRC)
                else:
                    x = self.ctx.kv_swap_in(self.sht, hc, nd, flags=aeg.FREE_SRC)
                self.ctx.layer_ready(x, -1, aeg.READY_WAIT_STREAM, cons.cuda_stream)
                e1.record(cons)
                e1.synchronize()
            self.ctx.layer_ready(x, -1, aeg.READY_BLOCK)
            self.ctx.xfer_release(x)
            ms = e0.elapsed_time(e1)
            k = self.ctx.kernel_stats(aeg.K_GATHER if name == "swap_out" else aeg.K_SCATTER)
            out[name] = {"GBps": round(self.n * self.sh.block_bytes() / (ms * 1e6), 2), "ms": round(ms, 1),
                         "kernel_GBps": round(k[1] / (k[2] * 1e6), 1) if k[2] else None,
                         "kernel_launches": k[0], "kernel_ms_total": round(k[2], 2),
                         "nvml_pcie": pc.summary()}
        self.ops.append((hc, nd))
        self.src_c = nd
        return out


# ----------------------------------------------------------------------------------- legs
def chunk_memcpy_baseline(aeg, torch, ctx, sht, src_blocks, reps=2):
    """The per-block memcpy the paper's swap amounts to for paged KV ("memcpy(async)"
    Fig. 10; vLLM-style swap_blocks): one cudaMemcpyAsync per (block, layer) chunk, device blocks ->
    host blocks, then host -> fresh device blocks, on one stream (copy engines only).  Same blocks
    and placement as the library's swap; timed with CUDA events.  Returns GB/s per direction."""
    from aeg_inputs import dev as D
    sh = aeg.KVShape.of(sht)
    n = len(src_blocks)
    hc = ctx.kv_alloc(aeg.POOL_HOST, sht, n)
    nd = ctx.kv_alloc(aeg.POOL_DEVICE, sht, n)
    dbase, _ = ctx.pool_region(aeg.POOL_DEVICE)
    hbase, _ = ctx.pool_region(aeg.POOL_HOST)
    so, ho, no = (chunk_offsets(ctx, p, sht, b) for p, b in ((0, src_blocks), (1, hc), (0, nd)))
    s = new_stream(torch)
    out = {}
    for name, args in (("d2h", (hbase, ho, dbase, so)), ("h2d", (dbase, no, hbase, ho))):
        ts = []
        for _ in range(reps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            D.copy_chunks(*args, sh.chunk_bytes(), s.cuda_stream)
            e1.record(s)
            e1.synchronize()
            ts.append(e0.elapsed_time(e1))
        out[name + "_GBps"] = round(n * sh.block_bytes() / (min(ts) * 1e6), 2)
    out["memcpy_calls_per_direction"] = int(so.size)
    out["chunk_bytes"] = sh.chunk_bytes()
    ctx.kv_free(aeg.POOL_HOST, hc)
    ctx.kv_free(aeg.POOL_DEVICE, nd)
    return out


def small_chunk_leg(aeg, torch, kernel, model="yi-9b", gib=1):
    """Swap-out / swap-in of `gib` GiB of a small-chunk KV shape (Yi-9B: 48 layers x 32 KiB chunks,
    the configs[3] model with the smallest chunk) through the library, next to the per-chunk memcpy
    baseline on the same blocks.  Correctness: the round trip is the identity on every chunk."""
    import aeg_inputs as gi
    from aeg_inputs import dev as D
    sht = gi.KV_SHAPES[model]
    sh = aeg.KVShape.of(sht)
    n = (gib * GIB) // sh.block_bytes()
    ctx = aeg.Context(0, aeg.default_config(device_kv_bytes=3 * gib * GIB + GIB, host_kv_bytes=gib * GIB + GIB,
                                            kernel=kernel, flags=aeg.CFG_TIMING))
    dbase, _ = ctx.pool_region(0)
    hbase, _ = ctx.pool_region(1)
    src = ctx.kv_alloc(0, sht, n)
    keys = np.array([gi.kv_key(3, 0, i, l) for i in range(n) for l in range(sh.num_layers)], np.uint64)
    seed = gi.kv_seed(4)
    D.fill_chunks(dbase, chunk_offsets(ctx, 0, sht, src), keys, sh.chunk_bytes(), seed)
    s = new_stream(torch)
    res = {}
    for it in range(3):
        hc = ctx.kv_alloc(1, sht, n)
        nd = ctx.kv_alloc(0, sht, n)
        ms = []
        for kind in ("out", "in"):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            ctx.stream_fence(s.cuda_stream)
            x = ctx.kv_swap_out(sht, src, hc, flags=aeg.FREE_SRC) if kind == "out" else \
                ctx.kv_swap_in(sht, hc, nd, flags=aeg.FREE_SRC)
            ctx.layer_ready(x, -1, aeg.READY_WAIT_STREAM, s.cuda_stream)
            e1.record(s)
            e1.synchronize()
            ctx.layer_ready(x, -1, aeg.READY_BLOCK)
            ctx.xfer_release(x)
            ms.append(e0.elapsed_time(e1))
        src = nd
        if it > 0:
            res.setdefault("out", []).append(ms[0])
            res.setdefault("in", []).append(ms[1])
    bad, _ = D.verify_chunks(dbase, chunk_offsets(ctx, 0, sht, src), keys, sh.chunk_bytes(), seed)
    ctx.reclaim(True)
    base = chunk_memcpy_baseline(aeg, torch, ctx, sht, src)
    ctx.shutdown()
    b = n * sh.block_bytes()
    return {"workload": f"{model} KV ({n} blocks x {sh.num_layers} layers, {sh.chunk_bytes() >> 10} KiB chunks, "
                        f"{b / GIB:.2f} GiB) swap-out and swap-in, each alone",
            "swap_out_GBps": round(b / (min(res["out"]) * 1e6), 2), "swap_in_GBps": round(b / (min(res["in"]) * 1e6), 2),
            "per_chunk_memcpy": base, "bit_exact": bad == 0}



def c1_leg(aeg, torch, kernel, reps=200, pack_mib=0):
    """configs[0] (tiny: 2 layers, 4 KV heads, d=64, fp16, 16-token blocks, 8 requests <= 256
    tokens, 75 blocks, 2.3 MiB) swap round trip: launch/latency-bound, so report the per-round-trip
    latency (GPU: consumer-stream events from the fence to the swap-in's last layer; wall: the two
    API calls + host sync) and the host enqueue time of each call.  Whole-image oracle parity of the
    same workload: tests/test_gpu_swap.py.  Here: identity on every chunk after all round trips."""
    import aeg_inputs as gi
    from aeg_inputs import dev as D
    sht = gi.KV_SHAPES["tiny"]
    sh = aeg.KVShape.of(sht)
    lens = gi.request_lengths(1, 8, 1, 256, forced=(1, 16, 17, 255, 256))
    nb = sum(-(-t // 16) for t in lens)
    kib = 1024
    # staging slots of 8 MiB: one segment per layer (the planner keeps >= 4 segments, so a 2-layer
    # transfer is never packed into one: the swap-in's H2D of layer 0 overlaps the swap-out's D2H of
    # layer 1 — 147 vs 172 us as one packed segment); 1 MiB slots would cut each layer in two (more
    # segments, ~2x the enqueue time, tools/enqueue_probe.py)
    ctx = aeg.Context(0, aeg.default_config(device_kv_bytes=32 * 256 * kib, host_kv_bytes=32 * 256 * kib,
                                            dev_slab_bytes=256 * kib, host_slab_bytes=256 * kib,
                                            staging_slot_bytes=8 << 20, staging_slots=2, stage_ring_bytes=2 << 20,
                                            stage_chunk_bytes=1 << 20, device_weight_bytes=2 << 20,
                                            table_arena_bytes=2 << 20, host_threads=1, kernel=kernel,
                                            pack_layer_mib=pack_mib))
    dbase, _ = ctx.pool_region(0)
    src = ctx.kv_alloc(0, sht, nb)
    keys = np.array([gi.kv_key(1, 0, i, l) for i in range(nb) for l in range(sh.num_layers)], np.uint64)
    seed = gi.kv_seed(1)
    D.fill_chunks(dbase, chunk_offsets(ctx, 0, sht, src), keys, sh.chunk_bytes(), seed)
    s = new_stream(torch)
    gpu_us, wall_us, enq_us = [], [], []
    for it in range(reps + 10):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        t0 = time.perf_counter()
        e0.record(s)
        ctx.stream_fence(s.cuda_stream)
        hc = ctx.kv_alloc(1, sht, nb)
        nd = ctx.kv_alloc(0, sht, nb)
        t1 = time.perf_counter()
        x = ctx.kv_swap_out(sht, src, hc, flags=aeg.FREE_SRC)
        t2 = time.perf_counter()
        y = ctx.kv_swap_in(sht, hc, nd, flags=aeg.FREE_SRC)
        t3 = time.perf_counter()
        ctx.layer_ready(y, -1, aeg.READY_WAIT_STREAM, s.cuda_stream)
        e1.record(s)
        e1.synchronize()
        t4 = time.perf_counter()
        ctx.layer_ready(x, -1, aeg.READY_BLOCK)
        ctx.xfer_release(x)
        ctx.xfer_release(y)
        src = nd
        if it >= 10:
            gpu_us.append(e0.elapsed_time(e1) * 1e3)
            wall_us.append((t4 - t0) * 1e6)
            enq_us.append(((t2 - t1) * 1e6, (t3 - t2) * 1e6))
    bad, _ = D.verify_chunks(dbase, chunk_offsets(ctx, 0, sht, src), keys, sh.chunk_bytes(), seed)
    ctx.shutdown()
    med = lambda v: round(statistics.median(v), 1)  # noqa: E731
    return {"workload": f"configs[0] tiny KV, 8 requests ({nb} blocks, {nb * sh.block_bytes() / 2**20:.2f} MiB): "
                        "swap-out + swap-in round trip, one at a time",
            "round_trip_gpu_us_p50": med(gpu_us), "round_trip_wall_us_p50": med(wall_us),
            "enqueue_us_p50": {"swap_out": med([a for a, _ in enq_us]), "swap_in": med([b for _, b in enq_us])},
            "reps": reps, "bit_exact": bad == 0}


def pcie_calibration(torch, dist=None):
    """Plain cudaMemcpy of 1 GiB pinned <-> device: the copy engines' measured ceiling here.  With
    several ranks every phase starts after a barrier, so all GPUs copy at once (the ceiling the
    replicas share: PCIe switch uplinks, host DRAM)."""
    sync = dist.barrier if dist is not None and dist.world > 1 else (lambda: None)
    h = torch.empty(GIB, dtype=torch.uint8, pin_memory=True)
    d = torch.empty(GIB, dtype=torch.uint8, device="cuda")
    out = {}
    s = new_stream(torch)
    for name, fn in (("h2d", lambda: d.copy_(h, non_blocking=True)), ("d2h", lambda: h.copy_(d, non_blocking=True))):
        sync()
        with torch.cuda.stream(s):
            fn()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(3):
                fn()
            e1.record()
        e1.synchronize()
        out[name] = 3 * GIB / (e0.elapsed_time(e1) * 1e6)
    # both directions at once (the ceiling of the round-trip `value`): 3 x 1 GiB each way
    h2 = torch.empty(GIB, dtype=torch.uint8, pin_memory=True)
    d2 = torch.empty(GIB, dtype=torch.uint8, device="cuda")
    s2 = new_stream(torch)
    torch.cuda.synchronize()
    sync()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    s2.wait_event(e0)
    for _ in range(3):
        with torch.cuda.stream(s):
            d.copy_(h, non_blocking=True)
        with torch.cuda.stream(s2):
            h2.copy_(d2, non_blocking=True)
    s.wait_stream(s2)
    e1.record(s)
    e1.synchronize()
    out["bidir_total"] = 6 * GIB / (e0.elapsed_time(e1) * 1e6)
    del h, d, h2, d2
    if dist is not None and dist.world > 1:   # all ranks at once: the aggregate the replicas can reach
        out["bidir_total_all_ranks"] = dist.sum(out["bidir_total"])
        out["h2d_all_ranks"] = dist.sum(out["h2d"])
        out["d2h_all_ranks"] = dist.sum(out["d2h"])
    return out


def host_facts():
    """The box the numbers were taken on: CPU count / model, memory, NUMA nodes, the
    GPU's NUMA node."""
    import platform
    f = {"cpus": os.cpu_count(), "machine": platform.machine()}
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                f["cpu_model"] = line.split(":", 1)[1].strip()
                break
        for line in open("/proc/meminfo"):
            if line.startswith("MemTotal"):
                f["mem_gib"] = round(int(line.split()[1]) / 2**20, 1)
                break
        f["numa_nodes"] = len([d for d in os.listdir("/sys/devices/system/node") if d.startswith("node")])
    except OSError:
        pass
    f["all_core_host_memcpy_GBps"] = host_memcpy_ceiling()
    try:   # how the GPUs reach the host and each other (PCIe switches shared by GPUs bound the replicas)
        r = subprocess.run(["nvidia-smi", "topo", "-m"], capture_output=True, text=True, timeout=30)
        import re
        f["nvidia_smi_topo"] = [" ".join(l.split()) for l in re.sub(r"\x1b\[[0-9;]*m", "", r.stdout).splitlines()
                                if l.strip() and not l.lstrip().startswith(("Legend", "X ", "SYS", "NODE", "PHB",
                                                                            "PXB", "PIX", "NV#"))][:20]
    except (OSError, subprocess.SubprocessError):
        pass
    return f


def host_memcpy_ceiling(mib=256, reps=4):
    """Context row: all-core host memcpy GB/s (one thread per core, each copying its
    own 256 MiB buffer; NumPy releases the GIL), counting read + write bytes like the oracle's GB/s
    counts payload only once per direction -- here payload bytes copied."""
    import threading
    n = os.cpu_count() or 1
    bufs = [(np.ones(mib << 20, np.uint8), np.ones(mib << 20, np.uint8)) for _ in range(n)]

    def work(a, b):
        for _ in range(reps):
            np.copyto(b, a)
    ths = [threading.Thread(target=work, args=ab) for ab in bufs]
    t0 = time.perf_counter()
    for t in ths:
        t.start()
    for t in ths:
        t.join()
    dt = time.perf_counter() - t0
    return round(n * reps * (mib << 20) / dt / 1e9, 1)


def model_caches(names):
    """Host Model Caches (pageable) with generated bf16 content."""
    import aeg_inputs as gi
    from aeg_inputs import dev as D
    descs, caches = {}, {}
    for m, nm in enumerate(names):
        ts = gi.model_tensors(nm)
        sizes = [t["rows"] * t["cols"] * 2 for t in ts]
        offs = np.cumsum([0] + [-(-s // 256) * 256 for s in sizes])
        buf = np.empty(int(offs[-1]), dtype=np.uint8)
        for k, (o, s) in enumerate(zip(offs, sizes)):
            D.host_fill(buf[o:o + s], gi.w_seed(3), gi.weight_key(m, k), threads=16)
        caches[nm] = buf
        descs[nm] = [dict(host_src=buf.ctypes.data + int(o), rows=t["rows"], cols=t["cols"], elem_bytes=2,
                          layer=t["layer"], split=t["split"], groups=t["groups"]) for t, o in zip(ts, offs)]
    return descs, caches


def switch_leg(aeg, torch, n_switch, kernel, descs, mode="staged", caches=None, kv_out="after"):
    """configs[3]: token-level switch among Qwen-1.8B / Llama-7B / Yi-9B shapes on one GPU.
    staged  : switch(A->B) = swap-out of A's 1 GiB decode KV (D2H) || staging of B's weights through
              the pinned Stage Buffer (H2D, Fig. 9 3.a) -> swap-in of B's KV.
    prefetch: B's weights were prefetched right after A's in the weights region during A's turn
              (Fig. 8(b)); the switch relocates them to the buffer start on the
              device (Fig. 9 3.b, N1) || A's KV out -> B's KV in; then C's prefetch starts.
    Latency = switch start -> last (first) layer ready for a per-layer consumer that waits on the
    weights layer l+1 (and 0) and KV layer l, on the device timeline (CUDA events)."""
    import aeg_inputs as gi
    from aeg_inputs import dev as D
    names = list(descs)
    shapes = {n: gi.KV_SHAPES[n] for n in names}
    wsize = {nm: sum(d["rows"] * d["cols"] * 2 + 255 & ~255 for d in descs[nm]) for nm in names}
    wmax = max(wsize.values())
    region = wmax + 64 * MIB if mode == "staged" else 2 * wmax + 128 * MIB
    cfg = aeg.default_config(device_kv_bytes=8 * GIB, host_kv_bytes=8 * GIB, device_weight_bytes=region,
                             kernel=kernel, host_threads=12)
    if int(os.environ.get("AEG_STAGE_CHUNK_MIB", "0")):
        cfg.stage_chunk_bytes = int(os.environ["AEG_STAGE_CHUNK_MIB"]) * MIB
    ctx = aeg.Context(0, cfg)
    reg_s = None
    if mode == "direct":   # page-lock the Model Caches once ("no pinning during scaling")
        t0 = time.time()
        for nm in names:
            ctx.host_register(caches[nm].ctypes.data, caches[nm].nbytes)
        reg_s = time.time() - t0
    kv = {}
    for nm in names:
        sh = shapes[nm]
        n = GIB // (sh[0] * 2 * sh[1] * sh[2] * sh[3] * sh[4])
        kv[nm] = (ctx.kv_alloc(aeg.POOL_HOST, sh, n), n)
    cur = names[0]
    db = ctx.kv_alloc(aeg.POOL_DEVICE, shapes[cur], kv[cur][1])
    y = ctx.kv_swap_in(shapes[cur], kv[cur][0], db, flags=aeg.FREE_SRC)
    ctx.layer_ready(y, -1, aeg.READY_BLOCK)
    kv[cur] = (db, kv[cur][1])
    offs, x = ctx.weights_stage(descs[cur])
    ctx.layer_ready(x, -1, aeg.READY_BLOCK)
    pre = None   # (model, xfer, offset of its first tensor)
    if mode == "prefetch":
        ctx.weights_reset(-(-wsize[cur] // 256) * 256)
        o, xp = ctx.weights_stage(descs[names[1]])
        pre = (names[1], xp, int(o[0]), o)
    cons = new_stream(torch)
    res = []
    diag_ms = None
    order = [names[(i + 1) % len(names)] for i in range(n_switch + 3)]
    for i, nxt in enumerate(order):
        if pre is not None:   # the decode turn of `cur` hides the prefetch
            ctx.layer_ready(pre[1], -1, aeg.READY_BLOCK)
        e0 = torch.cuda.Event(enable_timing=True)
        e0.record(cons)
        ctx.stream_fence(cons.cuda_stream)

        def a_kv_out(a=cur):                                                           # A's KV out (D2H)
            hb = ctx.kv_alloc(aeg.POOL_HOST, shapes[a], kv[a][1])
            x = ctx.kv_swap_out(shapes[a], kv[a][0], hb, flags=aeg.FREE_SRC)
            kv[a] = (hb, kv[a][1])
            return x
        xo = a_kv_out() if kv_out == "concurrent" else None
        # B's KV goes first: the copy engine serves one busy H2D stream until it drains
        # (profiles/r01/ce_probe.txt), so KV queued behind a model's weights would land last
        nsh = shapes[nxt]
        db = ctx.kv_alloc(aeg.POOL_DEVICE, nsh, kv[nxt][1])
        xi = ctx.kv_swap_in(nsh, kv[nxt][0], db, flags=aeg.FREE_SRC)                  # B's KV in
        kv[nxt] = (db, kv[nxt][1])
        if mode in ("staged", "direct"):
            ctx.weights_reset(0)
            wo, xw = ctx.weights_stage(descs[nxt])                                     # B's weights in
            wl = lambda l: min(l, ctx.xfer_layers(xw) - 1)  # noqa: E731
        else:
            assert pre[0] == nxt
            xw = ctx.weights_relocate(pre[2], 0, wsize[nxt])                           # 3.b: on-device copy
            wo = [int(x) - pre[2] for x in pre[3]]
            ctx.xfer_release(pre[1])
            wl = lambda l: 0  # noqa: E731
        diag = {}
        if i == 3:   # one switch: when does each piece land (device timeline, separate streams)?
            # KV probes first: a weights-layer wait blocks the host until the pipeline records it
            probes = {"kv_l0": (xi, 0), "kv_last": (xi, nsh[0] - 1), "kv_out_all": (xo, -1),
                      "weights_l0": (xw, wl(0)), "weights_l1": (xw, wl(1)), "weights_all": (xw, -1)}
            if xo is None:
                del probes["kv_out_all"]
            for name, (xx, l) in probes.items():
                ds = new_stream(torch)
                ctx.layer_ready(xx, l, aeg.READY_WAIT_STREAM, ds.cuda_stream)
                de = torch.cuda.Event(enable_timing=True)
                de.record(ds)
                diag[name] = de
        ev = []
        for l in range(nsh[0]):
            if l == 0:
                ctx.layer_ready(xw, wl(0), aeg.READY_WAIT_STREAM, cons.cuda_stream)
            ctx.layer_ready(xw, wl(l + 1), aeg.READY_WAIT_STREAM, cons.cuda_stream)
            ctx.layer_ready(xi, l, aeg.READY_WAIT_STREAM, cons.cuda_stream)
            e = torch.cuda.Event(enable_timing=True)
            e.record(cons)
            ev.append(e)
        ctx.layer_ready(xw, -1, aeg.READY_WAIT_STREAM, cons.cuda_stream)
        e_end = torch.cuda.Event(enable_timing=True)
        e_end.record(cons)
        if xo is None:
            # PCIe duplex costs each direction ~10 % here (bidirectional memcpy ~99 GB/s total vs
            # 55-57 one way), so A's KV-out waits until B has landed and overlaps B's decode
            # instead of B's load (ordered after the consumer stream: aeg_stream_fence)
            ctx.stream_fence(cons.cuda_stream)
            xo = a_kv_out()
            if diag:
                ds = new_stream(torch)
                ctx.layer_ready(xo, -1, aeg.READY_WAIT_STREAM, ds.cuda_stream)
                de = torch.cuda.Event(enable_timing=True)
                de.record(ds)
                diag["kv_out_all"] = de
        e_end.synchronize()
        for xx in (xo, xw, xi):
            ctx.layer_ready(xx, -1, aeg.READY_BLOCK)
            ctx.xfer_release(xx)
        kvb = kv[nxt][1] * nsh[0] * 2 * nsh[1] * nsh[2] * nsh[3] * nsh[4]
        if diag:
            torch.cuda.synchronize()
            diag_ms = {k: round(e0.elapsed_time(v), 2) for k, v in diag.items()}
            diag_ms["to"] = nxt
        if i >= 3:
            res.append(dict(to=nxt, first_ms=e0.elapsed_time(ev[0]), last_ms=e0.elapsed_time(e_end),
                            bytes_h2d=(0 if mode == "prefetch" else wsize[nxt]) + kvb))
        if i == len(order) - 1:   # bit-exact check of the running model's weights (TP=1: the tensors)
            base, _, _ = ctx.weights_region()
            m = names.index(nxt)
            bad = 0
            for k in (0, len(descs[nxt]) // 2, len(descs[nxt]) - 1):
                d = descs[nxt][k]
                nb = d["rows"] * d["cols"] * 2
                o = int(wo[k])
                got = D.read(base + o, min(nb, 1 << 24))
                exp = gi.region_bytes(gi.w_seed(3), gi.weight_key(m, k), min(nb, 1 << 24))
                bad += int((got != exp).sum())
        cur = nxt
        if mode == "prefetch":   # next turn: prefetch the model after `cur` behind it
            nn = names[(names.index(cur) + 1) % len(names)]
            ctx.weights_reset(-(-wsize[cur] // 256) * 256)
            o, xp = ctx.weights_stage(descs[nn])
            pre = (nn, xp, int(o[0]), o)
    if pre is not None:
        ctx.layer_ready(pre[1], -1, aeg.READY_BLOCK)
    wchunks, wfill, wslot = ctx.weights_stats()
    ctx.shutdown()
    per = {}
    for nm in names:
        r = [x for x in res if x["to"] == nm]
        if not r:
            continue
        lat = sorted(x["last_ms"] for x in r)
        per[nm] = {"switches": len(r), "last_layer_ms_p50": round(statistics.median(lat), 2),
                   "last_layer_ms_p90": round(lat[int(0.9 * (len(lat) - 1))], 2),
                   "first_layer_ms_p50": round(statistics.median(x["first_ms"] for x in r), 2),
                   "h2d_bytes": int(r[0]["bytes_h2d"]), "weights_bytes": int(wsize[nm]),
                   "h2d_GBps": round(r[0]["bytes_h2d"] / (statistics.median(lat) * 1e6), 1),
                   # N4: Eq. 4 (garbled) predicted and solved for beta on this B200,
                   # under both readings: literal T = size / BW * beta, and DESIGN reading 19
                   # T = size / (BW * beta) (an inefficiency lengthens T); paper beta = 0.625
                   "eq4_weights_ms_at_64GBps": {
                       "literal": round(wsize[nm] / PCIE_NOMINAL * BETA / 1e6, 1),
                       "reading19": round(wsize[nm] / (PCIE_NOMINAL * BETA) / 1e6, 1)},
                   "eq4_beta_fit": None if mode == "prefetch" else {
                       "literal": round(PCIE_NOMINAL * 1e9 * statistics.median(lat) / 1e3 / wsize[nm], 3),
                       "reading19": round(wsize[nm] / (PCIE_NOMINAL * 1e9 * statistics.median(lat) / 1e3), 3),
                       "reading19_all_h2d_bytes": round(r[0]["bytes_h2d"] / (PCIE_NOMINAL * 1e9 * statistics.median(lat) / 1e3), 3),
                       "what": "size = the model's weight bytes (Eq. 4's Model Size), T = last-layer-ready "
                               "latency of the switch, which also carries 1 GiB of KV over the same H2D link; "
                               "reading19_all_h2d_bytes uses weights + KV bytes (the link's own efficiency)"}}
    how = {"staged": "weights staged through the 2 GiB pinned Stage Buffer by host threads (3.a)",
           "direct": "weights DMA'd straight from the page-locked Model Cache (registered once)",
           "prefetch": "weights prefetched during the previous turn, relocated on-device at the switch (3.b)"}[mode]
    return {"workload": f"configs[3] 3-model switch (Qwen-1.8B, Llama-7B, Yi-9B shapes), 1 GiB KV each; {how}; "
                        f"A's KV out {'after B has landed' if kv_out == 'after' else 'concurrent with B loading'}",
            "per_model": per, "weights_bit_exact_sample": bad == 0, "register_s": reg_s,
            "landing_ms_one_switch": diag_ms,
            "weight_pipeline": {"chunks": wchunks, "issuer_wait_fill_ms": round(wfill, 1),
                                "fill_wait_slot_ms": round(wslot, 1)}}


def migrate_leg(aeg, torch, kernel, n_req=16, src_layout=None, dst_layout=None):
    """configs[2] shapes on one GPU: Llama-2-13B KV hand-off through the fused migrate kernel into
    another context's pool (peer mapped in-process, the same kernel that stores over NVLink when the
    peer is another GPU).  Checked against the generator at the destination blocks' chunks (identity
    under relabelling), located through the library's block table."""
    import aeg_inputs as gi
    from aeg_inputs import dev as D
    sht = gi.KV_SHAPES["llama-2-13b"]
    sh = aeg.KVShape.of(sht)
    lens = gi.request_lengths(3, n_req, 512, 4096)
    n = sum(-(-t // 16) for t in lens)
    slab = 1 * GIB + 256 * MIB
    nslab = -(-n // (slab // sh.block_bytes())) + 1
    mk = lambda lay: aeg.Context(0, aeg.default_config(device_kv_bytes=nslab * slab, host_kv_bytes=GIB,  # noqa: E731
                                                       dev_slab_bytes=slab, dev_slab_layout=lay, kernel=kernel,
                                                       flags=aeg.CFG_TIMING))
    a = mk(aeg.LAYER_MAJOR if src_layout is None else src_layout)
    b = mk(aeg.BLOCK_MAJOR if dst_layout is None else dst_layout)
    sc = a.kv_alloc(0, sht, n)
    dc = b.kv_alloc(0, sht, n)
    abase, _ = a.pool_region(0)
    bbase, _ = b.pool_region(0)
    seed = gi.kv_seed(3)
    offs = chunk_offsets(a, 0, sht, sc)
    keys = [gi.kv_key(1, i // 4096, i % 4096, l) for i in range(n) for l in range(sh.num_layers)]
    D.fill_chunks(abase, offs, keys, sh.chunk_bytes(), seed)
    a.import_peer(1, b.export_ipc())

    def timed(reps, flags=0):
        out = []
        for it in range(reps + 2):
            a.kernel_stats_reset()
            s = new_stream(torch)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            a.stream_fence(s.cuda_stream)
            x = a.kv_migrate(sht, sc, 1, dc, flags=flags)
            a.layer_ready(x, -1, aeg.READY_WAIT_STREAM, s.cuda_stream)
            e1.record(s)
            e1.synchronize()
            a.xfer_release(x)
            if it >= 2:
                out.append(e0.elapsed_time(e1))
        return out

    # SM budget of the hand-off (aeg_set_migrate_ctas): CTAs of 256 threads, ~one per SM up to 148
    sweep = {}
    for ctas in (8, 16, 32, 64, 148):
        a.set_migrate_ctas(ctas)
        sweep[ctas] = round(n * sh.block_bytes() / (min(timed(2)) * 1e6), 1)
    a.set_migrate_ctas(0)
    ce_ms = min(timed(2, aeg.MIGRATE_CE))   # copy-engine route: gather kernel + CE D2D commands
    doffs = chunk_offsets(b, 0, sht, dc)
    bad_ce, _ = D.verify_chunks(bbase, doffs, keys, sh.chunk_bytes(), seed)
    D.fill_chunks(bbase, doffs, [gi.poison_key(gi.TAG_DST, int(o)) for o in doffs], sh.chunk_bytes(), seed)
    times = timed(4)
    nl, nbytes, kms = a.kernel_stats(aeg.K_MIGRATE)
    bad, _ = D.verify_chunks(bbase, doffs, keys, sh.chunk_bytes(), seed)
    # baseline on the same blocks: one cudaMemcpyAsync (copy engine, D2D) per (block, layer) chunk
    s = new_stream(torch)
    bt = []
    for _ in range(2):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        D.copy_chunks(bbase, doffs, abase, offs, sh.chunk_bytes(), s.cuda_stream)
        e1.record(s)
        e1.synchronize()
        bt.append(e0.elapsed_time(e1))
    a.shutdown()
    b.shutdown()
    payload = n * sh.block_bytes()
    ms = statistics.median(times)
    return {"workload": f"configs[2] Llama-2-13B hand-off, {n_req} requests ({n} blocks), 1 GPU (peer pool "
                        "in-process; NVLink path needs >= 2 GPUs)",
            "payload_bytes": payload, "ms": round(ms, 3), "GBps_payload": round(payload / (ms * 1e6), 1),
            "hbm_GBps": round(2 * payload / (ms * 1e6), 1), "kernel_launches_per_xfer": nl,
            "kernel_ms_per_xfer": round(kms, 3), "bit_exact": bad == 0,
            "GBps_payload_by_ctas": sweep,
            "ce_route_GBps_payload": round(payload / (ce_ms * 1e6), 1), "ce_route_bit_exact": bad_ce == 0,
            "per_chunk_memcpy_baseline_GBps_payload": round(payload / (min(bt) * 1e6), 1),
            "per_chunk_memcpy_calls": int(len(offs))}


def migrate_leg_two_device(aeg, torch, kernel, n_req=16):
    """configs[2] between two GPUs of ONE process (rank 0 of an N >= 2 run, every GPU visible): the
    prefill context on cuda:0 migrates n_req Llama-2-13B requests into the pool of a decode context
    on cuda:1 mapped directly (aeg_import_peer's same-process cross-device branch:
    cudaDeviceEnablePeerAccess, 16-byte stores into the peer aperture over NVLink).  Reports GB/s
    by CTA budget and the smallest budget reaching 0.70 x 900 GB/s; bit-exact at the destination."""
    import aeg_inputs as gi
    from aeg_inputs import dev as D
    if torch.cuda.device_count() < 2:
        return {"skipped": "needs two visible GPUs"}
    sht = gi.KV_SHAPES["llama-2-13b"]
    sh = aeg.KVShape.of(sht)
    lens = gi.request_lengths(3, n_req, 512, 4096)
    n = sum(-(-t // 16) for t in lens)
    slab = GIB + 256 * MIB
    nslab = -(-n // (slab // sh.block_bytes())) + 1
    mk = lambda dev, lay: aeg.Context(dev, aeg.default_config(  # noqa: E731
        device_kv_bytes=nslab * slab, host_kv_bytes=GIB, dev_slab_bytes=slab, dev_slab_layout=lay, kernel=kernel,
        flags=aeg.CFG_TIMING))
    a = mk(0, aeg.LAYER_MAJOR)
    b = mk(1, aeg.BLOCK_MAJOR)
    try:
        sc, dc = a.kv_alloc(0, sht, n), b.kv_alloc(0, sht, n)
        abase, _ = a.pool_region(0)
        bbase, _ = b.pool_region(0)
        seed = gi.kv_seed(3)
        keys = [gi.kv_key(1, 7, i, l) for i in range(n) for l in range(sh.num_layers)]
        torch.cuda.set_device(0)
        D.fill_chunks(abase, chunk_offsets(a, 0, sht, sc), keys, sh.chunk_bytes(), seed)
        D.sync()
        a.import_peer(1, b.export_ipc())
        s = torch.cuda.Stream(device=0)

        def timed(reps, flags=0):
            out = []
            for it in range(reps + 1):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(s)
                a.stream_fence(s.cuda_stream)
                x = a.kv_migrate(sht, sc, 1, dc, flags=flags)
                a.layer_ready(x, -1, aeg.READY_WAIT_STREAM, s.cuda_stream)
                e1.record(s)
                e1.synchronize()
                a.xfer_release(x)
                if it:
                    out.append(e0.elapsed_time(e1))
            return out
        payload = n * sh.block_bytes()
        sweep = {}
        for ctas in (8, 16, 32, 48, 64, 96, 148):
            a.set_migrate_ctas(ctas)
            sweep[ctas] = round(payload / (min(timed(2)) * 1e6), 1)
        a.set_migrate_ctas(0)
        ce_ms = min(timed(2, aeg.MIGRATE_CE))
        ms = statistics.median(timed(4))
        torch.cuda.set_device(1)
        bad, _ = D.verify_chunks(bbase, chunk_offsets(b, 0, sht, dc), keys, sh.chunk_bytes(), seed)
        torch.cuda.set_device(0)
        ok = [c for c, v in sorted(sweep.items()) if v >= 0.70 * NVLINK_NOMINAL]
        return {"workload": f"configs[2] Llama-2-13B hand-off, {n_req} requests ({n} blocks), cuda:0 -> cuda:1 in "
                            "one process (direct peer mapping, NVLink)",
                "payload_bytes": payload, "ms": round(ms, 3), "GBps": round(payload / (ms * 1e6), 1),
                "frac_of_nvlink_nominal": round(payload / (ms * 1e6) / NVLINK_NOMINAL, 3),
                "GBps_by_ctas": sweep, "ctas_for_70pct_nvlink": ok[0] if ok else None, "bit_exact": bad == 0,
                "ce_route_GBps": round(payload / (ce_ms * 1e6), 1),
                "ce_route_frac_of_measured_peer_copy": round(payload / (ce_ms * 1e6) / NVLINK_PEER_COPY, 3)}
    finally:
        torch.cuda.set_device(0)
        a.shutdown()
        b.shutdown()


def _nccl_sendrecv(torch, dist, pairs, nbytes, reps=4):
    """NCCL point-to-point of one hand-off's payload as ONE contiguous buffer per pair (no block
    tables, no gather/scatter: an upper bound for an NCCL-based hand-off).  Max-over-ranks device
    time of the median rep."""
    td = dist.td
    rank = dist.rank
    peer = {a_: b_ for a_, b_ in pairs}
    peer.update({b_: a_ for a_, b_ in pairs})
    buf = torch.empty(nbytes, dtype=torch.uint8, device="cuda") if rank in peer else None
    ts = []
    for _ in range(reps + 1):   # every rank takes part in the barrier / max, paired or not
        dist.barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        if buf is not None and any(a_ == rank for a_, _ in pairs):
            td.send(buf, peer[rank])
        elif buf is not None:
            td.recv(buf, peer[rank])
        e1.record()
        e1.synchronize()
        ts.append(dist.max(e0.elapsed_time(e1)))
    del buf
    ms = statistics.median(ts[1:])
    return {"ms": round(ms, 3), "GBps_per_pair": round(nbytes / (ms * 1e6), 1)}


def migrate_leg_dist(aeg, torch, dist, kernel, n_req=16):
    """configs[2] across GPUs: prefill rank i hands n_req Llama-2-13B-shaped requests to decode rank
    i + N/2 over NVLink/NVSwitch (fused gather -> remote 16-byte stores), per-layer IPC events.
    Aggregate GB/s = all pairs' payload / max-over-ranks device time."""
    import aeg_inputs as gi
    from aeg_inputs import dev as D
    from paper_conf_sosp_xiang0qyzyzl0025_b200 import dist as PD
    world, rank = dist.world, dist.rank
    sht = gi.KV_SHAPES["llama-2-13b"]
    sh = aeg.KVShape.of(sht)
    lens = gi.request_lengths(3, n_req, 512, 4096)
    n = sum(-(-t // 16) for t in lens)
    slab = GIB + 256 * MIB
    nslab = -(-n // (slab // sh.block_bytes())) + 1
    cfg = aeg.default_config(device_kv_bytes=nslab * slab, host_kv_bytes=GIB, dev_slab_bytes=slab,
                             dev_slab_layout=aeg.LAYER_MAJOR if PD.role(rank, world) == "prefill" else aeg.BLOCK_MAJOR,
                             kernel=kernel, flags=aeg.CFG_TIMING)
    ctx = aeg.Context(dist.device, cfg)
    base, _ = ctx.pool_region(0)
    seed = gi.kv_seed(3)
    PD.connect(ctx, rank)
    prefill = PD.role(rank, world) == "prefill"
    dst = None if prefill else [int(b) for b in ctx.kv_alloc(0, sht, n)]
    handles = PD.exchange(dst)
    pairs = PD.handoff_pairs(world)
    src = None
    if prefill:
        src = ctx.kv_alloc(0, sht, n)
        offs = chunk_offsets(ctx, 0, sht, src)
        keys = [gi.kv_key(1, rank, i, l) for i in range(n) for l in range(sh.num_layers)]
        D.fill_chunks(base, offs, keys, sh.chunk_bytes(), seed)
    dst_by_rank = {d: np.array(h, np.uint64) for d, h in enumerate(handles) if h}

    def hand_off(round_pairs):
        """One timed round: every prefill rank migrates to its partner; the decode side waits per
        layer on the imported IPC events.  Returns the max-over-ranks device time (ms)."""
        dist.barrier()
        ms = 0.0
        xs = {}
        if prefill:
            s = new_stream(torch)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            ctx.stream_fence(s.cuda_stream)
            xs = PD.handoff(ctx, sht, src, round_pairs, rank, dst_by_rank)
            for x in xs.values():
                ctx.layer_ready(x, -1, aeg.READY_WAIT_STREAM, s.cuda_stream)
            e1.record(s)
            e1.synchronize()
            ms = e0.elapsed_time(e1)
        blobs = PD.exchange({d: ctx.xfer_export(x) for d, x in xs.items()})
        if not prefill:
            for sender, m in enumerate(blobs):
                if m and rank in m:
                    xi = ctx.xfer_import(sender, m[rank])
                    for l in range(sh.num_layers):
                        ctx.layer_ready(xi, l, aeg.READY_BLOCK)
                    ctx.xfer_release(xi)
        for x in xs.values():
            ctx.xfer_release(x)
        return dist.max(ms)

    ctx.kernel_stats_reset()
    times = [hand_off(pairs) for _ in range(5)][1:]
    kl, kb, kms = ctx.kernel_stats(aeg.K_MIGRATE)   # prefill ranks: 5 rounds of migrate launches
    k_gbps = dist.max(kb / 2 / (kms * 1e6) if kms > 0 else 0.0)   # payload bytes over the link
    sweep = {}   # SM budget of the hand-off: how many SMs saturate the link
    for ctas in (8, 16, 32, 64, 148):
        ctx.set_migrate_ctas(ctas)
        sweep[ctas] = round(len(pairs) * n * sh.block_bytes() / (min(hand_off(pairs) for _ in range(2)) * 1e6), 1)
    ctx.set_migrate_ctas(0)
    per_pair_target = 0.70 * NVLINK_NOMINAL
    ok_ctas = [c for c, v in sorted(sweep.items()) if v / len(pairs) >= per_pair_target]
    bad = 0
    if not prefill:
        sender = [s_ for s_, d in pairs if d == rank][0]
        offs = chunk_offsets(ctx, 0, sht, dst)
        keys = [gi.kv_key(1, sender, i, l) for i in range(n) for l in range(sh.num_layers)]
        bad, _ = D.verify_chunks(base, offs, keys, sh.chunk_bytes(), seed)
    bad = dist.sum(bad)
    # the library's copy-engine route (AEG_MIGRATE_CE: gather kernel + CE commands over NVLink, no
    # SMs on the decode GPU), every pair at once, max-over-ranks device time
    lib_err = []

    def ce_lib_round():
        dist.barrier()
        ms = 0.0
        if prefill and not lib_err:
            try:
                s = new_stream(torch)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(s)
                ctx.stream_fence(s.cuda_stream)
                xs = PD.handoff(ctx, sht, src, pairs, rank, dst_by_rank, flags=aeg.MIGRATE_CE)
                for x in xs.values():
                    ctx.layer_ready(x, -1, aeg.READY_WAIT_STREAM, s.cuda_stream)
                e1.record(s)
                e1.synchronize()
                for x in xs.values():
                    ctx.xfer_release(x)
                ms = e0.elapsed_time(e1)
            except Exception as e:  # noqa: BLE001  (every rank must still reach the max below)
                lib_err.append(f"{type(e).__name__}: {e}")
                ms = -1e9
        return dist.max(ms)
    lib_ce_ms = min(ce_lib_round() for _ in range(3))
    lib_failed = dist.sum(1 if lib_err else 0)
    lib_ce = ({"error": lib_err[0] if lib_err else "failed on another rank"} if lib_failed or lib_ce_ms <= 0 else
              {"GBps_aggregate": round(len(pairs) * n * sh.block_bytes() / (lib_ce_ms * 1e6), 1),
               "GBps_per_pair": round(n * sh.block_bytes() / (lib_ce_ms * 1e6), 1),
               "what": "aeg_kv_migrate(AEG_MIGRATE_CE): gather kernel into staging, copy-engine commands "
                       "into the peer pool"})
    # CE-vs-SM: the same chunks paged -> paged, one cudaMemcpyAsync per (block,
    # layer) chunk (copy engines, zero SMs) into the partner's pool mapped here (aeg_peer_region);
    # decode ranks send their chunk offsets.  Max-over-ranks device time of one round, all pairs.
    doffs_by_rank = PD.exchange(None if prefill else chunk_offsets(ctx, 0, sht, dst).tolist())
    ce_err = []

    def ce_round():
        dist.barrier()
        ms = 0.0
        if prefill and not ce_err:
            try:
                d = [d_ for s_, d_ in pairs if s_ == rank][0]
                pbase, _ = ctx.peer_region(d)
                s = new_stream(torch)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(s)
                D.copy_chunks(pbase, np.asarray(doffs_by_rank[d], np.uint64), base, offs, sh.chunk_bytes(),
                                    s.cuda_stream)
                e1.record(s)
                e1.synchronize()
                ms = e0.elapsed_time(e1)
            except Exception as e:  # noqa: BLE001  (every rank must still reach the max below)
                ce_err.append(f"{type(e).__name__}: {e}")
                ms = -1e9
        return dist.max(ms)
    ce_ms = min(ce_round() for _ in range(3))
    failed = dist.sum(1 if ce_err else 0)
    ce = ({"error": ce_err[0] if ce_err else "failed on another rank"} if failed or ce_ms <= 0 else
          {"GBps_aggregate": round(len(pairs) * n * sh.block_bytes() / (ce_ms * 1e6), 1),
           "what": "one cudaMemcpyAsync per (block, layer) chunk into the peer pool, copy engines only"})
    # SURVEY §8(d) C3 for N >= 4: all-to-all, every prefill rank -> every decode rank, round-robin
    a2a = None
    if world >= 4:
        h = world // 2
        t_rounds = [hand_off(PD.handoff_pairs(world, "all2all", r)) for r in range(h)]
        a2a = {"rounds": h, "ms_total": round(sum(t_rounds), 3),
               "GBps_aggregate": round(h * len(pairs) * n * sh.block_bytes() / (sum(t_rounds) * 1e6), 1)}
    ctx.shutdown()
    nccl = None
    if dist.backend == "nccl":   # comparison baseline (not the product): NCCL send/recv of the same
        nccl = _nccl_sendrecv(torch, dist, pairs, n * sh.block_bytes())   # payload, contiguous
    ms = statistics.median(times)
    payload = len(pairs) * n * sh.block_bytes()
    return {"workload": f"configs[2] Llama-2-13B hand-off, {n_req} requests per pair, pairs {pairs}",
            "nccl_sendrecv_contiguous_baseline": nccl, "per_chunk_ce_route": ce, "library_ce_route": lib_ce,
            "payload_bytes": payload, "ms": round(ms, 3), "GBps_aggregate": round(payload / (ms * 1e6), 1),
            "GBps_per_pair": round(payload / len(pairs) / (ms * 1e6), 1), "peak_per_direction_nominal": NVLINK_NOMINAL,
            "frac_of_nvlink_nominal_per_pair": round(payload / len(pairs) / (ms * 1e6) / NVLINK_NOMINAL, 3),
            "frac_of_measured_peer_copy_per_pair": round(payload / len(pairs) / (ms * 1e6) / NVLINK_PEER_COPY, 3),
            "kernel_GBps_payload_max_rank": round(k_gbps, 1), "kernel_launches_per_xfer": int(kl // 5) if kl else 0,
            "GBps_aggregate_by_ctas": sweep,
            "ctas_for_70pct_nvlink_per_pair": ok_ctas[0] if ok_ctas else None,
            "bit_exact": bad == 0, "all_to_all": a2a}


def _host_route_geometry(aeg, n_req):
    import aeg_inputs as gi
    sht = gi.KV_SHAPES["llama-2-13b"]
    sh = aeg.KVShape.of(sht)
    lens = gi.request_lengths(3, n_req, 512, 4096)
    n = sum(-(-t // 16) for t in lens)
    slab = GIB + 256 * MIB
    nslab = -(-n // (slab // sh.block_bytes())) + 1
    return sht, sh, n, slab, nslab


def _dbg(*a):
    if os.environ.get("AEG_DEBUG_ROUTE"):
        print(f"[{os.getpid()} {time.time():.3f}]", *a, file=sys.stderr, flush=True)


def _host_route_decode(conn, n_req):
    """Decode instance D of the host-route leg (a separate process on the same GPU): imports the
    prefill instance's node-shared CPU KV cache once, then per hand-off swaps the request in from
    there (C->D, aeg_kv_swap_in_from) waiting only on P's per-layer IPC events, and stamps the GPU
    clock when its last layer is ready."""
    try:
        import torch
        import aeg_inputs as gi
        from aeg_inputs import dev as D
        import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg
        sht, sh, n, slab, nslab = _host_route_geometry(aeg, n_req)
        ctx = aeg.Context(0, aeg.default_config(device_kv_bytes=nslab * slab, host_kv_bytes=GIB, dev_slab_bytes=slab,
                                                dev_slab_layout=aeg.BLOCK_MAJOR))
        base, _ = ctx.pool_region(0)
        _dbg("D: ctx up")
        ctx.import_peer(0, conn.recv())
        _dbg("D: peer imported")
        t = torch.zeros(1, dtype=torch.int64, device="cuda")
        s = new_stream(torch)
        D.stamp(t.data_ptr(), s.cuda_stream)   # load every kernel now: a module load later would wait
        s.synchronize()                        # behind P's gate kernel
        conn.send("ready")
        keys = np.array([gi.kv_key(1, i // 4096, i % 4096, l) for i in range(n) for l in range(sh.num_layers)], np.uint64)
        while True:
            m = conn.recv()
            if m == "bye":
                break
            hb, xblob = m
            xo = ctx.xfer_import(0, xblob)
            _dbg("D: events imported")
            dc = ctx.kv_alloc(0, sht, n)
            xi = ctx.kv_swap_in_from(sht, 0, np.array(hb, dtype=np.uint64), dc, after=xo)       # ③④⑤
            _dbg("D: swap-in enqueued")
            ctx.layer_ready(xi, -1, aeg.READY_WAIT_STREAM, s.cuda_stream)
            D.stamp(t.data_ptr(), s.cuda_stream)
            conn.send(ctx.xfer_export(xi))
            _dbg("D: exported")
            s.synchronize()
            bad, _ = D.verify_chunks(base, chunk_offsets(ctx, 0, sht, dc), keys, sh.chunk_bytes(), gi.kv_seed(3))
            ctx.xfer_release(xi)
            ctx.xfer_release(xo)
            ctx.kv_free(0, dc)
            conn.send((int(t.item()), int(bad)))
        ctx.shutdown()
    except BaseException:
        import traceback
        conn.send(("error", traceback.format_exc()))


def host_route_leg(aeg, torch, kernel, n_req=4, reps=4):
    """NEXT-2, the paper's own P->C->D route (Fig. 10) measured: prefill instance
    P (this process) swaps a hand-off of n_req Llama-2-13B requests out to its part of the node-shared
    pinned CPU KV cache (P->C), decode instance D (another process, same GPU) swaps it in from there
    (C->D) with per-layer IPC-event waits, so the two PCIe directions overlap layer by layer; P keeps
    the CPU blocks in its move list until D's swap-in completes (aeg_kv_free_after).  Latency = GPU
    clock from P's start to D's last layer ready (%globaltimer, shared by both processes)."""
    import multiprocessing as mp
    import aeg_inputs as gi
    from aeg_inputs import dev as D
    sht, sh, n, slab, nslab = _host_route_geometry(aeg, n_req)
    a = aeg.Context(0, aeg.default_config(device_kv_bytes=nslab * slab, host_kv_bytes=nslab * slab,
                                          dev_slab_bytes=slab, host_slab_bytes=slab, kernel=kernel,
                                          flags=aeg.CFG_SHARED_HOST))
    cm = mp.get_context("spawn")
    parent, child = cm.Pipe()
    p = cm.Process(target=_host_route_decode, args=(child, n_req))
    p.start()
    child.close()

    def recv():
        if not parent.poll(300):
            raise RuntimeError("decode process did not answer")
        m = parent.recv()
        if isinstance(m, tuple) and len(m) == 2 and m[0] == "error":
            raise RuntimeError("decode process failed:\n" + m[1])
        return m

    res = []
    try:
        abase, _ = a.pool_region(0)
        src = a.kv_alloc(0, sht, n)
        keys = [gi.kv_key(1, i // 4096, i % 4096, l) for i in range(n) for l in range(sh.num_layers)]
        D.fill_chunks(abase, chunk_offsets(a, 0, sht, src), keys, sh.chunk_bytes(), gi.kv_seed(3))
        D.sync()
        parent.send(a.export_ipc())
        if recv() != "ready":
            raise RuntimeError("decode process handshake")
        ts = torch.zeros(2, dtype=torch.int64, device="cuda")
        s, s2 = new_stream(torch), new_stream(torch)
        alone = []   # P->C with no concurrent C->D: the shared region's one-direction rate
        for _ in range(3):
            hc = a.kv_alloc(1, sht, n)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            a.stream_fence(s.cuda_stream)
            xo = a.kv_swap_out(sht, src, hc)
            a.layer_ready(xo, -1, aeg.READY_WAIT_STREAM, s.cuda_stream)
            e1.record(s)
            e1.synchronize()
            alone.append(e0.elapsed_time(e1))
            a.xfer_release(xo)
            a.kv_free(1, hc)
            a.reclaim(True)
        gate = D.Gate()
        for _ in range(reps + 1):
            hc = a.kv_alloc(1, sht, n)
            _dbg("P: rep")
            gate.close_on(s.cuda_stream)          # everything is enqueued on both sides before it starts
            D.stamp(ts.data_ptr(), s.cuda_stream)
            a.stream_fence(s.cuda_stream)
            xo = a.kv_swap_out(sht, src, hc)                                                       # ①②
            parent.send(([int(b) for b in hc], a.xfer_export(xo)))
            _dbg("P: swap-out enqueued + sent")
            xd = a.xfer_import(1, recv())
            _dbg("P: D's events imported")
            a.layer_ready(xo, -1, aeg.READY_WAIT_STREAM, s2.cuda_stream)
            D.stamp(ts.data_ptr() + 8, s2.cuda_stream)
            a.kv_free_after(1, hc, xd)            # the CPU blocks stay in P's move list until D is done
            gate.open()
            _dbg("P: gate open")
            t_end, bad = recv()
            _dbg("P: rep done")
            torch.cuda.synchronize()
            t0, t_out = (int(x) for x in ts.tolist())
            a.xfer_release(xo)
            a.xfer_release(xd)
            res.append((t_out - t0, t_end - t0, bad))
        parent.send("bye")
    finally:
        p.join(timeout=60)
        if p.is_alive():
            p.kill()
        a.shutdown()
    res = res[1:]
    b = n * sh.block_bytes()
    out_ns = statistics.median(r[0] for r in res)
    e2e_ns = statistics.median(r[1] for r in res)
    return {"workload": f"configs[2] Llama-2-13B hand-off of {n_req} requests ({n} blocks, {b / GIB:.2f} GiB) through "
                        "the node-shared pinned CPU cache, P and D in two processes on one GPU",
            "p_to_c_ms": round(out_ns / 1e6, 2), "p_to_c_GBps": round(b / out_ns, 1),
            "p_to_c_alone_GBps": round(b / (min(alone[1:]) * 1e6), 1),
            "p_to_c_alone_frac_of_pcie_nominal": round(b / (min(alone[1:]) * 1e6) / PCIE_NOMINAL, 3),
            "p_to_d_ms": round(e2e_ns / 1e6, 2), "p_to_d_GBps": round(b / e2e_ns, 1),
            "both_directions_GBps_over_p_to_d": round(2 * b / e2e_ns, 1),
            "note": "P->C and C->D overlap layer by layer, so p_to_c_GBps is one direction of a duplex "
                    "transfer (this box's duplex memcpy ceiling is in pcie_memcpy_GBps.bidir_total); "
                    "p_to_c_alone_GBps is the same swap-out into the shared region with D idle",
            "bit_exact": all(r[2] == 0 for r in res), "reps": len(res)}


def sparse_model_cache(name, m, tp_rank, tp_size, seed, threads=16, min_sparse=MIB):
    """Host Model Cache of a whole model (pageable) laid out as model_caches()
    does, but only TP rank `tp_rank`'s shard bytes are materialised: the rest of the anonymous
    MAP_NORESERVE mapping is never touched, so a 144.6 GB Qwen-72B cache costs one rank's 36 GB of
    host RAM.  Materialised bytes equal the dense content (the generator is counter-based)."""
    import mmap
    import aeg_inputs as gi
    from aeg_inputs import dev as D
    ts = gi.model_tensors(name)
    sizes = [t["rows"] * t["cols"] * 2 for t in ts]
    offs = np.cumsum([0] + [-(-x // 256) * 256 for x in sizes])
    mm = mmap.mmap(-1, int(offs[-1]), flags=mmap.MAP_PRIVATE | mmap.MAP_ANONYMOUS | getattr(mmap, "MAP_NORESERVE", 0x4000))
    if hasattr(mmap, "MADV_NOHUGEPAGE"):
        mm.madvise(mmap.MADV_NOHUGEPAGE)
    buf = np.frombuffer(mm, dtype=np.uint8)
    base = buf.ctypes.data
    touched = 0
    for k, (t, o, n) in enumerate(zip(ts, offs, sizes)):
        o, rb, key = int(o), t["cols"] * 2, gi.weight_key(m, k)
        if t["split"] == gi.REPLICATED or n < min_sparse or tp_size == 1:
            D.host_fill(buf[o:o + n], seed, key, threads=threads)
            touched += n
        elif t["split"] in (gi.COL, gi.VOCAB):
            g_rows = t["rows"] // t["groups"]
            part = g_rows // tp_size
            for g in range(t["groups"]):
                a = (g * g_rows + tp_rank * part) * rb
                assert a % 8 == 0
                D.host_fill(buf[o + a:o + a + part * rb], seed, key + a // 8, threads=threads)
                touched += part * rb
        else:   # ROW: the rank's column slice of every row
            w = rb // tp_size
            D.host_fill_2d(base + o + tp_rank * w, t["rows"], rb, w, seed, key + tp_rank * w // 8, threads=threads)
            touched += t["rows"] * w
    descs = [dict(host_src=base + int(o), rows=t["rows"], cols=t["cols"], elem_bytes=2, layer=t["layer"],
                  split=t["split"], groups=t["groups"]) for t, o in zip(ts, offs)]
    return descs, (mm, buf), touched


def _c5_check_weights(aeg, ctx, name, m, seed, tp_rank, tp_size, got_offs, picks):
    """Sampled check of staged shards at the offsets the library returned: each expected shard is cut
    from the generator's dense tensor by its split's definition (the row/column ranges the input
    builder materialised).  The oracle's O8 check of the same run is tests/test_gpu_c5.py."""
    import aeg_inputs as gi
    from aeg_inputs import dev as D
    ts = gi.model_tensors(name)
    base, _, _ = ctx.weights_region()
    bad = 0
    for k in picks:
        t = ts[k]
        rows, cb = t["rows"], t["cols"] * 2
        full = gi.region_bytes(seed, gi.weight_key(m, k), rows * cb).reshape(rows, cb)
        if t["split"] == gi.REPLICATED:
            exp = full
        elif t["split"] in (gi.COL, gi.VOCAB):
            g, p = rows // t["groups"], rows // t["groups"] // tp_size
            exp = np.concatenate([full[q * g + tp_rank * p:q * g + (tp_rank + 1) * p] for q in range(t["groups"])])
        else:
            w = cb // tp_size
            exp = full[:, tp_rank * w:(tp_rank + 1) * w]
        exp = np.ascontiguousarray(exp).reshape(-1)
        bad += int((D.read(base + int(got_offs[k]), exp.size) != exp).sum())
    return bad == 0, len(picks)


def c5_leg(aeg, torch, kernel, dist=None, tp_rank=1, tp_size=4, reps=3, model="qwen-72b", check=None):
    """configs[4]: Qwen-72B TP=4 scale-up.  The decode instance's rank r stages its 36.1 GB weight
    shard (Megatron col/row/vocab split, host threads -> pinned Stage Buffer -> PCIe, PAPER.md:
    1343-1354) while its prefill partner hands it 2 GiB of KV (Qwen-72B-TP4 shape, H=16 per rank)
    through the fused migrate kernel (PAPER.md:2096-2098 layout).  One GPU: one rank pair, the
    prefill side a second context on the same GPU (the same kernel stores over NVLink when the peer
    is another GPU); with 8 ranks: ranks 0-3 prefill, 4-7 decode, rank i -> i + 4.
    Reports per-rank weights GB/s, KV hand-off GB/s and the scale-up time (both ready).
    `check(ctx, model, m, seed, tp_rank, tp_size, offsets, picks)` replaces the sampled weights
    check (the GPU test passes the oracle's)."""
    import aeg_inputs as gi
    from aeg_inputs import dev as D
    world = 1 if dist is None else dist.world
    rank = 0 if dist is None else dist.rank
    device = 0 if dist is None else dist.device
    decode = world == 1 or rank >= world // 2
    prefill = world == 1 or rank < world // 2
    if world > 1:
        tp_rank = rank % (world // 2)
    seed_w, seed_kv = gi.w_seed(5), gi.kv_seed(5)
    sht = gi.KV_SHAPES["qwen-72b-tp4"]
    sh = aeg.KVShape.of(sht)
    n_kv = (2 * GIB) // sh.block_bytes()
    slab = 10 * 64 * MIB * 2            # 1.25 GiB: 128 blocks of 10 MiB
    nslab = -(-n_kv // (slab // sh.block_bytes())) + 1
    out = {"workload": f"configs[4] {model} TP=4 scale-up: one decode rank stages its weight shard (staged 3.a) "
                       f"while its prefill partner migrates {n_kv} blocks ({n_kv * sh.block_bytes() / GIB:.2f} GiB) "
                       "of KV to it" + (" (1 GPU: both ranks' contexts on it)" if world == 1 else f", {world} ranks")}
    descs, keep, touched, wctx, a, b = None, None, 0, None, None, None
    t0 = time.time()
    if decode:
        descs, keep, touched = sparse_model_cache(model, 7, tp_rank, tp_size, seed_w)
        shard_total = sum(-(-(d["rows"] * d["cols"] * 2 // (1 if d["split"] == gi.REPLICATED else tp_size)) // 256) * 256
                          for d in descs)
        wctx = aeg.Context(device, aeg.default_config(device_kv_bytes=nslab * slab, host_kv_bytes=GIB,
                                                      dev_slab_bytes=slab, dev_slab_layout=aeg.BLOCK_MAJOR,
                                                      device_weight_bytes=shard_total + 64 * MIB, kernel=kernel,
                                                      host_threads=12, flags=aeg.CFG_TIMING))
        b = wctx
    out["model_cache_build_s"] = round(time.time() - t0, 1)
    out["model_cache_touched_bytes"] = touched
    if prefill:
        a = aeg.Context(device, aeg.default_config(device_kv_bytes=nslab * slab, host_kv_bytes=GIB, dev_slab_bytes=slab,
                                                   dev_slab_layout=aeg.LAYER_MAJOR, kernel=kernel, flags=aeg.CFG_TIMING))
    # pools + destination handles
    if world == 1:
        a.import_peer(1, b.export_ipc())
        peer_of = {0: 1}
        dst = b.kv_alloc(0, sht, n_kv)
    else:
        from paper_conf_sosp_xiang0qyzyzl0025_b200 import dist as PD
        ctx = a if prefill else b
        PD.connect(ctx, rank)
        dst = None if prefill else b.kv_alloc(0, sht, n_kv)
        handles = PD.exchange(None if prefill else [int(x) for x in dst])
        peer_of = {rank: rank + world // 2} if prefill else {}
        dst_by_rank = {d: np.array(h, np.uint64) for d, h in enumerate(handles) if h}
    src = None
    if prefill:
        src = a.kv_alloc(0, sht, n_kv)
        abase, _ = a.pool_region(0)
        D.fill_chunks(abase, chunk_offsets(a, 0, sht, src),
                      [gi.kv_key(5, rank, i, l) for i in range(n_kv) for l in range(sh.num_layers)], sh.chunk_bytes(), seed_kv)
    dst_handles = dst if world == 1 else (dst_by_rank.get(rank + world // 2) if prefill else None)
    D.sync()

    def one(do_w, do_kv):
        if dist is not None:
            dist.barrier()
        s = new_stream(torch)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        xw = xk = None
        if decode and do_w:
            b.stream_fence(s.cuda_stream)
            b.weights_reset(0)
            offs, xw = b.weights_stage(descs, tp_rank, tp_size)
        if prefill and do_kv:
            a.stream_fence(s.cuda_stream)
            xk = a.kv_migrate(sht, src, peer_of[rank], dst_handles)
        if xw is not None:
            b.layer_ready(xw, -1, aeg.READY_WAIT_STREAM, s.cuda_stream)
        if xk is not None:
            a.layer_ready(xk, -1, aeg.READY_WAIT_STREAM, s.cuda_stream)
        e1.record(s)
        e1.synchronize()
        ms = e0.elapsed_time(e1) if (xw is not None or xk is not None) else 0.0
        if xw is not None:
            b.xfer_release(xw)
        if xk is not None:
            a.xfer_release(xk)
        return ms if dist is None else dist.max(ms)

    w_ms = [one(True, False) for _ in range(reps)]
    k_ms = [one(False, True) for _ in range(reps + 2)][2:]
    both = [one(True, True) for _ in range(reps)]
    w_ok, picks = True, 0
    if decode:
        n_t = len(descs)
        pick = [0, 1, 2, 3, 4, 5, 6, 7, n_t // 2 + 3, n_t - 2]
        b.weights_reset(0)
        offs, x = b.weights_stage(descs, tp_rank, tp_size)
        b.layer_ready(x, -1, aeg.READY_BLOCK)
        b.xfer_release(x)
        w_ok, picks = (check or _c5_check_weights)(aeg, b, model, 7, seed_w, tp_rank, tp_size, offs, pick)
    kv_bad = 0
    if decode:
        sender = 0 if world == 1 else rank - world // 2
        bbase, _ = b.pool_region(0)
        kv_bad, _ = D.verify_chunks(bbase, chunk_offsets(b, 0, sht, dst),
                                    [gi.kv_key(5, sender, i, l) for i in range(n_kv) for l in range(sh.num_layers)],
                                    sh.chunk_bytes(), seed_kv)
    shard = 0 if not decode else sum(d["rows"] * d["cols"] * 2 // (1 if d["split"] == gi.REPLICATED else tp_size)
                                     for d in descs)
    for c in (a, b):
        if c is not None:
            c.shutdown()
    del keep
    n_dec = 1 if world == 1 else world // 2
    if dist is not None:
        shard = dist.max(shard)
        kv_bad = dist.sum(kv_bad)
        w_ok = dist.sum(0 if w_ok else 1) == 0
        picks = int(dist.sum(picks))
        out["model_cache_build_s"] = round(dist.max(out["model_cache_build_s"]), 1)
        out["model_cache_touched_bytes"] = int(dist.max(touched))
    kvb = n_kv * sh.block_bytes()
    wm, km, bm = statistics.median(w_ms), statistics.median(k_ms), statistics.median(both)
    out.update({"tp_size": tp_size, "decode_ranks": n_dec, "shard_bytes_per_rank": int(shard),
                "weights_ms": round(wm, 1), "weights_GBps_per_rank": round(shard / (wm * 1e6), 1),
                "weights_frac_of_pcie_nominal": round(shard / (wm * 1e6) / PCIE_NOMINAL, 3),
                "kv_bytes_per_pair": kvb, "kv_ms": round(km, 3), "kv_GBps_per_pair": round(kvb / (km * 1e6), 1),
                "kv_peer": "same GPU (HBM)" if world == 1 else "NVLink",
                "scale_up_ms": round(bm, 1), "scale_up_ms_all": [round(x, 1) for x in both],
                "aggregate_h2d_GBps": round(n_dec * shard / (bm * 1e6), 1),
                "weights_bit_exact_sample": bool(w_ok), "weights_tensors_checked": picks,
                "kv_bit_exact": kv_bad == 0})
    return out


def allocator_leg(aeg, reps=20):
    """H1 control overhead ("tracking indices in the unified cache"): the slab
    allocator of a host-only context with the C2 geometry (82 GiB device pool, 1 GiB slabs, aged by
    the same churn), timed per aeg_kv_alloc / aeg_kv_free call through the Python binding (the
    1-block call shows the binding's own per-call cost)."""
    import aeg_inputs as gi
    cfg = aeg.default_config(device_kv_bytes=82 * GIB, host_kv_bytes=40 * GIB,
                             flags=aeg.CFG_HOST_ONLY | aeg.CFG_NO_DAEMON)
    ctx = aeg.Context(0, cfg)
    sh = QWEN7B
    _, blocks = c2_requests(64)
    live = []
    for op, v in gi.churn_ops(2, capacity_blocks=12 * (GIB // (8 * MIB)), hi_blocks=96):
        if op == "alloc":
            live.append(ctx.kv_alloc(0, sh, v))
        elif live[v] is not None:
            ctx.kv_free(0, live[v])
            live[v] = None
    pa, pf, ba, bf, one = [], [], [], [], []
    clk = time.perf_counter_ns
    for _ in range(reps):
        hs = []
        for b in blocks:
            t0 = clk()
            hs.append(ctx.kv_alloc(0, sh, b))
            pa.append(clk() - t0)
        for h in hs:
            t0 = clk()
            ctx.kv_free(0, h)
            pf.append(clk() - t0)
        t0 = clk()
        h = ctx.kv_alloc(0, sh, sum(blocks))
        t1 = clk()
        ctx.kv_free(0, h)
        ba.append(t1 - t0)
        bf.append(clk() - t1)
    for _ in range(1000):
        t0 = clk()
        h = ctx.kv_alloc(0, sh, 1)
        one.append(clk() - t0)
        ctx.kv_free(0, h)
    ctx.shutdown()
    n = sum(blocks)
    med = lambda v: round(statistics.median(v) / 1e3, 2)  # noqa: E731
    return {"workload": f"C2 geometry, aged pool; 64 per-request calls ({n} Qwen-7B blocks) and one {n}-block call",
            "per_request_alloc_us_p50": med(pa), "per_request_free_us_p50": med(pf),
            "batch_alloc_us": med(ba), "batch_free_us": med(bf),
            "batch_alloc_ns_per_block": round(statistics.median(ba) / n, 1),
            "batch_free_ns_per_block": round(statistics.median(bf) / n, 1),
            "one_block_call_us_p50": med(one), "includes": "Python ctypes call overhead"}


def overlap_leg(aeg, torch, kernel, work_us=500, reps=5, pack_mib=0):
    """North star: "decoding of layer i overlaps the transfer of layer i+1".  A 1 GiB Llama-7B KV
    batch (32 layers) is swapped in while a synthetic decode step does `work_us` of work per layer
    (a spin kernel ~ one layer of a 7B decode step).  per_layer: layer l's work waits only on layer
    l's event (aeg_layer_ready WAIT_STREAM per layer); whole: it waits for the whole transfer (the
    paper's per-request granularity).  Times are device-side, from the swap-in
    call to the end of the last layer's work."""
    import aeg_inputs as gi
    from aeg_inputs import dev as D
    sh = gi.KV_SHAPES["llama-7b"]
    bb = sh[0] * 2 * sh[1] * sh[2] * sh[3] * sh[4]
    n = GIB // bb
    ctx = aeg.Context(0, aeg.default_config(device_kv_bytes=4 * GIB, host_kv_bytes=4 * GIB, kernel=kernel,
                                            pack_layer_mib=pack_mib))
    # clock64 cycles per microsecond at the current SM clock
    cyc_per_us = torch.cuda.get_device_properties(0).clock_rate / 1e3 if hasattr(
        torch.cuda.get_device_properties(0), "clock_rate") else 1965.0
    out = {}
    try:
        hb = ctx.kv_alloc(aeg.POOL_HOST, sh, n)
        cons = new_stream(torch)
        for mode in ("per_layer", "whole"):
            ts = []
            for _ in range(reps):
                db = ctx.kv_alloc(aeg.POOL_DEVICE, sh, n)
                torch.cuda.synchronize()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(cons)
                ctx.stream_fence(cons.cuda_stream)
                x = ctx.kv_swap_in(sh, hb, db)
                if mode == "whole":
                    ctx.layer_ready(x, -1, aeg.READY_WAIT_STREAM, cons.cuda_stream)
                for l in range(sh[0]):
                    if mode == "per_layer":
                        ctx.layer_ready(x, l, aeg.READY_WAIT_STREAM, cons.cuda_stream)
                    D.spin(int(work_us * cyc_per_us), cons.cuda_stream)
                e1.record(cons)
                e1.synchronize()
                ts.append(e0.elapsed_time(e1))
                ctx.layer_ready(x, -1, aeg.READY_BLOCK)
                ctx.xfer_release(x)
                ctx.kv_free(aeg.POOL_DEVICE, db)
            out[mode + "_ms"] = round(statistics.median(ts), 2)
    finally:
        ctx.shutdown()
    out.update({"workload": f"1 GiB Llama-7B KV swap-in ({n} blocks x 32 layers), {work_us} us of decode work "
                            "per layer", "decode_work_ms": round(sh[0] * work_us / 1e3, 1),
                "saved_ms": round(out["whole_ms"] - out["per_layer_ms"], 2)})
    return out


def kernel_alone_leg(aeg, kernel, shape=None):
    """kernel_alone_once over blocks spread like the step's, plus the contiguous best case (SURVEY
    §8(d): blocks allocated in order from a fresh pool)."""
    out = kernel_alone_once(aeg, kernel, shape, spread_gib=16)
    out["contiguous"] = kernel_alone_once(aeg, kernel, shape, spread_gib=0)
    return out


# one layer of Qwen-7B-sized chunks (256 KiB): 4,096 blocks are one 1 GiB staging segment, i.e. one
# gather and one scatter launch — the step's launch size (3,970 x 256 KiB) — with no copy-engine DMA
# running during either kernel (the D2H starts after the gather, the scatter after the H2D)
ALONE_SHAPE = (1, 32, 128, 2, 16)


def kernel_alone_once(aeg, kernel, shape=None, spread_gib=16, layer_gib=1):
    """The dominant kernels without the step's concurrent PCIe DMA: a swap-out and a swap-in of one
    layer of layer_gib (one gather and one scatter launch of the step's size), timed by the library's
    CUDA events (AEG_CFG_TIMING); best of 3.  The blocks are paged like the step's: a
    seeded random set kept out of a spread_gib pool that was filled and then mostly freed, so both
    kernels walk block tables spread over the whole pool (spread_gib = 0: the contiguous best case)."""
    import aeg_inputs as gi
    shape = shape or ALONE_SHAPE
    sh = aeg.KVShape.of(shape)
    n = (layer_gib * GIB) // sh.chunk_bytes()
    total = n * sh.block_bytes()
    ctx = aeg.Context(0, aeg.default_config(device_kv_bytes=max(spread_gib * GIB, total + GIB),
                                            host_kv_bytes=total + GIB, kernel=kernel, flags=aeg.CFG_TIMING))
    best = {}
    try:
        if spread_gib:
            every = ctx.kv_alloc(aeg.POOL_DEVICE, shape, (spread_gib * GIB) // sh.block_bytes())
            keep = gi.rng(47).permutation(len(every))
            ctx.kv_free(aeg.POOL_DEVICE, every[np.sort(keep[n:])])
            dev = every[np.sort(keep[:n])]
        else:   # contiguous best case: a fresh pool, blocks in order (whole-slab runs per layer)
            dev = ctx.kv_alloc(aeg.POOL_DEVICE, shape, n)
        for _ in range(4):
            ctx.kernel_stats_reset()
            host = ctx.kv_alloc(aeg.POOL_HOST, shape, n)
            x = ctx.kv_swap_out(shape, dev, host, flags=aeg.FREE_SRC)
            ctx.layer_ready(x, -1, aeg.READY_BLOCK)
            dev = ctx.kv_alloc(aeg.POOL_DEVICE, shape, n)
            y = ctx.kv_swap_in(shape, host, dev, flags=aeg.FREE_SRC)
            ctx.layer_ready(y, -1, aeg.READY_BLOCK)
            ctx.xfer_release(x)
            ctx.xfer_release(y)
            for kind, name in ((aeg.K_GATHER, "gather"), (aeg.K_SCATTER, "scatter")):
                nl, nb, ms = ctx.kernel_stats(kind)
                if ms > 0:
                    best[name] = max(best.get(name, 0.0), nb / (ms * 1e6))
    finally:
        ctx.shutdown()
    return {k: round(v, 1) for k, v in best.items()}


def per_request_sync_leg(aeg, torch, kernel, h2d_GBps=None, n_req=32, pack_mib=0):
    """Fig. 15 (right) on B200: the per-request KV cache transfer overhead.  n_req
    Qwen-7B requests with ShareGPT-like lengths (lognormal prompt + output, seeded) sit in the host
    pool; the scheduler issues one swap-in per request back to back (per-request transfers and
    readiness) and the decode side waits per request.  Per request: device time
    from the first issue to its last layer ready; its ideal is the cumulative bytes over the plain
    H2D memcpy rate of this box; overhead = ready - ideal.  Also the host enqueue time per call."""
    import aeg_inputs as gi
    sh = QWEN7B
    bb = aeg.KVShape.of(sh).block_bytes()
    g = gi.rng(31)
    lens = [int(g.lognormal(np.log(600), 0.8)) + int(g.lognormal(np.log(300), 0.8)) for _ in range(n_req)]
    nblk = [-(-max(1, t) // 16) for t in lens]
    ctx = aeg.Context(0, aeg.default_config(device_kv_bytes=(sum(nblk) * bb // GIB + 4) * GIB,
                                            host_kv_bytes=(sum(nblk) * bb // GIB + 4) * GIB, kernel=kernel,
                                            pack_layer_mib=pack_mib))
    try:
        host = [ctx.kv_alloc(aeg.POOL_HOST, sh, n) for n in nblk]
        cons = new_stream(torch)
        rows = []
        for rep in range(3):
            dev = [ctx.kv_alloc(aeg.POOL_DEVICE, sh, n) for n in nblk]
            torch.cuda.synchronize()
            e0 = torch.cuda.Event(enable_timing=True)
            e0.record(cons)
            ctx.stream_fence(cons.cuda_stream)
            xs, evs, enq = [], [], []
            for h, d in zip(host, dev):
                t0 = time.perf_counter()
                xs.append(ctx.kv_swap_in(sh, h, d))
                enq.append((time.perf_counter() - t0) * 1e6)
                # the decode side waits for this request right away (an event recorded later would
                # time the host's enqueue, not the request): ready = its last layer has landed
                ctx.layer_ready(xs[-1], -1, aeg.READY_WAIT_STREAM, cons.cuda_stream)
                e = torch.cuda.Event(enable_timing=True)
                e.record(cons)
                evs.append(e)
            evs[-1].synchronize()
            ready = [e0.elapsed_time(e) for e in evs]
            for x in xs:
                ctx.xfer_release(x)
            for d in dev:
                ctx.kv_free(aeg.POOL_DEVICE, d)
            if rep:
                rows.append((ready, enq))
    finally:
        ctx.shutdown()
    ready = [statistics.median(r[0][i] for r in rows) for i in range(n_req)]
    enq = sorted(e for r in rows for e in r[1])
    cum = np.cumsum([n * bb for n in nblk])
    out = {"workload": f"{n_req} Qwen-7B requests, ShareGPT-like lengths (mean {int(np.mean(lens))} tokens, "
                       f"{sum(nblk)} blocks, {cum[-1] / GIB:.2f} GiB), one swap-in per request, back to back",
           "ready_ms_p50": round(float(np.median(ready)), 2), "ready_ms_max": round(max(ready), 2),
           "per_request_transfer_ms_p50": round(float(np.median(np.diff([0.0] + ready))), 3),
           "enqueue_us_p50": round(enq[len(enq) // 2], 1), "enqueue_us_p90": round(enq[int(0.9 * (len(enq) - 1))], 1),
           "GBps": round(cum[-1] / (ready[-1] * 1e6), 1)}
    if h2d_GBps:
        over = [r - c / (h2d_GBps * 1e6) for r, c in zip(ready, cum)]
        out.update({"overhead_vs_memcpy_ms_p50": round(float(np.median(over)), 3),
                    "overhead_vs_memcpy_ms_max": round(max(over), 3), "h2d_memcpy_GBps": round(h2d_GBps, 1)})
    return out


class OracleSample:
    """The oracle as it stands (NumPy, one host core for its copies) on a bounded, resident sample
    of the C2 workload: swap-out + swap-in of `blocks` Qwen-7B blocks between byte-image pools
    (oracle/kv.py).  Setup (pool images, oracle allocators) is outside rep(); rep() is one sample
    step: swap-out of the blocks to host blocks, then swap-in into fresh device blocks."""

    def __init__(self, blocks=512):
        from oracle import kv as OK
        from oracle.shape import KVShape
        from oracle.slab import SlabPool
        self.OK = OK
        self.sh = sh = KVShape(*QWEN7B)
        self.blocks = blocks
        k = GIB // sh.block_bytes()
        ns = -(-blocks // k)
        self.dg = OK.PoolGeom(2 * ns * GIB, GIB, 0)          # source slabs + destination slabs
        self.hg = OK.PoolGeom(ns * GIB, GIB, 0)
        self.dev = np.zeros(self.dg.nbytes, np.uint8)
        self.dev[: blocks * sh.block_bytes()] = 1
        self.host = np.zeros(self.hg.nbytes, np.uint8)
        od, oh = SlabPool(self.dg.nbytes, GIB), SlabPool(self.hg.nbytes, GIB)
        self.src = od.alloc(sh, blocks)
        self.dst = od.alloc(sh, blocks)
        self.hb = oh.alloc(sh, blocks)

    def bytes_per_rep(self):
        return 2 * self.blocks * self.sh.block_bytes()

    def rep(self):
        OK = self.OK
        self.host = OK.swap_out(self.dev, self.dg, self.host, self.hg, self.sh, self.src, self.hb)
        self.dev = OK.swap_in(self.host, self.hg, self.dev, self.dg, self.sh, self.hb, self.dst)

    def describe(self, reps, t):
        return (f"{reps} x swap-out+swap-in of {self.blocks} of the 3970 configs[1] Qwen-7B blocks "
                f"({self.blocks * self.sh.block_bytes() >> 20} MiB each way, resident byte images) through "
                f"oracle/kv.py, {t:.1f} s timed (setup excluded); GB/s extrapolates linearly to the full "
                "31 GiB/direction step")


def gpu_local_cpus(index=0):
    """Host cores on GPU `index`'s NUMA node (sysfs local_cpulist of its PCI device), or None."""
    try:
        r = subprocess.run(["nvidia-smi", "--query-gpu=pci.bus_id", "--format=csv,noheader", "-i", str(index)],
                           capture_output=True, text=True, timeout=30)
        bus = r.stdout.strip().lower()
        if bus.count(":") == 2 and len(bus.split(":")[0]) == 8:   # 00000000:1B:00.0 -> 0000:1b:00.0
            bus = bus[4:]
        cpus = set()
        for part in open(f"/sys/bus/pci/devices/{bus}/local_cpulist").read().strip().split(","):
            a, _, b = part.partition("-")
            cpus.update(range(int(a), int(b or a) + 1))
        return cpus or None
    except (OSError, ValueError, subprocess.SubprocessError):
        return None


class one_core:
    """Pin this process to one host core for the oracle's timing (single-threaded, a
    core on the GPU's NUMA node when sysfs says which)."""

    def __enter__(self):
        self.aff = os.sched_getaffinity(0) if hasattr(os, "sched_getaffinity") else None
        if self.aff:
            near = (gpu_local_cpus() or set()) & set(self.aff)
            self.core = min(near or self.aff)
            self.gpu_local = bool(near)
            os.sched_setaffinity(0, {self.core})
        return self

    def describe(self):
        return {"core_id": getattr(self, "core", None), "on_gpu_numa_node": getattr(self, "gpu_local", None)}

    def __exit__(self, *a):
        if self.aff:
            os.sched_setaffinity(0, self.aff)


def cpu_baseline(blocks=512, min_s=10.0):
    """cpu_baseline leg of our arm: OracleSample timed for >= min_s seconds on one core."""
    o = OracleSample(blocks)
    reps, t = 0, 0.0
    with one_core() as pin:
        while (reps == 0 or t < min_s) and reps < 50:
            t0 = time.perf_counter()
            o.rep()
            t += time.perf_counter() - t0
            reps += 1
    return {"value": round(o.bytes_per_rep() * reps / t / 1e9, 3), "unit": "GB/s", "cores": 1, "kind": "oracle",
            "sample": o.describe(reps, t), "pinning": pin.describe()}


# ----------------------------------------------------------------------------------- arms
def run_reference(args):
    """Reference arm = the oracle (task ③/④): each step is one OracleSample rep (a bounded 4 GiB
    sample of the configs[1] round trip), timed alone; setup is outside the timed region."""
    world, rank, local = dist_env()
    if rank != 0:
        return 0
    o = OracleSample(512)
    with one_core() as pin:
        for _ in range(args.warmup):
            o.rep()
        t = 0.0
        for _ in range(args.steps):
            t0 = time.perf_counter()
            o.rep()
            t += time.perf_counter() - t0
    value = o.bytes_per_rep() * args.steps / t / 1e9
    full = 2 * sum(c2_requests(args.requests)[1]) * o.sh.block_bytes()
    out = {"impl": "reference", "metric": METRIC, "value": round(value, 3), "unit": "GB/s", "n_gpus": args.gpus,
           "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(1e3 * t / args.steps, 1),
           "ms_per_full_step_extrapolated": round(1e3 * full / (value * 1e9), 1),
           "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "bf16", "data": "synthetic",
           "config": {"workload": "configs[1] Qwen-7B 64-request swap round trip (bounded sample: "
                                  f"{o.blocks} of {sum(c2_requests(args.requests)[1])} blocks per step)",
                      "requests": args.requests},
           "cpu_baseline": {"value": round(value, 3), "unit": "GB/s", "cores": 1, "kind": "oracle",
                            "sample": o.describe(args.steps, t), "pinning": pin.describe()},
           "e2e": {"value": round(value, 3), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)
    return 0


def run_ours(args):
    import torch
    import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg
    from paper_conf_sosp_xiang0qyzyzl0025_b200 import build
    world, rank, local = dist_env()
    if rank == 0:   # compiled from the checked-out sources on this box, never a shipped binary
        build.build(force=os.environ.get("AEG_BENCH_NO_REBUILD") != "1")
    dist = Dist(world, rank, local)
    dist.barrier()
    kernel = {"auto": aeg.KERNEL_AUTO, "lsu": aeg.KERNEL_LSU, "bulk": aeg.KERNEL_BULK, "bulkw": aeg.KERNEL_BULKW,
              "warp": aeg.KERNEL_WARP}[args.kernel]
    n_req = args.requests
    if world > 1:   # keep the pinned host pools inside host RAM when several ranks share a node
        import psutil
        per_rank = psutil.virtual_memory().available / world
        while n_req > 4 and sum(c2_requests(n_req)[1]) * 8 * MIB * 1.3 > per_rank:
            n_req //= 2
    sb = SwapBench(aeg, QWEN7B, n_req, kernel, slot_mib=args.slot_mib, slots=args.slots,
                   dma_piece_mib=args.dma_piece_mib,
                   churn_slabs=args.churn_slabs).setup()
    sb.sink = torch.zeros(1, dtype=torch.int64, device="cuda")
    cons = new_stream(torch)
    bytes_step = 2 * sb.n * sb.sh.block_bytes()
    log(f"[rank {rank}] C2: {sb.n} blocks ({sb.n * sb.sh.block_bytes() / GIB:.2f} GiB), ctx init {sb.init_s:.1f} s")
    for _ in range(args.warmup):
        sb.step(torch, cons)
    sb.ctx.kernel_stats_reset()
    dist.barrier()
    with Clocks(dist.device) as clk, PcieCounters(dist.device) as pcnt:
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        marks = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
        e0.record(cons)
        for i in range(args.steps):
            sb.step(torch, cons)
            marks[i].record(cons)
        e1.record(cons)
        e1.synchronize()
    dist.barrier()
    ms_total = dist.max(e0.elapsed_time(e1))
    # N > 1: each replica's own rate (the ranks share PCIe switch uplinks and host DRAM)
    rank_ms = dist.gather_obj(e0.elapsed_time(e1)) if world > 1 else None
    clocks = clk.summary()
    pcie_counters = pcnt.summary()
    ms_step = ms_total / args.steps
    per_step = sorted(dist.max(a.elapsed_time(b)) for a, b in zip([e0] + marks[:-1], marks))
    pct = lambda q: round(per_step[min(len(per_step) - 1, int(q * (len(per_step) - 1) + 0.5))], 2)  # noqa: E731
    total_bytes = dist.sum(bytes_step * args.steps)
    value = total_bytes / (ms_total * 1e6)
    g = sb.ctx.kernel_stats(aeg.K_GATHER)
    s = sb.ctx.kernel_stats(aeg.K_SCATTER)
    f = sb.ctx.kernel_stats(aeg.K_FETCH)   # the block-table fetch kernel of each transfer
    launches_all = int(dist.sum(g[0] + s[0] + f[0]))
    hbm, hbm_src = peaks()
    # dominant kernel = gather (HBM bound): algorithmic bytes per launch / mean CUDA-event duration
    g_per_launch_bytes = g[1] / max(1, g[0])
    g_ms = g[2] / max(1, g[0])
    g_ach = g_per_launch_bytes / (g_ms * 1e6) if g_ms > 0 else 0.0
    s_ach = (s[1] / max(1, s[0])) / ((s[2] / max(1, s[0])) * 1e6) if s[2] > 0 else 0.0
    core = {
        "metric": METRIC, "value": round(value, 2), "unit": "GB/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(ms_step, 2),
        "step_ms_p10_p50_p90": [pct(0.1), pct(0.5), pct(0.9)], "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "bf16", "data": "synthetic",
        "config": {"workload": "configs[1]: Qwen-7B-shaped KV (32 layers, 32 KV heads, d=128, bf16, 16-token "
                               f"blocks), {n_req}-request decode batch swapped out and back in per step",
                   "requests": n_req, "requests_per_rank": n_req,
                   "requests_note": (None if n_req == args.requests else
                                     f"reduced from {args.requests} per rank so that {world} ranks' pinned "
                                     "host pools fit this node's RAM; per-rank work differs from N=1"),
                   "tokens": int(sum(sb.lens)), "blocks": sb.n,
                   "bytes_per_direction": sb.n * sb.sh.block_bytes(), "slab": "1 GiB layer-major",
                   "placement": "device pool aged by seeded churn", "l2": "inputs larger than L2 (32 GiB/step)",
                   "kernel": args.kernel, "staging_slot_mib": sb.cfg.staging_slot_bytes >> 20,
                   "dma_piece_mib": sb.cfg.dma_piece_mib,
                   "staging_slots": sb.cfg.staging_slots, "parallelism": f"replicas x{world}"},
        "roofline": {"bound": "hbm", "kernel": "gather (swap-out, H2)", "achieved": round(g_ach, 1),
                     "peak": hbm, "peak_source": hbm_src, "unit": "GB/s",
                     "frac": round(g_ach / hbm, 3), "traffic": ncu_traffic("gather", int(g_per_launch_bytes)),
                     "algorithmic_bytes_per_launch": int(g_per_launch_bytes), "launches": g[0],
                     "mean_launch_ms": round(g_ms, 4), "scatter_achieved": round(s_ach, 1)},
        "pcie": {"bound": "pcie", "achieved_round_trip": round(bytes_step / (ms_step * 1e6), 1),
                 "achieved_per_direction": round(bytes_step / 2 / (ms_step * 1e6), 1),
                 "peak_per_direction_nominal": PCIE_NOMINAL,
                 "frac_of_duplex_nominal": round(bytes_step / (ms_step * 1e6) / (2 * PCIE_NOMINAL), 3)},
        "clocks": clocks,
        "pcie_counters": pcie_counters,
        "gpu_launches": launches_all,
        "consumer_launches": args.steps * sb.L,
    }
    if rank_ms:
        core["per_rank_GBps"] = [round(bytes_step * args.steps / (m * 1e6), 1) for m in rank_ms]
    # Side legs are bounded: a hung leg must not lose the headline line, so after leg_budget_s a
    # watchdog prints the core line with the legs completed so far and ends the process.
    import threading
    partial, print_lock, printed = {}, threading.Lock(), []

    def on_leg_timeout():
        with print_lock:
            if rank == 0 and not printed:
                line = dict(core)
                line.update({"side_legs_timed_out_after_s": args.leg_budget_s, "side_legs_completed": partial})
                print(json.dumps(line), flush=True)
                printed.append(1)
        os._exit(0)
    watchdog = threading.Timer(args.leg_budget_s, on_leg_timeout)
    watchdog.daemon = True
    watchdog.start()
    out = {}
    if not args.profile:
        pc = pcie_calibration(torch, dist)
        # e2e: the same step through the public Python API, wall clock, after a host sync each step
        e2e = None
        if not args.no_e2e:
            ts, fl = [], []
            for _ in range(max(3, args.steps // 2)):
                torch.cuda.synchronize()
                t0 = time.perf_counter()
                ev = []
                sb.step(torch, cons, first_layer=ev)
                cons.synchronize()
                ts.append(time.perf_counter() - t0)
                fl.append((ev[0].elapsed_time(ev[1]), ev[0].elapsed_time(ev[2]), ev[0].elapsed_time(ev[3]))
                          + sb.enqueue_ms)
            e2e_t = dist.max(statistics.median(ts))   # the job's step ends when the slowest rank's does
            e2e = {"value": round(dist.sum(bytes_step) / e2e_t / 1e9, 2), "unit": "GB/s",
                   # whole job, like `value` (every rank's copies)
                   "h2d_bytes_per_step": int(dist.sum(bytes_step // 2 + 2 * sb.n * 8)),
                   "d2h_bytes_per_step": int(dist.sum(bytes_step // 2)),
                   "how": "wall clock around the Python-API calls of one step incl. host sync",
                   "round_trip_layer0_ready_ms_p50": round(statistics.median(f[0] for f in fl), 2),
                   "round_trip_last_layer_ready_ms_p50": round(statistics.median(f[1] for f in fl), 2),
                   "swap_out_layer0_landed_ms_p50": round(statistics.median(f[2] for f in fl), 2),
                   "enqueue_ms_p50": {"swap_out": round(statistics.median(f[3] for f in fl), 2),
                                      "swap_in": round(statistics.median(f[4] for f in fl), 2)}}
        partial["e2e"] = e2e
        def leg(name, fn):
            """A side leg that fails reports its error in the line instead of losing the whole line."""
            try:
                r = fn()
            except Exception as e:  # noqa: BLE001
                import traceback
                log(f"[rank {rank}] leg {name} failed:\n" + traceback.format_exc())
                r = {"error": f"{type(e).__name__}: {e}"}
            partial[name] = r
            return r

        one_dir = leg("one_direction", lambda: sb.one_direction(torch, cons))
        ver = leg("verify", sb.verify)
        base = leg("memcpy_baseline", lambda: chunk_memcpy_baseline(aeg, torch, sb.ctx, sb.sht, sb.src_c))
        if world > 1:   # every rank checks its own pools; the line reports all of them
            ver["ranks_failed"] = int(dist.sum(0 if ver.get("ok") else 1))
            ver["ok"] = ver["ranks_failed"] == 0
        sb.ctx.shutdown()

        def b2b():
            import psutil
            need = 2 * sb.n * sb.sh.block_bytes() + 12 * GIB   # second host batch + slack
            if world > 1 or psutil.virtual_memory().available < need + 16 * GIB:
                return None
            bb = SwapBench(aeg, QWEN7B, n_req, kernel, dev_batches=3, host_batches=2, timing=False).setup()
            try:
                bb.back_to_back(torch, cons, 2)          # warm-up
                runs = [bb.back_to_back(torch, cons, 6) for _ in range(2)]
                r = max(runs, key=lambda q: q["GBps"])
                r["GBps_runs"] = [q["GBps"] for q in runs]
                v = bb.verify()
                r["bit_exact"] = bool(v.get("ok"))
                r["what"] = ("configs[1] round trips back to back, no host sync between them (rules ❷❸ order "
                             "them per layer); context sized for 2 in flight")
                return r
            finally:
                bb.ctx.shutdown()
        back2back = leg("back_to_back", b2b)
        if args.no_migrate:
            mig = None
        elif world > 1:
            mig = leg("migrate", lambda: migrate_leg_dist(aeg, torch, dist, kernel, args.migrate_requests))
            if rank == 0 and dist.local == 0:   # the cross-device branch of aeg_import_peer, one process
                mig["two_device_same_process"] = leg("migrate_two_device",
                                                     lambda: migrate_leg_two_device(aeg, torch, kernel))
                # bulk copies (cp.async.bulk) storing into another GPU's memory are not relied on by
                # AUTO; opt-in only, and then in a throw-away process so a fault cannot touch this one
                if args.probe_peer_bulk:
                    mig["two_device_bulkw_stores_probe"] = leg("two_device_bulkw", two_device_bulkw_probe)
            dist.barrier()
        else:
            mig = leg("migrate", lambda: migrate_leg(aeg, torch, kernel, args.migrate_requests))
        sw = None
        if not (args.no_switch or world > 1):
            t0 = time.time()
            descs, caches = model_caches(["qwen-1.8b", "llama-7b", "yi-9b"])
            gen_s = time.time() - t0
            sw = {"staged": leg("switch_staged", lambda: switch_leg(aeg, torch, args.switches, kernel, descs, "staged")),
                  "prefetch": leg("switch_prefetch",
                                  lambda: switch_leg(aeg, torch, args.switches, kernel, descs, "prefetch")),
                  "direct": leg("switch_direct",
                                lambda: switch_leg(aeg, torch, args.switches, kernel, descs, "direct", caches)),
                  "model_cache_gen_s": round(gen_s, 1)}
            del caches
        ovl = None if args.no_switch or world > 1 else leg("overlap", lambda: overlap_leg(aeg, torch, kernel))
        alone = leg("kernel_alone", lambda: kernel_alone_leg(aeg, kernel))
        prs = None if world > 1 else leg("per_request_sync", lambda: per_request_sync_leg(
            aeg, torch, kernel, h2d_GBps=pc.get("h2d")))
        if args.no_c5:
            c5 = None
        elif world in (1, 8):
            c5 = leg("c5", lambda: c5_leg(aeg, torch, kernel, dist if world > 1 else None, model=args.c5_model))
        else:
            c5 = {"skipped": "configs[4] is the 8-GPU TP=4 layout (one rank pair on 1 GPU); not defined for N=%d" % world}
        small = None if world > 1 else leg("small_chunk", lambda: small_chunk_leg(aeg, torch, kernel))
        c1 = None if world > 1 else leg("c1", lambda: c1_leg(aeg, torch, kernel))
        small_tp4 = None if world > 1 else leg("small_chunk_tp4",
                                               lambda: small_chunk_leg(aeg, torch, kernel, model="yi-9b-tp4"))
        route = None if world > 1 else leg("host_route", lambda: host_route_leg(aeg, torch, kernel))
        alloc = leg("allocator", lambda: allocator_leg(aeg)) if rank == 0 else None
        cpu = None if args.no_cpu or rank != 0 else leg("cpu_baseline", cpu_baseline)
        out.update({"e2e": e2e, "verify": ver, "one_direction": one_dir, "pcie_memcpy_GBps": {k: round(v, 1) for k, v in pc.items()},
                    "switch": sw, "migrate": mig, "per_layer_overlap": ovl, "per_request_sync": prs, "c5": c5,
                    "kernel_alone": alone,
                    "allocator": alloc,
                    "per_chunk_memcpy_baseline": base, "small_chunk": small, "small_chunk_tp4": small_tp4, "c1": c1, "back_to_back": back2back,
                    "host_route": route,
                    "host": host_facts(),
                    "cpu_baseline": cpu})
        if not ver.get("ok"):
            log("VERIFICATION FAILED", ver)
    else:
        sb.ctx.shutdown()
    if rank == 0:
        res = json.loads(json.dumps(core))
        res.update(out)
        ka = out.get("kernel_alone") or {}
        if ka.get("gather"):   # context: the same kernel with no concurrent DMA (one 1 GiB launch)
            res["roofline"]["alone_achieved"] = ka["gather"]
            res["roofline"]["alone_frac"] = round(ka["gather"] / hbm, 3)
            res["roofline"]["alone_scatter_achieved"] = ka.get("scatter")
        res["paper_context"] = paper_context(out)
        pm = out.get("pcie_memcpy_GBps") or {}
        if pm.get("bidir_total"):   # the round trip against this box's own duplex copy-engine ceiling
            res["pcie"]["measured_bidir_memcpy_GBps"] = round(pm["bidir_total"], 1)
            res["pcie"]["frac_of_measured_bidir"] = round(value / pm["bidir_total"], 3)
        if pm.get("bidir_total_all_ranks"):   # N > 1: `value` is all ranks' bytes; ceiling = all GPUs at once
            res["pcie"]["scope"] = "achieved_* and measured_bidir_memcpy_GBps: rank 0; *_all_ranks: every GPU at once"
            res["pcie"]["measured_bidir_memcpy_GBps_all_ranks"] = round(pm["bidir_total_all_ranks"], 1)
            res["pcie"]["frac_of_measured_bidir"] = round(value / pm["bidir_total_all_ranks"], 3)
        od = out.get("one_direction")
        if od and "error" not in od:   # each direction alone against PCIe Gen5 x16 nominal 64 GB/s (target >= 0.80)
            res["pcie"]["swap_out_alone_GBps"] = od["swap_out"]["GBps"]
            res["pcie"]["swap_in_alone_GBps"] = od["swap_in"]["GBps"]
            res["pcie"]["swap_out_alone_frac"] = round(od["swap_out"]["GBps"] / PCIE_NOMINAL, 3)
            res["pcie"]["swap_in_alone_frac"] = round(od["swap_in"]["GBps"] / PCIE_NOMINAL, 3)
        with print_lock:
            if not printed:
                print(json.dumps(res), flush=True)
                printed.append(1)
    watchdog.cancel()
    dist.close()
    return 0


def paper_context(out):
    """The paper's own auto-scaling-overhead numbers, with the GPUs it reports them on, next to this
    run's corresponding measurements (context only: other hardware, other workloads)."""
    def pick(*path):
        v = out
        for k in path:
            if not isinstance(v, dict):
                return None
            v = v.get(k)
        return v
    return {
        "note": "context only: the paper's testbed is 8x H800 80 GB per node (PCIe Gen5, NVLink; PAPER.md:1598-1601) "
                "and its models are served end to end; here one B200 and synthetic KV / random-init weights",
        "auto_scaling_latency": {
            "paper": "< 1 s, about half near-instantaneous thanks to prefetch (7B/9B/13B models, H800; "
                     "PAPER.md:2020-2025, Fig. 15 left)",
            "ours_llama7b_switch_ms_p50": {m: pick("switch", m, "per_model", "llama-7b", "last_layer_ms_p50")
                                           for m in ("staged", "direct", "prefetch")}},
        "kv_sync_overhead_per_request": {
            "paper": "< 1 s per request in total (Fig. 15 right, PAPER.md:2025-2029)",
            "ours_overhead_vs_memcpy_ms_p50_max": [pick("per_request_sync", "overhead_vs_memcpy_ms_p50"),
                                                   pick("per_request_sync", "overhead_vs_memcpy_ms_max")]},
        "weight_load_bandwidth": {
            "paper": "vLLM baseline 2.83 GB/s per GPU over PCIe 4.0 (LLaMA-13B TP=2; PAPER.md:1173-1181)",
            "ours_staged_llama7b_h2d_GBps": pick("switch", "staged", "per_model", "llama-7b", "h2d_GBps")},
    }


def two_device_bulkw_probe(timeout_s=300):
    """Run migrate_leg_two_device with the BULKW kernel forced (bulk stores into the peer GPU) in a
    separate process; returns its JSON or what went wrong."""
    env = {k: v for k, v in os.environ.items() if k not in ("RANK", "LOCAL_RANK", "WORLD_SIZE")}
    try:
        r = subprocess.run([sys.executable, os.path.abspath(__file__), "--two-device-probe"], capture_output=True,
                           text=True, timeout=timeout_s, env=env)
    except subprocess.TimeoutExpired:
        return {"error": f"timed out after {timeout_s} s"}
    for line in reversed(r.stdout.splitlines()):
        if line.startswith("{"):
            return json.loads(line)
    return {"error": f"rc {r.returncode}", "stderr_tail": r.stderr[-400:]}


def main():
    args = parse()
    if args.two_device_probe:
        import torch
        import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg
        print(json.dumps(migrate_leg_two_device(aeg, torch, aeg.KERNEL_BULKW)), flush=True)
        return 0
    if args.impl == "reference":
        return run_reference(args)
    return run_ours(args)


if __name__ == "__main__":
    sys.exit(main())
