"""Local paged->paged hand-off (configs[2] Llama-2-13B, 16 requests, LM -> BM, one GPU): device time
of one aeg_kv_migrate with and without the library's per-launch timing events, for the library as
built (tools/gpu_migrate_pack.sh rebuilds it per layers-per-launch packing).  Prints one JSON line."""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402,F401
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg  # noqa: E402
import aeg_inputs as gi  # noqa: E402
from aeg_inputs import dev as D  # noqa: E402

GIB, MIB = bench.GIB, bench.MIB


def run(timing, n_req=16, reps=6):
    sht = gi.KV_SHAPES["llama-2-13b"]
    sh = aeg.KVShape.of(sht)
    lens = gi.request_lengths(3, n_req, 512, 4096)
    n = sum(-(-t // 16) for t in lens)
    slab = GIB + 256 * MIB
    nslab = -(-n // (slab // sh.block_bytes())) + 1
    mk = lambda lay: aeg.Context(0, aeg.default_config(  # noqa: E731
        device_kv_bytes=nslab * slab, host_kv_bytes=GIB, dev_slab_bytes=slab, dev_slab_layout=lay,
        flags=aeg.CFG_TIMING if timing else 0))
    a, b = mk(aeg.LAYER_MAJOR), mk(aeg.BLOCK_MAJOR)
    try:
        sc, dc = a.kv_alloc(0, sht, n), b.kv_alloc(0, sht, n)
        abase, _ = a.pool_region(0)
        bbase, _ = b.pool_region(0)
        seed = gi.kv_seed(3)
        keys = [gi.kv_key(1, i // 4096, i % 4096, l) for i in range(n) for l in range(sh.num_layers)]
        D.fill_chunks(abase, bench.chunk_offsets(a, 0, sht, sc), keys, sh.chunk_bytes(), seed)
        a.import_peer(1, b.export_ipc())
        s = torch.cuda.Stream()
        ts = []
        for it in range(reps + 2):
            a.kernel_stats_reset()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            a.stream_fence(s.cuda_stream)
            x = a.kv_migrate(sht, sc, 1, dc)
            a.layer_ready(x, -1, aeg.READY_WAIT_STREAM, s.cuda_stream)
            e1.record(s)
            e1.synchronize()
            a.xfer_release(x)
            if it >= 2:
                ts.append(e0.elapsed_time(e1))
        nl, nb, kms = a.kernel_stats(aeg.K_MIGRATE)
        bad, _ = D.verify_chunks(bbase, bench.chunk_offsets(b, 0, sht, dc), keys, sh.chunk_bytes(), seed)
        ms = statistics.median(ts)
        return {"timing_events": timing, "launches": nl, "ms": round(ms, 3), "ms_min": round(min(ts), 3),
                "hbm_GBps": round(2 * n * sh.block_bytes() / (ms * 1e6), 1),
                "hbm_GBps_best": round(2 * n * sh.block_bytes() / (min(ts) * 1e6), 1),
                "kernel_ms": round(kms, 3) if timing else None, "bit_exact": bad == 0}
    finally:
        a.shutdown()
        b.shutdown()


if __name__ == "__main__":
    print(json.dumps({"variant": os.environ.get("AEG_CXX_EXTRA", "default"), "runs": [run(True), run(False)]}),
          flush=True)
