"""Local migrate kernel vs block count, pool layouts and kernel (one GPU, same-process peer)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg  # noqa: E402

L, B = aeg.LAYER_MAJOR, aeg.BLOCK_MAJOR
NAMES = {aeg.KERNEL_AUTO: "auto", aeg.KERNEL_LSU: "lsu", aeg.KERNEL_BULK: "bulk", aeg.KERNEL_BULKW: "bulkw"}
for n_req in (16, 4):
    for sl, dl in ((L, B), (L, L), (B, B), (B, L)):
        for k in (aeg.KERNEL_LSU, aeg.KERNEL_BULK, aeg.KERNEL_BULKW):
            r = bench.migrate_leg(aeg, torch, k, n_req, sl, dl)
            print(json.dumps({"n_req": n_req, "src": "LM" if sl == L else "BM", "dst": "LM" if dl == L else "BM",
                              "kernel": NAMES[k], "hbm_GBps": r["hbm_GBps"],
                              "launches": r["kernel_launches_per_xfer"], "ok": r["bit_exact"]}), flush=True)
