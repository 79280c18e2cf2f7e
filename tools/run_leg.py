"""Run one bench.py side leg alone on cuda:0 and print its JSON (development / profiling helper).
    python tools/run_leg.py c5|migrate|overlap [kernel]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg  # noqa: E402
from paper_conf_sosp_xiang0qyzyzl0025_b200 import build  # noqa: E402

build.build()
leg = sys.argv[1]
kernel = {"auto": aeg.KERNEL_AUTO, "lsu": aeg.KERNEL_LSU, "bulk": aeg.KERNEL_BULK}[sys.argv[2] if len(sys.argv) > 2 else "auto"]
fn = {"c5": lambda: bench.c5_leg(aeg, torch, kernel), "migrate": lambda: bench.migrate_leg(aeg, torch, kernel),
      "overlap": lambda: bench.overlap_leg(aeg, torch, kernel),
      "small_chunk": lambda: bench.small_chunk_leg(aeg, torch, kernel)}[leg]
print(json.dumps(fn()), flush=True)
