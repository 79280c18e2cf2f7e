"""Run one bench.py side leg alone on cuda:0 and print its JSON (development / profiling helper).
    python tools/run_leg.py c5|migrate|overlap|small_chunk|switch|host_route|kernel_alone [auto|lsu|bulk]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg  # noqa: E402
from paper_conf_sosp_xiang0qyzyzl0025_b200 import build  # noqa: E402


def switch_cmp(kernel):
    """configs[3] switch with A's KV-out concurrent with B's load vs after it, per weight mode."""
    descs, caches = bench.model_caches(["qwen-1.8b", "llama-7b", "yi-9b"])
    out = {}
    for mode in ("staged", "prefetch", "direct"):
        for kv_out in ("concurrent", "after"):
            r = bench.switch_leg(aeg, torch, 12, kernel, descs, mode, caches if mode == "direct" else None, kv_out)
            key = f"{mode}/{kv_out}"
            out[key] = {k: (v["last_layer_ms_p50"], v["first_layer_ms_p50"]) for k, v in r["per_model"].items()}
            out[key]["landing"] = r["landing_ms_one_switch"]
            print(json.dumps({key: out[key]}), flush=True)
    return out


def main():
    build.build()
    leg = sys.argv[1]
    kernel = {"auto": aeg.KERNEL_AUTO, "lsu": aeg.KERNEL_LSU, "bulk": aeg.KERNEL_BULK, "bulkw": aeg.KERNEL_BULKW}[
        sys.argv[2] if len(sys.argv) > 2 else "auto"]
    fn = {"c5": lambda: bench.c5_leg(aeg, torch, kernel),
          "migrate": lambda: bench.migrate_leg(aeg, torch, kernel),
          "overlap": lambda: bench.overlap_leg(aeg, torch, kernel),
          "small_chunk": lambda: bench.small_chunk_leg(aeg, torch, kernel),
          "switch": lambda: switch_cmp(kernel),
          "host_route": lambda: bench.host_route_leg(aeg, torch, kernel),
          "kernel_alone": lambda: bench.kernel_alone_leg(aeg, kernel)}[leg]
    print(json.dumps(fn()), flush=True)


if __name__ == "__main__":
    main()
