"""Short run of the fused migrate kernel (configs[2] Llama-2-13B shapes, same-GPU peer pool) for ncu:
    ncu --set full -k regex:copy_ python tools/profile_migrate.py"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_sosp_xiang0qyzyzl0025_b200 as aeg  # noqa: E402

if __name__ == "__main__":
    print(bench.migrate_leg(aeg, torch, aeg.KERNEL_AUTO))
