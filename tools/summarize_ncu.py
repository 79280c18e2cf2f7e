"""Summarise ncu captures into profiles/ncu_summary.json (read here, no GPU needed):
    python tools/summarize_ncu.py gpurun_out/ncu_final
Per kernel role (gather = copy_*<1,0>, scatter = copy_*<0,1>, migrate = copy_*<1,1>): launches in
the full capture, mean duration, DRAM bytes per launch (read + write), DRAM throughput % of peak,
and the kernel-time totals from the launch list (cold, serialised)."""
import collections
import csv
import io
import json
import os
import subprocess
import sys

ROLE = {"<1, 0>": "gather", "<0, 1>": "scatter", "<1, 1>": "migrate", "<0, 0>": "memmove"}


def role(name):
    for k, v in ROLE.items():
        if k in name:
            return v
    return None


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    return rows[0], rows[2:]


def main(d):
    summ = {}
    for rep in ("swap.ncu-rep", "migrate.ncu-rep"):
        p = os.path.join(d, rep)
        if not os.path.exists(p):
            continue
        h, rows = raw(p)
        g = lambda r, k: r[h.index(k)]  # noqa: E731
        by = collections.defaultdict(list)
        for r in rows:
            ro = role(g(r, "Kernel Name"))
            if ro:
                by[ro].append(r)
        for ro, rs in by.items():
            # keep the full-size launches (the largest grid-work ones) for per-launch figures
            dur = [float(g(r, "gpu__time_duration.sum")) for r in rs]
            rd = [float(g(r, "dram__bytes_read.sum")) for r in rs]
            wr = [float(g(r, "dram__bytes_write.sum")) for r in rs]
            pct = [float(g(r, "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed")) for r in rs]
            top = sorted(range(len(rs)), key=lambda i: -(rd[i] + wr[i]))[: max(1, len(rs) // 2)]
            summ[ro] = {"kernel": g(rs[0], "Kernel Name")[:80], "capture": f"{d}/{rep}", "launches_captured": len(rs),
                        "duration_us": round(sum(dur[i] for i in top) / len(top), 2),
                        "dram_bytes_per_launch": int(1e6 * sum(rd[i] + wr[i] for i in top) / len(top)),
                        "dram_read_bytes_per_launch": int(1e6 * sum(rd[i] for i in top) / len(top)),
                        "dram_throughput_pct_mean": round(sum(pct[i] for i in top) / len(top), 1),
                        "grid": g(rs[0], "Grid Size"), "block": g(rs[0], "Block Size")}
    lp = os.path.join(d, "launches_bench.csv")
    if os.path.exists(lp):
        rows = list(csv.reader(open(lp)))
        i0 = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
        h, data = rows[i0], rows[i0 + 1:]
        tot = collections.Counter()
        cnt = collections.Counter()
        for r in data:
            if len(r) < len(h) or r[h.index("Metric Name")] != "gpu__time_duration.sum":
                continue
            nm = r[h.index("Kernel Name")]
            key = role(nm) if role(nm) else nm.split("(")[0][-40:]
            tot[key] += float(r[h.index("Metric Value")].replace(",", ""))
            cnt[key] += 1
        summ["launch_list"] = {k: {"launches": cnt[k], "total_us": round(v / 1e3, 1)} for k, v in tot.most_common()}
    json.dump(summ, open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles",
                                      "ncu_summary.json"), "w"), indent=1)
    print(json.dumps(summ, indent=1))


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/ncu_final")
