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


def fullsize(csv_path, alg_bytes, capture):
    """Merge a single-pass launch list (gpu__time_duration + dram__bytes_{read,write}, one row per
    metric) of the bench's own full-size step into profiles/ncu_summary.json under gather/scatter:
    per-launch DRAM traffic next to the algorithmic bytes of the same launch (bench.py roofline)."""
    txt = open(csv_path).read()
    rows = list(csv.DictReader(io.StringIO(txt[txt.index('"ID"'):])))
    by = collections.defaultdict(lambda: collections.defaultdict(list))
    names = {}
    for r in rows:
        ro = role(r["Kernel Name"])
        if ro:
            by[ro][r["Metric Name"]].append(float(r["Metric Value"].replace(",", "")))
            names[ro] = r["Kernel Name"].split("::")[-1][:60] + f" grid {r['Grid Size']} block {r['Block Size']}"
    out_p = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles", "ncu_summary.json")
    summ = json.load(open(out_p)) if os.path.exists(out_p) else {}
    for ro, m in by.items():
        n = len(m["gpu__time_duration.sum"])
        rd, wr = sum(m["dram__bytes_read.sum"]) / n, sum(m["dram__bytes_write.sum"]) / n
        dur = sum(m["gpu__time_duration.sum"]) / n
        if ro in summ and "16" in summ[ro].get("capture", ""):
            summ[ro + "_set_full_16req"] = summ.pop(ro)
        summ[ro] = {"kernel": names[ro], "capture": capture, "launches": n,
                    "algorithmic_bytes_per_launch": int(alg_bytes),
                    "dram_bytes_per_launch": int(rd + wr), "dram_read_bytes_per_launch": int(rd),
                    "dram_write_bytes_per_launch": int(wr), "duration_us_cold_serialised": round(dur / 1e3, 2),
                    "algorithmic_GBps_cold_serialised": round(alg_bytes / dur, 1),
                    "traffic_over_algorithmic": round((rd + wr) / alg_bytes, 4)}
    json.dump(summ, open(out_p, "w"), indent=1)
    print(json.dumps(summ, indent=1))


if __name__ == "__main__":
    if len(sys.argv) > 1 and sys.argv[1] == "--fullsize":
        fullsize(sys.argv[2], int(sys.argv[3]), sys.argv[4])
    else:
        main(sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/ncu_final")
