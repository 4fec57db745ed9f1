"""Summarise an ncu launch list + --set full captures into profiles/<round>/ (dev tool).

usage: python tools/ncu_summary.py gpurun_out r01 [config]
Writes profiles/<round>/ncu_summary.md, profiles/<round>/launch_shares.csv and
profiles/ncu_traffic.json (per-launch DRAM traffic of each kernel class, read by bench.py).
       python tools/ncu_summary.py gpurun_out r01 --captures-only NAME.md [title]
summarises only the .ncu-rep captures into profiles/<round>/NAME.md.
"""
import collections
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
METRICS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "dram read"),
    ("dram__bytes_write.sum", "dram write"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram % peak"),
    ("lts__throughput.avg.pct_of_peak_sustained_elapsed", "L2 % peak"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "SM % peak"),
    ("pcie__read_bytes.sum.per_second", "PCIe read"),
    ("l1tex__m_xbar2l1tex_read_bytes.sum", "L2->L1 read"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps active %"),
    ("launch__grid_size", "grid"),
    ("launch__registers_per_thread", "regs"),
    ("smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio", "stall long_sb"),
    ("smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio", "stall short_sb"),
    ("smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio", "stall barrier"),
    ("smsp__average_warps_issue_stalled_lg_throttle_per_issue_active.ratio", "stall lg_throttle"),
]
CLASS = {"k_gather": "gather", "k_ondemand": "ondemand", "k_static": "static", "k_classify": "classify",
         "k_finalize": "finalize"}


def kclass(name):
    for k, v in CLASS.items():
        if k in name:
            return v
    return None


def to_bytes(v, unit):
    f = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(unit)
    return float(v) * f if f else None


def captures(src):
    lines = []
    for rep in sorted(x for x in os.listdir(src) if x.endswith(".ncu-rep")):
        raw = subprocess.run(["ncu", "-i", os.path.join(src, rep), "--page", "raw", "--csv"],
                             capture_output=True, text=True).stdout
        rr = list(csv.reader(io.StringIO(raw)))
        if len(rr) < 3:
            continue
        h, u = rr[0], rr[1]
        for r in rr[2:]:
            name = r[h.index("Kernel Name")].split("(ascetic::")[0].replace("void ", "").replace("ascetic::<unnamed>::", "")
            lines += [f"## `{name}` (`{rep}`, `ncu --set full`)", "", "| metric | value | unit |", "|---|---|---|"]
            for m, label in METRICS:
                if m in h:
                    i = h.index(m)
                    lines.append(f"| {label} (`{m}`) | {r[i]} | {u[i]} |")
            lines.append("")
    return lines


def main():
    src, rnd = sys.argv[1], sys.argv[2]
    out_dir = os.path.join(ROOT, "profiles", rnd)
    os.makedirs(out_dir, exist_ok=True)
    if len(sys.argv) > 4 and sys.argv[3] == "--captures-only":
        title = sys.argv[5] if len(sys.argv) > 5 else "ncu captures"
        lines = [f"# {title}", ""] + captures(src)
        open(os.path.join(out_dir, sys.argv[4]), "w").write("\n".join(lines) + "\n")
        print("\n".join(lines))
        return
    cfg = sys.argv[3] if len(sys.argv) > 3 else "c2"
    lines = [f"# ncu summary — round {rnd[1:]}, workload {cfg} (bench.py --steps 1 --warmup 3)", ""]
    # ---- launch list
    rows = list(csv.reader(open(os.path.join(src, "launches.csv"))))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    hdr = rows[hi]
    ki, vi, ui = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
    agg = collections.defaultdict(lambda: [0, 0.0])
    for r in rows[hi + 1:]:
        name = r[ki].split("(")[0].replace("void ", "").replace("ascetic::<unnamed>::", "")
        v = float(r[vi].replace(",", ""))
        v *= {"nsecond": 1e-6, "ns": 1e-6, "usecond": 1e-3, "us": 1e-3, "msecond": 1.0, "ms": 1.0,
              "second": 1e3, "s": 1e3}.get(r[ui], 1.0)
        agg[name][0] += 1
        agg[name][1] += v
    tot = sum(v[1] for v in agg.values())
    lines += ["## Launch list (`ncu --metrics gpu__time_duration.sum --clock-control none`, serialised, cold)", "",
              "| kernel | launches | total ms | share |", "|---|---|---|---|"]
    with open(os.path.join(out_dir, "launch_shares.csv"), "w") as f:
        f.write("kernel,launches,total_ms,share\n")
        for k, v in sorted(agg.items(), key=lambda x: -x[1][1]):
            lines.append(f"| `{k}` | {v[0]} | {v[1]:.3f} | {v[1] / tot:.3f} |")
            f.write(f"{k},{v[0]},{v[1]:.4f},{v[1] / tot:.4f}\n")
    lines += ["", f"Total device time in the listed launches: {tot:.2f} ms", ""]
    # ---- full captures
    traffic = {}
    for rep in sorted(x for x in os.listdir(src) if x.endswith(".ncu-rep")):
        raw = subprocess.run(["ncu", "-i", os.path.join(src, rep), "--page", "raw", "--csv"],
                             capture_output=True, text=True).stdout
        rr = list(csv.reader(io.StringIO(raw)))
        if len(rr) < 3:
            continue
        h, u = rr[0], rr[1]
        for r in rr[2:]:
            name = r[h.index("Kernel Name")].split("(")[0].replace("void ", "").replace("ascetic::<unnamed>::", "")
            lines += [f"## `{name}` (`{rep}`, `ncu --set full`)", "", "| metric | value | unit |", "|---|---|---|"]
            vals = {}
            for m, label in METRICS:
                if m in h:
                    i = h.index(m)
                    lines.append(f"| {label} (`{m}`) | {r[i]} | {u[i]} |")
                    vals[m] = (r[i], u[i])
            lines.append("")
            c = kclass(name)
            if c and "dram__bytes_read.sum" in vals:
                rb = to_bytes(vals["dram__bytes_read.sum"][0].replace(",", ""), vals["dram__bytes_read.sum"][1])
                wb = to_bytes(vals["dram__bytes_write.sum"][0].replace(",", ""), vals["dram__bytes_write.sum"][1])
                if rb is not None and wb is not None:
                    traffic[c] = rb + wb
    open(os.path.join(out_dir, "ncu_summary.md"), "w").write("\n".join(lines) + "\n")
    tp = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    d = json.load(open(tp)) if os.path.exists(tp) else {}
    d.setdefault(cfg, {}).update(traffic)
    d["_note"] = ("dram__bytes_read.sum + dram__bytes_write.sum of ONE launch per kernel class from "
                  "ncu --set full (profiles/<round>/ncu_summary.md); bench.py copies the dominant kernel's value")
    json.dump(d, open(tp, "w"), indent=1)
    print("\n".join(lines))


if __name__ == "__main__":
    main()
