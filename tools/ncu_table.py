"""Markdown table of ncu --set full captures (dev tool): one row per launch (the `--top` longest per
kernel), with duration, DRAM and L2 throughput, L2 sector traffic and hit rates, atomics.

    python tools/ncu_table.py OUT.md "title" gpurun_out/prof_a.ncu-rep [more.ncu-rep ...] [--top 2]
"""
import collections
import csv
import io
import subprocess
import sys

COLS = [
    ("gpu__time_duration.sum", "us", 1e-3),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "DRAM %", 1),
    ("dram__bytes_read.sum", "DRAM rd MB", 1e-6),
    ("lts__throughput.avg.pct_of_peak_sustained_elapsed", "L2 %", 1),
    ("lts__t_sectors.sum.pct_of_peak_sustained_elapsed", "L2 sectors %", 1),
    ("lts__t_sectors.sum", "L2 sectors M", 1e-6),
    ("lts__t_sector_hit_rate.pct", "L2 hit %", 1),
    ("l1tex__t_sector_hit_rate.pct", "L1 hit %", 1),
    ("l1tex__t_requests_pipe_lsu_mem_global_op_atom.sum", "atom req M", 1e-6),
    ("l1tex__t_requests_pipe_lsu_mem_global_op_red.sum", "red req M", 1e-6),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps %", 1),
    ("smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio", "stall long_sb", 1),
    ("pcie__read_bytes.sum.per_second", "PCIe rd GB/s", 1e-9),
]
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1, "usecond": 1e3, "msecond": 1e6,
         "second": 1e9, "ns": 1, "us": 1e3, "ms": 1e6, "s": 1e9, "byte/s": 1, "Kbyte/s": 1e3, "Mbyte/s": 1e6,
         "Gbyte/s": 1e9, "Tbyte/s": 1e12}


def rows_of(rep):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rr = list(csv.reader(io.StringIO(raw)))
    if len(rr) < 3:
        return []
    h, u = rr[0], rr[1]
    out = []
    for r in rr[2:]:
        name = r[h.index("Kernel Name")]
        name = name.split("(DevState")[0].split("(ascetic")[0].replace("void ", "").replace("ascetic::<unnamed>::", "")
        name = name.replace("(anonymous namespace)::", "").replace("ascetic::", "").replace("<unnamed>::", "")
        name = name.replace("unnamed>::", "").split("(Queues")[0]
        vals = {}
        for m, _, sc in COLS:
            if m in h:
                i = h.index(m)
                try:
                    v = float(r[i].replace(",", ""))
                except ValueError:
                    continue
                if u[i] in SCALE and ("bytes" in m or "duration" in m):
                    v *= SCALE[u[i]]
                vals[m] = v * sc
        out.append((name, vals))
    return out


def main():
    args = sys.argv[1:]
    top = 2
    if "--top" in args:
        i = args.index("--top")
        top = int(args[i + 1])
        del args[i:i + 2]
    out, title, reps = args[0], args[1], args[2:]
    lines = [f"# {title}", "", "| capture | kernel | " + " | ".join(c[1] for c in COLS) + " |",
             "|---|---|" + "---|" * len(COLS)]
    for rep in reps:
        per = collections.defaultdict(list)
        for name, vals in rows_of(rep):
            per[name].append(vals)
        for name, lst in per.items():
            lst.sort(key=lambda v: -v.get("gpu__time_duration.sum", 0))
            for vals in lst[:top]:
                cells = [f"{vals[m]:.3g}" if m in vals else "" for m, _, _ in COLS]
                lines.append(f"| `{rep.split('/')[-1]}` | `{name}` | " + " | ".join(cells) + " |")
    open(out, "w").write("\n".join(lines) + "\n")
    print("\n".join(lines))


if __name__ == "__main__":
    main()
