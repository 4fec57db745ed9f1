"""Launch-list shares from an ncu --csv log (dev tool): per kernel, launches, total device ms, share.
    python tools/launch_shares.py gpurun_out/launches_c4.csv > profiles/r02/launch_shares_c4.md"""
import collections
import csv
import sys

UNIT = {"nsecond": 1e-6, "ns": 1e-6, "usecond": 1e-3, "us": 1e-3, "msecond": 1, "ms": 1, "second": 1e3, "s": 1e3}


def main():
    rows = list(csv.reader(open(sys.argv[1])))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    h = rows[hi]
    ki, mi, vi, ui = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"), h.index("Metric Unit")
    agg = collections.defaultdict(lambda: [0, 0.0])
    for r in rows[hi + 1:]:
        if r[mi] != "gpu__time_duration.sum":
            continue
        name = r[ki].split("(")[0].replace("void ", "")
        for p in ("ascetic::<unnamed>::", "ascetic::(anonymous namespace)::", "ascetic::"):
            name = name.replace(p, "")
        agg[name][0] += 1
        agg[name][1] += float(r[vi].replace(",", "")) * UNIT.get(r[ui], 1.0)
    tot = sum(v[1] for v in agg.values())
    print("| kernel | launches | total ms | share |\n|---|---|---|---|")
    for k, v in sorted(agg.items(), key=lambda x: -x[1][1]):
        print(f"| `{k}` | {v[0]} | {v[1]:.3f} | {v[1] / tot:.3f} |")
    print(f"\nTotal device time in the listed launches: {tot:.2f} ms")


if __name__ == "__main__":
    main()
