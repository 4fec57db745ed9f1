"""Resident (budget >= CSR) edge-kernel throughput, A/B of the SSSP/CC min-update forms (dev tool, GPU).
Prints per algorithm and relax mode: run ms, static-hit kernel time, static G arcs/s and the
algorithmic HBM rate (b_e + 4 bytes per arc).
    python tools/resident_ab.py --graph rmat24 | c3
"""
import argparse
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen as gg                              # noqa: E402
import paper_conf_icpp_tangzwgzwy21_b200 as asc    # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--graph", default="rmat24")
    ap.add_argument("--algos", default="bfs,sssp,cc,pr")
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--pr-iters", type=int, default=5)
    ap.add_argument("--pr-segments", default="0,67108864", help="PR: pr_segment values to A/B")
    a = ap.parse_args()
    asc.set_device(0)
    graphs = {}
    for algo in a.algos.split(","):
        w = algo == "sssp"
        if w not in graphs:
            if a.graph == "c3":
                c = gg.CONFIGS["c3"]
                graphs[w] = gg.rmat(c["scale"], c["tuples"], seed=c["seed"], permute=True, n=c["n"], weights=w)
            else:
                graphs[w] = gg.rmat(int(a.graph[4:]), seed=2, weights=w)
        g = graphs[w]
        src = int(np.argmax(np.diff(g.off.astype(np.int64))))
        asc.load_csr(g.off, g.nbr, pairs=g.pairs, symmetric=True, sorted_rows=True)
        asc.set_budget(int(1.2 * g.csr_bytes))
        modes = [1, 2] if algo in ("sssp", "cc") else ([int(x) for x in a.pr_segments.split(",")] if algo == "pr" else [0])
        for mode in modes:
            if algo == "pr":
                asc.set_option("pr_segment", mode)
            else:
                asc.set_option("relax_mode", mode)
            best = None
            for _ in range(a.reps):
                asc.run(algo, src, a.pr_iters if algo == "pr" else 0)
                st, _ = asc.stats(per_iter=False)
                if best is None or st["time_run_s"] < best["time_run_s"]:
                    best = st
            st = best
            ex = st["time_run_s"] - st["time_fill_s"]
            rate = st["static_arcs"] / max(1e-12, st["time_static_s"])
            print(f"{a.graph} {algo:4s} {'pr_segment' if algo == 'pr' else 'relax'}={mode} passes={st['pr_segment_passes']} n={g.n} m={g.m} iters={st['iterations']} run {st['time_run_s']*1e3:8.2f} ms "
                  f"excl fill {ex*1e3:8.2f} ms static {st['time_static_s']*1e3:8.2f} ms finalize {st['time_finalize_s']*1e3:6.2f} ms "
                  f"classify {st['time_classify_s']*1e3:6.2f} ms  static {rate/1e9:6.1f} G arcs/s = "
                  f"{rate * (g.b_e + 4) / 1e12:5.2f} TB/s algorithmic  whole {st['active_arcs_total']/ex/1e9:6.1f} GTEPS excl fill",
                  flush=True)
        asc.set_option("relax_mode", 0)
        asc.set_option("pr_segment", 128 << 20)
    asc.unload()


if __name__ == "__main__":
    main()
