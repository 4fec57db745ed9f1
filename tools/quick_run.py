"""Quick single run of one config on the GPU with per-iteration phase timings (dev tool)."""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402

import graphgen as gg  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--algo", default="sssp")
    ap.add_argument("--scale", type=int, default=20)
    ap.add_argument("--frac-budget", type=float, default=0.5)
    ap.add_argument("--xfer", type=int, default=0)
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--iters", type=int, default=0)
    ap.add_argument("--config", default="")
    ap.add_argument("--gather-ctas", type=int, default=0)
    ap.add_argument("--chunk-cap", type=int, default=0)
    ap.add_argument("--sweep", action="store_true")
    ap.add_argument("--quiet", action="store_true")
    ap.add_argument("--budget-mult", type=float, default=0.0, help="budget = mult x CSR bytes (config runs)")
    ap.add_argument("--algo-override", default="")
    ap.add_argument("--scale-override", type=int, default=0)
    ap.add_argument("--sweep-ctas", default="148,296,444,592,1184")
    ap.add_argument("--buffers", default="3", help="comma list: run once per chunk-buffer count")
    ap.add_argument("--static-ctas", default="0", help="comma list of static CTAs per SM (0 = default)")
    ap.add_argument("--sweep-caps", default="0,32,8")
    a = ap.parse_args()
    import paper_conf_icpp_tangzwgzwy21_b200 as asc
    t0 = time.time()
    if a.config:
        cfg = dict(gg.CONFIGS[a.config])
        want_w = (a.algo_override or cfg["algo"]) == "sssp"
        g = gg.rmat(a.scale_override or cfg["scale"], cfg["tuples"] if not a.scale_override else None, seed=cfg["seed"],
                    permute=cfg["permute"], n=cfg["n"] if not a.scale_override else 0, weights=want_w, name=a.config)
        budget = gg.config_budget(a.config, g) if a.budget_mult <= 0 else int(a.budget_mult * g.csr_bytes)
        algo = gg.CONFIGS[a.config]["algo"] if a.algo_override == "" else a.algo_override
        iters = gg.CONFIGS[a.config].get("iters", 0) if a.iters == 0 else a.iters
    else:
        g = gg.rmat(a.scale, seed=2, weights=(a.algo == "sssp"))
        budget = int(a.frac_budget * g.csr_bytes)
        algo, iters = a.algo, a.iters
    print(f"gen {time.time()-t0:.1f}s n={g.n} m={g.m}", flush=True)
    t0 = time.time()
    asc.load_csr(g.off, g.nbr, pairs=g.pairs, symmetric=True, sorted_rows=True)   # as bench.py
    print(f"load {time.time()-t0:.2f}s", flush=True)
    asc.set_budget(budget)
    asc.set_option("xfer_mode", a.xfer)
    asc.set_option("gather_ctas", a.gather_ctas)
    asc.set_option("chunk_cap", a.chunk_cap)
    src = gg.sources(g, 1, seed=1)[0]
    if a.sweep:
        for gc in [int(x) for x in a.sweep_ctas.split(',')]:
            for cc in [int(x) << 20 for x in a.sweep_caps.split(',')]:
                asc.set_option("gather_ctas", gc)
                asc.set_option("chunk_cap", cc)
                best = None
                for r in range(2):
                    asc.run(algo, src, iters)
                    st, _ = asc.stats(per_iter=False)
                    if best is None or st["time_run_s"] < best["time_run_s"]:
                        best = st
                print(f"gather_ctas={gc:5d} chunk_cap={cc>>20:4d}MiB run_ms={best['time_run_s']*1e3:8.2f} "
                      f"gather_GBs={best['gather_bytes']/max(best['time_gather_s'],1e-9)/1e9:6.2f} "
                      f"ondemand_ms={best['time_ondemand_s']*1e3:7.2f} chunks={best['chunks_total']} "
                      f"GTEPS={best['active_arcs_total']/best['time_run_s']/1e9:.3f}", flush=True)
        asc.set_option("gather_ctas", a.gather_ctas)
        asc.set_option("chunk_cap", a.chunk_cap)
    for nb, sc in [(int(x), int(y)) for x in a.buffers.split(",") for y in a.static_ctas.split(",")]:
      asc.set_option("chunk_buffers", nb)
      asc.set_option("static_ctas_per_sm", sc)
      print("static_ctas_per_sm", sc, end=" ")
      asc.set_budget(budget)
      for r in range(a.reps):
        asc.run(algo, src, iters)
        st, its = asc.stats()
        print("buffers", nb, json.dumps({k: st[k] for k in ["iterations", "s", "h2d_payload_bytes", "h2d_static_fill_bytes",
                                              "active_arcs_total", "chunks_total", "dma_chunks", "gather_chunks",
                                              "time_run_s", "time_fill_s", "time_h2d_busy_s", "gteps",
                                              "chunk_cap"]}), flush=True)
        b_e = g.b_e
        ks = {"static": (st["static_arcs"] * (b_e + 4), st["time_static_s"]),
              "ondemand": (st["ondemand_arcs"] * (b_e + 4), st["time_ondemand_s"]),
              "gather": (st["gather_bytes"], st["time_gather_s"]),
              "classify": (0, st["time_classify_s"]), "finalize": (0, st["time_finalize_s"])}
        print("  kernels:", {k: (round(t * 1e3, 3), round(b / t / 1e9, 1) if t > 0 else 0) for k, (b, t) in ks.items()},
              f"GTEPS={st['active_arcs_total'] / st['time_run_s'] / 1e9:.2f} "
              f"static_Garcs/s={st['static_arcs'] / max(st['time_static_s'], 1e-9) / 1e9:.1f}", flush=True)
    for i in ([] if a.quiet else its):
        print({k: (round(v, 3) if isinstance(v, float) else v) for k, v in i.items() if k != "digest"})


if __name__ == "__main__":
    main()
