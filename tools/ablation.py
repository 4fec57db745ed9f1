"""Ablations of SURVEY §8(f) NEXT(1), the paper's Fig. 8 / 10 / 11 on synthetic graphs:
  * static-fraction sweep R in {0 (everything on demand, the Subway-like self-baseline), 0.2 ...
    1.0} next to Eq. 2's R (K = 0.1) at the config's budget (Fig. 10);
  * overlap of static computing with the transfer on / off (Fig. 8, "overlapping savings",
    P:1196-1245);
  * budget sweep at Eq. 2's R (Fig. 11).
Writes one JSON line per run and a markdown table. usage: python tools/ablation.py c2 [c3 c4]"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import graphgen as gg  # noqa: E402


def main():
    import paper_conf_icpp_tangzwgzwy21_b200 as asc
    cfgs = sys.argv[1:] or ["c2"]
    rows = []
    for key in cfgs:
        c = gg.CONFIGS[key]
        g = gg.config_graph(key)
        budget = gg.config_budget(key, g)
        algo = c["algo"]
        iters = 5 if algo == "pr" else 0
        src = gg.sources(g, 1, seed=c["seed"])[0]
        asc.load_csr(g.off, g.nbr, pairs=g.pairs)

        def one(label, nbytes, frac, overlap=1, rear=0, eq3=0, replace=0, run_algo=None, tol=10000):
            asc.set_option("overlap", overlap)
            asc.set_option("static_placement", rear)
            asc.set_option("repartition", eq3)
            asc.set_option("replace_chunks", replace)
            asc.set_option("prd_tol_ppm", tol)
            asc.set_budget(nbytes, frac)
            ra = run_algo or algo
            best = None
            for _ in range(2):
                asc.run(ra, src, iters if ra == algo else 0)
                st, _ = asc.stats(per_iter=False)
                if best is None or st["time_run_s"] < best["time_run_s"]:
                    best = st
            r = dict(config=key, study=label if ra == algo else f"{label} ({ra}, tol {tol} ppm, "
                     f"{best['iterations']} it)", repartitions=best["repartitions"],
                     budget_frac_of_csr=round(nbytes / g.csr_bytes, 3),
                     R=round(best["static_fraction_used"], 4), overlap=overlap, run_ms=round(best["time_run_s"] * 1e3, 2),
                     gteps=round(best["active_arcs_total"] / best["time_run_s"] / 1e9, 3),
                     fill_gb=round(best["h2d_static_fill_bytes"] / 1e9, 3),
                     miss_gb=round(best["h2d_payload_bytes"] / 1e9, 3),
                     replace_k=replace, swaps=best["swaps_total"], replace_gb=round(best["h2d_replace_bytes"] / 1e9, 3),
                     replace_ms=round(best["time_replace_s"] * 1e3, 2), host_ms=round(best["time_host_s"] * 1e3, 2),
                     h2d_gb=round((best["h2d_static_fill_bytes"] + best["h2d_payload_bytes"]
                                   + best["h2d_replace_bytes"]) / 1e9, 3))
            rows.append(r)
            print(json.dumps(r), flush=True)

        only = os.environ.get("ABLATION_ONLY", "")
        one("eq2", budget, -1.0)
        if only == "replace":
            # §3.4 data replacement: K chunk swaps per iteration, counter by algorithm
            for K in [16, 256, 4096]:
                one("replace", budget, -1.0, replace=K)
            for seed in [1, 2]:   # §5 random initial chunks
                asc.set_option("placement_seed", seed)
                one(f"random-fill seed {seed}", budget, -1.0, rear=2)
        elif only == "prd":
            # PageRank-delta (Subway's PR) on the config graph and budget
            for tol in [10000, 300000]:
                one("prd", budget, -1.0, run_algo="prd", tol=tol)
        elif os.environ.get("ABLATION_QUICK") != "1":
            for R in [0.0, 0.2, 0.4, 0.6, 0.8, 0.9, 0.95, 1.0]:
                one("R-sweep", budget, R)
            one("overlap-off", budget, -1.0, overlap=0)
            for f in [0.25, 0.5, 0.75, 1.0]:
                one("budget-sweep", int(f * g.csr_bytes), -1.0)
        if only not in ("replace", "prd"):
            one("rear-fill", budget, -1.0, rear=1)
            one("eq3-repartition", budget, -1.0, eq3=1)
        asc.set_option("overlap", 1)
        asc.set_option("replace_chunks", 0)
        asc.set_option("static_placement", 0)
        asc.set_option("repartition", 0)
        asc.unload()
        del g
    out = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "gpurun_out", "ablation.md")
    with open(out, "w") as f:
        f.write("| config | study | budget/CSR | R | overlap | K | run ms | GTEPS | fill GB | miss GB | swaps | "
                "replace GB | replace ms | host ms | H2D GB |\n")
        f.write("|---|---|---|---|---|---|---|---|---|---|---|---|---|---|---|\n")
        for r in rows:
            f.write(f"| {r['config']} | {r['study']} | {r['budget_frac_of_csr']} | {r['R']} | {r['overlap']} | "
                    f"{r['replace_k']} | {r['run_ms']} | {r['gteps']} | {r['fill_gb']} | {r['miss_gb']} | "
                    f"{r['swaps']} | {r['replace_gb']} | {r['replace_ms']} | {r['host_ms']} | {r['h2d_gb']} |\n")
    print(open(out).read())


if __name__ == "__main__":
    t0 = time.time()
    main()
    print(f"total {time.time() - t0:.1f}s")
