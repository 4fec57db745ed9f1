"""Transfer-engine A/B on a config (dev tool, GPU): gap bridging and copy-engine long runs.
    python tools/gather_ab.py --config c4 --gaps 0,64,256,1024 --ce 0,1048576
Prints per setting: best run ms, GTEPS, gather payload rate, the SM gather's load/payload ratio."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen as gg                              # noqa: E402
import paper_conf_icpp_tangzwgzwy21_b200 as asc    # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c4")
    ap.add_argument("--gaps", default="0,64,256,1024")
    ap.add_argument("--ce", default="0,1048576")
    ap.add_argument("--reps", type=int, default=2)
    ap.add_argument("--span", default="0,85", help="span_density percentages (0 = no span DMA)")
    ap.add_argument("--ratio", default="200", help="span_max_ratio percentages")
    a = ap.parse_args()
    c = gg.CONFIGS[a.config]
    algo = c["algo"]
    g = gg.config_graph(a.config)
    budget = gg.config_budget(a.config, g)
    src = gg.sources(g, 1, seed=c["seed"])[0]
    iters = c.get("iters", 0) if algo == "pr" else 0
    asc.set_device(0)
    asc.load_csr(g.off, g.nbr, pairs=g.pairs, symmetric=True)
    asc.set_budget(budget)
    asc.run(algo, src, iters)
    for rnd in range(2):                                  # two interleaved rounds
        for ce, gap, sp, ra in [(int(c_), int(g_), int(s_), int(r_)) for s_ in a.span.split(",") for c_ in a.ce.split(",")
                                for g_ in a.gaps.split(",") for r_ in a.ratio.split(",")]:
            if True:
                asc.set_option("span_max_ratio", ra)
                asc.set_option("ce_min_run", ce)
                asc.set_option("gap_bridge", gap)
                asc.set_option("span_density", sp)
                best = None
                for _ in range(a.reps):
                    asc.run(algo, src, iters)
                    st, _ = asc.stats(per_iter=False)
                    if best is None or st["time_run_s"] < best["time_run_s"]:
                        best = st
                st = best
                sm = st["gather_bytes"] - st["gather_ce_bytes"]
                print(f"round {rnd} {a.config} span={sp:3d} ratio={ra:4d} ce_min_run={ce:8d} gap={gap:5d} run {st['time_run_s']*1e3:8.1f} ms "
                      f"{st['gteps']:6.2f} GTEPS  gather {st['gather_bytes']/1e9:6.2f} GB in {st['time_gather_s']*1e3:7.1f} ms "
                      f"= {st['gather_bytes']/max(1e-9, st['time_gather_s'])/1e9:5.1f} GB/s (CE {st['gather_ce_bytes']/1e9:5.2f} GB)  "
                      f"SM load/payload {st['gather_load_bytes']/max(1, sm):.3f}  dma {st['dma_bytes']/1e9:5.2f} GB "
                      f"{st['dma_bytes']/max(1e-9, st['time_dma_s'])/1e9:5.1f} GB/s  span {st['span_chunks']} windows "
                      f"{st['span_payload_bytes']/1e9:.2f} GB payload in {st['span_link_bytes']/1e9:.2f} GB", flush=True)
    asc.unload()


if __name__ == "__main__":
    main()
