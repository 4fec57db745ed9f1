"""Probe: fill / swap throughput of the chunk-copy kernel and the host cost of the replacement
step on C2 (random placement fill vs front DMA fill; K sweep with per-iteration timing)."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen as gg  # noqa: E402


def main():
    import paper_conf_icpp_tangzwgzwy21_b200 as asc
    key = sys.argv[1] if len(sys.argv) > 1 else "c2"
    g = gg.config_graph(key)
    budget = gg.config_budget(key, g)
    c = gg.CONFIGS[key]
    src = gg.sources(g, 1, seed=c["seed"])[0]
    asc.load_csr(g.off, g.nbr, pairs=g.pairs)
    for placement, K in [(0, 0), (2, 0), (0, 4096)]:
        asc.set_option("static_placement", placement)
        asc.set_option("replace_chunks", K)
        asc.set_budget(budget)
        for rep in range(2):
            t0 = time.time()
            asc.run(c["algo"], src, 5 if c["algo"] == "pr" else 0)
            wall = time.time() - t0
        st, its = asc.stats()
        print(json.dumps(dict(placement=placement, K=K, run_ms=round(st["time_run_s"] * 1e3, 2), wall_ms=round(wall * 1e3, 1),
                              fill_gb=st["h2d_static_fill_bytes"] / 1e9, fill_ms=round(st["time_fill_s"] * 1e3, 2),
                              fill_gbs=round(st["h2d_static_fill_bytes"] / max(st["time_fill_s"], 1e-9) / 1e9, 2),
                              replace_gb=st["h2d_replace_bytes"] / 1e9, replace_ms=round(st["time_replace_s"] * 1e3, 2),
                              host_ms=round(st["time_host_s"] * 1e3, 2), miss_gb=st["h2d_payload_bytes"] / 1e9,
                              swaps=st["swaps_total"], s=st["s"])), flush=True)
        for i in its:
            print("  ", {k: i[k] for k in ["t", "nA", "swaps", "ms_h2d", "ms_total", "ms_link_tail", "s_static"]})
    asc.set_option("static_placement", 0)
    asc.set_option("replace_chunks", 0)


if __name__ == "__main__":
    main()
