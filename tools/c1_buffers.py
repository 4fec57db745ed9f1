"""C1 (BFS RMAT-16, 25 % budget) run time vs the number of chunk buffers, 0 = auto (dev tool)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen as gg                              # noqa: E402
import paper_conf_icpp_tangzwgzwy21_b200 as asc    # noqa: E402

g = gg.config_graph("c1")
budget = gg.config_budget("c1", g)
srcs = gg.sources(g, 8, seed=1)
asc.set_device(0)
for nb in [2, 3, 4, 0, 2, 3, 4, 0]:
    asc.unload()
    asc.load_csr(g.off, g.nbr, pairs=g.pairs, symmetric=True)
    asc.set_option("chunk_buffers", nb)
    asc.set_budget(budget)
    for s in srcs[:3]:
        asc.run("bfs", s, 0)                        # warm-up
    ms, arcs = 0.0, 0
    for s in srcs:
        asc.run("bfs", s, 0)
        st = asc.stats(per_iter=False)[0]
        ms += st["time_run_s"] * 1e3
        arcs += st["active_arcs_total"]
    print(f"chunk_buffers={nb}: {ms / len(srcs):.3f} ms per run, {arcs / ms / 1e6:.3f} GTEPS, chunks/run "
          f"{st['chunks_total']}")
