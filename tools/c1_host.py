"""C1: wall time of ascetic_run vs the library's device-timed run, with per-phase timing on/off (dev tool)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen as gg                              # noqa: E402
import paper_conf_icpp_tangzwgzwy21_b200 as asc    # noqa: E402

g = gg.config_graph("c1")
budget = gg.config_budget("c1", g)
srcs = gg.sources(g, 8, seed=1)
asc.set_device(0)
asc.load_csr(g.off, g.nbr, pairs=g.pairs, symmetric=True)
asc.set_budget(budget)
for timing in [1, 0, 1, 0]:
    asc.set_option("timing", timing)
    for s in srcs[:3]:
        asc.run("bfs", s, 0)
    wall, lib = 0.0, 0.0
    for s in srcs:
        t0 = time.perf_counter()
        asc.run("bfs", s, 0)
        wall += time.perf_counter() - t0
        lib += asc.stats(per_iter=False)[0]["time_run_s"]
    print(f"timing={timing}: wall {wall / len(srcs) * 1e3:.3f} ms per run, library run {lib / len(srcs) * 1e3:.3f} ms")
