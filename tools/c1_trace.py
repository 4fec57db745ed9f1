"""ASCETIC_TRACE timeline of one C1 BFS run (dev tool): python tools/c1_trace.py (set ASCETIC_TRACE=1)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen as gg                              # noqa: E402
import paper_conf_icpp_tangzwgzwy21_b200 as asc    # noqa: E402

g = gg.config_graph("c1")
budget = gg.config_budget("c1", g)
src = gg.sources(g, 1, seed=1)[0]
asc.set_device(0)
asc.load_csr(g.off, g.nbr, pairs=g.pairs, symmetric=True)
asc.set_budget(budget)
for rep in range(4):
    t0 = time.perf_counter()
    asc.run("bfs", src, 0)
    t1 = time.perf_counter()
st, its = asc.stats()
print(f"wall {1e3 * (t1 - t0):.3f} ms, run {st['time_run_s'] * 1e3:.3f} ms, fill {st['time_fill_s'] * 1e3:.3f} ms, "
      f"host {st['time_host_s'] * 1e3:.3f} ms, launches {st['kernel_launches']}, iters {st['iterations']}", file=sys.stderr)
for i in its:
    print(f"t={i['t']} |A|={i['nA']} runs={i['nruns']} chunks={i['chunks']} mode={i['mode']} cls={i['ms_classify']:.3f} "
          f"st={i['ms_static']:.3f} od={i['ms_ondemand']:.3f} h2d={i['ms_h2d']:.3f} fin={i['ms_finalize']:.3f} "
          f"tot={i['ms_total']:.3f}", file=sys.stderr)
