"""One resident run (budget 1.2 x CSR) per listed algorithm, for ncu captures of the static-hit
kernels (dev tool).  python tools/resident_one.py --graph rmat24 --algos cc,sssp"""
import argparse
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen as gg                              # noqa: E402
import paper_conf_icpp_tangzwgzwy21_b200 as asc    # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--graph", default="rmat24")
ap.add_argument("--algos", default="cc")
a = ap.parse_args()
asc.set_device(0)
for algo in a.algos.split(","):
    w = algo == "sssp"
    if a.graph == "c3":
        c = gg.CONFIGS["c3"]
        g = gg.rmat(c["scale"], c["tuples"], seed=c["seed"], permute=True, n=c["n"], weights=w)
    else:
        g = gg.rmat(int(a.graph[4:]), seed=2, weights=w)
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    asc.load_csr(g.off, g.nbr, pairs=g.pairs, symmetric=True, sorted_rows=True)
    asc.set_budget(int(1.2 * g.csr_bytes))
    asc.run(algo, src, 3 if algo == "pr" else 0)
    st, _ = asc.stats(per_iter=False)
    print(a.graph, algo, st["iterations"], st["time_static_s"], st["static_arcs"], flush=True)
asc.unload()
