"""C5 on ONE GPU (out-of-core variant): RMAT-29, 40 GB device budget. BFS parity vs the oracle at
full size, PR 2 iterations parity, PR 43 iterations timing. Dev tool (long: generation ~8 min)."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402

import graphgen as gg  # noqa: E402


def main():
    import paper_conf_icpp_tangzwgzwy21_b200 as asc
    import oracle
    t0 = time.time()
    g = gg.config_graph("c5")
    print(f"gen {time.time() - t0:.1f}s n={g.n} m={g.m} csr={g.csr_bytes / 1e9:.1f} GB", flush=True)
    budget = gg.config_budget("c5", g)
    t0 = time.time()
    asc.load_csr(g.off, g.nbr)
    asc.set_budget(budget)
    print(f"load+budget {time.time() - t0:.1f}s", flush=True)
    keys = ["iterations", "s", "h2d_payload_bytes", "h2d_static_fill_bytes", "active_arcs_total", "time_run_s",
            "time_fill_s", "gteps", "chunk_cap", "vertex_state_bytes", "static_bytes"]
    src = gg.sources(g, 1, seed=5)[0]
    for r in range(2):
        asc.run("bfs", src)
        st, its = asc.stats()
        print("bfs", json.dumps({k: st[k] for k in keys}), flush=True)
    res = asc.get_result().copy()
    p = oracle.placer(g.off, 4, budget)
    stat = oracle.static_prefix(g.n, p.s)
    t0 = time.time()
    ref = oracle.run("bfs", g.off, g.nbr, src=src, is_static=stat)
    print(f"oracle bfs {time.time() - t0:.1f}s", flush=True)
    F = ["nA", "nH", "nM", "nruns", "active_arcs", "hit_arcs", "miss_bytes", "digest"]
    print("bfs values equal", bool(np.array_equal(res, ref.values)),
          "records equal", [{f: i[f] for f in F} for i in its] == [{f: x[f] for f in F} for x in ref.records],
          flush=True)
    asc.run("pr", 0, 2)
    res = asc.get_result().astype(np.float64)
    st, its = asc.stats()
    print("pr2", json.dumps({k: st[k] for k in keys}), flush=True)
    t0 = time.time()
    ref = oracle.run("pr", g.off, g.nbr, max_iters=2, is_static=stat)
    print(f"oracle pr2 {time.time() - t0:.1f}s", flush=True)
    rel = np.abs(res - ref.values) / ref.values
    print("pr2 max rel", float(rel.max()), "L1", float(np.abs(res - ref.values).sum()),
          "records equal", [{f: i[f] for f in F} for i in its] == [{f: x[f] for f in F} for x in ref.records],
          flush=True)
    asc.run("pr", 0, 43)
    st, its = asc.stats()
    print("pr43", json.dumps({k: st[k] for k in keys}), flush=True)
    asc.unload()


if __name__ == "__main__":
    main()
