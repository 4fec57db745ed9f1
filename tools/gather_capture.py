"""One C4 CC run with the SM gather only (no copy-engine runs, no span DMA), for an ncu capture of gather launches
whose payload is known: iteration 1's windows are full chunks of chunk_cap bytes (dev tool).
    ncu --set full -k regex:k_gather16 -s 1 -c 2 -o prof python tools/gather_capture.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen as gg                              # noqa: E402
import paper_conf_icpp_tangzwgzwy21_b200 as asc    # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "c4"
c = gg.CONFIGS[cfg]
g = gg.config_graph(cfg)
asc.set_device(0)
asc.load_csr(g.off, g.nbr, pairs=g.pairs, symmetric=True, sorted_rows=True)
asc.set_option("ce_min_run", 0)
asc.set_option("span_density", 0)
asc.set_budget(gg.config_budget(cfg, g))
src = gg.sources(g, 1, seed=c["seed"])[0]
asc.run(c["algo"], src, 0)
st, its = asc.stats()
print("chunk_cap", st["chunk_cap"], "per-iteration (mode, chunks, miss bytes):",
      [(i["mode"], i["chunks"], i["miss_bytes"]) for i in its], flush=True)
asc.unload()
