"""Per-iteration miss-run statistics of one C2 run (dev tool): how long the miss runs are, which
transfer mode each iteration took, and its link rate. python tools/c2_iters.py"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen as gg                              # noqa: E402
import paper_conf_icpp_tangzwgzwy21_b200 as asc    # noqa: E402

g = gg.config_graph("c2")
budget = gg.config_budget("c2", g)
src = gg.sources(g, 1, seed=2)[0]
asc.set_device(0)
asc.load_csr(g.off, g.nbr, pairs=g.pairs, symmetric=True)
asc.set_budget(budget)
for rep in range(2):
    asc.run("sssp", src, 0)
st, its = asc.stats()
print(f"run {st['time_run_s'] * 1e3:.1f} ms, fill {st['time_fill_s'] * 1e3:.1f} ms, payload {st['h2d_payload_bytes'] / 1e9:.3f} GB")
for i in its:
    avg = i["miss_bytes"] / max(1, i["nruns"])
    gbs = i["miss_bytes"] / max(1e-9, i["ms_h2d"] * 1e-3) / 1e9
    print(f"t={i['t']:2d} |A|={i['nA']:9d} |M|={i['nM']:9d} runs={i['nruns']:9d} miss={i['miss_bytes'] / 1e6:8.1f} MB "
          f"avg_run={avg:9.0f} B mode={i['mode']} h2d={i['ms_h2d']:7.2f} ms ({gbs:5.1f} GB/s)")
