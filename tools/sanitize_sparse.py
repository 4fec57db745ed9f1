"""Small emulated P = 3 runs with the sparse exchange, for compute-sanitizer (dev tool)."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen as gg                              # noqa: E402
import paper_conf_icpp_tangzwgzwy21_b200 as asc    # noqa: E402

asc.set_device(0)
for algo in ["bfs", "sssp", "cc"]:
    g = gg.rmat(10, seed=5, weights=(algo == "sssp"))
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    asc.unload()
    asc.emulate_ranks(3)
    asc.load_csr(g.off, g.nbr, pairs=g.pairs, symmetric=True)
    asc.set_option("chunk_cap", 4096)
    asc.set_budget(g.csr_bytes // 8, 0.4)
    outs = []
    for d in [0, 1]:
        asc.set_option("sparse_exchange", d)
        asc.run(algo, src, 0)
        outs.append(asc.get_result().copy())
        print(algo, "d", d, "sparse iterations", asc.stats()[0]["sparse_exchanges"])
    assert np.array_equal(outs[0], outs[1])
asc.unload()
print("ok")
