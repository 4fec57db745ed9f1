"""Dense vs sparse exchange (ASCETIC_OPT_SPARSE_EXCHANGE) with P emulated ranks on one GPU: per-run
time, exchange time (sum of the per-iteration ms_exchange spans), iterations that went sparse, and
a bit-exact check of sparse against dense. Dev tool: python tools/sparse_ab.py [scale] [P]."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen as gg                              # noqa: E402
import paper_conf_icpp_tangzwgzwy21_b200 as asc    # noqa: E402

scale = int(sys.argv[1]) if len(sys.argv) > 1 else 22
P = int(sys.argv[2]) if len(sys.argv) > 2 else 4
asc.set_device(0)
for algo in ["bfs", "sssp", "cc"]:
    g = gg.rmat(scale, seed=2, weights=(algo == "sssp"))
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    asc.unload()
    asc.emulate_ranks(P)
    asc.load_csr(g.off, g.nbr, pairs=g.pairs, symmetric=True)
    asc.set_budget(g.csr_bytes // (2 * P))
    res = {}
    for d in [0, 8, 0, 8]:
        asc.set_option("sparse_exchange", d)
        asc.run(algo, src, 0)
        st, its = asc.stats()
        xm = sum(i["ms_exchange"] for i in its)
        r = asc.get_result().copy()
        if d in res:
            assert np.array_equal(res[d], r)
        res[d] = r
        print(f"{algo} P={P} scale={scale} d={d}: run {st['time_run_s'] * 1e3:.2f} ms, exchange {xm:.2f} ms, "
              f"iters {st['iterations']}, sparse {st['sparse_exchanges']}, pair bytes {st['sparse_exchange_bytes']}",
              flush=True)
    assert np.array_equal(res[0], res[8]), algo
    asc.set_option("sparse_exchange", 0)
asc.unload()
asc.emulate_ranks(1)
print("sparse == dense: ok")
