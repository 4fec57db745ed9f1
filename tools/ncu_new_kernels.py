"""Driver for ncu captures of the round's new kernels on RMAT-22: §3.4 replacement
(k_chunk_access, k_copy_chunks, k_apply_swaps, k_static_rebits, static kernels with the slot
remap) on SSSP, and PageRank-delta (k_ondemand<4>, k_static_*<4>, k_finalize_prd)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import graphgen as gg  # noqa: E402


def main():
    import paper_conf_icpp_tangzwgzwy21_b200 as asc
    which = sys.argv[1] if len(sys.argv) > 1 else "all"
    if which in ("all", "replace"):
        g = gg.rmat(22, seed=2, weights=True)
        src = int(np.argmax(np.diff(g.off.astype(np.int64))))
        asc.load_csr(g.off, g.nbr, pairs=True)
        asc.set_option("replace_chunks", 1024)
        asc.set_budget(g.csr_bytes // 2)
        for _ in range(2):
            asc.run("sssp", src)
        st, _ = asc.stats(per_iter=False)
        print("replace", st["swaps_total"], st["h2d_replace_bytes"], st["time_run_s"])
        asc.set_option("replace_chunks", 0)
        asc.unload()
    if which == "resident":   # static-hit kernels alone (budget above the CSR), SSSP and CC
        for algo in ("sssp", "cc"):
            g = gg.rmat(23, seed=2, weights=(algo == "sssp"))
            src = int(np.argmax(np.diff(g.off.astype(np.int64))))
            asc.load_csr(g.off, g.nbr, pairs=g.pairs)
            asc.set_budget(int(g.csr_bytes * 1.2))
            for _ in range(2):
                asc.run(algo, src)
            st, _ = asc.stats(per_iter=False)
            print("resident", algo, st["time_static_s"], st["static_arcs"])
            asc.unload()
    if which in ("all", "prd"):
        g = gg.rmat(22, seed=3)
        asc.load_csr(g.off, g.nbr)
        asc.set_budget(g.csr_bytes // 2)
        for _ in range(2):
            asc.run("prd", 0)
        st, _ = asc.stats(per_iter=False)
        print("prd", st["iterations"], st["time_run_s"], st["gteps"])
        asc.unload()


if __name__ == "__main__":
    main()
