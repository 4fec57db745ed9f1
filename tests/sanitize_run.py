"""Small end-to-end runs of every algorithm for compute-sanitizer (memcheck / racecheck /
synccheck): tiny chunks (many chunk windows, lists split across chunks), hub splitting,
gather and DMA transfer modes, and 2 emulated ranks; §3.4 replacement, random initial content
and PageRank-delta. Checks results against the oracle."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))   # repo root

import numpy as np  # noqa: E402

import graphgen as gg  # noqa: E402
import oracle  # noqa: E402


def main():
    import paper_conf_icpp_tangzwgzwy21_b200 as asc
    bad = 0
    for world in (1, 2):
        asc.unload()
        asc.emulate_ranks(world)
        for algo in ["bfs", "sssp", "cc", "pr"]:
            g = gg.rmat(9, seed=5, weights=(algo == "sssp"))
            src = int(np.argmax(np.diff(g.off.astype(np.int64))))
            it = 4 if algo == "pr" else 0
            for xfer, cap, hub in [(1, 64, 32), (2, 0, 2048), (0, 1024, 64)]:
                asc.unload()
                asc.load_csr(g.off, g.nbr, pairs=g.pairs)
                asc.set_option("xfer_mode", xfer)
                asc.set_option("chunk_cap", cap)
                asc.set_option("hub_degree", hub)
                asc.set_budget(g.csr_bytes // (3 * world), 0.4)
                asc.run(algo, src, it)
                res = asc.get_result()
                bounds = oracle.partition(g.off, world)
                st = np.zeros(g.n, dtype=np.uint8)
                for k in range(world):
                    lo, hi = int(bounds[k]), int(bounds[k + 1])
                    p = oracle.placer(g.off[lo:hi + 1] - g.off[lo], g.b_e, g.csr_bytes // (3 * world), 0.4)
                    st[lo:lo + p.s] = 1
                ref = oracle.run(algo, g.off, g.nbr, src=src, max_iters=it, is_static=st)
                ok = (np.max(np.abs(res - ref.values) / ref.values) < 1e-5) if algo == "pr" else np.array_equal(res, ref.values)
                bad += 0 if ok else 1
                print(f"world={world} {algo} xfer={xfer} cap={cap} hub={hub}: {'ok' if ok else 'MISMATCH'}", flush=True)
    # §3.4 replacement, random initial content and PageRank-delta (one and two ranks)
    for world in (1, 2):
        asc.unload()
        asc.emulate_ranks(world)
        for algo, placement, K in [("bfs", 0, 8), ("sssp", 2, 8), ("cc", 2, 0), ("prd", 0, 4), ("prd", 2, 0)]:
            g = gg.rmat(12, seed=6, weights=(algo == "sssp"))
            src = int(np.argmax(np.diff(g.off.astype(np.int64))))
            asc.unload()
            asc.load_csr(g.off, g.nbr, pairs=g.pairs)
            asc.set_option("static_placement", placement)
            asc.set_option("replace_chunks", K)
            asc.set_option("chunk_cap", 4096)
            asc.set_option("hub_degree", 64)
            budget = g.csr_bytes // (3 * world)
            asc.set_budget(budget)
            asc.run(algo, src, 0)
            res = asc.get_result()
            bounds = oracle.partition(g.off, world)
            ms = [oracle.placer(g.off[int(bounds[k]):int(bounds[k + 1]) + 1] - g.off[int(bounds[k])], g.b_e, budget).Ms
                  for k in range(world)]
            ref = oracle.run_hot(algo, g.off, g.nbr, static_bytes=ms, src=src, kswap=K, bounds=bounds,
                                 random_seed=1 if placement == 2 else None)
            exp = ref.values.astype(np.float32) if algo == "prd" else ref.values
            ok = np.array_equal(res, exp)
            bad += 0 if ok else 1
            print(f"world={world} {algo} placement={placement} K={K}: {'ok' if ok else 'MISMATCH'}", flush=True)
    # round-2 paths: span-DMA windows (forced), copy-engine long runs beside the gather, the PR slice pull,
    # RED.MIN updates (default), one and two ranks
    for world in (1, 2):
        asc.unload()
        asc.emulate_ranks(world)
        for algo, opts in [("bfs", {"xfer_mode": 3, "span_density": 50}), ("sssp", {"xfer_mode": 3, "span_density": 0}),
                           ("cc", {"xfer_mode": 1, "ce_min_run": 512}), ("pr", {"xfer_mode": 1, "ce_min_run": 512}),
                           ("pr", {"pr_segment": 2048}), ("prd", {"xfer_mode": 3, "span_density": 85})]:
            g = gg.rmat(10, seed=7, weights=(algo == "sssp"))
            src = int(np.argmax(np.diff(g.off.astype(np.int64))))
            it = 4 if algo == "pr" else 0
            asc.unload()
            asc.load_csr(g.off, g.nbr, pairs=g.pairs, sorted_rows=True)
            asc.set_option("chunk_cap", 2048)
            asc.set_option("hub_degree", 64)
            for k, v in opts.items():
                asc.set_option(k, v)
            budget = (20 * g.csr_bytes) if "pr_segment" in opts else g.csr_bytes // (3 * world)
            asc.set_budget(budget, 0.4)
            asc.run(algo, src, it)
            res = asc.get_result()
            bounds = oracle.partition(g.off, world)
            st = np.zeros(g.n, dtype=np.uint8)
            for k in range(world):
                lo, hi = int(bounds[k]), int(bounds[k + 1])
                p = oracle.placer(g.off[lo:hi + 1] - g.off[lo], g.b_e, budget, 0.4)
                st[lo:lo + p.s] = 1
            ref = oracle.run(algo, g.off, g.nbr, src=src, max_iters=it, is_static=st)
            if algo == "pr":
                ok = np.max(np.abs(res - ref.values) / ref.values) < 1e-5
            else:
                ok = np.array_equal(res, ref.values.astype(np.float32) if algo == "prd" else ref.values)
            bad += 0 if ok else 1
            print(f"world={world} {algo} {opts}: {'ok' if ok else 'MISMATCH'}", flush=True)
            for k, v in [("xfer_mode", 0), ("span_density", 85), ("ce_min_run", 1 << 20), ("pr_segment", 128 << 20)]:
                asc.set_option(k, v)
    for k, v in [("static_placement", 0), ("replace_chunks", 0), ("chunk_cap", 0), ("hub_degree", 2048)]:
        asc.set_option(k, v)
    asc.unload()
    asc.emulate_ranks(1)
    print("mismatches:", bad)
    sys.exit(1 if bad else 0)


if __name__ == "__main__":
    main()
