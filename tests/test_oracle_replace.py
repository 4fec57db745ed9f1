"""Pins for the oracle's §3.4 data replacement (oracle.c or_run_hot).

* a hand-worked example (tests/golden/replace_bfs_worked.txt),
* the special case K = 0, which must reduce to the already-pinned front-prefix run,
* the closed form for all-active PageRank with the last-iteration counter (no chunk is ever
  hotter than a resident one, so nothing moves),
* a vectorised restatement over scipy BFS level sets (np.add.at chunk counters, lexsort
  selection) for several chunks, K and graph seeds,
* results never depend on the replacement (it moves bytes, not values).
"""
import os

import numpy as np
import pytest
import scipy.sparse as sp
from scipy.sparse import csgraph

import graphgen as gg
import oracle
from tests import pins

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
CHUNK = 16384


def worked_graph():
    lists = [[1] * 4096, [2] * 4096, [3] * 1024, [4] * 512 + [5] * 512, [], [6] * 6144, [0] * 50]
    off = np.zeros(len(lists) + 1, dtype=np.uint64)
    off[1:] = np.cumsum([len(x) for x in lists])
    nbr = np.array([v for x in lists for v in x], dtype=np.uint32)
    return off, nbr


def test_replace_worked_example():
    off, nbr = worked_graph()
    rows = [list(map(int, ln.split())) for ln in open(os.path.join(GOLDEN, "replace_bfs_worked.txt"))
            if ln.strip() and not ln.startswith("#")]
    r = oracle.run_hot("bfs", off, nbr, static_bytes=32768, src=2, kswap=1)
    cols = ["t", "nA", "nH", "nM", "nruns", "active_arcs", "hit_arcs", "miss_bytes", "s", "swaps", "replace_bytes"]
    assert [[rec[c] for c in cols] for rec in r.records] == rows
    np.testing.assert_array_equal(r.values, [4, 5, 0, 1, 2, 2, 3])
    assert r.h2d_payload == 61640 and r.replace_bytes == 32768 and r.iterations == 6
    r0 = oracle.run_hot("bfs", off, nbr, static_bytes=32768, src=2, kswap=0)
    assert r0.h2d_payload == 32968 and r0.replace_bytes == 0


@pytest.mark.parametrize("algo", ["bfs", "sssp", "cc", "pr"])
def test_replace_k0_is_the_front_prefix_run(algo):
    g = gg.rmat(12, seed=5, weights=(algo == "sssp"))
    b_e = 8 if algo == "sssp" else 4
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    for frac in (0.0, 0.3, 0.77, 1.0):
        p = oracle.placer(g.off, b_e, g.csr_bytes // 2, frac=frac)
        iters = 6 if algo == "pr" else 0
        a = oracle.run(algo, g.off, g.nbr, src=src, max_iters=iters, is_static=oracle.static_prefix(g.n, p.s))
        b = oracle.run_hot(algo, g.off, g.nbr, static_bytes=p.Ms, src=src, max_iters=iters, kswap=0)
        assert a.records == b.records, frac           # includes s: chunk rule == front prefix
        np.testing.assert_array_equal(a.values, b.values)
        assert b.replace_bytes == 0


def test_replace_pr_last_iteration_counter_never_swaps():
    """All-active PR (A_t = V): every full chunk holds 16384/b_e accessed arcs each iteration, so
    with h = last iteration's accesses no non-resident chunk is hotter than a resident one."""
    g = gg.rmat(12, seed=6)
    p = oracle.placer(g.off, 4, g.csr_bytes // 3)
    assert 0 < p.Ms < 4 * g.m
    r = oracle.run_hot("pr", g.off, g.nbr, static_bytes=p.Ms, max_iters=5, kswap=64, policy="last")
    assert r.replace_bytes == 0 and all(x["swaps"] == 0 for x in r.records)
    # the cumulative counter sees the same equal counts: still no swap
    r2 = oracle.run_hot("pr", g.off, g.nbr, static_bytes=p.Ms, max_iters=5, kswap=64, policy="cumulative")
    assert r2.replace_bytes == 0


def restated_bfs_replacement(off, nbr, src, Ms, K, res0=None):
    """§3.4 restated with numpy over scipy's BFS level sets (independent of oracle.c's loops)."""
    n = off.size - 1
    A = sp.csr_matrix((np.ones(nbr.size), nbr.astype(np.int64), off.astype(np.int64)), shape=(n, n))
    lev = csgraph.shortest_path(A, directed=True, unweighted=True, indices=src)
    L = int(lev[np.isfinite(lev)].max())
    o = off.astype(np.int64)
    D = 4 * int(o[-1])
    NC = (D + CHUNK - 1) // CHUNK
    res = np.zeros(NC, dtype=bool)
    res[:(Ms + CHUNK - 1) // CHUNK] = True
    if res0 is not None:
        res = np.array(res0, dtype=bool)
    h = np.zeros(NC, dtype=np.int64)
    a_byte, e_byte = 4 * o[:-1], 4 * o[1:]
    deg = o[1:] - o[:-1]
    arc_chunk = (4 * np.arange(o[-1])) // CHUNK
    owner = np.repeat(np.arange(n), deg)

    def static_set():
        st = np.empty(n, dtype=bool)
        for v in range(n):
            if deg[v] == 0:
                st[v] = a_byte[v] == 0 or res[(a_byte[v] - 1) // CHUNK]
            else:
                st[v] = res[a_byte[v] // CHUNK:(e_byte[v] - 1) // CHUNK + 1].all()
        return st

    st = static_set()
    recs = []
    for t in range(L + 1):
        act = lev == t
        rec = pins.records_from_sets([act], off, 4, 0)[0]
        hit, miss = act & st, act & ~st
        rec.update(t=t, nH=int(hit.sum()), nM=int(miss.sum()), nruns=pins.runs_of(miss),
                   hit_arcs=int(deg[hit].sum()), miss_bytes=int(4 * deg[miss].sum()), s=int(st.sum()))
        np.add.at(h, arc_chunk[act[owner]], 1)
        ids = np.arange(NC)
        hot = ids[~res][np.lexsort((ids[~res], -h[~res]))][:K]
        cold = ids[res][np.lexsort((ids[res], h[res]))][:K]
        sw, by = 0, 0
        for hi_, co in zip(hot, cold):
            if not h[hi_] > h[co]:
                break
            res[hi_], res[co] = True, False
            sw += 1
            by += min(CHUNK, D - CHUNK * int(hi_))
        rec.update(swaps=sw, replace_bytes=by)
        if sw:
            st = static_set()
        recs.append(rec)
    return recs


@pytest.mark.parametrize("seed,K,frac", [(1, 1, 0.3), (2, 4, 0.5), (3, 16, 0.2), (4, 64, 0.6)])
def test_replace_bfs_vs_restatement(seed, K, frac):
    g = gg.rmat(12, seed=seed)
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    p = oracle.placer(g.off, 4, g.csr_bytes, frac=frac)
    got = oracle.run_hot("bfs", g.off, g.nbr, static_bytes=p.Ms, src=src, kswap=K)
    exp = restated_bfs_replacement(g.off, g.nbr, src, p.Ms, K)
    assert got.records == exp
    assert sum(r["swaps"] for r in got.records) > 0


@pytest.mark.parametrize("algo", ["bfs", "sssp", "cc"])
def test_replace_never_changes_results(algo):
    g = gg.rmat(12, seed=8, weights=(algo == "sssp"))
    b_e = 8 if algo == "sssp" else 4
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    p = oracle.placer(g.off, b_e, g.csr_bytes // 3)
    plain = oracle.run(algo, g.off, g.nbr, src=src, is_static=oracle.static_prefix(g.n, p.s))
    hot = oracle.run_hot(algo, g.off, g.nbr, static_bytes=p.Ms, src=src, kswap=32)
    np.testing.assert_array_equal(plain.values, hot.values)
    assert hot.replace_bytes > 0
    for r in hot.records:
        assert r["replace_bytes"] <= CHUNK * r["swaps"]
        assert r["miss_bytes"] + b_e * r["hit_arcs"] == b_e * r["active_arcs"]


def test_replace_multi_rank_k0_matches_front_and_splits():
    g = gg.rmat(12, seed=9)
    P = 3
    b = oracle.partition(g.off, P)
    ms, st = [], np.zeros(g.n, dtype=np.uint8)
    for k in range(P):
        lo, hi = int(b[k]), int(b[k + 1])
        sub = g.off[lo:hi + 1] - g.off[lo]
        p = oracle.placer(sub, 4, int(0.4 * 4 * int(sub[-1])))
        ms.append(p.Ms)
        st[lo:lo + p.s] = 1
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    front = oracle.run("bfs", g.off, g.nbr, src=src, is_static=st, bounds=b)
    k0 = oracle.run_hot("bfs", g.off, g.nbr, static_bytes=ms, src=src, kswap=0, bounds=b)
    assert front.records == k0.records
    k8 = oracle.run_hot("bfs", g.off, g.nbr, static_bytes=ms, src=src, kswap=8, bounds=b)
    np.testing.assert_array_equal(front.values, k8.values)
    assert [r["rank"] for r in k8.records[:P]] == list(range(P))


@pytest.mark.parametrize("nc,ns,seed", [(1, 1, 1), (10, 3, 1), (1000, 250, 7), (5000, 4999, 3), (64, 0, 2)])
def test_random_chunks_are_the_smallest_keys(nc, ns, seed):
    """§5 random initial content: the ns chunks with the smallest
    splitmix64((seed << 32) ^ c) keys (the digest's splitmix, pinned in tests/pins.py)."""
    res = oracle.random_chunks(nc, ns, seed)
    assert res.sum() == min(ns, nc)
    keys = np.array([pins.splitmix(((seed << 32) ^ c) & pins.M64) for c in range(nc)], dtype=object)
    if 0 < ns < nc:
        assert max(keys[res]) < min(keys[~res])


@pytest.mark.parametrize("seed,K", [(1, 0), (5, 0), (2, 8)])
def test_random_initial_content_vs_restatement(seed, K):
    g = gg.rmat(12, seed=12)
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    p = oracle.placer(g.off, 4, g.csr_bytes, frac=0.35)
    nc = (4 * g.m + CHUNK - 1) // CHUNK
    res0 = oracle.random_chunks(nc, (p.Ms + CHUNK - 1) // CHUNK, seed)
    got = oracle.run_hot("bfs", g.off, g.nbr, static_bytes=p.Ms, src=src, kswap=K, random_seed=seed)
    assert got.records == restated_bfs_replacement(g.off, g.nbr, src, p.Ms, K, res0=res0)
    front = oracle.run_hot("bfs", g.off, g.nbr, static_bytes=p.Ms, src=src, kswap=K)
    np.testing.assert_array_equal(got.values, front.values)
    assert got.records[0]["s"] != front.records[0]["s"]      # a different static set
