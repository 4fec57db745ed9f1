"""Pins for the CPU oracle (oracle/oracle.c) against things other than itself.

Every pin restates a definition independently (tests/pins.py, scipy, closed forms,
hand values in tests/golden/) so a plausible mistake in the oracle fails one of them.
"""
import itertools
import os

import numpy as np
import pytest
import scipy.sparse as sp
from scipy.sparse import csgraph

import graphgen as gg
import oracle
from tests import pins

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


# ------------------------------------------------------------------ placer (Eq. 1 / Eq. 2)
def _golden_eq2():
    rows = []
    for line in open(os.path.join(GOLDEN, "eq2_hand_values.txt")):
        line = line.strip()
        if not line or line.startswith("#"):
            continue
        d, m, r = line.split()[:3]
        rows.append((float(d), float(m), float(r)))
    return rows


@pytest.mark.parametrize("D,M,R", _golden_eq2())
def test_placer_eq2_hand_values(D, M, R):
    """Eq. 2 with K = 0.1 against hand-computed values."""
    U = 16384 * 1000
    m = int(round(D * U / 4))
    B = int(round(M * U))
    off = np.array([0, m], dtype=np.uint64)
    p = oracle.placer(off, 4, B)
    assert p.R == pytest.approx(R, abs=1e-9)
    # Ms = R*B floored to 16 KiB, never above D
    assert p.Ms % 16384 == 0
    assert p.Ms <= p.D
    assert p.R * B - 16384 < p.Ms <= max(p.R * B, 0) + 1e-6 or p.Ms == p.D
    # Eq. 1: (D - Ms) K + Ms <= M, with equality up to the 16 KiB floor when R in (0,1)
    lhs = (p.D - p.Ms) * 0.1 + p.Ms
    if 0 < R < 1:
        assert lhs <= B + 1e-6
        assert B - lhs < 16384
    assert p.C == B - p.Ms
    assert p.cap == (p.C // 2) // 16 * 16


def test_placer_prefix_and_frac():
    g = gg.rmat(12, seed=7)
    for budget in [0, 1000, 50_000, g.csr_bytes // 4, g.csr_bytes, 10 * g.csr_bytes]:
        for frac in [-1.0, 0.0, 0.3, 1.0]:
            p = oracle.placer(g.off, 4, budget, frac)
            # s = max{v : b_e off[v] <= Ms}, by searchsorted on the byte offsets
            s = int(np.searchsorted(4 * g.off.astype(np.int64), p.Ms, side="right")) - 1
            assert p.s == s
            assert p.static_bytes == 4 * int(g.off[s]) <= p.Ms
            if frac >= 0:
                assert p.R == frac
            if budget >= 4 * g.m and frac < 0:
                assert p.R == 1.0
    # R = 1 with B >= D: whole graph static
    p = oracle.placer(g.off, 4, 4 * g.m + 16384, -1.0)
    assert p.s == g.n


def test_placer_nan_and_negative_clamp():
    off = np.array([0, 1000], dtype=np.uint64)
    p = oracle.placer(off, 4, 10, -1.0)   # K D >> M => R < 0 -> 0
    assert p.R == 0.0 and p.Ms == 0 and p.s == 0


def test_rear_start_is_smallest_fitting_suffix():
    g = gg.rmat(11, seed=9)
    o = g.off.astype(np.int64)
    for Ms in [0, 100, 16384, 4 * g.m // 3, 4 * g.m, 10 * g.m]:
        s_lo = oracle.rear_start(g.off, 4, Ms)
        assert 4 * (o[-1] - o[s_lo]) <= Ms
        assert s_lo == 0 or 4 * (o[-1] - o[s_lo - 1]) > Ms


def test_partition_edge_balanced():
    g = gg.rmat(12, seed=3)
    for P in [1, 2, 3, 4, 8]:
        b = oracle.partition(g.off, P)
        assert b[0] == 0 and b[P] == g.n
        offs = g.off.astype(np.int64)
        for k in range(1, P):
            target = -(-(k * g.m) // P)
            assert b[k] == int(np.searchsorted(offs, target, side="left"))
        assert np.all(np.diff(b.astype(np.int64)) >= 0)


# ------------------------------------------------------------------ digest
def test_digest_matches_python_ints():
    rng = np.random.default_rng(0)
    for n in [0, 1, 31, 32, 33, 100, 1000]:
        a = rng.random(n) < 0.3
        assert oracle.digest(a) == pins.digest(a)
    # sensitivity: one bit changes the digest
    a = np.zeros(77, dtype=bool)
    b = a.copy(); b[76] = True
    assert oracle.digest(a) != oracle.digest(b)


# ------------------------------------------------------------------ BFS
def _all_graphs(n):
    pairs = list(itertools.combinations(range(n), 2))
    for mask in range(1 << len(pairs)):
        e = [pairs[i] for i in range(len(pairs)) if mask >> i & 1]
        yield e


@pytest.mark.parametrize("n", [1, 2, 3, 4, 5])
def test_bfs_exhaustive_tiny(n):
    """Every undirected simple graph on n <= 5 vertices x every source vs textbook queue BFS."""
    for e in _all_graphs(n):
        src = np.array([a for a, b in e], dtype=np.uint32)
        dst = np.array([b for a, b in e], dtype=np.uint32)
        g = gg.from_edges(n, src, dst)
        adj = pins.adjacency(g.off, g.nbr)
        for s in range(n):
            r = oracle.run("bfs", g.off, g.nbr, src=s)
            np.testing.assert_array_equal(r.values, pins.bfs_queue(adj, s))
            levels = r.values
            reached = levels != pins.INF
            assert r.iterations == (int(levels[reached].max()) + 1 if reached.any() else 0)


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_bfs_vs_scipy_and_records(seed):
    g = gg.random_graph(600, 900, seed) if seed < 3 else gg.rmat(10, seed=seed)
    deg = np.diff(g.off.astype(np.int64))
    src = int(np.argmax(deg))
    A = sp.csr_matrix((np.ones(g.m), g.nbr.astype(np.int64), g.off.astype(np.int64)), shape=(g.n, g.n))
    dist = csgraph.shortest_path(A, unweighted=True, indices=src)
    s_static = g.n // 3
    r = oracle.run("bfs", g.off, g.nbr, src=src, is_static=oracle.static_prefix(g.n, s_static))
    exp = np.where(np.isinf(dist), pins.INF, dist).astype(np.uint32)
    np.testing.assert_array_equal(r.values, exp)
    # records: A_t = {v : level(v) = t}
    L = int(exp[exp != pins.INF].max())
    sets = [exp == t for t in range(L + 1)]
    assert r.records == pins.records_from_sets(sets, g.off, 4, s_static)
    # closed form: total miss bytes = 4 * sum of degrees of reached non-static vertices
    reached = exp != pins.INF
    ns = np.arange(g.n) >= s_static
    assert r.h2d_payload == 4 * int(deg[reached & ns].sum())


def test_bfs_invariants_rmat():
    g = gg.rmat(13, seed=11)
    deg = np.diff(g.off.astype(np.int64))
    src = int(np.argmax(deg))
    r = oracle.run("bfs", g.off, g.nbr, src=src)
    lev = r.values.astype(np.int64)
    u = np.repeat(np.arange(g.n), deg)
    v = g.nbr.astype(np.int64)
    both = (lev[u] != pins.INF) & (lev[v] != pins.INF)
    assert np.all(np.abs(lev[u][both] - lev[v][both]) <= 1)
    # reached <=> same component as src
    A = sp.csr_matrix((np.ones(g.m), v, g.off.astype(np.int64)), shape=(g.n, g.n))
    _, lab = csgraph.connected_components(A, directed=False)
    np.testing.assert_array_equal(lev != pins.INF, lab == lab[src])
    # every reached v != src has a neighbour at level - 1
    has_parent = np.zeros(g.n, dtype=bool)
    ok = both & (lev[u] == lev[v] - 1)
    has_parent[v[ok]] = True
    reached = lev != pins.INF
    reached[src] = False
    assert np.all(has_parent[reached])


def test_bfs_max_iters():
    g = gg.rmat(10, seed=5)
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    full = oracle.run("bfs", g.off, g.nbr, src=src)
    part = oracle.run("bfs", g.off, g.nbr, src=src, max_iters=2)
    assert part.iterations == 2
    assert part.records == full.records[:2]
    np.testing.assert_array_equal(part.values, np.where(full.values <= 2, full.values, pins.INF))


# ------------------------------------------------------------------ SSSP
def _weighted_edges(g):
    ids, w = g.ids(), g.weights()
    deg = np.diff(g.off.astype(np.int64))
    u = np.repeat(np.arange(g.n), deg)
    return list(zip(u.tolist(), ids.tolist(), w.tolist()))


@pytest.mark.parametrize("n", [2, 3, 4])
def test_sssp_exhaustive_tiny_vs_matrix_bellman_ford(n):
    """All graphs on n <= 4 vertices with seeded weights; values AND Jacobi active sets."""
    for k, e in enumerate(_all_graphs(n)):
        src = np.array([a for a, b in e], dtype=np.uint32)
        dst = np.array([b for a, b in e], dtype=np.uint32)
        g = gg.from_edges(n, src, dst, weights=True, seed=k + 1)
        ew = _weighted_edges(g)
        for s in range(n):
            r = oracle.run("sssp", g.off, g.nbr, src=s, is_static=oracle.static_prefix(n, n // 2))
            init = [pins.INF] * n
            init[s] = 0
            x, sets = pins.bf_dense(n, ew, init)
            np.testing.assert_array_equal(r.values, x)
            A0 = np.zeros(n, dtype=bool); A0[s] = True
            seq = [A0] + [c for c in sets if c.any()]
            assert r.records == pins.records_from_sets(seq, g.off, 8, n // 2)


@pytest.mark.parametrize("seed", [1, 2])
def test_sssp_vs_dijkstra(seed):
    g = gg.random_graph(500, 1500, seed, weights=True) if seed == 1 else gg.rmat(10, seed=seed, weights=True)
    ids, w = g.ids().astype(np.int64), g.weights().astype(np.float64)
    A = sp.csr_matrix((w, ids, g.off.astype(np.int64)), shape=(g.n, g.n))
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    d = csgraph.dijkstra(A, indices=src)
    r = oracle.run("sssp", g.off, g.nbr, src=src)
    exp = np.where(np.isinf(d), pins.INF, d).astype(np.uint32)
    np.testing.assert_array_equal(r.values, exp)
    assert g.weights().min() >= 1 and g.weights().max() <= 64


def test_sssp_records_vs_matrix_form():
    g = gg.random_graph(60, 150, 9, weights=True)
    ew = _weighted_edges(g)
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    init = [pins.INF] * g.n
    init[src] = 0
    x, sets = pins.bf_dense(g.n, ew, init)
    A0 = np.zeros(g.n, dtype=bool); A0[src] = True
    r = oracle.run("sssp", g.off, g.nbr, src=src, is_static=oracle.static_prefix(g.n, 25))
    np.testing.assert_array_equal(r.values, x)
    assert r.records == pins.records_from_sets([A0] + [c for c in sets if c.any()], g.off, 8, 25)


def test_sssp_invariants_rmat():
    g = gg.rmat(12, seed=13, weights=True)
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    r = oracle.run("sssp", g.off, g.nbr, src=src)
    dist = r.values.astype(np.int64)
    deg = np.diff(g.off.astype(np.int64))
    u = np.repeat(np.arange(g.n), deg)
    v, w = g.ids().astype(np.int64), g.weights().astype(np.int64)
    reach = dist[u] != pins.INF
    assert np.all(dist[v][reach] <= dist[u][reach] + w[reach])          # triangle inequality
    tight = np.zeros(g.n, dtype=bool)
    t = reach & (dist[v] == dist[u] + w)
    tight[v[t]] = True
    rv = dist != pins.INF
    rv[src] = False
    assert np.all(tight[rv])                                            # every reached v has a tight in-arc


# ------------------------------------------------------------------ CC
@pytest.mark.parametrize("n", [1, 2, 3, 4, 5])
def test_cc_exhaustive_tiny(n):
    for e in _all_graphs(n):
        src = np.array([a for a, b in e], dtype=np.uint32)
        dst = np.array([b for a, b in e], dtype=np.uint32)
        g = gg.from_edges(n, src, dst)
        # union-find min-ID labels
        parent = list(range(n))

        def find(x):
            while parent[x] != x:
                x = parent[x]
            return x
        for a, b in e:
            ra, rb = find(a), find(b)
            if ra != rb:
                parent[max(ra, rb)] = min(ra, rb)
        exp = np.array([find(v) for v in range(n)], dtype=np.uint32)
        r = oracle.run("cc", g.off, g.nbr)
        np.testing.assert_array_equal(r.values, exp)


@pytest.mark.parametrize("seed", [1, 2])
def test_cc_vs_scipy_and_records(seed):
    g = gg.random_graph(300, 280, seed) if seed == 1 else gg.rmat(11, seed=seed)
    A = sp.csr_matrix((np.ones(g.m), g.nbr.astype(np.int64), g.off.astype(np.int64)), shape=(g.n, g.n))
    ncomp, lab = csgraph.connected_components(A, directed=False)
    minid = np.full(ncomp, g.n)
    np.minimum.at(minid, lab, np.arange(g.n))
    exp = minid[lab].astype(np.uint32)
    r = oracle.run("cc", g.off, g.nbr, is_static=oracle.static_prefix(g.n, g.n // 2))
    np.testing.assert_array_equal(r.values, exp)
    # invariants: label constant on edges, label[v] <= v, idempotent
    deg = np.diff(g.off.astype(np.int64))
    u = np.repeat(np.arange(g.n), deg)
    assert np.all(r.values[u] == r.values[g.nbr])
    assert np.all(r.values <= np.arange(g.n))
    assert np.all(r.values[r.values] == r.values)
    if g.n <= 400:
        edges = [(int(a), int(b), 0) for a, b in zip(u, g.nbr)]
        x, sets = pins.bf_dense(g.n, edges, list(range(g.n)))
        seq = [np.ones(g.n, dtype=bool)] + [c for c in sets if c.any()]
        assert r.records == pins.records_from_sets(seq, g.off, 4, g.n // 2)


# ------------------------------------------------------------------ PageRank
@pytest.mark.parametrize("seed", [1, 2, 3])
def test_pr_vs_dense_matrix(seed):
    g = gg.random_graph(400, 1200, seed) if seed < 3 else gg.rmat(9, seed=seed)
    iters = 20
    r = oracle.run("pr", g.off, g.nbr, max_iters=iters, is_static=oracle.static_prefix(g.n, g.n // 3))
    exp = pins.pr_dense(g.off, g.nbr, iters)
    np.testing.assert_allclose(r.values, exp, rtol=1e-12, atol=0)
    assert abs(r.values.sum() - 1.0) < 1e-12                    # mass conserved
    assert r.iterations == iters
    # A_t = V every iteration; closed-form miss bytes b_e (m - off[s])
    s = g.n // 3
    for rec in r.records:
        assert rec["nA"] == g.n and rec["miss_bytes"] == 4 * (g.m - int(g.off[s]))
        assert rec["nruns"] == (1 if s < g.n else 0)


def test_pr_regular_graph_closed_form():
    n = 64
    src = np.arange(n, dtype=np.uint32)
    dst = ((np.arange(n) + 1) % n).astype(np.uint32)   # cycle: 2-regular
    g = gg.from_edges(n, src, dst)
    r = oracle.run("pr", g.off, g.nbr, max_iters=43)
    np.testing.assert_allclose(r.values, np.full(n, 1.0 / n), rtol=1e-14)


def test_pr_converges_toward_linear_solve():
    g = gg.rmat(9, seed=4)
    n = g.n
    r = oracle.run("pr", g.off, g.nbr, max_iters=43)
    # stationary vector from a linear solve of r = (1-d)/n + d (P r), with dangling mass spread uniformly
    deg = np.diff(g.off.astype(np.int64)).astype(np.float64)
    M = np.zeros((n, n))
    for u in range(n):
        for e in range(int(g.off[u]), int(g.off[u + 1])):
            M[int(g.nbr[e]), u] += 1.0 / deg[u]
    M[:, deg == 0] = 1.0 / n
    d = 0.85
    rstar = np.linalg.solve(np.eye(n) - d * M, np.full(n, (1 - d) / n))
    assert np.abs(r.values - rstar).sum() <= 2 * 0.85 ** 43


def test_pr_requires_iters():
    g = gg.rmat(6, seed=1)
    with pytest.raises(ValueError):
        oracle.run("pr", g.off, g.nbr, max_iters=0)


# ------------------------------------------------------------------ multi-rank simulation
@pytest.mark.parametrize("algo", ["bfs", "cc", "sssp"])
def test_multi_rank_records_split_global(algo):
    g = gg.rmat(11, seed=21, weights=(algo == "sssp"))
    P = 4
    b = oracle.partition(g.off, P)
    ids = g.ids()
    b_e = 8 if algo == "sssp" else 4
    # per-rank placer on the rebased rows, union of per-rank prefixes
    st = np.zeros(g.n, dtype=np.uint8)
    for k in range(P):
        lo, hi = int(b[k]), int(b[k + 1])
        sub = g.off[lo:hi + 1] - g.off[lo]
        p = oracle.placer(sub, b_e, budget=int(0.3 * b_e * int(sub[-1])))
        st[lo:lo + p.s] = 1
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    one = oracle.run(algo, g.off, g.nbr, src=src, is_static=st)
    multi = oracle.run(algo, g.off, g.nbr, src=src, is_static=st, bounds=b)
    np.testing.assert_array_equal(one.values, multi.values)      # results partition-independent
    assert one.h2d_payload == multi.h2d_payload
    for t, rec in enumerate(one.records):
        parts = multi.records[t * P:(t + 1) * P]
        assert [p["rank"] for p in parts] == list(range(P))
        for f in ["nH", "nM", "active_arcs", "hit_arcs", "miss_bytes"]:
            assert sum(p[f] for p in parts) == rec[f]
        assert all(p["digest"] == rec["digest"] and p["nA"] == rec["nA"] for p in parts)
        assert sum(p["nruns"] for p in parts) >= rec["nruns"]
    del ids


def test_oracle_zero_budget_r0_moves_every_reached_list_once():
    """R = 0 (Subway-like): BFS moves every reached list exactly once (Table 5)."""
    g = gg.rmat(12, seed=2)
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    r = oracle.run("bfs", g.off, g.nbr, src=src, is_static=np.zeros(g.n, dtype=np.uint8))
    deg = np.diff(g.off.astype(np.int64))
    assert r.h2d_payload == 4 * int(deg[r.values != pins.INF].sum())
    r1 = oracle.run("bfs", g.off, g.nbr, src=src, is_static=np.ones(g.n, dtype=np.uint8))
    assert r1.h2d_payload == 0


def two_communities(half=600, seed=3):
    """Two random communities [0, half) and [half, 2 half) joined by one bridge: a BFS from the
    second one keeps its early frontiers out of the static front prefix (Eq. 3 fires)."""
    rng = np.random.default_rng(seed)
    a = rng.integers(0, half, (4 * half, 2))
    b = rng.integers(half, 2 * half, (4 * half, 2))
    e = np.concatenate([a, b, [[half - 1, half]]]).astype(np.uint32)
    return gg.from_edges(2 * half, e[:, 0], e[:, 1])


def test_eq3_repartition_vs_restatement():
    """Eq. 3 restated over scipy BFS level sets: when V_ondemand > C and
    V_static/M_static < 0.5 V/D, M_static -= M_static V/D (16 KiB floor), prefix recomputed."""
    g = two_communities()
    deg = np.diff(g.off.astype(np.int64))
    A = sp.csr_matrix((np.ones(g.m), g.nbr.astype(np.int64), g.off.astype(np.int64)), shape=(g.n, g.n))
    src = 900
    lev = csgraph.shortest_path(A, unweighted=True, indices=src)
    L = int(lev[np.isfinite(lev)].max())
    budget = g.csr_bytes // 2
    p = oracle.placer(g.off, 4, budget)
    D = 4.0 * g.m
    Ms, s = p.Ms, p.s
    recs = []
    for t in range(L + 1):
        act = lev == t
        V, Vs, Vo = 4.0 * deg[act].sum(), 4.0 * deg[act & (np.arange(g.n) < s)].sum(), 4.0 * deg[act & (np.arange(g.n) >= s)].sum()
        if Ms > 0 and Vo > budget - Ms and Vs / Ms < 0.5 * V / D:
            new = (Ms - min(int(np.floor(Ms * V / D)), Ms)) // 16384 * 16384
            if new < Ms:
                Ms = new
                s = int(np.searchsorted(4 * g.off.astype(np.int64), Ms, side="right")) - 1
        recs.append(pins.records_from_sets([act], g.off, 4, s)[0] | {"t": t})
    got = oracle.run("bfs", g.off, g.nbr, src=src, is_static=oracle.static_prefix(g.n, p.s),
                     eq3_budget=budget, eq3_ms=p.Ms)
    assert got.repartitions >= 1
    assert got.records == recs
    plain = oracle.run("bfs", g.off, g.nbr, src=src, is_static=oracle.static_prefix(g.n, p.s))
    np.testing.assert_array_equal(got.values, plain.values)        # Eq. 3 moves bytes, never results
    assert got.h2d_payload != plain.h2d_payload


@pytest.mark.parametrize("n,p_active,p_static", [(1, 1.0, 0.0), (37, 0.5, 0.3), (1000, 0.3, 0.5), (5000, 0.9, 0.1),
                                                 (64, 1.0, 1.0), (64, 0.0, 0.5)])
def test_classify_vs_vectorized(n, p_active, p_static):
    """or_classify (plain loop) vs a vectorised numpy construction of the same sets/runs/offsets."""
    rng = np.random.default_rng(n)
    deg = rng.integers(0, 9, n)
    off = np.concatenate([[0], np.cumsum(deg)]).astype(np.uint64)
    a = rng.random(n) < p_active
    s = rng.random(n) < p_static
    for b_e in (4, 8):
        c = oracle.classify(off, b_e, a, s)
        np.testing.assert_array_equal(c["hits"], np.nonzero(a & s)[0])
        miss = a & ~s
        np.testing.assert_array_equal(c["misses"], np.nonzero(miss)[0])
        edges = np.diff(np.concatenate([[0], miss.astype(np.int8), [0]]))
        np.testing.assert_array_equal(c["run_b"], np.nonzero(edges == 1)[0])
        np.testing.assert_array_equal(c["run_e"], np.nonzero(edges == -1)[0])
        mbytes = np.where(miss, deg * b_e, 0)
        cum = np.concatenate([[0], np.cumsum(mbytes)])
        np.testing.assert_array_equal(c["run_dst"], cum[c["run_b"]])
