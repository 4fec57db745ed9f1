"""Pins for the oracle's PageRank-delta (algo "prd", oracle.c; Subway's
frontier-driven PR, Table 1). Readings R28-R30 in DESIGN.md:
fixed point Q = 2^56, d = 17/20, res_0 = floor(3Q/20n), tau = floor(res_0 * ppm / 1e6).

* tau = 0, T iterations: every vertex is active every round, so r + res is the truncated Jacobi
  power series sum_{k=0}^{T} (d A D^-1)^k b (dense fp64 matrix products), up to one quantum
  per arc and round of truncation;
* tau > 0: the result is a tau-approximate fixed point of x = b + d A D^-1 x (every absorbed
  residual was pushed; what is left is <= tau per vertex);
* degenerate graphs (no arcs, one vertex, dangling vertices).
"""
import numpy as np
import pytest

import graphgen as gg
import oracle

Q = 2.0 ** 56


def dense(g):
    n = g.n
    A = np.zeros((n, n))
    for u in range(n):
        for e in range(int(g.off[u]), int(g.off[u + 1])):
            A[int(g.nbr[e]), u] += 1.0
    deg = np.diff(g.off.astype(np.int64)).astype(np.float64)
    return A, deg


@pytest.fixture(autouse=True)
def _tol():
    yield
    oracle.set_prd_tol(10000)


@pytest.mark.parametrize("scale,T", [(6, 1), (7, 5), (8, 12)])
def test_prd_tau0_is_the_power_series(scale, T):
    g = gg.rmat(scale, seed=4)
    oracle.set_prd_tol(0)
    r = oracle.run("prd", g.off, g.nbr, max_iters=T)
    assert r.iterations == T
    A, deg = dense(g)
    M = 0.85 * A / np.where(deg > 0, deg, 1.0)[None, :]
    b = np.full(g.n, float((3 * (1 << 56)) // (20 * g.n))) / Q
    x, term = b.copy(), b.copy()
    for _ in range(T):
        term = M @ term
        x += term
    # truncation: at most one quantum per arc per round (floor of d res / deg), plus conversion
    bound = (T * g.m + g.n) / Q + 1e-15 * x
    assert np.all(np.abs(r.values - x) <= bound)
    assert np.all(r.values <= x + 1e-15 * x)          # truncation only ever removes mass
    assert r.records[0]["nA"] == g.n                   # tau = 0: every vertex with residual > 0 is active
    assert all(rec["nA"] >= int((M.sum(axis=1) > 0).sum()) for rec in r.records[1:])


@pytest.mark.parametrize("ppm", [1000, 10000, 300000])
def test_prd_tau_is_an_approximate_fixed_point(ppm):
    g = gg.rmat(9, seed=5)
    oracle.set_prd_tol(ppm)
    r = oracle.run("prd", g.off, g.nbr)
    A, deg = dense(g)
    res0 = (3 * (1 << 56)) // (20 * g.n)
    tau = (res0 * ppm // 1000000) / Q
    b = res0 / Q
    x = r.values
    # x = r + res with res <= tau; r was pushed: x - b - d A D^-1 (x - res) = -truncation
    lhs = x - b - 0.85 * (A @ (x / np.where(deg > 0, deg, 1.0) * (deg > 0)))
    slack = 0.85 * (A @ np.where(deg > 0, tau / np.where(deg > 0, deg, 1.0), 0.0))
    trunc = (r.iterations * (A.sum(axis=1) + 1)) / Q
    assert np.all(lhs <= 1e-13 * x)
    assert np.all(lhs >= -slack - trunc - 1e-13 * x)
    assert r.records[-1]["nA"] > 0 and r.iterations > 1
    # partial activity (Table 1: PR's active edges are a fraction of the graph per iteration)
    if ppm >= 300000:
        assert min(rec["active_arcs"] for rec in r.records) < g.m


def test_prd_degenerate():
    g = gg.from_edges(5, np.zeros(0, np.uint32), np.zeros(0, np.uint32))
    r = oracle.run("prd", g.off, g.nbr)
    res0 = (3 * (1 << 56)) // (20 * 5)
    assert r.iterations == 1
    np.testing.assert_array_equal(r.values, np.full(5, res0 / Q))
    one = gg.from_edges(1, np.zeros(0, np.uint32), np.zeros(0, np.uint32))
    r1 = oracle.run("prd", one.off, one.nbr)
    assert r1.iterations == 1 and r1.values[0] == ((3 << 56) // 20) / Q
