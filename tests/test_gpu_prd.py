"""GPU parity of PageRank-delta (ASCETIC_PRD, Subway's frontier-driven
PR). Integer fixed-point residuals make everything bit-exact against the
oracle: fp32 ranks, per-iteration active sets and bytes."""
import numpy as np
import pytest

import graphgen as gg
import oracle

pytestmark = pytest.mark.gpu

REC = ["nA", "nH", "nM", "nruns", "active_arcs", "hit_arcs", "miss_bytes", "digest", "swaps", "replace_bytes"]


@pytest.fixture()
def asc():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import paper_conf_icpp_tangzwgzwy21_b200 as m
    m.unload()
    yield m
    for k, v in [("prd_tol_ppm", 10000), ("xfer_mode", 0), ("chunk_cap", 0), ("replace_chunks", 0), ("hub_degree", 2048)]:
        m.set_option(k, v)
    oracle.set_prd_tol(10000)
    m.unload()
    m.emulate_ranks(1)


def _check(asc, g, ppm, its, st, res, max_iters=0, kswap=0, Ms=None):
    oracle.set_prd_tol(ppm)
    if kswap:
        ref = oracle.run_hot("prd", g.off, g.nbr, static_bytes=Ms, max_iters=max_iters, kswap=kswap)
    else:
        p_s = st["s"]
        ref = oracle.run("prd", g.off, g.nbr, max_iters=max_iters, is_static=oracle.static_prefix(g.n, p_s))
    np.testing.assert_array_equal(res, ref.values.astype(np.float32))
    assert st["iterations"] == ref.iterations
    assert len(its) == len(ref.records)
    for a, b in zip(its, ref.records):
        for f in REC:
            assert a[f] == b[f], (b["t"], f, a[f], b[f])
    assert st["h2d_payload_bytes"] == ref.h2d_payload


@pytest.mark.parametrize("ppm", [1000, 10000, 300000])
@pytest.mark.parametrize("frac", [-1.0, 0.0, 0.6])
@pytest.mark.parametrize("xfer", [1, 2])
def test_prd_parity(asc, ppm, frac, xfer):
    g = gg.rmat(13, seed=51)
    asc.load_csr(g.off, g.nbr)
    asc.set_option("prd_tol_ppm", ppm)
    asc.set_option("xfer_mode", xfer)
    asc.set_option("chunk_cap", 1 << 15)
    asc.set_budget(g.csr_bytes // 3, frac)
    asc.run("prd", 0)
    st, its = asc.stats()
    _check(asc, g, ppm, its, st, asc.get_result().copy())
    assert st["iterations"] > 3


def test_prd_hubs_directed_and_max_iters(asc):
    """Directed RMAT lists (no symmetry needed for push), hub pieces, a max_iters cut."""
    u = gg.rmat(14, seed=52)
    src = np.repeat(np.arange(u.n, dtype=np.uint32), np.diff(u.off.astype(np.int64)))
    keep = (src.astype(np.int64) * 7 + u.nbr) % 3 != 0                  # drop a third of the arcs: directed
    g = gg.from_edges(u.n, src[keep], u.nbr[keep], symmetrize=False)
    asc.load_csr(g.off, g.nbr, symmetric=False)
    asc.set_option("hub_degree", 64)
    asc.set_budget(g.csr_bytes // 2)
    for mi in (0, 3):
        asc.run("prd", 0, mi)
        st, its = asc.stats()
        _check(asc, g, 10000, its, st, asc.get_result().copy(), max_iters=mi)


def test_prd_with_replacement(asc):
    g = gg.rmat(14, seed=53)
    budget = g.csr_bytes // 3
    asc.load_csr(g.off, g.nbr)
    asc.set_option("prd_tol_ppm", 200000)
    asc.set_option("replace_chunks", 32)
    asc.set_budget(budget)
    asc.run("prd", 0)
    st, its = asc.stats()
    p = oracle.placer(g.off, 4, budget)
    _check(asc, g, 200000, its, st, asc.get_result().copy(), kswap=32, Ms=p.Ms)


@pytest.mark.parametrize("P", [2, 3, 4])
def test_prd_emulated_ranks(asc, P):
    """P ranks on one GPU: pushes into per-rank increment arrays, SUM exchange, dense finalize;
    per-rank records and the fp32 ranks bit-exact against the oracle's multi-rank simulation."""
    g = gg.rmat(13, seed=54)
    budget = g.csr_bytes // (3 * P)
    asc.emulate_ranks(P)
    asc.load_csr(g.off, g.nbr)
    asc.set_option("prd_tol_ppm", 50000)
    asc.set_budget(budget, 0.5)
    asc.run("prd", 0)
    st, its = asc.stats()
    b = oracle.partition(g.off, P)
    stat = np.zeros(g.n, dtype=np.uint8)
    for k in range(P):
        lo, hi = int(b[k]), int(b[k + 1])
        stat[lo:lo + oracle.placer(g.off[lo:hi + 1] - g.off[lo], 4, budget, 0.5).s] = 1
    oracle.set_prd_tol(50000)
    ref = oracle.run("prd", g.off, g.nbr, is_static=stat, bounds=b)
    np.testing.assert_array_equal(asc.get_result(), ref.values.astype(np.float32))
    assert [i["rank"] for i in its] == [r["rank"] for r in ref.records]
    for a, r in zip(its, ref.records):
        for f in REC:
            assert a[f] == r[f], (r["t"], r["rank"], f)


def test_prd_rmat20_parity(asc):
    """A larger PageRank-delta run (RMAT-20, 33 M arcs, many chunk windows and hub pieces)."""
    g = gg.rmat(20, seed=55)
    budget = g.csr_bytes // 2
    asc.load_csr(g.off, g.nbr)
    asc.set_budget(budget)
    asc.run("prd", 0)
    st, its = asc.stats()
    _check(asc, g, 10000, its, st, asc.get_result().copy())
