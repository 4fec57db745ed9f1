"""Parity at BASELINE.json's full sizes, in the configuration bench.py times.

C2 (SSSP, RMAT-24, 50 % budget): the oracle finishes a whole run in ~1.5 s on the box's
cores, so values AND every per-iteration record are compared in full.
C3 (PR, friendster-shaped, 11 GB): two full PR iterations compared vertex by vertex against
the fp64 oracle; the 43-iteration run is checked through properties that hold at any size
(mass = 1, A_t = V, closed-form miss bytes b_e (m - off[s]) every iteration, one run).
"""
import numpy as np
import pytest

import graphgen as gg
import oracle

pytestmark = pytest.mark.gpu

REC = ["nA", "nH", "nM", "nruns", "active_arcs", "hit_arcs", "miss_bytes", "digest"]


@pytest.fixture(scope="module")
def asc():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import paper_conf_icpp_tangzwgzwy21_b200 as m
    yield m
    m.unload()


def test_c2_full_parity(asc):
    g = gg.config_graph("c2")
    budget = gg.config_budget("c2", g)
    asc.load_csr(g.off, g.nbr, pairs=True)
    asc.set_budget(budget)
    p = oracle.placer(g.off, 8, budget)
    st_static = oracle.static_prefix(g.n, p.s)
    for src in gg.sources(g, 8, seed=2)[:2]:          # the first bench sources
        asc.run("sssp", src)
        st, its = asc.stats()
        res = asc.get_result()
        ref = oracle.run("sssp", g.off, g.nbr, src=src, is_static=st_static)
        np.testing.assert_array_equal(res, ref.values)
        assert st["iterations"] == ref.iterations
        assert [{f: i[f] for f in REC} for i in its] == [{f: r[f] for f in REC} for r in ref.records]
        assert st["h2d_payload_bytes"] == ref.h2d_payload
        assert st["h2d_static_fill_bytes"] == p.static_bytes
        assert st["s"] == p.s


def test_c3_full_pr(asc):
    g = gg.config_graph("c3")
    budget = gg.config_budget("c3", g)
    asc.load_csr(g.off, g.nbr)
    asc.set_budget(budget)
    p = oracle.placer(g.off, 4, budget)
    # two full iterations, every vertex
    asc.run("pr", 0, 2)
    res = asc.get_result().astype(np.float64)
    ref = oracle.run("pr", g.off, g.nbr, max_iters=2, is_static=oracle.static_prefix(g.n, p.s))
    rel = np.abs(res - ref.values) / ref.values
    assert rel.max() <= 1e-5, rel.max()
    assert np.abs(res - ref.values).sum() <= 1e-6
    st, its = asc.stats()
    assert [{f: i[f] for f in REC} for i in its] == [{f: r[f] for f in REC} for r in ref.records]
    # the configured 43 iterations: properties that hold at any size
    asc.run("pr", 0, 43)
    st, its = asc.stats()
    r43 = asc.get_result().astype(np.float64)
    assert st["iterations"] == 43 and len(its) == 43
    assert abs(r43.sum() - 1.0) < 1e-4
    assert (r43 > 0).all()
    for i in its:
        assert i["nA"] == g.n and i["nruns"] == (1 if p.s < g.n else 0)
        assert i["miss_bytes"] == 4 * (g.m - int(g.off[p.s]))
        assert i["active_arcs"] == g.m
    assert st["h2d_payload_bytes"] == 43 * 4 * (g.m - int(g.off[p.s]))


_C2 = {}


def _c2():
    if "g" not in _C2:
        _C2["g"] = gg.config_graph("c2")
    return _C2["g"]


@pytest.mark.parametrize("placement,K", [(0, 256), (2, 0)])
def test_c2_full_replacement_and_random_fill(asc, placement, K):
    """§3.4 replacement (K = 256 swaps per iteration) and the random initial chunks at the bench
    size: values, every record (incl. swaps, swap bytes, |S|) and all bytes bit-exact."""
    g = _c2()
    budget = gg.config_budget("c2", g)
    asc.load_csr(g.off, g.nbr, pairs=True)
    asc.set_option("static_placement", placement)
    asc.set_option("replace_chunks", K)
    try:
        asc.set_budget(budget)
        src = gg.sources(g, 8, seed=2)[0]
        asc.run("sssp", src)
        st, its = asc.stats()
        res = asc.get_result()
    finally:
        asc.set_option("static_placement", 0)
        asc.set_option("replace_chunks", 0)
    p = oracle.placer(g.off, 8, budget)
    ref = oracle.run_hot("sssp", g.off, g.nbr, static_bytes=p.Ms, src=src, kswap=K,
                         random_seed=1 if placement == 2 else None)
    np.testing.assert_array_equal(res, ref.values)
    f = REC + ["swaps", "replace_bytes"]
    assert [{k: i[k] for k in f} for i in its] == [{k: r[k] for k in f} for r in ref.records]
    assert [i["s_static"] for i in its] == [r["s"] for r in ref.records]
    assert st["h2d_payload_bytes"] == ref.h2d_payload and st["h2d_replace_bytes"] == ref.replace_bytes
