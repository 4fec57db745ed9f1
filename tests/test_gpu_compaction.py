"""Kernel-level parity of GenDataMap + compaction: the classify kernel's
hit queues, miss queue + 64-bit arc prefix + list starts, maximal miss runs + byte offsets and
totals, bit-exact against oracle.classify on given active sets — random densities, ragged n,
many 8192-vertex tiles (decoupled look-back across tiles), runs spanning tiles, and the
degenerate cases (empty frontier, all active, all static, no static, alternating bits)."""
import numpy as np
import pytest

import graphgen as gg
import oracle

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def asc():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import paper_conf_icpp_tangzwgzwy21_b200 as m
    m.unload()
    yield m
    m.unload()


def _check(asc, g, active, s_static, hub=2048):
    b_e = g.b_e
    got = asc.debug_classify(active)
    stat = oracle.static_prefix(g.n, s_static).astype(bool)
    ref = oracle.classify(g.off, b_e, active, stat)
    deg = np.diff(g.off.astype(np.int64))
    hits = ref["hits"][deg[ref["hits"]] > 0]
    dh = deg[hits]
    np.testing.assert_array_equal(got["hit_small"], hits[dh < 32])
    np.testing.assert_array_equal(got["hit_med"], hits[(dh >= 32) & (dh < hub)])
    np.testing.assert_array_equal(got["hit_hub"], hits[dh >= hub])
    pieces = (dh[dh >= hub] + 4095) // 4096
    np.testing.assert_array_equal(got["hub_pre"], np.concatenate([[0], np.cumsum(pieces)[:-1]]).astype(np.uint32)
                                  if pieces.size else np.zeros(0, np.uint32))
    assert got["n_pieces"] == int(pieces.sum())
    mq = ref["misses"][deg[ref["misses"]] > 0]
    np.testing.assert_array_equal(got["missq"], mq)
    pre = np.concatenate([[0], np.cumsum(deg[mq])[:-1]]) if mq.size else np.zeros(0)
    np.testing.assert_array_equal(got["missq_pre"], pre.astype(np.uint64))
    np.testing.assert_array_equal(got["missq_src"], g.off[mq])
    np.testing.assert_array_equal(got["run_b"], ref["run_b"])
    np.testing.assert_array_equal(got["run_e"], ref["run_e"])
    np.testing.assert_array_equal(got["run_dst"].astype(np.uint64) * b_e, ref["run_dst"])
    assert got["miss_arcs"] * b_e == int(b_e * deg[ref["misses"]].sum())
    assert got["nA"] == int(active.sum()) and got["nH"] == ref["hits"].size and got["nM"] == ref["misses"].size
    assert got["active_arcs"] == int(deg[active].sum()) and got["hit_arcs"] == int(deg[ref["hits"]].sum())
    assert got["digest"] == oracle.digest(active)


@pytest.mark.parametrize("scale", [10, 14, 17])
def test_compaction_random_frontiers(asc, scale):
    g = gg.rmat(scale, seed=scale)
    asc.load_csr(g.off, g.nbr)
    asc.set_budget(g.csr_bytes // 3, 0.45)
    s = oracle.placer(g.off, 4, g.csr_bytes // 3, 0.45).s
    rng = np.random.default_rng(scale)
    for p in [0.001, 0.05, 0.5, 0.97]:
        _check(asc, g, rng.random(g.n) < p, s)


def test_compaction_degenerate_sets(asc):
    g = gg.rmat(15, seed=3)          # 32768 vertices = 4 tiles
    n = g.n
    asc.load_csr(g.off, g.nbr)
    for frac in [0.0, 1.0, 0.37]:
        asc.set_budget(g.csr_bytes, frac)
        s = oracle.placer(g.off, 4, g.csr_bytes, frac).s
        alt = np.zeros(n, bool); alt[::2] = True
        blocks = np.zeros(n, bool); blocks[100:20000] = True        # one run across tiles
        edge = np.zeros(n, bool); edge[[0, n - 1]] = True
        for a in [np.zeros(n, bool), np.ones(n, bool), alt, ~alt, blocks, edge]:
            _check(asc, g, a, s)


@pytest.mark.parametrize("n", [1, 31, 32, 33, 8191, 8192, 8193, 40001])
def test_compaction_ragged_sizes(asc, n):
    g = gg.random_graph(n, 3 * n, seed=n)
    asc.load_csr(g.off, g.nbr)
    asc.set_option("hub_degree", 32)
    asc.set_budget(max(64, g.csr_bytes // 2), 0.5)
    s = oracle.placer(g.off, 4, max(64, g.csr_bytes // 2), 0.5).s
    rng = np.random.default_rng(n)
    _check(asc, g, rng.random(n) < 0.6, s, hub=32)
    asc.set_option("hub_degree", 2048)


def test_compaction_weighted_bytes(asc):
    g = gg.rmat(13, seed=8, weights=True)
    asc.load_csr(g.off, g.nbr, pairs=True)
    asc.set_budget(g.csr_bytes // 4)
    s = oracle.placer(g.off, 8, g.csr_bytes // 4).s
    rng = np.random.default_rng(1)
    _check(asc, g, rng.random(g.n) < 0.3, s)
