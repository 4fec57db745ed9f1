"""P > 1 on one GPU: ascetic_emulate_ranks drives P rank parts through the same per-rank
code path as the NCCL build (owned ranges, per-rank placer/static region/transfer engine,
per-iteration exchange). Checked against the oracle's multi-rank simulation
(oracle.run(..., bounds=...)): results equal P = 1, per-rank records and bytes bit-exact."""
import numpy as np
import pytest

import graphgen as gg
import oracle

pytestmark = pytest.mark.gpu

REC = ["t", "rank", "nA", "nH", "nM", "nruns", "active_arcs", "hit_arcs", "miss_bytes", "digest"]


@pytest.fixture()
def asc():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import paper_conf_icpp_tangzwgzwy21_b200 as m
    m.unload()
    yield m
    m.unload()
    m.emulate_ranks(1)


def _rank_static(g, bounds, budget, frac):
    st = np.zeros(g.n, dtype=np.uint8)
    for k in range(len(bounds) - 1):
        lo, hi = int(bounds[k]), int(bounds[k + 1])
        p = oracle.placer(g.off[lo:hi + 1] - g.off[lo], g.b_e, budget, frac)
        st[lo:lo + p.s] = 1
    return st


@pytest.mark.parametrize("P", [2, 3, 4])
@pytest.mark.parametrize("algo", ["bfs", "sssp", "cc", "pr"])
def test_emulated_ranks_match_oracle(asc, P, algo):
    g = gg.rmat(12, seed=31, weights=(algo == "sssp"))
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    budget = g.csr_bytes // (4 * P)
    frac = 0.4
    iters = 8 if algo == "pr" else 0
    asc.emulate_ranks(P)
    asc.load_csr(g.off, g.nbr, pairs=g.pairs)
    asc.set_option("chunk_cap", 4096)
    asc.set_budget(budget, frac)
    asc.run(algo, src, iters)
    st, its = asc.stats()
    res = asc.get_result().copy()
    asc.set_option("chunk_cap", 0)
    bounds = oracle.partition(g.off, P)
    np.testing.assert_array_equal(asc.partition(g.off, P), bounds)
    stat = _rank_static(g, bounds, budget, frac)
    ref = oracle.run(algo, g.off, g.nbr, src=src, max_iters=iters, is_static=stat, bounds=bounds)
    one = oracle.run(algo, g.off, g.nbr, src=src, max_iters=iters, is_static=stat)
    if algo == "pr":
        rel = np.abs(res.astype(np.float64) - one.values) / one.values
        assert rel.max() <= 1e-5
        assert np.abs(res.astype(np.float64) - one.values).sum() <= 1e-6
    else:
        np.testing.assert_array_equal(res, one.values)       # results are those of P = 1
    assert st["world"] == P and st["iterations"] == ref.iterations
    assert [{f: i[f] for f in REC} for i in its] == [{f: r[f] for f in REC} for r in ref.records]
    assert st["h2d_payload_bytes"] == ref.h2d_payload


def test_emulated_uneven_partition_with_hub(asc):
    """A star (one hub holding most arcs) makes a rank own a single vertex."""
    n = 500
    src = np.zeros(n - 1, dtype=np.uint32)
    dst = np.arange(1, n, dtype=np.uint32)
    extra_s = np.arange(1, n - 1, dtype=np.uint32)
    g = gg.from_edges(n, np.concatenate([src, extra_s]), np.concatenate([dst, extra_s + 1]))
    P = 4
    asc.emulate_ranks(P)
    asc.load_csr(g.off, g.nbr)
    asc.set_budget(g.csr_bytes // 8, 0.5)
    asc.run("cc")
    st, its = asc.stats()
    bounds = oracle.partition(g.off, P)
    stat = _rank_static(g, bounds, g.csr_bytes // 8, 0.5)
    ref = oracle.run("cc", g.off, g.nbr, is_static=stat, bounds=bounds)
    np.testing.assert_array_equal(asc.get_result(), ref.values)
    assert [{f: i[f] for f in REC} for i in its] == [{f: r[f] for f in REC} for r in ref.records]


@pytest.mark.parametrize("P", [2, 3, 5])
@pytest.mark.parametrize("algo", ["bfs", "sssp", "cc", "prd"])
def test_fused_exchange_matches_oracle(asc, P, algo):
    """ASCETIC_OPT_FUSED_EXCHANGE: the finalize reads every rank's next bitmap / values /
    increments from the other parts' memory (peer memory on a multi-GPU box) between two
    barriers instead of the collective + copy-back; results and per-rank records unchanged."""
    g = gg.rmat(12, seed=33, weights=(algo == "sssp"))
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    budget = g.csr_bytes // (4 * P)
    asc.emulate_ranks(P)
    asc.load_csr(g.off, g.nbr, pairs=g.pairs)
    asc.set_option("fused_exchange", 1)
    asc.set_option("chunk_cap", 4096)
    try:
        asc.set_budget(budget, 0.4)
        for rep in range(2):                        # second run reuses the peer tables and buffers
            asc.run(algo, src)
            st, its = asc.stats()
            res = asc.get_result().copy()
            bounds = oracle.partition(g.off, P)
            stat = _rank_static(g, bounds, budget, 0.4)
            ref = oracle.run(algo, g.off, g.nbr, src=src, is_static=stat, bounds=bounds)
            exp = ref.values.astype(np.float32) if algo == "prd" else ref.values
            np.testing.assert_array_equal(res, exp)
            assert [{f: i[f] for f in REC} for i in its] == [{f: r[f] for f in REC} for r in ref.records]
        asc.set_option("fused_exchange", 0)          # and back to the collectives on the same parts
        asc.run(algo, src)
        np.testing.assert_array_equal(asc.get_result(), exp)
    finally:
        asc.set_option("fused_exchange", 0)
        asc.set_option("chunk_cap", 0)


def _bfs_sparse_prediction(g, levels, bounds, iters, d, P):
    """(sparse iterations, pair bytes) of the BFS sparse exchange, from the oracle's levels."""
    n = g.n
    deg = np.diff(g.off.astype(np.int64))
    src_of = np.repeat(np.arange(n, dtype=np.int64), deg)
    dst = g.nbr.astype(np.int64)
    lv = levels.astype(np.int64)
    cap = max(1, n // (64 * d * P))
    sparse, byt = 0, 0
    for t in range(iters):
        hit = (lv[src_of] == t) & (lv[dst] == t + 1)
        counts = [np.unique(dst[hit & (src_of >= int(bounds[r])) & (src_of < int(bounds[r + 1]))]).size
                  for r in range(P)]
        if max(counts) <= cap:
            sparse += 1
            byt += 8 * sum(counts)
    return sparse, byt


@pytest.mark.parametrize("P", [2, 3, 5])
@pytest.mark.parametrize("algo", ["bfs", "sssp", "cc"])
@pytest.mark.parametrize("d", [1, 8, 2000])
def test_sparse_exchange_matches_oracle(asc, P, algo, d):
    """ASCETIC_OPT_SPARSE_EXCHANGE: each rank's lowered (id, value) pairs (BFS:
    newly reached ids) are exchanged and applied with atomicMin + next bit when every rank has at
    most n/(d P) of them (BFS n/(64 d P)), else the dense MIN / OR runs. d = 1, 8: mostly sparse;
    d = 2000: a cap of 1 pair, so nearly every iteration falls back to dense. Values and every
    per-rank record equal the oracle either way."""
    g = gg.rmat(12, seed=35, weights=(algo == "sssp"))
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    budget = g.csr_bytes // (4 * P)
    asc.emulate_ranks(P)
    asc.load_csr(g.off, g.nbr, pairs=g.pairs, symmetric=True)
    asc.set_option("sparse_exchange", d)
    asc.set_option("chunk_cap", 4096)
    try:
        asc.set_budget(budget, 0.4)
        for rep in range(2):                        # second run reuses the pair buffers
            asc.run(algo, src)
            st, its = asc.stats()
            res = asc.get_result().copy()
            bounds = oracle.partition(g.off, P)
            ref = oracle.run(algo, g.off, g.nbr, src=src, is_static=_rank_static(g, bounds, budget, 0.4),
                             bounds=bounds)
            np.testing.assert_array_equal(res, ref.values)
            assert [{f: i[f] for f in REC} for i in its] == [{f: r[f] for f in REC} for r in ref.records]
            if algo == "bfs":
                # exact: rank r's pairs at level t are the ids it newly reached, i.e. the level-(t+1)
                # vertices adjacent to its owned level-t vertices; the level goes sparse iff every
                # rank has at most max(1, n / (64 d P)) of them, and moves 8 bytes per pair
                cnt, byt = _bfs_sparse_prediction(g, ref.values, bounds, st["iterations"], d, P)
                assert st["sparse_exchanges"] == cnt and st["sparse_exchange_bytes"] == byt
            elif d == 1 or d == 8:
                assert st["sparse_exchanges"] >= 1 and st["sparse_exchange_bytes"] > 0
            else:
                assert st["sparse_exchanges"] < st["iterations"]
        asc.set_option("sparse_exchange", 0)         # back to dense on the same parts
        asc.run(algo, src)
        np.testing.assert_array_equal(asc.get_result(), ref.values)
        assert asc.stats()[0]["sparse_exchanges"] == 0
    finally:
        asc.set_option("sparse_exchange", 0)
        asc.set_option("chunk_cap", 0)


@pytest.mark.parametrize("algo", ["cc", "pr"])
def test_reload_same_shape_new_partition(asc, algo):
    """Two graphs with the same n and m but different offsets, loaded back to back with P = 2:
    the second load must re-cut the rank ranges (each part's owned range and range-sized queues),
    so per-rank records follow the new partition and PR's slice exchange shares the right slices."""
    g1 = gg.rmat(11, seed=41)
    n = g1.n
    # relabel v -> n-1-v: same n and m, mirrored degree sequence, so other edge-balanced bounds
    deg = np.diff(g1.off.astype(np.int64))
    src = np.repeat(np.arange(n, dtype=np.int64), deg)
    g2 = gg.from_edges(n, (n - 1 - src).astype(np.uint32), (n - 1 - g1.nbr.astype(np.int64)).astype(np.uint32),
                       symmetrize=False, keep_dups=True)
    assert g2.m == g1.m and not np.array_equal(oracle.partition(g1.off, 2), oracle.partition(g2.off, 2))
    P, frac = 2, 0.4
    asc.emulate_ranks(P)
    iters = 6 if algo == "pr" else 0
    for g in (g1, g2):
        budget = g.csr_bytes // (4 * P)
        asc.load_csr(g.off, g.nbr)
        asc.set_option("chunk_cap", 4096)
        asc.set_budget(budget, frac)
        asc.run(algo, 0, iters)
        st, its = asc.stats()
        res = asc.get_result().copy()
        asc.set_option("chunk_cap", 0)
        bounds = oracle.partition(g.off, P)
        stat = _rank_static(g, bounds, budget, frac)
        ref = oracle.run(algo, g.off, g.nbr, max_iters=iters, is_static=stat, bounds=bounds)
        assert [{f: i[f] for f in REC} for i in its] == [{f: r[f] for f in REC} for r in ref.records]
        if algo == "pr":
            rel = np.abs(res.astype(np.float64) - ref.values) / ref.values
            assert rel.max() <= 1e-5
        else:
            np.testing.assert_array_equal(res, ref.values)


def test_kept_static_region_follows_placement(asc):
    """keep_static with a placement change (random -> front, front -> rear): the kept Static Region
    no longer holds what the new placement expects, so the next run must refill it."""
    g = gg.rmat(12, seed=43)
    asc.emulate_ranks(1)
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    budget = g.csr_bytes // 3
    asc.load_csr(g.off, g.nbr)
    asc.set_option("keep_static", 1)
    try:
        for placement in (2, 0, 1, 0):
            asc.set_option("static_placement", placement)
            asc.set_budget(budget)
            asc.run("bfs", src)
            st, _ = asc.stats()
            assert st["h2d_static_fill_bytes"] > 0, placement    # refilled after every change
            p = oracle.placer(g.off, 4, budget)
            if placement == 1:
                stat = oracle.static_rear(g.n, oracle.rear_start(g.off, 4, p.Ms))
                ref = oracle.run("bfs", g.off, g.nbr, src=src, is_static=stat)
            elif placement == 2:
                ref = oracle.run_hot("bfs", g.off, g.nbr, static_bytes=p.Ms, src=src, kswap=0, random_seed=1)
            else:
                ref = oracle.run("bfs", g.off, g.nbr, src=src, is_static=oracle.static_prefix(g.n, p.s))
            np.testing.assert_array_equal(asc.get_result(), ref.values)
            assert st["h2d_payload_bytes"] == ref.h2d_payload
        asc.run("bfs", src)                                        # unchanged: the region is kept
        assert asc.stats()[0]["h2d_static_fill_bytes"] == 0
    finally:
        asc.set_option("keep_static", 0)
        asc.set_option("static_placement", 0)


@pytest.mark.parametrize("fused", [0, 1])
@pytest.mark.parametrize("algo", ["sssp", "cc"])
def test_emulated_red_min(asc, algo, fused):
    """RED.MIN updates with P = 3 emulated ranks (MIN exchange or fused peer finalize)."""
    P = 3
    g = gg.rmat(12, seed=37, weights=(algo == "sssp"))
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    budget = g.csr_bytes // (4 * P)
    asc.emulate_ranks(P)
    asc.load_csr(g.off, g.nbr, pairs=g.pairs)
    asc.set_option("relax_mode", 2)
    asc.set_option("fused_exchange", fused)
    asc.set_option("chunk_cap", 4096)
    try:
        asc.set_budget(budget, 0.4)
        asc.run(algo, src)
        st, its = asc.stats()
        res = asc.get_result().copy()
    finally:
        asc.set_option("relax_mode", 0)
        asc.set_option("fused_exchange", 0)
        asc.set_option("chunk_cap", 0)
    bounds = oracle.partition(g.off, P)
    ref = oracle.run(algo, g.off, g.nbr, src=src, is_static=_rank_static(g, bounds, budget, 0.4), bounds=bounds)
    np.testing.assert_array_equal(res, ref.values)
    assert [{f: i[f] for f in REC} for i in its] == [{f: r[f] for f in REC} for r in ref.records]
