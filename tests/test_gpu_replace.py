"""GPU parity of the §3.4 data replacement (ASCETIC_OPT_REPLACE_CHUNKS; PAPER.md P:878-955,
Fig. 6) against the oracle's or_run_hot: per-iteration records including the static-vertex
count, the swaps and their bytes, bit-exact; results unchanged (PR within tolerance).
The static-hit kernels read swapped-in chunks through the slot table (sidx<REMAP>)."""
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
    for k, v in [("replace_chunks", 0), ("replace_policy", 0), ("chunk_cap", 0), ("xfer_mode", 0),
                 ("hub_degree", 2048), ("static_placement", 0), ("placement_seed", 1)]:
        m.set_option(k, v)
    m.unload()
    m.emulate_ranks(1)


def _check(its, ref, P=1):
    assert len(its) == len(ref.records)
    for a, b in zip(its, ref.records):
        for f in REC:
            assert a[f] == b[f], f"t={b['t']} rank={b['rank']} {f}: gpu {a[f]} oracle {b[f]}"
        assert a["s_static"] == b["s"], (b["t"], a["s_static"], b["s"])


def _values_ok(algo, res, ref):
    if algo == "pr":
        rel = np.abs(res.astype(np.float64) - ref.values) / ref.values
        assert rel.max() <= 1e-5
        assert np.abs(res.astype(np.float64) - ref.values).sum() <= 1e-6
    else:
        np.testing.assert_array_equal(res, ref.values)


def test_replace_worked_example_on_gpu(asc):
    from tests.test_oracle_replace import worked_graph
    off, nbr = worked_graph()
    asc.load_csr(off, nbr, symmetric=False)
    asc.set_option("replace_chunks", 1)
    asc.set_budget(32768 + 3 * 16384, 0.41)                   # Ms = floor(0.41 B / 16 KiB) 16 KiB = 32 KiB
    asc.run("bfs", 2)
    st, its = asc.stats()
    ref = oracle.run_hot("bfs", off, nbr, static_bytes=32768, src=2, kswap=1)
    assert st["static_reserved"] == 32768 and st["h2d_static_fill_bytes"] == 32768
    np.testing.assert_array_equal(asc.get_result(), [4, 5, 0, 1, 2, 2, 3])
    _check(its, ref)
    assert st["h2d_replace_bytes"] == 32768 and st["swaps_total"] == 2
    assert st["h2d_payload_bytes"] == 61640


@pytest.mark.parametrize("algo", ["bfs", "sssp", "cc", "pr"])
@pytest.mark.parametrize("K", [1, 16, 512])
@pytest.mark.parametrize("xfer", [1, 2])
def test_replace_parity(asc, algo, K, xfer):
    g = gg.rmat(14, seed=41, weights=(algo == "sssp"))
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    iters = 6 if algo == "pr" else 0
    budget = g.csr_bytes // 3
    asc.load_csr(g.off, g.nbr, pairs=g.pairs)
    asc.set_option("replace_chunks", K)
    asc.set_option("xfer_mode", xfer)
    asc.set_option("chunk_cap", 1 << 16)
    asc.set_budget(budget)
    p = oracle.placer(g.off, g.b_e, budget)
    ref = oracle.run_hot(algo, g.off, g.nbr, static_bytes=p.Ms, src=src, max_iters=iters, kswap=K)
    for rep in range(2):                                       # every run restarts from the front chunks
        asc.run(algo, src, iters)
        st, its = asc.stats()
        _values_ok(algo, asc.get_result().copy(), ref)
        _check(its, ref)
        assert st["h2d_static_fill_bytes"] == p.Ms
        assert st["h2d_replace_bytes"] == ref.replace_bytes
        assert st["h2d_payload_bytes"] == ref.h2d_payload
    if algo != "pr":
        assert ref.replace_bytes > 0
        # swapped-in chunks are read by the static-hit kernels: some hits lie outside the front prefix
        assert any(r["s"] != ref.records[0]["s"] for r in ref.records)


@pytest.mark.parametrize("algo", ["bfs", "sssp", "cc"])
def test_replace_hub_lists_across_slots(asc, algo):
    """Lists spanning many chunks (hub kernel, CTA pieces) read through the slot table."""
    g = gg.rmat(15, seed=43, weights=(algo == "sssp"))
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    budget = g.csr_bytes // 2
    asc.load_csr(g.off, g.nbr, pairs=g.pairs)
    asc.set_option("replace_chunks", 64)
    asc.set_option("hub_degree", 64)
    asc.set_budget(budget, 0.6)
    asc.run(algo, src)
    st, its = asc.stats()
    p = oracle.placer(g.off, g.b_e, budget, 0.6)
    ref = oracle.run_hot(algo, g.off, g.nbr, static_bytes=p.Ms, src=src, kswap=64)
    np.testing.assert_array_equal(asc.get_result(), ref.values)
    _check(its, ref)


@pytest.mark.parametrize("policy", [1, 2])
def test_replace_policy_override(asc, policy):
    g = gg.rmat(13, seed=44)
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    budget = g.csr_bytes // 3
    asc.load_csr(g.off, g.nbr)
    asc.set_option("replace_chunks", 32)
    asc.set_option("replace_policy", policy)
    asc.set_budget(budget)
    asc.run("cc", src)
    st, its = asc.stats()
    p = oracle.placer(g.off, 4, budget)
    ref = oracle.run_hot("cc", g.off, g.nbr, static_bytes=p.Ms, kswap=32,
                         policy="cumulative" if policy == 1 else "last")
    np.testing.assert_array_equal(asc.get_result(), ref.values)
    _check(its, ref)


@pytest.mark.parametrize("P", [2, 3])
@pytest.mark.parametrize("algo", ["bfs", "sssp", "cc"])
def test_replace_emulated_ranks(asc, P, algo):
    g = gg.rmat(13, seed=45, weights=(algo == "sssp"))
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    budget = g.csr_bytes // (3 * P)
    asc.emulate_ranks(P)
    asc.load_csr(g.off, g.nbr, pairs=g.pairs)
    asc.set_option("replace_chunks", 16)
    asc.set_budget(budget)
    asc.run(algo, src)
    st, its = asc.stats()
    b = oracle.partition(g.off, P)
    ms = [oracle.placer(g.off[int(b[k]):int(b[k + 1]) + 1] - g.off[int(b[k])], g.b_e, budget).Ms for k in range(P)]
    ref = oracle.run_hot(algo, g.off, g.nbr, static_bytes=ms, src=src, kswap=16, bounds=b)
    np.testing.assert_array_equal(asc.get_result(), ref.values)
    assert [i["rank"] for i in its] == [r["rank"] for r in ref.records]
    _check(its, ref)
    assert st["h2d_replace_bytes"] == ref.replace_bytes


def test_replace_rejects_rear_and_eq3(asc):
    g = gg.rmat(11, seed=46)
    asc.load_csr(g.off, g.nbr)
    asc.set_option("replace_chunks", 4)
    asc.set_option("static_placement", 1)
    with pytest.raises(asc.AsceticError):
        asc.set_budget(g.csr_bytes // 3)
    asc.set_option("static_placement", 0)
    asc.set_budget(g.csr_bytes // 3)
    asc.set_option("repartition", 1)
    with pytest.raises(asc.AsceticError):
        asc.run("bfs", 0)
    asc.set_option("repartition", 0)


@pytest.mark.parametrize("algo", ["bfs", "sssp", "cc", "pr"])
@pytest.mark.parametrize("seed,K", [(1, 0), (7, 0), (3, 32)])
def test_random_initial_content(asc, algo, seed, K):
    """§5 random initial content: the seeded chunk set is filled by the chunk-copy
    kernel, S is rebuilt from the residency; with and without §3.4 swaps on top."""
    g = gg.rmat(14, seed=47, weights=(algo == "sssp"))
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    iters = 5 if algo == "pr" else 0
    budget = g.csr_bytes // 3
    asc.load_csr(g.off, g.nbr, pairs=g.pairs)
    asc.set_option("static_placement", 2)
    asc.set_option("placement_seed", seed)
    asc.set_option("replace_chunks", K)
    asc.set_budget(budget)
    p = oracle.placer(g.off, g.b_e, budget)
    ref = oracle.run_hot(algo, g.off, g.nbr, static_bytes=p.Ms, src=src, max_iters=iters, kswap=K, random_seed=seed)
    for rep in range(2):
        asc.run(algo, src, iters)
        st, its = asc.stats()
        _values_ok(algo, asc.get_result().copy(), ref)
        _check(its, ref)
        assert st["s"] == ref.records[0]["s"]
        assert st["h2d_payload_bytes"] == ref.h2d_payload
        assert st["h2d_replace_bytes"] == ref.replace_bytes


@pytest.mark.parametrize("P", [2, 3])
def test_random_initial_content_ranks(asc, P):
    """Per-rank random chunk sets; rank payload starts are not 16-byte aligned (4-byte copy path)."""
    g = gg.rmat(13, seed=48)
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    budget = g.csr_bytes // (3 * P)
    asc.emulate_ranks(P)
    asc.load_csr(g.off, g.nbr)
    asc.set_option("static_placement", 2)
    asc.set_option("placement_seed", 5)
    asc.set_budget(budget)
    asc.run("cc", src)
    st, its = asc.stats()
    b = oracle.partition(g.off, P)
    ms = [oracle.placer(g.off[int(b[k]):int(b[k + 1]) + 1] - g.off[int(b[k])], 4, budget).Ms for k in range(P)]
    ref = oracle.run_hot("cc", g.off, g.nbr, static_bytes=ms, src=src, kswap=0, bounds=b, random_seed=5)
    np.testing.assert_array_equal(asc.get_result(), ref.values)
    _check(its, ref)
