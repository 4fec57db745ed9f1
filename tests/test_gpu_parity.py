"""GPU parity: the CUDA path (through the C ABI) vs the CPU oracle, element by element.

Bit-exact: BFS levels, SSSP distances, CC labels, per-iteration active sets (digest,
|A|, |H|, |M|, #runs, active/hit arcs) and per-iteration transferred bytes.
PageRank (fp32 on the GPU vs fp64 oracle): max per-vertex relative error <= 1e-5 and
L1 <= 1e-6 after the same number of iterations (BASELINE.json north_star).
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


def _oracle(algo, g, src, s_static, max_iters=0):
    return oracle.run(algo, g.off, g.nbr, src=src, max_iters=max_iters, is_static=oracle.static_prefix(g.n, s_static))


def _check_records(its, ref):
    assert len(its) == len(ref.records)
    for t, (a, b) in enumerate(zip(its, ref.records)):
        assert a["t"] == t
        for f in REC:
            assert a[f] == b[f], f"iteration {t} field {f}: gpu {a[f]} oracle {b[f]}"


def _run(asc, g, algo, src=0, budget=None, frac=-1.0, max_iters=0, chunk_cap=0, xfer=0, hub=2048):
    asc.load_csr(g.off, g.nbr, pairs=g.pairs, symmetric=True)
    asc.set_option("chunk_cap", chunk_cap)
    asc.set_option("xfer_mode", xfer)
    asc.set_option("hub_degree", hub)
    asc.set_budget(budget if budget is not None else g.csr_bytes // 4, frac)
    asc.run(algo, src, max_iters)
    st, its = asc.stats()
    return st, its, asc.get_result().copy()


def _pr_ok(gpu, ref):
    rel = np.abs(gpu.astype(np.float64) - ref) / np.abs(ref)
    l1 = np.abs(gpu.astype(np.float64) - ref).sum()
    assert rel.max() <= 1e-5, rel.max()
    assert l1 <= 1e-6, l1


ALGO_GRAPHS = {
    "bfs": dict(scale=12, weights=False),
    "sssp": dict(scale=12, weights=True),
    "cc": dict(scale=12, weights=False),
    "pr": dict(scale=12, weights=False),
}


@pytest.mark.parametrize("algo", ["bfs", "sssp", "cc", "pr"])
@pytest.mark.parametrize("frac", [-1.0, 0.0, 1.0, 0.5])
@pytest.mark.parametrize("xfer", [1, 2])
def test_parity_small(asc, algo, frac, xfer):
    cfg = ALGO_GRAPHS[algo]
    g = gg.rmat(cfg["scale"], seed=3, weights=cfg["weights"])
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    iters = 10 if algo == "pr" else 0
    st, its, res = _run(asc, g, algo, src=src, frac=frac, max_iters=iters, xfer=xfer, chunk_cap=4096)
    p = oracle.placer(g.off, g.b_e, g.csr_bytes // 4, frac)
    assert st["s"] == p.s and st["static_bytes"] == p.static_bytes
    ref = _oracle(algo, g, src, p.s, max_iters=iters)
    assert st["iterations"] == ref.iterations
    _check_records(its, ref)
    assert st["h2d_payload_bytes"] == ref.h2d_payload
    assert st["active_arcs_total"] == ref.active_arcs_total
    if algo == "pr":
        _pr_ok(res, ref.values)
    else:
        np.testing.assert_array_equal(res, ref.values)


@pytest.mark.parametrize("algo", ["bfs", "sssp", "cc"])
def test_parity_tiny_chunks_split_hubs(asc, algo):
    """16-byte chunks force every hub list across many chunks; hub threshold 32 forces multi-CTA hubs."""
    g = gg.rmat(10, seed=7, weights=(algo == "sssp"))
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    st, its, res = _run(asc, g, algo, src=src, frac=0.3, chunk_cap=16, xfer=1, hub=32)
    p = oracle.placer(g.off, g.b_e, g.csr_bytes // 4, 0.3)
    ref = _oracle(algo, g, src, p.s)
    np.testing.assert_array_equal(res, ref.values)
    _check_records(its, ref)


def test_parity_pr_tiny_chunks(asc):
    g = gg.rmat(10, seed=8)
    st, its, res = _run(asc, g, "pr", frac=0.2, max_iters=7, chunk_cap=48, xfer=1, hub=32)
    p = oracle.placer(g.off, 4, g.csr_bytes // 4, 0.2)
    ref = _oracle("pr", g, 0, p.s, max_iters=7)
    _check_records(its, ref)
    _pr_ok(res, ref.values)


@pytest.mark.parametrize("n", [1, 2, 31, 33, 65, 1000])
def test_edge_sizes_random(asc, n):
    """n not a multiple of 32, tiny graphs, isolated vertices."""
    g = gg.random_graph(n, 2 * n, seed=n)
    for algo in ["bfs", "cc"]:
        src = 0
        st, its, res = _run(asc, g, algo, src=src, budget=max(64, g.csr_bytes // 3), frac=0.5, chunk_cap=32)
        p = oracle.placer(g.off, 4, max(64, g.csr_bytes // 3), 0.5)
        ref = _oracle(algo, g, src, p.s)
        np.testing.assert_array_equal(res, ref.values)
        _check_records(its, ref)


def test_isolated_source(asc):
    n = 100
    src = np.array([1, 2, 3], dtype=np.uint32)
    dst = np.array([2, 3, 4], dtype=np.uint32)
    g = gg.from_edges(n, src, dst)
    st, its, res = _run(asc, g, "bfs", src=50, frac=0.5, chunk_cap=16)
    assert st["iterations"] == 1
    assert res[50] == 0 and (np.delete(res, 50) == 0xFFFFFFFF).all()
    assert its[0]["active_arcs"] == 0 and its[0]["miss_bytes"] == 0


def test_max_iters_and_repeat_runs(asc):
    g = gg.rmat(11, seed=4)
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    _run(asc, g, "bfs", src=src)
    for k in [1, 2, 3]:
        asc.run("bfs", src, k)
        st, its = asc.stats()
        res = asc.get_result()
        p = oracle.placer(g.off, 4, g.csr_bytes // 4)
        ref = _oracle("bfs", g, src, p.s, max_iters=k)
        np.testing.assert_array_equal(res, ref.values)
        _check_records(its, ref)


def test_c1_config_full(asc):
    """BASELINE config 1: BFS on RMAT-16 at 25 % of CSR bytes, Eq. 2 split, default chunking."""
    g = gg.config_graph("c1")
    budget = gg.config_budget("c1", g)
    for src in gg.sources(g, 4, seed=1):
        for xfer in [0, 1, 2]:
            st, its, res = _run(asc, g, "bfs", src=src, budget=budget, xfer=xfer)
            p = oracle.placer(g.off, 4, budget)
            ref = _oracle("bfs", g, src, p.s)
            np.testing.assert_array_equal(res, ref.values)
            _check_records(its, ref)
            assert st["h2d_static_fill_bytes"] == p.static_bytes
            assert st["h2d_payload_bytes"] == ref.h2d_payload


def test_resident_r1_moves_no_payload(asc):
    g = gg.rmat(12, seed=2)
    st, its, res = _run(asc, g, "cc", budget=10 * g.csr_bytes)
    assert st["s"] == g.n and st["h2d_payload_bytes"] == 0
    ref = _oracle("cc", g, 0, g.n)
    np.testing.assert_array_equal(res, ref.values)


def test_errors_on_gpu(asc):
    g = gg.rmat(8, seed=1)
    asc.load_csr(g.off, g.nbr, symmetric=False)
    asc.set_budget(g.csr_bytes)
    with pytest.raises(asc.AsceticError):
        asc.run("cc")                      # CC needs SYMMETRIC
    with pytest.raises(asc.AsceticError):
        asc.run("sssp", 0)                 # SSSP needs weights
    with pytest.raises(asc.AsceticError):
        asc.run("bfs", g.n)                # source out of range
    with pytest.raises(asc.AsceticError):
        asc.run("pr", 0, 0)                # PR needs iterations
    with pytest.raises(asc.AsceticError) as e:
        asc.set_budget(10, 0.0)            # on-demand chunk below 16 bytes
    assert e.value.code == asc.ENOMEM


def test_load_variants_copy_wgt_validate(asc):
    """COPY (library-owned pinned copy), separate weight array (interleaved by the library),
    VALIDATE, and duplicate arcs / self-loops kept in the CSR (degree counts multiplicity)."""
    g = gg.rmat(11, seed=12, weights=True)
    ids, w = g.ids().copy(), g.weights().copy()
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    p = oracle.placer(g.off, 8, g.csr_bytes // 3)
    ref = _oracle("sssp", g, src, p.s)
    for kw in [dict(copy=True), dict(validate=True)]:
        asc.load_csr(g.off, g.nbr, pairs=True, **kw)
        asc.set_budget(g.csr_bytes // 3)
        asc.run("sssp", src)
        np.testing.assert_array_equal(asc.get_result(), ref.values)
    asc.load_csr(g.off, ids, wgt=w)                       # separate weights
    asc.set_budget(g.csr_bytes // 3)
    asc.run("sssp", src)
    np.testing.assert_array_equal(asc.get_result(), ref.values)
    st, its = asc.stats()
    _check_records(its, ref)
    # multigraph with self-loops: the oracle and the engine both count multiplicity
    n = 300
    rng = np.random.default_rng(5)
    s_ = rng.integers(0, n, 2000).astype(np.uint32)
    d_ = rng.integers(0, n, 2000).astype(np.uint32)
    gm = gg.from_edges(n, s_, d_, keep_dups=True)
    for algo in ["bfs", "cc"]:
        st, its, res = _run(asc, gm, algo, src=0, budget=gm.csr_bytes // 2, frac=0.5, chunk_cap=64)
        pm = oracle.placer(gm.off, 4, gm.csr_bytes // 2, 0.5)
        refm = _oracle(algo, gm, 0, pm.s)
        np.testing.assert_array_equal(res, refm.values)
        _check_records(its, refm)


@pytest.mark.parametrize("opt,val", [("overlap", 0), ("keep_static", 1), ("chunk_buffers", 2),
                                     ("chunk_buffers", 3), ("chunk_buffers", 8), ("gather_ctas", 1), ("static_ctas_per_sm", 1),
                                     ("timing", 0), ("timing", 2), ("relax_mode", 1), ("relax_mode", 2), ("ce_min_run", 0),
                                     ("ce_min_run", 2048), ("gap_bridge", 0), ("gap_bridge", 4096)])
def test_options_do_not_change_results(asc, opt, val):
    """Tuning knobs change scheduling only: results, records and bytes stay bit-exact."""
    g = gg.rmat(12, seed=14, weights=True)
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    asc.load_csr(g.off, g.nbr, pairs=True)
    asc.set_option(opt, val)
    asc.set_budget(g.csr_bytes // 4)
    p = oracle.placer(g.off, 8, g.csr_bytes // 4)
    ref = _oracle("sssp", g, src, p.s)
    for rep in range(2):                                   # keep_static: 2nd run skips the fill
        asc.run("sssp", src)
        st, its = asc.stats()
        np.testing.assert_array_equal(asc.get_result(), ref.values)
        _check_records(its, ref)
        assert st["h2d_payload_bytes"] == ref.h2d_payload
        if opt == "keep_static" and rep == 1:
            assert st["h2d_static_fill_bytes"] == 0
        else:
            assert st["h2d_static_fill_bytes"] == p.static_bytes
    defaults = {"overlap": 1, "keep_static": 0, "chunk_buffers": 0, "gather_ctas": 0, "static_ctas_per_sm": 0,
                "timing": 1, "relax_mode": 0, "ce_min_run": 1 << 20, "gap_bridge": 0}
    asc.set_option(opt, defaults[opt])


@pytest.mark.parametrize("prefetch", [0, 1])
@pytest.mark.parametrize("nbuf", [2, 3, 5])
def test_pr_cross_iteration_prefetch(asc, prefetch, nbuf):
    """PR with copy-engine DMA chunks and the next-iteration prefetch: many small chunks per
    iteration so prefetched buffers wrap around; results and per-iteration bytes unchanged."""
    g = gg.rmat(12, seed=21)
    asc.load_csr(g.off, g.nbr)
    asc.set_option("prefetch", prefetch)
    asc.set_option("chunk_buffers", nbuf)
    asc.set_option("xfer_mode", 2)
    asc.set_option("chunk_cap", 4096)
    asc.set_budget(g.csr_bytes // 3, 0.5)
    asc.run("pr", 0, 9)
    st, its = asc.stats()
    res = asc.get_result().copy()
    asc.set_option("prefetch", 1)
    asc.set_option("chunk_buffers", 0)
    asc.set_option("xfer_mode", 0)
    asc.set_option("chunk_cap", 0)
    p = oracle.placer(g.off, 4, g.csr_bytes // 3, 0.5)
    ref = _oracle("pr", g, 0, p.s, max_iters=9)
    _check_records(its, ref)
    _pr_ok(res, ref.values)
    assert st["dma_chunks"] == st["chunks_total"] > 9 * nbuf
    assert st["dma_bytes"] == st["h2d_payload_bytes"] == ref.h2d_payload


@pytest.mark.parametrize("algo", ["bfs", "sssp", "cc", "pr"])
def test_rear_static_placement(asc, algo):
    """Rear initial content (§5): the static set is the suffix of whole lists
    that fits in Ms; records, bytes and results vs the oracle on that set."""
    g = gg.rmat(12, seed=17, weights=(algo == "sssp"))
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    iters = 6 if algo == "pr" else 0
    budget = g.csr_bytes // 3
    asc.load_csr(g.off, g.nbr, pairs=g.pairs)
    asc.set_option("static_placement", 1)
    asc.set_option("chunk_cap", 8192)
    asc.set_budget(budget)
    asc.run(algo, src, iters)
    st, its = asc.stats()
    res = asc.get_result().copy()
    asc.set_option("static_placement", 0)
    asc.set_option("chunk_cap", 0)
    p = oracle.placer(g.off, g.b_e, budget)
    s_lo = oracle.rear_start(g.off, g.b_e, p.Ms)
    ref = oracle.run(algo, g.off, g.nbr, src=src, max_iters=iters, is_static=oracle.static_rear(g.n, s_lo))
    assert st["s"] == g.n - s_lo
    assert st["h2d_static_fill_bytes"] == g.b_e * (int(g.off[-1]) - int(g.off[s_lo]))
    _check_records(its, ref)
    if algo == "pr":
        _pr_ok(res, ref.values)
    else:
        np.testing.assert_array_equal(res, ref.values)


@pytest.mark.parametrize("algo", ["bfs", "sssp", "cc"])
def test_eq3_repartition_parity(asc, algo):
    """Eq. 3 adaptive re-partition (ASCETIC_OPT_REPARTITION): the shrink decisions, the static
    prefix per iteration, every record and the results match the oracle's Eq. 3."""
    from tests.test_oracle import two_communities
    g = two_communities()
    if algo == "sssp":
        s_, d_ = np.repeat(np.arange(g.n), np.diff(g.off.astype(np.int64))).astype(np.uint32), g.nbr
        g = gg.from_edges(g.n, s_, d_, weights=True)
    budget = g.csr_bytes // 2
    asc.load_csr(g.off, g.nbr, pairs=g.pairs)
    asc.set_option("repartition", 1)
    asc.set_budget(budget)
    src = 900
    for rep in range(2):                                   # the split resets for every run
        asc.run(algo, src)
        st, its = asc.stats()
        res = asc.get_result().copy()
        p = oracle.placer(g.off, g.b_e, budget)
        ref = oracle.run(algo, g.off, g.nbr, src=src, is_static=oracle.static_prefix(g.n, p.s),
                         eq3_budget=budget, eq3_ms=p.Ms)
        np.testing.assert_array_equal(res, ref.values)
        _check_records(its, ref)
        assert [i["s_static"] for i in its] == [r["s"] for r in ref.records]
        assert st["repartitions"] == ref.repartitions
        assert st["h2d_payload_bytes"] == ref.h2d_payload
    if algo == "bfs":
        assert ref.repartitions >= 1
    asc.set_option("repartition", 0)


@pytest.mark.parametrize("shift", [1, 2, 3, 37, 102])
@pytest.mark.parametrize("algo", ["bfs", "sssp", "cc", "pr"])
def test_gather_unaligned_host_arrays(asc, algo, shift):
    """The zero-copy gather reads 16-byte-aligned cover units of the host CSR, and enumerates long
    pieces by 512-byte host block: host arrays that start 4, 8 or 12 bytes past a 16-byte boundary
    and at other phases of a 512-byte block (shift in words from a 16-byte boundary), with chunk
    windows that cut runs anywhere, must still deliver exactly the missed lists."""
    cfg = ALGO_GRAPHS[algo]
    g = gg.rmat(cfg["scale"], seed=11, weights=cfg["weights"])
    buf = np.zeros(g.nbr.size + 136, dtype=np.uint32)
    base = (-(buf.ctypes.data // 4)) % 4             # word offset of a 16-byte boundary
    nbr = buf[base + shift: base + shift + g.nbr.size]
    nbr[:] = g.nbr
    assert nbr.ctypes.data % 16 == 4 * (shift % 4)
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    iters = 6 if algo == "pr" else 0
    for cap in (4096, 200):
        asc.load_csr(g.off, nbr, pairs=g.pairs, symmetric=True)
        asc.set_option("chunk_cap", cap)
        asc.set_option("xfer_mode", 1)
        asc.set_budget(g.csr_bytes // 4, 0.3)
        asc.run(algo, src, iters)
        st, its = asc.stats()
        res = asc.get_result().copy()
        asc.set_option("chunk_cap", 0)
        asc.set_option("xfer_mode", 0)
        p = oracle.placer(g.off, g.b_e, g.csr_bytes // 4, 0.3)
        ref = _oracle(algo, g, src, p.s, max_iters=iters)
        _check_records(its, ref)
        if algo == "pr":
            _pr_ok(res, ref.values)
        else:
            np.testing.assert_array_equal(res, ref.values)


@pytest.mark.parametrize("mib,nb", [(11, 2), (13, 3)])
def test_auto_chunk_buffers(asc, mib, nb):
    """Auto chunk buffers (option 0): 3 buffers of C/3, or 2 when C/3 < 4 MiB; results unchanged."""
    g = gg.config_graph("c1")
    budget = mib << 20
    asc.load_csr(g.off, g.nbr)
    asc.set_option("chunk_buffers", 0)
    asc.set_budget(budget, 0.0)                            # R = 0: C = B
    src = gg.sources(g, 1, seed=1)[0]
    asc.run("bfs", src)
    st, its = asc.stats()
    assert st["chunk_buffers"] == nb
    assert st["chunk_cap"] == min(budget // nb, 4 * g.m) // 16 * 16
    ref = _oracle("bfs", g, src, 0)
    np.testing.assert_array_equal(asc.get_result(), ref.values)
    _check_records(its, ref)


def test_pr_bitwise_reproducible(asc):
    """PR sums are combined in 2^-62 fixed point (integer atomics), so two runs with the same
    options give bitwise-identical fp32 ranks, whatever order the hub-piece and chunk-segment
    partials land in (DESIGN R31); still within the tolerance of the fp64 oracle."""
    g = gg.rmat(14, seed=31)
    asc.load_csr(g.off, g.nbr)
    asc.set_option("hub_degree", 64)                       # many multi-CTA hub rows
    asc.set_option("chunk_cap", 3000)                      # rows split across chunks and segments
    asc.set_option("xfer_mode", 1)
    asc.set_budget(g.csr_bytes // 3, 0.4)
    runs = []
    for _ in range(3):
        asc.run("pr", 0, 12)
        runs.append(asc.get_result().copy())
    asc.set_option("hub_degree", 2048)
    asc.set_option("chunk_cap", 0)
    asc.set_option("xfer_mode", 0)
    assert all(np.array_equal(r.view(np.uint32), runs[0].view(np.uint32)) for r in runs[1:])
    p = oracle.placer(g.off, 4, g.csr_bytes // 3, 0.4)
    ref = _oracle("pr", g, 0, p.s, max_iters=12)
    _pr_ok(runs[0], ref.values)
    assert abs(runs[0].astype(np.float64).sum() - 1.0) <= 1e-5


@pytest.mark.parametrize("mode", [1, 2])
@pytest.mark.parametrize("algo", ["sssp", "cc"])
def test_relax_modes_resident_and_out_of_core(asc, mode, algo):
    """Both SSSP/CC min-update forms (atomicMin + next bit, RED.MIN + dense finalize) give the same
    values, active sets and bytes, resident (all lists static) and out of core."""
    g = gg.rmat(13, seed=19, weights=(algo == "sssp"))
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    asc.set_option("relax_mode", mode)
    try:
        for budget in (10 * g.csr_bytes, g.csr_bytes // 4):
            st, its, res = _run(asc, g, algo, src=src, budget=budget)
            p = oracle.placer(g.off, g.b_e, budget)
            ref = _oracle(algo, g, src, p.s)
            np.testing.assert_array_equal(res, ref.values)
            _check_records(its, ref)
            assert st["h2d_payload_bytes"] == ref.h2d_payload
    finally:
        asc.set_option("relax_mode", 0)


@pytest.mark.parametrize("shift", [0, 1])
@pytest.mark.parametrize("algo", ["bfs", "sssp", "cc", "pr"])
def test_hybrid_gather_copy_engine_long_runs(asc, algo, shift):
    """Gather-mode iterations with long runs: runs >= CE_MIN_RUN bytes go to the copy engines on a
    second copy stream while the SM gather (skipping their vertices, bridging small holes) moves the
    rest of each chunk window. Small windows cut long runs across chunks; the host array may start
    off a 16-byte boundary. Values, records and bytes equal the oracle's; the CE path must run."""
    cfg = ALGO_GRAPHS[algo]
    g = gg.rmat(cfg["scale"], seed=23, weights=cfg["weights"])
    buf = np.zeros(g.nbr.size + 8, dtype=np.uint32)
    base = (-(buf.ctypes.data // 4)) % 4
    nbr = buf[base + shift: base + shift + g.nbr.size]
    nbr[:] = g.nbr
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    iters = 6 if algo == "pr" else 0
    ce_total = 0
    for cap, ce in ((3000, 1024), (1 << 16, 256), (1 << 16, 4096)):
        asc.load_csr(g.off, nbr, pairs=g.pairs, symmetric=True)
        asc.set_option("chunk_cap", cap)
        asc.set_option("xfer_mode", 1)
        asc.set_option("ce_min_run", ce)
        asc.set_option("gap_bridge", 64)
        asc.set_budget(g.csr_bytes // 4, 0.3)
        asc.run(algo, src, iters)
        st, its = asc.stats()
        res = asc.get_result().copy()
        for k, v in (("chunk_cap", 0), ("xfer_mode", 0), ("ce_min_run", 1 << 20), ("gap_bridge", 0)):
            asc.set_option(k, v)
        p = oracle.placer(g.off, g.b_e, g.csr_bytes // 4, 0.3)
        ref = _oracle(algo, g, src, p.s, max_iters=iters)
        _check_records(its, ref)
        assert st["h2d_payload_bytes"] == ref.h2d_payload == st["gather_bytes"]
        if algo == "pr":
            _pr_ok(res, ref.values)
        else:
            np.testing.assert_array_equal(res, ref.values)
        ce_total += st["gather_ce_bytes"]
        # the SM gather loads at least the payload it moves (cover units, bridged holes)
        assert st["gather_load_bytes"] >= st["gather_bytes"] - st["gather_ce_bytes"]
    assert ce_total > 0


@pytest.mark.parametrize("resident", [True, False])
def test_pr_segmented_pull(asc, resident):
    """PR static pull in neighbour-id slices (ASCETIC_OPT_PR_SEGMENT, sorted rows): a small slice size
    forces several passes with per-row / per-piece cursors; ranks within tolerance of the oracle,
    records and bytes unchanged, bitwise reproducible, and close to the unsegmented pull."""
    g = gg.rmat(14, seed=33)
    budget = 10 * g.csr_bytes if resident else g.csr_bytes // 3
    res = {}
    for seg in (0, 16 << 10):                              # 4n = 64 KiB: 4 slices (capped by mean degree / 8)
        asc.load_csr(g.off, g.nbr, sorted_rows=True)
        asc.set_option("pr_segment", seg)
        asc.set_option("hub_degree", 256)                  # hub pieces get cursors too
        asc.set_budget(budget)
        asc.run("pr", 0, 8)
        st, its = asc.stats()
        res[seg] = asc.get_result().copy()
        if seg:
            assert st["pr_segment_passes"] >= 2
            asc.run("pr", 0, 8)
            assert np.array_equal(asc.get_result().view(np.uint32), res[seg].view(np.uint32))
        else:
            assert st["pr_segment_passes"] == 0
    asc.set_option("pr_segment", 128 << 20)
    asc.set_option("hub_degree", 2048)
    p = oracle.placer(g.off, 4, budget)
    ref = _oracle("pr", g, 0, p.s, max_iters=8)
    _check_records(its, ref)
    _pr_ok(res[16 << 10], ref.values)
    assert np.abs(res[16 << 10].astype(np.float64) - res[0]).max() <= 1e-6 * res[0].max()


def test_sorted_flag_validated(asc):
    g = gg.rmat(10, seed=5)
    asc.load_csr(g.off, g.nbr, sorted_rows=True, validate=True)       # generator rows are sorted
    bad = g.nbr.copy()
    deg = np.diff(g.off.astype(np.int64))
    v = int(np.argmax(deg))
    a = int(g.off[v])
    bad[a], bad[a + 1] = bad[a + 1], bad[a]
    with pytest.raises(asc.AsceticError):
        asc.load_csr(g.off, bad, sorted_rows=True, validate=True)
    asc.unload()


@pytest.mark.parametrize("density", [0, 50, 85])
@pytest.mark.parametrize("algo", ["bfs", "sssp", "cc", "pr", "prd"])
def test_span_dma_windows(asc, algo, density):
    """Span-DMA iterations (XFER_MODE 3): windows are host ranges of cap bytes over the miss stream's
    span; windows at least `density` % full are one DMA of their host bytes read in place by the
    on-demand kernels (span_base addressing), sparser ones are gathered. density 0 = every window
    DMA'd. Values, records and payload bytes equal the oracle's; the span path must run."""
    g = gg.rmat(12, seed=27, weights=(algo == "sssp"))
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    iters = 6 if algo in ("pr",) else 0
    asc.load_csr(g.off, g.nbr, pairs=g.pairs, symmetric=True)
    asc.set_option("chunk_cap", 4096)
    asc.set_option("xfer_mode", 3)
    asc.set_option("span_density", density)
    try:
        asc.set_budget(g.csr_bytes // 4, 0.3)
        asc.run(algo, src, iters)
        st, its = asc.stats()
        res = asc.get_result().copy()
    finally:
        asc.set_option("chunk_cap", 0)
        asc.set_option("xfer_mode", 0)
        asc.set_option("span_density", 85)
    p = oracle.placer(g.off, g.b_e, g.csr_bytes // 4, 0.3)
    ref = _oracle(algo, g, src, p.s, max_iters=iters)
    _check_records(its, ref)
    assert st["h2d_payload_bytes"] == ref.h2d_payload
    if algo == "pr":
        _pr_ok(res, ref.values)
    elif algo == "prd":
        np.testing.assert_array_equal(res, ref.values.astype(np.float32))
    else:
        np.testing.assert_array_equal(res, ref.values)
    assert st["span_chunks"] > 0 and st["span_link_bytes"] >= st["span_payload_bytes"] > 0
    assert any(i["mode"] == 3 for i in its)


@pytest.mark.parametrize("fv", [0, 1, 2])
@pytest.mark.parametrize("nbuf,xfer", [(0, 0), (3, 0), (2, 1), (4, 1)])
def test_bfs_fused_visit(asc, fv, nbuf, xfer):
    """ASCETIC_OPT_FUSED_VISIT: BFS's On-demand Computing done by the gather as the ids land (small-chunk
    pipeline with fv = 1, every gathered chunk with fv = 2) gives the same levels, records and bytes
    as the separate on-demand kernel (fv = 0). Small chunk caps give many chunks per level."""
    g = gg.rmat(13, seed=31)
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    asc.load_csr(g.off, g.nbr)
    asc.set_option("fused_visit", fv)
    asc.set_option("chunk_buffers", nbuf)
    asc.set_option("xfer_mode", xfer)
    asc.set_option("chunk_cap", 8192)
    asc.set_budget(g.csr_bytes // 4)
    p = oracle.placer(g.off, 4, g.csr_bytes // 4)
    ref = _oracle("bfs", g, src, p.s)
    for rep in range(2):
        asc.run("bfs", src)
        st, its = asc.stats()
        np.testing.assert_array_equal(asc.get_result(), ref.values)
        _check_records(its, ref)
        assert st["h2d_payload_bytes"] == ref.h2d_payload
    asc.set_option("fused_visit", 1)
    asc.set_option("chunk_buffers", 0)
    asc.set_option("xfer_mode", 0)
    asc.set_option("chunk_cap", 0)
