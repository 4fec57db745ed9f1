"""The NCCL back end on one GPU: ascetic_comm_init(rank 0, world 1, unique id) builds a one-rank
NCCL communicator, so every exchange step of the multi-GPU path (the bitmap
all-gather + OR, the MIN all-reduce, the fp64 SUM + slice broadcasts of PR, the u64 SUM of
PRD, the stream-ordered barriers and the CUDA-IPC handle all-gather of the fused exchange)
runs through the dlopen'ed libnccl instead of the emulation. With one rank the exchange is an
identity, so results, per-iteration records and bytes must equal the oracle's single-GPU run."""
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
    m.emulate_ranks(1)
    m.comm_init(0, 1, m.get_unique_id(), 0)
    yield m
    m.unload()
    m.comm_init(0, 1, None, 0)          # no id: drops the communicator


@pytest.mark.parametrize("fused", [0, 1])
@pytest.mark.parametrize("algo", ["bfs", "sssp", "cc", "pr", "prd"])
def test_nccl_one_rank_matches_oracle(asc, algo, fused):
    g = gg.rmat(12, seed=37, weights=(algo == "sssp"))
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    budget = g.csr_bytes // 4
    iters = 6 if algo == "pr" else 0
    asc.load_csr(g.off, g.nbr, pairs=g.pairs, symmetric=True)
    asc.set_option("fused_exchange", fused)
    asc.set_option("chunk_cap", 4096)
    try:
        asc.set_budget(budget, 0.4)
        p = oracle.placer(g.off, g.b_e, budget, 0.4)
        ref = oracle.run(algo, g.off, g.nbr, src=src, max_iters=iters, is_static=oracle.static_prefix(g.n, p.s))
        for rep in range(2):                 # the second run reuses the communicator, IPC maps, buffers
            asc.run(algo, src, iters)
            st, its = asc.stats()
            res = asc.get_result().copy()
            assert st["world"] == 1 and st["iterations"] == ref.iterations
            if algo == "pr":
                rel = np.abs(res.astype(np.float64) - ref.values) / ref.values
                assert rel.max() <= 1e-5 and np.abs(res.astype(np.float64) - ref.values).sum() <= 1e-6
            else:
                exp = ref.values.astype(np.float32) if algo == "prd" else ref.values
                np.testing.assert_array_equal(res, exp)
            assert [{f: i[f] for f in REC} for i in its] == [{f: r[f] for f in REC} for r in ref.records]
            assert st["h2d_payload_bytes"] == ref.h2d_payload
    finally:
        asc.set_option("fused_exchange", 0)
        asc.set_option("chunk_cap", 0)


def test_nccl_one_rank_reload_reopens_peers(asc):
    """A new graph shape re-allocates every buffer; the fused exchange must re-map (all-gather
    fresh IPC handles), not reuse mappings of freed allocations."""
    asc.set_option("fused_exchange", 1)
    try:
        for scale, seed in [(10, 41), (12, 42), (11, 43)]:
            g = gg.rmat(scale, seed=seed)
            asc.load_csr(g.off, g.nbr, symmetric=True)
            asc.set_budget(g.csr_bytes // 3, -1.0)
            asc.run("cc")
            p = oracle.placer(g.off, 4, g.csr_bytes // 3)
            ref = oracle.run("cc", g.off, g.nbr, is_static=oracle.static_prefix(g.n, p.s))
            np.testing.assert_array_equal(asc.get_result(), ref.values)
    finally:
        asc.set_option("fused_exchange", 0)


@pytest.mark.parametrize("algo", ["bfs", "sssp", "cc"])
def test_nccl_one_rank_sparse_exchange(asc, algo):
    """ASCETIC_OPT_SPARSE_EXCHANGE through libnccl: the count and pair all-gathers run on the
    one-rank communicator (nothing foreign to apply), the finalize takes the merged next bitmap."""
    g = gg.rmat(12, seed=39, weights=(algo == "sssp"))
    src = int(np.argmax(np.diff(g.off.astype(np.int64))))
    budget = g.csr_bytes // 4
    asc.load_csr(g.off, g.nbr, pairs=g.pairs, symmetric=True)
    asc.set_option("sparse_exchange", 1)
    asc.set_option("chunk_cap", 4096)
    try:
        asc.set_budget(budget, 0.4)
        p = oracle.placer(g.off, g.b_e, budget, 0.4)
        ref = oracle.run(algo, g.off, g.nbr, src=src, is_static=oracle.static_prefix(g.n, p.s))
        asc.run(algo, src)
        st, its = asc.stats()
        assert st["world"] == 1 and st["sparse_exchanges"] >= 1
        np.testing.assert_array_equal(asc.get_result(), ref.values)
        assert [{f: i[f] for f in REC} for i in its] == [{f: r[f] for f in REC} for r in ref.records]
    finally:
        asc.set_option("sparse_exchange", 0)
        asc.set_option("chunk_cap", 0)
