"""World-size-2 multi-process test of the partitioned (P > 1) path's host logic, on CPU.

Two processes (torch.distributed, gloo, 127.0.0.1) each take one 1D edge-balanced vertex
range from the library's own host partitioner (ascetic_partition) and place their Static
Region with the library's host placer (ascetic_place) under their own budget. They then
run the per-iteration protocol of SURVEY §8(e) — classify the OWNED active vertices, push
along owned out-lists, exchange (BFS: OR of next bitmaps by reduce-scatter-OR + all-gather; CC: MIN all-reduce
of labels; PR: SUM of dangling partials + all-gather of contrib slices; PRD: SUM of the
integer residual increments), finalize on the
replicated state — with numpy standing in for the kernels and gloo for NCCL. Per-rank
records and results must equal the oracle's multi-rank simulation and the P = 1 result.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
INF = 0xFFFFFFFF


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _runs(mask):
    return int(mask[0]) + int(np.count_nonzero(mask[1:] & ~mask[:-1])) if mask.size else 0


def _record(t, rank, A, stat, lo, hi, deg, b_e, digest):
    a = A[lo:hi]
    h = a & stat[lo:hi]
    m = a & ~stat[lo:hi]
    d = deg[lo:hi]
    return dict(t=t, rank=rank, nA=int(A.sum()), nH=int(h.sum()), nM=int(m.sum()), nruns=_runs(m),
                active_arcs=int(d[a].sum()), hit_arcs=int(d[h].sum()), miss_bytes=int(b_e * d[m].sum()),
                digest=digest, s=int(stat[lo:hi].sum()), swaps=0, replace_bytes=0)


def _or_allgather(mask):
    """The BFS exchange of Comm::or_words: reduce-scatter-OR of the 32-bit bitmap words by
    point-to-point slices (rank r owns words [r S, min((r+1) S, nw)), S = ceil(nw / P)), then an
    all-gather of the ORed slices padded to S words."""
    P, me = dist.get_world_size(), dist.get_rank()
    n = mask.size
    nw = (n + 31) // 32
    words = np.zeros(nw * 32, dtype=np.uint8)
    words[:n] = mask
    words = np.packbits(words.reshape(-1, 32)[:, ::-1], axis=1)[:, ::-1].copy().view(np.uint32).reshape(-1)
    S = (nw + P - 1) // P

    def ln(r):
        return 0 if r * S >= nw else min(S, nw - r * S)

    reqs, recv = [], {}
    for r in range(P):
        if r == me:
            continue
        if ln(r):
            reqs.append(dist.isend(torch.from_numpy(words[r * S: r * S + ln(r)].astype(np.int64)), r))
        if ln(me):
            recv[r] = torch.empty(ln(me), dtype=torch.int64)
            reqs.append(dist.irecv(recv[r], r))
    for rq in reqs:
        rq.wait()
    mine = words[me * S: me * S + ln(me)].astype(np.int64)
    for r, t in recv.items():
        mine |= t.numpy()
    pad = np.zeros(S, dtype=np.int64)
    pad[: ln(me)] = mine
    parts = [torch.empty(S, dtype=torch.int64) for _ in range(P)]
    dist.all_gather(parts, torch.from_numpy(pad))
    allw = np.concatenate([p.numpy() for p in parts])[:nw].astype(np.uint32)
    bits = np.unpackbits(allw.view(np.uint8).reshape(-1, 4)[:, ::-1], axis=1)[:, ::-1].reshape(-1)
    return bits[:n].astype(bool)


def _worker(rank, world, port, algo, q):
    import sys
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import graphgen as gg
        import oracle
        import paper_conf_icpp_tangzwgzwy21_b200 as asc
        g = gg.rmat(10, seed=17)
        n, off, nbr = g.n, g.off, g.nbr
        deg = np.diff(off.astype(np.int64))
        bounds = asc.partition(off, world)                   # the library's host partitioner
        lo, hi = int(bounds[rank]), int(bounds[rank + 1])
        budget = g.csr_bytes // 6
        pl = asc.place(off[lo:hi + 1], 4, budget, 0.5)       # the library's host placer, this rank's rows
        stat = np.zeros(n, dtype=bool)
        stat[lo:lo + pl["s"]] = True
        allstat = [None] * world
        dist.all_gather_object(allstat, stat)                # every rank's static set (for the oracle check)
        stat_all = np.logical_or.reduce(allstat)
        src_all = np.repeat(np.arange(n), deg)
        recs, t = [], 0
        if algo == "bfs":
            s = int(np.argmax(deg))
            level = np.full(n, INF, dtype=np.uint64)
            level[s] = 0
            A = np.zeros(n, dtype=bool); A[s] = True
            visited = A.copy()
            while A.any():
                recs.append(_record(t, rank, A, stat_all, lo, hi, deg, 4, oracle.digest(A)))
                own = np.zeros(n, dtype=bool); own[lo:hi] = A[lo:hi]
                sel = own[src_all]
                nxt = np.zeros(n, dtype=bool)
                nxt[nbr[sel]] = True
                nxt &= ~visited
                nxt = _or_allgather(nxt)                     # exchange: OR of next bitmaps
                visited |= nxt
                level[nxt] = t + 1
                A = nxt
                t += 1
            vals = level.astype(np.uint32)
        elif algo == "bfs_sparse":
            # BFS with the sparse exchange (d = 1): newly reached ids, all-gathered padded to the
            # largest count, when every rank has at most n / (64 P); else the bitmap OR
            s = int(np.argmax(deg))
            cap = max(1, n // (64 * world))
            level = np.full(n, INF, dtype=np.uint64)
            level[s] = 0
            A = np.zeros(n, dtype=bool); A[s] = True
            visited = A.copy()
            n_sparse = n_dense = 0
            while A.any():
                recs.append(_record(t, rank, A, stat_all, lo, hi, deg, 4, oracle.digest(A)))
                own = np.zeros(n, dtype=bool); own[lo:hi] = A[lo:hi]
                sel = own[src_all]
                nxt = np.zeros(n, dtype=bool)
                nxt[nbr[sel]] = True
                nxt &= ~visited
                ids = np.flatnonzero(nxt)
                cnt = torch.tensor([ids.size], dtype=torch.int64)
                cnts = [torch.zeros_like(cnt) for _ in range(world)]
                dist.all_gather(cnts, cnt)
                maxc = max(int(c.item()) for c in cnts)
                if maxc <= cap:
                    buf = torch.zeros(maxc, dtype=torch.int64)
                    buf[: ids.size] = torch.from_numpy(ids)
                    bufs = [torch.zeros_like(buf) for _ in range(world)]
                    dist.all_gather(bufs, buf)
                    for b_, c_ in zip(bufs, cnts):
                        nxt[b_[: int(c_.item())].numpy()] = True
                    n_sparse += 1
                else:
                    nxt = _or_allgather(nxt)
                    n_dense += 1
                visited |= nxt
                level[nxt] = t + 1
                A = nxt
                t += 1
            assert n_sparse >= 1 and n_dense >= 1, (n_sparse, n_dense)
            vals = level.astype(np.uint32)
        elif algo == "cc_sparse":
            # CC with the sparse MIN exchange (ASCETIC_OPT_SPARSE_EXCHANGE, d = 8): each rank's
            # lowered (id, label) pairs, all-gathered padded to the largest count and applied with
            # MIN, when every rank has at most n / (8 P) of them; else the dense MIN all-reduce
            s = 0
            cap = max(1, n // (8 * world))
            lab = np.arange(n, dtype=np.int64)
            A = np.ones(n, dtype=bool)
            n_sparse = n_dense = 0
            while A.any():
                recs.append(_record(t, rank, A, stat_all, lo, hi, deg, 4, oracle.digest(A)))
                snap = lab.copy()
                own = np.zeros(n, dtype=bool); own[lo:hi] = A[lo:hi]
                sel = own[src_all]
                np.minimum.at(lab, nbr[sel].astype(np.int64), snap[src_all[sel]])
                ids = np.flatnonzero(lab < snap)                 # this rank's next bits
                cnt = torch.tensor([ids.size], dtype=torch.int64)
                cnts = [torch.zeros_like(cnt) for _ in range(world)]
                dist.all_gather(cnts, cnt)
                maxc = max(int(c.item()) for c in cnts)
                if maxc <= cap:
                    buf = torch.zeros((maxc, 2), dtype=torch.int64)
                    buf[: ids.size, 0] = torch.from_numpy(ids)
                    buf[: ids.size, 1] = torch.from_numpy(lab[ids])
                    bufs = [torch.zeros_like(buf) for _ in range(world)]
                    dist.all_gather(bufs, buf)
                    nxt = np.zeros(n, dtype=bool)
                    nxt[ids] = True
                    for r_, (b_, c_) in enumerate(zip(bufs, cnts)):
                        if r_ == rank:
                            continue
                        pr = b_[: int(c_.item())].numpy()
                        np.minimum.at(lab, pr[:, 0], pr[:, 1])
                        nxt[pr[:, 0]] = True
                    A = nxt                                      # A_{t+1} = the merged next bits
                    n_sparse += 1
                else:
                    tl = torch.from_numpy(lab)
                    dist.all_reduce(tl, op=dist.ReduceOp.MIN)
                    lab = tl.numpy().copy()
                    A = lab < snap
                    n_dense += 1
                t += 1
            assert n_sparse >= 1 and n_dense >= 1, (n_sparse, n_dense)
            vals = lab.astype(np.uint32)
        elif algo == "cc":
            s = 0
            lab = np.arange(n, dtype=np.int64)
            A = np.ones(n, dtype=bool)
            while A.any():
                recs.append(_record(t, rank, A, stat_all, lo, hi, deg, 4, oracle.digest(A)))
                snap = lab.copy()
                own = np.zeros(n, dtype=bool); own[lo:hi] = A[lo:hi]
                sel = own[src_all]
                np.minimum.at(lab, nbr[sel].astype(np.int64), snap[src_all[sel]])
                tl = torch.from_numpy(lab)
                dist.all_reduce(tl, op=dist.ReduceOp.MIN)    # exchange: MIN of labels
                lab = tl.numpy().copy()
                A = lab < snap                               # A_{t+1} from the exchanged values
                t += 1
            vals = lab.astype(np.uint32)
        elif algo == "prd":
            # PageRank-delta (DESIGN R28-R30): integer residual increments, SUM all-reduce
            s = 0
            Q = 1 << 56
            res0 = (3 * Q) // (20 * n)
            tau = res0 * 10000 // 1000000
            r = np.zeros(n, dtype=np.uint64)
            res = np.full(n, res0, dtype=np.uint64)
            A = res > tau
            while A.any():
                recs.append(_record(t, rank, A, stat_all, lo, hi, deg, 4, oracle.digest(A)))
                r[A] += res[A]
                c = np.where(A & (deg > 0), (17 * res) // (20 * np.maximum(deg, 1).astype(np.uint64)), 0).astype(np.uint64)
                res[A] = 0
                own = np.zeros(n, dtype=bool); own[lo:hi] = A[lo:hi]
                sel = own[src_all]
                inc = np.zeros(n, dtype=np.uint64)
                np.add.at(inc, nbr[sel].astype(np.int64), c[src_all[sel]])
                ti = torch.from_numpy(inc.view(np.int64).copy())
                dist.all_reduce(ti)                          # exchange: SUM of the increments
                res += ti.numpy().view(np.uint64)
                A = res > tau
                t += 1
            vals = np.ldexp((r + res).astype(np.float64), -56)
        else:  # pr, pull
            s = 0
            iters = 6
            r = np.full(n, 1.0 / n)
            A = np.ones(n, dtype=bool)
            c = np.where(deg > 0, r / np.maximum(deg, 1), 0.0)
            dang = r[deg == 0].sum()
            for t in range(iters):
                recs.append(_record(t, rank, A, stat_all, lo, hi, deg, 4, oracle.digest(A)))
                sums = np.zeros(hi - lo)
                for v in range(lo, hi):
                    sums[v - lo] = c[nbr[off[v]:off[v + 1]]].sum()
                rn = 0.15 / n + 0.85 * (sums + dang / n)
                dpart = torch.tensor([rn[deg[lo:hi] == 0].sum()], dtype=torch.float64)
                dist.all_reduce(dpart)                       # exchange: SUM of dangling partials
                dang = float(dpart.item())
                cslice = np.where(deg[lo:hi] > 0, rn / np.maximum(deg[lo:hi], 1), 0.0)
                sl = [None] * world
                dist.all_gather_object(sl, (lo, cslice, rn))  # exchange: contrib slices
                for (a, cs, rr) in sl:
                    c[a:a + cs.size] = cs
                    r[a:a + cs.size] = rr
            vals = r
        out = [None] * world
        dist.all_gather_object(out, recs)
        if rank == 0:
            q.put(("ok", bounds.tolist(), pl, out, vals, int(s), stat_all))
    except Exception as e:  # surface worker failures
        q.put(("err", repr(e)))
        raise
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("algo", ["bfs", "bfs_sparse", "cc", "cc_sparse", "pr", "prd"])
def test_world2_gloo_protocol(algo):
    import graphgen as gg
    import oracle
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, algo, q)) for r in range(2)]
    for p in procs:
        p.start()
    msg = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
    assert msg[0] == "ok", msg
    _, bounds, pl, per_rank, vals, s, stat = msg
    g = gg.rmat(10, seed=17)
    assert bounds == oracle.partition(g.off, 2).tolist()
    o_pl = oracle.placer(g.off[bounds[0]:bounds[1] + 1] - g.off[bounds[0]], 4, g.csr_bytes // 6, 0.5)
    assert pl["s"] == o_pl.s and pl["static_bytes"] == o_pl.static_bytes and pl["cap"] == o_pl.cap
    iters = 6 if algo == "pr" else 0
    ref = oracle.run(algo.replace("_sparse", ""), g.off, g.nbr, src=s, max_iters=iters, is_static=stat.astype(np.uint8),
                     bounds=np.array(bounds, dtype=np.uint64))
    got = [rec for t in range(len(per_rank[0])) for rk in range(2) for rec in [per_rank[rk][t]]]
    assert got == ref.records
    if algo == "prd":
        np.testing.assert_array_equal(vals, ref.values)             # integer protocol: exact
    elif algo == "pr":
        np.testing.assert_allclose(vals, ref.values, rtol=1e-12)
    else:
        np.testing.assert_array_equal(vals, ref.values)
