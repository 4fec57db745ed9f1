"""Independent formulations used to PIN the oracle (never call oracle/ from here).

Each function restates a textbook / matrix-form definition, not the oracle's
frontier loop, so a dropped term, wrong index or transposed operand in
oracle.c shows up as a mismatch:
  * bfs_queue       — textbook queue BFS (levels = hop distance).
  * bf_dense        — Jacobi Bellman-Ford in matrix form over ALL vertices
                      (x_{t+1} = min(x_t, min_u x_t[u] + W[u, :])); its changed
                      set is the frontier the paper's push model activates
                      (P:650-652).
  * pr_dense        — PageRank power iteration as a dense matrix product.
  * runs_of         — maximal ID runs by a plain scan.
  * splitmix/digest — the digest written out with Python ints.
"""
from __future__ import annotations

from collections import deque

import numpy as np

INF = 0xFFFFFFFF
PHI = 0x9E3779B97F4A7C15
M64 = (1 << 64) - 1


def adjacency(off, ids):
    n = len(off) - 1
    return [list(map(int, ids[int(off[v]):int(off[v + 1])])) for v in range(n)]


def bfs_queue(adj, src):
    lev = [INF] * len(adj)
    lev[src] = 0
    q = deque([src])
    while q:
        u = q.popleft()
        for v in adj[u]:
            if lev[v] == INF:
                lev[v] = lev[u] + 1
                q.append(v)
    return np.array(lev, dtype=np.uint32)


def bf_dense(n, edges_w, init, max_rounds=None):
    """Jacobi relaxation in matrix form. edges_w: list of (u, v, w) arcs. init: initial x.
    Returns (final x, list of changed-sets per round, starting with the initial set)."""
    W = np.full((n, n), np.inf)
    for u, v, w in edges_w:
        W[u, v] = min(W[u, v], w)
    x = np.array([np.inf if a == INF else float(a) for a in init])
    sets = []
    cur = x.copy()
    # A_0 is given by the caller (source or all); rounds until no change
    r = 0
    while True:
        cand = np.min(cur[:, None] + W, axis=0) if n else cur
        nxt = np.minimum(cur, cand)
        changed = nxt < cur
        sets.append(changed)
        cur = nxt
        r += 1
        if not changed.any() or (max_rounds and r >= max_rounds):
            break
    out = np.array([INF if np.isinf(a) else int(a) for a in cur], dtype=np.uint32)
    return out, sets


def pr_dense(off, ids, iters, d=0.85):
    n = len(off) - 1
    A = np.zeros((n, n))  # A[v, u] = 1 for arc u->v (symmetric graphs: rows = lists)
    for u in range(n):
        for e in range(int(off[u]), int(off[u + 1])):
            A[int(ids[e]), u] += 1.0
    deg = np.diff(off.astype(np.int64)).astype(np.float64)
    r = np.full(n, 1.0 / n)
    for _ in range(iters):
        c = np.where(deg > 0, r / np.where(deg > 0, deg, 1.0), 0.0)
        dang = r[deg == 0].sum()
        r = (1 - d) / n + d * (A @ c + dang / n)
    return r


def runs_of(mask):
    runs, prev = 0, False
    for x in mask:
        if x and not prev:
            runs += 1
        prev = bool(x)
    return runs


def splitmix(z):
    z = (z + PHI) & M64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M64
    return z ^ (z >> 31)


def digest(active):
    n = len(active)
    s = 0
    for w in range((n + 31) // 32):
        word = 0
        for b in range(32):
            v = w * 32 + b
            if v < n and active[v]:
                word |= 1 << b
        s = (s + splitmix(w ^ ((word * PHI) & M64))) & M64
    return s


def records_from_sets(sets, off, b_e, s_static, rank_bounds=None):
    """Per-iteration records computed from explicit active sets (list of bool arrays)."""
    n = len(off) - 1
    deg = np.diff(off.astype(np.int64))
    st = np.zeros(n, dtype=bool)
    st[:s_static] = True
    bounds = [0, n] if rank_bounds is None else [int(x) for x in rank_bounds]
    out = []
    for t, A in enumerate(sets):
        A = np.asarray(A, dtype=bool)
        for g in range(len(bounds) - 1):
            lo, hi = bounds[g], bounds[g + 1]
            a = A[lo:hi]
            h = a & st[lo:hi]
            mm = a & ~st[lo:hi]
            out.append(dict(t=t, rank=g, nA=int(A.sum()), nH=int(h.sum()), nM=int(mm.sum()),
                            nruns=runs_of(mm), active_arcs=int(deg[lo:hi][a].sum()),
                            hit_arcs=int(deg[lo:hi][h].sum()), miss_bytes=int(b_e * deg[lo:hi][mm].sum()),
                            digest=digest(A), s=int(st[lo:hi].sum()), swaps=0, replace_bytes=0))
    return out
