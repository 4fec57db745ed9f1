"""CPU ORACLE for the Ascetic hot path — TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
legs may import this package. The product path (paper_conf_icpp_tangzwgzwy21_b200)
never imports it and shares no code with it (see oracle.c's header for the paper
passages each function follows; DESIGN.md §"Readings" lists the interpretations).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

BFS, SSSP, CC, PR, PRD = 0, 1, 2, 3, 4
ALGOS = {"bfs": BFS, "sssp": SSSP, "cc": CC, "pr": PR, "prd": PRD}
INF = 0xFFFFFFFF


class _Place(ctypes.Structure):
    _fields_ = [("R", ctypes.c_double), ("D", ctypes.c_uint64), ("B", ctypes.c_uint64),
                ("Ms", ctypes.c_uint64), ("s", ctypes.c_uint64), ("static_bytes", ctypes.c_uint64),
                ("C", ctypes.c_uint64), ("cap", ctypes.c_uint64)]


class _Iter(ctypes.Structure):
    _fields_ = [("t", ctypes.c_uint32), ("rank", ctypes.c_uint32), ("nA", ctypes.c_uint64),
                ("nH", ctypes.c_uint64), ("nM", ctypes.c_uint64), ("nruns", ctypes.c_uint64),
                ("active_arcs", ctypes.c_uint64), ("hit_arcs", ctypes.c_uint64),
                ("miss_bytes", ctypes.c_uint64), ("digest", ctypes.c_uint64), ("s", ctypes.c_uint64),
                ("swaps", ctypes.c_uint64), ("replace_bytes", ctypes.c_uint64)]


class _Summary(ctypes.Structure):
    _fields_ = [("iterations", ctypes.c_uint32), ("nrec", ctypes.c_uint32),
                ("h2d_payload", ctypes.c_uint64), ("active_arcs_total", ctypes.c_uint64),
                ("h2d_replace", ctypes.c_uint64)]


ITER_FIELDS = ["t", "rank", "nA", "nH", "nM", "nruns", "active_arcs", "hit_arcs", "miss_bytes", "digest", "s",
               "swaps", "replace_bytes"]


def build(force: bool = False) -> str:
    """Compile the oracle (building the checker is not using it)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-shared", "-fPIC", "-o", _LIB, _SRC, "-lm"])
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        lib.or_placer.argtypes = [ctypes.c_uint64, ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64,
                                  ctypes.c_double, ctypes.POINTER(_Place)]
        lib.or_partition.argtypes = [ctypes.c_uint64, ctypes.c_void_p, ctypes.c_uint32, ctypes.c_void_p]
        lib.or_digest.restype = ctypes.c_uint64
        lib.or_digest.argtypes = [ctypes.c_uint64, ctypes.c_void_p]
        lib.or_run_ex.argtypes = [ctypes.c_int, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint32,
                                  ctypes.c_uint32, ctypes.c_void_p, ctypes.c_uint32, ctypes.c_void_p,
                                  ctypes.c_void_p, ctypes.c_void_p, ctypes.POINTER(_Iter), ctypes.c_uint32,
                                  ctypes.POINTER(_Summary), ctypes.c_int, ctypes.c_uint64, ctypes.c_uint64,
                                  ctypes.POINTER(ctypes.c_uint64)]
        lib.or_run_hot.argtypes = [ctypes.c_int, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint32,
                                   ctypes.c_uint32, ctypes.c_uint32, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                   ctypes.POINTER(_Iter), ctypes.c_uint32, ctypes.POINTER(_Summary), ctypes.c_void_p,
                                   ctypes.c_uint32, ctypes.c_int, ctypes.c_int, ctypes.c_uint64]
        lib.or_random_chunks.argtypes = [ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_void_p]
        lib.or_set_prd_tol.argtypes = [ctypes.c_uint64]
        lib.or_threads.restype = ctypes.c_int
        lib.or_set_threads.argtypes = [ctypes.c_int]
        lib.or_classify.argtypes = [ctypes.c_uint64, ctypes.c_void_p, ctypes.c_uint32, ctypes.c_void_p, ctypes.c_void_p,
                                    ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                    ctypes.c_void_p, ctypes.c_void_p]
        _lib = lib
    return _lib


def threads() -> int:
    return int(_load().or_threads())


def set_threads(k: int) -> None:
    """OpenMP threads of the following runs (timing only; results do not depend on it except the
    fp64 summation order of PR's dangling mass)."""
    _load().or_set_threads(int(k))


@dataclass
class Placement:
    R: float
    D: int
    B: int
    Ms: int
    s: int
    static_bytes: int
    C: int
    cap: int


def placer(off: np.ndarray, b_e: int, budget: int, frac: float = -1.0) -> Placement:
    lib = _load()
    off = np.ascontiguousarray(off, dtype=np.uint64)
    p = _Place()
    lib.or_placer(off.size - 1, off.ctypes.data, b_e, budget, frac, ctypes.byref(p))
    return Placement(p.R, p.D, p.B, p.Ms, p.s, p.static_bytes, p.C, p.cap)


def rear_start(off: np.ndarray, b_e: int, Ms: int) -> int:
    """First vertex of the rear (suffix) static set placed in Ms bytes."""
    lib = _load()
    lib.or_rear_start.restype = ctypes.c_uint64
    lib.or_rear_start.argtypes = [ctypes.c_uint64, ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64]
    off = np.ascontiguousarray(off, dtype=np.uint64)
    return int(lib.or_rear_start(off.size - 1, off.ctypes.data, b_e, Ms))


def static_rear(n: int, s_lo: int) -> np.ndarray:
    st = np.zeros(n, dtype=np.uint8)
    st[s_lo:] = 1
    return st


def partition(off: np.ndarray, P: int) -> np.ndarray:
    lib = _load()
    off = np.ascontiguousarray(off, dtype=np.uint64)
    b = np.zeros(P + 1, dtype=np.uint64)
    lib.or_partition(off.size - 1, off.ctypes.data, P, b.ctypes.data)
    return b


def classify(off: np.ndarray, b_e: int, active: np.ndarray, is_static: np.ndarray) -> dict:
    """StaticNodes, On-demandNodes and the on-demand request's runs + byte offsets (Fig. 4)."""
    lib = _load()
    off = np.ascontiguousarray(off, dtype=np.uint64)
    n = off.size - 1
    a = np.ascontiguousarray(active, dtype=np.uint8)
    s = np.ascontiguousarray(is_static, dtype=np.uint8)
    hits = np.zeros(max(n, 1), dtype=np.uint32)
    misses = np.zeros(max(n, 1), dtype=np.uint32)
    rb = np.zeros(max(n, 1), dtype=np.uint32)
    re = np.zeros(max(n, 1), dtype=np.uint32)
    rd = np.zeros(max(n, 1), dtype=np.uint64)
    out = np.zeros(3, dtype=np.uint64)
    lib.or_classify(n, off.ctypes.data, b_e, a.ctypes.data, s.ctypes.data, hits.ctypes.data, misses.ctypes.data,
                    rb.ctypes.data, re.ctypes.data, rd.ctypes.data, out.ctypes.data)
    nh, nm, nr = (int(x) for x in out)
    return dict(hits=hits[:nh].copy(), misses=misses[:nm].copy(), run_b=rb[:nr].copy(), run_e=re[:nr].copy(),
                run_dst=rd[:nr].copy())


def digest(active: np.ndarray) -> int:
    a = np.ascontiguousarray(active, dtype=np.uint8)
    return int(_load().or_digest(a.size, a.ctypes.data))


@dataclass
class Result:
    values: np.ndarray          # uint32 levels/dists/labels, or float64 ranks
    iterations: int
    records: list[dict]
    h2d_payload: int
    active_arcs_total: int
    repartitions: int = 0
    replace_bytes: int = 0      # §3.4 swap bytes (run_hot)


def static_prefix(n: int, s: int) -> np.ndarray:
    st = np.zeros(n, dtype=np.uint8)
    st[:s] = 1
    return st


def run(algo: str | int, off: np.ndarray, nbr: np.ndarray, src: int = 0, max_iters: int = 0,
        is_static: np.ndarray | None = None, bounds: np.ndarray | None = None,
        eq3_budget: int = 0, eq3_ms: int = 0) -> Result:
    """Run the oracle. nbr = ids (bfs/cc/pr) or interleaved (id,w) pairs (sssp).
    eq3_budget > 0 applies the Eq. 3 re-partition (one rank; is_static = the front prefix placed
    in eq3_ms bytes of the budget)."""
    lib = _load()
    a = ALGOS[algo] if isinstance(algo, str) else algo
    off = np.ascontiguousarray(off, dtype=np.uint64)
    nbr = np.ascontiguousarray(nbr, dtype=np.uint32)
    n = off.size - 1
    st = np.zeros(n, dtype=np.uint8) if is_static is None else np.ascontiguousarray(is_static, dtype=np.uint8)
    P = 1 if bounds is None else len(bounds) - 1
    b = None if bounds is None else np.ascontiguousarray(bounds, dtype=np.uint64)
    res_u = np.zeros(max(n, 1), dtype=np.uint32)[:n]
    res_f = np.zeros(max(n, 1), dtype=np.float64)[:n]
    cap = (min(n + 2, 1 << 16) if a != PR else max(1, max_iters)) * P
    recs = (_Iter * cap)()
    s = _Summary()
    reparts = ctypes.c_uint64(0)
    rc = lib.or_run_ex(a, n, off.ctypes.data, nbr.ctypes.data if nbr.size else None, src, max_iters,
                       st.ctypes.data if n else None, P, b.ctypes.data if b is not None else None,
                       res_u.ctypes.data if n else None, res_f.ctypes.data if n else None, recs, cap, ctypes.byref(s),
                       1 if eq3_budget > 0 else 0, eq3_budget, eq3_ms, ctypes.byref(reparts))
    if rc != 0:
        raise ValueError(f"oracle rejected arguments (rc={rc})")
    records = [{f: int(getattr(recs[i], f)) for f in ITER_FIELDS} for i in range(s.nrec)]
    vals = res_f.copy() if a in (PR, PRD) else res_u.copy()
    return Result(vals, int(s.iterations), records, int(s.h2d_payload), int(s.active_arcs_total),
                  int(reparts.value))


def run_hot(algo: str | int, off: np.ndarray, nbr: np.ndarray, static_bytes, src: int = 0, max_iters: int = 0,
            kswap: int = 0, policy: str | None = None, bounds: np.ndarray | None = None,
            random_seed: int | None = None) -> Result:
    """Run with the §3.4 data replacement: 16 KiB chunks, hotness counters, up to
    `kswap` chunk swaps per iteration and rank. static_bytes = Ms (int, or one per rank).
    policy: "cumulative" (default for bfs/sssp/cc) or "last" (default for pr).
    random_seed: start from the seeded random chunk set (§5 random initial content) instead of the front."""
    lib = _load()
    a = ALGOS[algo] if isinstance(algo, str) else algo
    if policy is None:
        policy = "last" if a == PR else "cumulative"
    if policy not in ("cumulative", "last"):
        raise ValueError(policy)
    off = np.ascontiguousarray(off, dtype=np.uint64)
    nbr = np.ascontiguousarray(nbr, dtype=np.uint32)
    n = off.size - 1
    P = 1 if bounds is None else len(bounds) - 1
    b = None if bounds is None else np.ascontiguousarray(bounds, dtype=np.uint64)
    ms = np.ascontiguousarray(np.broadcast_to(np.asarray(static_bytes, dtype=np.uint64), (P,)), dtype=np.uint64)
    res_u = np.zeros(max(n, 1), dtype=np.uint32)[:n]
    res_f = np.zeros(max(n, 1), dtype=np.float64)[:n]
    cap = (min(n + 2, 1 << 16) if a != PR else max(1, max_iters)) * P
    recs = (_Iter * cap)()
    s = _Summary()
    rc = lib.or_run_hot(a, n, off.ctypes.data, nbr.ctypes.data if nbr.size else None, src, max_iters, P,
                        b.ctypes.data if b is not None else None, res_u.ctypes.data if n else None,
                        res_f.ctypes.data if n else None, recs, cap, ctypes.byref(s), ms.ctypes.data, kswap,
                        1 if policy == "cumulative" else 0, 0 if random_seed is None else 1,
                        0 if random_seed is None else int(random_seed))
    if rc != 0:
        raise ValueError(f"oracle rejected arguments (rc={rc})")
    records = [{f: int(getattr(recs[i], f)) for f in ITER_FIELDS} for i in range(s.nrec)]
    vals = res_f.copy() if a in (PR, PRD) else res_u.copy()
    return Result(vals, int(s.iterations), records, int(s.h2d_payload), int(s.active_arcs_total), 0,
                  int(s.h2d_replace))


def random_chunks(nc: int, ns: int, seed: int) -> np.ndarray:
    """Resident flags of the seeded random initial Static Region (ns of nc 16 KiB chunks)."""
    res = np.zeros(max(nc, 1), dtype=np.uint8)
    _load().or_random_chunks(nc, ns, seed, res.ctypes.data)
    return res[:nc].astype(bool)


def set_prd_tol(ppm: int) -> None:
    """PageRank-delta threshold tau = floor(res0 * ppm / 1e6), res0 = floor(3 * 2^56 / (20 n))."""
    _load().or_set_prd_tol(int(ppm))
