"""Seeded synthetic graph inputs (INPUT ONLY — no method arithmetic).

Shared by the CUDA path's tests/bench and by the oracle's tests, as the task
allows for seeded input generators. The recipes follow SURVEY.md §8(d) and are
restated in DESIGN.md ("Input recipe"): RMAT (a,b,c,d)=(0.57,0.19,0.19,0.05),
"RMAT-rand" permutation (Table 3), symmetrized, self-loops and
duplicates removed; SSSP weights uniform in 1..64 (PAPER.md P:993-995 names an
extra weight field; the distribution is SURVEY Q12's reading).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "graphgen.c")
_LIB = os.path.join(_HERE, "libgraphgen.so")
_lib = None


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O3", "-march=x86-64-v2", "-fopenmp", "-shared", "-fPIC",
                               "-o", _LIB, _SRC])
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        lib.gg_rmat_build.restype = ctypes.c_void_p
        lib.gg_rmat_build.argtypes = [ctypes.c_int, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint64,
                                      ctypes.c_int, ctypes.c_double, ctypes.c_double, ctypes.c_double]
        lib.gg_from_edges.restype = ctypes.c_void_p
        lib.gg_from_edges.argtypes = [ctypes.c_uint32, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_void_p,
                                      ctypes.c_int, ctypes.c_int]
        lib.gg_size.argtypes = [ctypes.c_void_p, ctypes.POINTER(ctypes.c_uint32), ctypes.POINTER(ctypes.c_uint64)]
        lib.gg_export.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                  ctypes.c_int, ctypes.c_uint64]
        lib.gg_free.argtypes = [ctypes.c_void_p]
        lib.gg_threads.restype = ctypes.c_int
        _lib = lib
    return _lib


@dataclass
class Graph:
    """CSR graph: off uint64[n+1], nbr uint32[m] (or [2m] interleaved (id,w) when pairs)."""
    n: int
    m: int
    off: np.ndarray
    nbr: np.ndarray
    pairs: bool = False
    name: str = ""

    @property
    def b_e(self) -> int:
        return 8 if self.pairs else 4

    @property
    def csr_bytes(self) -> int:
        """Edge payload + offsets (the 'CSR bytes' a percentage budget refers to)."""
        return self.b_e * self.m + 8 * (self.n + 1)

    def ids(self) -> np.ndarray:
        return self.nbr[0::2] if self.pairs else self.nbr

    def weights(self) -> np.ndarray:
        if not self.pairs:
            raise ValueError("graph has no weights")
        return self.nbr[1::2]


def _export(h, pairs: bool, wseed: int, name: str, alloc=None) -> Graph:
    """alloc(count, dtype) -> numpy array lets callers place the offsets and arcs (e.g. in pinned memory)."""
    lib = _load()
    n = ctypes.c_uint32()
    m = ctypes.c_uint64()
    lib.gg_size(h, ctypes.byref(n), ctypes.byref(m))
    off = (alloc(n.value + 1, np.uint64) if alloc is not None else np.empty(n.value + 1, dtype=np.uint64))[:n.value + 1]
    cnt = (2 if pairs else 1) * m.value
    nbr = (alloc(cnt, np.uint32) if alloc is not None else np.empty(max(1, cnt), dtype=np.uint32))[:cnt]
    lib.gg_export(h, off.ctypes.data, nbr.ctypes.data if nbr.size else None, None, 1 if pairs else 0, wseed)
    lib.gg_free(h)
    return Graph(n=n.value, m=m.value, off=off, nbr=nbr, pairs=pairs, name=name)


def rmat(scale: int, tuples: int | None = None, seed: int = 1, permute: bool = True, n: int = 0,
         weights: bool = False, abc=(0.57, 0.19, 0.19), name: str = "", alloc=None) -> Graph:
    """RMAT graph, symmetrized + deduplicated. `n` > 0 rejects endpoints >= n (exact n)."""
    lib = _load()
    if tuples is None:
        tuples = 16 << scale
    h = lib.gg_rmat_build(scale, tuples, n, seed, 1 if permute else 0, abc[0], abc[1], abc[2])
    if not h:
        raise ValueError("bad rmat parameters")
    return _export(h, weights, seed, name or f"rmat{scale}", alloc)


def from_edges(n: int, src, dst, symmetrize: bool = True, weights: bool = False, seed: int = 1,
               keep_dups: bool = False, name: str = "edges") -> Graph:
    lib = _load()
    src = np.ascontiguousarray(src, dtype=np.uint32)
    dst = np.ascontiguousarray(dst, dtype=np.uint32)
    h = lib.gg_from_edges(n, src.size, src.ctypes.data if src.size else None,
                          dst.ctypes.data if dst.size else None, 1 if symmetrize else 0, 1 if keep_dups else 0)
    return _export(h, weights, seed, name)


def random_graph(n: int, ne: int, seed: int, weights: bool = False) -> Graph:
    """Uniform random symmetric simple graph with ~ne undirected tuples (tests)."""
    rng = np.random.default_rng(seed)
    src = rng.integers(0, max(n, 1), size=ne, dtype=np.uint64).astype(np.uint32)
    dst = rng.integers(0, max(n, 1), size=ne, dtype=np.uint64).astype(np.uint32)
    return from_edges(n, src, dst, symmetrize=True, weights=weights, seed=seed, name=f"rand{n}")


# ---- the BASELINE.json configs as concrete inputs ----
CONFIGS = {
    "c1": dict(algo="bfs", scale=16, tuples=16 << 16, n=0, permute=True, seed=1, budget_frac=0.25,
               desc="BFS on RMAT scale-16, budget 25% of CSR bytes"),
    "c2": dict(algo="sssp", scale=24, tuples=16 << 24, n=0, permute=True, seed=2, budget_frac=0.50,
               desc="SSSP (w in 1..64) on RMAT scale-24, budget 50% of CSR bytes"),
    "c3": dict(algo="pr", scale=26, tuples=1_806_067_135, n=65_608_366, permute=True, seed=3,
               budget_bytes=11 * 10**9, iters=43,
               desc="PageRank 43 iterations on a friendster-shaped graph, 11 GB budget"),
    "c4": dict(algo="cc", scale=27, tuples=3_300_000_000, n=105_000_000, permute=False, seed=4,
               budget_frac=0.30, desc="CC on a uk-2007-shaped graph, budget 30% of CSR bytes"),
    "c5": dict(algo="bfs+pr", scale=29, tuples=16 << 29, n=0, permute=True, seed=5,
               budget_bytes=40 * 10**9, desc="BFS + PR on RMAT scale-29, 40 GB per GPU"),
}


def config_graph(key: str, scale_override: int | None = None, alloc=None) -> Graph:
    c = CONFIGS[key]
    scale = scale_override or c["scale"]
    tuples = c["tuples"] if scale_override is None else (16 << scale)
    n = c["n"] if scale_override is None else 0
    return rmat(scale, tuples, seed=c["seed"], permute=c["permute"], n=n,
                weights=(c["algo"] == "sssp"), name=key, alloc=alloc)


def config_budget(key: str, g: Graph) -> int:
    c = CONFIGS[key]
    if "budget_bytes" in c:
        return int(c["budget_bytes"])
    return int(c["budget_frac"] * g.csr_bytes)


def sources(g: Graph, count: int, seed: int) -> list[int]:
    """Seeded BFS/SSSP sources with deg > 0."""
    deg = np.diff(g.off.astype(np.int64))
    cand = np.nonzero(deg > 0)[0]
    if cand.size == 0:
        return [0] * count
    rng = np.random.default_rng(seed)
    return [int(x) for x in rng.choice(cand, size=count, replace=True)]


def threads() -> int:
    return int(_load().gg_threads())
