"""ascetic-b200: B200-native hot path of Ascetic (Tang et al., ICPP '21).

Thin ctypes binding over libascetic.so (include/ascetic.h). Argument marshalling only:
every step of the path (classification, compaction, transfer, edge kernels, finalize)
runs in the library's sm_100a kernels. There is NO CPU fallback: importing this package
without the built library raises.

    import paper_conf_icpp_tangzwgzwy21_b200 as asc
    asc.load_csr(off, nbr, symmetric=True)        # host CSR (uint64 off, uint32 nbr)
    asc.set_budget(bytes, static_fraction=-1.0)   # Eq. 2 split
    asc.run("bfs", source=0)                      # or "sssp", "cc", "pr"
    st, iters = asc.stats()
    levels = asc.get_result()
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libascetic.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is not built; run `python -c 'import __graft_entry__ as g; g.build()'` "
                      "(there is no CPU fallback)")

_lib = ctypes.CDLL(LIB_PATH)

OK, EINVAL, ESTATE, ENOMEM, EHOSTMEM, ECUDA, ENCCL, EUNSUPPORTED = 0, -1, -2, -3, -4, -5, -6, -7
STATUS = {0: "OK", -1: "EINVAL", -2: "ESTATE", -3: "ENOMEM", -4: "EHOSTMEM", -5: "ECUDA", -6: "ENCCL",
          -7: "EUNSUPPORTED"}
ALGOS = {"bfs": 0, "sssp": 1, "cc": 2, "pr": 3, "prd": 4}
SYMMETRIC, COPY, VALIDATE, PAIRS, SORTED = 1, 2, 4, 8, 16
OPTIONS = {"chunk_cap": 1, "xfer_mode": 2, "dma_min_run": 3, "overlap": 4, "keep_static": 5,
           "hub_degree": 6, "timing": 7, "gather_ctas": 8, "chunk_buffers": 9, "static_ctas_per_sm": 10,
           "prefetch": 11, "repartition": 12, "static_placement": 13, "replace_chunks": 14,
           "replace_policy": 15, "placement_seed": 16, "prd_tol_ppm": 17,
           "fused_exchange": 18, "sparse_exchange": 19, "relax_mode": 20,
           "ce_min_run": 21, "gap_bridge": 22, "pr_segment": 23,
           "span_density": 24, "span_max_ratio": 25,
           "fused_visit": 26}
INF = 0xFFFFFFFF


class Stats(ctypes.Structure):
    _fields_ = [("algo", ctypes.c_int32), ("iterations", ctypes.c_uint32),
                ("n", ctypes.c_uint64), ("m", ctypes.c_uint64), ("b_e", ctypes.c_uint32),
                ("rank", ctypes.c_uint32), ("world", ctypes.c_uint32),
                ("s", ctypes.c_uint64), ("budget_bytes", ctypes.c_uint64), ("static_reserved", ctypes.c_uint64),
                ("static_bytes", ctypes.c_uint64), ("ondemand_bytes", ctypes.c_uint64),
                ("chunk_cap", ctypes.c_uint64), ("static_fraction_used", ctypes.c_double),
                ("h2d_payload_bytes", ctypes.c_uint64), ("h2d_static_fill_bytes", ctypes.c_uint64),
                ("h2d_other_bytes", ctypes.c_uint64), ("d2h_bytes", ctypes.c_uint64),
                ("active_arcs_total", ctypes.c_uint64), ("chunks_total", ctypes.c_uint64),
                ("dma_chunks", ctypes.c_uint64), ("gather_chunks", ctypes.c_uint64),
                ("time_run_s", ctypes.c_double), ("time_fill_s", ctypes.c_double),
                ("time_h2d_busy_s", ctypes.c_double), ("gteps", ctypes.c_double),
                ("gteps_excl_fill", ctypes.c_double), ("vertex_state_bytes", ctypes.c_uint64),
                ("kernel_launches", ctypes.c_uint64), ("time_classify_s", ctypes.c_double),
                ("time_static_s", ctypes.c_double), ("static_arcs", ctypes.c_uint64),
                ("time_ondemand_s", ctypes.c_double), ("ondemand_arcs", ctypes.c_uint64),
                ("time_gather_s", ctypes.c_double), ("gather_bytes", ctypes.c_uint64),
                ("time_dma_s", ctypes.c_double), ("dma_bytes", ctypes.c_uint64),
                ("time_finalize_s", ctypes.c_double), ("time_host_s", ctypes.c_double),
                ("repartitions", ctypes.c_uint64), ("h2d_replace_bytes", ctypes.c_uint64),
                ("swaps_total", ctypes.c_uint64), ("time_replace_s", ctypes.c_double),
                ("sparse_exchanges", ctypes.c_uint64), ("sparse_exchange_bytes", ctypes.c_uint64),
                ("chunk_buffers", ctypes.c_uint32), ("reserved0", ctypes.c_uint32),
                ("gather_ce_bytes", ctypes.c_uint64), ("gather_load_bytes", ctypes.c_uint64),
                ("pr_segment_passes", ctypes.c_uint64), ("span_chunks", ctypes.c_uint64),
                ("span_link_bytes", ctypes.c_uint64), ("span_payload_bytes", ctypes.c_uint64)]


class IterStats(ctypes.Structure):
    _fields_ = [("t", ctypes.c_uint32), ("rank", ctypes.c_uint32),
                ("nA", ctypes.c_uint64), ("nH", ctypes.c_uint64), ("nM", ctypes.c_uint64), ("nruns", ctypes.c_uint64),
                ("active_arcs", ctypes.c_uint64), ("hit_arcs", ctypes.c_uint64), ("miss_bytes", ctypes.c_uint64),
                ("digest", ctypes.c_uint64), ("chunks", ctypes.c_uint32), ("mode", ctypes.c_uint32),
                ("ms_classify", ctypes.c_float), ("ms_static", ctypes.c_float), ("ms_ondemand", ctypes.c_float),
                ("ms_h2d", ctypes.c_float), ("ms_finalize", ctypes.c_float), ("ms_exchange", ctypes.c_float),
                ("ms_total", ctypes.c_float), ("ms_link_head", ctypes.c_float), ("ms_link_gaps", ctypes.c_float),
                ("ms_link_tail", ctypes.c_float), ("s_static", ctypes.c_uint64), ("swaps", ctypes.c_uint64),
                ("replace_bytes", ctypes.c_uint64)]


_lib.ascetic_load_csr.argtypes = [ctypes.c_uint64, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_void_p,
                                  ctypes.c_void_p, ctypes.c_uint32]
_lib.ascetic_set_budget.argtypes = [ctypes.c_uint64, ctypes.c_double]
_lib.ascetic_set_option.argtypes = [ctypes.c_int, ctypes.c_int64]
_lib.ascetic_run.argtypes = [ctypes.c_int, ctypes.c_uint32, ctypes.c_uint32]
_lib.ascetic_stats.argtypes = [ctypes.POINTER(Stats), ctypes.POINTER(IterStats), ctypes.c_uint32]
_lib.ascetic_get_result.argtypes = [ctypes.c_void_p, ctypes.c_uint64]
_lib.ascetic_get_unique_id.argtypes = [ctypes.c_void_p]
_lib.ascetic_comm_init.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_int]
_lib.ascetic_set_device.argtypes = [ctypes.c_int]
_lib.ascetic_unload.restype = None
_lib.ascetic_last_error.restype = ctypes.c_char_p
_lib.ascetic_version.restype = ctypes.c_char_p

EXPORTS = ["ascetic_load_csr", "ascetic_set_budget", "ascetic_set_option", "ascetic_run", "ascetic_stats",
           "ascetic_get_result", "ascetic_get_unique_id", "ascetic_comm_init", "ascetic_set_device",
           "ascetic_unload", "ascetic_last_error", "ascetic_version"]


class AsceticError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"{STATUS.get(code, code)}: {msg}")
        self.code = code


def _check(rc: int) -> int:
    if rc < 0:
        raise AsceticError(rc, _lib.ascetic_last_error().decode())
    return rc


# keep host arrays alive while the library pins them in place
_keep: dict = {}


def version() -> str:
    return _lib.ascetic_version().decode()


def set_device(device: int) -> None:
    _check(_lib.ascetic_set_device(device))


def load_csr(off: np.ndarray, nbr: np.ndarray, wgt: np.ndarray | None = None, *, symmetric: bool = True,
             pairs: bool = False, copy: bool = False, validate: bool = False, sorted_rows: bool = False) -> None:
    """off: uint64[n+1]; nbr: uint32[m] (or [2m] (id,w) pairs with pairs=True); wgt: uint32[m] or None.
    sorted_rows asserts ascending neighbour ids in every row (ASCETIC_SORTED)."""
    if off.dtype != np.uint64 or not off.flags.c_contiguous:
        raise TypeError("off must be a C-contiguous uint64 array")
    if nbr.dtype != np.uint32 or not nbr.flags.c_contiguous:
        raise TypeError("nbr must be a C-contiguous uint32 array")
    n = off.size - 1
    m = nbr.size // 2 if pairs else nbr.size
    flags = (SYMMETRIC if symmetric else 0) | (COPY if copy else 0) | (VALIDATE if validate else 0) | \
            (PAIRS if pairs else 0) | (SORTED if sorted_rows else 0)
    wp = None
    if wgt is not None:
        if wgt.dtype != np.uint32 or wgt.size != m:
            raise TypeError("wgt must be uint32[m]")
        wp = wgt.ctypes.data
    _check(_lib.ascetic_load_csr(n, m, off.ctypes.data, nbr.ctypes.data if nbr.size else None, wp, flags))
    _keep["csr"] = (off, nbr, wgt)


def set_budget(nbytes: int, static_fraction: float = -1.0) -> None:
    _check(_lib.ascetic_set_budget(int(nbytes), float(static_fraction)))


def set_option(name: str, value: int) -> None:
    _check(_lib.ascetic_set_option(OPTIONS[name], int(value)))


def run(algo: str, source: int = 0, max_iters: int = 0) -> None:
    _check(_lib.ascetic_run(ALGOS[algo], int(source), int(max_iters)))


def _sdict(s: ctypes.Structure) -> dict:
    return {f: getattr(s, f) for f, _ in s._fields_}


def stats(per_iter: bool = True) -> tuple[dict, list[dict]]:
    st = Stats()
    k = _check(_lib.ascetic_stats(ctypes.byref(st), None, 0))
    its = []
    if per_iter and k:
        arr = (IterStats * k)()
        _check(_lib.ascetic_stats(ctypes.byref(st), arr, k))
        its = [_sdict(arr[i]) for i in range(k)]
    return _sdict(st), its


def get_result(out: np.ndarray | None = None) -> np.ndarray:
    st = Stats()
    _check(_lib.ascetic_stats(ctypes.byref(st), None, 0))
    dt = np.float32 if st.algo in (ALGOS["pr"], ALGOS["prd"]) else np.uint32
    if out is None:
        out = np.empty(max(st.n, 1), dtype=dt)[: st.n]
    _check(_lib.ascetic_get_result(out.ctypes.data, out.nbytes))
    return out


def unload() -> None:
    _lib.ascetic_unload()
    _keep.clear()


PARITY_FIELDS = ["t", "nA", "nH", "nM", "nruns", "active_arcs", "hit_arcs", "miss_bytes", "digest"]


class Placement(ctypes.Structure):
    _fields_ = [("R", ctypes.c_double), ("D", ctypes.c_uint64), ("B", ctypes.c_uint64), ("Ms", ctypes.c_uint64),
                ("s", ctypes.c_uint64), ("static_bytes", ctypes.c_uint64), ("C", ctypes.c_uint64),
                ("cap", ctypes.c_uint64)]


_lib.ascetic_place.argtypes = [ctypes.c_uint64, ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_double,
                               ctypes.POINTER(Placement)]
EXPORTS.append("ascetic_place")
_lib.ascetic_emulate_ranks.argtypes = [ctypes.c_int]
_lib.ascetic_partition.argtypes = [ctypes.c_uint64, ctypes.c_void_p, ctypes.c_uint32, ctypes.c_void_p]
EXPORTS += ["ascetic_emulate_ranks", "ascetic_partition"]


class ClassifyOut(ctypes.Structure):
    _fields_ = [(f, ctypes.c_void_p) for f in ["hit_small", "hit_med", "hit_hub", "hub_pre", "missq", "missq_pre",
                                               "missq_src", "run_b", "run_e", "run_dst"]] + \
               [(f, ctypes.c_uint64) for f in ["cap", "n_small", "n_med", "n_hub", "n_pieces", "n_missq", "n_runs",
                                               "miss_arcs", "nA", "nH", "nM", "active_arcs", "hit_arcs", "digest"]]


_lib.ascetic_debug_classify.argtypes = [ctypes.c_int, ctypes.c_void_p, ctypes.c_uint64, ctypes.POINTER(ClassifyOut)]
EXPORTS.append("ascetic_debug_classify")


def debug_classify(active: np.ndarray, rank: int = 0) -> dict:
    """One classify+compaction of `active` (bool[n]) against the current StaticBitmap (test use)."""
    a = np.ascontiguousarray(active, dtype=bool)
    n = a.size
    words = np.packbits(np.concatenate([a, np.zeros((-n) % 32, bool)]).reshape(-1, 32)[:, ::-1], axis=1)
    words = np.ascontiguousarray(words[:, ::-1]).view(np.uint32).reshape(-1) if n else np.zeros(0, np.uint32)
    cap = max(n, 1)
    arr = {k: np.zeros(cap, dtype=np.uint32) for k in ["hit_small", "hit_med", "hit_hub", "hub_pre", "missq",
                                                      "run_b", "run_e"]}
    arr.update({k: np.zeros(cap, dtype=np.uint64) for k in ["missq_pre", "missq_src", "run_dst"]})
    o = ClassifyOut()
    for k, v in arr.items():
        setattr(o, k, v.ctypes.data)
    o.cap = cap
    _check(_lib.ascetic_debug_classify(rank, words.ctypes.data if words.size else None, words.size, ctypes.byref(o)))
    cnt = {"hit_small": o.n_small, "hit_med": o.n_med, "hit_hub": o.n_hub, "hub_pre": o.n_hub, "missq": o.n_missq,
           "missq_pre": o.n_missq, "missq_src": o.n_missq, "run_b": o.n_runs, "run_e": o.n_runs, "run_dst": o.n_runs}
    res = {k: v[:cnt[k]].copy() for k, v in arr.items()}
    res.update({f: getattr(o, f) for f in ["n_pieces", "miss_arcs", "nA", "nH", "nM", "active_arcs", "hit_arcs",
                                           "digest"]})
    return res


def partition(off: np.ndarray, parts: int) -> np.ndarray:
    """Host-only 1D edge-balanced rank boundaries (parts+1 entries)."""
    off = np.ascontiguousarray(off, dtype=np.uint64)
    b = np.zeros(parts + 1, dtype=np.uint64)
    _check(_lib.ascetic_partition(off.size - 1, off.ctypes.data, parts, b.ctypes.data))
    return b


def emulate_ranks(world: int) -> None:
    """Drive `world` ranks from this process on its single GPU (before load_csr)."""
    _check(_lib.ascetic_emulate_ranks(int(world)))


def get_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(_lib.ascetic_get_unique_id(buf))
    return buf.raw


def comm_init(rank: int, world: int, uid: bytes | None, device: int) -> None:
    """Join the NCCL exchange (one process per GPU), before load_csr."""
    buf = ctypes.create_string_buffer(uid, 128) if uid is not None else None
    _check(_lib.ascetic_comm_init(int(rank), int(world), buf, int(device)))


def init_distributed(device: int) -> tuple[int, int]:
    """torch.distributed plumbing only: rank 0's NCCL unique id is broadcast over the
    already-initialised default process group, then every rank calls comm_init."""
    import torch.distributed as dist
    rank, world = dist.get_rank(), dist.get_world_size()
    if world == 1:
        return rank, world
    obj = [get_unique_id() if rank == 0 else None]
    dist.broadcast_object_list(obj, src=0)
    comm_init(rank, world, obj[0], device)
    return rank, world
_lib.ascetic_struct_sizes.argtypes = [ctypes.c_void_p]
EXPORTS.append("ascetic_struct_sizes")


def struct_sizes() -> tuple[int, int, int]:
    out = (ctypes.c_uint64 * 3)()
    _check(_lib.ascetic_struct_sizes(out))
    return int(out[0]), int(out[1]), int(out[2])


if struct_sizes() != (ctypes.sizeof(Stats), ctypes.sizeof(IterStats), ctypes.sizeof(Placement)):
    raise ImportError(f"ctypes mirrors out of sync with ascetic.h: lib {struct_sizes()} vs "
                      f"{(ctypes.sizeof(Stats), ctypes.sizeof(IterStats), ctypes.sizeof(Placement))}")


def place(off: np.ndarray, b_e: int, nbytes: int, static_fraction: float = -1.0) -> dict:
    """Host-only Eq. 2 placement (what set_budget would choose)."""
    off = np.ascontiguousarray(off, dtype=np.uint64)
    p = Placement()
    _check(_lib.ascetic_place(off.size - 1, off.ctypes.data, b_e, int(nbytes), float(static_fraction),
                              ctypes.byref(p)))
    return _sdict(p)
