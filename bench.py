"""bench.py — end-to-end GTEPS of the Ascetic hot path under a capped device budget.

Contract (driver): `python bench.py --gpus N --steps K --warmup W` prints ONE JSON line.
A step = one full ascetic_run (classify+compact, static fill, static + on-demand edge
kernels, every H2D chunk, finalize, for all iterations) of the workload below. Default
workload = BASELINE.json configs[3], the largest configuration that runs on one GPU in a
bench-sized time: CC on the uk-2007-shaped graph (105 M vertices, 3.3 B tuples -> 6.4 B
arcs, 25.8 GB CSR) with the device edge budget capped at 30 % of the CSR bytes; the same
config is BASELINE.json's 1/2/4/8-GPU case. C1-C3 and C5 stay available with --config.

  value  = Σ active arcs / Σ step device time (CUDA events around each step), GTEPS;
           the graph is host-resident (that is the method) and already pinned/loaded.
  e2e    = same metric through the public API with every host<->device copy inside the
           step: load_csr (offsets H2D) + set_budget + run (fill + misses H2D) + get_result (D2H).
  roofline = dominant kernel of the step (by device time): algorithmic bytes / time vs
           the measured peak of its bound (host link: pinned H2D measured here; HBM:
           MEASURED_PEAKS.json hbm_gbs). See DESIGN.md §"Roofline".
`--impl reference` times the CPU oracle (oracle/) on the same workload instead.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

METRIC = "end-to-end GTEPS incl. H2D under capped HBM budget; H2D GB per run"


def _dist():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def _peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d.get("hbm_gbs", 6650.0)), "measured"
    return 6650.0, "fallback"


class Clocks:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md clocks line)."""

    FIELDS = ["index", "clocks.sm", "clocks.max.sm", "power.draw", "clocks_event_reasons.active",
              "clocks_event_reasons.hw_slowdown", "clocks_event_reasons.hw_thermal_slowdown",
              "clocks_event_reasons.sw_thermal_slowdown", "clocks_event_reasons.sw_power_cap"]

    def __init__(self, gpu: int):
        self.gpu = gpu
        self.path = f"/tmp/ascetic_clocks_{os.getpid()}.csv"
        self.p = None

    def start(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(self.gpu), "--query-gpu=" + ",".join(self.FIELDS),
                                       "--format=csv,noheader,nounits", "-lms", "100"],
                                      stdout=open(self.path, "w"), stderr=subprocess.DEVNULL)
        except Exception:
            self.p = None

    def stop(self) -> dict:
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.p.terminate()
        try:
            self.p.wait(timeout=5)
        except Exception:
            self.p.kill()
        sm, smax, reasons, power = [], [], set(), []
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in open(self.path):
            f = [x.strip() for x in line.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1])); smax.append(float(f[2])); power.append(float(f[3]))
            except ValueError:
                continue
            for nm, v in zip(names, f[5:9]):
                if v.lower() == "active":
                    reasons.add(nm)
        os.unlink(self.path)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(smax) if smax else None,
                "reasons": sorted(reasons), "samples": len(sm), "power_w_max": max(power) if power else None}


def _h2d_peak(torch, dev, reps: int = 5) -> float:
    """Pinned H2D copy-engine peak on this box: 1 GiB cudaMemcpyAsync, best of `reps` (GB/s)."""
    sz = 1 << 30
    h = torch.empty(sz, dtype=torch.uint8, pin_memory=True)
    g = torch.empty(sz, dtype=torch.uint8, device=dev)
    best = 0.0
    for _ in range(reps):
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); g.copy_(h, non_blocking=True); e1.record(); e1.synchronize()
        best = max(best, sz / (e0.elapsed_time(e1) / 1e3) / 1e9)
    del h, g
    return best


def _workload(cfg_key: str):
    import graphgen as gg
    c = gg.CONFIGS[cfg_key]
    return gg, c


def _config(args, c, g) -> dict:
    """The workload, identical in both arms (the driver compares the two config dicts)."""
    import graphgen as gg
    algo, iters = _algo(args, c)
    return {"workload": f"{args.config}: {c['desc']}", "algo": algo, "n": g.n, "m": g.m,
            "budget_bytes": gg.config_budget(args.config, g), "csr_bytes": g.csr_bytes,
            "pr_iterations": iters if algo == "pr" else None,
            "sources": "8 seeded sources with deg > 0 (seed = config seed), cycled over the steps"
            if algo in ("bfs", "sssp") else None}


def _algo(args, c):
    """(algorithm, PR iterations) of a config; C5 ("BFS + PageRank") runs one of them per bench line."""
    algo = c["algo"] if c["algo"] != "bfs+pr" else args.c5_algo
    iters = (c.get("iters") or args.c5_pr_iters) if algo == "pr" else 0
    return algo, iters


def shared_graph(config: str, barrier, local_rank: int, tag: str, alloc_local=None):
    """N > 1 on one node: local rank 0 generates the CSR ONCE into shared files (/dev/shm when it has
    room, else ASCETIC_SHM_DIR or /tmp), every rank maps them MAP_SHARED, so host RAM holds one copy
    whatever N is; each rank's library then pins only the arcs of its own rows.
    Returns (graph, cleanup, generation seconds)."""
    import graphgen as gg
    c = gg.CONFIGS[config]
    est = 8 * ((1 << c["scale"]) + 1) + (8 if c["algo"] == "sssp" else 4) * 2 * c["tuples"]
    d = "/dev/shm"
    try:
        st = os.statvfs(d)
        if st.f_bavail * st.f_frsize < est * 1.05:
            d = os.environ.get("ASCETIC_SHM_DIR", "/tmp")
    except OSError:
        d = os.environ.get("ASCETIC_SHM_DIR", "/tmp")
    base = os.path.join(d, f"ascetic_{config}_{tag}")
    gen_s = 0.0
    if local_rank == 0:
        files = []

        def alloc(count, dtype):
            path = f"{base}.{len(files)}"
            files.append(path)
            return np.memmap(path, dtype=dtype, mode="w+", shape=(max(1, count),))

        t0 = time.time()
        g = gg.config_graph(config, alloc=alloc)
        gen_s = time.time() - t0
        for a in (g.off, g.nbr):
            if isinstance(a.base, np.memmap):
                a.base.flush()
        json.dump({"n": g.n, "m": g.m, "pairs": g.pairs, "files": files}, open(base + ".json.tmp", "w"))
        os.replace(base + ".json.tmp", base + ".json")
    barrier()
    meta = json.load(open(base + ".json"))
    n, m, pairs = meta["n"], meta["m"], meta["pairs"]
    # read-write shared mappings (never written): page-locking a read-only mapping can be refused
    off = np.memmap(meta["files"][0], dtype=np.uint64, mode="r+")[: n + 1]
    cnt = (2 if pairs else 1) * m
    nbr = np.memmap(meta["files"][1], dtype=np.uint32, mode="r+")[:cnt]
    g = gg.Graph(n=n, m=m, off=off, nbr=nbr, pairs=pairs, name=config)

    def cleanup():
        barrier()
        if local_rank == 0:
            for f in meta["files"] + [base + ".json"]:
                try:
                    os.unlink(f)
                except OSError:
                    pass
    return g, cleanup, gen_s


def spans_cover(per: list) -> bool:
    """True when the library's per-phase CUDA-event spans cover every class of work in these steps
    (TIMING=1 gives small iterations one span, leaving their per-kernel times at 0)."""
    for s in per:
        if s["gather_bytes"] and not s["time_gather_s"]:
            return False
        if s["ondemand_arcs"] and not s["time_ondemand_s"]:
            return False
        if s["static_arcs"] and not s["time_static_s"]:
            return False
        if (s["h2d_payload_bytes"] + s["h2d_static_fill_bytes"]) and not s["time_h2d_busy_s"]:
            return False
        if s["iterations"] and not s["time_classify_s"]:
            return False
    return True


def roofline_of(per: list, steps: int, total_ms: float, b_e: int, n: int, h2d_peak: float, hbm_peak: float,
                hbm_src: str, config: str) -> dict:
    """Roofline entry of a bench line from the library's per-step stats (pure: unit-tested on CPU)."""
    # ---- per-kernel-class breakdown (library CUDA events on the launching streams)
    kern = {
        "gather": dict(time_s=sum(s["time_gather_s"] for s in per), bytes=sum(s["gather_bytes"] for s in per),
                       bound="host_link", peak=h2d_peak),
        "dma": dict(time_s=sum(s["time_dma_s"] + s["time_fill_s"] for s in per),
                    bytes=sum(s["dma_bytes"] + s["h2d_static_fill_bytes"] for s in per), bound="host_link",
                    peak=h2d_peak),
        "ondemand": dict(time_s=sum(s["time_ondemand_s"] for s in per),
                         bytes=sum(s["ondemand_arcs"] for s in per) * (b_e + 4), bound="hbm", peak=hbm_peak),
        "static": dict(time_s=sum(s["time_static_s"] for s in per),
                       bytes=sum(s["static_arcs"] for s in per) * (b_e + 4), bound="hbm", peak=hbm_peak),
        "classify": dict(time_s=sum(s["time_classify_s"] for s in per),
                         bytes=sum(s["iterations"] for s in per) * (n // 4) + 0, bound="hbm", peak=hbm_peak),
    }
    # the transfer path as a whole (the step's bound when out of core): every H2D byte of the step (static
    # fill + per-iteration miss payload, whichever engine moved it) over the copy streams' busy time
    kern["transfer"] = dict(time_s=sum(s["time_h2d_busy_s"] for s in per),
                            bytes=sum(s["h2d_static_fill_bytes"] + s["h2d_payload_bytes"] for s in per),
                            bound="host_link", peak=h2d_peak)
    for k_, d in kern.items():
        d["achieved"] = d["bytes"] / d["time_s"] / 1e9 if d["time_s"] > 0 else 0.0
        d["frac"] = d["achieved"] / d["peak"] if d["peak"] else 0.0
        d["share_of_step"] = d["time_s"] * 1e3 / total_ms if total_ms else 0.0
    # headline entry: the transfer path when it fills most of the step (out of core), else the
    # longest kernel class; "dominant_kernel" is always the longest class of our own kernels
    own = ("gather", "ondemand", "static", "classify")
    dom_kernel = max(own, key=lambda k_: kern[k_]["time_s"])
    dom = "transfer" if kern["transfer"]["share_of_step"] >= 0.5 else max(
        ("gather", "dma", "ondemand", "static", "classify"), key=lambda k_: kern[k_]["time_s"])
    dk = kern[dom]
    # the gather class = the transfer engine in gather mode: SM zero-copy gather + the copy-engine
    # long runs beside it (same chunk windows, union time)
    sm_b = sum(s["gather_bytes"] - s["gather_ce_bytes"] for s in per)
    kern["gather"].update(sm_bytes=sm_b, ce_bytes=sum(s["gather_ce_bytes"] for s in per),
                          sm_load_bytes=sum(s["gather_load_bytes"] for s in per),
                          launches=sum(s["gather_chunks"] for s in per))
    traffic, traffic_note = None, None
    tp = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    tj = {}
    if os.path.exists(tp):
        try:
            tj = json.load(open(tp)).get(config, {})
        except Exception:
            tj = {}
    tg = tj.get("gather")
    if isinstance(tg, dict) and "pcie_read_per_payload" in tg and kern["gather"]["launches"]:
        # gather launches: PCIe read bytes = ncu's measured PCIe bytes per payload byte (a capture of
        # full-window launches) x this run's SM payload per gather launch
        kern["gather"]["pcie_read_bytes_per_launch"] = tg["pcie_read_per_payload"] * sm_b / kern["gather"]["launches"]
    if dom == "transfer":
        # link bytes of the step: copy-engine bytes as moved (static fill, DMA'd runs, span windows
        # with their holes) + the SM gather's payload scaled by its measured PCIe bytes per payload byte
        ratio = tg.get("pcie_read_per_payload") if isinstance(tg, dict) else None
        ce = sum(s["h2d_static_fill_bytes"] + s["dma_bytes"] - s["span_payload_bytes"] + s["span_link_bytes"]
                 + s["gather_ce_bytes"] for s in per)
        if ratio or sm_b == 0:
            ratio = ratio or 0.0
            traffic = (ce + ratio * sm_b) / steps
            traffic_note = (f"per step: copy-engine bytes as moved ({ce / steps / 1e9:.2f} GB incl. span holes) + "
                            f"SM-gathered payload x {ratio:.3f} PCIe read bytes per payload byte "
                            f"(ncu pcie__read_bytes, {tg.get('source', 'ncu') if isinstance(tg, dict) else 'no SM gather'}); algorithmic bytes per step "
                            f"{dk['bytes'] / steps / 1e9:.2f} GB")
    else:
        t_ = tj.get(dom)
        if isinstance(t_, (int, float)):
            traffic = t_
            traffic_note = "dram__bytes_read.sum + dram__bytes_write.sum of one launch (ncu --set full)"
    roofline = {"kernel": dom, "bound": dk["bound"], "achieved": dk["achieved"], "peak": dk["peak"],
                "unit": "GB/s", "frac": dk["frac"], "traffic": traffic, "traffic_note": traffic_note,
                "dominant_kernel": {"name": dom_kernel, "achieved": kern[dom_kernel]["achieved"],
                                    "peak": kern[dom_kernel]["peak"], "frac": kern[dom_kernel]["frac"],
                                    "bound": kern[dom_kernel]["bound"],
                                    "share_of_step": kern[dom_kernel]["share_of_step"]},
                "peak_source": ("pinned H2D cudaMemcpyAsync 1 GiB, best of 5 copies before and 10 after the timed steps, in this run"
                                if dk["bound"] == "host_link" else f"MEASURED_PEAKS.json hbm_gbs ({hbm_src})"),
                "per_kernel": {k_: {kk: (round(vv, 6) if isinstance(vv, float) else vv) for kk, vv in d.items()}
                               for k_, d in kern.items()}}
    return roofline


def run_reference(args, ws, rank):
    """--impl reference: the oracle as it stands, on the host cores, same config/metric/unit."""
    if rank != 0:
        return 0
    import oracle
    gg, c = _workload(args.config)
    g = gg.config_graph(args.config)
    budget = gg.config_budget(args.config, g)
    p = oracle.placer(g.off, g.b_e, budget)
    st = oracle.static_prefix(g.n, p.s)
    algo, iters = _algo(args, c)
    if algo == "pr":
        iters = min(iters, args.ref_pr_iters)
    srcs = gg.sources(g, 8, seed=c["seed"])
    for i in range(args.warmup):
        oracle.run(algo, g.off, g.nbr, src=srcs[i % len(srcs)], max_iters=iters, is_static=st)
    arcs, secs, h2d = 0, 0.0, 0
    for i in range(args.steps):
        t0 = time.perf_counter()
        r = oracle.run(algo, g.off, g.nbr, src=srcs[(args.warmup + i) % len(srcs)], max_iters=iters, is_static=st)
        secs += time.perf_counter() - t0
        arcs += r.active_arcs_total
        h2d += r.h2d_payload + p.static_bytes
    v = arcs / secs / 1e9
    sample = (f"{args.steps} full oracle {algo.upper()} runs" + (f" of {iters} iterations" if algo == "pr" else "")
              + f" on the {args.config} graph (n={g.n}, m={g.m})")
    out = {"metric": METRIC, "value": v, "unit": "GTEPS", "impl": "reference", "n_gpus": ws,
           "steps": args.steps, "warmup": args.warmup, "ms_per_step": secs / args.steps * 1e3,
           "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u32" if algo != "pr" else "f64",
           "data": "synthetic", "config": _config(args, c, g),
           "run": {"h2d_gb_per_run_predicted": h2d / args.steps / 1e9,
                   "pr_iterations_per_step": iters if algo == "pr" else None},
           "cpu_baseline": {"value": v, "unit": "GTEPS", "cores": oracle.threads(), "kind": "oracle",
                            "sample": sample},
           "e2e": {"value": v, "unit": "GTEPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ascetic", choices=["ascetic", "reference"])
    ap.add_argument("--config", default="c4", choices=["c1", "c2", "c3", "c4", "c5"])
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--profile-steps", type=int, default=3,
                    help="extra steps with every phase timed, for the roofline breakdown when the timed steps "
                         "left small iterations as one span (after the timed region)")
    ap.add_argument("--no-pageable", action="store_true", help="skip the pageable-input load_csr measurement")
    ap.add_argument("--c5-algo", default="bfs", choices=["bfs", "pr"], help="C5 (BFS + PageRank): which one a step runs")
    ap.add_argument("--c5-pr-iters", type=int, default=43, help="C5 PageRank iterations per step")
    ap.add_argument("--cpu-seconds", type=float, default=15.0, help="bounded oracle sample for cpu_baseline")
    ap.add_argument("--ref-pr-iters", type=int, default=2, help="PR iterations per reference step (bounded)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--xfer", type=int, default=0)
    ap.add_argument("--opt", action="append", default=[], metavar="NAME=VALUE",
                    help="extra library option for A/B runs (ascetic_set_option), repeatable")
    ap.add_argument("--sparse-exchange", type=int, default=0,
                    help="N > 1, BFS/SSSP/CC: ASCETIC_OPT_SPARSE_EXCHANGE divisor d (0 = dense exchange)")
    args = ap.parse_args()
    ws, rank, local = _dist()
    if args.warmup < 3:
        print("warning: warmup < 3 violates the timing rules; using 3", file=sys.stderr)
        args.warmup = 3
    if args.impl == "reference":
        return run_reference(args, ws, rank)

    import torch
    import torch.distributed as dist
    dev = torch.device("cuda", local)
    torch.cuda.set_device(dev)
    if ws > 1:
        import datetime
        # generous timeout: the other ranks wait in a barrier while local rank 0 generates the shared
        # graph (C4 ~3 min, C5 ~8 min on 16 host cores)
        dist.init_process_group("nccl", device_id=dev, timeout=datetime.timedelta(minutes=60))
    import paper_conf_icpp_tangzwgzwy21_b200 as asc
    gg, c = _workload(args.config)
    algo, iters = _algo(args, c)

    h2d_peak = _h2d_peak(torch, dev)
    hbm_peak, hbm_src = _peaks()

    # graph offsets and arcs generated straight into pinned host memory (the method's host Edgelist)
    pinned = []

    def alloc(count, dtype):
        words = max(1, count) * np.dtype(dtype).itemsize // 4
        t = torch.empty(words, dtype=torch.int32, pin_memory=True)
        pinned.append(t)
        return t.numpy().view(dtype)

    cleanup = None
    if ws > 1:
        g, cleanup, gen_s = shared_graph(args.config, dist.barrier, local, os.environ.get("MASTER_PORT", "0"))
    else:
        t0 = time.time()
        g = gg.config_graph(args.config, alloc=alloc)
        gen_s = time.time() - t0
    srcs = gg.sources(g, 8, seed=c["seed"])
    if ws > 1:
        # 1D edge-balanced ranges, one per GPU; NCCL exchange inside the library.
        # Per-GPU budget = the config's budget rule applied to this rank's slice.
        asc.init_distributed(local)
        b = asc.partition(g.off, ws)
        lo, hi = int(b[rank]), int(b[rank + 1])
        slice_bytes = g.b_e * int(g.off[hi] - g.off[lo]) + 8 * (hi - lo + 1)
        budget = int(c["budget_frac"] * slice_bytes) if "budget_frac" in c else int(c["budget_bytes"])
    else:
        asc.set_device(local)
        budget = gg.config_budget(args.config, g)

    asc.load_csr(g.off, g.nbr, pairs=g.pairs, symmetric=True, sorted_rows=True)   # generator rows are sorted
    for kv in args.opt:                               # before set_budget: some shape the On-demand Region
        k_, v_ = kv.split("=", 1)
        asc.set_option(k_, int(v_))
    asc.set_budget(budget)
    asc.set_option("xfer_mode", args.xfer)
    asc.set_option("sparse_exchange", args.sparse_exchange)
    l2_flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)

    def step(i):
        asc.run(algo, srcs[i % len(srcs)], iters)

    def stats():                                      # host bookkeeping: read after a step's end event
        return asc.stats(per_iter=False)[0]

    for i in range(args.warmup):
        step(i)
    torch.cuda.synchronize()

    g500_edges = 0
    deg64 = np.diff(g.off.astype(np.int64)) if algo == "bfs" else None
    clocks = Clocks(local)
    clocks.start()
    time.sleep(1.0)                                   # the sampler's own start-up (NVML init) stays out of the steps
    per = []
    total_ms = 0.0
    for k in range(args.steps):
        l2_flush.fill_(k & 0xFF)                      # flush L2 between timed steps (outside the step)
        torch.cuda.synchronize()
        if ws > 1:
            dist.barrier()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record()
        step(args.warmup + k)
        e1.record()
        torch.cuda.synchronize()
        total_ms += e0.elapsed_time(e1)
        per.append(stats())
        if algo == "bfs":
            # Graph500 TEPS: undirected edges in the reached component, read after the
            # timed region; the graphs are symmetric, so that is half the reached vertices' arcs
            lv = asc.get_result()
            g500_edges += int(deg64[lv != 0xFFFFFFFF].sum()) // 2
    clk = clocks.stop()
    if ws > 1:
        tt = torch.tensor([total_ms], device=dev, dtype=torch.float64)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        total_ms = float(tt.item())

    def _sum_ranks(x: int) -> int:
        if ws == 1:
            return x
        tt = torch.tensor([x], device=dev, dtype=torch.int64)
        dist.all_reduce(tt)
        return int(tt.item())

    # every rank counts the arcs of ITS owned active vertices: the job total is the sum
    arcs = sum(s["active_arcs_total"] for s in per)
    arcs_all = _sum_ranks(arcs)
    value = arcs_all / (total_ms / 1e3) / 1e9
    fill = _sum_ranks(sum(s["h2d_static_fill_bytes"] for s in per))
    payload = _sum_ranks(sum(s["h2d_payload_bytes"] for s in per))
    lib_ms = sum(s["time_run_s"] for s in per) * 1e3
    # GTEPS excluding the static fill (the fill DMA's own events, max over ranks)
    fill_ms = sum(s["time_fill_s"] for s in per) * 1e3
    if ws > 1:
        tt = torch.tensor([fill_ms], device=dev, dtype=torch.float64)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        fill_ms = float(tt.item())
    value_excl_fill = arcs_all / ((total_ms - fill_ms) / 1e3) / 1e9 if total_ms > fill_ms else None

    # the link peak again, right after the timed steps (a measurement taken while the host was still busy
    # elsewhere, e.g. unpinning a previous process's memory, can read low): the best of both is the peak
    h2d_peak = max(h2d_peak, _h2d_peak(torch, dev, reps=10))
    roofline = roofline_of(per, args.steps, total_ms, g.b_e, g.n, h2d_peak, hbm_peak, hbm_src, args.config)
    if not spans_cover(per) and args.profile_steps > 0:
        # small iterations ran with one span each (TIMING=1 keeps per-phase events off the latency path),
        # so the per-kernel classes above are incomplete: take them from extra steps with every phase
        # timed, run AFTER the timed region (their event overhead never reaches `value`)
        asc.set_option("timing", 2)
        prof, prof_ms = [], 0.0
        for k in range(args.profile_steps):
            l2_flush.fill_(k & 0xFF)
            torch.cuda.synchronize()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record()
            step(args.warmup + k)
            e1.record()
            torch.cuda.synchronize()
            prof_ms += e0.elapsed_time(e1)
            prof.append(stats())
        asc.set_option("timing", int(dict(kv.split("=", 1) for kv in args.opt).get("timing", 1)))
        roofline = roofline_of(prof, args.profile_steps, prof_ms, g.b_e, g.n, h2d_peak, hbm_peak, hbm_src,
                               args.config)
        roofline["phase_spans"] = (f"{args.profile_steps} extra steps with every phase timed (TIMING=2), after "
                                   f"the timed region: {prof_ms / args.profile_steps:.3f} ms per step with the "
                                   f"events vs {total_ms / args.steps:.3f} timed")
    h2d_total = fill + payload
    span_holes = _sum_ranks(sum(s["span_link_bytes"] - s["span_payload_bytes"] for s in per))
    link = {"h2d_bytes": h2d_total, "h2d_busy_s": sum(s["time_h2d_busy_s"] for s in per),
            "achieved_gbs": h2d_total / (sum(s["time_h2d_busy_s"] for s in per) or 1) / 1e9,
            "whole_step_gbs": h2d_total / (total_ms / 1e3) / 1e9, "peak_gbs": h2d_peak}
    link["frac_busy"] = link["achieved_gbs"] / h2d_peak
    link["frac_step"] = link["whole_step_gbs"] / h2d_peak

    # ---- e2e: public API with host buffers, every copy inside the step
    e2e_ms, e2e_arcs, h2d_b, d2h_b = 0.0, 0, 0, 0
    e2e_parts = {}
    res = np.empty(g.n, dtype=np.float32 if algo == "pr" else np.uint32)
    res_pinned = torch.empty(max(1, g.n), dtype=torch.int32, pin_memory=True).numpy().view(res.dtype)[: g.n]
    for k in range(args.e2e_steps):
        l2_flush.fill_(k & 0xFF)
        torch.cuda.synchronize()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record()
        h0 = time.perf_counter()
        asc.load_csr(g.off, g.nbr, pairs=g.pairs, symmetric=True, sorted_rows=True)
        h1 = time.perf_counter()
        asc.set_budget(budget)
        asc.set_option("xfer_mode", args.xfer)
        asc.set_option("sparse_exchange", args.sparse_exchange)
        h2 = time.perf_counter()
        asc.run(algo, srcs[k % len(srcs)], iters)
        h3 = time.perf_counter()
        asc.get_result(res_pinned)
        h4 = time.perf_counter()
        e1.record()
        torch.cuda.synchronize()
        s_ = asc.stats(per_iter=False)[0]
        for key, v in (("load_csr", h1 - h0), ("set_budget", h2 - h1), ("run", h3 - h2), ("get_result", h4 - h3)):
            e2e_parts[key] = e2e_parts.get(key, 0.0) + v * 1e3 / max(1, args.e2e_steps)
        e2e_ms += e0.elapsed_time(e1)
        e2e_arcs += s_["active_arcs_total"]
        h2d_b += 8 * (g.n + 1) + s_["h2d_static_fill_bytes"] + s_["h2d_payload_bytes"]
        d2h_b += res_pinned.nbytes + s_["d2h_bytes"]
    if ws > 1:
        tt = torch.tensor([e2e_ms], device=dev, dtype=torch.float64)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        e2e_ms = float(tt.item())
        e2e_arcs, h2d_b, d2h_b = _sum_ranks(e2e_arcs), _sum_ranks(h2d_b), _sum_ranks(d2h_b)
    e2e = {"value": e2e_arcs / (e2e_ms / 1e3) / 1e9 if e2e_ms > 0 else None, "unit": "GTEPS",
           "h2d_bytes_per_step": h2d_b // max(1, args.e2e_steps), "d2h_bytes_per_step": d2h_b // max(1, args.e2e_steps),
           "steps": args.e2e_steps, "ms_per_step": e2e_ms / max(1, args.e2e_steps),
           "host_ms_per_call": {k: round(v, 3) for k, v in e2e_parts.items()},
           "note": "host arrays already page-locked (the bench generates them into pinned memory), so "
                   "load_csr is the offsets upload; see cold_pageable for a caller with pageable arrays"}

    # ---- a caller with PAGEABLE host arrays: load_csr pins the edge array in place
    # (cudaHostRegister, read-only) before the first run; reported next to the warm e2e
    if not args.no_pageable and ws == 1:
        nbr_pg = np.empty_like(g.nbr)                   # plain (pageable) numpy memory
        np.copyto(nbr_pg, g.nbr)
        t0 = time.perf_counter()
        asc.load_csr(g.off, nbr_pg, pairs=g.pairs, symmetric=True, sorted_rows=True)
        pin_ms = (time.perf_counter() - t0) * 1e3
        asc.set_budget(budget)
        torch.cuda.synchronize()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record()
        asc.run(algo, srcs[0], iters)
        e1.record()
        torch.cuda.synchronize()
        s_ = asc.stats(per_iter=False)[0]
        run_ms = e0.elapsed_time(e1)
        e2e["cold_pageable"] = {"load_csr_ms": round(pin_ms, 1), "run_ms": round(run_ms, 2),
                                "value": s_["active_arcs_total"] / ((pin_ms + run_ms) / 1e3) / 1e9,
                                "pinned_bytes": int(g.nbr.nbytes),
                                "note": "first call with pageable arrays: load_csr (page-locking the edge "
                                        "array) + one run, GTEPS over both"}
        asc.load_csr(g.off, g.nbr, pairs=g.pairs, symmetric=True, sorted_rows=True)   # unpins nbr_pg
        del nbr_pg

    # ---- CPU baseline: the oracle as it stands, bounded sample, rank 0 at N=1 only
    cpu = None
    if rank == 0 and ws == 1 and not args.no_cpu_baseline:
        import oracle
        p = oracle.placer(g.off, g.b_e, budget)
        stc = oracle.static_prefix(g.n, p.s)
        it_ = min(iters, args.ref_pr_iters) if algo == "pr" else 0
        a_, s_t, runs = 0, 0.0, 0
        while runs < 1 or (s_t < args.cpu_seconds and runs < 8):
            t0 = time.perf_counter()
            r = oracle.run(algo, g.off, g.nbr, src=srcs[runs % len(srcs)], max_iters=it_, is_static=stc)
            s_t += time.perf_counter() - t0
            a_ += r.active_arcs_total
            runs += 1
        cpu = {"value": a_ / s_t / 1e9, "unit": "GTEPS", "cores": oracle.threads(), "kind": "oracle",
               "sample": f"{runs} full oracle {algo.upper()} runs" + (f" of {it_} iterations" if algo == "pr" else "")
                         + f" from the bench sources on the same {args.config} graph ({s_t:.1f} s)"}
        if args.config in ("c1", "c2"):
            # a single-thread oracle figure too, for C1/C2: one run from the first source
            k0 = oracle.threads()
            oracle.set_threads(1)
            try:
                t0 = time.perf_counter()
                r = oracle.run(algo, g.off, g.nbr, src=srcs[0], max_iters=it_, is_static=stc)
                t1 = time.perf_counter() - t0
            finally:
                oracle.set_threads(k0)
            cpu["single_thread"] = {"value": r.active_arcs_total / t1 / 1e9, "unit": "GTEPS", "cores": 1,
                                    "sample": f"1 full oracle {algo.upper()} run from source {srcs[0]} ({t1:.1f} s)"}

    out = {"metric": METRIC, "value": value, "unit": "GTEPS", "n_gpus": ws, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": total_ms / args.steps, "higher_is_better": True,
           "scaling": "strong", "vs_baseline": None, "dtype": "u32" if algo != "pr" else "f32",
           "data": "synthetic",
           "config": _config(args, c, g),
           "run": {"budget_bytes_per_rank": budget, "static_vertices": per[0]["s"],
                   "static_fraction": per[0]["static_fraction_used"], "chunk_cap": per[0]["chunk_cap"],
                   "chunk_buffers": per[0]["chunk_buffers"],
                   "h2d_gb_per_run": h2d_total / args.steps / 1e9,
                   "h2d_fill_gb_per_run": fill / args.steps / 1e9,
                   "h2d_payload_gb_per_run": payload / args.steps / 1e9,
                   # bytes the copy engines and the SM gather actually requested: payload + the holes
                   # that span-DMA windows carry between missed lists (PCIe protocol overhead excluded)
                   "h2d_requested_gb_per_run": (h2d_total + span_holes) / args.steps / 1e9,
                   "iterations_per_run": statistics.mean(s["iterations"] for s in per),
                   "sources": srcs if algo in ("bfs", "sssp") else None,
                   "l2": "flushed (512 MiB write) between timed steps; graph > L2",
                   "graph_gen_s": round(gen_s, 2),
                   "options": args.opt or None,
                   "parallelism": f"{ws} process(es), one GPU each" + ("" if ws == 1 else
                                  ": 1D edge-balanced vertex ranges, per-rank static region and budget, "
                                  "NCCL exchange per iteration (OR / MIN / SUM + slice broadcast)"
                                  + (f"; sparse exchange d={args.sparse_exchange}, "
                                     f"{sum(s_['sparse_exchanges'] for s_ in per)} sparse iterations"
                                     if args.sparse_exchange else ""))},
           "gteps_excl_fill": value_excl_fill,
           "graph500_gteps": (g500_edges / (total_ms / 1e3) / 1e9) if algo == "bfs" else None,
           "roofline": roofline, "link": link, "cpu_baseline": cpu, "e2e": e2e,
           "gpu_launches": int(sum(s["kernel_launches"] for s in per)),
           "library_ms_per_step": lib_ms / args.steps,
           "clocks": clk}
    if rank == 0:
        print(json.dumps(out), flush=True)
    asc.unload()
    if cleanup is not None:
        cleanup()
    if ws > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
