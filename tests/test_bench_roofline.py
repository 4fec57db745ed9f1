"""bench.py's roofline entry from per-step library stats (pure function, CPU): the transfer path is
the headline when it fills most of the step, traffic combines copy-engine bytes with the measured
PCIe bytes per SM-gathered payload byte, and HBM-bound steps pick the longest kernel class."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402

STAT_KEYS = ["time_gather_s", "gather_bytes", "time_dma_s", "time_fill_s", "dma_bytes", "h2d_static_fill_bytes",
             "time_ondemand_s", "ondemand_arcs", "time_static_s", "static_arcs", "time_classify_s", "iterations",
             "gather_ce_bytes", "gather_load_bytes", "gather_chunks", "time_h2d_busy_s", "h2d_payload_bytes",
             "span_payload_bytes", "span_link_bytes"]


def _step(**kw):
    s = {k: 0 for k in STAT_KEYS}
    s.update(kw)
    return s


def test_transfer_bound_step_with_gather_and_span():
    # one C4-like step: 6 GB fill + 19.7 GB span (19.75 GB moved) + 8.2 GB gathered
    st = _step(time_gather_s=0.188, gather_bytes=8.2e9, gather_chunks=13, time_dma_s=0.358 + 0.36, time_fill_s=0.108,
               dma_bytes=19.75e9 + 19.72e9, h2d_static_fill_bytes=6.0e9, span_payload_bytes=19.72e9,
               span_link_bytes=19.75e9, h2d_payload_bytes=47.67e9, time_h2d_busy_s=1.01, iterations=6,
               time_ondemand_s=0.09, ondemand_arcs=6.4e9, time_static_s=0.02, static_arcs=2e9, time_classify_s=0.007)
    r = bench.roofline_of([st], 1, 1022.7, 4, 105_000_000, 55.6, 6553.6, "measured", "c4")
    assert r["kernel"] == "transfer" and r["bound"] == "host_link"
    assert abs(r["achieved"] - (6.0e9 + 47.67e9) / 1.01 / 1e9) < 1e-6
    assert abs(r["frac"] - r["achieved"] / 55.6) < 1e-9
    assert r["dominant_kernel"]["name"] == "gather"
    ratio = bench.json.load(open(os.path.join(ROOT, "profiles", "ncu_traffic.json")))["c4"]["gather"]["pcie_read_per_payload"]
    ce = 6.0e9 + (19.75e9 + 19.72e9) - 19.72e9 + 19.75e9
    assert abs(r["traffic"] - (ce + ratio * 8.2e9)) < 1.0
    assert r["per_kernel"]["gather"]["launches"] == 13


def test_hbm_bound_step_picks_longest_class_and_dma_only_config_traffic():
    st = _step(time_static_s=0.05, static_arcs=10e9, time_ondemand_s=0.01, ondemand_arcs=1e9, time_h2d_busy_s=0.01,
               time_fill_s=0.01, h2d_static_fill_bytes=0.5e9, time_classify_s=0.001, iterations=5)
    r = bench.roofline_of([st], 1, 70.0, 4, 1 << 24, 55.6, 6553.6, "measured", "c1")
    assert r["kernel"] == "static" and r["bound"] == "hbm" and r["unit"] == "GB/s"
    # DMA-only out-of-core step (C3-like): traffic = the copy-engine bytes
    st = _step(time_dma_s=2.7, dma_bytes=144.3e9, time_fill_s=0.19, h2d_static_fill_bytes=10.7e9,
               h2d_payload_bytes=144.3e9, time_h2d_busy_s=2.8, iterations=43)
    r = bench.roofline_of([st], 1, 2872.0, 4, 65_608_366, 55.6, 6553.6, "measured", "c3")
    assert r["kernel"] == "transfer" and abs(r["traffic"] - (10.7e9 + 144.3e9)) < 1.0


def test_spans_cover_detects_single_span_iterations():
    # every class with work has event time: the timed steps carry the breakdown
    full = _step(time_gather_s=0.1, gather_bytes=1e9, time_h2d_busy_s=0.1, h2d_payload_bytes=1e9, iterations=3,
                 time_classify_s=0.001, ondemand_arcs=1e6, time_ondemand_s=0.01, static_arcs=1e6, time_static_s=0.01)
    assert bench.spans_cover([full])
    # a C1-like step (TIMING=1: small iterations ran as one span each): work without per-phase time
    c1 = _step(gather_bytes=6e6, h2d_payload_bytes=6e6, iterations=7, time_classify_s=0.0002, ondemand_arcs=1e6)
    assert not bench.spans_cover([full, c1])
    # no work, no time needed
    assert bench.spans_cover([_step()])
