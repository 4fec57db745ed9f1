"""Per-iteration miss-run profile of one run (dev tool, GPU): how the miss payload of each
iteration splits by run length, how long the gaps between consecutive runs are, and what each
iteration's transfer achieved. Active sets come from the library itself (results after t
iterations, Jacobi semantics), so no oracle is involved.

    python tools/run_profile.py --config c4 [--scale 22]
"""
import argparse
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen as gg                              # noqa: E402
import paper_conf_icpp_tangzwgzwy21_b200 as asc    # noqa: E402

BUCKETS = [0, 256, 1024, 4096, 16384, 65536, 262144, 1 << 20, 1 << 62]


def runs_of(mask):
    """maximal runs [b, e) of True in mask"""
    m = np.concatenate([[False], mask, [False]]).astype(np.int8)
    d = np.diff(m)
    return np.nonzero(d == 1)[0], np.nonzero(d == -1)[0]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c4")
    ap.add_argument("--scale", type=int, default=None)
    args = ap.parse_args()
    c = gg.CONFIGS[args.config]
    algo = c["algo"] if c["algo"] != "bfs+pr" else "bfs"
    g = gg.config_graph(args.config, scale_override=args.scale)
    budget = gg.config_budget(args.config, g)
    off = g.off.astype(np.int64)
    src = gg.sources(g, 1, seed=c["seed"])[0] if algo in ("bfs", "sssp") else 0
    asc.set_device(0)
    asc.load_csr(g.off, g.nbr, pairs=g.pairs, symmetric=True)
    asc.set_budget(budget)
    asc.run(algo, src, 0)
    asc.run(algo, src, 0)
    st, its = asc.stats()
    s = st["s"]
    b_e = g.b_e
    print(f"{args.config} {algo} n={g.n} m={g.m} s={s} run {st['time_run_s'] * 1e3:.1f} ms "
          f"fill {st['time_fill_s'] * 1e3:.1f} ms payload {st['h2d_payload_bytes'] / 1e9:.3f} GB "
          f"gather {st['gather_bytes'] / 1e9:.2f} GB in {st['time_gather_s'] * 1e3:.1f} ms "
          f"dma {st['dma_bytes'] / 1e9:.2f} GB in {st['time_dma_s'] * 1e3:.1f} ms", flush=True)
    prev = None
    for t, it in enumerate(its):
        # A_t from the results after t and t-1 iterations
        if algo == "bfs":
            asc.run(algo, src, t + 1)
            lv = asc.get_result().copy()
            act = lv == t
        else:
            # A_0 = V (CC) or {src} (SSSP); A_t = {v : r_t < r_(t-1)}, r_t = values after t iterations
            if t == 0:
                act = np.zeros(g.n, bool)
                if algo == "cc":
                    act[:] = True
                    prev = np.arange(g.n, dtype=np.uint32)
                else:
                    act[src] = True
                    prev = np.full(g.n, 0xFFFFFFFF, dtype=np.uint32)
                    prev[src] = 0
            else:
                asc.run(algo, src, t)
                cur = asc.get_result().copy()
                act = cur < prev
                prev = cur
        miss = act.copy()
        miss[:s] = False
        b, e = runs_of(miss)
        rb = b_e * (off[e] - off[b])
        assert int(rb.sum()) == it["miss_bytes"], (t, int(rb.sum()), it["miss_bytes"])
        gaps = b_e * (off[b[1:]] - off[e[:-1]]) if b.size > 1 else np.zeros(0, np.int64)
        hist = np.histogram(rb, bins=BUCKETS, weights=rb)[0] / max(1, rb.sum())
        gh = [float((gaps < x).mean()) if gaps.size else 0.0 for x in (16, 64, 128, 256, 1024)]
        gbs = it["miss_bytes"] / max(1e-9, it["ms_h2d"] * 1e-3) / 1e9
        print(f"t={t} |A|={it['nA']} |M|={it['nM']} runs={it['nruns']} miss={it['miss_bytes'] / 1e6:.1f} MB "
              f"avg_run={rb.mean() if rb.size else 0:.0f} B mode={it['mode']} h2d={it['ms_h2d']:.2f} ms ({gbs:.1f} GB/s)",
              flush=True)
        print("   payload share by run bytes " + " ".join(f"<{BUCKETS[i + 1]}:{hist[i]:.3f}" for i in range(len(hist) - 1)))
        print("   gap fraction below 16/64/128/256/1024 B: " + " ".join(f"{x:.3f}" for x in gh)
              + f"  gap bytes / payload {gaps.sum() / max(1, rb.sum()):.3f}")
        # how much of the payload sits in host windows of W bytes that are >= 85 % payload (span-DMA
        # candidates at that window size)
        if b.size:
            hb = b_e * off[b]
            he = b_e * off[e]
            h0 = int(hb[0])
            parts = []
            for W in (1 << 20, 4 << 20, 16 << 20, 64 << 20, 256 << 20):
                nwin = int((int(he[-1]) - h0 + W - 1) // W)
                pay = np.zeros(nwin + 1, dtype=np.int64)
                # payload per window: split each run at window boundaries (runs are sorted and disjoint)
                cb = np.cumsum(np.concatenate([[0], (he - hb)]))          # payload before run i
                edges = h0 + W * np.arange(nwin + 1, dtype=np.int64)
                # payload below host position x = cb[j] + clip(x - hb[j], 0, len_j), j = last run with hb <= x
                j = np.searchsorted(hb, edges, side="right") - 1
                jj = np.clip(j, 0, hb.size - 1)
                below = np.where(j < 0, 0, cb[jj] + np.clip(edges - hb[jj], 0, he[jj] - hb[jj]))
                pay = np.diff(below)
                dense = pay >= 0.85 * W
                parts.append(f"W={W >> 20}MiB:{pay[dense].sum() / max(1, pay.sum()):.3f}")
            print("   payload share in >=85%-dense host windows " + " ".join(parts))
    asc.unload()


if __name__ == "__main__":
    main()
