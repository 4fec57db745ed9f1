// frontier.cu — GenDataMap + StaticNodes/On-demandNodes generation in ONE pass.
//
// Paper: StaticMap = ActiveBitmap AND StaticBitmap, On-demand Map = StaticMap XOR
// ActiveBitmap (Fig. 4; §3.1); StaticNodes are
// generated from StaticMap and handed to the Manager; On-demandNodes
// with their Degree generate the data request.
//
// B200 design (DESIGN.md §"Kernels / classify"): one CTA = 8 warps = 256 bitmap
// words = 8192 vertices. Each warp owns 32 consecutive words; per word every lane
// classifies one vertex with register bit ops (AND / AND-NOT, never materialising
// the maps), reads off[v], off[v+1] only for active vertices (coalesced 8-byte
// loads), and ballots/popcounts its class. The order-preserving compaction of the
// hit queues (3 degree buckets), the miss queue (+64-bit arc prefix) and the
// maximal miss runs (+64-bit destination offsets) is ONE decoupled look-back scan
// over a 32-byte multi-field value. Run ends are paired with run starts by rank,
// so a run may span any number of tiles. The last CTA to finish writes the totals
// straight into mapped pinned host memory: that is the only D2H per iteration.
#include "ascetic_internal.h"

namespace ascetic {

namespace {

constexpr unsigned FULL = 0xFFFFFFFFu;
constexpr unsigned long long PHI = 0x9E3779B97F4A7C15ull;

__device__ __forceinline__ unsigned long long mix64(unsigned long long z) {
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

// bits of word w that fall in the vertex range [vlo, vhi)
__device__ __forceinline__ uint32_t own_mask(uint32_t w, unsigned long long vlo, unsigned long long vhi) {
    const unsigned long long b = (unsigned long long)w * 32ull;
    const unsigned long long lo = vlo > b ? vlo : b;
    const unsigned long long hi = vhi < b + 32 ? vhi : b + 32;
    if (lo >= hi) return 0u;
    const uint32_t top = (uint32_t)(hi - b), bot = (uint32_t)(lo - b);
    const uint32_t upto = top == 32 ? FULL : ((1u << top) - 1u);
    return upto & ~((1u << bot) - 1u);
}

__device__ __forceinline__ unsigned long long wsum64(unsigned long long x) {
#pragma unroll
    for (int d = 16; d; d >>= 1) x += __shfl_xor_sync(FULL, x, d);
    return x;
}

__device__ __forceinline__ unsigned long long wexcl64(unsigned long long x, int lane) {
    unsigned long long inc = x;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        unsigned long long y = __shfl_up_sync(FULL, inc, d);
        if (lane >= d) inc += y;
    }
    return inc - x;
}

__device__ __forceinline__ uint32_t wexcl32(uint32_t x, int lane) {
    uint32_t inc = x;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        uint32_t y = __shfl_up_sync(FULL, inc, d);
        if (lane >= d) inc += y;
    }
    return inc - x;
}

__device__ __forceinline__ ScanVal sv_zero() {
    ScanVal z;
    z.small = z.med = z.hub = z.missq = z.runs = z.pieces = 0;
    z.miss_arcs = 0;
    return z;
}

__device__ __forceinline__ ScanVal sv_add(const ScanVal& a, const ScanVal& b) {
    ScanVal r;
    r.small = a.small + b.small;
    r.med = a.med + b.med;
    r.hub = a.hub + b.hub;
    r.missq = a.missq + b.missq;
    r.runs = a.runs + b.runs;
    r.pieces = a.pieces + b.pieces;
    r.miss_arcs = a.miss_arcs + b.miss_arcs;
    return r;
}

__device__ __forceinline__ ScanVal sv_warp_sum(ScanVal v) {
    ScanVal r;
    r.small = __reduce_add_sync(FULL, v.small);
    r.med = __reduce_add_sync(FULL, v.med);
    r.hub = __reduce_add_sync(FULL, v.hub);
    r.missq = __reduce_add_sync(FULL, v.missq);
    r.runs = __reduce_add_sync(FULL, v.runs);
    r.pieces = __reduce_add_sync(FULL, v.pieces);
    r.miss_arcs = wsum64(v.miss_arcs);
    return r;
}

__device__ __forceinline__ void sv_store_volatile(ScanVal* p, const ScanVal& v) {
    volatile uint32_t* q = reinterpret_cast<volatile uint32_t*>(p);
    q[0] = v.small; q[1] = v.med; q[2] = v.hub; q[3] = v.missq; q[4] = v.runs; q[5] = v.pieces;
    *reinterpret_cast<volatile unsigned long long*>(&p->miss_arcs) = v.miss_arcs;
}

__device__ __forceinline__ ScanVal sv_load_volatile(const ScanVal* p) {
    const volatile uint32_t* q = reinterpret_cast<const volatile uint32_t*>(p);
    ScanVal v;
    v.small = q[0]; v.med = q[1]; v.hub = q[2]; v.missq = q[3]; v.runs = q[4]; v.pieces = q[5];
    v.miss_arcs = *reinterpret_cast<const volatile unsigned long long*>(&p->miss_arcs);
    return v;
}

// WPW = bitmap words per warp: 32 (a tile = 8192 vertices) or, for small bitmaps that would leave most
// SMs idle, 4 (a tile = 1024 vertices: each warp's serial walk over its words is 8x shorter, which is
// what bounds a small graph's classify, ~30 us at C1's 8 tiles of 32 words)
template <int WPW>
__global__ void __launch_bounds__(kClassifyWarps * 32, 4) k_classify(ClassifyArgs a) {
    __shared__ uint32_t s_tile;
    __shared__ ScanVal s_warp[kClassifyWarps];
    __shared__ ScanVal s_excl;
    __shared__ unsigned long long s_ns[kClassifyWarps][6];

    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint32_t lt = (1u << lane) - 1u;
    const uint32_t le = lt | (1u << lane);
    if (threadIdx.x == 0) s_tile = atomicAdd(&a.tot->tile_counter, 1u);
    __syncthreads();
    const uint32_t tile = s_tile;
    const uint32_t w0 = tile * (kClassifyWarps * WPW) + warp * WPW;
    const uint32_t myw = w0 + lane;
    const bool mine_w = lane < WPW && myw < a.nwords;

    // A is replicated across ranks; this rank classifies only its owned range [vlo, vhi)
    // while |A| and the digest are taken over the whole bitmap.
    uint32_t myAll = 0, myS = 0;
    if (mine_w) { myAll = __ldg(a.A + myw); myS = __ldg(a.S + myw); }
    const uint32_t myA = myAll & own_mask(myw, a.vlo, a.vhi);
    const uint32_t myMiss = myA & ~myS;
    uint32_t prevMiss = 0, nextMiss = 0;
    if (w0 > 0 && w0 - 1 < a.nwords)
        prevMiss = __ldg(a.A + w0 - 1) & ~__ldg(a.S + w0 - 1) & own_mask(w0 - 1, a.vlo, a.vhi);
    if (w0 + WPW < a.nwords)
        nextMiss = __ldg(a.A + w0 + WPW) & ~__ldg(a.S + w0 + WPW) & own_mask(w0 + WPW, a.vlo, a.vhi);
    const uint32_t anyA = __ballot_sync(FULL, myA != 0);
    const uint32_t piece = a.piece_arcs;

    // Both phases walk the warp's 32 words one at a time (prefix order), but the offsets of the active
    // vertices are loaded kBatch words ahead: with few CTAs (small graphs) each dependent off[] load
    // chain costs ~0.5 us, so one load round trip per word made a C1 classify ~20 us.
    constexpr int kBatch = WPW < 8 ? WPW : 8;
    // ---------------- phase A: per-warp counts
    ScanVal mine = sv_zero();
    unsigned long long aArcs = 0, hArcs = 0;
    unsigned long long degA[kBatch];
    for (int j = 0; j < WPW; ++j) {
        if ((j & (kBatch - 1)) == 0) {
            const uint32_t any8 = (anyA >> j) & ((1u << kBatch) - 1u);
#pragma unroll
            for (int u = 0; u < kBatch; ++u) {
                degA[u] = 0;
                if ((any8 >> u) & 1u) {                      // warp-uniform
                    const uint32_t awu = __shfl_sync(FULL, myA, j + u);
                    const unsigned long long vu = (unsigned long long)(w0 + j + u) * 32ull + lane;
                    if ((awu >> lane) & 1u) degA[u] = __ldg(a.off + vu + 1) - __ldg(a.off + vu);
                }
            }
        }
        if (!((anyA >> j) & 1u)) continue;                    // warp-uniform
        const uint32_t aw = __shfl_sync(FULL, myA, j);
        const uint32_t sw = __shfl_sync(FULL, myS, j);
        const uint32_t pm = __shfl_sync(FULL, myMiss, (j + 31) & 31);
        const uint32_t carry_in = (j == 0 ? prevMiss : pm) >> 31;
        const bool act = (aw >> lane) & 1u;
        unsigned long long deg = 0;
#pragma unroll
        for (int u = 0; u < kBatch; ++u)
            if ((j & (kBatch - 1)) == u) deg = degA[u];
        const bool st = (sw >> lane) & 1u;
        const bool hit = act && st, miss = act && !st;
        aArcs += deg;
        if (hit) {
            hArcs += deg;
            if (deg > 0) {
                if (deg < kSmallDeg) mine.small++;
                else if (deg < a.hub_deg) mine.med++;
                else { mine.hub++; mine.pieces += (uint32_t)((deg + piece - 1) / piece); }
            }
        }
        if (miss) {
            mine.miss_arcs += deg;
            if (deg > 0) mine.missq++;
        }
        const uint32_t mw = aw & ~sw;
        const uint32_t starts = mw & ~((mw << 1) | carry_in);
        if (lane == 0) mine.runs += __popc(starts);
    }
    ScanVal wagg = sv_warp_sum(mine);
    {
        unsigned long long nA = __popc(myAll), nH = __popc(myA & myS), nM = __popc(myMiss);
        unsigned long long nS = wsum64((unsigned long long)__popc(myS & own_mask(myw, a.vlo, a.vhi)));
        if (lane == 0 && nS) atomicAdd(&a.tot->nS, nS);
        unsigned long long dg = mine_w ? mix64((unsigned long long)myw ^ ((unsigned long long)myAll * PHI)) : 0ull;
        nA = wsum64(nA); nH = wsum64(nH); nM = wsum64(nM); dg = wsum64(dg);
        aArcs = wsum64(aArcs); hArcs = wsum64(hArcs);
        if (lane == 0) {
            s_warp[warp] = wagg;
            s_ns[warp][0] = nA; s_ns[warp][1] = nH; s_ns[warp][2] = nM;
            s_ns[warp][3] = aArcs; s_ns[warp][4] = hArcs; s_ns[warp][5] = dg;
        }
    }
    __syncthreads();

    // ---------------- block aggregate + decoupled look-back (warp 0)
    if (warp == 0) {
        ScanVal agg = sv_zero();
        if (lane == 0) {
            for (int w = 0; w < kClassifyWarps; ++w) {
                ScanVal x = s_warp[w];
                s_warp[w] = agg;            // becomes the warp's exclusive offset in the block
                agg = sv_add(agg, x);
            }
            if (tile == 0) {
                sv_store_volatile(&a.tile_incl[0], agg);
                __threadfence();
                *reinterpret_cast<volatile uint32_t*>(&a.tile_flag[0]) = (a.epoch << 2) | 2u;
            } else {
                sv_store_volatile(&a.tile_agg[tile], agg);
                __threadfence();
                *reinterpret_cast<volatile uint32_t*>(&a.tile_flag[tile]) = (a.epoch << 2) | 1u;
            }
        }
        ScanVal excl = sv_zero();
        if (tile > 0) {
            int base = (int)tile - 1;
            while (true) {
                const int idx = base - lane;
                uint32_t st = 2;
                ScanVal val = sv_zero();
                if (idx >= 0) {
                    uint32_t f;
                    do {
                        f = *reinterpret_cast<volatile uint32_t*>(&a.tile_flag[idx]);
                    } while ((f >> 2) != a.epoch || (f & 3u) == 0u);
                    __threadfence();
                    st = f & 3u;
                    val = sv_load_volatile(st == 2 ? &a.tile_incl[idx] : &a.tile_agg[idx]);
                }
                const uint32_t incl_mask = __ballot_sync(FULL, st == 2);
                const int stop = incl_mask ? (__ffs(incl_mask) - 1) : 31;
                ScanVal c = (lane <= stop) ? val : sv_zero();
                excl = sv_add(excl, sv_warp_sum(c));
                if (incl_mask) break;
                base -= 32;
            }
            if (lane == 0) {
                sv_store_volatile(&a.tile_incl[tile], sv_add(excl, agg));
                __threadfence();
                *reinterpret_cast<volatile uint32_t*>(&a.tile_flag[tile]) = (a.epoch << 2) | 2u;
            }
        }
        if (lane == 0) s_excl = excl;
    }
    __syncthreads();

    // ---------------- phase B: scatter with the prefixes
    const ScanVal wb = sv_add(s_excl, s_warp[warp]);
    uint32_t bS = wb.small, bM = wb.med, bH = wb.hub, bQ = wb.missq, bR = wb.runs, bP = wb.pieces;
    unsigned long long bArcs = wb.miss_arcs;
    unsigned long long o0B[kBatch], degB[kBatch];
    for (int j = 0; j < WPW; ++j) {
        if ((j & (kBatch - 1)) == 0) {
            const uint32_t any8 = (anyA >> j) & ((1u << kBatch) - 1u);
#pragma unroll
            for (int u = 0; u < kBatch; ++u) {
                o0B[u] = 0; degB[u] = 0;
                if ((any8 >> u) & 1u) {                      // warp-uniform
                    const uint32_t awu = __shfl_sync(FULL, myA, j + u);
                    const unsigned long long vu = (unsigned long long)(w0 + j + u) * 32ull + lane;
                    if ((awu >> lane) & 1u) { o0B[u] = __ldg(a.off + vu); degB[u] = __ldg(a.off + vu + 1) - o0B[u]; }
                }
            }
        }
        if (!((anyA >> j) & 1u)) continue;
        const uint32_t aw = __shfl_sync(FULL, myA, j);
        const uint32_t sw = __shfl_sync(FULL, myS, j);
        const uint32_t pm = __shfl_sync(FULL, myMiss, (j + 31) & 31);
        const uint32_t nm = __shfl_sync(FULL, myMiss, (j + 1) & 31);
        const uint32_t carry_in = (j == 0 ? prevMiss : pm) >> 31;
        const uint32_t carry_out = (j == WPW - 1 ? nextMiss : nm) & 1u;
        const unsigned long long v = (unsigned long long)(w0 + j) * 32ull + lane;
        const bool act = (aw >> lane) & 1u;
        unsigned long long deg = 0, o0 = 0;
#pragma unroll
        for (int u = 0; u < kBatch; ++u)
            if ((j & (kBatch - 1)) == u) { deg = degB[u]; o0 = o0B[u]; }
        const bool st = (sw >> lane) & 1u;
        const bool hit = act && st, miss = act && !st;
        const uint32_t hw = aw & sw;
        if (hw) {
            const bool isS = hit && deg > 0 && deg < kSmallDeg;
            const bool isM = hit && deg >= kSmallDeg && deg < a.hub_deg;
            const bool isH = hit && deg >= a.hub_deg;
            const uint32_t balS = __ballot_sync(FULL, isS);
            const uint32_t balM = __ballot_sync(FULL, isM);
            const uint32_t balH = __ballot_sync(FULL, isH);
            if (isS) a.hq_small[bS + __popc(balS & lt)] = (uint32_t)v;
            if (isM) a.hq_med[bM + __popc(balM & lt)] = (uint32_t)v;
            if (balH) {
                const uint32_t pc = isH ? (uint32_t)((deg + piece - 1) / piece) : 0u;
                const uint32_t ex = wexcl32(pc, lane);
                if (isH) {
                    const uint32_t k = bH + __popc(balH & lt);
                    a.hq_hub[k] = (uint32_t)v;
                    a.hub_pre[k] = bP + ex;
                }
                bP += __shfl_sync(FULL, ex + pc, 31);
            }
            bS += __popc(balS); bM += __popc(balM); bH += __popc(balH);
        }
        const uint32_t mw = aw & ~sw;
        if (mw) {
            const unsigned long long md = miss ? deg : 0ull;
            const unsigned long long ex = wexcl64(md, lane);
            const unsigned long long tot = __shfl_sync(FULL, ex + md, 31);
            const bool isQ = miss && deg > 0;
            const uint32_t balQ = __ballot_sync(FULL, isQ);
            if (isQ) {
                const uint32_t k = bQ + __popc(balQ & lt);
                const unsigned long long pre = bArcs + ex;
                a.mq[k] = (uint32_t)v;
                a.mq_pre[k] = pre;
                a.mq_src[k] = o0;
                // every miss-stream tile start t*kEdgeTile inside [pre, pre+deg) maps to k
                const unsigned long long t1 = (pre + deg - 1) >> kEdgeTileShift;
                for (unsigned long long t = (pre + kEdgeTile - 1) >> kEdgeTileShift; t <= t1; ++t)
                    a.tile_first[t] = k;
            }
            const uint32_t starts = mw & ~((mw << 1) | carry_in);
            const uint32_t ends = mw & ~((mw >> 1) | (carry_out << 31));
            if ((starts >> lane) & 1u) {
                const uint32_t r = bR + __popc(starts & lt);
                a.run_b[r] = (uint32_t)v;
                a.run_dst[r] = bArcs + ex;
            }
            if ((ends >> lane) & 1u) {
                const uint32_t r = bR + __popc(starts & le) - 1u;
                a.run_e[r] = (uint32_t)(v + 1);
            }
            bQ += __popc(balQ);
            bR += __popc(starts);
            bArcs += tot;
        }
    }

    // ---------------- non-scan totals, completion, totals to host
    // Only the last CTA writes host (mapped) memory, so the others need only a GPU-scope fence before
    // their completion count (a system-scope fence in every CTA cost a PCIe round trip each).
    __shared__ uint32_t s_last;
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned long long t[6] = {0, 0, 0, 0, 0, 0};
        for (int w = 0; w < kClassifyWarps; ++w)
            for (int k = 0; k < 6; ++k) t[k] += s_ns[w][k];
        if (t[0]) atomicAdd(&a.tot->nA, t[0]);
        if (t[1]) atomicAdd(&a.tot->nH, t[1]);
        if (t[2]) atomicAdd(&a.tot->nM, t[2]);
        if (t[3]) atomicAdd(&a.tot->active_arcs, t[3]);
        if (t[4]) atomicAdd(&a.tot->hit_arcs, t[4]);
        atomicAdd(&a.tot->digest, t[5]);                 // Σ mod 2^64
        __threadfence();          // this CTA's queue / run writes before its completion count
        s_last = atomicAdd(&a.tot->done_counter, 1u) == a.ntiles - 1;
    }
    __syncthreads();
    if (!s_last) return;
    __threadfence();
    const ScanVal fin = sv_load_volatile(&a.tile_incl[a.ntiles - 1]);
    // the run list goes to the host only when the host will plan copy-engine DMAs from it (few,
    // long runs, or DMA forced): the first host_runs_cap runs, copied by the whole CTA
    const bool dma = fin.runs && (a.force_host_runs ||
                                  (fin.runs <= a.host_runs_cap && fin.miss_arcs >= (unsigned long long)fin.runs * a.dma_min_run_arcs));
    if (dma) {
        const uint32_t nr = min(fin.runs, a.host_runs_cap);
        const volatile uint32_t* rb = a.run_b;
        const volatile uint32_t* re = a.run_e;
        for (uint32_t r = threadIdx.x; r < nr; r += blockDim.x) {
            a.host_runs[2 * r] = rb[r];
            a.host_runs[2 * r + 1] = re[r];
        }
        __syncthreads();
    }
    if (threadIdx.x == 0) {
        volatile IterTotals* vt = a.tot;
        IterTotals* h = a.host_tot;
        h->nA = vt->nA; h->nH = vt->nH; h->nM = vt->nM; h->nS = vt->nS;
        h->active_arcs = vt->active_arcs; h->hit_arcs = vt->hit_arcs; h->digest = vt->digest;
        h->miss_arcs = fin.miss_arcs;
        h->n_small = fin.small; h->n_med = fin.med; h->n_hub = fin.hub;
        h->n_missq = fin.missq; h->n_runs = fin.runs; h->n_pieces = fin.pieces;
        h->host_runs = dma ? min(fin.runs, a.host_runs_cap) : 0u;
        a.tot->miss_arcs = fin.miss_arcs;
        a.tot->n_small = fin.small; a.tot->n_med = fin.med; a.tot->n_hub = fin.hub;
        a.tot->n_missq = fin.missq; a.tot->n_runs = fin.runs; a.tot->n_pieces = fin.pieces;
        // host span of the miss stream (the queue is in ascending id, so host order): first list's
        // start, last list's end; the other CTAs' queue writes are visible after the done count
        unsigned long long h0 = 0, h1 = 0;
        if (fin.missq) {
            const volatile unsigned long long* src = a.mq_src;
            const volatile unsigned long long* pre = a.mq_pre;
            h0 = src[0];
            h1 = src[fin.missq - 1] + (fin.miss_arcs - pre[fin.missq - 1]);
        }
        h->miss_h0 = h0; h->miss_h1 = h1;
        {   // the next classify's totals start from zero
            unsigned long long* z = reinterpret_cast<unsigned long long*>(a.tot_next);
            for (size_t i = 0; i < sizeof(IterTotals) / 8; ++i) z[i] = 0ull;
        }
        __threadfence_system();   // the CTA's host writes (runs, totals) before the ready flag
        *reinterpret_cast<volatile uint32_t*>(&h->ready) = 1u;
    }
}

}  // namespace

void launch_classify(const ClassifyArgs& a, cudaStream_t s) {
    if (a.ntiles == 0) return;
    if (a.words_per_warp == 4) k_classify<4><<<a.ntiles, kClassifyWarps * 32, 0, s>>>(a);
    else k_classify<32><<<a.ntiles, kClassifyWarps * 32, 0, s>>>(a);
    ++g_launches;
}

}  // namespace ascetic
