// engine.cu — run controller: placer, partition, transfer engine, per-iteration pipeline.
//
// One iteration (Fig. 4; Fig. 5), B200 version, per rank part:
//   compute stream cs : classify+compact  ──► host reads 96 B of totals (mapped memory)
//   cs                : static-hit kernels (Static Computing)
//   copy stream xs    : chunk k = miss-stream arcs [k*cap, (k+1)*cap) ->
//                       zero-copy SM gather or copy-engine DMA of runs
//                       buffer k%2 waits consumed[k-2]; records ready[k]
//   cs                : waits ready[k] -> on-demand kernel -> records consumed[k]
//   (P > 1)           : exchange: OR bitmaps (BFS) / MIN values (SSSP, CC)
//   cs                : finalize: next active set
//   (P > 1, PR)       : exchange: SUM dangling, share contrib slices
// Fragmenting when the request exceeds the On-demand Region (§3.3) is the
// chunk loop; the static compute overlaps the transfer (§3.2).
#include "engine.h"

#include <algorithm>
#include <array>
#include <atomic>
#include <chrono>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <thread>

namespace ascetic {

#define CK(call)                                                                                   \
    do {                                                                                           \
        cudaError_t e__ = (call);                                                                  \
        if (e__ != cudaSuccess)                                                                    \
            throw Error(ASCETIC_ECUDA, std::string(#call) + ": " + cudaGetErrorString(e__));       \
    } while (0)

enum { ALG_BFS = 0, ALG_SSSP = 1, ALG_CC = 2, ALG_PR = 3, ALG_PRD = 4 };

// ASCETIC_TRACE (the one environment knob; tracing only, never a kernel choice): 1 = print every timed
// span of a run to stderr (rank, iteration, phase, start and end ms), 2 = also split the static-hit
// phase by degree bucket. Either forces per-phase spans in every iteration.
static int trace_level() {
    static const int lv = [] { const char* e = std::getenv("ASCETIC_TRACE"); return e ? std::atoi(e) : 0; }();
    return lv;
}

// ------------------------------------------------------------------ placer / partition
Placement place(const uint64_t* off, uint64_t n, uint32_t b_e, uint64_t budget, double frac) {
    Placement p;
    const double K = 0.10;
    const uint64_t base = off[0];
    p.B = budget;
    p.D = (uint64_t)b_e * (off[n] - base);
    double R;
    if (frac >= 0.0 && frac <= 1.0) {
        R = frac;
    } else {
        R = (1.0 - K * (double)p.D / (double)budget) / (1.0 - K);   // Eq. 2
        if (!(R > 0.0)) R = 0.0;
        if (R > 1.0) R = 1.0;
    }
    p.R = R;
    uint64_t Ms = (uint64_t)std::floor(R * (double)budget / 16384.0) * 16384ull;  // 16 KB chunks
    if (Ms > p.D) Ms = p.D;
    p.Ms = Ms;
    // front prefix of whole lists: s = max{v : b_e (off[v]-base) <= Ms}
    const uint64_t lim = base + Ms / b_e;
    p.s = (uint64_t)(std::upper_bound(off, off + n + 1, lim) - off) - 1;
    p.static_bytes = (uint64_t)b_e * (off[p.s] - base);
    p.C = budget >= Ms ? budget - Ms : 0;
    p.cap = p.C / 2 / 16 * 16;
    return p;
}

std::vector<uint64_t> partition(const uint64_t* off, uint64_t n, uint32_t P) {
    std::vector<uint64_t> b(P + 1);
    const uint64_t m = off[n];
    b[0] = 0;
    for (uint32_t g = 1; g < P; ++g) {
        const uint64_t target = ((uint64_t)g * m + P - 1) / P;
        b[g] = (uint64_t)(std::lower_bound(off, off + n + 1, target) - off);
        if (b[g] > n) b[g] = n;
    }
    b[P] = n;
    return b;
}

// ------------------------------------------------------------------ event pool
cudaEvent_t EventPool::get() {
    if (used == ev.size()) {
        cudaEvent_t e;
        CK(cudaEventCreate(&e));
        ev.push_back(e);
    }
    return ev[used++];
}
EventPool::~EventPool() {
    for (auto e : ev) cudaEventDestroy(e);
}

// ------------------------------------------------------------------ helpers
template <typename T>
static void dalloc(T** p, size_t count, uint64_t* acct) {
    if (count == 0) count = 1;
    cudaError_t e = cudaMalloc((void**)p, count * sizeof(T));
    if (e != cudaSuccess) {
        cudaGetLastError();
        throw Error(ASCETIC_ENOMEM, "cudaMalloc of " + std::to_string(count * sizeof(T)) + " bytes failed");
    }
    if (acct) *acct += count * sizeof(T);
}

template <typename T>
static void dfree(T*& p) {
    if (p) cudaFree((void*)p);
    p = nullptr;
}

void HostGraph::release() {
    if (registered) { cudaHostUnregister(registered); registered = nullptr; reg_bytes = 0; }
    if (owned) { cudaFreeHost(owned); owned = nullptr; }
    nbr = nbr_dev = nullptr;
}

// ================================================================== Part
Part::Part(const HostGraph& g, const Options& o, int rank, uint64_t vlo, uint64_t vhi, int sm_count)
    : g_(g), o_(o), rank_(rank), vlo_(vlo), vhi_(vhi), sm_count_(sm_count) {}

Part::~Part() {
    if (cs_) cudaStreamSynchronize(cs_);
    if (xs_) cudaStreamSynchronize(xs_);
    free_regions();
    dfree(d_off_); dfree(d_A_); dfree(d_S_); dfree(d_next_); dfree(d_visited_); dfree(d_next2_);
    if (d_peers_) { cudaFree((void*)d_peers_); d_peers_ = nullptr; }
    dfree(d_val_); dfree(d_snap_); dfree(d_rank_); dfree(d_contrib_); dfree(d_sum_); dfree(d_dang_);
    dfree(d_pr_r_); dfree(d_pr_res_); dfree(d_pr_c_); dfree(d_pr_inc_);
    dfree(d_hq_small_); dfree(d_hq_med_); dfree(d_hq_hub_); dfree(d_hub_pre_);
    dfree(d_mq_); dfree(d_mq_pre_); dfree(d_mq_src_); dfree(d_tile_first_);
    dfree(d_run_b_); dfree(d_run_e_); dfree(d_run_dst_);
    dfree(d_tile_agg_); dfree(d_tile_incl_); dfree(d_tile_flag_); dfree(d_tot_);
    if (h_tot_) cudaFreeHost(h_tot_);
    if (h_runs_) cudaFreeHost(h_runs_);
    if (h_long_) cudaFreeHost(h_long_);
    if (h_win_) cudaFreeHost(h_win_);
    if (h_span_flag_) cudaFreeHost(h_span_flag_);
    if (h_long_flag_) cudaFreeHost(h_long_flag_);
    for (int i = 0; i < 2; ++i) { if (h_lint_[i]) cudaFreeHost(h_lint_[i]); dfree(d_lint_[i]); }
    dfree(d_long_cnt_); dfree(d_cover_); dfree(d_seg_cur_);
    if (h_cover_) { cudaFreeHost(h_cover_); h_cover_ = nullptr; }
    for (int i = 0; i < kMaxBuffers; ++i) {
        if (ce_done_[i]) cudaEventDestroy(ce_done_[i]);
        if (xfer_go_[i]) cudaEventDestroy(xfer_go_[i]);
    }
    if (xs2_) { cudaStreamSynchronize(xs2_); cudaStreamDestroy(xs2_); }
    for (cudaStream_t& x : xs34_) if (x) { cudaStreamSynchronize(x); cudaStreamDestroy(x); x = nullptr; }
    for (int i = 0; i < kMaxBuffers; ++i) {
        if (ready_[i]) cudaEventDestroy(ready_[i]);
        if (consumed_[i]) cudaEventDestroy(consumed_[i]);
    }
    if (ev_classified_) cudaEventDestroy(ev_classified_);
    if (ev_long_) cudaEventDestroy(ev_long_);
    if (ev_pipe_) cudaEventDestroy(ev_pipe_);
    free_hot();
    if (ev_acc_) cudaEventDestroy(ev_acc_);
    if (ev_swapped_) cudaEventDestroy(ev_swapped_);
    if (static_go_) cudaEventDestroy(static_go_);
    if (static_done_) cudaEventDestroy(static_done_);
    if (sync_ev_) cudaEventDestroy(sync_ev_);
    if (ss_) { cudaStreamSynchronize(ss_); cudaStreamDestroy(ss_); }
    if (cs_) cudaStreamDestroy(cs_);
    if (xs_) cudaStreamDestroy(xs_);
    cudaGetLastError();
}

void Part::alloc_vertex_state() {
    // priorities (numerically lower = higher): the transfer stream first (its gather CTAs are
    // few and must stay resident to keep the link busy); on-demand and static-hit kernels
    // share the SMs at equal priority (measured: starving the static kernels stretches PR
    // iterations, whose static pull is HBM-bound, by 20 %).
    int lo_pri = 0, hi_pri = 0;
    CK(cudaDeviceGetStreamPriorityRange(&lo_pri, &hi_pri));
    CK(cudaStreamCreateWithPriority(&cs_, cudaStreamNonBlocking, lo_pri));
    CK(cudaStreamCreateWithPriority(&xs_, cudaStreamNonBlocking, hi_pri));
    CK(cudaStreamCreateWithPriority(&ss_, cudaStreamNonBlocking, lo_pri));
    CK(cudaStreamCreateWithPriority(&xs2_, cudaStreamNonBlocking, hi_pri));
    for (cudaStream_t& x : xs34_) CK(cudaStreamCreateWithPriority(&x, cudaStreamNonBlocking, hi_pri));
    for (int i = 0; i < kMaxBuffers; ++i) {
        CK(cudaEventCreateWithFlags(&ready_[i], cudaEventDisableTiming));
        CK(cudaEventCreateWithFlags(&consumed_[i], cudaEventDisableTiming));
        CK(cudaEventCreateWithFlags(&ce_done_[i], cudaEventDisableTiming));
        CK(cudaEventCreateWithFlags(&xfer_go_[i], cudaEventDisableTiming));
    }
    CK(cudaEventCreateWithFlags(&static_go_, cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&static_done_, cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&sync_ev_, cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&ev_classified_, cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&ev_long_, cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&ev_pipe_, cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&ev_acc_, cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&ev_swapped_, cudaEventDisableTiming));
    const uint64_t n = g_.n, m = g_.m;
    vertex_bytes_ = 0;
    nwords_ = (uint32_t)((n + 31) / 32);
    // classify tiles: 32 words per warp, or 4 when that would leave more than half the SMs idle
    wpw_ = (nwords_ + kTileWords - 1) / kTileWords < (uint32_t)(2 * sm_count_) ? 4u : 32u;
    ntiles_ = (nwords_ + kClassifyWarps * wpw_ - 1) / (kClassifyWarps * wpw_);
    dalloc(&d_off_, n + 1, &vertex_bytes_);
    dalloc(&d_A_, nwords_, &vertex_bytes_);
    dalloc(&d_S_, nwords_, &vertex_bytes_);
    dalloc(&d_next_, nwords_, &vertex_bytes_);
    const uint64_t own = vhi_ - vlo_;
    dalloc(&d_hq_small_, own, &vertex_bytes_);
    dalloc(&d_hq_med_, own, &vertex_bytes_);
    hub_cap_ = std::min<uint64_t>(own, m / o_.hub_deg + 1);       // at most m / hub_deg hubs
    dalloc(&d_hq_hub_, hub_cap_, &vertex_bytes_);
    dalloc(&d_hub_pre_, hub_cap_, &vertex_bytes_);
    dalloc(&d_mq_, own, &vertex_bytes_);
    dalloc(&d_mq_pre_, own + 2, &vertex_bytes_);   // +2: the gather's TMA copies whole 16-byte pairs
    dalloc(&d_mq_src_, own + 2, &vertex_bytes_);
    dalloc(&d_tile_first_, (m >> kEdgeTileShift) + 2, &vertex_bytes_);
    dalloc(&d_run_b_, own / 2 + 1, &vertex_bytes_);
    dalloc(&d_run_e_, own / 2 + 1, &vertex_bytes_);
    dalloc(&d_run_dst_, own / 2 + 1, &vertex_bytes_);
    dalloc(&d_tile_agg_, ntiles_, &vertex_bytes_);
    dalloc(&d_tile_incl_, ntiles_, &vertex_bytes_);
    dalloc(&d_tile_flag_, ntiles_, &vertex_bytes_);
    dalloc(&d_tot_, 2, &vertex_bytes_);   // double-buffered: classify t zeroes the buffer of t+1
    CK(cudaMemset(d_tot_, 0, 2 * sizeof(IterTotals)));
    tot_buf_ = 0;
    CK(cudaMemset(d_tile_flag_, 0, (size_t)std::max<uint32_t>(ntiles_, 1) * 4));
    CK(cudaMemset(d_S_, 0, (size_t)std::max<uint32_t>(nwords_, 1) * 4));
    epoch_ = 0;
    cudaError_t e = cudaHostAlloc((void**)&h_tot_, sizeof(IterTotals), cudaHostAllocMapped | cudaHostAllocPortable);
    if (e != cudaSuccess) { cudaGetLastError(); throw Error(ASCETIC_EHOSTMEM, "cudaHostAlloc totals"); }
    e = cudaHostAlloc((void**)&h_runs_, 2ull * kRunsHostMax * sizeof(uint32_t), cudaHostAllocMapped | cudaHostAllocPortable);
    if (e != cudaSuccess) { cudaGetLastError(); throw Error(ASCETIC_EHOSTMEM, "cudaHostAlloc run list"); }
    e = cudaHostAlloc((void**)&h_win_, 8ull * (kSpanWinMax + 1), cudaHostAllocMapped | cudaHostAllocPortable);
    if (e == cudaSuccess) e = cudaHostAlloc((void**)&h_span_flag_, 8, cudaHostAllocMapped | cudaHostAllocPortable);
    if (e != cudaSuccess) { cudaGetLastError(); throw Error(ASCETIC_EHOSTMEM, "cudaHostAlloc span windows"); }
    e = cudaHostAlloc((void**)&h_long_, 3ull * kLongMax * 8, cudaHostAllocMapped | cudaHostAllocPortable);
    if (e == cudaSuccess) e = cudaHostAlloc((void**)&h_long_flag_, 8, cudaHostAllocMapped | cudaHostAllocPortable);
    for (int i = 0; i < 2 && e == cudaSuccess; ++i) e = cudaHostAlloc((void**)&h_lint_[i], 2ull * kLongMax * 8, cudaHostAllocPortable);
    if (e != cudaSuccess) { cudaGetLastError(); throw Error(ASCETIC_EHOSTMEM, "cudaHostAlloc long-run lists"); }
    dalloc(&d_long_cnt_, 2, &vertex_bytes_);
    for (int i = 0; i < 2; ++i) dalloc(&d_lint_[i], 2ull * kLongMax, &vertex_bytes_);
    dalloc(&d_cover_, 1, &vertex_bytes_);
    CK(cudaMallocHost(&h_cover_, sizeof(unsigned long long)));
}

void Part::alloc_algo_state(int algo, bool multi) {
    multi_ = multi;
    if (algo == ALG_PRD) {
        if (!d_pr_r_) {
            dalloc(&d_pr_r_, g_.n, &vertex_bytes_);
            dalloc(&d_pr_res_, g_.n, &vertex_bytes_);
            dalloc(&d_pr_c_, g_.n, &vertex_bytes_);
        }
        if (multi && !d_pr_inc_) {
            dalloc(&d_pr_inc_, g_.n, &vertex_bytes_);
            CK(cudaMemset(d_pr_inc_, 0, g_.n * 8));
        }
        if (!d_rank_) dalloc(&d_rank_, g_.n, &vertex_bytes_);
    } else if (algo == ALG_PR) {
        if (!d_rank_) {
            dalloc(&d_rank_, g_.n, &vertex_bytes_);
            dalloc(&d_contrib_, g_.n, &vertex_bytes_);
            dalloc(&d_sum_, g_.n, &vertex_bytes_);
            dalloc(&d_dang_, 2, &vertex_bytes_);
        }
    } else {
        if (!d_val_) dalloc(&d_val_, g_.n, &vertex_bytes_);
        if (algo == ALG_BFS && !d_visited_) dalloc(&d_visited_, nwords_, &vertex_bytes_);
        if (algo != ALG_BFS && !d_snap_) dalloc(&d_snap_, g_.n, &vertex_bytes_);
    }
    if (o_.hub_deg < 2048) {
        const uint64_t need = std::min<uint64_t>(vhi_ - vlo_, g_.m / o_.hub_deg + 1);
        if (need > hub_cap_) {
            dfree(d_hq_hub_); dfree(d_hub_pre_);
            dalloc(&d_hq_hub_, need, &vertex_bytes_);
            dalloc(&d_hub_pre_, need, &vertex_bytes_);
            hub_cap_ = need;
        }
    }
}

void Part::upload_off() {
    CK(cudaMemcpyAsync(d_off_, g_.off, (g_.n + 1) * sizeof(uint64_t), cudaMemcpyHostToDevice, cs_));
    static_valid_ = false;
}

void Part::free_regions() {
    dfree(arena_);
    arena_bytes_ = 0;
    d_static_ = nullptr;
    for (int i = 0; i < kMaxBuffers; ++i) d_chunk_[i] = nullptr;
    static_alloc_ = chunk_alloc_ = 0;
    nbuf_alloc_ = 0;
    static_valid_ = false;
}

// The edge budget is ONE arena of at most B bytes: the Static Region is its front
// [0, static_bytes) ⊆ [0, Ms), the On-demand Region [Ms, arena) is cut into nbuf_ chunk buffers.
// Moving Ms (Eq. 3 re-partition) keeps the static prefix in place and re-cuts the rest.
void Part::layout_regions(uint64_t Ms) {
    d_static_ = arena_;
    const uint64_t per = arena_bytes_ > Ms ? (arena_bytes_ - Ms) / (uint64_t)nbuf_ / 16 * 16 : 0;
    for (int i = 0; i < kMaxBuffers; ++i) d_chunk_[i] = (per && i < nbuf_) ? arena_ + Ms + (uint64_t)i * per : nullptr;
    chunk_alloc_ = per;
    cap_ = per;   // chunk-cap option (tuning only): never above the buffer
    if (o_.chunk_cap && o_.chunk_cap < cap_) cap_ = std::max<uint64_t>(16, o_.chunk_cap / 16 * 16);
}

void Part::set_budget(uint64_t bytes, double frac) {
    Placement p = place(g_.off + vlo_, vhi_ - vlo_, g_.b_e, bytes, frac);
    const uint64_t own = vhi_ - vlo_;
    stat_lo_ = vlo_;
    if (o_.placement == 1) {
        // rear initial content (§5): the suffix of whole lists that fits in Ms,
        // s_lo = min{v : b_e (off[vhi] - off[v]) <= Ms}
        const uint64_t* off = g_.off;
        const uint64_t lim = off[vhi_] - std::min<uint64_t>(p.Ms / g_.b_e, off[vhi_]);
        stat_lo_ = (uint64_t)(std::lower_bound(off + vlo_, off + vhi_ + 1, lim) - off);
        p.s = vhi_ - stat_lo_;
        p.static_bytes = (uint64_t)g_.b_e * (off[vhi_] - off[stat_lo_]);
    }
    if (p.s < own && p.cap < 16)
        throw Error(ASCETIC_ENOMEM, "budget leaves an On-demand chunk below 16 bytes (cap=" + std::to_string(p.cap) + ")");
    // On-demand Region C split into nb chunk buffers of floor(C/nb/16)*16 bytes (the placer's
    // `cap` is the 2-buffer figure; more buffers give the pipeline slack, same C)
    // auto (0): 3 buffers, or 2 when a third of C is under 4 MiB: per-chunk latency (~25 us of
    // gather + on-demand launch) then dominates and fewer, larger chunks win (C1 A/B on B200:
    // 2 / 3 / 4 buffers = 0.99 / 1.14 / 1.29 ms per run, profiles/r01/c1_chunk_buffers.log)
    const int nb = o_.chunk_buffers ? std::max(2, std::min(kMaxBuffers, o_.chunk_buffers))
                                    : (p.C / 3 < (4ull << 20) ? 2 : 3);
    // chunk buffers never need more than the rank's whole payload D
    const uint64_t per_buf = std::min<uint64_t>(p.C / (uint64_t)nb, std::max<uint64_t>(p.D, 16)) / 16 * 16;
    if (p.s < own && per_buf < 16)
        throw Error(ASCETIC_ENOMEM, "budget leaves an On-demand chunk below 16 bytes");
    // arena = Ms + nb chunk buffers (<= B); just the static prefix when everything is static
    const uint64_t want = std::max<uint64_t>(16, p.s < own ? p.Ms + (uint64_t)nb * per_buf : p.static_bytes);
    if (want != arena_bytes_ || nb != nbuf_alloc_) {
        free_regions();
        cudaError_t e = cudaMalloc((void**)&arena_, want);
        if (e != cudaSuccess) { cudaGetLastError(); throw Error(ASCETIC_ENOMEM, "edge-budget arena allocation"); }
        arena_bytes_ = want;
        nbuf_alloc_ = nb;
    } else if (p.s != pl_.s) {
        static_valid_ = false;
    }
    static_alloc_ = p.static_bytes;
    nbuf_ = nb;
    pl_ = p;
    ms_cur_ = p.Ms;
    s_cur_ = p.s;
    layout_regions(p.Ms);
    launch_set_range_bits(d_S_, nwords_, stat_lo_, stat_lo_ + p.s, cs_);   // StaticBitmap
    // §3.4 data replacement and the random initial content (§5): the Static Region
    // becomes ceil(Ms / 16 KiB) chunk slots, filled whole; only meaningful when some lists stay
    // outside it
    if (o_.replace_k > 0 && o_.placement == 1) throw Error(ASCETIC_EINVAL, "replacement needs the front or random placement");
    hot_ = (o_.replace_k > 0 || o_.placement == 2) && p.s < own && p.Ms > 0;
    if (hot_) {
        hNC_ = (p.D + kChunkBytes - 1) / kChunkBytes;
        hNS_ = (p.Ms + kChunkBytes - 1) / kChunkBytes;
        if (hNC_ > 0xFFFFFFF0ull) throw Error(ASCETIC_EINVAL, "too many 16 KiB chunks for replacement");
        init_chunks_.resize(hNS_);
        if (o_.placement == 2) {
            // the hNS_ chunks with the smallest splitmix64((seed << 32) ^ c), ties by c (DESIGN R27)
            std::vector<std::pair<uint64_t, uint32_t>> key(hNC_);
            for (uint64_t c = 0; c < hNC_; ++c) {
                uint64_t z = (o_.placement_seed << 32) ^ c;
                z += 0x9E3779B97F4A7C15ull;
                z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
                z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
                key[c] = {z ^ (z >> 31), (uint32_t)c};
            }
            std::nth_element(key.begin(), key.begin() + (hNS_ - 1), key.end());
            for (uint64_t i = 0; i < hNS_; ++i) init_chunks_[i] = key[i].second;
            std::sort(init_chunks_.begin(), init_chunks_.end());
        } else {
            for (uint64_t i = 0; i < hNS_; ++i) init_chunks_[i] = (uint32_t)i;
        }
        init_fill_bytes_ = 0;
        for (uint32_t c : init_chunks_) init_fill_bytes_ += std::min<uint64_t>(kChunkBytes, p.D - (uint64_t)c * kChunkBytes);
        if (hNC_ != hot_alloc_nc_ || o_.replace_k != hot_alloc_k_) {
            free_hot();
            dalloc(&d_slot_of_, hNC_, nullptr);
            dalloc(&d_acc_, hNC_, nullptr);
            dalloc(&d_init_, hNC_, nullptr);
            dalloc(&d_swap_, 3ull * std::max<uint32_t>(o_.replace_k, 1), nullptr);
            cudaError_t e = cudaHostAlloc((void**)&h_acc_, hNC_ * 4, cudaHostAllocPortable);
            if (e == cudaSuccess)
                e = cudaHostAlloc((void**)&h_swap_, 12ull * std::max<uint32_t>(o_.replace_k, 1), cudaHostAllocPortable);
            if (e != cudaSuccess) { cudaGetLastError(); throw Error(ASCETIC_EHOSTMEM, "cudaHostAlloc (replacement tables)"); }
            hot_alloc_nc_ = hNC_;
            hot_alloc_k_ = o_.replace_k;
        }
        CK(cudaMemcpyAsync(d_init_, init_chunks_.data(), hNS_ * 4, cudaMemcpyHostToDevice, cs_));
        hot_dirty_ = true;   // begin() installs the initial slots
    }
    // what the Static Region holds: a kept region (ASCETIC_OPT_KEEP_STATIC) is only reused when the
    // placement, its first vertex, its size and the slot layout are all unchanged
    const std::array<uint64_t, 6> key = {(uint64_t)o_.placement, o_.placement == 2 ? o_.placement_seed : 0ull,
                                         stat_lo_, p.s, hot_ ? p.Ms : 0ull, (uint64_t)hot_};
    if (key != static_key_) static_valid_ = false;
    static_key_ = key;
    CK(cudaStreamSynchronize(cs_));
}

void Part::free_hot() {
    dfree(d_slot_of_); dfree(d_acc_); dfree(d_swap_); dfree(d_init_);
    if (h_acc_) cudaFreeHost(h_acc_);
    if (h_swap_) cudaFreeHost(h_swap_);
    h_acc_ = h_swap_ = nullptr;
    hot_alloc_nc_ = 0;
    hot_alloc_k_ = 0;
}

// Eq. 3 (§3.3): after the data map of an iteration is generated, if the on-demand
// data exceed the On-demand Region and the Static Region is under-used (V_static / M_static <
// 0.5 V / D), shrink the Static Region by M_static * V / D (floored to 16 KiB) and
// hand that memory to the On-demand Region; the caller re-generates the data map.
bool Part::maybe_repartition(const IterTotals& T) {
    if (ms_cur_ == 0 || pl_.D == 0 || o_.placement != 0) return false;   // Eq. 3 shrinks a front prefix
    const double b_e = g_.b_e;
    const double V = b_e * (double)T.active_arcs, Vs = b_e * (double)T.hit_arcs, Vo = b_e * (double)T.miss_arcs;
    const double D = (double)pl_.D, Ms = (double)ms_cur_;
    const double C = (double)(pl_.B > ms_cur_ ? pl_.B - ms_cur_ : 0);
    if (!(Vo > C && Vs / Ms < 0.5 * V / D)) return false;
    const uint64_t delta = (uint64_t)std::floor(Ms * V / D);
    const uint64_t ms_new = (ms_cur_ - std::min(delta, ms_cur_)) / 16384ull * 16384ull;
    if (ms_new >= ms_cur_) return false;
    const uint64_t* off = g_.off + vlo_;
    const uint64_t lim = off[0] + ms_new / g_.b_e;
    const uint64_t s_new = (uint64_t)(std::upper_bound(off, off + (vhi_ - vlo_) + 1, lim) - off) - 1;
    CK(cudaStreamSynchronize(xs_));   // no transfer may still target the old chunk layout
    CK(cudaStreamSynchronize(xs2_));
    for (cudaStream_t x : xs34_) CK(cudaStreamSynchronize(x));
    static_valid_ = false;            // chunk buffers now overlay the old static tail
    ms_cur_ = ms_new;
    s_cur_ = s_new;
    layout_regions(ms_new);
    launch_set_range_bits(d_S_, nwords_, vlo_, vlo_ + s_new, cs_);
    st.repartitions += 1;
    return true;
}

DevState Part::dev_state(uint32_t iter) const {
    DevState d;
    d.off = d_off_; d.n = g_.n; d.nwords = nwords_;
    d.A = d_A_; d.S = d_S_; d.next = (fused_ && (iter & 1u)) ? d_next2_ : d_next_; d.visited = d_visited_;
    d.val = d_val_; d.snap = d_snap_;
    d.rank = d_rank_; d.contrib = d_contrib_; d.sum = d_sum_; d.dang = d_dang_;
    d.iter = iter;
    d.vlo = vlo_; d.vhi = vhi_;
    d.static_arc0 = g_.off ? g_.off[stat_lo_] : 0;
    d.slot_of = hot_ ? d_slot_of_ : nullptr;
    d.pr_r = d_pr_r_; d.pr_res = d_pr_res_; d.pr_c = d_pr_c_;
    d.pr_inc = multi_ ? d_pr_inc_ : nullptr;
    d.tau = prd_tau_;
    d.red_min = red_min_ ? 1u : 0u;
    return d;
}

Queues Part::queues(const IterTotals& T) const {
    Queues q;
    q.hq_small = d_hq_small_; q.hq_med = d_hq_med_; q.hq_hub = d_hq_hub_; q.hub_pre = d_hub_pre_;
    q.mq = d_mq_; q.mq_pre = d_mq_pre_; q.mq_src = d_mq_src_; q.tile_first = d_tile_first_;
    q.n_missq = T.n_missq; q.miss_arcs = T.miss_arcs;
    return q;
}

cudaEvent_t Part::mark(cudaStream_t s, bool always) {
    if (!timing_ || (!fine_ && !always)) return nullptr;
    cudaEvent_t e = pool_.get();
    CK(cudaEventRecord(e, s));
    return e;
}

void Part::span(cudaEvent_t a, cudaStream_t s, uint32_t t, int ph, int sub) {
    if (!timing_ || !a) return;
    cudaEvent_t e = pool_.get();
    CK(cudaEventRecord(e, s));
    spans_.push_back({a, e, t, ph, sub});
}

// ---- transfer engine: chunk = miss-stream arcs [lo, hi). mode 1: zero-copy SM gather over
// the miss queue; mode 2: copy-engine DMA of the run pieces intersecting the window.
void Part::transfer_chunk(const Queues& q, int buf, unsigned long long lo, unsigned long long hi, int mode,
                          cudaStream_t xs, const DevState* visit) {
    if (mode == 1) {
        const uint32_t b_e = g_.b_e;
        // the long runs of the window go to the copy engines on the second copy stream, concurrently
        // with the SM gather of the rest; both start after this chunk's buffer is free (xfer_go) and
        // the chunk is ready when both are done
        bool ce = false;
        if (nlint_) {
            size_t r = std::upper_bound(ldst_.begin(), ldst_.end(), lo) - ldst_.begin();
            r = r ? r - 1 : 0;
            const char* host = (const char*)g_.nbr;
            char* dst = (char*)d_chunk_[buf];
            for (; r < lb_.size(); ++r) {
                const unsigned long long a0 = g_.off[lb_[r]], a1 = g_.off[le_[r]];
                const unsigned long long s0 = ldst_[r], s1 = s0 + (a1 - a0);
                if (s0 >= hi) break;
                const unsigned long long p0 = std::max(s0, lo), p1 = std::min(s1, hi);
                if (p1 <= p0) continue;
                if (!ce) {
                    CK(cudaEventRecord(xfer_go_[buf], xs_));
                    CK(cudaStreamWaitEvent(xs2_, xfer_go_[buf], 0));
                    ce = true;
                }
                CK(cudaMemcpyAsync(dst + (p0 - lo) * b_e, host + (a0 + (p0 - s0)) * b_e, (p1 - p0) * b_e,
                                   cudaMemcpyHostToDevice, xs2_));
                st.gather_ce_bytes += (p1 - p0) * b_e;
            }
        }
        // default grid keeps ~1 MiB of PCIe reads in flight (CTAs x 256 lanes x 8 loads x b_e):
        // enough to saturate the link (~20 us of it), while a deeper queue only adds latency
        // and congests the memory system for the concurrently running edge kernels
        // (measured: 64 CTAs at b_e = 8 -> same 47 GB/s, 3x faster on-demand kernels than 296)
        const int ctas = o_.gather_ctas ? o_.gather_ctas : (int)(64u * 8u / b_e);
        launch_gather(q, g_.nbr_dev, g_.m, b_e, d_chunk_[buf], lo, hi, ctas, nlint_ ? d_lint_[lint_buf_] : nullptr,
                      nlint_, o_.gap_bridge, d_cover_, xs, visit);
        if (ce) {
            CK(cudaEventRecord(ce_done_[buf], xs2_));
            CK(cudaStreamWaitEvent(xs_, ce_done_[buf], 0));
        }
        return;
    }
    size_t r = std::upper_bound(rdst_.begin(), rdst_.end(), lo) - rdst_.begin();
    r = r ? r - 1 : 0;
    const char* host = (const char*)g_.nbr;
    char* dst = (char*)d_chunk_[buf];
    const uint32_t b_e = g_.b_e;
    for (; r < rb_.size(); ++r) {
        const unsigned long long a0 = g_.off[rb_[r]], a1 = g_.off[re_[r]];
        const unsigned long long s0 = rdst_[r], s1 = s0 + (a1 - a0);
        if (s0 >= hi) break;
        const unsigned long long p0 = std::max(s0, lo), p1 = std::min(s1, hi);
        if (p1 <= p0) continue;
        CK(cudaMemcpyAsync(dst + (p0 - lo) * b_e, host + (a0 + (p0 - s0)) * b_e, (p1 - p0) * b_e,
                           cudaMemcpyHostToDevice, xs));
    }
}

// Gather-mode iteration with runs of >= ce_min_run bytes: the copy engines move those (one
// cudaMemcpyAsync each, ~55 GB/s when long) while the SM gather does the many short ones. A small
// kernel lists the long runs into mapped memory; the host sorts them by stream position and hands
// the gather their stream intervals (H2D on the copy stream, before this iteration's gathers).
uint32_t Part::plan_long_runs(const IterTotals& T) {
    nlint_ = 0;
    lb_.clear(); le_.clear(); ldst_.clear();
    const unsigned long long min_arcs = std::max<uint64_t>(1, o_.ce_min_run / g_.b_e);
    *reinterpret_cast<volatile uint32_t*>(&h_long_flag_[0]) = 0;
    launch_long_runs(d_run_b_, d_run_e_, d_run_dst_, T.n_runs, d_off_, min_arcs, h_long_, kLongMax, d_long_cnt_,
                     d_long_cnt_ + 1, h_long_flag_, cs_);
    CK(cudaGetLastError());
    CK(cudaEventRecord(ev_long_, cs_));
    const volatile uint32_t* flag = h_long_flag_;
    uint32_t spins = 0;
    while (!flag[0]) {
        if ((++spins & 1023u) == 0) {
            const cudaError_t e = cudaEventQuery(ev_long_);
            if (e == cudaSuccess) break;
            if (e != cudaErrorNotReady) CK(e);
        }
    }
    if (!flag[0]) CK(cudaEventSynchronize(ev_long_));
    std::atomic_thread_fence(std::memory_order_acquire);
    const uint32_t c0 = flag[1];
    const uint32_t cnt = std::min<uint32_t>(c0, kLongMax);
    st.d2h_bytes += 8 + 24ull * cnt;
    if (!cnt) return 0;
    std::vector<uint32_t> idx(cnt);
    const volatile unsigned long long* L = h_long_;
    std::vector<unsigned long long> raw(3ull * cnt);
    for (uint64_t i = 0; i < 3ull * cnt; ++i) raw[i] = L[i];
    for (uint32_t i = 0; i < cnt; ++i) idx[i] = i;
    std::sort(idx.begin(), idx.end(), [&](uint32_t a, uint32_t b) { return raw[3 * a + 2] < raw[3 * b + 2]; });
    lint_buf_ ^= 1u;
    unsigned long long* li = h_lint_[lint_buf_];
    for (uint32_t k = 0; k < cnt; ++k) {
        const uint32_t i = idx[k];
        lb_.push_back((uint32_t)raw[3 * i]);
        le_.push_back((uint32_t)raw[3 * i + 1]);
        ldst_.push_back(raw[3 * i + 2]);
        li[2 * k] = raw[3 * i + 2];
        li[2 * k + 1] = raw[3 * i + 2] + (g_.off[raw[3 * i + 1]] - g_.off[raw[3 * i]]);
    }
    // staging buffer of parity p is rewritten two iterations later, after this copy ran (the host
    // reaches iteration t+2 only once classify(t+2) finished, which follows every chunk of t+1)
    CK(cudaMemcpyAsync(d_lint_[lint_buf_], li, 16ull * cnt, cudaMemcpyHostToDevice, xs_));
    st.h2d_other_bytes += 16ull * cnt;
    nlint_ = cnt;
    return cnt;
}

// Span-DMA iteration (mode 3): windows are host ranges of cap bytes over the miss stream's host span
// [miss_h0, miss_h1); a small kernel finds each window's first miss-stream position (mapped memory).
// False (stay in gather mode) when the span needs more windows than the table holds.
bool Part::plan_span_windows(const IterTotals& T) {
    const unsigned long long cap_arcs = cap_ / g_.b_e;
    const unsigned long long span = T.miss_h1 - T.miss_h0;
    const uint64_t nwin = (span + cap_arcs - 1) / cap_arcs;
    if (nwin == 0 || nwin > kSpanWinMax) return false;
    *reinterpret_cast<volatile uint32_t*>(&h_span_flag_[0]) = 0;
    Queues q = queues(T);
    launch_span_windows(q, T.miss_h0, T.miss_h1, cap_arcs, (uint32_t)nwin, h_win_, h_span_flag_, cs_);
    CK(cudaGetLastError());
    CK(cudaEventRecord(ev_long_, cs_));
    const volatile uint32_t* flag = h_span_flag_;
    uint32_t spins = 0;
    while (!flag[0]) {
        if ((++spins & 1023u) == 0) {
            const cudaError_t e = cudaEventQuery(ev_long_);
            if (e == cudaSuccess) break;
            if (e != cudaErrorNotReady) CK(e);
        }
    }
    if (!flag[0]) CK(cudaEventSynchronize(ev_long_));
    std::atomic_thread_fence(std::memory_order_acquire);
    st.d2h_bytes += 8ull * (nwin + 1);
    span_nwin_ = (uint32_t)nwin;
    return true;
}

void Part::begin(int algo, uint32_t source, uint32_t max_iters, bool timing) {
    algo_ = algo;
    if (algo == ALG_PRD) {   // tau = floor(res0 * ppm / 1e6), res0 = floor(3 * 2^56 / (20 n))  (DESIGN R29)
        const unsigned __int128 res0 = (3ull << 56) / (20ull * g_.n);
        prd_tau_ = (uint64_t)(res0 * o_.prd_tol_ppm / 1000000u);
    }
    max_iters_ = max_iters;
    gchunk_ = 0;
    prefetched_ = 0;
    timing_ = timing;
    // every run starts from the placer's split (an Eq. 3 shrink lasts for the run it happened in)
    if (ms_cur_ != pl_.Ms || s_cur_ != pl_.s) {
        ms_cur_ = pl_.Ms;
        s_cur_ = pl_.s;
        launch_set_range_bits(d_S_, nwords_, stat_lo_, stat_lo_ + pl_.s, cs_);
    }
    layout_regions(ms_cur_);
    if (hot_) {
        // every run starts from the front chunks [0, hNS_) in slots [0, hNS_) and a zero hotness table
        if (hot_dirty_) {
            slot_of_.assign(hNC_, kNoSlot);
            slot_chunk_ = init_chunks_;
            for (uint64_t i = 0; i < hNS_; ++i) slot_of_[init_chunks_[i]] = (uint32_t)i;
            CK(cudaMemcpyAsync(d_slot_of_, slot_of_.data(), hNC_ * 4, cudaMemcpyHostToDevice, cs_));
            CK(cudaStreamSynchronize(cs_));
            if (o_.placement == 2) launch_static_bits(dev_state(0), d_slot_of_, g_.b_e, cs_);
            else launch_set_range_bits(d_S_, nwords_, stat_lo_, stat_lo_ + pl_.s, cs_);
            static_valid_ = false;
            hot_dirty_ = false;
        }
        hot_h_.assign(hNC_, 0);
    }
    acc_pending_ = false;
    iters.clear();
    std::memset(&st, 0, sizeof st);
    pool_.reset();
    spans_.clear();
    host_s_ = 0.0;
    fine_ = true;
    launches0_ = g_launches;
    ev_start_ = pool_.get(); ev_fill0_ = pool_.get(); ev_fill1_ = pool_.get();
    CK(cudaEventRecord(ev_start_, cs_));
    CK(cudaMemsetAsync(d_cover_, 0, 8, cs_));
    // ---- static fill: ONE DMA of this rank's front prefix, counted in the run
    CK(cudaStreamWaitEvent(xs_, ev_start_, 0));
    CK(cudaEventRecord(ev_fill0_, xs_));
    // with slots the chunks are filled whole: Ms bytes for the front chunks (one DMA), the chosen
    // chunks for the random content (one zero-copy chunk-copy kernel)
    const uint64_t fill = hot_ ? init_fill_bytes_ : pl_.static_bytes;
    if (fill && !(o_.keep_static && static_valid_)) {
        if (hot_ && o_.placement == 2) {
            launch_copy_chunks(g_.nbr_dev, g_.off[vlo_] * (uint64_t)g_.b_e, pl_.D, d_init_, nullptr, (uint32_t)hNS_,
                               d_static_, xs_);
            CK(cudaGetLastError());
        } else {
            CK(cudaMemcpyAsync(d_static_, (const char*)g_.nbr + g_.off[stat_lo_] * g_.b_e, fill,
                               cudaMemcpyHostToDevice, xs_));
        }
        st.h2d_static_fill_bytes = fill;
        static_valid_ = true;
    }
    CK(cudaEventRecord(ev_fill1_, xs_));
    launch_init(algo, dev_state(0), source, cs_);
    CK(cudaGetLastError());
    // only the static-hit kernels read the Static Region: iteration 0's classify and its chunk
    // transfers (queued on the copy stream right behind the fill) need not wait for the fill
    CK(cudaStreamWaitEvent(ss_, ev_fill1_, 0));
}

void Part::classify(uint32_t t) {
    // ---- GenDataMap + compaction
    *reinterpret_cast<volatile uint32_t*>(&h_tot_->ready) = 0;
    ++epoch_;
    if (epoch_ >= (1u << 30)) {
        CK(cudaMemsetAsync(d_tile_flag_, 0, (size_t)ntiles_ * 4, cs_));
        epoch_ = 1;
    }
    ClassifyArgs ca;
    ca.A = d_A_; ca.S = d_S_; ca.off = d_off_; ca.n = g_.n; ca.vlo = vlo_; ca.vhi = vhi_;
    ca.nwords = nwords_; ca.ntiles = ntiles_; ca.words_per_warp = wpw_;
    ca.hub_deg = o_.hub_deg; ca.piece_arcs = kPieceArcs;
    ca.hq_small = d_hq_small_; ca.hq_med = d_hq_med_; ca.hq_hub = d_hq_hub_; ca.hub_pre = d_hub_pre_;
    ca.mq = d_mq_; ca.mq_pre = d_mq_pre_; ca.mq_src = d_mq_src_; ca.tile_first = d_tile_first_;
    ca.run_b = d_run_b_; ca.run_e = d_run_e_; ca.run_dst = d_run_dst_;
    ca.tile_agg = d_tile_agg_; ca.tile_incl = d_tile_incl_; ca.tile_flag = d_tile_flag_; ca.epoch = epoch_;
    ca.tot = d_tot_ + tot_buf_;            // zeroed by the previous classify's last CTA
    ca.tot_next = d_tot_ + (tot_buf_ ^ 1u);
    tot_buf_ ^= 1u;
    ca.host_tot = h_tot_;
    ca.host_runs = h_runs_; ca.host_runs_cap = kRunsHostMax;
    ca.force_host_runs = o_.xfer_mode == 2 ? 1u : 0u;
    ca.dma_min_run_arcs = o_.xfer_mode == 0 ? std::max<uint64_t>(1, o_.dma_min_run / g_.b_e) : ~0ull;
    // the iteration's start marks its wall time, with TIMING = 1 only when the previous iteration was
    // big enough for per-phase spans (a small run's event pairs cost more than its classify kernels)
    cudaEvent_t e0 = mark(cs_);
    launch_classify(ca, cs_);
    CK(cudaGetLastError());
    span(e0, cs_, t, PH_CLS);
    CK(cudaEventRecord(ev_classified_, cs_));
}

IterTotals Part::wait_classify() {
    // low-latency wait: spin on the flag the last classify CTA writes into mapped memory
    const volatile uint32_t* flag = &h_tot_->ready;
    uint32_t spins = 0;
    while (!*flag) {
        if ((++spins & 1023u) == 0) {
            const cudaError_t q = cudaEventQuery(ev_classified_);
            if (q == cudaSuccess) break;
            if (q != cudaErrorNotReady) CK(q);
        }
    }
    std::atomic_thread_fence(std::memory_order_acquire);
    IterTotals T = *const_cast<const IterTotals*>(h_tot_);
    if (!T.ready) {
        CK(cudaEventSynchronize(ev_classified_));
        T = *const_cast<const IterTotals*>(h_tot_);
    }
    st.d2h_bytes += sizeof(IterTotals);
    return T;
}

void Part::expand(uint32_t t, const IterTotals& T) {
    const auto th0 = std::chrono::steady_clock::now();
    const uint32_t b_e = g_.b_e;
    ascetic_iter_stats_t is{};
    is.t = t; is.rank = (uint32_t)rank_;
    is.nA = T.nA; is.nH = T.nH; is.nM = T.nM; is.nruns = T.n_runs;
    is.active_arcs = T.active_arcs; is.hit_arcs = T.hit_arcs; is.miss_bytes = T.miss_arcs * b_e;
    is.digest = T.digest;
    is.s_static = T.nS;
    const DevState d = dev_state(t);
    const Queues q = queues(T);
    // per-phase spans only for iterations big enough for them to matter (TIMING = 1): a small
    // iteration keeps its classify span (its wall time); its event pairs would cost more device and
    // host time than its kernels (C1: 0.28 ms device + 0.27 ms host per 1 ms run in round 1; bench
    // step 1.07 -> 0.87 ms when the threshold went from 2^20 arcs / 4 MiB to 2^23 arcs / 32 MiB)
    fine_ = o_.timing >= 2 || trace_level() > 0 || T.active_arcs >= (8ull << 20) || T.miss_arcs * b_e >= (32ull << 20);
    if (algo_ == ALG_PR) CK(cudaMemsetAsync(d_sum_ + vlo_, 0, (vhi_ - vlo_) * sizeof(unsigned long long), cs_));
    // ---- Static Computing, overlapping the transfer, on its own stream so
    // the on-demand kernels (and through them the chunk buffers' reuse) never queue behind it;
    // finalize joins it. The static buffer holds host arcs [off[vlo], off[vlo+s]); kernels
    // index it with rank-local arc numbers (arc - d.static_arc0), so 128-bit alignment is
    // that of the buffer itself.
    static_pending_ = false;
    static_launched_ = false;
    // §3.4: this iteration's accesses per 16 KiB chunk -> pinned host table, read by
    // replace() while the on-demand chunks stream (the server thread of Fig. 6)
    if (hot_ && o_.replace_k > 0 && !(max_iters_ && t + 1 == max_iters_)) {
        CK(cudaMemsetAsync(d_acc_, 0, hNC_ * 4, cs_));
        launch_chunk_access(d, q, T.n_small, T.n_med, T.n_hub, b_e, d_acc_, cs_);
        CK(cudaGetLastError());
        CK(cudaMemcpyAsync(h_acc_, d_acc_, hNC_ * 4, cudaMemcpyDeviceToHost, cs_));
        CK(cudaEventRecord(ev_acc_, cs_));
        acc_pending_ = true;
        st.d2h_bytes += hNC_ * 4;
    }
    if (T.n_small + T.n_med + T.n_hub) {
        CK(cudaEventRecord(static_go_, cs_));
        CK(cudaStreamWaitEvent(ss_, static_go_, 0));
        // persistent grid: 4 CTAs/SM leave room for the on-demand kernels; an iteration without
        // misses (resident lists only) takes every slot
        const int cps = o_.static_ctas_per_sm > 0 ? o_.static_ctas_per_sm : (T.miss_arcs ? 4 : 8);
        // PR with contrib beyond L2: pull in neighbour-id slices (rows must be sorted; front prefix only)
        uint32_t passes = 1;
        if (algo_ == ALG_PR && o_.pr_segment && (g_.flags & ASCETIC_SORTED) && !hot_ && 4ull * g_.n > o_.pr_segment * 3 / 2) {
            const uint64_t by_l2 = (4ull * g_.n + o_.pr_segment - 1) / o_.pr_segment;
            const uint64_t by_deg = T.nH ? T.hit_arcs / T.nH / 8 : 0;   // a pass must not cost more than it saves
            passes = (uint32_t)std::min<uint64_t>(by_l2, by_deg);
            if (passes >= 2) {
                const uint64_t need = (uint64_t)T.n_med + T.n_pieces + 2;
                if (need > seg_cur_n_) {
                    dfree(d_seg_cur_);
                    dalloc(&d_seg_cur_, need, &vertex_bytes_);
                    seg_cur_n_ = need;
                }
            }
        }
        if (passes >= 2) {
            cudaEvent_t e0 = mark(ss_);
            launch_static_pr_seg(d, q, d_static_, T.n_small, T.n_med, T.n_hub, T.n_pieces, kPieceArcs, passes, d_seg_cur_,
                                 d_seg_cur_ + T.n_med, cps * sm_count_, ss_);
            CK(cudaGetLastError());
            span(e0, ss_, t, PH_STATIC);
            st.pr_segment_passes = passes;
        } else if (trace_level() == 2 && timing_) {   // timeline of the three degree buckets
            for (int b = 0; b < 3; ++b) {
                cudaEvent_t e0 = mark(ss_);
                launch_static(algo_, d, q, d_static_, b == 0 ? T.n_small : 0, b == 1 ? T.n_med : 0,
                              b == 2 ? T.n_hub : 0, T.n_pieces, kPieceArcs, cps * sm_count_, ss_);
                CK(cudaGetLastError());
                span(e0, ss_, t, PH_STATIC, 1 + b);
            }
        } else {
            cudaEvent_t e0 = mark(ss_);
            launch_static(algo_, d, q, d_static_, T.n_small, T.n_med, T.n_hub, T.n_pieces, kPieceArcs, cps * sm_count_, ss_);
            CK(cudaGetLastError());
            span(e0, ss_, t, PH_STATIC);
        }
        CK(cudaEventRecord(static_done_, ss_));
        static_pending_ = true;
        static_launched_ = true;
    }
    st.static_arcs += T.hit_arcs;
    st.ondemand_arcs += T.miss_arcs;
    nlint_ = 0;
    // ---- On-demand request, fragmented into chunks
    const unsigned long long cap_arcs = cap_ / b_e;
    const unsigned long long miss = T.miss_arcs;
    uint32_t nchunks = miss ? (uint32_t)((miss + cap_arcs - 1) / cap_arcs) : 0;
    int mode = 1;
    if (nchunks) {
        if (o_.xfer_mode == 2) mode = 2;
        else if (o_.xfer_mode == 1 || o_.xfer_mode == 3) mode = 1;
        else mode = (T.n_runs <= kRunsHostMax && miss * b_e / std::max<uint32_t>(1, T.n_runs) >= o_.dma_min_run) ? 2 : 1;
        // span DMA: the miss stream is nearly contiguous on the host (few, small holes between its runs)
        // (forced with XFER_MODE 3 whatever the span, for tests: sparse windows are then gathered)
        if (mode == 1 && (o_.xfer_mode == 3 || (o_.xfer_mode == 0 && o_.span_density > 0 &&
                                                 miss * b_e >= o_.span_min_bytes &&
                                                 (double)(T.miss_h1 - T.miss_h0) <= o_.span_max_ratio * (double)miss)) &&
            plan_span_windows(T))
            mode = 3;
        if (mode == 2) {
            // the run list is already in mapped host memory (classify's last CTA copies the first
            // kRunsHostMax runs there when the iteration qualifies for DMAs): no device round trip
            // before the DMAs can be planned
            rb_.resize(T.n_runs); re_.resize(T.n_runs); rdst_.resize(T.n_runs);
            const volatile uint32_t* hr = h_runs_;
            const uint32_t nh = std::min<uint32_t>(T.host_runs, T.n_runs);
            for (uint32_t r = 0; r < nh; ++r) { rb_[r] = hr[2 * r]; re_[r] = hr[2 * r + 1]; }
            if (T.n_runs > nh) {   // forced DMA mode with a long run list (or none copied): fetch the rest
                CK(cudaMemcpy(rb_.data() + nh, d_run_b_ + nh, (T.n_runs - nh) * 4ull, cudaMemcpyDeviceToHost));
                CK(cudaMemcpy(re_.data() + nh, d_run_e_ + nh, (T.n_runs - nh) * 4ull, cudaMemcpyDeviceToHost));
            }
            st.d2h_bytes += T.n_runs * 8ull;
            unsigned long long acc = 0;
            for (uint32_t r = 0; r < T.n_runs; ++r) { rdst_[r] = acc; acc += g_.off[re_[r]] - g_.off[rb_[r]]; }
        }
        // long runs can only matter when the iteration moves many of them (32 x the threshold): a
        // small iteration would pay the listing kernel and its host round trip for nothing (C1)
        if (mode == 1 && o_.ce_min_run && T.n_runs && miss * b_e >= 32 * o_.ce_min_run) plan_long_runs(T);
        if (!o_.overlap && static_pending_) {   // ablation: the transfer waits for static computing
            CK(cudaStreamWaitEvent(xs_, static_done_, 0));
            CK(cudaStreamWaitEvent(xs2_, static_done_, 0));
        }
    }
    // chunks already transferred at the end of the previous iteration (PR prefetch) must be
    // exactly this iteration's first windows
    if (prefetched_ && (mode != 2 || miss != prefetch_miss_ || T.n_runs != prefetch_runs_))
        throw Error(ASCETIC_ECUDA, "internal: prefetched chunks do not match the iteration's miss stream");
    const uint64_t g0 = gchunk_;   // global chunk number of this iteration's chunk 0
    // small chunks (two buffers of < 4 MiB, e.g. C1's 0.3 MB; ~14 us gathers, latency-bound): each
    // buffer gets its own stream that runs the buffer's transfers AND its on-demand kernels in order,
    // so buffer reuse and transfer -> compute need no events (2 launches per chunk instead of 2 + 4
    // event calls) and chunk k+1's transfer runs beside chunk k's compute; the two streams join the
    // compute stream at the end. (C1: 0.868 -> 0.871 ms per step, i.e. the chunk pipeline is not
    // host-bound once the per-phase events are off.) Large chunks keep the event pipeline (copy
    // stream at the highest priority, compute on its own stream).
    // (up to 4 buffers: with BFS's fused visit a buffer's stream holds only gathers, so more buffers of
    // smaller chunks put more chunk transfers in flight at once)
    const bool alt = mode == 1 && nlint_ == 0 && nbuf_ <= 4 && cap_ < (4ull << 20) && prefetched_ == 0;
    cudaStream_t bst[4] = {xs_, xs2_, xs34_[0], xs34_[1]};
    if (alt && nchunks) {
        CK(cudaEventRecord(ev_pipe_, cs_));   // after the previous iteration's compute and this one's memsets
        for (int b = 0; b < nbuf_; ++b) CK(cudaStreamWaitEvent(bst[b], ev_pipe_, 0));
    }
    // windows: [k cap, (k+1) cap) of the miss stream, or (span mode) the host ranges of cap bytes
    // over the miss stream's span; a dense span window is one DMA of its host bytes and the
    // on-demand kernel reads it in place (span_base), a sparse one is gathered like mode 1
    // BFS: On-demand Computing of a gathered chunk fused into its gather (the ids are visited as they
    // land); not with copy-engine long runs beside the gather (their vertices are not in its lanes)
    const bool fuse = algo_ == ALG_BFS && b_e == 4 && nlint_ == 0 &&
                      (o_.fused_visit == 2 || (o_.fused_visit == 1 && alt));
    uint32_t nwin = nchunks;
    if (mode == 3) nwin = span_nwin_;
    uint32_t done = 0;
    for (uint32_t k = 0; k < nwin; ++k) {
        unsigned long long lo, hi, base = ~0ull, hbytes = 0;
        int wmode = mode;
        if (mode == 3) {
            lo = h_win_[k];
            hi = h_win_[k + 1];
            if (hi <= lo) continue;                                  // a hole-only window
            const unsigned long long H0 = T.miss_h0 + (unsigned long long)k * cap_arcs;
            const unsigned long long H1 = std::min<unsigned long long>(T.miss_h1, H0 + cap_arcs);
            if ((double)(hi - lo) >= o_.span_density * (double)(H1 - H0)) {
                wmode = 3;
                base = H0;
                hbytes = (H1 - H0) * b_e;
            } else {
                wmode = 1;
            }
        } else {
            lo = (unsigned long long)k * cap_arcs;
            hi = std::min(miss, lo + cap_arcs);
        }
        const uint64_t gk = g0 + done;
        const int buf = (int)(gk % (uint64_t)nbuf_);
        if (alt) {
            cudaStream_t sb = bst[buf];
            cudaEvent_t e0 = mark(sb);
            transfer_chunk(q, buf, lo, hi, 1, sb, fuse ? &d : nullptr);
            CK(cudaGetLastError());
            span(e0, sb, t, PH_GATHER);
            if (!fuse) {
                e0 = mark(sb);
                launch_ondemand(algo_, d, q, d_chunk_[buf], lo, hi, ~0ull, sb);
                CK(cudaGetLastError());
                span(e0, sb, t, PH_OND);
            }
            st.gather_bytes += (hi - lo) * b_e;
            ++st.gather_chunks;
            ++done;
            continue;
        }
        cudaStream_t xk = xs_;
        if (done >= prefetched_) {
            if (gk >= (uint64_t)nbuf_) CK(cudaStreamWaitEvent(xk, consumed_[buf], 0));   // buffer reuse
            cudaEvent_t e0 = mark(xk);
            if (wmode == 3) {
                CK(cudaMemcpyAsync(d_chunk_[buf], (const char*)g_.nbr + base * b_e, hbytes, cudaMemcpyHostToDevice, xk));
            } else {
                transfer_chunk(q, buf, lo, hi, wmode, xk, fuse && wmode == 1 ? &d : nullptr);
            }
            CK(cudaGetLastError());
            span(e0, xk, t, wmode == 1 ? PH_GATHER : PH_DMA);
            CK(cudaEventRecord(ready_[buf], xk));
        }
        if (wmode == 1) st.gather_bytes += (hi - lo) * b_e;
        else st.dma_bytes += (hi - lo) * b_e;
        if (wmode == 3) { st.span_link_bytes += hbytes; st.span_payload_bytes += (hi - lo) * b_e; ++st.span_chunks; }
        cudaEvent_t e0 = nullptr;
        CK(cudaStreamWaitEvent(cs_, ready_[buf], 0));
        if (!(fuse && wmode == 1)) {   // (fused: the gather already computed the chunk)
            e0 = mark(cs_);
            launch_ondemand(algo_, d, q, d_chunk_[buf], lo, hi, base, cs_);   // On-demand Computing
            CK(cudaGetLastError());
            span(e0, cs_, t, PH_OND);
        }
        CK(cudaEventRecord(consumed_[buf], cs_));
        if (wmode == 1) ++st.gather_chunks; else ++st.dma_chunks;
        ++done;
    }
    if (alt && done) {   // the buffers' last users, for whoever uses them next; finalize waits for all
        for (int b = 0; b < nbuf_; ++b) {
            CK(cudaEventRecord(consumed_[b], bst[b]));
            CK(cudaStreamWaitEvent(cs_, consumed_[b], 0));
        }
    }
    nchunks = done;
    gchunk_ = g0 + nchunks;
    prefetched_ = 0;
    // ---- PR: A_t = V every iteration, so the next iteration's miss stream is this one and its
    // transfer does not depend on this iteration's values. Issue the next iteration's first
    // chunks now (each still waits for its buffer's consumer): the link keeps streaming
    // through this iteration's tail, finalize and the next classify.
    if (algo_ == ALG_PR && mode == 2 && nchunks && o_.prefetch && !o_.repartition && !hot_ && t + 1 < max_iters_) {
        const uint32_t np = std::min<uint32_t>(nchunks, (uint32_t)nbuf_);
        for (uint32_t k = 0; k < np; ++k) {
            const uint64_t gk = gchunk_ + k;
            const int buf = (int)(gk % (uint64_t)nbuf_);
            const unsigned long long lo = (unsigned long long)k * cap_arcs;
            const unsigned long long hi = std::min(miss, lo + cap_arcs);
            if (gk >= (uint64_t)nbuf_) CK(cudaStreamWaitEvent(xs_, consumed_[buf], 0));
            cudaEvent_t e0 = mark(xs_);
            transfer_chunk(q, buf, lo, hi, mode, xs_);
            CK(cudaGetLastError());
            span(e0, xs_, t + 1, PH_DMA);
            CK(cudaEventRecord(ready_[buf], xs_));
        }
        prefetched_ = np;
        prefetch_miss_ = miss;
        prefetch_runs_ = T.n_runs;
    }
    is.chunks = nchunks;
    is.mode = nchunks ? (uint32_t)mode : 0u;
    st.chunks_total += nchunks;
    st.h2d_payload_bytes += is.miss_bytes;
    st.active_arcs_total += is.active_arcs;
    iters.push_back(is);
    host_s_ += std::chrono::duration<double>(std::chrono::steady_clock::now() - th0).count();
}

void Part::debug_classify(const uint32_t* active_words, uint64_t nwords, ascetic_classify_out_t* out) {
    if (nwords != nwords_) throw Error(ASCETIC_EINVAL, "active bitmap must have ceil(n/32) words");
    for (uint64_t w = 0; w < nwords; ++w) {   // bits beyond n must be clear
        const uint64_t lo = w * 32;
        if (lo + 32 > g_.n && (active_words[w] >> (g_.n - lo)) != 0 && g_.n - lo < 32)
            throw Error(ASCETIC_EINVAL, "active bitmap has bits set beyond n");
    }
    CK(cudaMemcpyAsync(d_A_, active_words, nwords * 4, cudaMemcpyHostToDevice, cs_));
    const bool timing = timing_;
    timing_ = false;
    classify(0);
    timing_ = timing;
    const IterTotals T = wait_classify();
    CK(cudaStreamSynchronize(cs_));
    out->n_small = T.n_small; out->n_med = T.n_med; out->n_hub = T.n_hub; out->n_pieces = T.n_pieces;
    out->n_missq = T.n_missq; out->n_runs = T.n_runs; out->miss_arcs = T.miss_arcs;
    out->nA = T.nA; out->nH = T.nH; out->nM = T.nM; out->active_arcs = T.active_arcs; out->hit_arcs = T.hit_arcs;
    out->digest = T.digest;
    auto get = [&](void* dst, const void* src, uint64_t count, size_t elem) {
        if (dst && count && count <= out->cap) CK(cudaMemcpy(dst, src, count * elem, cudaMemcpyDeviceToHost));
    };
    get(out->hit_small, d_hq_small_, T.n_small, 4);
    get(out->hit_med, d_hq_med_, T.n_med, 4);
    get(out->hit_hub, d_hq_hub_, T.n_hub, 4);
    get(out->hub_pre, d_hub_pre_, T.n_hub, 4);
    get(out->missq, d_mq_, T.n_missq, 4);
    get(out->missq_pre, d_mq_pre_, T.n_missq, 8);
    get(out->missq_src, d_mq_src_, T.n_missq, 8);
    get(out->run_b, d_run_b_, T.n_runs, 4);
    get(out->run_e, d_run_e_, T.n_runs, 4);
    get(out->run_dst, d_run_dst_, T.n_runs, 8);
}

void Part::join_static() {
    if (static_pending_) CK(cudaStreamWaitEvent(cs_, static_done_, 0));
    static_pending_ = false;
}

// §3.4 (Fig. 6; swaps "when GPU is processing the On-demand Region"):
// update the HotnessTable with this iteration's chunk accesses (cumulative for BFS/SSSP/CC, last
// iteration for PR), then swap the K hottest non-resident chunks (h desc, id asc)
// with the K coldest resident ones (h asc, id asc) while strictly hotter. The swap DMAs run on
// the copy stream after this iteration's miss chunks and static-hit kernels; slot table and
// StaticBitmap are updated on the compute stream before the next GenDataMap.
void Part::replace(uint32_t t) {
    if (!acc_pending_ || o_.replace_k == 0) return;
    acc_pending_ = false;
    const auto th0 = std::chrono::steady_clock::now();
    CK(cudaEventSynchronize(ev_acc_));
    const bool cum = o_.replace_policy == 1 || (o_.replace_policy == 0 && algo_ != ALG_PR);
    const uint32_t K = o_.replace_k;
    uint64_t* h = hot_h_.data();
    const uint32_t* acc = h_acc_;
    if (cum) for (uint64_t c = 0; c < hNC_; ++c) h[c] += acc[c];
    else for (uint64_t c = 0; c < hNC_; ++c) h[c] = acc[c];
    // K hottest non-resident chunks: bounded heap ordered by `better`, so its top is the worst kept
    auto better = [&](uint32_t a, uint32_t b) { return h[a] != h[b] ? h[a] > h[b] : a < b; };  // min-heap
    std::vector<uint32_t> hot;
    hot.reserve(K + 1);
    for (uint64_t c = 0; c < hNC_; ++c) {
        if (slot_of_[c] != kNoSlot) continue;
        if (hot.size() == K) {
            if (h[c] <= h[hot.front()]) continue;   // ascending ids: a tie never displaces
            std::pop_heap(hot.begin(), hot.end(), better);
            hot.back() = (uint32_t)c;
        } else {
            hot.push_back((uint32_t)c);
        }
        std::push_heap(hot.begin(), hot.end(), better);
    }
    std::sort(hot.begin(), hot.end(), better);
    // K coldest resident chunks (there are hNS_ of them: scan the slots)
    std::vector<uint32_t> cold(slot_chunk_);
    auto colder = [&](uint32_t a, uint32_t b) { return h[a] != h[b] ? h[a] < h[b] : a < b; };
    const size_t kc = std::min<size_t>(K, cold.size());
    std::partial_sort(cold.begin(), cold.begin() + kc, cold.end(), colder);
    uint32_t k = 0;
    uint64_t bytes = 0;
    while (k < hot.size() && k < kc && h[hot[k]] > h[cold[k]]) ++k;
    if (k) {
        const uint64_t x0 = g_.off[vlo_] * (uint64_t)g_.b_e;
        if (static_launched_) CK(cudaStreamWaitEvent(xs_, static_done_, 0));   // evicted slots no longer read
        cudaEvent_t e0 = mark(xs_);
        for (uint32_t i = 0; i < k; ++i) {
            const uint32_t cin = hot[i], cout = cold[i], slot = slot_of_[cout];
            slot_of_[cin] = slot;
            slot_of_[cout] = kNoSlot;
            slot_chunk_[slot] = cin;
            bytes += std::min<uint64_t>(kChunkBytes, pl_.D - (uint64_t)cin * kChunkBytes);
            h_swap_[i] = cin;
            h_swap_[k + i] = cout;
            h_swap_[2 * k + i] = slot;
        }
        // the swap list, then one zero-copy kernel copying the K incoming 16 KiB chunks from the
        // pinned host CSR into their slots (16 KiB contiguous reads run at the link's rate)
        CK(cudaMemcpyAsync(d_swap_, h_swap_, 12ull * k, cudaMemcpyHostToDevice, xs_));
        launch_copy_chunks(g_.nbr_dev, x0, pl_.D, d_swap_, d_swap_ + 2 * k, k, d_static_, xs_);
        CK(cudaGetLastError());
        span(e0, xs_, t, PH_REPL);
        CK(cudaEventRecord(ev_swapped_, xs_));
        CK(cudaStreamWaitEvent(cs_, ev_swapped_, 0));
        launch_apply_swaps(dev_state(t), d_slot_of_, d_swap_, k, g_.b_e, cs_);
        CK(cudaGetLastError());
        hot_dirty_ = true;
        static_valid_ = false;   // the region no longer holds the front prefix (keep_static)
    }
    if (!iters.empty()) { iters.back().swaps = k; iters.back().replace_bytes = bytes; }
    st.h2d_replace_bytes += bytes;
    st.swaps_total += k;
    host_s_ += std::chrono::duration<double>(std::chrono::steady_clock::now() - th0).count();
}

// ---- fused exchange: the finalize reads every rank's buffer from peer memory
void Part::set_fused(bool on) {
    fused_ = on;
    if (on && !d_next2_) {
        dalloc(&d_next2_, nwords_, &vertex_bytes_);
        CK(cudaMemset(d_next2_, 0, (size_t)std::max<uint32_t>(nwords_, 1) * 4));
    }
}

void Part::set_peers(int kind, const std::vector<void*>& ptrs) {
    const int P = (int)ptrs.size();
    if (!d_peers_ || peer_world_ != P) {
        if (d_peers_) cudaFree((void*)d_peers_);
        CK(cudaMalloc((void**)&d_peers_, 3 * (size_t)P * sizeof(void*)));
        peer_world_ = P;
    }
    CK(cudaMemcpyAsync(d_peers_ + (size_t)kind * P, ptrs.data(), (size_t)P * sizeof(void*), cudaMemcpyHostToDevice, cs_));
    CK(cudaStreamSynchronize(cs_));
}

void Part::finalize_fused(uint32_t t) {
    join_static();
    cudaEvent_t e0 = mark(cs_);
    const int kind = algo_ == ALG_BFS ? (int)(t & 1u) : 2;
    launch_finalize_peers(algo_, dev_state(t), d_peers_ + (size_t)kind * peer_world_, peer_world_, cs_);
    CK(cudaGetLastError());
    span(e0, cs_, t, PH_FIN);
}

void Part::clear_next(uint32_t b) {
    CK(cudaMemsetAsync(next_buf((int)b), 0, (size_t)nwords_ * 4, cs_));
}

void Part::clear_prd_inc() {
    if (d_pr_inc_) CK(cudaMemsetAsync(d_pr_inc_, 0, g_.n * 8, cs_));
}

void Part::finalize(uint32_t t, bool dense) {
    // ---- next active set, after the static-hit kernels
    join_static();
    cudaEvent_t e0 = mark(cs_);
    launch_finalize(algo_, dev_state(t), dense || red_min_, cs_);
    CK(cudaGetLastError());
    span(e0, cs_, t, PH_FIN);
}

void Part::end() {
    cudaEvent_t ev_end = pool_.get();
    join_static();
    CK(cudaEventRecord(ev_end, cs_));
    CK(cudaMemcpyAsync(h_cover_, d_cover_, 8, cudaMemcpyDeviceToHost, cs_));   // after every gather (cs_ joins them)
    CK(cudaStreamSynchronize(cs_));
    CK(cudaStreamSynchronize(xs_));
    CK(cudaStreamSynchronize(xs2_));
    for (cudaStream_t x : xs34_) CK(cudaStreamSynchronize(x));
    CK(cudaStreamSynchronize(ss_));
    float ms = 0.f, fill_ms = 0.f;
    CK(cudaEventElapsedTime(&ms, ev_start_, ev_end));
    CK(cudaEventElapsedTime(&fill_ms, ev_fill0_, ev_fill1_));
    double ph[PH_N] = {};
    const bool trace = trace_level() > 0;
    static const char* kPhName[PH_N] = {"classify", "static", "ondemand", "gather", "dma", "finalize", "exchange",
                                        "replace"};
    for (const Span& sp : spans_) {
        float a = 0.f;
        CK(cudaEventElapsedTime(&a, sp.a, sp.b));
        if (trace) {   // timeline: rank iter kernel-class start end (ms from run start)
            float s0 = 0.f;
            CK(cudaEventElapsedTime(&s0, ev_start_, sp.a));
            static const char* kSub[4] = {"", "_small", "_med", "_hub"};
            std::fprintf(stderr, "TRACE %d %u %s%s %.4f %.4f\n", rank_, sp.iter, kPhName[sp.ph], kSub[sp.sub & 3], s0, s0 + a);
        }
        ph[sp.ph] += a;
        if (sp.iter < iters.size()) {
            auto& is = iters[sp.iter];
            switch (sp.ph) {
                case PH_CLS: is.ms_classify += a; break;
                case PH_STATIC: is.ms_static += a; break;
                case PH_OND: is.ms_ondemand += a; break;
                case PH_GATHER: case PH_DMA: is.ms_h2d += a; break;
                case PH_XCH: is.ms_exchange += a; break;
                case PH_REPL: is.ms_h2d += a; break;
                default: is.ms_finalize += a; break;
            }
        }
    }
    // iteration wall time: from its classify launch to the next one (the last: to the run's end)
    std::vector<cudaEvent_t> cls_start(iters.size() + 1, nullptr);
    for (const Span& sp : spans_)
        if (sp.ph == PH_CLS && sp.iter < cls_start.size()) cls_start[sp.iter] = sp.a;
    std::vector<cudaEvent_t> x_first(iters.size(), nullptr), x_last(iters.size(), nullptr);
    for (const Span& sp : spans_) {
        if ((sp.ph == PH_GATHER || sp.ph == PH_DMA) && sp.iter < iters.size()) {
            if (!x_first[sp.iter]) x_first[sp.iter] = sp.a;
            x_last[sp.iter] = sp.b;
        }
    }
    for (size_t i = 0; i < iters.size(); ++i) {
        // to the next iteration's start (unmarked after a small iteration: no wall time then)
        cudaEvent_t a = cls_start[i], b = cls_start[i + 1] ? cls_start[i + 1] : (i + 1 < iters.size() ? nullptr : ev_end);
        float w = 0.f;
        if (a && b) CK(cudaEventElapsedTime(&w, a, b));
        iters[i].ms_total = w;
        if (a && b && x_first[i]) {
            float h = 0.f, span_ms = 0.f, tl = 0.f;
            CK(cudaEventElapsedTime(&h, a, x_first[i]));
            CK(cudaEventElapsedTime(&span_ms, x_first[i], x_last[i]));
            CK(cudaEventElapsedTime(&tl, x_last[i], b));
            iters[i].ms_link_head = h;
            iters[i].ms_link_gaps = span_ms - iters[i].ms_h2d;
            iters[i].ms_link_tail = tl;
        }
    }
    st.algo = algo_;
    st.iterations = (uint32_t)iters.size();
    st.n = g_.n; st.m = g_.m; st.b_e = g_.b_e;
    st.rank = (uint32_t)rank_;
    st.s = iters.empty() ? pl_.s : iters[0].s_static;   // static vertices at the start of the run
    st.budget_bytes = pl_.B;
    st.static_reserved = pl_.Ms;
    st.static_bytes = pl_.static_bytes;
    st.ondemand_bytes = pl_.C;
    st.chunk_cap = cap_;
    st.chunk_buffers = (uint32_t)nbuf_;
    st.static_fraction_used = pl_.R;
    {
        st.gather_load_bytes = *h_cover_ * 16ull;
    }
    st.time_run_s = ms / 1e3;
    st.time_fill_s = fill_ms / 1e3;
    st.time_classify_s = ph[PH_CLS] / 1e3;
    st.time_static_s = ph[PH_STATIC] / 1e3;
    st.time_ondemand_s = ph[PH_OND] / 1e3;
    st.time_gather_s = ph[PH_GATHER] / 1e3;
    st.time_dma_s = ph[PH_DMA] / 1e3;
    st.time_finalize_s = ph[PH_FIN] / 1e3;
    st.time_host_s = host_s_;
    st.time_h2d_busy_s = (ph[PH_GATHER] + ph[PH_DMA] + ph[PH_REPL] + fill_ms) / 1e3;
    st.time_replace_s = ph[PH_REPL] / 1e3;
    st.vertex_state_bytes = vertex_bytes_;
    st.kernel_launches = g_launches - launches0_;
}

// ================================================================== Engine
Engine::~Engine() {
    try { unload(); } catch (...) {}
}

void Engine::set_device(int dev) {
    if (state_ != 0) throw Error(ASCETIC_ESTATE, "set_device must precede load_csr");
    int cnt = 0;
    CK(cudaGetDeviceCount(&cnt));
    if (dev < 0 || dev >= cnt) throw Error(ASCETIC_EINVAL, "device out of range");
    device_ = dev;
}

void Engine::comm_init(int rank, int world, const void* uid, int device) {
    if (state_ != 0) throw Error(ASCETIC_ESTATE, "comm_init must precede load_csr");
    if (world < 1 || rank < 0 || rank >= world) throw Error(ASCETIC_EINVAL, "bad rank/world");
    if (world > 1 && !uid) throw Error(ASCETIC_EINVAL, "unique id is NULL");
    set_device(device);
    CK(cudaSetDevice(device_));
    emulate_ = 1;
    comm_.init_nccl(rank, world, uid);
}

void Engine::emulate_ranks(int world) {
    if (state_ != 0) throw Error(ASCETIC_ESTATE, "emulate_ranks must precede load_csr");
    if (world < 1 || world > 64) throw Error(ASCETIC_EINVAL, "emulated world must be in [1, 64]");
    comm_.init_emulated(world);
    emulate_ = world;
}

void Engine::load_csr(uint64_t n, uint64_t m, const uint64_t* off, const uint32_t* nbr, const uint32_t* wgt,
                      uint32_t flags) {
    if (!off) throw Error(ASCETIC_EINVAL, "off is NULL");
    if (n >= 0xFFFFFFFFull) throw Error(ASCETIC_EINVAL, "n must be < 2^32 - 1");
    if (m > 0 && !nbr) throw Error(ASCETIC_EINVAL, "nbr is NULL");
    if ((flags & ASCETIC_PAIRS) && wgt) throw Error(ASCETIC_EINVAL, "wgt given together with ASCETIC_PAIRS");
    if (off[0] != 0) throw Error(ASCETIC_EINVAL, "off[0] != 0");
    if (off[n] != m) throw Error(ASCETIC_EINVAL, "off[n] != m");
    const bool pairs = (flags & ASCETIC_PAIRS) || wgt;
    const uint32_t b_e = pairs ? 8u : 4u;
    if (flags & ASCETIC_VALIDATE) {
        const uint64_t step = (flags & ASCETIC_PAIRS) ? 2 : 1;
        for (uint64_t e = 0; e < m; ++e)
            if (nbr[e * step] >= n) throw Error(ASCETIC_EINVAL, "neighbour id >= n at arc " + std::to_string(e));
        if (flags & ASCETIC_SORTED)
            for (uint64_t v = 0; v < n; ++v)
                for (uint64_t e = off[v] + 1; e < off[v + 1]; ++e)
                    if (nbr[e * step] < nbr[(e - 1) * step])
                        throw Error(ASCETIC_EINVAL, "row " + std::to_string(v) + " is not sorted (ASCETIC_SORTED)");
    }
    if (device_ < 0) CK(cudaGetDevice(&device_));
    CK(cudaSetDevice(device_));
    CK(cudaDeviceGetAttribute(&sm_count_, cudaDevAttrMultiProcessorCount, device_));
    // same shape: keep every device allocation and stream (a reload is then offsets H2D and
    // host bookkeeping only); otherwise start from scratch. The rank ranges are part of the shape:
    // a part's owned range [vlo, vhi) and its range-sized queues are fixed at construction, so a
    // graph with the same n and m but other edge-balanced bounds rebuilds the parts.
    bool same_shape = state_ != 0 && n == g_.n && m == g_.m && b_e == g_.b_e;
    if (same_shape && comm_.world() > 1) same_shape = partition(off, n, (uint32_t)comm_.world()) == bounds_;
    if (state_ != 0 && !same_shape) unload();
    if (g_.owned) { cudaFreeHost(g_.owned); g_.owned = nullptr; }   // a registration may be kept (below)
    have_result_ = false;
    g_.n = n; g_.m = m; g_.b_e = b_e; g_.flags = flags;
    // offsets: used in place by the host planner (placer, partition, DMA planning) and DMA'd to
    // the device (full speed when the caller's array is pinned); ASCETIC_COPY keeps a private copy
    if (flags & ASCETIC_COPY) {
        g_.off_own.assign(off, off + n + 1);
        g_.off = g_.off_own.data();
    } else {
        g_.off_own.clear();
        g_.off = off;
    }
    // ---- rank ranges first: with one process per GPU a rank only ever reads the arcs of its own rows
    const int world = comm_.world();
    std::vector<uint64_t> nb = partition(off, n, (uint32_t)world);
    uint64_t a0 = 0, a1 = m;                         // arcs this process may read from the host
    if (!comm_.emulated() && world > 1) {
        a0 = std::min<uint64_t>(off[nb[comm_.rank()]], m);
        a1 = std::max<uint64_t>(a0, std::min<uint64_t>(off[nb[comm_.rank() + 1]], m));
    }
    // ---- pin the edge array (the On-demand Engine's Edgelist): this process's arc range
    // only (ranks share one host CSR, each pins its owned rows). Host arc x is always
    // addressed as nbr + b_e x; for a private copy of a slice `nbr` is the copy's virtual base.
    const size_t bytes = (size_t)b_e * m;
    if (bytes > 0) {
        const bool need_copy = (flags & ASCETIC_COPY) || wgt;
        if (need_copy) {
            if (g_.registered) { cudaHostUnregister(g_.registered); g_.registered = nullptr; g_.reg_bytes = 0; }
            // bytes [f0, f1) of the b_e layout, 16-byte aligned so the gather's cover units stay inside
            const uint64_t f0 = (uint64_t)b_e * a0 / 16 * 16;
            const uint64_t f1 = std::min<uint64_t>(((uint64_t)b_e * a1 + 15) / 16 * 16, bytes);
            cudaError_t e = cudaHostAlloc(&g_.owned, std::max<uint64_t>(f1 - f0, 16), cudaHostAllocPortable | cudaHostAllocMapped);
            if (e != cudaSuccess) { cudaGetLastError(); throw Error(ASCETIC_EHOSTMEM, "cudaHostAlloc failed"); }
            if (wgt) {
                uint32_t* dst = (uint32_t*)g_.owned;
                const uint64_t e0 = f0 / 8, e1 = f1 / 8;   // interleaved (id, w): 8 bytes per arc
                const unsigned nt = std::max(1u, std::min(16u, std::thread::hardware_concurrency()));
                std::vector<std::thread> th;
                for (unsigned t = 0; t < nt; ++t)
                    th.emplace_back([=] {
                        for (uint64_t e2 = e0 + t; e2 < e1; e2 += nt) {
                            dst[2 * (e2 - e0)] = nbr[e2];
                            dst[2 * (e2 - e0) + 1] = wgt[e2];
                        }
                    });
                for (auto& x : th) x.join();
            } else {
                std::memcpy(g_.owned, (const char*)nbr + f0, f1 - f0);
            }
            g_.nbr = (const char*)g_.owned - f0;
            void* dp = nullptr;
            CK(cudaHostGetDevicePointer(&dp, g_.owned, 0));
            g_.nbr_dev = (const char*)dp - f0;
        } else {
            // whole pages covering this process's arcs, clipped to the caller's array
            const uintptr_t base = (uintptr_t)nbr, pg = 4096;
            const uintptr_t lo = std::max<uintptr_t>(base, (base + (uintptr_t)b_e * a0) / pg * pg);
            const uintptr_t hi = std::min<uintptr_t>(base + bytes, (base + (uintptr_t)b_e * a1 + pg - 1) / pg * pg);
            const size_t rb = std::max<size_t>(hi > lo ? hi - lo : 0, 1);
            const bool keep = g_.registered == (void*)lo && g_.reg_bytes == rb;   // same range as before
            if (g_.registered && !keep) { cudaHostUnregister(g_.registered); g_.registered = nullptr; g_.reg_bytes = 0; }
            cudaPointerAttributes attr{};
            cudaError_t e = keep ? cudaSuccess : cudaPointerGetAttributes(&attr, (const void*)lo);
            if (e != cudaSuccess) cudaGetLastError();
            uintptr_t dbase = lo;                 // host address whose device alias is looked up
            if (!keep && e == cudaSuccess && attr.type == cudaMemoryTypeHost) {
                dbase = base;                     // already page-locked by the caller (cudaHostAlloc / pin_memory)
            } else if (!keep) {
                e = cudaHostRegister((void*)lo, rb, cudaHostRegisterPortable | cudaHostRegisterMapped | cudaHostRegisterReadOnly);
                if (e != cudaSuccess) {
                    cudaGetLastError();
                    e = cudaHostRegister((void*)lo, rb, cudaHostRegisterPortable | cudaHostRegisterMapped);
                }
                if (e != cudaSuccess) { cudaGetLastError(); throw Error(ASCETIC_EHOSTMEM, std::string("cudaHostRegister: ") + cudaGetErrorString(e)); }
                g_.registered = (void*)lo;
                g_.reg_bytes = rb;
            }
            g_.nbr = nbr;
            void* dp = nullptr;
            CK(cudaHostGetDevicePointer(&dp, (void*)dbase, 0));
            g_.nbr_dev = (const char*)dp - (dbase - base);
        }
    } else {
        g_.release();
    }
    g_.arc_lo = a0;
    g_.arc_hi = a1;
    // ---- rank parts: this process's ranks and their owned vertex ranges
    bounds_ = nb;
    if (!same_shape) {
        parts_.clear();
        if (comm_.emulated()) {
            for (int r = 0; r < world; ++r)
                parts_.emplace_back(new Part(g_, o_, r, bounds_[r], bounds_[r + 1], sm_count_));
        } else {
            const int r = comm_.rank();
            parts_.emplace_back(new Part(g_, o_, r, bounds_[r], bounds_[r + 1], sm_count_));
        }
        for (auto& p : parts_) p->alloc_vertex_state();
    }
    for (auto& p : parts_) p->upload_off();   // offsets H2D on every load (also resets the static region)
    for (auto& p : parts_) CK(cudaStreamSynchronize(p->cs()));
    {   // monotone offsets, checked on the device copy (one pass over 8(n+1) bytes of HBM)
        unsigned long long* d_bad = nullptr;
        CK(cudaMalloc(&d_bad, sizeof(unsigned long long)));
        CK(cudaMemset(d_bad, 0xFF, sizeof(unsigned long long)));
        launch_check_monotone(parts_[0]->dev_off(), n, d_bad, parts_[0]->cs());
        unsigned long long bad = 0;
        cudaError_t e = cudaMemcpy(&bad, d_bad, sizeof bad, cudaMemcpyDeviceToHost);
        cudaFree(d_bad);
        CK(e);
        if (bad != ~0ull) {
            unload();
            throw Error(ASCETIC_EINVAL, "off is not non-decreasing at v=" + std::to_string(bad));
        }
    }
    state_ = 1;
}

void Engine::set_budget(uint64_t bytes, double frac) {
    if (state_ == 0) throw Error(ASCETIC_ESTATE, "set_budget before load_csr");
    if (std::isnan(frac) || frac > 1.0) throw Error(ASCETIC_EINVAL, "static_fraction must be <= 1 (or < 0 for Eq. 2)");
    CK(cudaSetDevice(device_));
    state_ = 1;
    for (auto& p : parts_) p->set_budget(bytes, frac);   // every rank: its own budget B (§8(e))
    state_ = 2;
}

void Engine::set_option(int opt, int64_t value) {
    switch (opt) {
        case ASCETIC_OPT_CHUNK_CAP:
            if (value < 0) throw Error(ASCETIC_EINVAL, "chunk cap < 0");
            o_.chunk_cap = (uint64_t)value;
            break;
        case ASCETIC_OPT_XFER_MODE:
            if (value < 0 || value > 3) throw Error(ASCETIC_EINVAL, "xfer mode must be 0, 1, 2 or 3");
            o_.xfer_mode = (int)value;
            break;
        case ASCETIC_OPT_DMA_MIN_RUN: o_.dma_min_run = (uint64_t)std::max<int64_t>(0, value); break;
        case ASCETIC_OPT_OVERLAP: o_.overlap = value ? 1 : 0; break;
        case ASCETIC_OPT_KEEP_STATIC:
            o_.keep_static = value ? 1 : 0;
            for (auto& p : parts_) p->on_reload();
            break;
        case ASCETIC_OPT_HUB_DEGREE:
            if (value < 32 || value > (1ll << 30)) throw Error(ASCETIC_EINVAL, "hub degree must be in [32, 2^30]");
            o_.hub_deg = (uint32_t)value;
            break;
        case ASCETIC_OPT_TIMING:
            if (value < 0 || value > 2) throw Error(ASCETIC_EINVAL, "timing: 0 = off, 1 = auto, 2 = every phase");
            o_.timing = (int)value;
            break;
        case ASCETIC_OPT_GATHER_CTAS:
            if (value < 0 || value > 65535) throw Error(ASCETIC_EINVAL, "gather CTAs must be in [0, 65535]");
            o_.gather_ctas = (int)value;
            break;
        case ASCETIC_OPT_PREFETCH: o_.prefetch = value ? 1 : 0; break;
        case ASCETIC_OPT_REPARTITION: o_.repartition = value ? 1 : 0; break;
        case ASCETIC_OPT_STATIC_PLACEMENT:
            if (value < 0 || value > 2) throw Error(ASCETIC_EINVAL, "static placement: 0 = front, 1 = rear, 2 = random");
            o_.placement = (int)value;
            if (state_ == 2) state_ = 1;   // takes effect at the next set_budget
            break;
        case ASCETIC_OPT_REPLACE_CHUNKS:
            if (value < 0 || value > 65536) throw Error(ASCETIC_EINVAL, "replace chunks must be in [0, 65536]");
            o_.replace_k = (uint32_t)value;
            if (state_ == 2) state_ = 1;   // takes effect at the next set_budget
            break;
        case ASCETIC_OPT_PLACEMENT_SEED:
            o_.placement_seed = (uint64_t)value;
            if (state_ == 2) state_ = 1;
            break;
        case ASCETIC_OPT_PRD_TOL_PPM:
            if (value < 0 || value > 1000000000ll) throw Error(ASCETIC_EINVAL, "PRD tolerance must be in [0, 1e9] ppm");
            o_.prd_tol_ppm = (uint64_t)value;
            break;
        case ASCETIC_OPT_FUSED_EXCHANGE: o_.fused_exchange = value ? 1 : 0; break;
        case ASCETIC_OPT_SPARSE_EXCHANGE:
            if (value < 0 || value > 0xFFFFFFFFll) throw Error(ASCETIC_EINVAL, "sparse exchange divisor must be in [0, 2^32)");
            o_.sparse_exchange = (uint32_t)value;
            break;
        case ASCETIC_OPT_REPLACE_POLICY:
            if (value < 0 || value > 2) throw Error(ASCETIC_EINVAL, "replace policy: 0 = by algorithm, 1 = cumulative, 2 = last");
            o_.replace_policy = (int)value;
            break;
        case ASCETIC_OPT_STATIC_CTAS_PER_SM:
            if (value < 0 || value > 64) throw Error(ASCETIC_EINVAL, "static CTAs per SM must be in [0, 64]");
            o_.static_ctas_per_sm = (int)value;
            break;
        case ASCETIC_OPT_RELAX_MODE:
            if (value < 0 || value > 2) throw Error(ASCETIC_EINVAL, "relax mode: 0 = auto, 1 = atomicMin + next bit, 2 = RED.MIN + dense finalize");
            o_.relax_mode = (int)value;
            break;
        case ASCETIC_OPT_CE_MIN_RUN:
            if (value < 0) throw Error(ASCETIC_EINVAL, "copy-engine minimum run must be >= 0 bytes");
            o_.ce_min_run = (uint64_t)value;
            break;
        case ASCETIC_OPT_SPAN_DENSITY:
            if (value < 0 || value > 100) throw Error(ASCETIC_EINVAL, "span density must be a percentage in [0, 100]");
            o_.span_density = value / 100.0;
            break;
        case ASCETIC_OPT_SPAN_MAX_RATIO:
            if (value < 100 || value > 100000) throw Error(ASCETIC_EINVAL, "span ratio must be a percentage in [100, 100000]");
            o_.span_max_ratio = value / 100.0;
            break;
        case ASCETIC_OPT_PR_SEGMENT:
            if (value < 0) throw Error(ASCETIC_EINVAL, "PR segment bytes must be >= 0");
            o_.pr_segment = (uint64_t)value;
            break;
        case ASCETIC_OPT_GAP_BRIDGE:
            if (value < 0 || value > 65536) throw Error(ASCETIC_EINVAL, "gap bridge must be in [0, 65536] bytes");
            o_.gap_bridge = (uint32_t)value;
            break;
        case ASCETIC_OPT_FUSED_VISIT:
            if (value < 0 || value > 2) throw Error(ASCETIC_EINVAL, "fused visit must be 0, 1 or 2");
            o_.fused_visit = (int)value;
            break;
        case ASCETIC_OPT_CHUNK_BUFFERS:
            if (value != 0 && (value < 2 || value > 8)) throw Error(ASCETIC_EINVAL, "chunk buffers must be 0 (auto) or in [2, 8]");
            o_.chunk_buffers = (int)value;
            if (state_ == 2) state_ = 1;   // takes effect at the next set_budget
            break;
        default: throw Error(ASCETIC_EINVAL, "unknown option");
    }
}

void Engine::debug_classify(int rank, const uint32_t* active_words, uint64_t nwords, ascetic_classify_out_t* out) {
    if (state_ != 2) throw Error(ASCETIC_ESTATE, "debug_classify needs a loaded graph and a budget");
    if (!active_words || !out) throw Error(ASCETIC_EINVAL, "NULL argument");
    if (rank < 0 || rank >= (int)parts_.size()) throw Error(ASCETIC_EINVAL, "rank is not a local rank");
    CK(cudaSetDevice(device_));
    have_result_ = false;
    parts_[rank]->debug_classify(active_words, nwords, out);
}

// emulated ranks: every part's compute stream -> part 0's (the collectives run there) and back.
// Each part's sync event is re-recorded per use (a wait binds to the record enqueued before it).
void Engine::join() {
    cudaStream_t c0 = parts_[0]->cs();
    for (size_t i = 1; i < parts_.size(); ++i) {
        CK(cudaEventRecord(parts_[i]->sync_event(), parts_[i]->cs()));
        CK(cudaStreamWaitEvent(c0, parts_[i]->sync_event(), 0));
    }
}

void Engine::fork() {
    if (parts_.size() < 2) return;
    cudaEvent_t e = parts_[0]->sync_event();
    CK(cudaEventRecord(e, parts_[0]->cs()));
    for (size_t i = 1; i < parts_.size(); ++i) CK(cudaStreamWaitEvent(parts_[i]->cs(), e, 0));
}

void Engine::run(int algo, uint32_t source, uint32_t max_iters) {
    if (state_ != 2) throw Error(ASCETIC_ESTATE, state_ == 0 ? "run before load_csr" : "run before set_budget");
    if (algo < 0 || algo > 4) throw Error(ASCETIC_EINVAL, "unknown algorithm");
    if (algo == ALG_SSSP && g_.b_e != 8) throw Error(ASCETIC_EINVAL, "SSSP needs weights (ASCETIC_PAIRS or wgt)");
    if (algo != ALG_SSSP && g_.b_e != 4) throw Error(ASCETIC_EINVAL, "BFS/CC/PR take an unweighted CSR (b_e = 4)");
    if ((algo == ALG_BFS || algo == ALG_SSSP) && source >= g_.n) throw Error(ASCETIC_EINVAL, "source >= n");
    if (algo == ALG_PR && max_iters == 0) throw Error(ASCETIC_EINVAL, "PR needs max_iters >= 1");
    if ((algo == ALG_CC || algo == ALG_PR) && !(g_.flags & ASCETIC_SYMMETRIC))
        throw Error(ASCETIC_EINVAL, "CC and PR need ASCETIC_SYMMETRIC");
    if (g_.n == 0) throw Error(ASCETIC_EINVAL, "empty graph");
    if (o_.replace_k && o_.repartition) throw Error(ASCETIC_EINVAL, "replacement (§3.4) and Eq. 3 re-partition are exclusive");
    if (o_.repartition && o_.placement != 0) throw Error(ASCETIC_EINVAL, "Eq. 3 re-partition shrinks a front prefix");
    CK(cudaSetDevice(device_));
    have_result_ = false;
    const bool multi = comm_.active();
    const bool timing = o_.timing != 0;
    for (auto& p : parts_) p->alloc_algo_state(algo, multi);
    for (auto& p : parts_) p->set_fused(false);
    // fused exchange (P > 1, BFS/SSSP/CC/PRD): every part gets the world's buffer pointers
    const bool fused = multi && o_.fused_exchange && algo != ALG_PR;
    if (fused) {
        for (auto& p : parts_) p->set_fused(true);
        for (int kind = 0; kind < 3; ++kind) {
            if (kind < 2 && algo != ALG_BFS) continue;
            auto local = [&](Part& p) -> void* {
                if (kind < 2) return p.next_buf(kind);
                return algo == ALG_PRD ? (void*)p.prd_inc() : (void*)p.val();
            };
            std::vector<void*> world;
            if (comm_.emulated()) for (auto& p : parts_) world.push_back(local(*p));
            else world = comm_.open_peers(local(*parts_[0]));
            for (auto& p : parts_) p->set_peers(kind, world);
        }
    }
    // sparse exchange (collectives path, BFS / SSSP / CC): pair buffers sized before the timed run.
    // cap = n / (d P) pairs per rank; BFS n / (64 d P), a pair (8 B) replacing one bitmap bit
    const bool sparse_on = multi && !fused && o_.sparse_exchange &&
                           (algo == ALG_BFS || algo == ALG_SSSP || algo == ALG_CC);
    if (sparse_on) {
        const uint64_t dP = (uint64_t)o_.sparse_exchange * (uint64_t)comm_.world();
        const uint64_t c64 = algo == ALG_BFS ? g_.n / (64 * dP) : g_.n / dP;
        const uint32_t cap = (uint32_t)std::max<uint64_t>(1, std::min<uint64_t>(c64, g_.n));
        if (sp_cap_ != cap || sp_pairs_.size() != parts_.size()) {
            free_sparse();
            for (size_t i = 0; i < parts_.size(); ++i) {
                void* pp = nullptr;
                uint32_t* cc = nullptr;
                CK(cudaMalloc(&pp, (size_t)cap * 8));
                CK(cudaMalloc(&cc, 4));
                sp_pairs_.push_back(pp);
                sp_cnt_.push_back(cc);
            }
            sp_cap_ = cap;
        }
        comm_.reserve_sparse(cap, (int)parts_.size());
    }
    // SSSP/CC min updates: RED.MIN + dense finalize (default: resident RMAT-24 static-hit kernels -15 %
    // SSSP / -11 % CC, friendster-shaped CC -5 %, profiles/r02/resident_ab.md), unless the sparse
    // exchange needs this rank's next bits (it packs exactly the ids this rank lowered)
    const bool red = (algo == ALG_SSSP || algo == ALG_CC) && !sparse_on && o_.relax_mode != 1;
    for (auto& p : parts_) p->set_red_min(red);
    for (auto& p : parts_) p->begin(algo, source, max_iters, timing);
    Part& p0 = *parts_[0];
    std::vector<IterTotals> T(parts_.size());
    uint32_t t = 0;
    uint64_t sparse_iters = 0, sparse_bytes = 0;
    for (t = 0;; ++t) {
        if (max_iters && t == max_iters) break;
        bool dense_fin = true;   // false after a sparse exchange: A_{t+1} = the merged next bitmap
        for (auto& p : parts_) p->classify(t);
        for (size_t i = 0; i < parts_.size(); ++i) T[i] = parts_[i]->wait_classify();
        if (T[0].nA == 0) break;   // |A_t| is counted over the replicated bitmap: identical on every rank
        if (o_.repartition) {      // Eq. 3, then re-generate the data map
            for (size_t i = 0; i < parts_.size(); ++i) {
                if (parts_[i]->maybe_repartition(T[i])) {
                    parts_[i]->classify(t);
                    T[i] = parts_[i]->wait_classify();
                }
            }
        }
        for (size_t i = 0; i < parts_.size(); ++i) parts_[i]->expand(t, T[i]);
        if (fused) {
            // barrier 1: every rank's edge kernels are done before anyone reads its buffer
            for (auto& p : parts_) p->join_static();
            cudaEvent_t e0 = p0.mark(p0.cs());
            if (comm_.emulated()) { join(); fork(); } else comm_.barrier(p0.cs());
            p0.span(e0, p0.cs(), t, PH_XCH);
            // BFS: the other next buffer was last read before this barrier: clear it for t+1
            if (algo == ALG_BFS) for (auto& p : parts_) p->clear_next((t + 1) & 1u);
            for (auto& p : parts_) p->finalize_fused(t);
            if (algo != ALG_BFS) {
                // barrier 2: nobody overwrites its values / increments while a peer still reads them
                cudaEvent_t e1 = p0.mark(p0.cs());
                if (comm_.emulated()) { join(); fork(); } else comm_.barrier(p0.cs());
                p0.span(e1, p0.cs(), t, PH_XCH);
                if (algo == ALG_PRD) for (auto& p : parts_) p->clear_prd_inc();
            }
            for (auto& p : parts_) p->replace(t);
            continue;
        }
        if (multi && algo != ALG_PR) {
            // ---- exchange: OR of next bitmaps (BFS), MIN of values (SSSP, CC)
            for (auto& p : parts_) p->join_static();
            join();
            cudaEvent_t e0 = p0.mark(p0.cs());
            const uint64_t nw = (g_.n + 31) / 32;
            // SURVEY §8(e) sparse form (BFS / SSSP / CC): the ids (and values) each rank set in its
            // next bitmap this iteration, when every rank has at most `cap` of them; else dense
            auto try_sparse = [&]() -> bool {
                if (!sparse_on) return false;
                const uint32_t cap = sp_cap_;
                std::vector<uint32_t*> b, nx;
                for (auto& p : parts_) { b.push_back(p->val()); nx.push_back(p->next()); }
                for (size_t i = 0; i < parts_.size(); ++i)
                    launch_sparse_pack(nx[i], b[i], (uint32_t)nw, sp_pairs_[i], cap, sp_cnt_[i], p0.cs());
                uint64_t bytes = 0;
                const bool ok = comm_.sparse_min(b, nx, sp_pairs_, sp_cnt_, cap, p0.cs(), &bytes);
                if (ok) { ++sparse_iters; sparse_bytes += bytes; }
                return ok;
            };
            if (algo == ALG_BFS) {
                // BFS levels: a discovering rank holds t+1, the others INF, so MIN is right too
                if (!try_sparse()) {
                    std::vector<uint32_t*> b;
                    for (auto& p : parts_) b.push_back(p->next());
                    comm_.or_words(b, nw, p0.cs());
                }
            } else if (algo == ALG_PRD) {
                std::vector<unsigned long long*> b;
                for (auto& p : parts_) b.push_back(p->prd_inc());
                comm_.sum_u64(b, g_.n, p0.cs());
            } else {
                const bool sparse = try_sparse();
                if (!sparse) {
                    std::vector<uint32_t*> b;
                    for (auto& p : parts_) b.push_back(p->val());
                    comm_.min_u32(b, g_.n, p0.cs());
                }
                dense_fin = !sparse;
            }
            p0.span(e0, p0.cs(), t, PH_XCH);
            fork();
        }
        for (auto& p : parts_) p->finalize(t, multi && dense_fin);
        if (multi && algo == ALG_PR) {
            // ---- exchange: SUM of the fixed-point dangling partials (exact, so the total is the same
            // for every P), every rank's contrib slice to all
            join();
            cudaEvent_t e0 = p0.mark(p0.cs());
            std::vector<unsigned long long*> dg;
            std::vector<void*> cb;
            const int nxt = (int)((t + 1) & 1u);
            for (auto& p : parts_) { dg.push_back(p->dang() + nxt); cb.push_back(p->contrib()); }
            comm_.sum_u64(dg, 1, p0.cs());
            comm_.share_slices(cb, bounds_, 4, p0.cs());
            p0.span(e0, p0.cs(), t, PH_XCH);
            fork();
        }
        for (auto& p : parts_) p->replace(t);   // §3.4 swaps, effective at t+1
    }
    if (multi && algo == ALG_PR) {
        join();
        std::vector<void*> rk;
        for (auto& p : parts_) rk.push_back(p->rank_arr());
        comm_.share_slices(rk, bounds_, 4, p0.cs());
        fork();
    }
    if (algo == ALG_PRD)
        for (auto& p : parts_) launch_prd_output(p->dev_state(t), p->cs());   // rank = fp32((r + res) 2^-56)
    if (parts_.size() > 1) join();
    for (auto& p : parts_) p->end();
    // ---- aggregate the local parts (one with NCCL; all emulated ranks otherwise)
    st_ = p0.st;
    iters_.clear();
    const size_t niter = p0.iters.size();
    for (size_t i = 0; i < niter; ++i)
        for (auto& p : parts_)
            if (i < p->iters.size()) iters_.push_back(p->iters[i]);
    for (size_t i = 1; i < parts_.size(); ++i) {
        const auto& s = parts_[i]->st;
        st_.h2d_payload_bytes += s.h2d_payload_bytes;
        st_.h2d_static_fill_bytes += s.h2d_static_fill_bytes;
        st_.d2h_bytes += s.d2h_bytes;
        st_.active_arcs_total += s.active_arcs_total;
        st_.chunks_total += s.chunks_total;
        st_.dma_chunks += s.dma_chunks;
        st_.gather_chunks += s.gather_chunks;
        st_.static_arcs += s.static_arcs;
        st_.ondemand_arcs += s.ondemand_arcs;
        st_.gather_bytes += s.gather_bytes;
        st_.gather_ce_bytes += s.gather_ce_bytes;
        st_.gather_load_bytes += s.gather_load_bytes;
        st_.h2d_other_bytes += s.h2d_other_bytes;
        st_.dma_bytes += s.dma_bytes;
        st_.static_bytes += s.static_bytes;
        st_.vertex_state_bytes += s.vertex_state_bytes;
        st_.repartitions += s.repartitions;
        st_.h2d_replace_bytes += s.h2d_replace_bytes;
        st_.swaps_total += s.swaps_total;
        st_.time_replace_s = std::max(st_.time_replace_s, s.time_replace_s);
        st_.kernel_launches = std::max(st_.kernel_launches, s.kernel_launches);
    }
    st_.iterations = t;
    st_.sparse_exchanges = sparse_iters;
    st_.sparse_exchange_bytes = sparse_bytes;
    st_.world = (uint32_t)comm_.world();
    st_.rank = (uint32_t)comm_.rank();
    st_.gteps = st_.time_run_s > 0 ? (double)st_.active_arcs_total / st_.time_run_s / 1e9 : 0.0;
    const double ex = st_.time_run_s - st_.time_fill_s;
    st_.gteps_excl_fill = ex > 0 ? (double)st_.active_arcs_total / ex / 1e9 : 0.0;
    last_algo_ = algo;
    have_result_ = true;
}

int Engine::stats(ascetic_stats_t* out, ascetic_iter_stats_t* per_iter, uint32_t cap) const {
    if (!have_result_) throw Error(ASCETIC_ESTATE, "no completed run");
    if (out) *out = st_;
    if (per_iter) {
        const uint32_t k = std::min<uint32_t>(cap, (uint32_t)iters_.size());
        std::memcpy(per_iter, iters_.data(), k * sizeof(ascetic_iter_stats_t));
    }
    return (int)iters_.size();
}

void Engine::get_result(void* dst, uint64_t bytes) {
    if (!have_result_) throw Error(ASCETIC_ESTATE, "no completed run");
    if (!dst || bytes < 4 * g_.n) throw Error(ASCETIC_EINVAL, "result buffer must hold 4n bytes");
    CK(cudaSetDevice(device_));
    Part& p0 = *parts_[0];
    const void* src = (last_algo_ == ALG_PR || last_algo_ == ALG_PRD) ? (const void*)p0.rank_arr() : (const void*)p0.val();
    CK(cudaMemcpy(dst, src, 4 * g_.n, cudaMemcpyDeviceToHost));
}

void Engine::free_sparse() {
    for (void* p : sp_pairs_) if (p) cudaFree(p);
    for (uint32_t* c : sp_cnt_) if (c) cudaFree(c);
    sp_pairs_.clear();
    sp_cnt_.clear();
    sp_cap_ = 0;
}

void Engine::unload() {
    if (device_ >= 0) cudaSetDevice(device_);
    free_sparse();
    parts_.clear();
    g_.release();
    g_.off = nullptr;
    g_.off_own.clear();
    g_.off_own.shrink_to_fit();
    g_.n = g_.m = 0;
    state_ = 0;
    have_result_ = false;
    last_algo_ = -1;
    cudaGetLastError();
}

}  // namespace ascetic
