// engine.cu — run controller: placer, transfer engine, per-iteration pipeline.
//
// One iteration (Fig. 4; Fig. 5), B200 version:
//   compute stream cs : classify+compact  ──► host reads 80 B of totals (mapped)
//   cs                : static-hit kernels (Static Computing)
//   copy stream xs    : chunk k = miss-stream arcs [k*cap, (k+1)*cap) ->
//                       zero-copy SM gather or copy-engine DMA of runs
//                       buffer k%2 waits consumed[k-2]; records ready[k]
//   cs                : waits ready[k] -> on-demand kernel -> records consumed[k]
//   cs                : finalize: next active set
// Fragmenting when the request exceeds the On-demand Region (§3.3) is the
// chunk loop; the static compute overlaps the transfer (§3.2).
#include "engine.h"

#include <algorithm>
#include <atomic>
#include <chrono>
#include <cmath>
#include <cstring>
#include <thread>

namespace ascetic {

#define CK(call)                                                                                   \
    do {                                                                                           \
        cudaError_t e__ = (call);                                                                  \
        if (e__ != cudaSuccess)                                                                    \
            throw Error(ASCETIC_ECUDA, std::string(#call) + ": " + cudaGetErrorString(e__));       \
    } while (0)

enum { ALG_BFS = 0, ALG_SSSP = 1, ALG_CC = 2, ALG_PR = 3 };

// ------------------------------------------------------------------ placer
Placement place(const uint64_t* off, uint64_t n, uint32_t b_e, uint64_t budget, double frac) {
    Placement p;
    const double K = 0.10;
    p.B = budget;
    p.D = (uint64_t)b_e * off[n];
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
    // front prefix of whole lists: s = max{v : b_e off[v] <= Ms}
    const uint64_t lim = Ms / b_e;
    p.s = (uint64_t)(std::upper_bound(off, off + n + 1, lim) - off) - 1;
    p.static_bytes = (uint64_t)b_e * off[p.s];
    p.C = budget >= Ms ? budget - Ms : 0;
    p.cap = p.C / 2 / 16 * 16;
    return p;
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

// ------------------------------------------------------------------ load
void Engine::load_csr(uint64_t n, uint64_t m, const uint64_t* off, const uint32_t* nbr, const uint32_t* wgt,
                      uint32_t flags) {
    if (state_ != 0) unload();
    if (!off) throw Error(ASCETIC_EINVAL, "off is NULL");
    if (n >= 0xFFFFFFFFull) throw Error(ASCETIC_EINVAL, "n must be < 2^32 - 1");
    if (m > 0 && !nbr) throw Error(ASCETIC_EINVAL, "nbr is NULL");
    if ((flags & ASCETIC_PAIRS) && wgt) throw Error(ASCETIC_EINVAL, "wgt given together with ASCETIC_PAIRS");
    if (off[0] != 0) throw Error(ASCETIC_EINVAL, "off[0] != 0");
    for (uint64_t v = 0; v < n; ++v)
        if (off[v + 1] < off[v]) throw Error(ASCETIC_EINVAL, "off is not non-decreasing at v=" + std::to_string(v));
    if (off[n] != m) throw Error(ASCETIC_EINVAL, "off[n] != m");
    const bool pairs = (flags & ASCETIC_PAIRS) || wgt;
    const uint32_t b_e = pairs ? 8u : 4u;
    if (flags & ASCETIC_VALIDATE) {
        const uint64_t step = (flags & ASCETIC_PAIRS) ? 2 : 1;
        for (uint64_t e = 0; e < m; ++e)
            if (nbr[e * step] >= n) throw Error(ASCETIC_EINVAL, "neighbour id >= n at arc " + std::to_string(e));
    }
    if (device_ < 0) CK(cudaGetDevice(&device_));
    CK(cudaSetDevice(device_));
    CK(cudaDeviceGetAttribute(&sm_count_, cudaDevAttrMultiProcessorCount, device_));

    n_ = n; m_ = m; b_e_ = b_e; flags_ = flags;
    h_off_copy_.assign(off, off + n + 1);     // host planning copy (placer, DMA runs)
    h_off_ = h_off_copy_.data();
    // ---- pin the edge array (the On-demand Engine's Edgelist)
    const size_t bytes = (size_t)b_e * m;
    if (bytes > 0) {
        const bool need_copy = (flags & ASCETIC_COPY) || wgt;
        if (need_copy) {
            cudaError_t e = cudaHostAlloc(&h_owned_, bytes, cudaHostAllocPortable | cudaHostAllocMapped);
            if (e != cudaSuccess) { cudaGetLastError(); throw Error(ASCETIC_EHOSTMEM, "cudaHostAlloc failed"); }
            if (wgt) {
                uint32_t* dst = (uint32_t*)h_owned_;
                const unsigned nt = std::max(1u, std::min(16u, std::thread::hardware_concurrency()));
                std::vector<std::thread> th;
                for (unsigned t = 0; t < nt; ++t)
                    th.emplace_back([=] {
                        for (uint64_t e2 = t; e2 < m; e2 += nt) { dst[2 * e2] = nbr[e2]; dst[2 * e2 + 1] = wgt[e2]; }
                    });
                for (auto& x : th) x.join();
            } else {
                std::memcpy(h_owned_, nbr, bytes);
            }
            h_nbr_ = h_owned_;
        } else {
            cudaPointerAttributes attr{};
            cudaError_t e = cudaPointerGetAttributes(&attr, nbr);
            if (e != cudaSuccess) cudaGetLastError();
            if (e == cudaSuccess && attr.type == cudaMemoryTypeHost) {
                h_nbr_ = nbr;                       // already page-locked (cudaHostAlloc / pin_memory)
            } else {
                e = cudaHostRegister((void*)nbr, bytes,
                                     cudaHostRegisterPortable | cudaHostRegisterMapped | cudaHostRegisterReadOnly);
                if (e != cudaSuccess) {
                    cudaGetLastError();
                    e = cudaHostRegister((void*)nbr, bytes, cudaHostRegisterPortable | cudaHostRegisterMapped);
                }
                if (e != cudaSuccess) { cudaGetLastError(); throw Error(ASCETIC_EHOSTMEM, std::string("cudaHostRegister: ") + cudaGetErrorString(e)); }
                h_registered_ = (void*)nbr;
                h_nbr_ = nbr;
            }
        }
        void* dp = nullptr;
        CK(cudaHostGetDevicePointer(&dp, (void*)h_nbr_, 0));
        h_nbr_dev_ = dp;
    }
    // ---- streams
    int lo_pri = 0, hi_pri = 0;
    CK(cudaDeviceGetStreamPriorityRange(&lo_pri, &hi_pri));
    CK(cudaStreamCreateWithPriority(&cs_, cudaStreamNonBlocking, lo_pri));
    CK(cudaStreamCreateWithPriority(&xs_, cudaStreamNonBlocking, hi_pri));
    for (int i = 0; i < 2; ++i) {
        CK(cudaEventCreateWithFlags(&ready_[i], cudaEventDisableTiming));
        CK(cudaEventCreateWithFlags(&consumed_[i], cudaEventDisableTiming));
    }
    CK(cudaEventCreateWithFlags(&ev_classified_, cudaEventDisableTiming | cudaEventBlockingSync));
    alloc_vertex_state();
    CK(cudaMemcpyAsync(d_off_, off, (n + 1) * sizeof(uint64_t), cudaMemcpyHostToDevice, cs_));
    CK(cudaStreamSynchronize(cs_));
    state_ = 1;
}

void Engine::alloc_vertex_state() {
    vertex_bytes_ = 0;
    nwords_ = (uint32_t)((n_ + 31) / 32);
    ntiles_ = (nwords_ + kTileWords - 1) / kTileWords;
    dalloc(&d_off_, n_ + 1, &vertex_bytes_);
    dalloc(&d_A_, nwords_, &vertex_bytes_);
    dalloc(&d_S_, nwords_, &vertex_bytes_);
    dalloc(&d_next_, nwords_, &vertex_bytes_);
    dalloc(&d_hq_small_, n_, &vertex_bytes_);
    dalloc(&d_hq_med_, n_, &vertex_bytes_);
    const uint64_t nhub = std::min<uint64_t>(n_, m_ / opt_hub_deg_ + 1);   // at most m / hub_deg hubs
    dalloc(&d_hq_hub_, nhub, &vertex_bytes_);
    dalloc(&d_hub_pre_, nhub, &vertex_bytes_);
    dalloc(&d_mq_, n_, &vertex_bytes_);
    dalloc(&d_mq_pre_, n_, &vertex_bytes_);
    dalloc(&d_mq_src_, n_, &vertex_bytes_);
    dalloc(&d_tile_first_, (m_ >> kEdgeTileShift) + 2, &vertex_bytes_);
    dalloc(&d_run_b_, n_ / 2 + 1, &vertex_bytes_);
    dalloc(&d_run_e_, n_ / 2 + 1, &vertex_bytes_);
    dalloc(&d_run_dst_, n_ / 2 + 1, &vertex_bytes_);
    dalloc(&d_tile_agg_, ntiles_, &vertex_bytes_);
    dalloc(&d_tile_incl_, ntiles_, &vertex_bytes_);
    dalloc(&d_tile_flag_, ntiles_, &vertex_bytes_);
    dalloc(&d_tot_, 1, &vertex_bytes_);
    CK(cudaMemset(d_tile_flag_, 0, (size_t)std::max<uint32_t>(ntiles_, 1) * 4));
    CK(cudaMemset(d_S_, 0, (size_t)std::max<uint32_t>(nwords_, 1) * 4));
    epoch_ = 0;
    if (!h_tot_) {
        cudaError_t e = cudaHostAlloc((void**)&h_tot_, sizeof(IterTotals), cudaHostAllocMapped | cudaHostAllocPortable);
        if (e != cudaSuccess) { cudaGetLastError(); throw Error(ASCETIC_EHOSTMEM, "cudaHostAlloc totals"); }
    }
}

void Engine::alloc_algo_state(int algo) {
    if (algo == ALG_PR) {
        if (!d_rank_) {
            dalloc(&d_rank_, n_, &vertex_bytes_);
            dalloc(&d_contrib_, n_, &vertex_bytes_);
            dalloc(&d_sum_, n_, &vertex_bytes_);
            dalloc(&d_dang_, 2, &vertex_bytes_);
        }
    } else {
        if (!d_val_) {
            dalloc(&d_val_, n_, &vertex_bytes_);
        }
        if (algo == ALG_BFS && !d_visited_) dalloc(&d_visited_, nwords_, &vertex_bytes_);
        if (algo != ALG_BFS && !d_snap_) dalloc(&d_snap_, n_, &vertex_bytes_);
    }
}

void Engine::free_budget_regions() {
    dfree(d_static_);
    dfree(d_chunk_[0]);
    dfree(d_chunk_[1]);
    static_valid_ = false;
}

// ------------------------------------------------------------------ budget
void Engine::set_budget(uint64_t bytes, double frac) {
    if (state_ == 0) throw Error(ASCETIC_ESTATE, "set_budget before load_csr");
    if (std::isnan(frac) || frac > 1.0) throw Error(ASCETIC_EINVAL, "static_fraction must be <= 1 (or < 0 for Eq. 2)");
    CK(cudaSetDevice(device_));
    Placement p = place(h_off_, n_, b_e_, bytes, frac);
    if (p.s < n_ && p.cap < 16)
        throw Error(ASCETIC_ENOMEM, "budget leaves an On-demand chunk below 16 bytes (cap=" + std::to_string(p.cap) + ")");
    free_budget_regions();
    state_ = 1;
    pl_ = p;
    cap_ = p.cap;
    if (opt_chunk_cap_ && opt_chunk_cap_ < cap_) cap_ = std::max<uint64_t>(16, opt_chunk_cap_ / 16 * 16);
    if (p.static_bytes) {
        cudaError_t e = cudaMalloc(&d_static_, p.static_bytes);
        if (e != cudaSuccess) { cudaGetLastError(); throw Error(ASCETIC_ENOMEM, "static region allocation"); }
    }
    if (p.s < n_) {
        for (int i = 0; i < 2; ++i) {
            cudaError_t e = cudaMalloc(&d_chunk_[i], cap_);
            if (e != cudaSuccess) { cudaGetLastError(); free_budget_regions(); throw Error(ASCETIC_ENOMEM, "chunk allocation"); }
        }
    }
    launch_set_prefix_bits(d_S_, nwords_, p.s, cs_);   // StaticBitmap
    CK(cudaStreamSynchronize(cs_));
    state_ = 2;
}

void Engine::set_option(int opt, int64_t value) {
    switch (opt) {
        case ASCETIC_OPT_CHUNK_CAP:
            if (value < 0) throw Error(ASCETIC_EINVAL, "chunk cap < 0");
            opt_chunk_cap_ = (uint64_t)value;
            if (state_ == 2) {
                cap_ = pl_.cap;
                if (opt_chunk_cap_ && opt_chunk_cap_ < cap_) cap_ = std::max<uint64_t>(16, opt_chunk_cap_ / 16 * 16);
            }
            break;
        case ASCETIC_OPT_XFER_MODE:
            if (value < 0 || value > 2) throw Error(ASCETIC_EINVAL, "xfer mode must be 0, 1 or 2");
            opt_xfer_mode_ = (int)value;
            break;
        case ASCETIC_OPT_DMA_MIN_RUN: opt_dma_min_run_ = (uint64_t)std::max<int64_t>(0, value); break;
        case ASCETIC_OPT_OVERLAP: opt_overlap_ = value ? 1 : 0; break;
        case ASCETIC_OPT_KEEP_STATIC: opt_keep_static_ = value ? 1 : 0; static_valid_ = false; break;
        case ASCETIC_OPT_HUB_DEGREE:
            if (value < 32 || value > (1ll << 30)) throw Error(ASCETIC_EINVAL, "hub degree must be in [32, 2^30]");
            if ((uint32_t)value < opt_hub_deg_ && state_ != 0) {
                // hub arrays hold at most m / hub_deg entries; grow them
                const uint64_t nhub = std::min<uint64_t>(n_, m_ / (uint64_t)value + 1);
                dfree(d_hq_hub_); dfree(d_hub_pre_);
                dalloc(&d_hq_hub_, nhub, &vertex_bytes_);
                dalloc(&d_hub_pre_, nhub, &vertex_bytes_);
            }
            opt_hub_deg_ = (uint32_t)value;
            break;
        case ASCETIC_OPT_TIMING: opt_timing_ = value ? 1 : 0; break;
        case ASCETIC_OPT_GATHER_CTAS:
            if (value < 0 || value > 65535) throw Error(ASCETIC_EINVAL, "gather CTAs must be in [0, 65535]");
            opt_gather_ctas_ = (int)value;
            break;
        default: throw Error(ASCETIC_EINVAL, "unknown option");
    }
}

DevState Engine::dev_state(uint32_t iter) const {
    DevState d;
    d.off = d_off_; d.n = n_; d.nwords = nwords_;
    d.A = d_A_; d.S = d_S_; d.next = d_next_; d.visited = d_visited_;
    d.val = d_val_; d.snap = d_snap_;
    d.rank = d_rank_; d.contrib = d_contrib_; d.sum = d_sum_; d.dang = d_dang_;
    d.iter = iter;
    return d;
}

Queues Engine::queues(const IterTotals& T) const {
    Queues q;
    q.hq_small = d_hq_small_; q.hq_med = d_hq_med_; q.hq_hub = d_hq_hub_; q.hub_pre = d_hub_pre_;
    q.mq = d_mq_; q.mq_pre = d_mq_pre_; q.mq_src = d_mq_src_; q.tile_first = d_tile_first_;
    q.n_missq = T.n_missq; q.miss_arcs = T.miss_arcs;
    return q;
}

// ------------------------------------------------------------------ transfer engine
// chunk = miss-stream arcs [lo, hi). mode 1: zero-copy SM gather over the miss queue;
// mode 2: copy-engine DMA of the run pieces intersecting the window.
void Engine::transfer_chunk(const Queues& q, int buf, unsigned long long lo, unsigned long long hi, int mode,
                            const std::vector<uint32_t>& rb, const std::vector<uint32_t>& re,
                            const std::vector<unsigned long long>& rdst) {
    if (mode == 1) {
        launch_gather(q, h_nbr_dev_, b_e_, d_chunk_[buf], lo, hi, opt_gather_ctas_ ? opt_gather_ctas_ : 2 * sm_count_, xs_);
        return;
    }
    // first run whose stream range ends after lo
    size_t r = std::upper_bound(rdst.begin(), rdst.end(), lo) - rdst.begin();
    r = r ? r - 1 : 0;
    const char* host = (const char*)h_nbr_;
    char* dst = (char*)d_chunk_[buf];
    for (; r < rb.size(); ++r) {
        const unsigned long long a0 = h_off_[rb[r]], a1 = h_off_[re[r]];
        const unsigned long long s0 = rdst[r], s1 = s0 + (a1 - a0);
        if (s0 >= hi) break;
        const unsigned long long p0 = std::max(s0, lo), p1 = std::min(s1, hi);
        if (p1 <= p0) continue;
        CK(cudaMemcpyAsync(dst + (p0 - lo) * b_e_, host + (a0 + (p0 - s0)) * b_e_, (p1 - p0) * b_e_,
                           cudaMemcpyHostToDevice, xs_));
    }
}

// ------------------------------------------------------------------ run
void Engine::run(int algo, uint32_t source, uint32_t max_iters) {
    if (state_ != 2) throw Error(ASCETIC_ESTATE, state_ == 0 ? "run before load_csr" : "run before set_budget");
    if (algo < 0 || algo > 3) throw Error(ASCETIC_EINVAL, "unknown algorithm");
    if (algo == ALG_SSSP && b_e_ != 8) throw Error(ASCETIC_EINVAL, "SSSP needs weights (ASCETIC_PAIRS or wgt)");
    if (algo != ALG_SSSP && b_e_ != 4) throw Error(ASCETIC_EINVAL, "BFS/CC/PR take an unweighted CSR (b_e = 4)");
    if ((algo == ALG_BFS || algo == ALG_SSSP) && source >= n_) throw Error(ASCETIC_EINVAL, "source >= n");
    if (algo == ALG_PR && max_iters == 0) throw Error(ASCETIC_EINVAL, "PR needs max_iters >= 1");
    if ((algo == ALG_CC || algo == ALG_PR) && !(flags_ & ASCETIC_SYMMETRIC))
        throw Error(ASCETIC_EINVAL, "CC and PR need ASCETIC_SYMMETRIC");
    if (n_ == 0) throw Error(ASCETIC_EINVAL, "empty graph");
    CK(cudaSetDevice(device_));
    alloc_algo_state(algo);
    have_result_ = false;
    iters_.clear();
    std::memset(&st_, 0, sizeof st_);
    pool_.reset();
    const bool timing = opt_timing_ != 0;
    const unsigned long long launches0 = g_launches;

    // event pairs per kernel class, resolved after the run
    enum { PH_CLS, PH_STATIC, PH_OND, PH_GATHER, PH_DMA, PH_FIN, PH_N };
    struct Span { cudaEvent_t a, b; uint32_t iter; int ph; };
    std::vector<Span> spans;
    auto open_span = [&](cudaStream_t s) -> cudaEvent_t {
        if (!timing) return nullptr;
        cudaEvent_t e = pool_.get();
        CK(cudaEventRecord(e, s));
        return e;
    };
    auto close_span = [&](cudaEvent_t a, cudaStream_t s, uint32_t it, int ph) {
        if (!timing) return;
        cudaEvent_t e = pool_.get();
        CK(cudaEventRecord(e, s));
        spans.push_back({a, e, it, ph});
    };

    cudaEvent_t ev_start = pool_.get(), ev_end = pool_.get(), ev_fill0 = pool_.get(), ev_fill1 = pool_.get();
    CK(cudaEventRecord(ev_start, cs_));
    // ---- static fill: ONE DMA of the front prefix, counted in the run
    uint64_t fill_bytes = 0;
    CK(cudaStreamWaitEvent(xs_, ev_start, 0));
    CK(cudaEventRecord(ev_fill0, xs_));
    if (pl_.static_bytes && !(opt_keep_static_ && static_valid_)) {
        CK(cudaMemcpyAsync(d_static_, h_nbr_, pl_.static_bytes, cudaMemcpyHostToDevice, xs_));
        fill_bytes = pl_.static_bytes;
        static_valid_ = true;
    }
    CK(cudaEventRecord(ev_fill1, xs_));
    launch_init(algo, dev_state(0), source, cs_);
    CK(cudaGetLastError());
    CK(cudaStreamWaitEvent(cs_, ev_fill1, 0));

    const unsigned long long cap_arcs = cap_ / b_e_;
    std::vector<uint32_t> rb, re;
    std::vector<unsigned long long> rdst;
    double host_s = 0.0;
    uint32_t t = 0;
    for (t = 0;; ++t) {
        if (max_iters && t == max_iters) break;
        // ---- GenDataMap + compaction
        *reinterpret_cast<volatile uint32_t*>(&h_tot_->ready) = 0;
        CK(cudaMemsetAsync(d_tot_, 0, sizeof(IterTotals), cs_));
        ++epoch_;
        if (epoch_ >= (1u << 30)) {
            CK(cudaMemsetAsync(d_tile_flag_, 0, (size_t)ntiles_ * 4, cs_));
            epoch_ = 1;
        }
        ClassifyArgs ca;
        ca.A = d_A_; ca.S = d_S_; ca.off = d_off_; ca.n = n_; ca.nwords = nwords_; ca.ntiles = ntiles_;
        ca.hub_deg = opt_hub_deg_; ca.piece_arcs = kPieceArcs;
        ca.hq_small = d_hq_small_; ca.hq_med = d_hq_med_; ca.hq_hub = d_hq_hub_; ca.hub_pre = d_hub_pre_;
        ca.mq = d_mq_; ca.mq_pre = d_mq_pre_; ca.mq_src = d_mq_src_; ca.tile_first = d_tile_first_; ca.run_b = d_run_b_; ca.run_e = d_run_e_; ca.run_dst = d_run_dst_;
        ca.tile_agg = d_tile_agg_; ca.tile_incl = d_tile_incl_; ca.tile_flag = d_tile_flag_; ca.epoch = epoch_;
        ca.tot = d_tot_; ca.host_tot = h_tot_;
        cudaEvent_t e0 = open_span(cs_);
        launch_classify(ca, cs_);
        CK(cudaGetLastError());
        close_span(e0, cs_, t, PH_CLS);
        CK(cudaEventRecord(ev_classified_, cs_));
        // low-latency wait: spin on the flag the last classify CTA writes into mapped memory
        {
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
        }
        const auto th0 = std::chrono::steady_clock::now();
        const IterTotals T = *const_cast<const IterTotals*>(h_tot_);
        if (!T.ready) CK(cudaEventSynchronize(ev_classified_));
        st_.d2h_bytes += sizeof(IterTotals);
        if (T.nA == 0) break;

        ascetic_iter_stats_t is{};
        is.t = t; is.rank = 0;
        is.nA = T.nA; is.nH = T.nH; is.nM = T.nM; is.nruns = T.n_runs;
        is.active_arcs = T.active_arcs; is.hit_arcs = T.hit_arcs; is.miss_bytes = T.miss_arcs * b_e_;
        is.digest = T.digest;
        const DevState d = dev_state(t);
        const Queues q = queues(T);
        if (algo == ALG_PR) CK(cudaMemsetAsync(d_sum_, 0, n_ * sizeof(double), cs_));
        // ---- Static Computing, overlapping the transfer
        if (T.n_small + T.n_med + T.n_hub) {
            e0 = open_span(cs_);
            launch_static(algo, d, q, d_static_, T.n_small, T.n_med, T.n_hub, T.n_pieces, kPieceArcs, cs_);
            CK(cudaGetLastError());
            close_span(e0, cs_, t, PH_STATIC);
        }
        st_.static_arcs += T.hit_arcs;
        st_.ondemand_arcs += T.miss_arcs;
        // ---- On-demand request, fragmented into chunks
        const unsigned long long miss = T.miss_arcs;
        const uint32_t nchunks = miss ? (uint32_t)((miss + cap_arcs - 1) / cap_arcs) : 0;
        int mode = 1;
        if (nchunks) {
            if (opt_xfer_mode_ == 2) mode = 2;
            else if (opt_xfer_mode_ == 1) mode = 1;
            else mode = (T.n_runs <= kRunsHostMax && miss * b_e_ / std::max<uint32_t>(1, T.n_runs) >= opt_dma_min_run_) ? 2 : 1;
            if (mode == 2) {
                rb.resize(T.n_runs); re.resize(T.n_runs); rdst.resize(T.n_runs);
                CK(cudaMemcpy(rb.data(), d_run_b_, T.n_runs * 4ull, cudaMemcpyDeviceToHost));
                CK(cudaMemcpy(re.data(), d_run_e_, T.n_runs * 4ull, cudaMemcpyDeviceToHost));
                st_.d2h_bytes += T.n_runs * 8ull;
                unsigned long long acc = 0;
                for (uint32_t r = 0; r < T.n_runs; ++r) { rdst[r] = acc; acc += h_off_[re[r]] - h_off_[rb[r]]; }
            }
            if (!opt_overlap_) {
                cudaEvent_t es = pool_.get();
                CK(cudaEventRecord(es, cs_));
                CK(cudaStreamWaitEvent(xs_, es, 0));
            }
        }
        for (uint32_t k = 0; k < nchunks; ++k) {
            const int buf = k & 1;
            const unsigned long long lo = (unsigned long long)k * cap_arcs;
            const unsigned long long hi = std::min(miss, lo + cap_arcs);
            if (k >= 2) CK(cudaStreamWaitEvent(xs_, consumed_[buf], 0));
            e0 = open_span(xs_);
            transfer_chunk(q, buf, lo, hi, mode, rb, re, rdst);
            CK(cudaGetLastError());
            close_span(e0, xs_, t, mode == 2 ? PH_DMA : PH_GATHER);
            if (mode == 2) st_.dma_bytes += (hi - lo) * b_e_; else st_.gather_bytes += (hi - lo) * b_e_;
            CK(cudaEventRecord(ready_[buf], xs_));
            CK(cudaStreamWaitEvent(cs_, ready_[buf], 0));
            e0 = open_span(cs_);
            launch_ondemand(algo, d, q, d_chunk_[buf], lo, hi, cs_);   // On-demand Computing
            CK(cudaGetLastError());
            close_span(e0, cs_, t, PH_OND);
            CK(cudaEventRecord(consumed_[buf], cs_));
        }
        // ---- next active set
        e0 = open_span(cs_);
        launch_finalize(algo, d, cs_);
        CK(cudaGetLastError());
        close_span(e0, cs_, t, PH_FIN);
        is.chunks = nchunks;
        is.mode = nchunks ? (uint32_t)mode : 0u;
        st_.chunks_total += nchunks;
        if (nchunks && mode == 2) st_.dma_chunks += nchunks; else if (nchunks) st_.gather_chunks += nchunks;
        st_.h2d_payload_bytes += is.miss_bytes;
        st_.active_arcs_total += is.active_arcs;
        iters_.push_back(is);
        host_s += std::chrono::duration<double>(std::chrono::steady_clock::now() - th0).count();
    }
    CK(cudaEventRecord(ev_end, cs_));
    CK(cudaStreamSynchronize(cs_));
    CK(cudaStreamSynchronize(xs_));
    float ms = 0.f;
    CK(cudaEventElapsedTime(&ms, ev_start, ev_end));
    float fill_ms = 0.f;
    CK(cudaEventElapsedTime(&fill_ms, ev_fill0, ev_fill1));
    double ph[PH_N] = {0, 0, 0, 0, 0, 0};
    for (const Span& sp : spans) {
        float a = 0.f;
        CK(cudaEventElapsedTime(&a, sp.a, sp.b));
        ph[sp.ph] += a;
        if (sp.iter < iters_.size()) {
            auto& is = iters_[sp.iter];
            switch (sp.ph) {
                case PH_CLS: is.ms_classify += a; break;
                case PH_STATIC: is.ms_static += a; break;
                case PH_OND: is.ms_ondemand += a; break;
                case PH_GATHER: case PH_DMA: is.ms_h2d += a; break;
                default: is.ms_finalize += a; break;
            }
        }
    }
    for (auto& is : iters_)
        is.ms_total = is.ms_classify + is.ms_static + is.ms_ondemand + is.ms_finalize;
    st_.algo = algo;
    st_.iterations = t;
    st_.n = n_; st_.m = m_; st_.b_e = b_e_;
    st_.rank = 0; st_.world = 1;
    st_.s = pl_.s;
    st_.budget_bytes = pl_.B;
    st_.static_reserved = pl_.Ms;
    st_.static_bytes = pl_.static_bytes;
    st_.ondemand_bytes = pl_.C;
    st_.chunk_cap = cap_;
    st_.static_fraction_used = pl_.R;
    st_.h2d_static_fill_bytes = fill_bytes;
    st_.h2d_other_bytes = 0;
    st_.time_run_s = ms / 1e3;
    st_.time_fill_s = fill_ms / 1e3;
    st_.time_classify_s = ph[PH_CLS] / 1e3;
    st_.time_static_s = ph[PH_STATIC] / 1e3;
    st_.time_ondemand_s = ph[PH_OND] / 1e3;
    st_.time_gather_s = ph[PH_GATHER] / 1e3;
    st_.time_dma_s = ph[PH_DMA] / 1e3;
    st_.time_finalize_s = ph[PH_FIN] / 1e3;
    st_.time_host_s = host_s;
    st_.time_h2d_busy_s = (ph[PH_GATHER] + ph[PH_DMA] + fill_ms) / 1e3;
    st_.gteps = st_.time_run_s > 0 ? (double)st_.active_arcs_total / st_.time_run_s / 1e9 : 0.0;
    const double ex = st_.time_run_s - st_.time_fill_s;
    st_.gteps_excl_fill = ex > 0 ? (double)st_.active_arcs_total / ex / 1e9 : 0.0;
    st_.vertex_state_bytes = vertex_bytes_;
    st_.kernel_launches = g_launches - launches0;
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
    if (!dst || bytes < 4 * n_) throw Error(ASCETIC_EINVAL, "result buffer must hold 4n bytes");
    CK(cudaSetDevice(device_));
    const void* src = (last_algo_ == ALG_PR) ? (const void*)d_rank_ : (const void*)d_val_;
    CK(cudaMemcpy(dst, src, 4 * n_, cudaMemcpyDeviceToHost));
}

void Engine::unload() {
    if (state_ == 0 && !h_tot_) return;
    if (device_ >= 0) cudaSetDevice(device_);
    if (cs_) cudaStreamSynchronize(cs_);
    if (xs_) cudaStreamSynchronize(xs_);
    free_budget_regions();
    dfree(d_off_); dfree(d_A_); dfree(d_S_); dfree(d_next_); dfree(d_visited_);
    dfree(d_val_); dfree(d_snap_); dfree(d_rank_); dfree(d_contrib_); dfree(d_sum_); dfree(d_dang_);
    dfree(d_hq_small_); dfree(d_hq_med_); dfree(d_hq_hub_); dfree(d_hub_pre_);
    dfree(d_mq_); dfree(d_mq_pre_); dfree(d_mq_src_); dfree(d_tile_first_); dfree(d_run_b_); dfree(d_run_e_); dfree(d_run_dst_);
    dfree(d_tile_agg_); dfree(d_tile_incl_); dfree(d_tile_flag_); dfree(d_tot_);
    if (h_tot_) { cudaFreeHost(h_tot_); h_tot_ = nullptr; }
    if (h_registered_) { cudaHostUnregister(h_registered_); h_registered_ = nullptr; }
    if (h_owned_) { cudaFreeHost(h_owned_); h_owned_ = nullptr; }
    for (int i = 0; i < 2; ++i) {
        if (ready_[i]) cudaEventDestroy(ready_[i]);
        if (consumed_[i]) cudaEventDestroy(consumed_[i]);
        ready_[i] = consumed_[i] = nullptr;
    }
    if (ev_classified_) { cudaEventDestroy(ev_classified_); ev_classified_ = nullptr; }
    if (cs_) { cudaStreamDestroy(cs_); cs_ = nullptr; }
    if (xs_) { cudaStreamDestroy(xs_); xs_ = nullptr; }
    h_nbr_ = h_nbr_dev_ = nullptr;
    h_off_ = nullptr;
    h_off_copy_.clear();
    h_off_copy_.shrink_to_fit();
    n_ = m_ = 0;
    state_ = 0;
    have_result_ = false;
    last_algo_ = -1;
    cudaGetLastError();
}

}  // namespace ascetic
