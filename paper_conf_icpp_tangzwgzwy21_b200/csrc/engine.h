// engine.h — the host-side run controller behind the C ABI (include/ascetic.h).
//
//   HostGraph : the caller's CSR, pinned (the paper's host "Edgelist")
//   Part      : one rank's device engine — its owned vertex range [vlo, vhi), replicated
//               vertex state, its Static Region + On-demand Region, its two streams
//   Engine    : the ABI context; drives its local parts phase by phase
//               (classify -> static + transfer + on-demand -> exchange -> finalize) and owns
//               the Comm (NCCL across processes, or P ranks emulated on one GPU)
#pragma once
#include <array>
#include <cstdint>
#include <memory>
#include <stdexcept>
#include <string>
#include <vector>

#include <cuda_runtime.h>

#include "../../include/ascetic.h"
#include "ascetic_internal.h"
#include "comm.h"

namespace ascetic {

// An error that maps onto an ascetic_status at the ABI.
struct Error : std::runtime_error {
    int code;
    Error(int c, const std::string& m) : std::runtime_error(m), code(c) {}
};

// Eq. 1/Eq. 2 placement (§3.3; K = 0.10; 16 KiB) over the
// rows [0, n) of `off` (absolute offsets; the rows' first arc is off[0]).
struct Placement {
    double R = 0.0;
    uint64_t D = 0, B = 0, Ms = 0, s = 0, static_bytes = 0, C = 0, cap = 0;
};
Placement place(const uint64_t* off, uint64_t n, uint32_t b_e, uint64_t budget, double frac);

// 1D edge-balanced vertex ranges: b_0 = 0, b_P = n, b_g = min{v : off[v] >= ceil(g m / P)}.
std::vector<uint64_t> partition(const uint64_t* off, uint64_t n, uint32_t P);

struct EventPool {
    std::vector<cudaEvent_t> ev;
    size_t used = 0;
    cudaEvent_t get();
    void reset() { used = 0; }
    ~EventPool();
};

struct Options {
    uint64_t chunk_cap = 0;
    int xfer_mode = 0;
    uint64_t dma_min_run = 64 * 1024;
    int overlap = 1;
    int keep_static = 0;
    uint32_t hub_deg = 2048;
    int timing = 1;
    int gather_ctas = 0;
    int chunk_buffers = 0;   // On-demand Region split into this many chunk buffers of C/N bytes;
                             // 0 = auto: 3 (absorbs one slow on-demand kernel without stalling the
                             // link), 2 when C/3 < 4 MiB (chunks that small are latency-bound)
    int static_ctas_per_sm = 0;   // persistent grid of the static-hit kernels (0 = 4 per SM)
    int prefetch = 1;             // PR: issue the next iteration's first chunk transfers early
    int repartition = 0;          // Eq. 3 adaptive re-partition (off, as in the paper's evaluation)
    int placement = 0;            // initial static content: 0 = front prefix, 1 = rear suffix, 2 = random chunks
    uint64_t placement_seed = 1;  // seed of the random initial chunk set
    uint64_t prd_tol_ppm = 10000; // PageRank-delta threshold, ppm of the initial residual (1-d)/n
    int fused_exchange = 0;       // P > 1: exchange fused into finalize over peer memory (NVLink / IPC)
    uint32_t sparse_exchange = 0; // P > 1, SSSP/CC: sparse MIN when every rank has <= n/(d P) pairs (0 = off)
    uint32_t replace_k = 0;       // §3.4 data replacement: chunk swaps examined per iteration (0 = off)
    int replace_policy = 0;       // hotness counter: 0 = by algorithm, 1 = cumulative, 2 = last iteration
    int relax_mode = 0;           // SSSP/CC min update: 0 = auto, 1 = atomicMin + next bit, 2 = RED.MIN + dense finalize
    uint64_t ce_min_run = 1ull << 20;   // gather-mode iterations: runs >= this many bytes go to the copy engines (0 = off)
    uint64_t pr_segment = 128ull << 20; // PR static pull: neighbour-id slice of contrib per pass (0 = off; 128 MiB:
                                        // friendster-shaped resident pull -22 %, profiles/r02/prseg_ab_c3.log)
    double span_density = 0.85;         // span DMA of a window when payload >= this share of its host bytes (0 = off)
    uint64_t span_min_bytes = 64ull << 20;   // ... in iterations with at least this much payload
    double span_max_ratio = 2.0;        // ... whose host span is at most this many times the payload
    int fused_visit = 1;                // BFS gathered chunks: visit in the gather (1 = small chunks, 2 = all, 0 = off)
    uint32_t gap_bridge = 0;            // gather: also load host holes <= this many bytes between pieces (0 = off;
                                        // measured no gain: C2/C4 A/B, profiles/r02/gather_ab_c4.log)
};

struct HostGraph {
    uint64_t n = 0, m = 0;
    uint32_t b_e = 4, flags = 0;
    const uint64_t* off = nullptr;    // host offsets (caller's, or off_own): placer, partition, DMA planning
    std::vector<uint64_t> off_own;    // private copy with ASCETIC_COPY
    const void* nbr = nullptr;        // b_e bytes per arc, pinned
    const void* nbr_dev = nullptr;    // device-visible alias (zero-copy)
    void* owned = nullptr;            // library-owned pinned copy
    void* registered = nullptr;       // pinned in place by us: [registered, registered + reg_bytes)
    size_t reg_bytes = 0;
    uint64_t arc_lo = 0, arc_hi = 0;  // host arcs this process reads (its ranks' rows; all with emulation)
    void release();
};

enum { PH_CLS, PH_STATIC, PH_OND, PH_GATHER, PH_DMA, PH_FIN, PH_XCH, PH_REPL, PH_N };

class Part {
  public:
    Part(const HostGraph& g, const Options& o, int rank, uint64_t vlo, uint64_t vhi, int sm_count);
    ~Part();
    void alloc_vertex_state();
    void alloc_algo_state(int algo, bool multi);
    void upload_off();
    void set_budget(uint64_t bytes, double frac);
    void on_reload() { static_valid_ = false; }

    // one run, phase by phase
    void begin(int algo, uint32_t source, uint32_t max_iters, bool timing);
    void classify(uint32_t t);
    IterTotals wait_classify();
    void expand(uint32_t t, const IterTotals& T);
    void debug_classify(const uint32_t* active_words, uint64_t nwords, ascetic_classify_out_t* out);
    bool maybe_repartition(const IterTotals& T);   // Eq. 3; true = re-generate the data map
    void replace(uint32_t t);                      // §3.4: hotness update + chunk swaps (effective at t+1)
    void join_static();   // cs waits for this iteration's static-hit kernels
    void finalize(uint32_t t, bool dense);
    // fused exchange (P > 1): the peer tables and the finalize that reads every rank's buffer
    void set_fused(bool on);   // this run uses the fused exchange (allocates the second next buffer)
    void set_red_min(bool on) { red_min_ = on; }   // SSSP/CC: RED.MIN updates, A_{t+1} from val < snap
    void set_peers(int kind, const std::vector<void*>& ptrs);   // kind 0/1: next[0/1], 2: val or inc
    void finalize_fused(uint32_t t);
    void clear_next(uint32_t b);
    void clear_prd_inc();
    uint32_t* next_buf(int b) const { return b ? d_next2_ : d_next_; }
    void end();
    void span(cudaEvent_t a, cudaStream_t s, uint32_t t, int ph, int sub = 0);   // close a timed span
    cudaEvent_t mark(cudaStream_t s, bool always = false);          // open a timed span

    cudaStream_t cs() const { return cs_; }
    const unsigned long long* dev_off() const { return d_off_; }
    cudaEvent_t sync_event() const { return sync_ev_; }
    DevState dev_state(uint32_t iter) const;
    const Placement& placement() const { return pl_; }
    uint64_t cap() const { return cap_; }
    uint64_t vlo() const { return vlo_; }
    uint64_t vhi() const { return vhi_; }
    uint32_t* next() const { return d_next_; }
    uint32_t* val() const { return d_val_; }
    float* rank_arr() const { return d_rank_; }
    float* contrib() const { return d_contrib_; }
    unsigned long long* prd_inc() const { return d_pr_inc_; }
    unsigned long long* dang() const { return d_dang_; }
    uint64_t vertex_bytes() const { return vertex_bytes_; }

    // results of the last run
    ascetic_stats_t st{};
    std::vector<ascetic_iter_stats_t> iters;

  private:
    void transfer_chunk(const Queues& q, int buf, unsigned long long lo, unsigned long long hi, int mode,
                        cudaStream_t xs,
                        const DevState* visit = nullptr);
    uint32_t plan_long_runs(const IterTotals& T);   // gather mode: the long runs for the copy engines
    bool plan_span_windows(const IterTotals& T);    // span-DMA mode: the windows' miss-stream positions
    Queues queues(const IterTotals& T) const;
    void free_regions();
    void layout_regions(uint64_t Ms);

    const HostGraph& g_;
    const Options& o_;
    int rank_;
    uint64_t vlo_, vhi_;
    int sm_count_;
    int algo_ = 0;
    bool timing_ = true;
    bool fine_ = true;   // this iteration records per-phase spans
    // device vertex state
    uint32_t nwords_ = 0, ntiles_ = 0, wpw_ = 32;
    unsigned long long* d_off_ = nullptr;
    uint32_t *d_A_ = nullptr, *d_S_ = nullptr, *d_next_ = nullptr, *d_visited_ = nullptr;
    uint32_t *d_val_ = nullptr, *d_snap_ = nullptr;
    float *d_rank_ = nullptr, *d_contrib_ = nullptr;
    unsigned long long *d_pr_r_ = nullptr, *d_pr_res_ = nullptr, *d_pr_c_ = nullptr;   // PageRank-delta
    unsigned long long* d_pr_inc_ = nullptr;   // P > 1: residual increments of this rank's pushes
    bool multi_ = false;
    bool fused_ = false;
    bool red_min_ = false;
    uint32_t* d_next2_ = nullptr;              // fused exchange: next bitmaps double-buffered by iteration parity
    const void** d_peers_ = nullptr;           // [3][world] device pointers (next0, next1, val/inc)
    int peer_world_ = 0;
    uint64_t prd_tau_ = 0;
    unsigned long long *d_sum_ = nullptr, *d_dang_ = nullptr;   // PR, 2^-62 fixed point
    uint32_t *d_hq_small_ = nullptr, *d_hq_med_ = nullptr, *d_hq_hub_ = nullptr, *d_hub_pre_ = nullptr;
    uint32_t *d_mq_ = nullptr, *d_run_b_ = nullptr, *d_run_e_ = nullptr, *d_tile_first_ = nullptr;
    unsigned long long *d_mq_pre_ = nullptr, *d_mq_src_ = nullptr, *d_run_dst_ = nullptr;
    uint64_t hub_cap_ = 0;
    ScanVal *d_tile_agg_ = nullptr, *d_tile_incl_ = nullptr;
    uint32_t* d_tile_flag_ = nullptr;
    uint32_t epoch_ = 0;
    IterTotals* d_tot_ = nullptr;   // [2]
    uint32_t tot_buf_ = 0;
    IterTotals* h_tot_ = nullptr;   // mapped pinned
    uint32_t* h_runs_ = nullptr;    // mapped pinned (b, e) pairs of the first kRunsHostMax runs
    uint64_t vertex_bytes_ = 0;
    // edge budget regions (Eq. 1/2)
    Placement pl_{};
    char* arena_ = nullptr;          // the edge budget: Static Region + On-demand Region
    uint64_t arena_bytes_ = 0;
    uint64_t ms_cur_ = 0, s_cur_ = 0; // current split (Eq. 3 may shrink it during a run)
    uint64_t stat_lo_ = 0;            // first static vertex: vlo (front) or the rear suffix start
    void* d_static_ = nullptr;
    static constexpr int kMaxBuffers = 8;
    char* d_chunk_[kMaxBuffers] = {};
    int nbuf_ = 2, nbuf_alloc_ = 0;   // chunk buffers in use / allocated
    uint64_t cap_ = 0, static_alloc_ = 0, chunk_alloc_ = 0;
    bool static_valid_ = false;
    std::array<uint64_t, 6> static_key_{};   // placement, seed, first static vertex, s, slot bytes, slots on
    // streams / events
    cudaStream_t cs_ = nullptr, xs_ = nullptr, ss_ = nullptr;   // compute, copy, static-hit streams
    cudaEvent_t ready_[kMaxBuffers] = {}, consumed_[kMaxBuffers] = {};
    cudaEvent_t static_go_ = nullptr, static_done_ = nullptr, sync_ev_ = nullptr;
    bool static_pending_ = false;
    uint64_t gchunk_ = 0;            // chunks issued so far in this run (buffer = gchunk % nbuf)
    uint32_t prefetched_ = 0;        // next iteration's chunks already issued (PR prefetch)
    unsigned long long prefetch_miss_ = 0;
    uint32_t prefetch_runs_ = 0;
    uint32_t max_iters_ = 0;
    cudaEvent_t ev_classified_ = nullptr;
    EventPool pool_;
    struct Span { cudaEvent_t a, b; uint32_t iter; int ph; int sub; };
    std::vector<Span> spans_;
    cudaEvent_t ev_start_ = nullptr, ev_fill0_ = nullptr, ev_fill1_ = nullptr;
    double host_s_ = 0.0;
    unsigned long long launches0_ = 0;
    // §3.4 data replacement: the Static Region as hNS_ slots of 16 KiB over the rank's hNC_ chunks
    bool hot_ = false, hot_dirty_ = false, acc_pending_ = false, static_launched_ = false;
    uint64_t hNC_ = 0, hNS_ = 0, hot_alloc_nc_ = 0;
    uint32_t hot_alloc_k_ = 0;
    uint32_t *d_slot_of_ = nullptr, *d_acc_ = nullptr, *d_swap_ = nullptr;
    uint32_t *h_acc_ = nullptr, *h_swap_ = nullptr;     // pinned
    std::vector<uint32_t> slot_of_, slot_chunk_;       // host mirror: chunk -> slot, slot -> chunk
    std::vector<uint32_t> init_chunks_;                // initial resident chunks, ascending (slot i = init_chunks_[i])
    uint32_t* d_init_ = nullptr;                       // device copy of init_chunks_ (fill list)
    uint64_t init_fill_bytes_ = 0;
    std::vector<uint64_t> hot_h_;                      // HotnessTable (Fig. 6)
    cudaEvent_t ev_acc_ = nullptr, ev_swapped_ = nullptr;
    void free_hot();
    // DMA planning scratch
    std::vector<uint32_t> rb_, re_;
    std::vector<unsigned long long> rdst_;
    // hybrid gather: long runs by the copy engines on a second copy stream, the rest by the SM gather
    static constexpr uint32_t kLongMax = 1u << 16;
    unsigned long long* h_long_ = nullptr;          // mapped: (b, e, dst) x kLongMax, unordered
    uint32_t* h_long_flag_ = nullptr;               // mapped: [0] ready, [1] count
    uint32_t* d_long_cnt_ = nullptr;                // device: count, done
    unsigned long long* h_lint_[2] = {};            // pinned staging of the sorted stream intervals (by parity)
    unsigned long long* d_lint_[2] = {};            // device copies read by the gather
    uint32_t nlint_ = 0, lint_buf_ = 0;
    std::vector<uint32_t> lb_, le_;                  // this iteration's long runs, by stream position
    std::vector<unsigned long long> ldst_;
    cudaStream_t xs2_ = nullptr;
    cudaStream_t xs34_[2] = {nullptr, nullptr};   // small-chunk pipeline: buffers 2 and 3's own streams
    cudaEvent_t ce_done_[kMaxBuffers] = {}, xfer_go_[kMaxBuffers] = {}, ev_long_ = nullptr, ev_pipe_ = nullptr;
    unsigned long long* d_cover_ = nullptr;          // gather: 16-byte units loaded (link bytes / 16)
    unsigned long long* h_cover_ = nullptr;          // its pinned host copy, read after the run's end
    static constexpr uint32_t kSpanWinMax = 4096;
    unsigned long long* h_win_ = nullptr;            // mapped: span windows' first miss-stream positions (nwin + 1)
    uint32_t* h_span_flag_ = nullptr;                // mapped: [0] ready
    uint32_t span_nwin_ = 0;
    uint32_t* d_seg_cur_ = nullptr;                  // PR segmented pull: cursors (medium rows, then hub pieces)
    uint64_t seg_cur_n_ = 0;
    static constexpr uint32_t kPieceArcs = 4096;
    static constexpr uint32_t kRunsHostMax = 8192;
};

class Engine {
  public:
    ~Engine();
    void set_device(int dev);
    void comm_init(int rank, int world, const void* uid, int device);
    void emulate_ranks(int world);
    void load_csr(uint64_t n, uint64_t m, const uint64_t* off, const uint32_t* nbr, const uint32_t* wgt,
                  uint32_t flags);
    void set_budget(uint64_t bytes, double frac);
    void set_option(int opt, int64_t value);
    void debug_classify(int rank, const uint32_t* active_words, uint64_t nwords, ascetic_classify_out_t* out);
    void run(int algo, uint32_t source, uint32_t max_iters);
    int stats(ascetic_stats_t* out, ascetic_iter_stats_t* per_iter, uint32_t cap) const;
    void get_result(void* dst, uint64_t bytes);
    void unload();

  private:
    void join();                                      // all local parts' cs -> parts_[0].cs
    void fork();                                      // parts_[0].cs -> all local parts' cs

    int state_ = 0;   // 0 unloaded, 1 loaded, 2 ready
    int device_ = -1;
    int sm_count_ = 148;
    HostGraph g_;
    Options o_;
    Comm comm_;
    int emulate_ = 1;
    std::vector<std::unique_ptr<Part>> parts_;
    std::vector<uint64_t> bounds_;
    int last_algo_ = -1;
    bool have_result_ = false;
    ascetic_stats_t st_{};
    std::vector<ascetic_iter_stats_t> iters_;
    // sparse MIN exchange buffers, one per local part: (id, value) pairs and their count
    std::vector<void*> sp_pairs_;
    std::vector<uint32_t*> sp_cnt_;
    uint32_t sp_cap_ = 0;
    void free_sparse();
};

}  // namespace ascetic
