// ascetic_internal.h — device data layout and kernel launchers of libascetic.so.
//
// Layout in HBM (DESIGN.md §"Data layout"):
//   resident vertex state (outside the edge budget):
//     off      uint64[n+1]      CSR offsets
//     A, S     uint32[nw]       ActiveBitmap / StaticBitmap, nw = ceil(n/32)
//     next     uint32[nw]       next-frontier bits set by the edge kernels
//     visited  uint32[nw]       BFS only
//     val      uint32[n]        level / dist / label;  snap uint32[n] Jacobi snapshot (SSSP, CC)
//     rank f32[n], contrib f32[n], sum f64[n]  PageRank
//     hit queues (small / medium / hub) uint32, hub piece prefix uint32,
//     miss queue uint32 + its arc prefix uint64, miss runs (b,e) uint32 + dst uint64
//   edge budget B (Eq. 1/2):
//     static   b_e * off[s] bytes = host nbr bytes [0, b_e*off[s])   (Static Region)
//     chunk[2] cap bytes each                                        (On-demand Region)
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace ascetic {

constexpr uint32_t kInf = 0xFFFFFFFFu;
constexpr double kFxOne = 4611686018427387904.0;         // 2^62: PR sums are < 2 (Σ_v sum = Σ r <= 1)
constexpr int kClassifyWarps = 8;                       // words per tile = 8 * 32
constexpr int kTileWords = kClassifyWarps * 32;         // 256 words = 8192 vertices
constexpr uint32_t kSmallDeg = 32;                      // hit lists shorter than this: warp-cooperative
constexpr int kEdgeTileShift = 11;
constexpr int kEdgeTile = 1 << kEdgeTileShift;          // arcs per CTA tile of the miss stream

// Scan fields of the order-preserving compaction (one decoupled look-back pass).
struct ScanVal {
    uint32_t small, med, hub, missq, runs, pieces;
    unsigned long long miss_arcs;
};

// Per-iteration totals. Written by the last classify block into device memory AND
// into mapped pinned host memory (the only device->host traffic per iteration).
struct IterTotals {
    unsigned long long nA, nH, nM, active_arcs, hit_arcs, digest;
    unsigned long long miss_arcs;
    uint32_t n_small, n_med, n_hub, n_missq, n_runs, n_pieces;
    uint32_t tile_counter, done_counter;
    uint32_t ready;          // set to 1 last (host spin target)
    uint32_t host_runs;      // runs copied to the mapped run list (0 = not copied)
    unsigned long long nS;   // |S ∩ owned range| (static vertices of this rank in this iteration)
    unsigned long long miss_h0, miss_h1;   // host arc span of the miss stream: off[first miss], off[last miss + 1]
};

struct ClassifyArgs {
    const uint32_t* A;
    const uint32_t* S;
    const unsigned long long* off;
    uint64_t n;
    uint64_t vlo, vhi;                 // owned vertex range of this rank
    uint32_t nwords;
    uint32_t ntiles;
    uint32_t words_per_warp;           // 32, or 4 for small bitmaps (tile = kClassifyWarps * words_per_warp words)
    uint32_t hub_deg;
    uint32_t piece_arcs;
    uint32_t* hq_small;
    uint32_t* hq_med;
    uint32_t* hq_hub;
    uint32_t* hub_pre;                 // exclusive prefix of pieces per hub
    uint32_t* mq;                      // miss vertices with deg > 0, ascending
    unsigned long long* mq_pre;        // exclusive prefix of miss arcs at each mq entry
    unsigned long long* mq_src;        // off[v] of each mq entry (host arc index of its list)
    uint32_t* tile_first;              // [t] = mq index of the vertex holding miss arc t*kEdgeTile
    uint32_t* run_b;
    uint32_t* run_e;
    unsigned long long* run_dst;       // exclusive prefix of miss arcs at run start
    ScanVal* tile_agg;
    ScanVal* tile_incl;
    uint32_t* tile_flag;
    uint32_t epoch;
    IterTotals* tot;                   // device, zero on entry
    IterTotals* tot_next;              // device: zeroed by the last CTA for the next classify (no memset launch)
    IterTotals* host_tot;              // mapped pinned
    uint32_t* host_runs;               // mapped pinned: (b, e) of the first host_runs_cap runs, written (by the
    uint32_t host_runs_cap;            // last CTA) only when the host will plan DMAs: force_host_runs, or at
    uint32_t force_host_runs;          // most host_runs_cap runs averaging >= dma_min_run_arcs arcs
    unsigned long long dma_min_run_arcs;
};

// Device state handed to the edge / finalize kernels.
struct DevState {
    const unsigned long long* off;
    uint64_t n;
    uint32_t nwords;
    uint32_t* A;
    uint32_t* S;
    uint32_t* next;
    uint32_t* visited;
    uint32_t* val;
    uint32_t* snap;
    float* rank;
    float* contrib;
    // PR pull sums and dangling mass in 2^-62 fixed point (u64): every fp64 partial (a row, a hub
    // piece, a chunk segment of a row) is rounded once to the grid and added as an integer, so the
    // totals do not depend on the order the atomics land in (bitwise-reproducible ranks, DESIGN R31)
    unsigned long long* sum;
    unsigned long long* dang;   // [0] = current dangling mass, [1] = next
    uint32_t iter;         // t
    uint64_t vlo, vhi;     // owned vertex range (PR finalize)
    unsigned long long static_arc0;   // first arc held by the Static Region (off[vlo])
    // §3.4 replacement: Static Region = 16 KiB slots; slot_of[c] = slot of rank-local chunk c
    // (kNoSlot if not resident). nullptr = contiguous prefix (no remapping).
    const uint32_t* slot_of;
    // PageRank-delta (fixed point 2^-56): rank, residual, push value; tau = activation threshold
    unsigned long long *pr_r, *pr_res, *pr_c;
    unsigned long long* pr_inc;        // P > 1: this rank's increments (summed across ranks), else nullptr
    unsigned long long tau;
    uint32_t red_min;                  // SSSP/CC: fire-and-forget RED.MIN + dense finalize (no next bits)
};

constexpr uint32_t kNoSlot = 0xFFFFFFFFu;
constexpr int kChunkShift = 14;                          // §3.4 16 KB chunks
constexpr uint64_t kChunkBytes = 1ull << kChunkShift;

struct Queues {
    const uint32_t* hq_small;
    const uint32_t* hq_med;
    const uint32_t* hq_hub;
    const uint32_t* hub_pre;
    const uint32_t* mq;
    const unsigned long long* mq_pre;
    const unsigned long long* mq_src;
    const uint32_t* tile_first;
    uint32_t n_missq;
    unsigned long long miss_arcs;      // total miss-stream length (arcs)
};

// kernels launched by this library (bench's gpu_launches claim); defined in edges.cu
extern unsigned long long g_launches;

// ---- launchers (frontier.cu) ----
void launch_classify(const ClassifyArgs& a, cudaStream_t s);

// ---- launchers (edges.cu) ----
void launch_init(int algo, const DevState& d, uint32_t source, cudaStream_t s);
void launch_static(int algo, const DevState& d, const Queues& q, const void* static_base,
                   uint32_t n_small, uint32_t n_med, uint32_t n_hub, uint32_t n_pieces,
                   uint32_t piece_arcs, int max_ctas, cudaStream_t s);
// PR static pull in `passes` neighbour-id slices (contrib slice L2-resident per pass); small rows unsegmented;
// cur_med[n_med], cur_hub[npieces]: per-row / per-piece cursors (scratch). Front prefix only (no slot remap).
void launch_static_pr_seg(const DevState& d, const Queues& q, const void* sbase, uint32_t ns, uint32_t nm, uint32_t nh,
                          uint32_t npieces, uint32_t piece, uint32_t passes, uint32_t* cur_med, uint32_t* cur_hub,
                          int max_ctas, cudaStream_t s);
// on-demand computing of miss-stream arcs [lo, hi): chunk = the compacted stream (span_base = ~0) or
// the host arcs [span_base, ...) verbatim (span DMA)
void launch_ondemand(int algo, const DevState& d, const Queues& q, const void* chunk, unsigned long long lo,
                     unsigned long long hi, unsigned long long span_base, cudaStream_t s);
// span windows: for k in [0, nwin], the miss-stream position of host arc h0 + k * win (h1 for k = nwin)
void launch_span_windows(const Queues& q, unsigned long long h0, unsigned long long h1, unsigned long long win,
                         uint32_t nwin, unsigned long long* out, uint32_t* flag, cudaStream_t s);
// zero-copy gather of miss-stream arcs [lo, hi) into chunk; skips the vertices inside the sorted long
// stream intervals lint[2i, 2i+1) (copied by the copy engines), bridges host holes <= gap_bytes;
// adds the number of 16-byte host units it loads to *cover
void launch_gather(const Queues& q, const void* host_nbr, uint64_t m, uint32_t b_e, void* chunk,
                   unsigned long long lo, unsigned long long hi, int max_ctas, const unsigned long long* lint,
                   uint32_t nlint, uint32_t gap_bytes, unsigned long long* cover, cudaStream_t s,
                   const DevState* visit = nullptr);   // BFS: visit the landed ids in the gather (fused)
// long miss runs (>= min_arcs arcs): append (b, e, dst) of each into out[3*i] (mapped host memory,
// unordered, at most cap), count into *count; `flag` set to 1 by the last CTA (host spin target)
void launch_long_runs(const uint32_t* run_b, const uint32_t* run_e, const unsigned long long* run_dst, uint32_t n_runs,
                      const unsigned long long* off, unsigned long long min_arcs, unsigned long long* out, uint32_t cap,
                      uint32_t* count, uint32_t* done, uint32_t* flag, cudaStream_t s);
// §3.4: per-chunk accesses (active arcs) of this iteration's hit + miss queues into acc
void launch_chunk_access(const DevState& d, const Queues& q, uint32_t n_small, uint32_t n_med, uint32_t n_hub,
                         uint32_t b_e, uint32_t* acc, cudaStream_t s);
// §3.4: apply swaps (in[i] gets out[i]'s slot) and recompute S for the vertices touching the changed chunks
void launch_apply_swaps(const DevState& d, uint32_t* slot_of, const uint32_t* swaps /* in[k], out[k], slot[k] */,
                        uint32_t k, uint32_t b_e, cudaStream_t s);
// copy `count` 16 KiB chunks ids[i] of the rank's payload (host bytes x0 + 16 KiB * id, the last
// chunk clipped at D) from the mapped host CSR into slot slots[i] (or i) of the Static Region
void launch_copy_chunks(const void* host_dev, uint64_t x0, uint64_t D, const uint32_t* ids, const uint32_t* slots,
                        uint32_t count, void* dst, cudaStream_t s);
// S := {v in [vlo, vhi) : every chunk of v's list is resident} (full rebuild)
void launch_static_bits(const DevState& d, const uint32_t* slot_of, uint32_t b_e, cudaStream_t s);
// dense = values were exchanged (P > 1): SSSP/CC rebuild A from val < snap over all vertices
void launch_finalize(int algo, const DevState& d, bool dense, cudaStream_t s);
// fused exchange + finalize (P > 1): peers = device array of P pointers to every rank's buffer
// (BFS: next bitmaps, SSSP/CC: values, PRD: residual increments)
void launch_finalize_peers(int algo, const DevState& d, const void* const* peers, int P, cudaStream_t s);
// PRD: rank[v] = fp32((r + res) 2^-56)
void launch_prd_output(const DevState& d, cudaStream_t s);
// collectives' device side (comm.cu drives them)
void launch_or_reduce(uint32_t* dst, const uint32_t* gathered, uint32_t parts, uint64_t nw, cudaStream_t s);
void launch_or_into(uint32_t* dst, const uint32_t* src, uint64_t nw, cudaStream_t s);
void launch_min_into(uint32_t* dst, const uint32_t* src, uint64_t n, cudaStream_t s);
// sparse MIN exchange (SSSP / CC): pack this rank's improved (id, value) pairs (count zeroed first;
// at most cap written, *count = the full number), and apply P ranks' pairs (rank `skip` left out)
void launch_sparse_pack(const uint32_t* next, const uint32_t* val, uint32_t nwords, void* pairs, uint32_t cap,
                        uint32_t* count, cudaStream_t s);
void launch_sparse_apply(uint32_t* val, uint32_t* next, const void* pairs, uint64_t stride, const uint32_t* counts,
                         int P, int skip, uint32_t cap, cudaStream_t s);
void launch_add_u64(unsigned long long* dst, const unsigned long long* src, uint64_t n, cudaStream_t s);
// *bad := min{v : off[v+1] < off[v]} (left untouched when off[0..n] is non-decreasing)
void launch_check_monotone(const unsigned long long* off, uint64_t n, unsigned long long* bad, cudaStream_t s);
// bits := the vertex range [a, b)
void launch_set_range_bits(uint32_t* bits, uint32_t nwords, uint64_t a, uint64_t b, cudaStream_t s);

}  // namespace ascetic
