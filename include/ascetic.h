/*
 * ascetic.h — C ABI of libascetic.so, the B200-native hot path of Ascetic
 * (Tang et al., "Ascetic: Enhancing Cross-Iterations Data Efficiency in
 * Out-of-Memory Graph Processing on GPUs", ICPP '21).
 *
 * Citations: "P:NNN" = line NNN of the paper text; "§8(x)" = SURVEY.md.
 *
 * What the library does, per iteration of a push-based vertex-centric BSP
 * algorithm over a CSR graph whose edges exceed a capped device budget
 * (§3.1):
 *   1. GenDataMap: StaticMap = Active AND Static, On-demand Map = StaticMap XOR
 *      Active (Fig. 4), compacted into a hit queue and the
 *      on-demand request sized by degrees.
 *   2. Static Computing on the resident Static Region (Fig. 4 (3))
 *      overlapped with the On-demand transfer (Fig. 5).
 *   3. On-demand Computing on chunks of the On-demand Region, fragmented when the
 *      request exceeds the region (§3.3; Fig. 4 (5)).
 *   4. Next active set "generated based on the connected edges".
 * The device memory split follows Eq. 1/Eq. 2 (§3.3, K = 10 %,
 * P:856-859) with the front prefix as initial static content (§5).
 *
 * Conventions for every call:
 *   - returns ASCETIC_OK (0) or a negative ascetic_status; no C++ exception
 *     crosses the ABI; ascetic_last_error() gives a thread-local message.
 *   - one context per process (one GPU per process); calls are NOT thread-safe.
 *   - host pointers are plain host memory; the library never frees caller memory.
 *   - state machine: UNLOADED --load_csr--> LOADED --set_budget--> READY
 *     --run--> READY (run and set_budget may repeat); out-of-order => ESTATE.
 */
#ifndef ASCETIC_H
#define ASCETIC_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    ASCETIC_OK = 0,
    ASCETIC_EINVAL = -1,       /* bad argument (message says which) */
    ASCETIC_ESTATE = -2,       /* call out of order */
    ASCETIC_ENOMEM = -3,       /* device allocation failed, or budget too small for a chunk */
    ASCETIC_EHOSTMEM = -4,     /* host pin / allocation failed */
    ASCETIC_ECUDA = -5,        /* CUDA runtime error (message has cudaGetErrorString) */
    ASCETIC_ENCCL = -6,        /* collective error (multi-GPU) */
    ASCETIC_EUNSUPPORTED = -7  /* feature not built */
} ascetic_status;

typedef enum { ASCETIC_BFS = 0, ASCETIC_SSSP = 1, ASCETIC_CC = 2, ASCETIC_PR = 3,
               ASCETIC_PRD = 4  /* PageRank-delta: Subway's frontier-driven PR, see run() */
} ascetic_algo;

/* load_csr flags */
enum {
    ASCETIC_SYMMETRIC = 1u,   /* caller asserts both directions are stored; required for CC and PR */
    ASCETIC_COPY = 2u,        /* copy into library-owned pinned memory instead of pinning in place */
    ASCETIC_VALIDATE = 4u,    /* O(m) check that every neighbour id < n */
    ASCETIC_PAIRS = 8u,       /* nbr holds 2m uint32: interleaved (id, weight) per arc */
    ASCETIC_SORTED = 16u      /* caller asserts every row lists its neighbours in ascending id order (checked
                                 with ASCETIC_VALIDATE); lets PR pull in L2-sized neighbour-id slices */
};

/* Tuning knobs (ascetic_set_option). None changes what is computed or the
 * per-iteration payload bytes; they change chunking and the transfer mechanism. */
typedef enum {
    ASCETIC_OPT_CHUNK_CAP = 1,     /* bytes; 0 = from the placer (C/2). Clamped to the placer's cap, multiple of 16 */
    ASCETIC_OPT_XFER_MODE = 2,     /* 0 = auto, 1 = zero-copy SM gather only, 2 = copy-engine DMA of runs only,
                                      3 = span DMA where the miss stream's host span is at most 2x its payload
                                      (windows of cap host bytes; dense ones DMA'd whole and read in place,
                                      sparse ones gathered), else as 0 */
    ASCETIC_OPT_DMA_MIN_RUN = 3,   /* bytes: auto mode uses DMA when every run piece averages >= this */
    ASCETIC_OPT_OVERLAP = 4,       /* 1 (default) = static compute overlaps the transfer; 0 = serialize (ablation, Fig. 8) */
    ASCETIC_OPT_KEEP_STATIC = 5,   /* 1 = keep the Static Region filled across runs (fill counted once) ; default 0 */
    ASCETIC_OPT_HUB_DEGREE = 6,    /* hit-queue degree at/above which a list is split across CTAs (default 2048) */
    ASCETIC_OPT_TIMING = 7,        /* CUDA-event phase timing: 1 (default) = per-phase spans in iterations with >= 2^23
                                      active arcs or >= 32 MiB of misses, one span (the iteration) otherwise;
                                      2 = every phase of every iteration; 0 = off */
    ASCETIC_OPT_GATHER_CTAS = 8,   /* persistent CTAs of the zero-copy gather; 0 (default) = 512 / b_e (~1 MiB in flight) */
    ASCETIC_OPT_CHUNK_BUFFERS = 9, /* On-demand Region C split into N buffers of C/N (2..8; 0 = auto (default): 3, or 2
                                    when C/3 < 4 MiB); set before set_budget */
    ASCETIC_OPT_STATIC_CTAS_PER_SM = 10, /* persistent grid of the static-hit kernels, CTAs per SM (0 = default 4) */
    ASCETIC_OPT_PREFETCH = 11,     /* 1 (default): PR issues the next iteration's first chunk DMAs at the end of the
                                      current one (A_t = V, so the miss stream repeats); 0 = off */
    ASCETIC_OPT_REPARTITION = 12,  /* 1: Eq. 3 adaptive re-partition (§3.3) after each data map:
                                      if V_ondemand > C and V_static/M_static < 0.5 V/D, shrink the Static Region
                                      by M_static*V/D (floored to 16 KiB) and re-generate the map. Default 0, as
                                      in the paper's evaluation. Changes per-iteration bytes. */
    ASCETIC_OPT_STATIC_PLACEMENT = 13, /* initial static content (§5): 0 = front prefix (default),
                                      1 = rear suffix of whole lists fitting in Ms, 2 = random: the
                                      ceil(Ms/16 KiB) chunks with the smallest splitmix64((seed<<32) ^ c)
                                      (Static Region as 16 KiB slots, as with REPLACE_CHUNKS). Set before
                                      set_budget. */
    ASCETIC_OPT_REPLACE_CHUNKS = 14, /* §3.4 data replacement (Fig. 6): K = 16 KiB chunk swaps
                                      examined per iteration and rank (0 = off, the default; max 65536).
                                      The Static Region becomes Ms/16 KiB chunk slots (initially the front
                                      chunks, filled whole); after each iteration's data map, per-chunk access
                                      counters (active arcs read) update the hotness table; during on-demand
                                      computing the K hottest non-resident chunks replace the K coldest
                                      resident ones while strictly hotter, effective next iteration. A vertex
                                      is static iff every chunk its list touches is resident. Front
                                      or random placement; exclusive with Eq. 3. Set before set_budget.
                                      Changes bytes. */
    ASCETIC_OPT_REPLACE_POLICY = 15, /* hotness counter: 0 = by algorithm (default: cumulative for
                                      BFS/SSSP/CC, last iteration for PR), 1 = cumulative, 2 = last iteration */
    ASCETIC_OPT_PLACEMENT_SEED = 16, /* seed of the random initial content (default 1). Set before set_budget. */
    ASCETIC_OPT_PRD_TOL_PPM = 17,    /* PageRank-delta activation threshold tau in ppm of the initial residual
                                      (1-d)/n (default 10000 = 1 %) */
    ASCETIC_OPT_FUSED_EXCHANGE = 18, /* P > 1, BFS/SSSP/CC/PRD: 1 = fuse the per-iteration exchange into the
                                      finalize kernel, which reads every rank's next bitmap / values /
                                      increments straight from peer memory (CUDA IPC over NVLink with the NCCL
                                      back end; the other parts' buffers when emulated), between stream-ordered
                                      barriers; 0 (default) = NCCL collectives. Results are identical. */
    ASCETIC_OPT_SPARSE_EXCHANGE = 19,/* P > 1, BFS/SSSP/CC, collectives path: d >= 1 = sparse exchange (SURVEY
                                      §8(e)): each rank packs the (id, value) pairs it set in its next bitmap this
                                      iteration (lowered values; BFS: newly reached ids), the pairs are
                                      all-gathered and applied with atomicMin + next bit, whenever every rank has
                                      at most max(1, n / (d * P)) of them (BFS: n / (64 d P), a pair replaces a
                                      bitmap bit), else the dense ncclAllReduce(min) / bitmap OR; one 4P-byte host
                                      read per iteration decides. 0 (default) = dense always. 8 keeps the
                                      all-gather under the all-reduce's bytes. Results are identical. */
    ASCETIC_OPT_RELAX_MODE = 20,     /* SSSP/CC min updates: 1 = atomicMin, and the thread whose atomic lowered the
                                      value sets the vertex's next-frontier bit; 2 = fire-and-forget RED.MIN, and
                                      the finalize derives A_{t+1} = {v : val < snap} in one dense pass (Jacobi:
                                      the same set); 0 = auto (default) = 2 (resident static-hit kernels 5-15 % faster). The sparse
                                      exchange forces 1. Results are identical. */
    ASCETIC_OPT_CE_MIN_RUN = 21,     /* bytes (default 1 MiB, 0 = off): in gather-mode iterations the miss runs of at
                                      least this many bytes are copied by the copy engines (one cudaMemcpyAsync per
                                      run piece, on a second copy stream) while the SM gather moves the rest */
    ASCETIC_OPT_GAP_BRIDGE = 22,     /* bytes (default 0 = off): the SM gather also loads (and discards) host holes of
                                      at most this size between consecutive pieces of a warp's group, so the warp
                                      reads one contiguous block instead of two. Measured: no gain at 64 B, -1 % at
                                      256 B, -2..3 % at 1 KiB on C2/C4 (the link is not charged per block) */
    ASCETIC_OPT_PR_SEGMENT = 23,     /* bytes (default 128 MiB, 0 = off): with ASCETIC_SORTED rows and contrib (4n bytes)
                                      above 1.5x this, the resident (static) PR pull runs in J = ceil(4n / this)
                                      passes over neighbour-id slices, capped at the static rows' mean degree / 8,
                                      so each pass's contrib gathers hit L2 */
    ASCETIC_OPT_SPAN_DENSITY = 24,   /* percent (default 85, 0 = off): in auto mode an iteration with >= 64 MiB of
                                      misses whose host span is <= SPAN_MAX_RATIO x the payload moves each window of cap host
                                      bytes with ONE copy-engine DMA when its payload is >= this share of those
                                      bytes (the holes ride along, ~55 GB/s for the whole window), and
                                      gathers the sparser windows; the on-demand kernels read a DMA'd window in
                                      place. Payload accounting is unchanged; span_link_bytes counts the holes. */
    ASCETIC_OPT_SPAN_MAX_RATIO = 25, /* percent (default 200): auto span planning only when the miss stream's host
                                      span is at most this share of its payload (windows then decided one by one) */
    ASCETIC_OPT_FUSED_VISIT = 26     /* BFS, SM-gathered chunks: the gather visits the ids it lands (On-demand
                                      Computing P:694 fused into the transfer; the chunk is still written).
                                      1 (default) = for small chunks (two buffers of < 4 MiB, where the
                                      gather -> on-demand chain is the latency), 2 = every gathered chunk, 0 = off */
} ascetic_option;

typedef struct {
    int32_t algo;
    uint32_t iterations;          /* executed expansions with non-empty A_t (PR: max_iters) */
    uint64_t n, m;                /* vertices, stored arcs */
    uint32_t b_e;                 /* payload bytes per arc: 4, or 8 with ASCETIC_PAIRS */
    uint32_t rank, world;
    uint64_t s;                   /* static vertices are [0, s) (front prefix) at the start of the run */
    uint64_t budget_bytes;        /* B: Static + On-demand edge regions */
    uint64_t static_reserved;     /* Ms = R*B floored to 16 KiB */
    uint64_t static_bytes;        /* b_e * off[s] actually resident */
    uint64_t ondemand_bytes;      /* C = B - Ms */
    uint64_t chunk_cap;           /* bytes per on-demand chunk buffer: floor(C / chunk_buffers / 16) * 16 (or the
                                     CHUNK_CAP option, if smaller) */
    double static_fraction_used;  /* R */
    uint64_t h2d_payload_bytes;   /* Σ_t miss bytes (the parity target) */
    uint64_t h2d_static_fill_bytes;
    uint64_t h2d_other_bytes;     /* metadata H2D: the long-run stream intervals of hybrid gather iterations */
    uint64_t d2h_bytes;           /* run lists + counters read back */
    uint64_t active_arcs_total;   /* Σ_t Σ_{v∈A_t} deg(v) */
    uint64_t chunks_total;
    uint64_t dma_chunks, gather_chunks;
    double time_run_s;            /* ascetic_run wall time incl. fill, all H2D, all exchange */
    double time_fill_s;
    double time_h2d_busy_s;       /* copy-stream busy time (sum of chunk transfers, fill and swaps; per-phase
                                     spans exist only in iterations TIMING selects) */
    double gteps;                 /* active_arcs_total / time_run_s / 1e9 */
    double gteps_excl_fill;
    uint64_t vertex_state_bytes;  /* device bytes outside the edge budget */
    /* per-kernel-class device time (CUDA events on the launching stream) and algorithmic work */
    uint64_t kernel_launches;     /* kernels this library launched during the run */
    double time_classify_s;       /* classify+compact kernel */
    double time_static_s;         /* static-hit edge kernels */
    uint64_t static_arcs;         /* arcs they processed */
    double time_ondemand_s;       /* on-demand chunk edge kernels */
    uint64_t ondemand_arcs;
    double time_gather_s;         /* gather-mode chunk transfers: the zero-copy SM gather (with the copy-engine
                                     long runs beside it); CUDA events on the copy stream(s) */
    uint64_t gather_bytes;        /* payload of those chunks */
    double time_dma_s;            /* copy-engine chunk DMAs (runs and span windows) */
    uint64_t dma_bytes;           /* payload of those chunks (span windows: without their holes) */
    double time_finalize_s;
    double time_host_s;           /* host planning + waits between classify and the next launches */
    uint64_t repartitions;        /* Eq. 3 re-partitions performed (ASCETIC_OPT_REPARTITION) */
    uint64_t h2d_replace_bytes;   /* §3.4 swapped-in chunk bytes (ASCETIC_OPT_REPLACE_CHUNKS) */
    uint64_t swaps_total;         /* §3.4 chunk swaps performed */
    double time_replace_s;        /* copy-stream time of the swap DMAs */
    uint64_t sparse_exchanges;    /* iterations whose exchange went sparse (ASCETIC_OPT_SPARSE_EXCHANGE) */
    uint64_t sparse_exchange_bytes; /* (id, value) pair bytes all ranks contributed to those exchanges */
    uint32_t chunk_buffers;       /* On-demand Region buffers in use (auto: 3, or 2 when C/3 < 4 MiB) */
    uint32_t reserved0;
    uint64_t gather_ce_bytes;     /* part of gather_bytes moved by the copy engines (long runs, CE_MIN_RUN) */
    uint64_t gather_load_bytes;   /* host bytes the SM gather loaded: 16-byte cover units incl. bridged holes
                                     (vs gather_bytes - gather_ce_bytes of payload: the over-fetch) */
    uint64_t pr_segment_passes;   /* PR: neighbour-id slices of the static pull (0 = unsegmented) */
    uint64_t span_chunks;         /* span-DMA windows (XFER_MODE 3 / auto): one DMA of a window's host bytes */
    uint64_t span_link_bytes;     /* host bytes those DMAs moved (payload + the holes between the missed lists) */
    uint64_t span_payload_bytes;  /* payload inside them (counted in dma_bytes / h2d_payload_bytes) */
} ascetic_stats_t;

typedef struct {
    uint32_t t;
    uint32_t rank;
    uint64_t nA, nH, nM, nruns;
    uint64_t active_arcs, hit_arcs, miss_bytes;
    uint64_t digest;              /* Σ_w splitmix64(w ^ word_w * 0x9E3779B97F4A7C15) over A_t's bitmap */
    uint32_t chunks;
    uint32_t mode;                /* 1 = zero-copy gather, 2 = DMA */
    /* device time of each kernel class in this iteration (CUDA events); ms_total = the
     * iteration's wall time from its classify launch to the next iteration's */
    float ms_classify, ms_static, ms_ondemand, ms_h2d, ms_finalize, ms_exchange, ms_total;
    /* host-link idle inside the iteration: before its first chunk transfer, between its
     * chunk transfers, and after its last one (until the next iteration's classify) */
    float ms_link_head, ms_link_gaps, ms_link_tail;
    uint64_t s_static;            /* static vertices of this rank in this iteration (|S ∩ rank|) */
    uint64_t swaps;               /* §3.4: chunks swapped in during this iteration (effective at t+1) */
    uint64_t replace_bytes;       /* bytes of those chunks (16 KiB each; the rank's last chunk may be short) */
} ascetic_iter_stats_t;

/*
 * Load a CSR graph ("The graph is presented in the CSR format").
 *   n       vertices (< 2^32 - 1)
 *   m       stored arcs (both directions for symmetric graphs)
 *   off     host uint64[n+1], off[0] = 0, non-decreasing (checked on the device), off[n] = m
 *   nbr     host uint32[m] neighbour ids, or uint32[2m] (id, weight) pairs with ASCETIC_PAIRS
 *   wgt     host uint32[m] weights or NULL; if given (without PAIRS) the library builds
 *           its own interleaved pinned copy
 *   flags   ASCETIC_* load flags
 * Ownership: without ASCETIC_COPY the nbr array is pinned IN PLACE (cudaHostRegister,
 * read-only) and the off array is used in place by the host planner; both must stay alive and
 * unmodified until ascetic_unload() or the next load_csr. Memory already page-locked
 * (cudaHostAlloc / torch pin_memory) is used as is (pinned off uploads at the link's rate).
 * With ASCETIC_COPY the library keeps private copies of both.
 * Errors: EINVAL (off[0] != 0, non-monotone off, off[n] != m, ids >= n or (with SORTED) a row out of
 * order with VALIDATE, wgt with PAIRS), EHOSTMEM (pinning), ENOMEM/ECUDA (device offsets).
 */
int ascetic_load_csr(uint64_t n, uint64_t m, const uint64_t* off, const uint32_t* nbr,
                     const uint32_t* wgt, uint32_t flags);

/*
 * Split the device edge budget (§3.3):
 *   bytes            B = Static Region + On-demand Region (vertex state is accounted outside)
 *   static_fraction  R in [0,1] fixes the split; < 0 selects Eq. 2 with K = 0.10,
 *                    clamped to [0,1]. NaN or > 1 => EINVAL.
 * Ms = floor(R*B / 16 KiB) * 16 KiB (<= D), s = max{v : b_e*off[v] <= Ms}, C = B - Ms.
 * C is split into N chunk buffers (ASCETIC_OPT_CHUNK_BUFFERS; auto: 3, or 2 when C/3 < 4 MiB) of
 * floor(C/N/16)*16 bytes each (ascetic_placement_t.cap is the 2-buffer figure). Allocates one
 * arena of Ms + N buffers (<= B) once. ENOMEM if s < n and a buffer is below 16 bytes, or
 * allocation fails.
 */
int ascetic_set_budget(uint64_t bytes, double static_fraction);

/* The placement set_budget would choose, computed on the host only (no device, no state):
 * same arguments as set_budget plus the CSR offsets and payload bytes per arc. */
typedef struct {
    double R;
    uint64_t D, B, Ms, s, static_bytes, C, cap;
} ascetic_placement_t;
int ascetic_place(uint64_t n, const uint64_t* off, uint32_t b_e, uint64_t bytes, double static_fraction,
                  ascetic_placement_t* out);

/* Tuning knob (see ascetic_option). Valid in LOADED or READY state. */
int ascetic_set_option(int option, int64_t value);

/*
 * Run one algorithm to completion (SURVEY §8(c) definitions, Jacobi/BSP semantics):
 *   algo       ascetic_algo. SSSP needs weights (PAIRS or wgt). CC/PR need ASCETIC_SYMMETRIC.
 *   source     BFS/SSSP source (< n), ignored for CC/PR
 *   max_iters  0 = until the active set is empty; PR runs exactly max_iters (must be >= 1)
 * ASCETIC_PRD (PageRank-delta, frontier-driven) is computed in 2^-56 fixed
 * point with integer atomics, d = 17/20: res_0 = floor(3*2^56/(20n)), A_t = {v : res[v] > tau};
 * each active u moves res[u] into r[u] and pushes floor(17 res[u] / (20 deg u)) along its
 * out-arcs; the result is fp32((r + res) 2^-56). Bit-exact against the oracle (P > 1: the
 * integer increments are SUM-exchanged); no ASCETIC_SYMMETRIC needed.
 * The static fill (one H2D of the front prefix) is part of the run unless KEEP_STATIC
 * kept it from a previous run. Results stay on the device until ascetic_get_result.
 */
int ascetic_run(int algo, uint32_t source, uint32_t max_iters);

/* Statistics of the last run. per_iter may be NULL; up to cap entries are written.
 * Returns the number of iteration records available (>= 0) or a negative status. */
int ascetic_stats(ascetic_stats_t* out, ascetic_iter_stats_t* per_iter, uint32_t cap);

/* Copy the last run's result to host_dst: n x uint32 (levels / distances / labels,
 * UINT32_MAX = unreached) or n x float (PageRank, PageRank-delta). bytes must be >= 4n. */
int ascetic_get_result(void* host_dst, uint64_t bytes);

/* Multi-GPU (one process per GPU; the paper itself is single-GPU).
 * Vertices are cut into `world` 1D edge-balanced ranges (ascetic_partition); each rank owns
 * the out-lists of its range, has its own placer / Static Region / On-demand Region / transfer
 * engine under its own budget B, and keeps the vertex state replicated. One exchange per
 * iteration: OR of next-frontier bitmaps (BFS), MIN of values (SSSP, CC), SUM of the fp64
 * dangling mass + every rank's contrib slice (PR), SUM of the u64 residual increments (PRD).
 * Results equal the single-GPU run.
 *   ascetic_get_unique_id  rank 0: 128-byte NCCL unique id (EUNSUPPORTED if libnccl.so.2
 *                          cannot be loaded); share it out of band (torch.distributed)
 *   ascetic_comm_init      every rank, BEFORE load_csr; device = this rank's GPU
 *                          world = 1 with a unique id builds a one-rank NCCL communicator
 *                          (the exchange path runs through NCCL; used to test it on one GPU);
 *                          world = 1 with uid128 = NULL drops any communicator
 *   ascetic_emulate_ranks  drive `world` ranks from THIS process on its one GPU (each rank a
 *                          full engine with its own device state; collectives by device copies).
 *                          Same per-rank code path and per-rank statistics; for testing the
 *                          partitioned path without a multi-GPU box. BEFORE load_csr.
 * Statistics of a P > 1 run: per_iter holds one record per (iteration, local rank),
 * iteration-major; sums in ascetic_stats_t are over the local ranks. */
int ascetic_get_unique_id(void* out128);
int ascetic_comm_init(int rank, int world, const void* uid128, int device);
int ascetic_emulate_ranks(int world);

/* Host-only: the 1D edge-balanced rank boundaries (bounds[0] = 0, bounds[parts] = n,
 * bounds[g] = min{v : off[v] >= ceil(g*m/parts)}). bounds holds parts+1 entries. */
int ascetic_partition(uint64_t n, const uint64_t* off, uint32_t parts, uint64_t* bounds);

/* Device to use (before load_csr); default = current device. */
int ascetic_set_device(int device);

/* Release every device buffer and unpin host memory; back to UNLOADED. */
void ascetic_unload(void);

/* Thread-local message of the last failing call ("" if none). */
const char* ascetic_last_error(void);

/* Test/diagnostic entry point: run ONE GenDataMap + compaction (the classify kernel) of rank
 * `rank` (0 unless emulating ranks) on the active set given as host bitmap words (bit v%32 of
 * word v/32, nwords = ceil(n/32)) against the current StaticBitmap (READY state), and copy its
 * outputs to the caller's host arrays (each `cap` entries; counts are returned even when an
 * array is too small, in which case it is left unwritten). run_dst / missq_pre are in ARCS
 * (multiply by b_e for bytes). Overwrites the engine's active set. */
typedef struct {
    uint32_t *hit_small, *hit_med, *hit_hub, *hub_pre;    /* hit queues by degree bucket, ascending ids */
    uint32_t *missq;                                      /* missed vertices with deg > 0, ascending */
    uint64_t *missq_pre, *missq_src;                      /* exclusive miss-arc prefix; off[v] */
    uint32_t *run_b, *run_e;                              /* maximal runs [b, e) of the missed set */
    uint64_t *run_dst;                                    /* exclusive miss-arc prefix at each run start */
    uint64_t cap;
    uint64_t n_small, n_med, n_hub, n_pieces, n_missq, n_runs, miss_arcs;
    uint64_t nA, nH, nM, active_arcs, hit_arcs, digest;
} ascetic_classify_out_t;
int ascetic_debug_classify(int rank, const uint32_t* active_words, uint64_t nwords, ascetic_classify_out_t* out);

/* sizeof(ascetic_stats_t), sizeof(ascetic_iter_stats_t), sizeof(ascetic_placement_t) into out[0..2]
 * (lets bindings verify their struct mirrors). */
int ascetic_struct_sizes(uint64_t* out3);

/* Library version string. */
const char* ascetic_version(void);

#ifdef __cplusplus
}
#endif
#endif /* ASCETIC_H */
