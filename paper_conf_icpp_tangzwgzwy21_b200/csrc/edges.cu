// edges.cu — per-algorithm edge kernels, the zero-copy gather, init and finalize.
//
// Paper: Static Computing on the StaticNodes' edges straight from the Static Region
// (Fig. 4 (3)), On-demand Computing on the edges that landed in the
// On-demand Region (Fig. 4 (5)), the On-demand Engine's gather of OndemandEdges
// (P:593-596), and the next active set "generated based on the connected
// edges". Algorithms: BFS, SSSP, CC (push, Jacobi snapshots, SURVEY §8(c)
// Q2/Q3) and pull PageRank (d = 0.85).
//
// B200 design (DESIGN.md §"Kernels"):
//  * static hits are degree-bucketed: < 32 arcs -> one warp expands 32 lists with an
//    in-warp edge-balanced scan; 32..hub -> warp per list with 128-bit ld.global.nc;
//    >= hub -> the list is cut into fixed pieces, one CTA per piece (multi-CTA hubs).
//  * chunk kernels are edge-balanced: each CTA owns 2048 consecutive arcs of the
//    miss stream and maps arcs to sources through a shared-memory tile of the miss
//    queue's 64-bit prefix (one global binary search per CTA).
//  * the gather is a zero-copy SM copy: host arcs are read through the mapped pinned
//    CSR with the same arc->source map, so the host never needs the request list.
#include <algorithm>
#include <cstdlib>
#include <type_traits>

#include "ascetic_internal.h"

// Batching factors of the static-hit kernels, per algorithm: 16-byte loads per lane per round
// (8-byte arcs: SSSP; 4-byte arcs: the others) and 32-arc rounds per warp for short lists.
// Measured on B200, resident RMAT-24 at 8 CTAs/SM (profiles/r01/static_batching_ab.md):
// BFS gains nothing from batching (most arcs stop at the visited word), SSSP is best at 2/2
// (-14 %), CC/PRD at 2/4 (-10 %). ASC_* override them for tuning builds.
namespace ascetic { namespace {
template <int ALGO> constexpr int kU8 = 2;
template <int ALGO> constexpr int kU4 = (ALGO == 0) ? 1 : 2;
template <int ALGO> constexpr int kSmallRounds = (ALGO == 0) ? 1 : (ALGO == 1 ? 2 : 4);
} }
#ifdef ASC_U8
#define ASC_U8_OF(A) ASC_U8
#else
#define ASC_U8_OF(A) kU8<A>
#endif
#ifdef ASC_U4
#define ASC_U4_OF(A) ASC_U4
#else
#define ASC_U4_OF(A) kU4<A>
#endif
#ifdef ASC_SMALL_ROUNDS
#define ASC_SMALL_OF(A) ASC_SMALL_ROUNDS
#else
#define ASC_SMALL_OF(A) kSmallRounds<A>
#endif

namespace ascetic {

unsigned long long g_launches = 0;

namespace {

constexpr unsigned FULL = 0xFFFFFFFFu;
enum { BFS = 0, SSSP = 1, CC = 2, PR = 3, PRD = 4 };

// per-source value pushed along each arc: snapshot dist/label (u32), or PRD's fixed-point push c[u] (u64)
template <int ALGO>
using SrcVal = typename std::conditional<ALGO == PRD, unsigned long long, uint32_t>::type;

template <int ALGO>
__device__ __forceinline__ SrcVal<ALGO> src_val(const DevState& d, uint32_t u) {
    if constexpr (ALGO == PRD) return __ldg(d.pr_c + u);
    else if constexpr (ALGO == SSSP || ALGO == CC) return __ldg(d.snap + u);
    else return 0u;
}
constexpr double kDamp = 0.85;

// PR fixed point (DESIGN R31): one round-to-nearest per fp64 partial, integer sums thereafter
__device__ __forceinline__ unsigned long long to_fx(double x) { return __double2ull_rn(x * kFxOne); }
__device__ __forceinline__ double from_fx(unsigned long long x) { return __ull2double_rn(x) * (1.0 / kFxOne); }

// ------------------------------------------------------------------ L2 policy loads
// Adjacency lists and chunks are read once: stream them with L2 evict_first so they do not
// push the randomly accessed vertex state (dist / labels / bitmaps / contrib, the part of
// the working set with reuse) out of the 126 MB L2; the state is loaded with evict_last.
__device__ __forceinline__ unsigned long long pol_stream() {
    unsigned long long p;
    asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ unsigned long long pol_keep() {
    unsigned long long p;
    asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint4 ld_stream(const uint4* p) {
    uint4 x;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
                 : "=r"(x.x), "=r"(x.y), "=r"(x.z), "=r"(x.w) : "l"(p), "l"(pol_stream()));
    return x;
}
__device__ __forceinline__ uint2 ld_stream(const uint2* p) {
    uint2 x;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.u32 {%0,%1}, [%2], %3;"
                 : "=r"(x.x), "=r"(x.y) : "l"(p), "l"(pol_stream()));
    return x;
}
__device__ __forceinline__ uint32_t ld_stream(const uint32_t* p) {
    uint32_t x;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(x) : "l"(p), "l"(pol_stream()));
    return x;
}
// state written by atomics during the kernel: coherent load, kept in L2
__device__ __forceinline__ uint32_t ld_state(const uint32_t* p) {
    uint32_t x;
    asm volatile("ld.global.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(x) : "l"(p), "l"(pol_keep()));
    return x;
}
// state that is read-only during the kernel (visited bitmap, contrib)
__device__ __forceinline__ uint32_t ld_state_ro(const uint32_t* p) {
    uint32_t x;
    asm volatile("ld.global.nc.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(x) : "l"(p), "l"(pol_keep()));
    return x;
}

// ------------------------------------------------------------------ per-arc ops
__device__ __forceinline__ void set_next(const DevState& d, uint32_t v) {
    const uint32_t wi = v >> 5, bit = 1u << (v & 31);
    if (!(ld_state(d.next + wi) & bit)) atomicOr(d.next + wi, bit);
}

__device__ __forceinline__ void bfs_visit(const DevState& d, uint32_t v) {
    const uint32_t wi = v >> 5, bit = 1u << (v & 31);
    if (ld_state_ro(d.visited + wi) & bit) return;      // visited changes only in finalize
    if (ld_state(d.next + wi) & bit) return;
    atomicOr(d.next + wi, bit);
}

// SSSP / CC relax. Two forms with the same A_{t+1} (Jacobi: the set of vertices whose value ends
// the iteration below its snapshot): d.red_min = 0 waits for atomicMin's old value and sets the
// next bit when it lowered it; d.red_min = 1 issues a fire-and-forget RED.MIN and the dense
// finalize derives A_{t+1} = {v : val < snap} (no dependent atomic chain per improving arc).
__device__ __forceinline__ void min_update(const DevState& d, uint32_t v, uint32_t cand) {
    if (d.red_min) {
        atomicMin(d.val + v, cand);                      // result unused: compiles to RED.E.MIN
    } else {
        const uint32_t old = atomicMin(d.val + v, cand);
        if (cand < old) set_next(d, v);
    }
}

__device__ __forceinline__ void relax(const DevState& d, uint32_t v, uint32_t cand) {
    if (cand >= ld_state(d.val + v)) return;            // values only decrease within an iteration
    min_update(d, v, cand);
}

__device__ __forceinline__ uint32_t sat_add(uint32_t a, uint32_t w) {
    const unsigned long long c = (unsigned long long)a + w;
    return c > (unsigned long long)(kInf - 1) ? kInf - 1 : (uint32_t)c;
}

// PageRank-delta push (DESIGN R28-R30): res[v] += c[u] in 2^-56 fixed point (integer atomics,
// order-independent); the one thread whose add crosses tau marks v for the next active set.
__device__ __forceinline__ void prd_push(const DevState& d, uint32_t v, unsigned long long c) {
    if (c == 0) return;
    if (d.pr_inc) { atomicAdd(d.pr_inc + v, c); return; }   // P > 1: summed across ranks, then finalize
    const unsigned long long old = atomicAdd(d.pr_res + v, c);
    if (old <= d.tau && old + c > d.tau) set_next(d, v);
}

// one arc, push algorithms. `arc` points at b_e bytes: id (+ weight).
template <int ALGO>
__device__ __forceinline__ void push_arc(const DevState& d, SrcVal<ALGO> sval, uint32_t id, uint32_t w) {
    if constexpr (ALGO == BFS) bfs_visit(d, id);
    else if constexpr (ALGO == SSSP) relax(d, id, sat_add(sval, w));
    else if constexpr (ALGO == PRD) prd_push(d, id, sval);
    else relax(d, id, sval);
}

// N arcs of one lane at once, in phases so the lane keeps N state loads (then N atomics) in
// flight instead of one dependent load->atomic chain per arc: the static-hit kernels are
// latency-bound on these random 4-byte accesses (vmask bit j = arc j valid).
template <int ALGO, int N>
__device__ __forceinline__ void push_batch(const DevState& d, const SrcVal<ALGO> (&sv)[N], const uint32_t (&id)[N],
                                           const uint32_t (&w)[N], uint32_t vmask) {
    if constexpr (ALGO == PRD) {
        unsigned long long old[N];
#pragma unroll
        for (int j = 0; j < N; ++j) {
            old[j] = ~0ull;
            if (((vmask >> j) & 1u) && sv[j]) {
                if (d.pr_inc) atomicAdd(d.pr_inc + id[j], sv[j]);
                else old[j] = atomicAdd(d.pr_res + id[j], sv[j]);
            }
        }
#pragma unroll
        for (int j = 0; j < N; ++j)
            if (old[j] <= d.tau && old[j] + sv[j] > d.tau) set_next(d, id[j]);
    } else if constexpr (ALGO == BFS) {
        // visited words first (most arcs stop there), then the next words of the survivors only
        uint32_t vis[N], nx[N];
#pragma unroll
        for (int j = 0; j < N; ++j) vis[j] = ((vmask >> j) & 1u) ? ld_state_ro(d.visited + (id[j] >> 5)) : FULL;
#pragma unroll
        for (int j = 0; j < N; ++j) {
            const uint32_t bit = 1u << (id[j] & 31);
            nx[j] = (vis[j] & bit) ? FULL : ld_state(d.next + (id[j] >> 5));
        }
#pragma unroll
        for (int j = 0; j < N; ++j) {
            const uint32_t bit = 1u << (id[j] & 31);
            if (!((vis[j] | nx[j]) & bit)) atomicOr(d.next + (id[j] >> 5), bit);
        }
    } else {   // SSSP, CC: relax with the snapshot value
        uint32_t cand[N], cur[N];
#pragma unroll
        for (int j = 0; j < N; ++j) {
            cand[j] = (ALGO == SSSP) ? sat_add(sv[j], w[j]) : (uint32_t)sv[j];
            cur[j] = ((vmask >> j) & 1u) ? ld_state(d.val + id[j]) : 0u;
        }
#pragma unroll
        for (int j = 0; j < N; ++j) {
            if (cand[j] < cur[j]) min_update(d, id[j], cand[j]);
        }
    }
}

__device__ __forceinline__ double pr_in(const DevState& d, uint32_t id) {
    return (double)__uint_as_float(ld_state_ro(reinterpret_cast<const uint32_t*>(d.contrib) + id));
}

__device__ __forceinline__ uint32_t ub_u32(const uint32_t* a, uint32_t n, uint32_t x) {
    uint32_t lo = 0, hi = n;
    while (lo < hi) {
        const uint32_t mid = (lo + hi) >> 1;
        if (__ldg(a + mid) <= x) lo = mid + 1; else hi = mid;
    }
    return lo;
}

// §3.4 replacement: the Static Region is a set of 16 KiB slots; unit i (U-byte units) of the
// rank's payload lives at slot_of[chunk] * (16 KiB / U) + i mod (16 KiB / U). Without
// replacement the region is the contiguous front prefix (identity). An aligned 16-byte load
// never straddles a chunk, so the 128-bit body loop stays vectorised.
template <bool REMAP, int U>
__device__ __forceinline__ unsigned long long sidx(const DevState& d, unsigned long long i) {
    if (!REMAP) return i;
    constexpr unsigned long long per = kChunkBytes / U;
    return (unsigned long long)__ldg(d.slot_of + i / per) * per + (i % per);
}

// contiguous list [a0, a1) of arcs at base (b_e = 4 for ids, 8 for pairs), processed by
// `nthr` threads with index `tid`, 128-bit loads on the aligned body.
template <int ALGO, bool REMAP = false>
__device__ __forceinline__ double expand_list(const DevState& d, const void* base, unsigned long long a0,
                                              unsigned long long a1, SrcVal<ALGO> sval, int tid, int nthr) {
    double acc = 0.0;
    if (ALGO == SSSP) {
        const uint2* arcs = reinterpret_cast<const uint2*>(base);
        const unsigned long long h = min(a1, (a0 + 1) & ~1ull);      // 2 arcs per 16 B
        for (unsigned long long e = a0 + tid; e < h; e += nthr) {
            const uint2 x = ld_stream(arcs + sidx<REMAP, 8>(d, e));
            push_arc<ALGO>(d, sval, x.x, x.y);
        }
        const unsigned long long qb = h >> 1, qe = a1 >> 1;
        const uint4* q = reinterpret_cast<const uint4*>(base);
        // U x 16 B per lane per round (2U arcs): loads, then the state loads, then the atomics
        constexpr int U = ASC_U8_OF(ALGO);
        for (unsigned long long k = qb + tid; k < qe; k += (unsigned long long)U * nthr) {
            uint4 x[U];
            uint32_t vm = 0;
#pragma unroll
            for (int j = 0; j < U; ++j) {
                const unsigned long long kk = k + (unsigned long long)j * nthr;
                x[j] = make_uint4(0u, 0u, 0u, 0u);
                if (kk < qe) { x[j] = ld_stream(q + sidx<REMAP, 16>(d, kk)); vm |= 3u << (2 * j); }
            }
            SrcVal<ALGO> sv[2 * U];
            uint32_t id[2 * U], w[2 * U];
#pragma unroll
            for (int j = 0; j < U; ++j) {
                sv[2 * j] = sv[2 * j + 1] = sval;
                id[2 * j] = x[j].x; w[2 * j] = x[j].y; id[2 * j + 1] = x[j].z; w[2 * j + 1] = x[j].w;
            }
            push_batch<ALGO, 2 * U>(d, sv, id, w, vm);
        }
        for (unsigned long long e = max(h, qe << 1) + tid; e < a1; e += nthr) {
            const uint2 x = ld_stream(arcs + sidx<REMAP, 8>(d, e));
            push_arc<ALGO>(d, sval, x.x, x.y);
        }
    } else {
        const uint32_t* arcs = reinterpret_cast<const uint32_t*>(base);
        const unsigned long long h = min(a1, (a0 + 3) & ~3ull);      // 4 arcs per 16 B
        for (unsigned long long e = a0 + tid; e < h; e += nthr) {
            const uint32_t id = ld_stream(arcs + sidx<REMAP, 4>(d, e));
            if (ALGO == PR) acc += pr_in(d, id); else push_arc<ALGO>(d, sval, id, 0);
        }
        const unsigned long long qb = h >> 2, qe = a1 >> 2;
        const uint4* q = reinterpret_cast<const uint4*>(base);
        // push algorithms: 2 x 16 B per lane per round (8 arcs) so 8 state loads are in flight;
        // PR keeps 1 x 16 B per round (its 4 contrib gathers are independent loads already)
        constexpr int U = (ALGO == PR) ? 1 : ASC_U4_OF(ALGO);
        for (unsigned long long k = qb + tid; k < qe; k += (unsigned long long)U * nthr) {
            if constexpr (ALGO == PR) {
                const uint4 x = ld_stream(q + sidx<REMAP, 16>(d, k));
                acc += pr_in(d, x.x) + pr_in(d, x.y) + pr_in(d, x.z) + pr_in(d, x.w);
            } else {
                uint4 x[U];
                uint32_t vm = 0;
#pragma unroll
                for (int j = 0; j < U; ++j) {
                    const unsigned long long kk = k + (unsigned long long)j * nthr;
                    x[j] = make_uint4(0u, 0u, 0u, 0u);
                    if (kk < qe) { x[j] = ld_stream(q + sidx<REMAP, 16>(d, kk)); vm |= 15u << (4 * j); }
                }
                SrcVal<ALGO> sv[4 * U];
                uint32_t id[4 * U], w[4 * U];
#pragma unroll
                for (int j = 0; j < U; ++j) {
                    id[4 * j] = x[j].x; id[4 * j + 1] = x[j].y; id[4 * j + 2] = x[j].z; id[4 * j + 3] = x[j].w;
                }
#pragma unroll
                for (int j = 0; j < 4 * U; ++j) { sv[j] = sval; w[j] = 0u; }
                push_batch<ALGO, 4 * U>(d, sv, id, w, vm);
            }
        }
        for (unsigned long long e = max(h, qe << 2) + tid; e < a1; e += nthr) {
            const uint32_t id = ld_stream(arcs + sidx<REMAP, 4>(d, e));
            if (ALGO == PR) acc += pr_in(d, id); else push_arc<ALGO>(d, sval, id, 0);
        }
    }
    return acc;
}

__device__ __forceinline__ double warp_sum_d(double x) {
#pragma unroll
    for (int o = 16; o; o >>= 1) x += __shfl_xor_sync(FULL, x, o);
    return x;
}

// ------------------------------------------------------------------ static: small lists
// All three static-hit kernels are grid-stride loops over a capped, persistent grid: the
// hit work of an iteration can be tens of thousands of CTAs, and a grid that size would fill
// every SM slot and starve the on-demand kernels that gate chunk-buffer reuse (measured on the
// friendster-shaped PR: a 22 ms static pull stalled the transfer pipeline 13 ms per iteration).
template <int ALGO, bool REMAP>
__global__ void __launch_bounds__(256) k_static_small(DevState d, const uint32_t* __restrict__ q, uint32_t nq,
                                                      const void* __restrict__ sbase) {
    __shared__ double s_acc[8][32];
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
    for (uint32_t base = ((blockIdx.x * blockDim.x + threadIdx.x) >> 5) * 32; base < nq; base += nwarps * 32) {
        const uint32_t idx = base + lane;
        const bool valid = idx < nq;
        uint32_t u = 0, deg = 0;
        SrcVal<ALGO> sval = 0;
        unsigned long long start = 0;
        if (valid) {
            u = __ldg(q + idx);
            start = __ldg(d.off + u);
            deg = (uint32_t)(__ldg(d.off + u + 1) - start);
            sval = src_val<ALGO>(d, u);
        }
        uint32_t incl = deg;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(FULL, incl, o);
            if (lane >= o) incl += y;
        }
        const uint32_t excl = incl - deg;
        const uint32_t total = __shfl_sync(FULL, incl, 31);
        if constexpr (ALGO != PR) {
            // ASC_SMALL_ROUNDS rounds of 32 arcs per warp at once: each lane maps, loads and pushes
            // one arc per round
            constexpr int B = ASC_SMALL_OF(ALGO);
            for (uint32_t k0 = 0; k0 < total; k0 += 32u * B) {
                SrcVal<ALGO> sv[B];
                uint32_t id[B], w[B], vm = 0;
#pragma unroll
                for (int b = 0; b < B; ++b) {
                    const uint32_t k = k0 + 32u * b + lane;
                    int i = 0;
#pragma unroll
                    for (int step = 16; step >= 1; step >>= 1) {
                        const uint32_t x = __shfl_sync(FULL, incl, i + step - 1);
                        if (x <= k) i += step;
                    }
                    const unsigned long long ust = __shfl_sync(FULL, start, i);
                    const uint32_t uex = __shfl_sync(FULL, excl, i);
                    sv[b] = __shfl_sync(FULL, sval, i);
                    id[b] = 0u; w[b] = 0u;
                    if (k < total) {
                        const unsigned long long e = ust + (k - uex) - d.static_arc0;
                        if (ALGO == SSSP) {
                            const uint2 x = ld_stream(reinterpret_cast<const uint2*>(sbase) + sidx<REMAP, 8>(d, e));
                            id[b] = x.x; w[b] = x.y;
                        } else {
                            id[b] = ld_stream(reinterpret_cast<const uint32_t*>(sbase) + sidx<REMAP, 4>(d, e));
                        }
                        vm |= 1u << b;
                    }
                }
                push_batch<ALGO, B>(d, sv, id, w, vm);
            }
            continue;
        }
        if (ALGO == PR) s_acc[wib][lane] = 0.0;
        __syncwarp();
        for (uint32_t k0 = 0; k0 < total; k0 += 32) {
            const uint32_t k = k0 + lane;
            int i = 0;
#pragma unroll
            for (int step = 16; step >= 1; step >>= 1) {
                const uint32_t x = __shfl_sync(FULL, incl, i + step - 1);
                if (x <= k) i += step;
            }
            const unsigned long long ust = __shfl_sync(FULL, start, i);
            const uint32_t uex = __shfl_sync(FULL, excl, i);
            const SrcVal<ALGO> usv = __shfl_sync(FULL, sval, i);
            const bool ok = k < total;
            const unsigned long long e = ust + (k - uex) - d.static_arc0;   // index into the Static Region
            if (ALGO == PR) {
                double x = ok ? pr_in(d, ld_stream(reinterpret_cast<const uint32_t*>(sbase) + sidx<REMAP, 4>(d, e))) : 0.0;
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const double y = __shfl_up_sync(FULL, x, o);
                    const int oi = __shfl_up_sync(FULL, i, o);
                    if (lane >= o && oi == i) x += y;
                }
                const int ni = __shfl_down_sync(FULL, i, 1);
                const bool nok = __shfl_down_sync(FULL, (int)ok, 1);
                const bool last = ok && (lane == 31 || !nok || ni != i);
                if (last) s_acc[wib][i] += x;
                __syncwarp();
            } else if (ok) {
                if (ALGO == SSSP) {
                    const uint2 x = ld_stream(reinterpret_cast<const uint2*>(sbase) + sidx<REMAP, 8>(d, e));
                    push_arc<ALGO>(d, usv, x.x, x.y);
                } else {
                    push_arc<ALGO>(d, usv, ld_stream(reinterpret_cast<const uint32_t*>(sbase) + sidx<REMAP, 4>(d, e)), 0);
                }
            }
        }
        if (ALGO == PR && valid) d.sum[u] = to_fx(s_acc[wib][lane]);
        __syncwarp();
    }
}

// ------------------------------------------------------------------ static: warp per list
template <int ALGO, bool REMAP>
__global__ void __launch_bounds__(256) k_static_med(DevState d, const uint32_t* __restrict__ q, uint32_t nq,
                                                    const void* __restrict__ sbase) {
    const int lane = threadIdx.x & 31;
    const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
    for (uint32_t w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; w < nq; w += nwarps) {
        const uint32_t u = __ldg(q + w);
        const unsigned long long a0 = __ldg(d.off + u), a1 = __ldg(d.off + u + 1);
        const SrcVal<ALGO> sval = src_val<ALGO>(d, u);
        double acc = expand_list<ALGO, REMAP>(d, sbase, a0 - d.static_arc0, a1 - d.static_arc0, sval, lane, 32);
        if (ALGO == PR) {
            acc = warp_sum_d(acc);
            if (lane == 0) d.sum[u] = to_fx(acc);
        }
    }
}

// ------------------------------------------------------------------ static: hubs, CTA per piece
template <int ALGO, bool REMAP>
__global__ void __launch_bounds__(256) k_static_hub(DevState d, const uint32_t* __restrict__ hq,
                                                    const uint32_t* __restrict__ pre, uint32_t nh, uint32_t npieces,
                                                    uint32_t piece_arcs, const void* __restrict__ sbase) {
    __shared__ double s_red[8];
    for (uint32_t b = blockIdx.x; b < npieces; b += gridDim.x) {
        const uint32_t h = ub_u32(pre, nh, b) - 1;
        const uint32_t u = __ldg(hq + h);
        const uint32_t pidx = b - __ldg(pre + h);
        const unsigned long long o0 = __ldg(d.off + u), o1 = __ldg(d.off + u + 1);
        const unsigned long long a0 = o0 + (unsigned long long)pidx * piece_arcs;
        const unsigned long long a1 = min(o1, a0 + piece_arcs);
        const SrcVal<ALGO> sval = src_val<ALGO>(d, u);
        double acc = expand_list<ALGO, REMAP>(d, sbase, a0 - d.static_arc0, a1 - d.static_arc0, sval, threadIdx.x,
                                              blockDim.x);
        if (ALGO == PR) {
            acc = warp_sum_d(acc);
            if ((threadIdx.x & 31) == 0) s_red[threadIdx.x >> 5] = acc;
            __syncthreads();
            if (threadIdx.x == 0) {
                double t = 0.0;
                for (int w = 0; w < (int)(blockDim.x >> 5); ++w) t += s_red[w];
                atomicAdd(d.sum + u, to_fx(t));
            }
            __syncthreads();
        }
    }
}

// ------------------------------------------------------------------ PR pull, column-segmented
// When contrib (4n bytes) is larger than L2, a pull row's 4-byte contrib gathers each fetch a 32-byte
// DRAM sector (friendster-shaped resident PR: ~7x sector amplification, DRAM-saturated at 111 G
// arcs/s). Segmented pull: J passes, pass j gathers only neighbours in [lo_id, hi_id), a slice of
// contrib that stays L2-resident, so its gathers hit. Rows are sorted by neighbour id, so each row's
// pass-j arcs are the next contiguous stretch of its list: a per-row cursor (indexed by hit-queue
// position; per piece for hubs) resumes where pass j-1 stopped — every arc is read once over all
// passes, plus one boundary probe per row and pass. Partial sums are added in 2^-62 fixed point
// (rows: owner-exclusive; hub pieces: integer atomics), so the order of passes and pieces does not
// change a bit of the result. Small rows (< 32 arcs) keep the unsegmented kernel.
// first index in [lo, hi) whose id is >= key (ids ascend), found by the warp with 32-ary probing
__device__ __forceinline__ unsigned long long warp_lower_bound(const uint32_t* __restrict__ ids, unsigned long long lo,
                                                               unsigned long long hi, uint32_t key, int lane) {
    while (hi - lo > 32) {
        const unsigned long long step = (hi - lo + 31) / 32;
        const unsigned long long i = lo + (unsigned long long)lane * step;
        const bool below = i < hi && __ldg(ids + i) < key;
        const uint32_t c = __popc(__ballot_sync(FULL, below));   // probes below key: a prefix of the lanes
        if (c == 0) return lo;
        const unsigned long long nlo = lo + (unsigned long long)(c - 1) * step + 1;
        hi = min(hi, lo + (unsigned long long)c * step);
        lo = nlo;
    }
    const unsigned long long i = lo + lane;
    const bool below = i < hi && __ldg(ids + i) < key;
    return lo + __popc(__ballot_sync(FULL, below));
}

// pass j of a medium row: [cursor, first arc with id >= hi_id), found by a warp search, then the
// same vectorised pull as the unsegmented kernel over that stretch
template <bool FIRST>
__global__ void __launch_bounds__(256) k_static_med_pr_seg(DevState d, const uint32_t* __restrict__ q, uint32_t nq,
                                                           const uint32_t* __restrict__ sbase, uint32_t* __restrict__ cur,
                                                           uint32_t hi_id) {
    const int lane = threadIdx.x & 31;
    const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
    for (uint32_t w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; w < nq; w += nwarps) {
        const uint32_t u = __ldg(q + w);
        const unsigned long long a0 = __ldg(d.off + u) - d.static_arc0, a1 = __ldg(d.off + u + 1) - d.static_arc0;
        const unsigned long long p = a0 + (FIRST ? 0u : cur[w]);
        const unsigned long long e = warp_lower_bound(sbase, p, a1, hi_id, lane);
        double acc = e > p ? expand_list<PR, false>(d, sbase, p, e, 0u, lane, 32) : 0.0;
        acc = warp_sum_d(acc);
        if (lane == 0) {
            cur[w] = (uint32_t)(e - a0);
            if (acc != 0.0) d.sum[u] += to_fx(acc);
        }
    }
}

// pass j of a hub piece: warp 0 finds the stretch, the CTA pulls it
template <bool FIRST>
__global__ void __launch_bounds__(256) k_static_hub_pr_seg(DevState d, const uint32_t* __restrict__ hq,
                                                           const uint32_t* __restrict__ pre, uint32_t nh,
                                                           uint32_t npieces, uint32_t piece_arcs,
                                                           const uint32_t* __restrict__ sbase, uint32_t* __restrict__ cur,
                                                           uint32_t hi_id) {
    __shared__ double s_red[8];
    __shared__ unsigned long long s_end;
    for (uint32_t b = blockIdx.x; b < npieces; b += gridDim.x) {
        const uint32_t h = ub_u32(pre, nh, b) - 1;
        const uint32_t u = __ldg(hq + h);
        const uint32_t pidx = b - __ldg(pre + h);
        const unsigned long long o0 = __ldg(d.off + u) - d.static_arc0, o1 = __ldg(d.off + u + 1) - d.static_arc0;
        const unsigned long long a0 = o0 + (unsigned long long)pidx * piece_arcs;
        const unsigned long long a1 = min(o1, a0 + piece_arcs);
        const unsigned long long p = a0 + (FIRST ? 0u : cur[b]);
        if (threadIdx.x < 32) {
            const unsigned long long e = warp_lower_bound(sbase, p, a1, hi_id, threadIdx.x);
            if (threadIdx.x == 0) s_end = e;
        }
        __syncthreads();
        const unsigned long long e = s_end;
        double acc = e > p ? expand_list<PR, false>(d, sbase, p, e, 0u, threadIdx.x, blockDim.x) : 0.0;
        acc = warp_sum_d(acc);
        if ((threadIdx.x & 31) == 0) s_red[threadIdx.x >> 5] = acc;
        __syncthreads();
        if (threadIdx.x == 0) {
            double t = 0.0;
            for (int w = 0; w < (int)(blockDim.x >> 5); ++w) t += s_red[w];
            cur[b] = (uint32_t)(e - a0);
            if (t != 0.0) atomicAdd(d.sum + u, to_fx(t));
        }
        __syncthreads();
    }
}

// ------------------------------------------------------------------ miss-stream tiles
// Tile t = miss-stream arcs [t*2048, (t+1)*2048), clipped to the chunk window [lo, hi).
// tile_first[t] (written by k_classify) is the miss-queue index of the vertex holding arc
// t*2048, so a CTA stages the covering queue entries [tile_first[t], tile_first[t+1]]
// (at most 2049) without any global search. Inside the tile each warp owns 256
// consecutive arcs and maps them to vertices 32 at a time with one shared-memory load,
// one __reduce_or_sync and one popcount per arc (warp-cooperative merge path).
struct Tile {
    unsigned long long t_lo, t_hi;
    uint32_t i0, cnt;
};

__device__ __forceinline__ Tile tile_of(const Queues& q, unsigned long long t, unsigned long long lo,
                                        unsigned long long hi) {
    Tile x;
    x.t_lo = max(lo, t << kEdgeTileShift);
    x.t_hi = min(hi, (t + 1) << kEdgeTileShift);
    x.i0 = __ldg(q.tile_first + t);
    const unsigned long long ntot = (q.miss_arcs + kEdgeTile - 1) >> kEdgeTileShift;
    const uint32_t i1 = (t + 1 < ntot) ? __ldg(q.tile_first + t + 1) : q.n_missq - 1u;
    x.cnt = i1 - x.i0 + 1u;
    return x;
}

// largest k in [lo, cnt) with s_pre[k] <= p (s_pre[lo] <= p guaranteed)
__device__ __forceinline__ uint32_t find_local(const unsigned long long* s_pre, uint32_t lo, uint32_t cnt,
                                               unsigned long long p) {
    uint32_t hi = cnt;
    while (hi - lo > 1) {
        const uint32_t mid = (lo + hi) >> 1;
        if (s_pre[mid] <= p) lo = mid; else hi = mid;
    }
    return lo;
}

// lanes take arcs p..p+31; k = local index of the vertex holding arc p. Returns this lane's vertex.
__device__ __forceinline__ uint32_t warp_map(const unsigned long long* s_pre, uint32_t cnt, uint32_t k,
                                             unsigned long long p, int lane) {
    const uint32_t idx = k + 1u + (uint32_t)lane;
    const unsigned long long b = idx < cnt ? s_pre[idx] : ~0ull;
    const unsigned long long r = b - p;            // >= 1 for every entry after k
    const uint32_t bit = r < 32ull ? (1u << (uint32_t)r) : 0u;
    const uint32_t mask = __reduce_or_sync(FULL, bit);
    return k + (uint32_t)__popc(mask & ((2u << lane) - 1u));
}

// ------------------------------------------------------------------ on-demand compute
// Tile metadata is read straight from the queues (L1-cached), no shared memory: the kernel can
// co-reside with any kernel whatever the SM's L1/shared split (a 33 KB/CTA staged variant could
// not start on SMs configured for the shared-memory-free static kernels).
// A chunk holds either the compacted miss stream [lo, hi) (arc a at a - lo), or, for a span DMA, the
// host arcs [span_base, ...) verbatim (arc a of queue vertex k at off[v_k] + (a - pre_k) - span_base).
template <int ALGO>
struct TileView {
    const unsigned long long* pre;
    const unsigned long long* src;
    const uint32_t* u;
    const DevState* d;
    unsigned long long lo, span_base;
    __device__ __forceinline__ uint32_t vtx(uint32_t k) const { return __ldg(u + k); }
    __device__ __forceinline__ SrcVal<ALGO> val(uint32_t k) const { return src_val<ALGO>(*d, __ldg(u + k)); }
    __device__ __forceinline__ unsigned long long at(uint32_t k, unsigned long long a) const {
        return span_base == ~0ull ? a - lo : __ldg(src + k) + (a - __ldg(pre + k)) - span_base;
    }
};

template <int ALGO>
__device__ __forceinline__ void ondemand_tile(const DevState& d, const Queues& q, const void* __restrict__ chunk,
                                              unsigned long long lo, unsigned long long hi, unsigned long long t,
                                              unsigned long long span_base) {
    const Tile x = tile_of(q, t, lo, hi);
    TileView<ALGO> tv;
    tv.pre = q.mq_pre + x.i0;
    tv.src = q.mq_src + x.i0;
    tv.u = q.mq + x.i0;
    tv.d = &d;
    tv.lo = lo;
    tv.span_base = span_base;
    const unsigned long long* s_pre = tv.pre;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const unsigned long long pw = x.t_lo + (unsigned long long)warp * 256ull;
    if (pw >= x.t_hi) return;
    const unsigned long long pe = min(x.t_hi, pw + 256ull);
    uint32_t k = find_local(s_pre, 0, x.cnt, pw);
    if constexpr (ALGO == PRD) {
        // 2 phases: map + chunk loads for the warp's 8 groups of 32 arcs, then the residual atomics
        uint32_t id[8];
        unsigned long long c[8];
#pragma unroll
        for (int g = 0; g < 8; ++g) {
            const unsigned long long p = pw + 32ull * g;
            const uint32_t mk = warp_map(s_pre, x.cnt, k, p, lane);
            k = __shfl_sync(FULL, mk, 31);
            const unsigned long long a = p + lane;
            id[g] = kInf;
            c[g] = tv.val(mk);
            if (a < pe) id[g] = ld_stream(reinterpret_cast<const uint32_t*>(chunk) + tv.at(mk, a));
        }
#pragma unroll
        for (int g = 0; g < 8; ++g)
            if (id[g] != kInf) prd_push(d, id[g], c[g]);
    } else if constexpr (ALGO == BFS) {
        // span chunks only (compacted BFS chunks use k_ondemand_bfs): map, load ids, then visit
        uint32_t id[8], w8[8];
        SrcVal<ALGO> sv[8];
        uint32_t vm = 0;
#pragma unroll
        for (int g = 0; g < 8; ++g) {
            const unsigned long long p = pw + 32ull * g;
            const uint32_t mk = warp_map(s_pre, x.cnt, k, p, lane);
            k = __shfl_sync(FULL, mk, 31);
            const unsigned long long a = p + lane;
            id[g] = 0u; w8[g] = 0u; sv[g] = 0u;
            if (a < pe) { id[g] = ld_stream(reinterpret_cast<const uint32_t*>(chunk) + tv.at(mk, a)); vm |= 1u << g; }
        }
        push_batch<BFS, 8>(d, sv, id, w8, vm);
    } else if constexpr (ALGO == SSSP || ALGO == CC) {
        // 3 phases over the warp's 8 groups of 32 arcs: map + chunk loads, state loads, atomics
        uint32_t id[8], cand[8], cur[8];
#pragma unroll
        for (int g = 0; g < 8; ++g) {
            const unsigned long long p = pw + 32ull * g;
            const uint32_t mk = warp_map(s_pre, x.cnt, k, p, lane);
            k = __shfl_sync(FULL, mk, 31);
            const unsigned long long a = p + lane;
            id[g] = kInf;
            if (a < pe) {
                if (ALGO == SSSP) {
                    const uint2 e = ld_stream(reinterpret_cast<const uint2*>(chunk) + tv.at(mk, a));
                    id[g] = e.x;
                    cand[g] = sat_add(tv.val(mk), e.y);
                } else {
                    id[g] = ld_stream(reinterpret_cast<const uint32_t*>(chunk) + tv.at(mk, a));
                    cand[g] = tv.val(mk);
                }
            }
        }
#pragma unroll
        for (int g = 0; g < 8; ++g) cur[g] = id[g] != kInf ? ld_state(d.val + id[g]) : 0u;
#pragma unroll
        for (int g = 0; g < 8; ++g) {
            if (id[g] != kInf && cand[g] < cur[g]) min_update(d, id[g], cand[g]);
        }
    } else {
        // PR pull: partial row sums of the chunk's arcs. Same 3 phases: map + chunk loads,
        // contrib gathers (8 in flight per lane), then one segmented warp reduction per group
        // (rows are contiguous runs of lanes) with one fp64 atomicAdd per row segment.
        uint32_t mk8[8], id8[8];
        double v8[8];
#pragma unroll
        for (int g = 0; g < 8; ++g) {
            const unsigned long long p = pw + 32ull * g;
            mk8[g] = warp_map(s_pre, x.cnt, k, p, lane);
            k = __shfl_sync(FULL, mk8[g], 31);
            const unsigned long long a = p + lane;
            id8[g] = a < pe ? ld_stream(reinterpret_cast<const uint32_t*>(chunk) + tv.at(mk8[g], a)) : kInf;
        }
#pragma unroll
        for (int g = 0; g < 8; ++g) v8[g] = id8[g] != kInf ? pr_in(d, id8[g]) : 0.0;
#pragma unroll
        for (int g = 0; g < 8; ++g) {
            const bool ok = id8[g] != kInf;
            double v = v8[g];
            const int key = ok ? (int)mk8[g] : -1 - lane;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const double y = __shfl_up_sync(FULL, v, o);
                const int ok2 = __shfl_up_sync(FULL, key, o);
                if (lane >= o && ok2 == key) v += y;
            }
            const int nk = __shfl_down_sync(FULL, key, 1);
            if (ok && (lane == 31 || nk != key)) atomicAdd(d.sum + tv.vtx(mk8[g]), to_fx(v));
        }
    }
}

// one CTA per 2048-arc tile of the chunk window
template <int ALGO>
__global__ void __launch_bounds__(256) k_ondemand_g(DevState d, Queues q, const void* __restrict__ chunk,
                                                    unsigned long long lo, unsigned long long hi,
                                                    unsigned long long span_base) {
    const unsigned long long t0 = lo >> kEdgeTileShift, t1 = (hi - 1) >> kEdgeTileShift;
    for (unsigned long long t = t0 + blockIdx.x; t <= t1; t += gridDim.x)
        ondemand_tile<ALGO>(d, q, chunk, lo, hi, t, span_base);
}

// BFS needs no source: 128-bit loads straight over the chunk.
__global__ void __launch_bounds__(256) k_ondemand_bfs(DevState d, const uint32_t* __restrict__ chunk,
                                                      unsigned long long len) {
    const unsigned long long nq4 = len >> 2;
    const uint4* c4 = reinterpret_cast<const uint4*>(chunk);
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    for (unsigned long long i = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; i < nq4; i += stride) {
        const uint4 x = ld_stream(c4 + i);
        bfs_visit(d, x.x); bfs_visit(d, x.y); bfs_visit(d, x.z); bfs_visit(d, x.w);
    }
    const unsigned long long t = (nq4 << 2) + (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (t < len) bfs_visit(d, ld_stream(chunk + t));
}

// ------------------------------------------------------------------ zero-copy gather (transfer engine)
// TMA bulk copy (cp.async.bulk, global -> shared, completion on an mbarrier) of the tile metadata
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(unsigned long long* b, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(smem_u32(b)), "r"(count) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(unsigned long long* b, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(smem_u32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, unsigned long long* b) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 :: "r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned long long* b, uint32_t phase) {
    uint32_t done = 0;
    while (!done)
        asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                     : "=r"(done) : "r"(smem_u32(b)), "r"(phase) : "memory");
}
// host (mapped pinned) 16-byte load, not allocated in L1: read once, and keeping it out of L1
// leaves the concurrent static-hit kernels their L1 hits on vertex state (C2 static 14.9 -> 12.1 ms,
// C4-shaped 13.8 -> 11.0 ms; the gather rate is unchanged)
__device__ __forceinline__ uint4 ld_host16(const uint4* p) {
    uint4 x;
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(x.x), "=r"(x.y), "=r"(x.z), "=r"(x.w) : "l"(p));
    return x;
}

// 16-byte cover gather (default). Measured on the box (tools/zc_align.cu, profiles/r01/zc_align.log):
// zero-copy reads of random host runs reach ~44 GB/s with 4-byte loads, ~48 with 8-byte and
// ~50 with 16-byte loads, even when the runs start 4-byte aligned and the 16-byte cover is read
// (the extra bytes sit in sectors that are fetched anyway). So lanes here load 16-byte-aligned
// units of host memory: per warp segment of 256 stream arcs, the missed vertices are grouped
// into pieces (maximal runs whose lists are adjacent on the host: one stream->host offset per
// piece), each piece's cover units are enumerated across the warp (a unit shared by two
// vertices of one piece is loaded once), and every lane stores the piece words its unit holds
// at their stream position. `hoff` = the host array's byte offset from its 16-byte-aligned base.
// Gap bridging (option, off by default): a piece whose next piece starts at most `gap_words` later
// also loads the hole units between them (not stored), so the warp instruction reads one contiguous
// block instead of two. Random SM reads run at ~90 M regions/s up to 512 B each (tools/zc_gran.cu)
// and 89-96 % of the gaps between C4's miss runs are < 16 B (profiles/r02/run_profile_c4.log), but
// bridging did not raise the rate (profiles/r02/gather_ab_c4.log): regions adjacent inside one
// instruction are not what the link charges for.
// Long runs: stream intervals lint[2i, 2i+1) (sorted, disjoint; whole vertices) go through the copy
// engines instead (Part::transfer_chunk); their vertices are skipped here.
// VISIT (BFS, 4-byte arcs): On-demand Computing fused into the landing of the chunk -- each word
// the gather stores is a neighbour id, visited right there (visited-word loads of the lane's words
// batched, then a fire-and-forget OR into next for the unvisited ones), so the chunk needs no
// separate on-demand kernel. The chunk is still written (the On-demand Region holds the data as
// before); what goes is one kernel launch per chunk and the chunk re-read. Used for small chunks,
// where the gather -> on-demand launch chain is the latency of the iteration (C1).
template <int BE, int NG, bool VISIT>
__global__ void __launch_bounds__(256) k_gather16(Queues q, const uint4* __restrict__ host, uint32_t hoff,
                                                  unsigned long long w_end, uint32_t* __restrict__ chunk,
                                                  unsigned long long lo, unsigned long long hi,
                                                  const unsigned long long* __restrict__ lint, uint32_t nlint,
                                                  uint32_t gap_words, unsigned long long* __restrict__ cover,
                                                  DevState d) {
    static_assert(!VISIT || BE == 4, "fused visit: BFS arcs are bare 4-byte ids");
    // tile metadata (the miss-queue prefix and host offsets of the tile's vertices) staged in shared
    // memory by TMA: one elected thread bulk-copies both contiguous slices (16-byte aligned, so from
    // the even index at or below i0; the queues carry 2 elements of padding) and every thread waits
    // on the mbarrier. (Reading the metadata through L1 instead gathers at the same rate, but its L1
    // traffic slows the concurrent static-hit kernels.)
    __shared__ alignas(16) unsigned long long s_pre_raw[kEdgeTile + 4];
    __shared__ alignas(16) unsigned long long s_src_raw[kEdgeTile + 4];
    __shared__ alignas(8) unsigned long long s_bar;
    constexpr unsigned long long AW = BE / 4;                 // words per arc
    const unsigned long long w_off = hoff / 4;                // host word index of arc 0
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const unsigned long long t0 = lo >> kEdgeTileShift, t1 = (hi - 1) >> kEdgeTileShift;
    if (threadIdx.x == 0) mbar_init(&s_bar, 1);
    __syncthreads();
    uint32_t phase = 0;
    for (unsigned long long t = t0 + blockIdx.x; t <= t1; t += gridDim.x) {
        const Tile x = tile_of(q, t, lo, hi);
        const uint32_t sh = x.i0 & 1u;
        __syncthreads();                                      // the previous tile's readers are done
        if (threadIdx.x == 0) {
            const uint32_t bytes = ((x.cnt + sh + 1u) & ~1u) * 8u;
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // generic reads before async writes
            mbar_expect_tx(&s_bar, 2u * bytes);
            bulk_g2s(s_pre_raw, q.mq_pre + (x.i0 - sh), bytes, &s_bar);
            bulk_g2s(s_src_raw, q.mq_src + (x.i0 - sh), bytes, &s_bar);
        }
        mbar_wait(&s_bar, phase);
        phase ^= 1u;
        const unsigned long long* s_pre = s_pre_raw + sh;
        const unsigned long long* s_src = s_src_raw + sh;
        const unsigned long long pw = x.t_lo + (unsigned long long)warp * 256ull;
        if (pw >= x.t_hi) continue;
        const unsigned long long pe = min(x.t_hi, pw + 256ull);
        const uint32_t kfirst = find_local(s_pre, 0, x.cnt, pw);
        const uint32_t klast = find_local(s_pre, kfirst, x.cnt, pe - 1);
        // long intervals that can touch this segment: the last one starting at or before pw, and the next
        uint32_t li = 0;
        if (nlint) {
            uint32_t L = 0, R = nlint;                               // first interval starting after pw
            while (L < R) { const uint32_t mid = (L + R) >> 1; if (__ldg(lint + 2 * mid) <= pw) L = mid + 1; else R = mid; }
            li = L ? L - 1 : 0;
        }
        for (uint32_t kb = kfirst; kb <= klast; kb += 32) {
            // lane <-> vertex j of the segment: stream arcs [a0, a1), host arcs [h0, h1)
            const uint32_t j = kb + (uint32_t)lane;
            bool v = j <= klast;
            unsigned long long a0 = 0, a1 = 0, h0 = 0;
            if (v) {
                const unsigned long long pj = s_pre[j];
                const unsigned long long ej = (j + 1 < x.cnt) ? s_pre[j + 1] : ~0ull;
                a0 = max(pw, pj);
                a1 = max(a0, min(pe, ej));
                h0 = s_src[j] + (a0 - pj);
                // a vertex inside a long run (runs are whole vertices) is the copy engines' job
                for (uint32_t k = li; k < li + 2 && k < nlint; ++k)
                    if (a0 >= __ldg(lint + 2 * k) && a0 < __ldg(lint + 2 * k + 1)) v = false;
                if (!v) a0 = a1 = h0 = 0;
            }
            const unsigned long long h1 = h0 + (a1 - a0);
            const unsigned long long ph1 = __shfl_up_sync(FULL, h1, 1);
            const bool pv = __shfl_up_sync(FULL, v, 1);
            const bool start = v && (lane == 0 || !pv || h0 != ph1);
            const uint32_t smask = __ballot_sync(FULL, start);
            const uint32_t vmask = __ballot_sync(FULL, v);
            const uint32_t brk = __ballot_sync(FULL, start || !v);          // piece boundaries and holes
            const int ps = 31 - __clz(smask & ((2u << lane) - 1u));          // this lane's piece start
            const uint32_t after = lane == 31 ? 0u : (brk & ~((2u << lane) - 1u));
            const int pl = after ? (__ffs(after) - 2) : (31 - __clz(vmask)); // and its last lane
            const unsigned long long W0 = w_off + __shfl_sync(FULL, h0, ps & 31) * AW;   // piece host words [W0, W1)
            const unsigned long long W1 = w_off + __shfl_sync(FULL, h1, pl & 31) * AW;
            const unsigned long long D0 = (__shfl_sync(FULL, a0, ps & 31) - lo) * AW;    // chunk word of W0
            const unsigned long long hw0 = w_off + h0 * AW, hw1 = w_off + h1 * AW;
            // cover units of this lane's words not already covered by the previous lane of the piece
            const unsigned long long u0 = start ? (hw0 >> 2) : ((hw0 + 3) >> 2);
            unsigned long long u1 = (hw1 + 3) >> 2;
            // bridge to the next piece of this group when the hole is at most gap_words: its units are
            // loaded by this (the piece's last) lane and fall outside [W0, W1), so nothing is stored
            const unsigned long long nh0 = __shfl_down_sync(FULL, hw0, 1);
            const bool nstart = __shfl_down_sync(FULL, start, 1);
            if (v && lane == pl && lane < 31 && nstart && nh0 > hw1 && nh0 - hw1 <= gap_words)
                u1 = max(u1, nh0 >> 2);
            const uint32_t cnt = (v && hw1 > hw0 && u1 > u0) ? (uint32_t)(u1 - u0) : 0u;
            uint32_t incl = cnt;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t y = __shfl_up_sync(FULL, incl, o);
                if (lane >= o) incl += y;
            }
            const uint32_t units = __shfl_sync(FULL, incl, 31);
            if (lane == 0 && units) atomicAdd(cover, (unsigned long long)units);   // 16-byte units read
            // a piece of >= 32 units (512 B) starts at an enumeration slot congruent to its first host
            // unit mod 32, so each of its warp loads covers exactly one 512-byte host block: random
            // runs read at 51 GB/s that way vs 49 with 2 KB warp segments at arbitrary offsets
            // (tools/zc_seg.cu, profiles/r02/zc_seg.log). Up to 31 idle slots per long piece; short
            // pieces stay packed. Pads of the warp's long pieces are resolved in lane order.
            {
                const bool lstart = start && cnt && ((W1 + 3) >> 2) - (W0 >> 2) >= 32ull;
                uint32_t m = __ballot_sync(FULL, lstart), S = 0, shift = 0;
                while (m) {
                    const int l = __ffs(m) - 1;
                    m &= m - 1u;
                    const uint32_t e_l = __shfl_sync(FULL, incl - cnt, l) + S;
                    // (units count from the 16-byte-aligned array base: add its phase in the 512 B block)
                    const uint32_t blk = (uint32_t)(reinterpret_cast<uintptr_t>(host) >> 4);
                    const uint32_t pad = ((uint32_t)__shfl_sync(FULL, (uint32_t)u0, l) + blk - e_l) & 31u;
                    S += pad;
                    if (lane >= l) shift += pad;
                }
                incl += shift;
            }
            const uint32_t excl = incl - cnt;
            const uint32_t total = __shfl_sync(FULL, incl, 31);   // enumeration slots incl. the pads
            for (uint32_t b = 0; b < total; b += 32u * NG) {
                // NG groups of 32 units: all loads first (NG x 16 B in flight per lane), then the stores
                uint4 val[NG];
                unsigned long long uw[NG], pw0[NG], pw1[NG], pd0[NG];
#pragma unroll
                for (int g = 0; g < NG; ++g) {
                    const uint32_t tt = b + 32u * g + (uint32_t)lane;
                    int i = 0;
#pragma unroll
                    for (int step = 16; step >= 1; step >>= 1) {
                        const uint32_t y = __shfl_sync(FULL, incl, i + step - 1);
                        if (y <= tt) i += step;
                    }
                    const unsigned long long uo = __shfl_sync(FULL, u0, i);
                    const uint32_t eo = __shfl_sync(FULL, excl, i);
                    pw0[g] = __shfl_sync(FULL, W0, i);
                    pw1[g] = __shfl_sync(FULL, W1, i);
                    pd0[g] = __shfl_sync(FULL, D0, i);
                    uw[g] = ~0ull;
                    if (tt < total && tt >= eo) {                 // (below eo: a pad slot, idle)
                        uw[g] = uo + (tt - eo);
                        // the array's first / last unit may stick out of [w_off, w_end): read those
                        // word by word in the store phase, never outside the caller's array
                        if (uw[g] * 4 >= w_off && uw[g] * 4 + 4 <= w_end) val[g] = ld_host16(host + uw[g]);
                    }
                }
#pragma unroll
                for (int g = 0; g < NG; ++g) {
                    if (uw[g] == ~0ull) continue;
                    if (!(uw[g] * 4 >= w_off && uw[g] * 4 + 4 <= w_end)) {
                        const uint32_t* hw = reinterpret_cast<const uint32_t*>(host) + uw[g] * 4;
                        uint32_t x4[4];
#pragma unroll
                        for (int c = 0; c < 4; ++c) {
                            const unsigned long long w = uw[g] * 4 + c;
                            x4[c] = (w >= w_off && w < w_end) ? hw[c] : 0u;
                        }
                        val[g] = make_uint4(x4[0], x4[1], x4[2], x4[3]);
                    }
                    const uint32_t wv[4] = {val[g].x, val[g].y, val[g].z, val[g].w};
#pragma unroll
                    for (int c = 0; c < 4; ++c) {
                        const unsigned long long w = uw[g] * 4 + c;
                        if (w >= pw0[g] && w < pw1[g]) chunk[pd0[g] + (w - pw0[g])] = wv[c];
                    }
                }
                if constexpr (VISIT) {
                    // the lane's NG x 4 landed ids: all visited-word loads first, then the ORs
                    uint32_t vw[NG][4];
#pragma unroll
                    for (int g = 0; g < NG; ++g) {
#pragma unroll
                        for (int c = 0; c < 4; ++c) {
                            const unsigned long long w = uw[g] * 4 + c;
                            const uint32_t id = c == 0 ? val[g].x : c == 1 ? val[g].y : c == 2 ? val[g].z : val[g].w;
                            vw[g][c] = (uw[g] != ~0ull && w >= pw0[g] && w < pw1[g]) ? ld_state_ro(d.visited + (id >> 5)) : ~0u;
                        }
                    }
#pragma unroll
                    for (int g = 0; g < NG; ++g) {
#pragma unroll
                        for (int c = 0; c < 4; ++c) {
                            const uint32_t id = c == 0 ? val[g].x : c == 1 ? val[g].y : c == 2 ? val[g].z : val[g].w;
                            const uint32_t bit = 1u << (id & 31);
                            if (!(vw[g][c] & bit)) atomicOr(d.next + (id >> 5), bit);   // result unused: RED.OR
                        }
                    }
                }
            }
        }
    }
}

// Long miss runs for the copy engines: runs are maximal id ranges of M_t, so a run's host bytes are
// one contiguous range b_e [off[b], off[e]); those >= min_arcs arcs are appended (unordered) with
// their stream offset into mapped host memory for the host to sort and issue as DMAs.
__global__ void __launch_bounds__(256) k_long_runs(const uint32_t* __restrict__ run_b, const uint32_t* __restrict__ run_e,
                                                   const unsigned long long* __restrict__ run_dst, uint32_t n_runs,
                                                   const unsigned long long* __restrict__ off, unsigned long long min_arcs,
                                                   unsigned long long* out, uint32_t cap, uint32_t* count,
                                                   uint32_t* done, uint32_t* flag) {
    for (uint32_t r = blockIdx.x * blockDim.x + threadIdx.x; r < n_runs; r += gridDim.x * blockDim.x) {
        const uint32_t b = run_b[r], e = run_e[r];
        if (__ldg(off + e) - __ldg(off + b) >= min_arcs) {
            const uint32_t i = atomicAdd(count, 1u);
            if (i < cap) { out[3 * i] = b; out[3 * i + 1] = e; out[3 * i + 2] = run_dst[r]; }
        }
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence_system();                                    // this CTA's host writes first
        if (atomicAdd(done, 1u) == gridDim.x - 1) {
            __threadfence();
            flag[1] = *reinterpret_cast<volatile uint32_t*>(count);
            __threadfence_system();
            *reinterpret_cast<volatile uint32_t*>(flag) = 1u;
        }
    }
}

// Span windows (span-DMA iterations): window k is the host arc range [h0 + k win, h0 + (k+1) win) ∩
// [h0, h1); out[k] = the miss-stream position of its first missed arc (lists are host-ordered like
// the stream, so it is the first queue vertex whose list ends after the boundary, entered at the
// boundary). One CTA; the host spins on flag (mapped memory).
__global__ void __launch_bounds__(1024) k_span_windows(Queues q, unsigned long long h0, unsigned long long h1,
                                                       unsigned long long win, uint32_t nwin,
                                                       unsigned long long* out, uint32_t* flag) {
    const uint32_t nq = q.n_missq;
    for (uint32_t k = threadIdx.x; k <= nwin; k += blockDim.x) {
        const unsigned long long H = k == nwin ? h1 : min(h1, h0 + (unsigned long long)k * win);
        uint32_t L = 0, R = nq;                            // first j with end_j > H
        while (L < R) {
            const uint32_t mid = (L + R) >> 1;
            const unsigned long long pre = __ldg(q.mq_pre + mid);
            const unsigned long long end = __ldg(q.mq_src + mid) +
                                           ((mid + 1 < nq ? __ldg(q.mq_pre + mid + 1) : q.miss_arcs) - pre);
            if (end > H) R = mid; else L = mid + 1;
        }
        unsigned long long pos = q.miss_arcs;
        if (L < nq) {
            const unsigned long long s = __ldg(q.mq_src + L);
            pos = __ldg(q.mq_pre + L) + (H > s ? H - s : 0ull);
        }
        out[k] = pos;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence_system();
        *reinterpret_cast<volatile uint32_t*>(flag) = 1u;
    }
}

// ------------------------------------------------------------------ init / finalize
__global__ void k_fill_u32(uint32_t* p, uint64_t n, uint32_t v) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
        p[i] = v;
}

__global__ void k_iota_u32(uint32_t* a, uint32_t* b, uint64_t n) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
        a[i] = (uint32_t)i;
        b[i] = (uint32_t)i;
    }
}

// bits = exactly the vertex range [a, b)
__global__ void k_range_bits(uint32_t* bits, uint32_t nwords, uint64_t a, uint64_t b) {
    for (uint64_t w = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; w < nwords; w += (uint64_t)gridDim.x * blockDim.x) {
        const uint64_t base = w * 32;
        const uint64_t lo = a > base ? a : base, hi = b < base + 32 ? b : base + 32;
        uint32_t x = 0u;
        if (lo < hi) {
            const uint32_t top = (uint32_t)(hi - base), bot = (uint32_t)(lo - base);
            x = (top == 32 ? FULL : ((1u << top) - 1u)) & ~((1u << bot) - 1u);
        }
        bits[w] = x;
    }
}

__global__ void k_set_source(DevState d, uint32_t src, int algo) {
    d.val[src] = 0;
    if (algo == SSSP) d.snap[src] = 0;
    d.A[src >> 5] |= 1u << (src & 31);
    if (algo == BFS) d.visited[src >> 5] |= 1u << (src & 31);
}

__global__ void k_pr_init(DevState d) {
    const double r0 = 1.0 / (double)d.n;
    double dang = 0.0;
    for (uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v < d.n; v += (uint64_t)gridDim.x * blockDim.x) {
        const unsigned long long deg = d.off[v + 1] - d.off[v];
        d.rank[v] = (float)r0;
        d.contrib[v] = deg ? (float)(r0 / (double)deg) : 0.0f;
        if (!deg) dang += r0;
    }
    dang = warp_sum_d(dang);
    if ((threadIdx.x & 31) == 0 && dang != 0.0) atomicAdd(d.dang, to_fx(dang));
}

// PRD (DESIGN R28-R30): r = 0, res = res0; A_0 = {v : res0 > tau} absorbs at once
__global__ void k_prd_init(DevState d, unsigned long long res0) {
    const bool act = res0 > d.tau;
    for (uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v < d.n; v += (uint64_t)gridDim.x * blockDim.x) {
        const unsigned long long deg = d.off[v + 1] - d.off[v];
        d.pr_r[v] = act ? res0 : 0ull;
        d.pr_res[v] = act ? 0ull : res0;
        d.pr_c[v] = act && deg ? (17ull * res0) / (20ull * deg) : 0ull;
    }
    if (act)
        for (uint64_t w = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; w < d.nwords; w += (uint64_t)gridDim.x * blockDim.x) {
            const uint64_t base = w * 32;
            const uint32_t cnt = (uint32_t)min((uint64_t)32, d.n - base);
            d.A[w] = cnt == 32 ? FULL : ((1u << cnt) - 1u);
        }
}

// PRD finalize: A_{t+1} = the vertices whose residual crossed tau this iteration; each absorbs
// r += res, c = floor(17 res / (20 deg)), res = 0 (the push value of iteration t+1)
__global__ void k_finalize_prd(DevState d) {
    for (uint32_t w = blockIdx.x * blockDim.x + threadIdx.x; w < d.nwords; w += gridDim.x * blockDim.x) {
        const uint32_t nx = d.next[w];
        d.A[w] = nx;
        if (nx) {
            d.next[w] = 0;
            uint32_t b = nx;
            while (b) {
                const int i = __ffs(b) - 1;
                b &= b - 1;
                const uint64_t v = (uint64_t)w * 32 + i;
                const unsigned long long x = d.pr_res[v], deg = d.off[v + 1] - d.off[v];
                d.pr_r[v] += x;
                d.pr_c[v] = deg ? (17ull * x) / (20ull * deg) : 0ull;
                d.pr_res[v] = 0ull;
            }
        }
    }
}

// Dense finalize kernels (after an exchange, or reading peers): one thread per vertex, one warp per
// 32-vertex bitmap word built with a ballot, so every warp load instruction reads 128 contiguous bytes
// of each value array (one line, also when the array is a peer's over NVLink) and lane 0 writes the word.
#define FOR_EACH_WORD_WARP(d, w, v, lane)                                                                     \
    const int lane = threadIdx.x & 31;                                                                        \
    for (uint64_t w = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; w < (d).nwords;                \
         w += ((uint64_t)gridDim.x * blockDim.x) >> 5)                                                       \
        if (const uint64_t v = w * 32 + (uint64_t)lane; true)

// PRD finalize after the cross-rank SUM of the increments (P > 1): res += inc over all vertices,
// A_{t+1} = {v : res > tau}, the active absorb; identical on every rank (replicated state)
__global__ void __launch_bounds__(256) k_finalize_prd_dense(DevState d) {
    FOR_EACH_WORD_WARP(d, w, v, lane) {
        bool act = false;
        if (v < d.n) {
            const unsigned long long inc = d.pr_inc[v];
            if (inc) {                                   // inc = 0: res <= tau already (not active, unchanged)
                d.pr_inc[v] = 0ull;
                const unsigned long long x = d.pr_res[v] + inc;
                if (x > d.tau) {
                    const unsigned long long deg = d.off[v + 1] - d.off[v];
                    act = true;
                    d.pr_r[v] += x;
                    d.pr_c[v] = deg ? (17ull * x) / (20ull * deg) : 0ull;
                    d.pr_res[v] = 0ull;
                } else {
                    d.pr_res[v] = x;
                }
            }
        }
        const uint32_t bits = __ballot_sync(FULL, act);
        if (lane == 0) { d.A[w] = bits; d.next[w] = 0; }
    }
}

// ---- fused exchange + finalize (P > 1): each rank reads every rank's buffer straight from peer
// memory (NVLink peers mapped with CUDA IPC; the other parts' buffers when ranks are emulated on
// one GPU) and builds A_{t+1} in the same pass — no gathered copy, no separate reduce kernel.
// Loads bypass L1 (ld.global.cg): the peers wrote these buffers before the stream barrier.
template <typename T>
__device__ __forceinline__ T ld_peer(const T* p) { return __ldcg(p); }

// BFS: A = (OR_p next_p) & ~visited; every rank applies the same update to its replicated state
__global__ void k_finalize_bfs_peers(DevState d, const uint32_t* const* __restrict__ peers, int P) {
    for (uint32_t w = blockIdx.x * blockDim.x + threadIdx.x; w < d.nwords; w += gridDim.x * blockDim.x) {
        uint32_t nx = 0;
        for (int p = 0; p < P; ++p) nx |= ld_peer(peers[p] + w);
        const uint32_t vis = d.visited[w];
        const uint32_t nw = nx & ~vis;
        d.A[w] = nw;
        if (nw) {
            d.visited[w] = vis | nw;
            uint32_t b = nw;
            while (b) {
                const int i = __ffs(b) - 1;
                b &= b - 1;
                d.val[(uint64_t)w * 32 + i] = d.iter + 1;
            }
        }
    }
}

// SSSP / CC: val = MIN_p val_p, A = {v : val < snap}, snap = val (a peer may be writing its own
// val with the same minimum concurrently: every value read is >= the minimum, so MIN is exact)
__global__ void __launch_bounds__(256) k_finalize_min_peers(DevState d, const uint32_t* const* __restrict__ peers, int P) {
    FOR_EACH_WORD_WARP(d, w, v, lane) {
        bool act = false;
        if (v < d.n) {
            uint32_t x = kInf;
            for (int p = 0; p < P; ++p) x = min(x, ld_peer(peers[p] + v));
            const uint32_t y = d.snap[v];
            if (x < y) { act = true; d.snap[v] = x; }
            if (x != d.val[v]) d.val[v] = x;
        }
        const uint32_t bits = __ballot_sync(FULL, act);
        if (lane == 0) { d.A[w] = bits; d.next[w] = 0; }
    }
}

// PRD: res += SUM_p inc_p (integers: exact in any order), A = {res > tau}, absorb
__global__ void __launch_bounds__(256) k_finalize_prd_peers(DevState d, const unsigned long long* const* __restrict__ peers,
                                                            int P) {
    FOR_EACH_WORD_WARP(d, w, v, lane) {
        bool act = false;
        if (v < d.n) {
            unsigned long long inc = 0;
            for (int p = 0; p < P; ++p) inc += ld_peer(peers[p] + v);
            if (inc) {
                const unsigned long long x = d.pr_res[v] + inc;
                if (x > d.tau) {
                    const unsigned long long deg = d.off[v + 1] - d.off[v];
                    act = true;
                    d.pr_r[v] += x;
                    d.pr_c[v] = deg ? (17ull * x) / (20ull * deg) : 0ull;
                    d.pr_res[v] = 0ull;
                } else {
                    d.pr_res[v] = x;
                }
            }
        }
        const uint32_t bits = __ballot_sync(FULL, act);
        if (lane == 0) { d.A[w] = bits; d.next[w] = 0; }
    }
}

__global__ void k_add_u64(unsigned long long* __restrict__ dst, const unsigned long long* __restrict__ src, uint64_t n) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
        dst[i] += src[i];
}

// PRD output: rank = (r + res) * 2^-56, u64 -> fp64 -> fp32, both round-to-nearest
__global__ void k_prd_output(DevState d) {
    for (uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v < d.n; v += (uint64_t)gridDim.x * blockDim.x)
        d.rank[v] = __double2float_rn(__ull2double_rn(d.pr_r[v] + d.pr_res[v]) * 0x1p-56);
}

__global__ void k_finalize_bfs(DevState d) {
    for (uint32_t w = blockIdx.x * blockDim.x + threadIdx.x; w < d.nwords; w += gridDim.x * blockDim.x) {
        const uint32_t nx = d.next[w];
        const uint32_t vis = d.visited[w];
        const uint32_t nw = nx & ~vis;
        d.A[w] = nw;
        if (nx) d.next[w] = 0;
        if (nw) {
            d.visited[w] = vis | nw;
            uint32_t b = nw;
            while (b) {
                const int i = __ffs(b) - 1;
                b &= b - 1;
                d.val[(uint64_t)w * 32 + i] = d.iter + 1;
            }
        }
    }
}

__global__ void k_finalize_minlabel(DevState d) {
    for (uint32_t w = blockIdx.x * blockDim.x + threadIdx.x; w < d.nwords; w += gridDim.x * blockDim.x) {
        const uint32_t nx = d.next[w];
        d.A[w] = nx;
        if (nx) {
            d.next[w] = 0;
            uint32_t b = nx;
            while (b) {
                const int i = __ffs(b) - 1;
                b &= b - 1;
                const uint64_t v = (uint64_t)w * 32 + i;
                d.snap[v] = d.val[v];
            }
        }
    }
}

// r' = (1-d)/n + d (sum + dang/n) in fp64, stored fp32; contrib = fp32(r'/deg);
// next dangling mass accumulated from the fp64 r', per warp, into the fixed-point total.
__global__ void k_finalize_pr(DevState d, int cur) {
    const double inv_n = 1.0 / (double)d.n;
    const double dc = from_fx(d.dang[cur]);
    double dn = 0.0;
    for (uint64_t v = d.vlo + (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v < d.vhi;
         v += (uint64_t)gridDim.x * blockDim.x) {
        const double r = (1.0 - kDamp) * inv_n + kDamp * (from_fx(d.sum[v]) + dc * inv_n);
        const unsigned long long deg = __ldg(d.off + v + 1) - __ldg(d.off + v);
        d.rank[v] = (float)r;
        d.contrib[v] = deg ? (float)(r / (double)deg) : 0.0f;
        if (!deg) dn += r;
    }
    dn = warp_sum_d(dn);
    if ((threadIdx.x & 31) == 0 && dn != 0.0) atomicAdd(d.dang + (cur ^ 1), to_fx(dn));
}

// P > 1: values were MIN-exchanged, so A_{t+1} = {v : val[v] < snap[v]} over every vertex
__global__ void __launch_bounds__(256) k_finalize_minlabel_dense(DevState d) {
    FOR_EACH_WORD_WARP(d, w, v, lane) {
        bool act = false;
        if (v < d.n) {
            const uint32_t x = d.val[v], y = d.snap[v];
            if (x < y) { act = true; d.snap[v] = x; }
        }
        const uint32_t bits = __ballot_sync(FULL, act);
        if (lane == 0) { d.A[w] = bits; d.next[w] = 0; }
    }
}

__global__ void k_or_reduce(uint32_t* __restrict__ dst, const uint32_t* __restrict__ g, uint32_t parts, uint64_t nw) {
    for (uint64_t w = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; w < nw; w += (uint64_t)gridDim.x * blockDim.x) {
        uint32_t x = 0;
        for (uint32_t p = 0; p < parts; ++p) x |= g[(uint64_t)p * nw + w];
        dst[w] = x;
    }
}

__global__ void k_or_into(uint32_t* __restrict__ dst, const uint32_t* __restrict__ src, uint64_t nw) {
    for (uint64_t w = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; w < nw; w += (uint64_t)gridDim.x * blockDim.x)
        dst[w] |= src[w];
}

__global__ void k_min_into(uint32_t* __restrict__ dst, const uint32_t* __restrict__ src, uint64_t n) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
        dst[i] = min(dst[i], src[i]);
}

// sparse MIN exchange (SSSP / CC): this rank's improvements of the iteration as
// (id, value) pairs. A vertex's next bit is set iff this rank lowered its value below the
// iteration-start snapshot, which every rank shares, so the pairs of all ranks reproduce the MIN.
// Order of the pairs is irrelevant (MIN commutes); `count` may exceed `cap` (then the caller
// falls back to the dense exchange and nothing past cap is written).
__global__ void __launch_bounds__(256) k_sparse_pack(const uint32_t* __restrict__ next, const uint32_t* __restrict__ val,
                                                     uint32_t nwords, uint2* __restrict__ out, uint32_t cap,
                                                     uint32_t* __restrict__ count) {
    const int lane = threadIdx.x & 31;
    for (uint32_t w0 = blockIdx.x * blockDim.x; w0 < nwords; w0 += gridDim.x * blockDim.x) {   // warp-uniform trip count
        const uint32_t w = w0 + threadIdx.x;
        const uint32_t bits = w < nwords ? next[w] : 0u;
        const uint32_t c = __popc(bits);
        uint32_t incl = c;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(FULL, incl, o);
            if (lane >= o) incl += y;
        }
        const uint32_t tot = __shfl_sync(FULL, incl, 31);
        uint32_t base = 0;
        if (lane == 31 && tot) base = atomicAdd(count, tot);
        base = __shfl_sync(FULL, base, 31);
        uint32_t i = base + incl - c;
        uint32_t b = bits;
        while (b) {
            const int k = __ffs(b) - 1;
            b &= b - 1;
            const uint32_t v = w * 32u + (uint32_t)k;
            if (i < cap) out[i] = make_uint2(v, val[v]);
            ++i;
        }
    }
}

// apply the other ranks' pairs: val = min(val, x), next bit set (every pair is below the shared
// snapshot, so the vertex is active at t+1 whichever rank lowered it). pairs of rank p at
// pairs + p * stride, counts[p] of them; rank `skip` (this one) is left out.
__global__ void __launch_bounds__(256) k_sparse_apply(uint32_t* __restrict__ val, uint32_t* __restrict__ next,
                                                      const uint2* __restrict__ pairs, uint64_t stride,
                                                      const uint32_t* __restrict__ counts, int P, int skip, uint32_t cap) {
    for (int p = 0; p < P; ++p) {
        if (p == skip) continue;
        const uint32_t c = min(counts[p], cap);
        const uint2* src = pairs + (uint64_t)p * stride;
        for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < c; i += gridDim.x * blockDim.x) {
            const uint2 x = src[i];
            atomicMin(val + x.x, x.y);
            atomicOr(next + (x.x >> 5), 1u << (x.x & 31u));
        }
    }
}

__global__ void k_check_monotone(const unsigned long long* __restrict__ off, uint64_t n, unsigned long long* bad) {
    for (uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x)
        if (off[v + 1] < off[v]) atomicMin(bad, (unsigned long long)v);
}

// ------------------------------------------------------------------ §3.4 data replacement
// Accesses of this iteration per 16 KiB chunk: every active list with deg > 0 is
// in exactly one of the hit queues or the miss queue; its arcs [a, e) (rank-local) add their
// overlap with each chunk they touch. Consecutive queue entries are ascending vertex ids, so
// neighbouring lanes mostly hit the same chunk: single-chunk lists are combined per warp
// (match + reduce) before the atomic.
__global__ void __launch_bounds__(256) k_chunk_access(DevState d, Queues q, uint32_t n_small, uint32_t n_med,
                                                      uint32_t n_hub, uint32_t epc_shift, uint32_t* __restrict__ acc) {
    const unsigned long long total = (unsigned long long)n_small + n_med + n_hub + q.n_missq;
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    const unsigned long long x0 = d.static_arc0;
    for (unsigned long long i0 = (unsigned long long)blockIdx.x * blockDim.x; i0 < total; i0 += stride) {
        const unsigned long long i = i0 + threadIdx.x;
        uint32_t key = 0xFFFFFFFFu, val = 0;
        if (i < total) {
            unsigned long long j = i;
            uint32_t v;
            if (j < n_small) v = __ldg(q.hq_small + j);
            else if ((j -= n_small) < n_med) v = __ldg(q.hq_med + j);
            else if ((j -= n_med) < n_hub) v = __ldg(q.hq_hub + j);
            else v = __ldg(q.mq + (j - n_hub));
            const unsigned long long a = __ldg(d.off + v) - x0, e = __ldg(d.off + v + 1) - x0;
            const unsigned long long c0 = a >> epc_shift, c1 = (e - 1) >> epc_shift;
            if (c0 == c1) {
                key = (uint32_t)c0;
                val = (uint32_t)(e - a);
            } else {
                for (unsigned long long c = c0; c <= c1; ++c) {
                    const unsigned long long lo = max(a, c << epc_shift), hi = min(e, (c + 1) << epc_shift);
                    atomicAdd(acc + c, (uint32_t)(hi - lo));
                }
            }
        }
        const uint32_t peers = __match_any_sync(FULL, key);
        const uint32_t sum = __reduce_add_sync(peers, val);
        if (key != 0xFFFFFFFFu && (threadIdx.x & 31) == __ffs(peers) - 1) atomicAdd(acc + key, sum);
    }
}

// Swap i: chunk in[i] takes the slot of chunk out[i] (the swap DMAs already landed). Then the
// StaticBitmap is recomputed for every vertex touching a changed chunk: v is static iff all
// chunks of its list are resident; a degree-0 vertex at arc x belongs to chunk (x-1)/epc.
__global__ void k_apply_swaps(uint32_t* __restrict__ slot_of, const uint32_t* __restrict__ sw, uint32_t k) {
    // sw = [in[0..k), out[0..k), slot[0..k)]: in and out are disjoint chunk sets
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < k; i += gridDim.x * blockDim.x) {
        slot_of[sw[i]] = sw[2 * k + i];
        slot_of[sw[k + i]] = kNoSlot;
    }
}

__device__ __forceinline__ bool chunks_resident(const uint32_t* slot_of, unsigned long long a, unsigned long long e,
                                                uint32_t epc_shift) {
    if (e == a) return a == 0 || slot_of[(a - 1) >> epc_shift] != kNoSlot;
    for (unsigned long long c = a >> epc_shift; c <= (e - 1) >> epc_shift; ++c)
        if (slot_of[c] == kNoSlot) return false;
    return true;
}

// one warp per changed chunk (2k of them: the swapped-in and the evicted)
__global__ void __launch_bounds__(256) k_static_rebits(DevState d, const uint32_t* __restrict__ slot_of,
                                                       const uint32_t* __restrict__ sw, uint32_t nchg,
                                                       uint32_t epc_shift) {
    const int lane = threadIdx.x & 31;
    const uint32_t w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    if (w >= nchg) return;
    const unsigned long long x0 = d.static_arc0;
    const unsigned long long c = sw[w];
    const unsigned long long lo = x0 + (c << epc_shift), hi = x0 + ((c + 1) << epc_shift);
    // first v in [vlo, vhi) with off[v+1] > lo (its list ends after the chunk starts)
    unsigned long long L = d.vlo, R = d.vhi;
    while (L < R) {
        const unsigned long long mid = (L + R) >> 1;
        if (d.off[mid + 1] > lo) R = mid; else L = mid + 1;
    }
    for (unsigned long long v0 = L;; v0 += 32) {
        const unsigned long long v = v0 + lane;
        bool in = false;
        if (v < d.vhi) {
            const unsigned long long a = d.off[v], e = d.off[v + 1];
            in = a <= hi;
            if (in) {
                const uint32_t bit = 1u << (v & 31);
                if (chunks_resident(slot_of, a - x0, e - x0, epc_shift)) atomicOr(d.S + (v >> 5), bit);
                else atomicAnd(d.S + (v >> 5), ~bit);
            }
        }
        if (!__any_sync(FULL, in)) break;
    }
}

// S over the owned range from the chunk residency (random initial content): one warp per
// 32-vertex word, the word written whole (a part's S holds only its own range's bits)
__global__ void __launch_bounds__(256) k_static_bits_all(DevState d, const uint32_t* __restrict__ slot_of,
                                                         uint32_t epc_shift) {
    const int lane = threadIdx.x & 31;
    const uint64_t w0 = d.vlo >> 5, w1 = (d.vhi + 31) >> 5;
    const uint64_t nw = (uint64_t)gridDim.x * blockDim.x >> 5;
    for (uint64_t w = w0 + ((blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5); w < w1; w += nw) {
        const uint64_t v = w * 32 + lane;
        bool st = false;
        if (v >= d.vlo && v < d.vhi)
            st = chunks_resident(slot_of, __ldg(d.off + v) - d.static_arc0, __ldg(d.off + v + 1) - d.static_arc0,
                                 epc_shift);
        const uint32_t word = __ballot_sync(FULL, st);
        if (lane == 0) d.S[w] = word;
    }
}

// Chunk copy (random fill, §3.4 swaps): CTA i copies chunk ids[i] (16 KiB, clipped at D) from the
// mapped host CSR to its slot; 16 B loads when the rank's payload start is 16-byte aligned,
// 4 B otherwise; all of a thread's loads are issued before its stores.
__global__ void __launch_bounds__(256) k_copy_chunks(const char* __restrict__ host, unsigned long long x0,
                                                     unsigned long long D, const uint32_t* __restrict__ ids,
                                                     const uint32_t* __restrict__ slots, uint32_t count,
                                                     char* __restrict__ dst) {
    for (uint32_t i = blockIdx.x; i < count; i += gridDim.x) {
        const unsigned long long c = ids[i], slot = slots ? slots[i] : i;
        const unsigned long long o = c << kChunkShift;
        const unsigned long long len = min((unsigned long long)kChunkBytes, D - o);
        const char* src = host + x0 + o;
        char* out = dst + (slot << kChunkShift);
        if ((x0 & 15ull) == 0 && len == kChunkBytes) {
            const uint4* s4 = reinterpret_cast<const uint4*>(src);
            uint4* d4 = reinterpret_cast<uint4*>(out);
            uint4 v[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) v[j] = s4[threadIdx.x + 256 * j];
#pragma unroll
            for (int j = 0; j < 4; ++j) d4[threadIdx.x + 256 * j] = v[j];
        } else {
            const uint32_t* s1 = reinterpret_cast<const uint32_t*>(src);
            uint32_t* d1 = reinterpret_cast<uint32_t*>(out);
            for (unsigned long long j = threadIdx.x; j < len / 4; j += blockDim.x) d1[j] = s1[j];
        }
    }
}

inline unsigned blocks_for(unsigned long long n, int per_block, unsigned cap = 148u * 16u) {
    unsigned long long b = (n + per_block - 1) / per_block;
    if (b < 1) b = 1;
    return (unsigned)(b > cap ? cap : b);
}

template <int ALGO, bool REMAP>
void static_launch_t(const DevState& d, const Queues& q, const void* sbase, uint32_t ns, uint32_t nm, uint32_t nh,
                     uint32_t npieces, uint32_t piece, int max_ctas, cudaStream_t s) {
    auto cap = [&](unsigned long long b) { return (unsigned)(b < (unsigned long long)max_ctas ? b : max_ctas); };
    if (ns) { k_static_small<ALGO, REMAP><<<cap((ns + 255) / 256), 256, 0, s>>>(d, q.hq_small, ns, sbase); ++g_launches; }
    if (nm) { k_static_med<ALGO, REMAP><<<cap((nm + 7) / 8), 256, 0, s>>>(d, q.hq_med, nm, sbase); ++g_launches; }
    if (nh) {
        k_static_hub<ALGO, REMAP><<<cap(npieces), 256, 0, s>>>(d, q.hq_hub, q.hub_pre, nh, npieces, piece, sbase);
        ++g_launches;
    }
}

template <int ALGO>
void static_launch(const DevState& d, const Queues& q, const void* sbase, uint32_t ns, uint32_t nm, uint32_t nh,
                   uint32_t npieces, uint32_t piece, int max_ctas, cudaStream_t s) {
    if (d.slot_of) static_launch_t<ALGO, true>(d, q, sbase, ns, nm, nh, npieces, piece, max_ctas, s);
    else static_launch_t<ALGO, false>(d, q, sbase, ns, nm, nh, npieces, piece, max_ctas, s);
}

}  // namespace

void launch_static(int algo, const DevState& d, const Queues& q, const void* sbase, uint32_t ns, uint32_t nm,
                   uint32_t nh, uint32_t npieces, uint32_t piece, int max_ctas, cudaStream_t s) {
    switch (algo) {
        case PRD: static_launch<PRD>(d, q, sbase, ns, nm, nh, npieces, piece, max_ctas, s); break;
        case BFS: static_launch<BFS>(d, q, sbase, ns, nm, nh, npieces, piece, max_ctas, s); break;
        case SSSP: static_launch<SSSP>(d, q, sbase, ns, nm, nh, npieces, piece, max_ctas, s); break;
        case CC: static_launch<CC>(d, q, sbase, ns, nm, nh, npieces, piece, max_ctas, s); break;
        default: static_launch<PR>(d, q, sbase, ns, nm, nh, npieces, piece, max_ctas, s); break;
    }
}

void launch_static_pr_seg(const DevState& d, const Queues& q, const void* sbase, uint32_t ns, uint32_t nm, uint32_t nh,
                          uint32_t npieces, uint32_t piece, uint32_t passes, uint32_t* cur_med, uint32_t* cur_hub,
                          int max_ctas, cudaStream_t s) {
    auto cap = [&](unsigned long long b) { return (unsigned)(b < (unsigned long long)max_ctas ? b : max_ctas); };
    const uint32_t* sb = reinterpret_cast<const uint32_t*>(sbase);
    if (ns) { k_static_small<PR, false><<<cap((ns + 255) / 256), 256, 0, s>>>(d, q.hq_small, ns, sbase); ++g_launches; }
    const uint64_t slice = (d.n + passes - 1) / passes;
    for (uint32_t j = 0; j < passes; ++j) {
        const uint32_t hi_id = (uint32_t)std::min<uint64_t>(d.n, (j + 1) * slice);
        if (nm) {
            if (j == 0) k_static_med_pr_seg<true><<<cap((nm + 7) / 8), 256, 0, s>>>(d, q.hq_med, nm, sb, cur_med, hi_id);
            else k_static_med_pr_seg<false><<<cap((nm + 7) / 8), 256, 0, s>>>(d, q.hq_med, nm, sb, cur_med, hi_id);
            ++g_launches;
        }
        if (nh) {
            if (j == 0)
                k_static_hub_pr_seg<true><<<cap(npieces), 256, 0, s>>>(d, q.hq_hub, q.hub_pre, nh, npieces, piece, sb, cur_hub, hi_id);
            else
                k_static_hub_pr_seg<false><<<cap(npieces), 256, 0, s>>>(d, q.hq_hub, q.hub_pre, nh, npieces, piece, sb, cur_hub, hi_id);
            ++g_launches;
        }
    }
}

void launch_chunk_access(const DevState& d, const Queues& q, uint32_t n_small, uint32_t n_med, uint32_t n_hub,
                         uint32_t b_e, uint32_t* acc, cudaStream_t s) {
    const unsigned long long total = (unsigned long long)n_small + n_med + n_hub + q.n_missq;
    if (!total) return;
    const uint32_t epc_shift = kChunkShift - (b_e == 8 ? 3 : 2);
    k_chunk_access<<<blocks_for(total, 256), 256, 0, s>>>(d, q, n_small, n_med, n_hub, epc_shift, acc);
    ++g_launches;
}

void launch_apply_swaps(const DevState& d, uint32_t* slot_of, const uint32_t* sw, uint32_t k, uint32_t b_e,
                        cudaStream_t s) {
    if (!k) return;
    const uint32_t epc_shift = kChunkShift - (b_e == 8 ? 3 : 2);
    k_apply_swaps<<<blocks_for(k, 256), 256, 0, s>>>(slot_of, sw, k);
    k_static_rebits<<<(2 * k + 7) / 8, 256, 0, s>>>(d, slot_of, sw, 2 * k, epc_shift);
    g_launches += 2;
}

void launch_copy_chunks(const void* host_dev, uint64_t x0, uint64_t D, const uint32_t* ids, const uint32_t* slots,
                        uint32_t count, void* dst, cudaStream_t s) {
    if (!count) return;
    // 64 CTAs x 16 KiB = 1 MiB of host reads in flight (the transfer engine's sizing)
    k_copy_chunks<<<count < 64u ? count : 64u, 256, 0, s>>>(reinterpret_cast<const char*>(host_dev), x0, D, ids, slots,
                                                          count, reinterpret_cast<char*>(dst));
    ++g_launches;
}

void launch_static_bits(const DevState& d, const uint32_t* slot_of, uint32_t b_e, cudaStream_t s) {
    const uint32_t epc_shift = kChunkShift - (b_e == 8 ? 3 : 2);
    const unsigned long long words = ((d.vhi + 31) >> 5) - (d.vlo >> 5);
    if (!words) return;
    k_static_bits_all<<<blocks_for(words, 8), 256, 0, s>>>(d, slot_of, epc_shift);
    ++g_launches;
}

void launch_ondemand(int algo, const DevState& d, const Queues& q, const void* chunk,
                     unsigned long long lo, unsigned long long hi, unsigned long long span_base, cudaStream_t s) {
    if (hi <= lo) return;
    const unsigned long long len = hi - lo;
    const unsigned tiles = (unsigned)(((hi - 1) >> kEdgeTileShift) - (lo >> kEdgeTileShift) + 1);
    if (algo == BFS && span_base != ~0ull) {
        k_ondemand_g<BFS><<<tiles, 256, 0, s>>>(d, q, chunk, lo, hi, span_base);
        ++g_launches;
        return;
    }
    if (algo == BFS) {
        k_ondemand_bfs<<<blocks_for(len, 256 * 4), 256, 0, s>>>(d, reinterpret_cast<const uint32_t*>(chunk), len);
        ++g_launches;
        return;
    }
    switch (algo) {
        case SSSP: k_ondemand_g<SSSP><<<tiles, 256, 0, s>>>(d, q, chunk, lo, hi, span_base); break;
        case CC: k_ondemand_g<CC><<<tiles, 256, 0, s>>>(d, q, chunk, lo, hi, span_base); break;
        case PRD: k_ondemand_g<PRD><<<tiles, 256, 0, s>>>(d, q, chunk, lo, hi, span_base); break;
        default: k_ondemand_g<PR><<<tiles, 256, 0, s>>>(d, q, chunk, lo, hi, span_base); break;
    }
    ++g_launches;
}

void launch_gather(const Queues& q, const void* host_nbr, uint64_t m, uint32_t b_e, void* chunk,
                   unsigned long long lo, unsigned long long hi, int max_ctas, const unsigned long long* lint,
                   uint32_t nlint, uint32_t gap_bytes, unsigned long long* cover, cudaStream_t s,
                   const DevState* visit) {
    if (hi <= lo) return;
    const unsigned long long tiles = ((hi - 1) >> kEdgeTileShift) - (lo >> kEdgeTileShift) + 1;
    const unsigned grid = (unsigned)(tiles < (unsigned long long)max_ctas ? tiles : (unsigned long long)max_ctas);
    const uintptr_t hp = reinterpret_cast<uintptr_t>(host_nbr);
    const uint4* base = reinterpret_cast<const uint4*>(hp & ~(uintptr_t)15);
    const uint32_t hoff = (uint32_t)(hp & 15);
    uint32_t* c = reinterpret_cast<uint32_t*>(chunk);
    const unsigned long long w_end = hoff / 4 + m * (b_e / 4);   // host words from the aligned base
    // units loaded per lane per round: a 256-arc warp segment of 8-byte arcs is 128 units plus up to
    // one per piece boundary, so 4 per lane (128) usually needs a second, nearly empty round; 6 took
    // C2's gather from 44.6-44.7 to 45.0 GB/s (profiles/r01/gather_ng_ab.log; 5 and 8 within noise of
    // 6). 4-byte arcs: 64 units per segment, 4 per lane fits.
    const DevState none{};
    if (b_e == 8) k_gather16<8, 6, false><<<grid, 256, 0, s>>>(q, base, hoff, w_end, c, lo, hi, lint, nlint, gap_bytes / 4, cover, none);
    else if (visit) k_gather16<4, 4, true><<<grid, 256, 0, s>>>(q, base, hoff, w_end, c, lo, hi, lint, nlint, gap_bytes / 4, cover, *visit);
    else k_gather16<4, 4, false><<<grid, 256, 0, s>>>(q, base, hoff, w_end, c, lo, hi, lint, nlint, gap_bytes / 4, cover, none);
    ++g_launches;
}

void launch_long_runs(const uint32_t* run_b, const uint32_t* run_e, const unsigned long long* run_dst, uint32_t n_runs,
                      const unsigned long long* off, unsigned long long min_arcs, unsigned long long* out, uint32_t cap,
                      uint32_t* count, uint32_t* done, uint32_t* flag, cudaStream_t s) {
    cudaMemsetAsync(count, 0, 4, s);
    cudaMemsetAsync(done, 0, 4, s);
    k_long_runs<<<blocks_for(n_runs ? n_runs : 1, 256, 148u * 4u), 256, 0, s>>>(run_b, run_e, run_dst, n_runs, off,
                                                                                min_arcs, out, cap, count, done, flag);
    ++g_launches;
}

void launch_span_windows(const Queues& q, unsigned long long h0, unsigned long long h1, unsigned long long win,
                         uint32_t nwin, unsigned long long* out, uint32_t* flag, cudaStream_t s) {
    k_span_windows<<<1, 1024, 0, s>>>(q, h0, h1, win, nwin, out, flag);
    ++g_launches;
}

void launch_init(int algo, const DevState& d, uint32_t source, cudaStream_t s) {
    const unsigned gb = blocks_for(d.n, 256);
    cudaMemsetAsync(d.A, 0, (size_t)d.nwords * 4, s);
    cudaMemsetAsync(d.next, 0, (size_t)d.nwords * 4, s);
    switch (algo) {
        case BFS:
            cudaMemsetAsync(d.visited, 0, (size_t)d.nwords * 4, s);
            k_fill_u32<<<gb, 256, 0, s>>>(d.val, d.n, kInf);
            ++g_launches;
            k_set_source<<<1, 1, 0, s>>>(d, source, algo);
            ++g_launches;
            break;
        case SSSP:
            k_fill_u32<<<gb, 256, 0, s>>>(d.val, d.n, kInf);
            ++g_launches;
            k_fill_u32<<<gb, 256, 0, s>>>(d.snap, d.n, kInf);
            ++g_launches;
            k_set_source<<<1, 1, 0, s>>>(d, source, algo);
            ++g_launches;
            break;
        case CC:
            k_iota_u32<<<gb, 256, 0, s>>>(d.val, d.snap, d.n);
            ++g_launches;
            k_range_bits<<<blocks_for(d.nwords, 256), 256, 0, s>>>(d.A, d.nwords, 0, d.n);
            ++g_launches;
            break;
        case PRD: {
            const unsigned long long res0 = (3ull << 56) / (20ull * d.n);   // floor((1-d) Q / n)
            k_prd_init<<<gb, 256, 0, s>>>(d, res0);
            ++g_launches;
            break;
        }
        default:
            cudaMemsetAsync(d.dang, 0, 2 * sizeof(unsigned long long), s);
            k_pr_init<<<gb, 256, 0, s>>>(d);
            ++g_launches;
            k_range_bits<<<blocks_for(d.nwords, 256), 256, 0, s>>>(d.A, d.nwords, 0, d.n);
            ++g_launches;
            break;
    }
}

void launch_finalize(int algo, const DevState& d, bool dense, cudaStream_t s) {
    switch (algo) {
        case BFS: k_finalize_bfs<<<blocks_for(d.nwords, 256), 256, 0, s>>>(d); break;
        case PRD:
            if (dense) k_finalize_prd_dense<<<blocks_for(d.nwords, 8), 256, 0, s>>>(d);
            else k_finalize_prd<<<blocks_for(d.nwords, 256), 256, 0, s>>>(d);
            break;
        case SSSP:
        case CC:
            if (dense) k_finalize_minlabel_dense<<<blocks_for(d.nwords, 8), 256, 0, s>>>(d);
            else k_finalize_minlabel<<<blocks_for(d.nwords, 256), 256, 0, s>>>(d);
            break;
        default: {
            const int cur = (int)(d.iter & 1u);
            cudaMemsetAsync(d.dang + (cur ^ 1), 0, sizeof(unsigned long long), s);
            k_finalize_pr<<<blocks_for(d.vhi > d.vlo ? d.vhi - d.vlo : 1, 256), 256, 0, s>>>(d, cur);
            break;
        }
    }
    ++g_launches;
}

void launch_prd_output(const DevState& d, cudaStream_t s) {
    k_prd_output<<<blocks_for(d.n, 256), 256, 0, s>>>(d);
    ++g_launches;
}

void launch_or_reduce(uint32_t* dst, const uint32_t* gathered, uint32_t parts, uint64_t nw, cudaStream_t s) {
    k_or_reduce<<<blocks_for(nw, 256), 256, 0, s>>>(dst, gathered, parts, nw);
    ++g_launches;
}

void launch_or_into(uint32_t* dst, const uint32_t* src, uint64_t nw, cudaStream_t s) {
    k_or_into<<<blocks_for(nw, 256), 256, 0, s>>>(dst, src, nw);
    ++g_launches;
}

void launch_sparse_pack(const uint32_t* next, const uint32_t* val, uint32_t nwords, void* pairs, uint32_t cap,
                        uint32_t* count, cudaStream_t s) {
    cudaMemsetAsync(count, 0, 4, s);
    k_sparse_pack<<<blocks_for(nwords, 256), 256, 0, s>>>(next, val, nwords, reinterpret_cast<uint2*>(pairs), cap, count);
    ++g_launches;
}

void launch_sparse_apply(uint32_t* val, uint32_t* next, const void* pairs, uint64_t stride, const uint32_t* counts,
                         int P, int skip, uint32_t cap, cudaStream_t s) {
    k_sparse_apply<<<blocks_for(cap, 256, 148u * 4u), 256, 0, s>>>(val, next, reinterpret_cast<const uint2*>(pairs),
                                                                    stride, counts, P, skip, cap);
    ++g_launches;
}

void launch_min_into(uint32_t* dst, const uint32_t* src, uint64_t n, cudaStream_t s) {
    k_min_into<<<blocks_for(n, 256), 256, 0, s>>>(dst, src, n);
    ++g_launches;
}

void launch_finalize_peers(int algo, const DevState& d, const void* const* peers, int P, cudaStream_t s) {
    const unsigned g = blocks_for(d.nwords, 256), gw = blocks_for(d.nwords, 8);
    switch (algo) {
        case BFS: k_finalize_bfs_peers<<<g, 256, 0, s>>>(d, reinterpret_cast<const uint32_t* const*>(peers), P); break;
        case SSSP:
        case CC: k_finalize_min_peers<<<gw, 256, 0, s>>>(d, reinterpret_cast<const uint32_t* const*>(peers), P); break;
        case PRD:
            k_finalize_prd_peers<<<gw, 256, 0, s>>>(d, reinterpret_cast<const unsigned long long* const*>(peers), P);
            break;
        default: return;
    }
    ++g_launches;
}

void launch_add_u64(unsigned long long* dst, const unsigned long long* src, uint64_t n, cudaStream_t s) {
    k_add_u64<<<blocks_for(n, 256), 256, 0, s>>>(dst, src, n);
    ++g_launches;
}

void launch_check_monotone(const unsigned long long* off, uint64_t n, unsigned long long* bad, cudaStream_t s) {
    if (!n) return;
    k_check_monotone<<<blocks_for(n, 256), 256, 0, s>>>(off, n, bad);
    ++g_launches;
}

void launch_set_range_bits(uint32_t* bits, uint32_t nwords, uint64_t a, uint64_t b, cudaStream_t s) {
    if (nwords) { k_range_bits<<<blocks_for(nwords, 256), 256, 0, s>>>(bits, nwords, a, b); ++g_launches; }
}

}  // namespace ascetic
