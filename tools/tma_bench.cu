// tma_bench.cu — does a TMA bulk copy (cp.async.bulk global->shared) read mapped pinned host
// memory over PCIe more efficiently than SM loads? (dev microbenchmark, not the product)
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/tma_bench tools/tma_bench.cu
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <cstring>
#include <vector>
#include <random>
#include <algorithm>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); exit(1);} } while (0)

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t cnt) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(smem_u32(b)), "r"(cnt));
}
__device__ __forceinline__ void mbar_expect(uint64_t* b, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(smem_u32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* b) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 :: "r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t phase) {
    uint32_t done = 0;
    while (!done)
        asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                     : "=r"(done) : "r"(smem_u32(b)), "r"(phase) : "memory");
}

// contiguous: CTA-stride over CH-byte chunks; 1 bulk copy in flight per CTA, threads store smem->global
template <int CH>
__global__ void __launch_bounds__(256) tma_copy(const char* __restrict__ src, char* __restrict__ dst, size_t nch) {
    extern __shared__ __align__(128) char smem[];
    __shared__ __align__(8) uint64_t bar;
    if (threadIdx.x == 0) { mbar_init(&bar, 1); asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
    __syncthreads();
    uint32_t phase = 0;
    for (size_t c = blockIdx.x; c < nch; c += gridDim.x) {
        if (threadIdx.x == 0) { mbar_expect(&bar, CH); bulk_g2s(smem, src + c * CH, CH, &bar); }
        mbar_wait(&bar, phase);
        phase ^= 1;
        const uint4* s4 = reinterpret_cast<const uint4*>(smem);
        uint4* d4 = reinterpret_cast<uint4*>(dst + c * CH);
        for (int i = threadIdx.x; i < CH / 16; i += blockDim.x) d4[i] = s4[i];
        __syncthreads();
    }
}

// gather: one warp per run piece (<= SLOT bytes); lane 0 issues the bulk copy of the 16-byte
// aligned superset [a & ~15, (b + 15) & ~15) into the warp's slot, the warp copies the exact
// 8-byte elements to dst at the run's stream offset
template <int SLOT>
__global__ void __launch_bounds__(256) tma_gather(const char* __restrict__ src, const uint64_t* __restrict__ pa,
                                                  const uint32_t* __restrict__ plen, const uint64_t* __restrict__ pdst,
                                                  uint32_t npieces, uint64_t* __restrict__ dst) {
    extern __shared__ __align__(128) char smem[];
    __shared__ __align__(8) uint64_t bar[8];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    char* slot = smem + warp * (SLOT + 32);
    if (lane == 0) { mbar_init(&bar[warp], 1); asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
    __syncwarp();
    uint32_t phase = 0;
    const uint32_t nw = gridDim.x * 8;
    for (uint32_t i = blockIdx.x * 8 + warp; i < npieces; i += nw) {
        const uint64_t a = pa[i], len = plen[i];
        const uint64_t a16 = a & ~15ull, b16 = (a + len + 15) & ~15ull;
        if (lane == 0) { mbar_expect(&bar[warp], (uint32_t)(b16 - a16)); bulk_g2s(slot, src + a16, (uint32_t)(b16 - a16), &bar[warp]); }
        mbar_wait(&bar[warp], phase);
        phase ^= 1;
        const uint64_t* s8 = reinterpret_cast<const uint64_t*>(slot + (a - a16));
        uint64_t* d8 = dst + pdst[i] / 8;
        for (uint32_t k = lane; k < len / 8; k += 32) d8[k] = s8[k];
        __syncwarp();
    }
}

// baseline: SM loads, one warp per piece
__global__ void __launch_bounds__(256) ld_gather(const uint64_t* __restrict__ src, const uint64_t* __restrict__ pa,
                                                 const uint32_t* __restrict__ plen, const uint64_t* __restrict__ pdst,
                                                 uint32_t npieces, uint64_t* __restrict__ dst) {
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t nw = gridDim.x * 8;
    for (uint32_t i = blockIdx.x * 8 + warp; i < npieces; i += nw) {
        const uint64_t* s8 = src + pa[i] / 8;
        uint64_t* d8 = dst + pdst[i] / 8;
        const uint32_t n = plen[i] / 8;
        for (uint32_t k = lane; k < n; k += 32) d8[k] = s8[k];
    }
}

// baseline 2: the product gather's load shape -- 16-byte loads of the piece's 16-byte-aligned cover
// (k_gather16), one warp per piece, NG units in flight per lane; each lane stores the 8-byte words
// of its unit that fall inside the piece
template <int NG>
__global__ void __launch_bounds__(256) ld16_gather(const uint4* __restrict__ src, const uint64_t* __restrict__ pa,
                                                   const uint32_t* __restrict__ plen, const uint64_t* __restrict__ pdst,
                                                   uint32_t npieces, uint64_t* __restrict__ dst) {
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t nw = gridDim.x * 8;
    for (uint32_t i = blockIdx.x * 8 + warp; i < npieces; i += nw) {
        const uint64_t a = pa[i], b = a + plen[i];
        const uint64_t u0 = a >> 4, u1 = (b + 15) >> 4;
        uint64_t* d8 = dst + pdst[i] / 8;
        for (uint64_t u = u0; u < u1; u += 32 * NG) {
            uint4 v[NG];
#pragma unroll
            for (int g = 0; g < NG; ++g) {
                const uint64_t uu = u + 32 * g + lane;
                if (uu < u1) v[g] = src[uu];
            }
#pragma unroll
            for (int g = 0; g < NG; ++g) {
                const uint64_t uu = u + 32 * g + lane;
                if (uu >= u1) continue;
                const uint64_t w0 = uu * 16, w1 = w0 + 8;
                if (w0 >= a && w0 < b) d8[(w0 - a) / 8] = ((uint64_t)v[g].y << 32) | v[g].x;
                if (w1 >= a && w1 < b) d8[(w1 - a) / 8] = ((uint64_t)v[g].w << 32) | v[g].z;
            }
        }
    }
}

// TMA gather with two slots per warp: the bulk copy of piece i+1 is in flight while the warp
// stores piece i
template <int SLOT>
__global__ void __launch_bounds__(256) tma_gather2(const char* __restrict__ src, const uint64_t* __restrict__ pa,
                                                   const uint32_t* __restrict__ plen, const uint64_t* __restrict__ pdst,
                                                   uint32_t npieces, uint64_t* __restrict__ dst) {
    extern __shared__ __align__(128) char smem[];
    __shared__ __align__(8) uint64_t bar[16];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    char* slot[2] = {smem + (2 * warp) * (SLOT + 32), smem + (2 * warp + 1) * (SLOT + 32)};
    if (lane == 0) {
        mbar_init(&bar[2 * warp], 1); mbar_init(&bar[2 * warp + 1], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncwarp();
    uint32_t phase[2] = {0, 0};
    const uint32_t nw = gridDim.x * 8;
    auto issue = [&](uint32_t i, int k) {
        const uint64_t a = pa[i], len = plen[i];
        const uint64_t a16 = a & ~15ull, b16 = (a + len + 15) & ~15ull;
        if (lane == 0) { mbar_expect(&bar[2 * warp + k], (uint32_t)(b16 - a16)); bulk_g2s(slot[k], src + a16, (uint32_t)(b16 - a16), &bar[2 * warp + k]); }
    };
    uint32_t i = blockIdx.x * 8 + warp;
    int k = 0;
    if (i < npieces) issue(i, 0);
    for (; i < npieces; i += nw, k ^= 1) {
        if (i + nw < npieces) issue(i + nw, k ^ 1);
        mbar_wait(&bar[2 * warp + k], phase[k]);
        phase[k] ^= 1;
        const uint64_t a = pa[i], len = plen[i];
        const uint64_t* s8 = reinterpret_cast<const uint64_t*>(slot[k] + (a - (a & ~15ull)));
        uint64_t* d8 = dst + pdst[i] / 8;
        for (uint32_t q = lane; q < len / 8; q += 32) d8[q] = s8[q];
        __syncwarp();
    }
}

int main() {
    const size_t bytes = 512ull << 20;
    char* h; CK(cudaHostAlloc((void**)&h, bytes + 4096, cudaHostAllocMapped | cudaHostAllocPortable));
    memset(h, 1, bytes);
    char* d; CK(cudaMalloc((void**)&d, bytes));
    char* hd; CK(cudaHostGetDevicePointer((void**)&hd, h, 0));
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    auto timeit = [&](auto fn, const char* name, double nbytes) {
        fn(); CK(cudaDeviceSynchronize());
        float best = 1e9;
        for (int r = 0; r < 5; ++r) {
            cudaEventRecord(e0); fn(); cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
            float ms; cudaEventElapsedTime(&ms, e0, e1); best = std::min(best, ms);
        }
        CK(cudaGetLastError());
        printf("%-56s %8.2f GB/s  (%.3f ms)\n", name, nbytes / (best / 1e3) / 1e9, best);
    };
    timeit([&] { cudaMemcpyAsync(d, h, bytes, cudaMemcpyHostToDevice); }, "DMA cudaMemcpyAsync 512MiB", bytes);
    CK(cudaFuncSetAttribute(tma_copy<16384>, cudaFuncAttributeMaxDynamicSharedMemorySize, 16384));
    CK(cudaFuncSetAttribute(tma_copy<65536>, cudaFuncAttributeMaxDynamicSharedMemorySize, 65536));
    for (int grid : {148, 296, 592, 1184}) {
        char nm[96];
        snprintf(nm, sizeof nm, "TMA bulk 16KiB contiguous grid=%d", grid);
        timeit([&] { tma_copy<16384><<<grid, 256, 16384>>>(hd, d, bytes / 16384); }, nm, bytes);
        if (grid <= 296) {
            snprintf(nm, sizeof nm, "TMA bulk 64KiB contiguous grid=%d", grid);
            timeit([&] { tma_copy<65536><<<grid, 256, 65536>>>(hd, d, bytes / 65536); }, nm, bytes);
        }
    }
    CK(cudaFuncSetAttribute(tma_gather<4096>, cudaFuncAttributeMaxDynamicSharedMemorySize, 8 * (4096 + 32)));
    CK(cudaFuncSetAttribute(tma_gather2<4096>, cudaFuncAttributeMaxDynamicSharedMemorySize, 16 * (4096 + 32)));
    for (int avg_bytes : {256, 768, 1100, 2048, 8192, 65536}) {
        std::mt19937_64 rng(avg_bytes);
        std::vector<uint64_t> pa, pd; std::vector<uint32_t> pl;
        uint64_t total = 0;
        const uint64_t want = 128ull << 20;
        while (total < want) {
            uint64_t len = 8 * (1 + rng() % (2 * avg_bytes / 8 - 1));
            uint64_t st = 8 * (rng() % ((bytes - len) / 8));
            for (uint64_t o = 0; o < len; o += 4096 - 16) {            // pieces fit a 4 KiB slot with the superset
                const uint64_t l = std::min<uint64_t>(4096 - 16, len - o);
                pa.push_back(st + o); pl.push_back((uint32_t)l); pd.push_back(total + o);
            }
            total += len;
        }
        uint64_t *dpa, *dpd; uint32_t* dpl;
        CK(cudaMalloc(&dpa, pa.size() * 8)); CK(cudaMalloc(&dpd, pd.size() * 8)); CK(cudaMalloc(&dpl, pl.size() * 4));
        CK(cudaMemcpy(dpa, pa.data(), pa.size() * 8, cudaMemcpyHostToDevice));
        CK(cudaMemcpy(dpd, pd.data(), pd.size() * 8, cudaMemcpyHostToDevice));
        CK(cudaMemcpy(dpl, pl.data(), pl.size() * 4, cudaMemcpyHostToDevice));
        for (int grid : {148, 444, 1184}) {
            char nm[128];
            snprintf(nm, sizeof nm, "TMA gather runs avg %dB (%zu pieces) grid=%d", avg_bytes, pa.size(), grid);
            timeit([&] { tma_gather<4096><<<grid, 256, 8 * (4096 + 32)>>>(hd, dpa, dpl, dpd, (uint32_t)pa.size(), (uint64_t*)d); }, nm, (double)total);
            snprintf(nm, sizeof nm, "ld  gather runs avg %dB grid=%d", avg_bytes, grid);
            timeit([&] { ld_gather<<<grid, 256>>>((const uint64_t*)hd, dpa, dpl, dpd, (uint32_t)pa.size(), (uint64_t*)d); }, nm, (double)total);
            snprintf(nm, sizeof nm, "ld16 cover gather (k_gather16 shape) avg %dB grid=%d", avg_bytes, grid);
            timeit([&] { ld16_gather<4><<<grid, 256>>>((const uint4*)hd, dpa, dpl, dpd, (uint32_t)pa.size(), (uint64_t*)d); }, nm, (double)total);
            snprintf(nm, sizeof nm, "TMA gather 2 slots/warp avg %dB grid=%d", avg_bytes, grid);
            timeit([&] { tma_gather2<4096><<<grid, 256, 16 * (4096 + 32)>>>(hd, dpa, dpl, dpd, (uint32_t)pa.size(), (uint64_t*)d); }, nm, (double)total);
        }
        cudaFree(dpa); cudaFree(dpd); cudaFree(dpl);
    }
    return 0;
}
