// zc_bench.cu — host-link microbenchmarks on the B200 box (dev tool, not the product):
// pinned H2D DMA vs SM zero-copy reads of mapped pinned memory, contiguous and gathered.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o zc_bench tools/zc_bench.cu
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <vector>
#include <algorithm>
#include <random>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); exit(1);} } while (0)

template <int V, int HINT>
__global__ void zc_copy(const uint4* __restrict__ src, uint4* __restrict__ dst, size_t n16) {
    size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
    size_t stride = (size_t)gridDim.x * blockDim.x;
    if (V == 16) {
        for (; i < n16; i += stride) {
            uint4 x;
            if (HINT == 1) asm volatile("ld.global.nc.L1::no_allocate.L2::256B.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(x.x), "=r"(x.y), "=r"(x.z), "=r"(x.w) : "l"(src + i));
            else if (HINT == 2) asm volatile("ld.global.nc.L1::no_allocate.L2::128B.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(x.x), "=r"(x.y), "=r"(x.z), "=r"(x.w) : "l"(src + i));
            else x = src[i];
            dst[i] = x;
        }
    } else {
        const uint32_t* s = (const uint32_t*)src;
        uint32_t* d = (uint32_t*)dst;
        size_t n4 = n16 * 4;
        for (; i < n4; i += stride) {
            uint32_t x;
            if (HINT == 1) asm volatile("ld.global.nc.L1::no_allocate.L2::256B.u32 %0, [%1];" : "=r"(x) : "l"(s + i));
            else x = s[i];
            d[i] = x;
        }
    }
}

// unrolled: each thread issues U independent 16B loads before storing
template <int U>
__global__ void zc_copy_unroll(const uint4* __restrict__ src, uint4* __restrict__ dst, size_t n16) {
    size_t base = (size_t)blockIdx.x * blockDim.x * U + threadIdx.x;
    size_t stride = (size_t)gridDim.x * blockDim.x * U;
    for (; base < n16; base += stride) {
        uint4 x[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            size_t i = base + (size_t)u * blockDim.x;
            if (i < n16) x[u] = src[i];
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
            size_t i = base + (size_t)u * blockDim.x;
            if (i < n16) dst[i] = x[u];
        }
    }
}

// gather: runs (start, len) in 8-byte units, prefix dst; thread per output element
__global__ void zc_gather8(const uint64_t* __restrict__ src, const uint64_t* __restrict__ rstart,
                           const uint64_t* __restrict__ rpre, uint32_t nruns, uint64_t* __restrict__ dst, uint64_t total) {
    uint64_t p = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (; p < total; p += stride) {
        uint32_t lo = 0, hi = nruns;
        while (hi - lo > 1) { uint32_t mid = (lo + hi) >> 1; if (rpre[mid] <= p) lo = mid; else hi = mid; }
        dst[p] = src[rstart[lo] + (p - rpre[lo])];
    }
}

int main() {
    const size_t bytes = 512ull << 20;
    void* h; CK(cudaHostAlloc(&h, bytes, cudaHostAllocMapped | cudaHostAllocPortable));
    memset(h, 1, bytes);
    void* d; CK(cudaMalloc(&d, bytes));
    void* hd; CK(cudaHostGetDevicePointer(&hd, h, 0));
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    auto timeit = [&](auto fn, const char* name, double nbytes) {
        fn(); CK(cudaDeviceSynchronize());
        float best = 1e9;
        for (int r = 0; r < 5; ++r) {
            cudaEventRecord(e0); fn(); cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
            float ms; cudaEventElapsedTime(&ms, e0, e1); best = std::min(best, ms);
        }
        printf("%-48s %8.2f GB/s  (%.3f ms)\n", name, nbytes / (best / 1e3) / 1e9, best);
    };
    timeit([&] { cudaMemcpyAsync(d, h, bytes, cudaMemcpyHostToDevice); }, "DMA cudaMemcpyAsync 512MiB", bytes);
    const size_t n16 = bytes / 16;
    for (int grid : {148, 296, 592, 1184, 2368}) {
        char nm[96];
        snprintf(nm, sizeof nm, "zc 4B  grid=%d", grid);
        timeit([&] { zc_copy<4, 0><<<grid, 256>>>((const uint4*)hd, (uint4*)d, n16); }, nm, bytes);
        snprintf(nm, sizeof nm, "zc 16B grid=%d", grid);
        timeit([&] { zc_copy<16, 0><<<grid, 256>>>((const uint4*)hd, (uint4*)d, n16); }, nm, bytes);
        snprintf(nm, sizeof nm, "zc 16B L2::256B grid=%d", grid);
        timeit([&] { zc_copy<16, 1><<<grid, 256>>>((const uint4*)hd, (uint4*)d, n16); }, nm, bytes);
        snprintf(nm, sizeof nm, "zc 16B x4 unroll grid=%d", grid);
        timeit([&] { zc_copy_unroll<4><<<grid, 256>>>((const uint4*)hd, (uint4*)d, n16); }, nm, bytes);
    }
    // gather of short runs (lists of ~avg arcs of 8 B) from random positions
    for (int avg : {3, 6, 24, 96, 1024}) {
        std::mt19937_64 rng(avg);
        const uint64_t nel = bytes / 8;
        std::vector<uint64_t> rs, rp;
        uint64_t total = 0;
        const uint64_t want = 128ull << 20 >> 3;   // 128 MiB of gathered payload
        while (total < want) {
            uint64_t len = 1 + rng() % (2 * avg - 1);
            uint64_t st = rng() % (nel - len);
            rs.push_back(st); rp.push_back(total); total += len;
        }
        uint64_t *drs, *drp;
        CK(cudaMalloc(&drs, rs.size() * 8)); CK(cudaMalloc(&drp, rp.size() * 8));
        CK(cudaMemcpy(drs, rs.data(), rs.size() * 8, cudaMemcpyHostToDevice));
        CK(cudaMemcpy(drp, rp.data(), rp.size() * 8, cudaMemcpyHostToDevice));
        char nm[96];
        snprintf(nm, sizeof nm, "zc gather 8B runs avg=%d arcs (%zu runs)", avg, rs.size());
        timeit([&] { zc_gather8<<<2368, 256>>>((const uint64_t*)hd, drs, drp, (uint32_t)rs.size(), (uint64_t*)d, total); }, nm, total * 8.0);
        cudaFree(drs); cudaFree(drp);
    }
    return 0;
}
