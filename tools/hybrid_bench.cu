// hybrid_bench.cu — dev tool: does host-thread gather + copy-engine DMA, running concurrently
// with the SM zero-copy gather, raise payload throughput over PCIe above zero-copy alone?
// Workload: random ascending runs of ~1.1 KB (8-byte arcs), like C2's dense iterations.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/hybrid_bench tools/hybrid_bench.cu -lpthread
#include <algorithm>
#include <atomic>
#include <chrono>
#include <cstdint>
#include <cstdio>
#include <cstring>
#include <random>
#include <thread>
#include <vector>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); exit(1);} } while (0)

__global__ void zc_gather8(const uint64_t* __restrict__ src, const uint64_t* __restrict__ rstart,
                           const uint64_t* __restrict__ rpre, uint32_t nruns, uint64_t* __restrict__ dst, uint64_t total) {
    // warp-cooperative: 8 groups of 32 arcs per warp, loads first (like k_gather)
    const int lane = threadIdx.x & 31;
    const uint64_t nwarps = (uint64_t)gridDim.x * blockDim.x / 32;
    for (uint64_t w = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) / 32; w * 256 < total; w += nwarps) {
        uint64_t from[8];
        for (int g = 0; g < 8; ++g) {
            uint64_t p = w * 256 + g * 32 + lane;
            if (p >= total) { from[g] = ~0ull; continue; }
            uint32_t lo = 0, hi = nruns;
            while (hi - lo > 1) { uint32_t mid = (lo + hi) >> 1; if (rpre[mid] <= p) lo = mid; else hi = mid; }
            from[g] = rstart[lo] + (p - rpre[lo]);
        }
        uint64_t v[8];
        for (int g = 0; g < 8; ++g) if (from[g] != ~0ull) v[g] = src[from[g]];
        for (int g = 0; g < 8; ++g) if (from[g] != ~0ull) dst[w * 256 + g * 32 + lane] = v[g];
    }
}

int main() {
    const size_t host_bytes = 8ull << 30;
    uint64_t* h; CK(cudaHostAlloc((void**)&h, host_bytes, cudaHostAllocMapped | cudaHostAllocPortable));
    for (size_t i = 0; i < host_bytes / 8; i += 512) h[i] = i;
    uint64_t* hd; CK(cudaHostGetDevicePointer((void**)&hd, h, 0));
    const uint64_t nel = host_bytes / 8;
    std::mt19937_64 rng(7);
    std::vector<uint64_t> rs, rp;
    const uint64_t want = (2048ull << 20) / 8;   // 2 GiB payload
    uint64_t total = 0, pos = 0;
    const uint64_t gap_avg = (nel - want) / (want / 138);
    while (total < want) {
        uint64_t len = 1 + rng() % 275;            // ~138 arcs = 1.1 KB average
        pos += rng() % (2 * gap_avg + 1);
        if (pos + len >= nel) break;
        rs.push_back(pos); rp.push_back(total); total += len; pos += len;
    }
    printf("runs=%zu payload=%.2f GB avg run=%.0f B\n", rs.size(), total * 8 / 1e9, total * 8.0 / rs.size());
    uint64_t *drs, *drp, *d;
    CK(cudaMalloc(&drs, rs.size() * 8)); CK(cudaMalloc(&drp, rp.size() * 8));
    CK(cudaMemcpy(drs, rs.data(), rs.size() * 8, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(drp, rp.data(), rp.size() * 8, cudaMemcpyHostToDevice));
    CK(cudaMalloc(&d, total * 8));
    cudaStream_t sz, sd; CK(cudaStreamCreateWithFlags(&sz, cudaStreamNonBlocking)); CK(cudaStreamCreateWithFlags(&sd, cudaStreamNonBlocking));
    const size_t stage_bytes = 32ull << 20;
    const int nstage = 4;
    uint64_t* stage[nstage];
    for (int i = 0; i < nstage; ++i) CK(cudaHostAlloc((void**)&stage[i], stage_bytes, cudaHostAllocPortable));

    for (double f : {0.0, 0.2, 0.3, 0.4, 0.5, 1.0}) {
        for (int nthreads : {8, 12}) {
            if (f == 0.0 && nthreads != 8) continue;
            // split: first (1-f) of runs by zero-copy kernel, the rest by CPU gather + DMA
            size_t split = (size_t)((1.0 - f) * rs.size());
            uint64_t zc_total = split < rs.size() ? rp[split] : total;
            CK(cudaDeviceSynchronize());
            auto t0 = std::chrono::steady_clock::now();
            if (zc_total) zc_gather8<<<64, 256, 0, sz>>>(hd, drs, drp, (uint32_t)std::min(split, rs.size()), d, zc_total);
            // CPU path: pieces of stage_bytes, threads gather, main issues DMA
            size_t r = split;
            uint64_t out = zc_total;
            int si = 0;
            std::vector<cudaEvent_t> done(nstage);
            for (auto& ev : done) CK(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
            std::vector<bool> used(nstage, false);
            while (r < rs.size()) {
                size_t r0 = r; uint64_t bytes = 0;
                while (r < rs.size()) {
                    uint64_t len = (r + 1 < rs.size() ? rp[r + 1] : total) - rp[r];
                    if (bytes + len * 8 > stage_bytes && r > r0) break;
                    bytes += len * 8; ++r;
                }
                if (used[si]) CK(cudaEventSynchronize(done[si]));
                uint64_t* st = stage[si];
                std::vector<std::thread> th;
                for (int t = 0; t < nthreads; ++t)
                    th.emplace_back([&, t] {
                        size_t a = r0 + (r - r0) * t / nthreads, b = r0 + (r - r0) * (t + 1) / nthreads;
                        for (size_t q = a; q < b; ++q) {
                            uint64_t len = (q + 1 < rs.size() ? rp[q + 1] : total) - rp[q];
                            memcpy(st + (rp[q] - rp[r0]), h + rs[q], len * 8);
                        }
                    });
                for (auto& x : th) x.join();
                CK(cudaMemcpyAsync(d + out, st, bytes, cudaMemcpyHostToDevice, sd));
                CK(cudaEventRecord(done[si], sd));
                used[si] = true;
                out += bytes / 8;
                si = (si + 1) % nstage;
            }
            CK(cudaDeviceSynchronize());
            double s = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
            printf("cpu_fraction=%.1f threads=%2d  payload %.2f GB in %.1f ms = %.2f GB/s\n", f, nthreads, total * 8 / 1e9,
                   s * 1e3, total * 8 / s / 1e9);
            for (auto& e : done) cudaEventDestroy(e);
        }
    }
    return 0;
}
