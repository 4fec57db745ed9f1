// zc_align.cu — zero-copy gather of random host runs: load width x start alignment (dev tool).
//   mode 0: 16 B loads, runs start 16 B aligned (lengths multiple of 16)
//   mode 1: 4 B loads, lane = consecutive word (a warp instruction covers 128 B), 16 B-aligned starts
//   mode 2: 4 B loads, 4 B-aligned starts (what k_gather<4> does inside one run)
//   mode 3: 16 B loads of the 16 B-aligned cover of a 4 B-aligned run, words outside dropped
//   mode 4: 8 B loads, 8 B-aligned starts (k_gather<8>)
// Host array 4 GB (cudaHostAlloc, mapped); 512 MB moved per measurement; one warp per run.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o zc_align tools/zc_align.cu
#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <random>
#include <vector>

#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); exit(1);} } while (0)

template <int MODE>
__global__ void __launch_bounds__(256) gather(const char* __restrict__ host, const uint64_t* __restrict__ start,
                                              uint32_t len, uint32_t nruns, char* __restrict__ dst) {
    const int lane = threadIdx.x & 31;
    const uint32_t nw = (gridDim.x * blockDim.x) >> 5;
    for (uint32_t r = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; r < nruns; r += nw) {
        const uint64_t s = start[r];
        char* d = dst + (uint64_t)r * len;
        if (MODE == 0) {
            const uint4* src = reinterpret_cast<const uint4*>(host + s);
            uint4* o = reinterpret_cast<uint4*>(d);
            const uint32_t n = len / 16;
            for (uint32_t b = 0; b < n; b += 256) {
                uint4 v[8];
#pragma unroll
                for (int j = 0; j < 8; ++j) if (b + j * 32 + lane < n) v[j] = src[b + j * 32 + lane];
#pragma unroll
                for (int j = 0; j < 8; ++j) if (b + j * 32 + lane < n) o[b + j * 32 + lane] = v[j];
            }
        } else if (MODE == 1 || MODE == 2) {
            const uint32_t* src = reinterpret_cast<const uint32_t*>(host + s);
            uint32_t* o = reinterpret_cast<uint32_t*>(d);
            const uint32_t n = len / 4;
            for (uint32_t b = 0; b < n; b += 256) {
                uint32_t v[8];
#pragma unroll
                for (int j = 0; j < 8; ++j) if (b + j * 32 + lane < n) v[j] = src[b + j * 32 + lane];
#pragma unroll
                for (int j = 0; j < 8; ++j) if (b + j * 32 + lane < n) o[b + j * 32 + lane] = v[j];
            }
        } else if (MODE == 4) {
            const uint2* src = reinterpret_cast<const uint2*>(host + s);
            uint2* o = reinterpret_cast<uint2*>(d);
            const uint32_t n = len / 8;
            for (uint32_t b = 0; b < n; b += 256) {
                uint2 v[8];
#pragma unroll
                for (int j = 0; j < 8; ++j) if (b + j * 32 + lane < n) v[j] = src[b + j * 32 + lane];
#pragma unroll
                for (int j = 0; j < 8; ++j) if (b + j * 32 + lane < n) o[b + j * 32 + lane] = v[j];
            }
        } else {   // MODE 3: aligned 16 B cover, scalar stores of the words inside [s, s + len)
            const uint64_t a0 = s & ~15ull, a1 = (s + len + 15) & ~15ull;
            const uint4* src = reinterpret_cast<const uint4*>(host + a0);
            uint32_t* o = reinterpret_cast<uint32_t*>(d);
            const uint32_t n = (uint32_t)((a1 - a0) / 16);
            const int64_t shift = (int64_t)(s - a0) / 4;   // words before the run in the first unit
            const int64_t nwords = len / 4;
            for (uint32_t b = 0; b < n; b += 256) {
                uint4 v[8];
#pragma unroll
                for (int j = 0; j < 8; ++j) if (b + j * 32 + lane < n) v[j] = src[b + j * 32 + lane];
#pragma unroll
                for (int j = 0; j < 8; ++j) {
                    const int64_t u = b + j * 32 + lane;
                    if (u >= n) continue;
                    const int64_t w0 = u * 4 - shift;
                    const uint32_t x[4] = {v[j].x, v[j].y, v[j].z, v[j].w};
#pragma unroll
                    for (int q = 0; q < 4; ++q)
                        if (w0 + q >= 0 && w0 + q < nwords) o[w0 + q] = x[q];
                }
            }
        }
    }
}

int main() {
    const size_t S = 4ull << 30, moved = 512ull << 20;
    void* h = nullptr;
    CK(cudaHostAlloc(&h, S, cudaHostAllocMapped | cudaHostAllocPortable));
    memset(h, 1, S);
    char* hd = nullptr;
    CK(cudaHostGetDevicePointer((void**)&hd, h, 0));
    char* d = nullptr;
    CK(cudaMalloc(&d, moved + (1 << 20)));
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    const uint32_t lens[] = {64, 256, 1024, 4096, 65536};
    const char* names[] = {"16B ld, 16B-aligned", "4B ld, 16B-aligned", "4B ld, 4B-aligned", "16B cover, 4B-aligned",
                           "8B ld, 8B-aligned"};
    for (uint32_t L : lens) {
        const uint32_t nruns = (uint32_t)(moved / L);
        for (int mode = 0; mode < 5; ++mode) {
            const uint64_t al = (mode == 0 || mode == 1) ? 16 : (mode == 4 ? 8 : 4);
            std::vector<uint64_t> st(nruns);
            std::mt19937_64 rng(L * 7 + mode);
            for (auto& x : st) x = (rng() % ((S - L - 64) / al)) * al;
            uint64_t* dst_ = nullptr;
            CK(cudaMalloc(&dst_, nruns * 8ull));
            CK(cudaMemcpy(dst_, st.data(), nruns * 8ull, cudaMemcpyHostToDevice));
            for (int grid : {64, 148, 296}) {
                float best = 1e30f;
                for (int rep = 0; rep < 3; ++rep) {
                    cudaEventRecord(e0);
                    switch (mode) {
                        case 0: gather<0><<<grid, 256>>>(hd, dst_, L, nruns, d); break;
                        case 1: gather<1><<<grid, 256>>>(hd, dst_, L, nruns, d); break;
                        case 2: gather<2><<<grid, 256>>>(hd, dst_, L, nruns, d); break;
                        case 3: gather<3><<<grid, 256>>>(hd, dst_, L, nruns, d); break;
                        default: gather<4><<<grid, 256>>>(hd, dst_, L, nruns, d); break;
                    }
                    cudaEventRecord(e1);
                    CK(cudaEventSynchronize(e1));
                    float ms;
                    cudaEventElapsedTime(&ms, e0, e1);
                    best = std::min(best, ms);
                }
                printf("L=%6u %-24s grid=%3d : %6.2f GB/s payload\n", L, names[mode], grid, moved / best / 1e6);
            }
            cudaFree(dst_);
        }
    }
    return 0;
}
