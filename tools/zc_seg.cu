// zc_seg.cu — zero-copy gather of long host runs cut into per-warp segments (dev tool): does the
// segment length, or where the segment boundaries fall relative to 512-byte host blocks, change the
// rate? k_gather16 gives each warp 256 stream arcs (1 KB at 4-byte arcs, 2 KB at 8-byte arcs), so a
// long run is read as consecutive warp segments whose boundaries sit at arbitrary host offsets.
//   mode 0: segments of SEG bytes at stream offsets (host boundaries at the run's random alignment)
//   mode 1: segment boundaries moved to the next 512-byte host block boundary (first segment shorter)
//   mode 2: segments at stream offsets, but each warp load of a segment covers one 512-byte host block
//           (the segment's first load starts at its block, lanes before the segment idle): k_gather16
//           since the long-piece alignment
// One warp per segment, 16-byte cover loads, NG units in flight per lane, each lane stores its words.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o tools/zc_seg tools/zc_seg.cu
#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <random>
#include <vector>

#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e_)); exit(1);} } while (0)

// segment i: host bytes [ha[i], hb[i]) (16-byte multiples), stream offset d[i]
template <bool ALIGN>
__global__ void __launch_bounds__(256) seg_gather(const uint4* __restrict__ host, const uint64_t* __restrict__ ha,
                                                  const uint64_t* __restrict__ hb, const uint64_t* __restrict__ dd,
                                                  uint32_t nseg, uint4* __restrict__ dst) {
    const int lane = threadIdx.x & 31;
    const uint32_t nw = gridDim.x * 8;
    for (uint32_t i = blockIdx.x * 8 + (threadIdx.x >> 5); i < nseg; i += nw) {
        const uint64_t u0 = ha[i] >> 4, u1 = hb[i] >> 4;
        uint4* d = dst + (dd[i] >> 4);
        for (uint64_t u = ALIGN ? (u0 & ~31ull) : u0; u < u1; u += 32 * 6) {
            uint4 v[6];
#pragma unroll
            for (int g = 0; g < 6; ++g) {
                const uint64_t uu = u + 32 * g + lane;
                if (uu >= u0 && uu < u1) v[g] = host[uu];
            }
#pragma unroll
            for (int g = 0; g < 6; ++g) {
                const uint64_t uu = u + 32 * g + lane;
                if (uu >= u0 && uu < u1) d[uu - u0] = v[g];
            }
        }
    }
}

int main() {
    const size_t bytes = 4ull << 30;
    char* h;
    CK(cudaHostAlloc((void**)&h, bytes, cudaHostAllocMapped | cudaHostAllocPortable));
    memset(h, 1, bytes);
    char* hd;
    CK(cudaHostGetDevicePointer((void**)&hd, h, 0));
    const size_t want = 512ull << 20;
    uint4* dst;
    CK(cudaMalloc(&dst, want + (1 << 20)));
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    for (uint64_t run : {(uint64_t)4096, (uint64_t)16384, (uint64_t)65536}) {
        for (uint64_t seg : {(uint64_t)1024, (uint64_t)2048, (uint64_t)4096, (uint64_t)8192, (uint64_t)1 << 30}) {
            for (int mode : {0, 1, 2}) {
                if (seg >= run && mode >= 1) continue;
                std::mt19937_64 rng(run * 7 + seg);
                std::vector<uint64_t> ha, hb, dd;
                uint64_t total = 0;
                while (total < want) {
                    const uint64_t a = 16 * (rng() % ((bytes - run) / 16));
                    const uint64_t b = a + run;
                    uint64_t p = a;
                    while (p < b) {
                        uint64_t q = std::min<uint64_t>(b, p + seg);
                        if (mode == 1 && q < b) q = std::max<uint64_t>(p + 16, q & ~511ull);   // end at a 512 B host block
                        ha.push_back(p); hb.push_back(q); dd.push_back(total + (p - a));
                        p = q;
                    }
                    total += run;
                }
                uint64_t *dha, *dhb, *ddd;
                CK(cudaMalloc(&dha, ha.size() * 8)); CK(cudaMalloc(&dhb, hb.size() * 8)); CK(cudaMalloc(&ddd, dd.size() * 8));
                CK(cudaMemcpy(dha, ha.data(), ha.size() * 8, cudaMemcpyHostToDevice));
                CK(cudaMemcpy(dhb, hb.data(), hb.size() * 8, cudaMemcpyHostToDevice));
                CK(cudaMemcpy(ddd, dd.data(), dd.size() * 8, cudaMemcpyHostToDevice));
                float best = 1e9;
                for (int r = 0; r < 4; ++r) {
                    cudaEventRecord(e0);
                    if (mode == 2) seg_gather<true><<<64, 256>>>((const uint4*)hd, dha, dhb, ddd, (uint32_t)ha.size(), dst);
                    else seg_gather<false><<<64, 256>>>((const uint4*)hd, dha, dhb, ddd, (uint32_t)ha.size(), dst);
                    cudaEventRecord(e1);
                    CK(cudaEventSynchronize(e1));
                    float ms; cudaEventElapsedTime(&ms, e0, e1);
                    if (r) best = std::min(best, ms);
                }
                CK(cudaGetLastError());
                printf("run %6llu B  seg %10llu B  %s  %zu segments  %6.2f GB/s\n", (unsigned long long)run,
                       (unsigned long long)seg, mode == 1 ? "512B-aligned ends      " : mode == 2 ? "stream offs, loads alnd" : "stream offsets         ", ha.size(),
                       total / (best / 1e3) / 1e9);
                cudaFree(dha); cudaFree(dhb); cudaFree(ddd);
            }
        }
    }
    return 0;
}
