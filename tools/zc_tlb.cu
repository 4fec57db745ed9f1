// zc_tlb.cu — does the size / page backing of the pinned host array change SM zero-copy read
// rates? (dev tool, not the product). Reads runs of L bytes at random 16-byte-aligned offsets
// of a host array of S bytes (S = 0.5 GB vs 24 GB), backed by cudaHostAlloc, malloc +
// cudaHostRegister, or malloc + madvise(MADV_HUGEPAGE) + cudaHostRegister; plus copy-engine DMA
// of the same runs.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o zc_tlb tools/zc_tlb.cu
#include <sys/mman.h>

#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <random>
#include <vector>

#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); exit(1);} } while (0)

// one warp per run (grid-stride over runs); 8 x 16 B loads per lane in flight
__global__ void __launch_bounds__(256) gather_runs(const uint4* __restrict__ host, const uint64_t* __restrict__ start16,
                                                   uint32_t len16, uint32_t nruns, uint4* __restrict__ dst) {
    const int lane = threadIdx.x & 31;
    const uint32_t nw = (gridDim.x * blockDim.x) >> 5;
    for (uint32_t r = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; r < nruns; r += nw) {
        const uint4* s = host + start16[r];
        uint4* d = dst + (uint64_t)r * len16;
        for (uint32_t b = 0; b < len16; b += 256) {
            uint4 v[8];
#pragma unroll
            for (int j = 0; j < 8; ++j) {
                const uint32_t i = b + j * 32 + lane;
                if (i < len16) v[j] = s[i];
            }
#pragma unroll
            for (int j = 0; j < 8; ++j) {
                const uint32_t i = b + j * 32 + lane;
                if (i < len16) d[i] = v[j];
            }
        }
    }
}

static float time_ms(cudaEvent_t a, cudaEvent_t b) { float x; cudaEventElapsedTime(&x, a, b); return x; }

int main() {
    const size_t sizes[] = {512ull << 20, 24ull << 30};
    const uint32_t lens[] = {1024, 16384, 262144};
    const size_t moved = 512ull << 20;   // bytes per measurement
    uint4* d = nullptr;
    CK(cudaMalloc(&d, moved));
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    cudaStream_t st;
    cudaStreamCreate(&st);
    for (int backing = 0; backing < 3; ++backing) {
        for (size_t S : sizes) {
            void* h = nullptr;
            if (backing == 0) {
                CK(cudaHostAlloc(&h, S, cudaHostAllocMapped | cudaHostAllocPortable));
            } else {
                h = aligned_alloc(2u << 20, S);
                if (backing == 2) madvise(h, S, MADV_HUGEPAGE);
                memset(h, 1, S);
                CK(cudaHostRegister(h, S, cudaHostRegisterMapped | cudaHostRegisterPortable));
            }
            if (backing == 0) memset(h, 1, S);
            void* hd = nullptr;
            CK(cudaHostGetDevicePointer(&hd, h, 0));
            const char* bn[] = {"cudaHostAlloc", "malloc+register", "malloc+THP+register"};
            for (uint32_t L : lens) {
                const uint32_t nruns = (uint32_t)(moved / L);
                std::vector<uint64_t> st16(nruns);
                std::mt19937_64 rng(L + S);
                for (auto& x : st16) x = (rng() % ((S - L) / 16));
                uint64_t* dst16 = nullptr;
                CK(cudaMalloc(&dst16, nruns * 8ull));
                CK(cudaMemcpy(dst16, st16.data(), nruns * 8ull, cudaMemcpyHostToDevice));
                for (int grid : {64, 148}) {
                    float best = 1e30f;
                    for (int rep = 0; rep < 3; ++rep) {
                        cudaEventRecord(e0, st);
                        gather_runs<<<grid, 256, 0, st>>>((const uint4*)hd, dst16, L / 16, nruns, d);
                        cudaEventRecord(e1, st);
                        CK(cudaEventSynchronize(e1));
                        best = std::min(best, time_ms(e0, e1));
                    }
                    printf("%-22s S=%6.1f GB L=%7u SM-gather grid=%3d : %6.2f GB/s\n", bn[backing], S / 1e9, L, grid,
                           moved / best / 1e6);
                }
                {   // copy engine, one cudaMemcpyAsync per run (L >= 16 KiB only)
                    if (L >= 16384) {
                        float best = 1e30f;
                        for (int rep = 0; rep < 2; ++rep) {
                            cudaEventRecord(e0, st);
                            for (uint32_t r = 0; r < nruns; ++r)
                                cudaMemcpyAsync((char*)d + (size_t)r * L, (const char*)h + st16[r] * 16, L,
                                                cudaMemcpyHostToDevice, st);
                            cudaEventRecord(e1, st);
                            CK(cudaEventSynchronize(e1));
                            best = std::min(best, time_ms(e0, e1));
                        }
                        printf("%-22s S=%6.1f GB L=%7u DMA per run        : %6.2f GB/s\n", bn[backing], S / 1e9, L,
                               moved / best / 1e6);
                    }
                }
                cudaFree(dst16);
            }
            if (backing == 0) cudaFreeHost(h);
            else { cudaHostUnregister(h); free(h); }
        }
    }
    return 0;
}
