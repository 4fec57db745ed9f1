// zc_gran.cu — cost model of SM zero-copy reads over PCIe (dev tool): which unit does the link
// charge for, the warp instruction, the 128-byte line, the 32-byte sector, or the byte?
//
// Every warp load instruction reads 32 x 16 B = 512 B as K = 512 / P pieces of P bytes, each piece
// at an independent random position aligned to A bytes. 8 instructions per lane are issued before
// the stores (like k_gather16). Host array 4 GB (cudaHostAlloc, mapped); 1 GB moved per point.
//   P = 512, A = 512 : 4 full lines per instruction (random 512 B blocks)
//   P = 128, A = 128 : 4 random full lines
//   P = 64,  A = 64  : 8 random half lines
//   P = 32,  A = 32  : 16 random sectors
//   P = 16,  A = 16  : 32 random 16 B units
//   P = 128, A = 16  : 4 random 128 B pieces, most straddling two lines
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/zc_gran tools/zc_gran.cu
#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <random>
#include <vector>

#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); exit(1);} } while (0)

__device__ __forceinline__ uint4 ld_host16(const uint4* p) {
    uint4 x;
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(x.x), "=r"(x.y), "=r"(x.z), "=r"(x.w) : "l"(p));
    return x;
}

// starts[i] = byte offset of piece i; a lane's unit = (piece l / U, unit l % U), U = P / 16
__global__ void __launch_bounds__(256) rd(const char* __restrict__ host, const uint64_t* __restrict__ starts,
                                          uint32_t P, uint64_t ninstr, uint4* __restrict__ dst) {
    const int lane = threadIdx.x & 31;
    const uint32_t U = P / 16, K = 32 / U;
    const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    const uint64_t w0 = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    for (uint64_t i0 = w0 * 8; i0 < ninstr; i0 += nw * 8) {
        uint4 v[8];
#pragma unroll
        for (int j = 0; j < 8; ++j) {
            const uint64_t ins = i0 + j;
            if (ins < ninstr) {
                const uint64_t s = starts[ins * K + lane / U] + 16ull * (lane % U);
                v[j] = ld_host16(reinterpret_cast<const uint4*>(host + s));
            }
        }
#pragma unroll
        for (int j = 0; j < 8; ++j)
            if (i0 + j < ninstr) dst[((i0 + j) * 32 + lane) & ((1u << 22) - 1)] = v[j];
    }
}

int main() {
    const size_t S = 4ull << 30, moved = 1ull << 30;
    void* h = nullptr;
    CK(cudaHostAlloc(&h, S, cudaHostAllocMapped | cudaHostAllocPortable));
    memset(h, 1, S);
    char* hd = nullptr;
    CK(cudaHostGetDevicePointer((void**)&hd, h, 0));
    uint4* d = nullptr;
    CK(cudaMalloc(&d, (1u << 22) * 16ull));
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    struct Pt { uint32_t P, A; };
    const Pt pts[] = {{512, 512}, {512, 16}, {256, 256}, {256, 16}, {128, 128}, {128, 16}, {64, 64}, {64, 16},
                      {32, 32}, {16, 16}};
    const uint64_t ninstr = moved / 512;
    for (const Pt& p : pts) {
        const uint64_t npieces = ninstr * (512 / p.P);
        std::vector<uint64_t> st(npieces);
        std::mt19937_64 rng(p.P * 131 + p.A);
        for (auto& x : st) x = (rng() % ((S - 1024) / p.A)) * p.A;
        uint64_t* ds = nullptr;
        CK(cudaMalloc(&ds, npieces * 8ull));
        CK(cudaMemcpy(ds, st.data(), npieces * 8ull, cudaMemcpyHostToDevice));
        for (int grid : {64, 148, 296, 592}) {
            float best = 1e30f;
            for (int rep = 0; rep < 3; ++rep) {
                cudaEventRecord(e0);
                rd<<<grid, 256>>>(hd, ds, p.P, ninstr, d);
                cudaEventRecord(e1);
                CK(cudaEventSynchronize(e1));
                float ms;
                cudaEventElapsedTime(&ms, e0, e1);
                best = std::min(best, ms);
            }
            const double s = best / 1e3;
            // lines touched per piece: 1 if aligned inside a line, else ceil over the straddle
            printf("P=%4u A=%4u grid=%3d : %6.2f GB/s useful  %7.1f M pieces/s  %7.1f M instr/s\n", p.P, p.A, grid,
                   moved / s / 1e9, npieces / s / 1e6, ninstr / s / 1e6);
        }
        cudaFree(ds);
    }
    return 0;
}
