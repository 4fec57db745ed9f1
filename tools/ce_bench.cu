// ce_bench.cu — copy-engine H2D of scattered host runs (dev tool): one cudaMemcpyAsync per run from
// a 4 GB pinned host array at random 4-byte-aligned offsets into a device buffer, round-robin over
// S streams, 2 GiB per point. Tells at which run size the copy engines beat the SM gather (45-50 GB/s)
// and whether more streams (copy engines) hide the per-copy overhead.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ce_bench tools/ce_bench.cu
#include <algorithm>
#include <chrono>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <random>
#include <vector>

#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); exit(1);} } while (0)

int main() {
    const size_t S = 4ull << 30, moved = 2ull << 30;
    int ae = 0;
    CK(cudaDeviceGetAttribute(&ae, cudaDevAttrAsyncEngineCount, 0));
    printf("asyncEngineCount = %d\n", ae);
    char* h = nullptr;
    CK(cudaHostAlloc((void**)&h, S, cudaHostAllocPortable));
    memset(h, 1, S);
    char* d = nullptr;
    CK(cudaMalloc(&d, moved + (64 << 20)));
    std::vector<cudaStream_t> st(16);
    for (auto& s : st) CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    for (size_t L : {16ull << 10, 64ull << 10, 128ull << 10, 256ull << 10, 1ull << 20, 4ull << 20, 64ull << 20}) {
        const size_t n = moved / L;
        std::vector<size_t> off(n);
        std::mt19937_64 rng(L);
        for (auto& x : off) x = (rng() % ((S - L) / 4)) * 4;
        for (int ns : {1, 2, 4, 8, 16}) {
            double best = 1e30, host_us = 0;
            for (int rep = 0; rep < 2; ++rep) {
                CK(cudaDeviceSynchronize());
                CK(cudaEventRecord(e0, st[0]));
                for (int k = 1; k < ns; ++k) CK(cudaStreamWaitEvent(st[k], e0, 0));
                const auto t0 = std::chrono::steady_clock::now();
                for (size_t i = 0; i < n; ++i)
                    CK(cudaMemcpyAsync(d + i * L, h + off[i], L, cudaMemcpyHostToDevice, st[i % ns]));
                const auto t1 = std::chrono::steady_clock::now();
                for (int k = 1; k < ns; ++k) {
                    cudaEvent_t ek;
                    CK(cudaEventCreateWithFlags(&ek, cudaEventDisableTiming));
                    CK(cudaEventRecord(ek, st[k]));
                    CK(cudaStreamWaitEvent(st[0], ek, 0));
                    cudaEventDestroy(ek);
                }
                CK(cudaEventRecord(e1, st[0]));
                CK(cudaEventSynchronize(e1));
                float ms;
                cudaEventElapsedTime(&ms, e0, e1);
                if (ms < best) { best = ms; host_us = std::chrono::duration<double, std::micro>(t1 - t0).count() / n; }
            }
            printf("run %8zu B  streams %2d : %6.2f GB/s  (%6.2f us per copy on the device, %5.2f us host enqueue)\n", L, ns,
                   moved / (best / 1e3) / 1e9, best * 1e3 / n, host_us);
        }
    }
    return 0;
}
