// reg_bench.cu — can page-locking a large pageable edge array be split across host threads, and do
// copy-engine DMAs and SM zero-copy reads still run at full rate across the split points? (dev tool)
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o tools/reg_bench tools/reg_bench.cu -lpthread
#include <chrono>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <thread>
#include <vector>

#include <cuda_runtime.h>
#include <sys/mman.h>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e_)); exit(1);} } while (0)

static double now() { return std::chrono::duration<double>(std::chrono::steady_clock::now().time_since_epoch()).count(); }

__global__ void zc_read(const uint4* __restrict__ src, uint4* __restrict__ dst, size_t n) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) dst[i] = src[i];
}

int main(int argc, char** argv) {
    const size_t gib = 1ull << 30;
    const size_t bytes = (argc > 1 ? atoll(argv[1]) : 24) * gib;
    int can = 0;
    CK(cudaDeviceGetAttribute(&can, cudaDevAttrCanUseHostPointerForRegisteredMem, 0));
    printf("canUseHostPointerForRegisteredMem = %d\n", can);
    char* h = (char*)mmap(nullptr, bytes, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
    if (h == MAP_FAILED) { printf("mmap failed\n"); return 1; }
    {   // touch (first-touch in parallel)
        std::vector<std::thread> th;
        for (int t = 0; t < 16; ++t)
            th.emplace_back([=] { for (size_t o = t * (bytes / 16); o < (t + 1) * (bytes / 16); o += 4096) h[o] = (char)o; });
        for (auto& x : th) x.join();
    }
    char* d;
    CK(cudaMalloc(&d, 2 * gib));
    cudaStream_t s; CK(cudaStreamCreate(&s));
    cudaEvent_t e0, e1; CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
    for (int nt : {1, 2, 4, 8, 16}) {
        const size_t piece = (bytes / nt + 4095) / 4096 * 4096;
        double t0 = now();
        std::vector<std::thread> th;
        std::vector<cudaError_t> err(nt, cudaSuccess);
        for (int t = 0; t < nt; ++t)
            th.emplace_back([&, t] {
                const size_t o = t * piece, l = std::min(piece, bytes - o);
                err[t] = cudaHostRegister(h + o, l, cudaHostRegisterPortable | cudaHostRegisterMapped | cudaHostRegisterReadOnly);
            });
        for (auto& x : th) x.join();
        double t1 = now();
        for (int t = 0; t < nt; ++t) if (err[t] != cudaSuccess) { printf("register failed: %s\n", cudaGetErrorString(err[t])); return 1; }
        void* dp = nullptr;
        CK(cudaHostGetDevicePointer(&dp, h, 0));
        // 1 GiB DMA straddling the first split point, and an SM zero-copy read of the same range
        const size_t at = nt > 1 ? piece - gib / 2 : bytes / 2 - gib / 2;
        float ms_dma = 0, ms_zc = 0;
        for (int r = 0; r < 3; ++r) {
            double h0 = now();
            CK(cudaEventRecord(e0, s));
            CK(cudaMemcpyAsync(d, h + at, gib, cudaMemcpyHostToDevice, s));
            double h1 = now();
            CK(cudaEventRecord(e1, s));
            CK(cudaEventSynchronize(e1));
            CK(cudaEventElapsedTime(&ms_dma, e0, e1));
            if (r == 2) printf("  memcpy enqueue %.3f ms (async if << transfer)\n", 1e3 * (h1 - h0));
        }
        for (int r = 0; r < 3; ++r) {
            CK(cudaEventRecord(e0, s));
            zc_read<<<296, 256, 0, s>>>((const uint4*)((char*)dp + at), (uint4*)d, gib / 16);
            CK(cudaEventRecord(e1, s));
            CK(cudaEventSynchronize(e1));
            CK(cudaEventElapsedTime(&ms_zc, e0, e1));
        }
        CK(cudaGetLastError());
        double t2 = now();
        for (int t = 0; t < nt; ++t) CK(cudaHostUnregister(h + t * piece));
        double t3 = now();
        printf("%2d threads: register %.1f ms (%.1f GB/s), unregister %.1f ms, DMA across split %.2f GB/s, SM zero-copy %.2f GB/s, dev==host %d\n",
               nt, 1e3 * (t1 - t0), bytes / (t1 - t0) / 1e9, 1e3 * (t3 - t2), gib / (ms_dma / 1e3) / 1e9,
               gib / (ms_zc / 1e3) / 1e9, (int)(dp == (void*)h));
    }
    return 0;
}
