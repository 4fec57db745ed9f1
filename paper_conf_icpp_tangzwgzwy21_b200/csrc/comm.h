// comm.h — the per-iteration exchange of the multi-GPU path (the paper itself
// is single-GPU). One process per GPU, 1D vertex ranges, replicated vertex state:
//   BFS       : OR of the next-frontier bitmaps        (NCCL has no bitwise OR: reduce-scatter-OR over
//               point-to-point slices + OR kernel, then all-gather of the ORed slices)
//   SSSP / CC : MIN of the value arrays               (ncclAllReduce min)
//   PR        : SUM of the 2^-62 fixed-point dangling partials (exact) + every rank's contrib slice to all ranks
//   PRD       : SUM of the u64 residual increments   (ncclAllReduce sum, exact: integers)
// Two back ends behind one interface:
//   NCCL     — across processes (libnccl.so.2 is dlopen'ed on first use, so single-GPU
//              runs never load it and torch's own NCCL is reused when already loaded);
//   emulated — P ranks driven by ONE process on ONE GPU (each rank a full engine part with
//              its own device state); the same collectives done with device copies and
//              reduction kernels. It runs the identical per-rank code path, which is how the
//              P > 1 path is tested on a single GPU.
#pragma once
#include <cstdint>
#include <string>
#include <vector>

#include <cuda_runtime.h>

namespace ascetic {

class Comm {
  public:
    // NCCL back end
    static void unique_id(void* out128);
    void init_nccl(int rank, int world, const void* uid128);
    // emulated back end: `world` ranks, all local
    void init_emulated(int world);
    void destroy();
    ~Comm() { destroy(); }

    bool active() const { return world_ > 1 || nccl_comm_ != nullptr; }
    bool emulated() const { return emulated_; }
    int world() const { return world_; }
    int rank() const { return rank_; }

    // Collectives over all ranks. `local` = this process's buffers: one per local rank
    // (1 with NCCL, world with emulation). Everything is enqueued on `s`.
    void or_words(const std::vector<uint32_t*>& local, uint64_t nw, cudaStream_t s);
    void min_u32(const std::vector<uint32_t*>& local, uint64_t n, cudaStream_t s);
    // sparse MIN (SSSP / CC, small frontiers): every rank's (id, value) improvement pairs
    // (pairs[i]: count[i] of them, device u32, packed by launch_sparse_pack with capacity cap) go to
    // every rank and are applied by atomicMin + next bit. Reads the counts on the host (one sync);
    // returns false, having changed nothing, when some rank has more than cap pairs (the caller then
    // runs min_u32). All ranks take the same decision: they see the same counts.
    // allocate sparse_min's host count buffer and (NCCL) its gather buffer for `cap` pairs per rank
    void reserve_sparse(uint32_t cap, int local_parts);
    bool sparse_min(const std::vector<uint32_t*>& val, const std::vector<uint32_t*>& next,
                    const std::vector<void*>& pairs, const std::vector<uint32_t*>& count, uint32_t cap,
                    cudaStream_t s, uint64_t* bytes_out = nullptr);
    // element-wise SUM of n uint64 per rank (PageRank-delta residual increments), in place
    void sum_u64(const std::vector<unsigned long long*>& local, uint64_t n, cudaStream_t s);
    // Fused exchange support (NCCL back end): map every rank's `local` device allocation into this
    // process with CUDA IPC (handles all-gathered over NCCL on every call; a peer's mapping is reused while its handle is unchanged); returns the
    // world pointers, this rank's own at index rank(). Collective: every rank calls it.
    std::vector<void*> open_peers(void* local);
    // stream-ordered barrier over all ranks (a 4-byte ncclAllReduce); no-op when emulated
    void barrier(cudaStream_t s);
    // rank r owns elements [bounds[r], bounds[r+1]) of an elem_bytes array; afterwards every
    // rank holds every slice
    void share_slices(const std::vector<void*>& local, const std::vector<uint64_t>& bounds, uint32_t elem_bytes,
                      cudaStream_t s);

  private:
    int world_ = 1, rank_ = 0;
    bool emulated_ = false;
    void* nccl_comm_ = nullptr;
    uint32_t* scratch_ = nullptr;
    uint64_t scratch_words_ = 0;
    int* barrier_buf_ = nullptr;
    uint32_t* sp_counts_ = nullptr;      // device: all ranks' pair counts (NCCL)
    uint32_t* sp_counts_host_ = nullptr; // pinned: the same on the host
    void* sp_gather_ = nullptr;          // device: all ranks' pairs (NCCL), world x cap
    uint64_t sp_gather_bytes_ = 0;
    struct PeerMap {   // an opened CUDA IPC mapping of a peer's allocation
        int rank;
        unsigned char handle[64];   // CUDA_IPC_HANDLE_SIZE
        void* ptr;
    };
    std::vector<PeerMap> peer_maps_;
};

}  // namespace ascetic
