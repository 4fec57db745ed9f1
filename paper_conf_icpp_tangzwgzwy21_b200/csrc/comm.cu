// comm.cu — NCCL (dlopen) and single-GPU emulated collectives for the per-iteration exchange.
#include "comm.h"

#include <dlfcn.h>
#include <nccl.h>   // types and enums only; every function is resolved with dlsym

#include <algorithm>
#include <cstring>

#include "ascetic_internal.h"
#include "engine.h"

namespace ascetic {

namespace {

struct NcclApi {
    bool loaded = false;
    ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
    ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
    ncclResult_t (*AllReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*AllGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*Broadcast)(const void*, void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*Send)(const void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*Recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*GroupStart)() = nullptr;
    ncclResult_t (*GroupEnd)() = nullptr;
    const char* (*GetErrorString)(ncclResult_t) = nullptr;
};

NcclApi& nccl() {
    static NcclApi api;
    if (api.loaded) return api;
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL | RTLD_NOLOAD);   // torch's, if already loaded
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (!h) throw Error(ASCETIC_EUNSUPPORTED, std::string("cannot load libnccl.so.2: ") + dlerror());
    auto sym = [&](const char* name) {
        void* p = dlsym(h, name);
        if (!p) throw Error(ASCETIC_EUNSUPPORTED, std::string("libnccl lacks ") + name);
        return p;
    };
    api.GetUniqueId = (decltype(api.GetUniqueId))sym("ncclGetUniqueId");
    api.CommInitRank = (decltype(api.CommInitRank))sym("ncclCommInitRank");
    api.CommDestroy = (decltype(api.CommDestroy))sym("ncclCommDestroy");
    api.AllReduce = (decltype(api.AllReduce))sym("ncclAllReduce");
    api.AllGather = (decltype(api.AllGather))sym("ncclAllGather");
    api.Broadcast = (decltype(api.Broadcast))sym("ncclBroadcast");
    api.Send = (decltype(api.Send))sym("ncclSend");
    api.Recv = (decltype(api.Recv))sym("ncclRecv");
    api.GroupStart = (decltype(api.GroupStart))sym("ncclGroupStart");
    api.GroupEnd = (decltype(api.GroupEnd))sym("ncclGroupEnd");
    api.GetErrorString = (decltype(api.GetErrorString))sym("ncclGetErrorString");
    api.loaded = true;
    return api;
}

void NC(ncclResult_t r, const char* what) {
    if (r != ncclSuccess) throw Error(ASCETIC_ENCCL, std::string(what) + ": " + nccl().GetErrorString(r));
}

void CKc(cudaError_t e, const char* what) {
    if (e != cudaSuccess) throw Error(ASCETIC_ECUDA, std::string(what) + ": " + cudaGetErrorString(e));
}

}  // namespace

void Comm::unique_id(void* out128) {
    ncclUniqueId id;
    NC(nccl().GetUniqueId(&id), "ncclGetUniqueId");
    std::memcpy(out128, &id, sizeof id);
}

void Comm::init_nccl(int rank, int world, const void* uid128) {
    destroy();
    if (world < 1 || rank < 0 || rank >= world) throw Error(ASCETIC_EINVAL, "bad rank/world");
    world_ = world; rank_ = rank; emulated_ = false;
    // world 1 without an id: no communicator (single GPU). world 1 WITH an id: a one-rank NCCL
    // communicator, so the whole exchange path (collectives, barriers, IPC handle exchange)
    // runs through NCCL on one GPU — how that path is exercised without a multi-GPU box.
    if (world == 1 && !uid128) return;
    ncclUniqueId id;
    std::memcpy(&id, uid128, sizeof id);
    ncclComm_t c = nullptr;
    NC(nccl().CommInitRank(&c, world, id, rank), "ncclCommInitRank");
    nccl_comm_ = c;
}

void Comm::init_emulated(int world) {
    destroy();
    if (world < 1) throw Error(ASCETIC_EINVAL, "world must be >= 1");
    world_ = world; rank_ = 0; emulated_ = world > 1;
}

void Comm::destroy() {
    for (auto& m : peer_maps_) cudaIpcCloseMemHandle(m.ptr);
    peer_maps_.clear();
    if (barrier_buf_) { cudaFree(barrier_buf_); barrier_buf_ = nullptr; }
    if (nccl_comm_) { nccl().CommDestroy((ncclComm_t)nccl_comm_); nccl_comm_ = nullptr; }
    if (scratch_) { cudaFree(scratch_); scratch_ = nullptr; scratch_words_ = 0; }
    if (sp_counts_) { cudaFree(sp_counts_); sp_counts_ = nullptr; }
    if (sp_counts_host_) { cudaFreeHost(sp_counts_host_); sp_counts_host_ = nullptr; }
    if (sp_gather_) { cudaFree(sp_gather_); sp_gather_ = nullptr; sp_gather_bytes_ = 0; }
    world_ = 1; rank_ = 0; emulated_ = false;
}

void Comm::or_words(const std::vector<uint32_t*>& local, uint64_t nw, cudaStream_t s) {
    if (!active() || nw == 0) return;
    if (emulated_) {
        for (size_t p = 1; p < local.size(); ++p) launch_or_into(local[0], local[p], nw, s);
        for (size_t p = 1; p < local.size(); ++p)
            CKc(cudaMemcpyAsync(local[p], local[0], nw * 4, cudaMemcpyDeviceToDevice, s), "or copy-back");
        return;
    }
    // NCCL has no bitwise OR: reduce-scatter-OR by point-to-point slices, then all-gather the ORed
    // slices. Rank r owns words [r*S, min((r+1)*S, nw)), S = ceil(nw/P); every rank sends each peer
    // that peer's slice and ORs the P copies of its own: 2 (P-1)/P * nw words on the wire per rank
    // (an all-gather of whole bitmaps + local OR would move (P-1) * nw).
    const uint64_t P = (uint64_t)world_, me = (uint64_t)rank_;
    const uint64_t S = (nw + P - 1) / P;
    auto len = [&](uint64_t r) -> uint64_t { return r * S >= nw ? 0 : std::min(S, nw - r * S); };
    const uint64_t need = 2 * P * S;
    if (scratch_words_ < need) {
        if (scratch_) cudaFree(scratch_);
        CKc(cudaMalloc(&scratch_, need * 4), "exchange scratch");
        scratch_words_ = need;
    }
    uint32_t* recv = scratch_;           // [P][len(me)]: every rank's copy of my slice
    uint32_t* gath = scratch_ + P * S;   // [P][S]: the ORed slices, gathered in place
    const uint64_t lm = len(me);
    if (lm) CKc(cudaMemcpyAsync(recv + me * lm, local[0] + me * S, lm * 4, cudaMemcpyDeviceToDevice, s), "own slice");
    NC(nccl().GroupStart(), "ncclGroupStart");
    for (uint64_t r = 0; r < P; ++r) {
        if (r == me) continue;
        if (len(r)) NC(nccl().Send(local[0] + r * S, len(r), ncclUint32, (int)r, (ncclComm_t)nccl_comm_, s), "ncclSend(slice)");
        if (lm) NC(nccl().Recv(recv + r * lm, lm, ncclUint32, (int)r, (ncclComm_t)nccl_comm_, s), "ncclRecv(slice)");
    }
    NC(nccl().GroupEnd(), "ncclGroupEnd");
    if (lm) launch_or_reduce(gath + me * S, recv, (uint32_t)P, lm, s);
    NC(nccl().AllGather(gath + me * S, gath, S, ncclUint32, (ncclComm_t)nccl_comm_, s), "ncclAllGather(ORed slices)");
    CKc(cudaMemcpyAsync(local[0], gath, nw * 4, cudaMemcpyDeviceToDevice, s), "bitmap copy-back");
}

void Comm::min_u32(const std::vector<uint32_t*>& local, uint64_t n, cudaStream_t s) {
    if (!active() || n == 0) return;
    if (emulated_) {
        for (size_t p = 1; p < local.size(); ++p) launch_min_into(local[0], local[p], n, s);
        for (size_t p = 1; p < local.size(); ++p)
            CKc(cudaMemcpyAsync(local[p], local[0], n * 4, cudaMemcpyDeviceToDevice, s), "min copy-back");
        return;
    }
    NC(nccl().AllReduce(local[0], local[0], n, ncclUint32, ncclMin, (ncclComm_t)nccl_comm_, s), "ncclAllReduce(min)");
}

void Comm::reserve_sparse(uint32_t cap, int local_parts) {
    if (!active()) return;
    if (!sp_counts_host_)
        CKc(cudaMallocHost(&sp_counts_host_, sizeof(uint32_t) * (size_t)std::max(world_, local_parts)), "sparse counts");
    if (emulated_) return;
    if (!sp_counts_) CKc(cudaMalloc(&sp_counts_, sizeof(uint32_t) * (size_t)world_), "sparse counts");
    const uint64_t want = (uint64_t)world_ * cap * 8ull;
    if (sp_gather_bytes_ < want) {
        if (sp_gather_) cudaFree(sp_gather_);
        CKc(cudaMalloc(&sp_gather_, want), "sparse gather");
        sp_gather_bytes_ = want;
    }
}

bool Comm::sparse_min(const std::vector<uint32_t*>& val, const std::vector<uint32_t*>& next,
                      const std::vector<void*>& pairs, const std::vector<uint32_t*>& count, uint32_t cap,
                      cudaStream_t s, uint64_t* bytes_out) {
    if (!active()) return true;
    const int L = (int)val.size();   // local ranks: world when emulated, 1 with NCCL
    if (!sp_counts_host_) CKc(cudaMallocHost(&sp_counts_host_, sizeof(uint32_t) * (size_t)std::max(world_, L)), "sparse counts");
    if (emulated_) {
        for (int i = 0; i < L; ++i)
            CKc(cudaMemcpyAsync(sp_counts_host_ + i, count[i], 4, cudaMemcpyDeviceToHost, s), "sparse counts d2h");
    } else {
        if (!sp_counts_) CKc(cudaMalloc(&sp_counts_, sizeof(uint32_t) * (size_t)world_), "sparse counts");
        NC(nccl().AllGather(count[0], sp_counts_, 1, ncclUint32, (ncclComm_t)nccl_comm_, s), "ncclAllGather(sparse counts)");
        CKc(cudaMemcpyAsync(sp_counts_host_, sp_counts_, 4 * (size_t)world_, cudaMemcpyDeviceToHost, s), "sparse counts d2h");
    }
    CKc(cudaStreamSynchronize(s), "sparse counts sync");
    uint32_t maxc = 0;
    uint64_t total = 0;
    for (int r = 0; r < world_; ++r) { maxc = std::max(maxc, sp_counts_host_[r]); total += sp_counts_host_[r]; }
    if (maxc > cap) return false;
    if (bytes_out) *bytes_out = total * 8ull;
    if (maxc == 0) return true;
    if (emulated_) {
        // every part applies every other part's pairs; all packs were enqueued before, on s
        for (int q = 0; q < L; ++q)
            for (int p = 0; p < L; ++p)
                if (p != q) launch_sparse_apply(val[q], next[q], pairs[p], 0, count[p], 1, -1, maxc, s);
        return true;
    }
    const uint64_t need = (uint64_t)world_ * maxc * 8ull;
    if (sp_gather_bytes_ < need) {
        if (sp_gather_) cudaFree(sp_gather_);
        const uint64_t want = (uint64_t)world_ * cap * 8ull;   // sized once for the largest exchange
        CKc(cudaMalloc(&sp_gather_, want), "sparse gather");
        sp_gather_bytes_ = want;
    }
    NC(nccl().AllGather(pairs[0], sp_gather_, 2ull * maxc, ncclUint32, (ncclComm_t)nccl_comm_, s),
       "ncclAllGather(sparse pairs)");
    launch_sparse_apply(val[0], next[0], sp_gather_, maxc, sp_counts_, world_, rank_, maxc, s);
    return true;
}

void Comm::sum_u64(const std::vector<unsigned long long*>& local, uint64_t n, cudaStream_t s) {
    if (!active() || n == 0) return;
    if (emulated_) {
        for (size_t p = 1; p < local.size(); ++p) launch_add_u64(local[0], local[p], n, s);
        for (size_t p = 1; p < local.size(); ++p)
            CKc(cudaMemcpyAsync(local[p], local[0], n * 8, cudaMemcpyDeviceToDevice, s), "sum copy-back");
        return;
    }
    NC(nccl().AllReduce(local[0], local[0], n, ncclUint64, ncclSum, (ncclComm_t)nccl_comm_, s), "ncclAllReduce(sum u64)");
}

std::vector<void*> Comm::open_peers(void* local) {
    if (emulated_ || !active()) throw Error(ASCETIC_EINVAL, "open_peers needs the NCCL back end");
    // Always collective: every rank all-gathers its current handle, whatever its cache holds
    // (a rank that re-allocated while another did not must not leave that one waiting in a
    // skipped all-gather). A peer mapping is reused only while the peer's handle is unchanged.
    cudaIpcMemHandle_t h;
    CKc(cudaIpcGetMemHandle(&h, local), "cudaIpcGetMemHandle");
    char* dbuf = nullptr;
    CKc(cudaMalloc(&dbuf, sizeof h * (size_t)(world_ + 1)), "ipc handle buffer");
    CKc(cudaMemcpy(dbuf + sizeof h * (size_t)world_, &h, sizeof h, cudaMemcpyHostToDevice), "ipc handle H2D");
    NC(nccl().AllGather(dbuf + sizeof h * (size_t)world_, dbuf, sizeof h, ncclInt8, (ncclComm_t)nccl_comm_, 0),
       "ncclAllGather(ipc handles)");
    std::vector<cudaIpcMemHandle_t> all(world_);
    cudaError_t e = cudaMemcpy(all.data(), dbuf, sizeof h * (size_t)world_, cudaMemcpyDeviceToHost);
    cudaFree(dbuf);
    CKc(e, "ipc handles D2H");
    std::vector<void*> ptrs(world_, nullptr);
    for (int p = 0; p < world_; ++p) {
        if (p == rank_) { ptrs[p] = local; continue; }
        for (auto& m : peer_maps_)
            if (m.rank == p && std::memcmp(m.handle, &all[p], sizeof h) == 0) { ptrs[p] = m.ptr; break; }
        if (ptrs[p]) continue;
        CKc(cudaIpcOpenMemHandle(&ptrs[p], all[p], cudaIpcMemLazyEnablePeerAccess), "cudaIpcOpenMemHandle");
        PeerMap m;
        m.rank = p; m.ptr = ptrs[p];
        std::memcpy(m.handle, &all[p], sizeof h);
        peer_maps_.push_back(m);
    }
    return ptrs;
}

void Comm::barrier(cudaStream_t s) {
    if (emulated_ || !active()) return;
    if (!barrier_buf_) {
        CKc(cudaMalloc(&barrier_buf_, sizeof(int)), "barrier buffer");
        CKc(cudaMemset(barrier_buf_, 0, sizeof(int)), "barrier buffer");
    }
    NC(nccl().AllReduce(barrier_buf_, barrier_buf_, 1, ncclInt32, ncclMax, (ncclComm_t)nccl_comm_, s), "barrier");
}

void Comm::share_slices(const std::vector<void*>& local, const std::vector<uint64_t>& bounds, uint32_t elem_bytes,
                        cudaStream_t s) {
    if (!active()) return;
    if (emulated_) {
        for (size_t r = 0; r < local.size(); ++r) {
            const uint64_t off = bounds[r] * elem_bytes, len = (bounds[r + 1] - bounds[r]) * elem_bytes;
            if (!len) continue;
            for (size_t p = 0; p < local.size(); ++p)
                if (p != r)
                    CKc(cudaMemcpyAsync((char*)local[p] + off, (const char*)local[r] + off, len, cudaMemcpyDeviceToDevice, s),
                        "slice copy");
        }
        return;
    }
    NC(nccl().GroupStart(), "ncclGroupStart");
    for (int r = 0; r < world_; ++r) {
        const uint64_t off = bounds[r] * elem_bytes, len = (bounds[r + 1] - bounds[r]) * elem_bytes;
        if (!len) continue;
        char* p = (char*)local[0] + off;
        NC(nccl().Broadcast(p, p, len, ncclInt8, r, (ncclComm_t)nccl_comm_, s), "ncclBroadcast(slice)");
    }
    NC(nccl().GroupEnd(), "ncclGroupEnd");
}

}  // namespace ascetic
