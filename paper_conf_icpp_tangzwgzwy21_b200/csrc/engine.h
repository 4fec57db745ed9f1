// engine.h — the host-side run controller behind the C ABI (include/ascetic.h).
#pragma once
#include <cstdint>
#include <stdexcept>
#include <string>
#include <vector>

#include <cuda_runtime.h>

#include "../../include/ascetic.h"
#include "ascetic_internal.h"

namespace ascetic {

// An error that maps onto an ascetic_status at the ABI.
struct Error : std::runtime_error {
    int code;
    Error(int c, const std::string& m) : std::runtime_error(m), code(c) {}
};

// Eq. 1/Eq. 2 placement (§3.3; K = 0.10; 16 KiB).
struct Placement {
    double R = 0.0;
    uint64_t D = 0, B = 0, Ms = 0, s = 0, static_bytes = 0, C = 0, cap = 0;
};
Placement place(const uint64_t* off, uint64_t n, uint32_t b_e, uint64_t budget, double frac);

struct EventPool {
    std::vector<cudaEvent_t> ev;
    size_t used = 0;
    cudaEvent_t get();
    void reset() { used = 0; }
    ~EventPool();
};

class Engine {
  public:
    ~Engine();
    void set_device(int dev);
    void load_csr(uint64_t n, uint64_t m, const uint64_t* off, const uint32_t* nbr, const uint32_t* wgt,
                  uint32_t flags);
    void set_budget(uint64_t bytes, double frac);
    void set_option(int opt, int64_t value);
    void run(int algo, uint32_t source, uint32_t max_iters);
    int stats(ascetic_stats_t* out, ascetic_iter_stats_t* per_iter, uint32_t cap) const;
    void get_result(void* dst, uint64_t bytes);
    void unload();
    int state() const { return state_; }

  private:
    void alloc_vertex_state();
    void alloc_algo_state(int algo);
    void free_budget_regions();
    void transfer_chunk(const Queues& q, int buf, unsigned long long lo, unsigned long long hi, int mode,
                        const std::vector<uint32_t>& rb, const std::vector<uint32_t>& re,
                        const std::vector<unsigned long long>& rdst);
    DevState dev_state(uint32_t iter) const;
    Queues queues(const IterTotals& T) const;

    int state_ = 0;  // 0 unloaded, 1 loaded, 2 ready
    int device_ = -1;
    // graph (host)
    uint64_t n_ = 0, m_ = 0;
    uint32_t b_e_ = 4, flags_ = 0;
    const uint64_t* h_off_ = nullptr;
    std::vector<uint64_t> h_off_copy_;
    const void* h_nbr_ = nullptr;        // b_e bytes per arc, pinned
    const void* h_nbr_dev_ = nullptr;    // device-visible alias (zero-copy)
    void* h_owned_ = nullptr;            // library-owned pinned copy
    void* h_registered_ = nullptr;       // pinned in place by us
    // device vertex state
    uint32_t nwords_ = 0, ntiles_ = 0;
    unsigned long long* d_off_ = nullptr;
    uint32_t *d_A_ = nullptr, *d_S_ = nullptr, *d_next_ = nullptr, *d_visited_ = nullptr;
    uint32_t *d_val_ = nullptr, *d_snap_ = nullptr;
    float *d_rank_ = nullptr, *d_contrib_ = nullptr;
    double *d_sum_ = nullptr, *d_dang_ = nullptr;
    uint32_t *d_hq_small_ = nullptr, *d_hq_med_ = nullptr, *d_hq_hub_ = nullptr, *d_hub_pre_ = nullptr;
    uint32_t *d_mq_ = nullptr, *d_run_b_ = nullptr, *d_run_e_ = nullptr;
    unsigned long long *d_mq_pre_ = nullptr, *d_run_dst_ = nullptr, *d_mq_src_ = nullptr;
    uint32_t* d_tile_first_ = nullptr;
    int sm_count_ = 148;
    int opt_gather_ctas_ = 0;       // 0 = 2 x SMs
    ScanVal *d_tile_agg_ = nullptr, *d_tile_incl_ = nullptr;
    uint32_t* d_tile_flag_ = nullptr;
    uint32_t epoch_ = 0;
    IterTotals* d_tot_ = nullptr;
    IterTotals* h_tot_ = nullptr;   // mapped pinned
    uint64_t vertex_bytes_ = 0;
    // edge budget regions
    Placement pl_{};
    void* d_static_ = nullptr;
    void* d_chunk_[2] = {nullptr, nullptr};
    uint64_t cap_ = 0;              // effective chunk capacity (bytes)
    bool static_valid_ = false;     // KEEP_STATIC: static region already holds the prefix
    // streams/events
    cudaStream_t cs_ = nullptr, xs_ = nullptr;
    cudaEvent_t ready_[2] = {nullptr, nullptr}, consumed_[2] = {nullptr, nullptr};
    cudaEvent_t ev_classified_ = nullptr;
    EventPool pool_;
    // options
    uint64_t opt_chunk_cap_ = 0;
    int opt_xfer_mode_ = 0;
    uint64_t opt_dma_min_run_ = 64 * 1024;
    int opt_overlap_ = 1;
    int opt_keep_static_ = 0;
    uint32_t opt_hub_deg_ = 2048;
    int opt_timing_ = 1;
    static constexpr uint32_t kPieceArcs = 4096;
    static constexpr uint32_t kRunsHostMax = 8192;
    // results / stats
    int last_algo_ = -1;
    bool have_result_ = false;
    ascetic_stats_t st_{};
    std::vector<ascetic_iter_stats_t> iters_;
};

}  // namespace ascetic
