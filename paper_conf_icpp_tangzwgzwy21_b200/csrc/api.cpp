// api.cpp — the extern "C" boundary (include/ascetic.h). Every entry point maps
// C++ errors to an ascetic_status and a thread-local message; nothing throws across.
#include <cstring>
#include <new>
#include <string>

#include "engine.h"

namespace {
thread_local std::string g_err;
ascetic::Engine* g_engine = nullptr;

ascetic::Engine& engine() {
    if (!g_engine) g_engine = new ascetic::Engine();
    return *g_engine;
}

template <typename F>
int guarded(F&& f) {
    try {
        g_err.clear();
        return f();
    } catch (const ascetic::Error& e) {
        g_err = e.what();
        return e.code;
    } catch (const std::bad_alloc&) {
        g_err = "host allocation failed";
        return ASCETIC_EHOSTMEM;
    } catch (const std::exception& e) {
        g_err = e.what();
        return ASCETIC_ECUDA;
    } catch (...) {
        g_err = "unknown error";
        return ASCETIC_ECUDA;
    }
}
}  // namespace

extern "C" {

int ascetic_load_csr(uint64_t n, uint64_t m, const uint64_t* off, const uint32_t* nbr, const uint32_t* wgt,
                     uint32_t flags) {
    return guarded([&] { engine().load_csr(n, m, off, nbr, wgt, flags); return 0; });
}

int ascetic_set_budget(uint64_t bytes, double static_fraction) {
    return guarded([&] { engine().set_budget(bytes, static_fraction); return 0; });
}

int ascetic_place(uint64_t n, const uint64_t* off, uint32_t b_e, uint64_t bytes, double static_fraction,
                  ascetic_placement_t* out) {
    return guarded([&] {
        if (!off || !out) throw ascetic::Error(ASCETIC_EINVAL, "NULL argument");
        if (b_e != 4 && b_e != 8) throw ascetic::Error(ASCETIC_EINVAL, "b_e must be 4 or 8");
        if (static_fraction != static_fraction || static_fraction > 1.0)
            throw ascetic::Error(ASCETIC_EINVAL, "static_fraction must be <= 1 (or < 0 for Eq. 2)");
        const ascetic::Placement p = ascetic::place(off, n, b_e, bytes, static_fraction);
        out->R = p.R; out->D = p.D; out->B = p.B; out->Ms = p.Ms; out->s = p.s;
        out->static_bytes = p.static_bytes; out->C = p.C; out->cap = p.cap;
        return 0;
    });
}

int ascetic_debug_classify(int rank, const uint32_t* active_words, uint64_t nwords, ascetic_classify_out_t* out) {
    return guarded([&] { engine().debug_classify(rank, active_words, nwords, out); return 0; });
}

int ascetic_set_option(int option, int64_t value) {
    return guarded([&] { engine().set_option(option, value); return 0; });
}

int ascetic_run(int algo, uint32_t source, uint32_t max_iters) {
    return guarded([&] { engine().run(algo, source, max_iters); return 0; });
}

int ascetic_stats(ascetic_stats_t* out, ascetic_iter_stats_t* per_iter, uint32_t cap) {
    return guarded([&] { return engine().stats(out, per_iter, cap); });
}

int ascetic_get_result(void* host_dst, uint64_t bytes) {
    return guarded([&] { engine().get_result(host_dst, bytes); return 0; });
}

int ascetic_get_unique_id(void* out128) {
    return guarded([&] {
        if (!out128) throw ascetic::Error(ASCETIC_EINVAL, "out128 is NULL");
        ascetic::Comm::unique_id(out128);
        return 0;
    });
}

int ascetic_comm_init(int rank, int world, const void* uid128, int device) {
    return guarded([&] { engine().comm_init(rank, world, uid128, device); return 0; });
}

int ascetic_emulate_ranks(int world) {
    return guarded([&] { engine().emulate_ranks(world); return 0; });
}

int ascetic_partition(uint64_t n, const uint64_t* off, uint32_t parts, uint64_t* bounds) {
    return guarded([&] {
        if (!off || !bounds || parts < 1) throw ascetic::Error(ASCETIC_EINVAL, "bad argument");
        const auto b = ascetic::partition(off, n, parts);
        for (uint32_t i = 0; i <= parts; ++i) bounds[i] = b[i];
        return 0;
    });
}

int ascetic_set_device(int device) {
    return guarded([&] { engine().set_device(device); return 0; });
}

void ascetic_unload(void) {
    guarded([&] { engine().unload(); return 0; });
}

const char* ascetic_last_error(void) { return g_err.c_str(); }

int ascetic_struct_sizes(uint64_t* out3) {
    if (!out3) return ASCETIC_EINVAL;
    out3[0] = sizeof(ascetic_stats_t);
    out3[1] = sizeof(ascetic_iter_stats_t);
    out3[2] = sizeof(ascetic_placement_t);
    return 0;
}

const char* ascetic_version(void) { return "ascetic-b200 0.1 (sm_100a)"; }

}  // extern "C"
