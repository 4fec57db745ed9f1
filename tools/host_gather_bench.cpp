// host_gather_bench.cpp — can host threads gather short adjacency lists faster than the link?
// g++ -O3 -march=native -pthread -o tools/host_gather_bench tools/host_gather_bench.cpp
#include <chrono>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <random>
#include <thread>
#include <vector>

int main() {
    const size_t n8 = (4ull << 30) / 8;
    uint64_t* src = (uint64_t*)aligned_alloc(4096, n8 * 8);
    for (size_t i = 0; i < n8; ++i) src[i] = i;
    const size_t want = 256ull << 20 >> 3;
    uint64_t* dst = (uint64_t*)aligned_alloc(4096, want * 8 + 4096);
    for (int avg : {3, 6, 24, 60, 96, 1024}) {
        std::mt19937_64 rng(avg);
        std::vector<uint64_t> rs, rp;
        uint64_t total = 0;
        while (total < want) {
            uint64_t len = 1 + rng() % (2 * avg - 1);
            if (total + len > want) len = want - total;
            // ascending starts like a miss stream (ids ascending)
            rs.push_back(0); rp.push_back(total); total += len;
        }
        // ascending random starts
        uint64_t gap_room = n8 - total;
        std::vector<uint64_t> gaps(rs.size());
        for (auto& g : gaps) g = rng() % (2 * gap_room / rs.size() + 1);
        uint64_t pos = 0;
        for (size_t r = 0; r < rs.size(); ++r) {
            pos += gaps[r];
            if (pos + (r + 1 < rs.size() ? rp[r + 1] - rp[r] : total - rp[r]) > n8) pos = 0;
            rs[r] = pos;
            pos += (r + 1 < rs.size() ? rp[r + 1] - rp[r] : total - rp[r]);
        }
        for (int nt : {1, 4, 8, 16}) {
            double best = 1e9;
            for (int rep = 0; rep < 3; ++rep) {
                auto t0 = std::chrono::steady_clock::now();
                std::vector<std::thread> th;
                for (int t = 0; t < nt; ++t)
                    th.emplace_back([&, t] {
                        size_t nr = rs.size();
                        size_t a = nr * t / nt, b = nr * (t + 1) / nt;
                        for (size_t r = a; r < b; ++r) {
                            uint64_t len = (r + 1 < nr ? rp[r + 1] : total) - rp[r];
                            memcpy(dst + rp[r], src + rs[r], len * 8);
                        }
                    });
                for (auto& x : th) x.join();
                double s = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
                best = std::min(best, s);
            }
            printf("avg=%5d arcs(8B) runs=%8zu threads=%2d  %7.2f GB/s\n", avg, rs.size(), nt, total * 8 / best / 1e9);
        }
    }
    return 0;
}
