// cpu_gather_bench.cpp — host-side random row gather rate (phase 1 of a staged miss path).
//   g++ -O3 -march=native -pthread -o cg tools/cpu_gather_bench.cpp
//   ./cg <table_GB> <row_bytes> <rows> <thp 0/1>
#include <sys/mman.h>
#include <emmintrin.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <random>
#include <thread>
#include <vector>

int main(int argc, char** argv) {
    const double GB = argc > 1 ? atof(argv[1]) : 32;
    const size_t R = argc > 2 ? atoll(argv[2]) : 512;
    const size_t n = argc > 3 ? atoll(argv[3]) : 200000;
    const int thp = argc > 4 ? atoi(argv[4]) : 1;
    const size_t N = (size_t)(GB * 1e9) / R, bytes = N * R;
    uint8_t* t = (uint8_t*)mmap(nullptr, bytes, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
    if (thp) madvise(t, bytes, MADV_HUGEPAGE);
    {
        std::vector<std::thread> th;
        const int T = 16;
        for (int k = 0; k < T; ++k)
            th.emplace_back([&, k] { memset(t + bytes / T * k, k + 1, bytes / T + (k == T - 1 ? bytes % T : 0)); });
        for (auto& x : th) x.join();
    }
    std::vector<int32_t> rows(n);
    std::mt19937_64 rng(1);
    for (auto& r : rows) r = (int32_t)(rng() % N);
    uint8_t* stage = (uint8_t*)aligned_alloc(64, n * R);
    for (int T : {1, 2, 4, 8, 12, 16}) {
        for (int pf : {0, 1}) {   // 1 = non-temporal stores
            double best = 0;
            for (int rep = 0; rep < 3; ++rep) {
                auto t0 = std::chrono::steady_clock::now();
                std::vector<std::thread> th;
                for (int k = 0; k < T; ++k)
                    th.emplace_back([&, k] {
                        const size_t lo = n * k / T, hi = n * (k + 1) / T;
                        for (size_t i = lo; i < hi; ++i) {
                            if (pf) {
                                const __m128i* sp = (const __m128i*)(t + (size_t)rows[i] * R);
                                __m128i* dp = (__m128i*)&stage[i * R];
                                for (size_t c = 0; c < R / 16; ++c) _mm_stream_si128(dp + c, _mm_loadu_si128(sp + c));
                            } else {
                                memcpy(&stage[i * R], t + (size_t)rows[i] * R, R);
                            }
                        }
                        _mm_sfence();
                    });
                for (auto& x : th) x.join();
                const double s = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
                best = std::max(best, n * R / s / 1e9);
            }
            printf("table %.0f GB R=%zu thp=%d threads=%2d nt_store=%d: %.1f GB/s\n", GB, R, thp, T, pf, best);
        }
    }
    return 0;
}
