// gd_hostpool.cu — host worker pool for phase 1 of the staged miss path (host code only).
//
// GNNDrive's extractor loads missed rows from storage into a host staging buffer before
// the GPU transfer ("two-phase extraction").  Here the storage stand-in is
// the pinned host table, and phase 1 is a multi-threaded CPU gather of the missed rows
// into a contiguous pinned staging slot, run from a CUDA host function on the library's
// host-gather stream; phase 2 (k_stage_copy) pulls the slot over the host link with
// contiguous, translation-friendly reads.
#include <emmintrin.h>   // SSE2 streaming stores (baseline x86-64)
#include <xmmintrin.h>   // _mm_prefetch

#include <algorithm>
#include <cstdlib>

#include <atomic>
#include <chrono>
#include <condition_variable>
#include <cstring>
#include <functional>
#include <mutex>
#include <thread>
#include <vector>

#include "gd_hostpool.h"

namespace gd {

struct HostGatherPool::Impl {
    std::vector<std::thread> workers;
    std::mutex mu;
    std::condition_variable cv_work, cv_done;
    // generation / active / stop are atomics so that idle workers and the waiting caller can
    // spin on them for a short while before sleeping on the condition variables: the chunks of
    // a batch arrive back to back, and a futex wake-up of 12 helpers plus the join cost tens of
    // microseconds per chunk (env GD_POOL_SPIN = spin iterations, 0 = sleep at once)
    std::atomic<uint64_t> generation{0};
    std::atomic<int> active{0};
    std::atomic<bool> stop{false};
    int spin = 4000;
    // current job
    const uint8_t* src = nullptr;
    const int32_t* rows = nullptr;
    uint8_t* dst = nullptr;
    int64_t n = 0, R = 0, P = 1;
    bool nt = true;
    std::atomic<int64_t> next{0};
    static constexpr int64_t kChunk = 256;

    // Row copy with non-temporal stores: the staging slot is read next by the GPU over
    // PCIe, so keeping it out of the CPU caches avoids snoop hits on dirty lines, and
    // streaming stores skip the read-for-ownership of every destination line.
    static void copy_row(uint8_t* d, const uint8_t* s, int64_t R, bool nt) {
        if (!nt) {
            std::memcpy(d, s, (size_t)R);
        } else if ((R & 15) == 0 && (((uintptr_t)d) & 15) == 0) {
            const __m128i* sp = (const __m128i*)s;
            __m128i* dp = (__m128i*)d;
            const int64_t n16 = R >> 4;
            int64_t c = 0;
            for (; c + 4 <= n16; c += 4) {
                const __m128i a = _mm_loadu_si128(sp + c), b = _mm_loadu_si128(sp + c + 1);
                const __m128i e = _mm_loadu_si128(sp + c + 2), f = _mm_loadu_si128(sp + c + 3);
                _mm_stream_si128(dp + c, a);
                _mm_stream_si128(dp + c + 1, b);
                _mm_stream_si128(dp + c + 2, e);
                _mm_stream_si128(dp + c + 3, f);
            }
            for (; c < n16; ++c) _mm_stream_si128(dp + c, _mm_loadu_si128(sp + c));
        } else {
            std::memcpy(d, s, (size_t)R);
        }
    }

    int64_t pf_env = -1;   // prefetch distance in rows from env GD_GATHER_PF (0 = off), else byte-based

    // Prefetch distance: ~4 KB of rows ahead (8 rows of 512 B, 4 of 1 KB, 2 of 1.5 KB), so the
    // lines in flight per thread stay within the core's fill buffers whatever the row width
    // (a fixed 8 rows asked for 192 lines ahead with mag240m's 1536-byte rows).
    int64_t pf_rows() const { return pf_env >= 0 ? pf_env : std::max<int64_t>(2, 4096 / std::max<int64_t>(1, R)); }

    const uint8_t* row_ptr(int64_t v) const { return src + (v < P ? v : v % P) * R; }
    // (prefetching into L2 instead, _MM_HINT_T1, and 16 rows ahead were measured within the
    // box's run-to-run noise: papers100m 405-461 batches/s for all four combinations)
    void prefetch_row(const uint8_t* p) const {
        for (int64_t c = 0; c < R; c += 64) _mm_prefetch((const char*)p + c, _MM_HINT_T0);
    }

    void work() {
        while (true) {
            const int64_t lo = next.fetch_add(kChunk, std::memory_order_relaxed);
            if (lo >= n) break;
            const int64_t hi = lo + kChunk < n ? lo + kChunk : n;
            // software prefetch `pf` rows ahead: random rows over a table far larger than
            // the caches and the TLB reach are latency-bound per thread; prefetching every
            // line of row j + pf keeps ~pf rows of misses (and their page walks) in flight
            const int64_t pf = pf_rows();
            for (int64_t j = lo; j < hi && j < lo + pf; ++j) prefetch_row(row_ptr(rows[j]));
            for (int64_t j = lo; j < hi; ++j) {
                if (j + pf < hi) prefetch_row(row_ptr(rows[j + pf]));
                copy_row(dst + j * R, row_ptr(rows[j]), R, nt);
            }
        }
        _mm_sfence();   // streaming stores globally visible before the GPU pull is released
    }

    void loop() {
        uint64_t seen = 0;
        while (true) {
            bool got = false;
            for (int i = 0; i < spin && !got; ++i) {
                if (stop.load(std::memory_order_acquire)) return;
                got = generation.load(std::memory_order_acquire) != seen;
                if (!got) _mm_pause();
            }
            if (!got) {
                std::unique_lock<std::mutex> lk(mu);
                cv_work.wait(lk, [&] { return stop.load() || generation.load() != seen; });
                if (stop.load()) return;
            }
            seen = generation.load(std::memory_order_acquire);
            work();
            if (active.fetch_sub(1, std::memory_order_acq_rel) == 1) {
                std::lock_guard<std::mutex> lk(mu);
                cv_done.notify_one();
            }
        }
    }
};

HostGatherPool::HostGatherPool(int threads) : impl_(new Impl) {
    // the calling (CUDA callback) thread works too, so spawn threads-1 helpers
    if (const char* e = std::getenv("GD_GATHER_PF")) impl_->pf_env = std::max(0, std::atoi(e));
    if (const char* e = std::getenv("GD_POOL_SPIN")) impl_->spin = std::max(0, std::atoi(e));
    for (int t = 1; t < threads; ++t) impl_->workers.emplace_back([this] { impl_->loop(); });
}

HostGatherPool::~HostGatherPool() {
    {
        std::lock_guard<std::mutex> lk(impl_->mu);
        impl_->stop.store(true);
    }
    impl_->cv_work.notify_all();
    for (auto& w : impl_->workers) w.join();
    delete impl_;
}

int HostGatherPool::threads() const { return (int)impl_->workers.size() + 1; }

double HostGatherPool::gather(const uint8_t* src, const int32_t* rows, int64_t n, int64_t R, uint8_t* dst,
                              int64_t P, bool nt) {
    const auto t0 = std::chrono::steady_clock::now();
    if (n > 0) {
        Impl& I = *impl_;
        {
            std::lock_guard<std::mutex> lk(I.mu);
            I.src = src;
            I.rows = rows;
            I.dst = dst;
            I.n = n;
            I.R = R;
            I.P = P;
            I.nt = nt;
            I.next.store(0, std::memory_order_relaxed);
            I.active.store((int)I.workers.size(), std::memory_order_relaxed);
            I.generation.fetch_add(1, std::memory_order_release);   // publishes the job fields
        }
        I.cv_work.notify_all();
        I.work();
        for (int i = 0; i < I.spin && I.active.load(std::memory_order_acquire) != 0; ++i) _mm_pause();
        if (I.active.load(std::memory_order_acquire) != 0) {
            std::unique_lock<std::mutex> lk(I.mu);
            I.cv_done.wait(lk, [&] { return I.active.load() == 0; });
        }
    }
    return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
}

}  // namespace gd
