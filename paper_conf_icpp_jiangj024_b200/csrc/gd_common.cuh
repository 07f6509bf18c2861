// gd_common.cuh — device helpers shared by the sm_100a kernels of libgd.so:
// error plumbing, handle header, Philox4x32-10, decoupled look-back tile scan,
// open-addressing hash primitives.  Independent of oracle/ (no shared code).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <utility>
#include <vector>

#include "../../include/gd.h"

namespace gd {

// ---------------------------------------------------------------- errors (host)
gd_status set_error(gd_status s, const std::string& msg);
gd_status cuda_error(cudaError_t e, const char* what);
#define GD_CUDA(call)                                              \
    do {                                                           \
        cudaError_t e_ = (call);                                   \
        if (e_ != cudaSuccess) return ::gd::cuda_error(e_, #call); \
    } while (0)

constexpr uint32_t kMagicGraph = 0x47444752u;   // "GDGR"
constexpr uint32_t kMagicBuffer = 0x47444246u;  // "GDBF"

struct HandleHdr {
    uint32_t magic;
    int device;
    unsigned int* dev_status;   // sticky GD_DEV_* bits (device memory)
};

struct DeviceGuard {            // switch to the handle's device for one API call
    int prev = -1;
    explicit DeviceGuard(int dev) {
        cudaGetDevice(&prev);
        if (prev != dev) cudaSetDevice(dev);
    }
    ~DeviceGuard() {
        int cur = -1;
        cudaGetDevice(&cur);
        if (prev >= 0 && cur != prev) cudaSetDevice(prev);
    }
};

// Debug trace (env GD_DEBUG_KERNELS=1): synchronise after each launch and log it.
bool debug_kernels();
void debug_after(const char* what, cudaStream_t s);
#define GD_DEBUG_AFTER(what, s)                       \
    do {                                              \
        if (::gd::debug_kernels()) ::gd::debug_after(what, s); \
    } while (0)

// Pointer kind: true if `p` is device-accessible memory of the current context
// (device / managed), false for host memory (pageable or pinned).
bool is_device_pointer(const void* p);
// Device address of page-locked (mapped) host memory, nullptr for anything else.
const void* mapped_host_pointer(const void* p);

// ------------------------------------------------------------ programmatic dependent launch
// Kernels of a stream-ordered chain (sampling hops, bookkeeping) start with GD_PDL_ENTRY():
// wait for the preceding kernel's completion and memory flush (griddepcontrol.wait; a no-op
// without the launch attribute), then let the next kernel of the chain be scheduled
// (griddepcontrol.launch_dependents), so its launch overlaps this kernel's tail instead of
// following it.  Nothing may touch memory before the wait.
#define GD_PDL_ENTRY()                                        \
    do {                                                      \
        asm volatile("griddepcontrol.wait;" ::: "memory");    \
        asm volatile("griddepcontrol.launch_dependents;");    \
    } while (0)

bool pdl_enabled();   // GD_PDL=0 turns the launch attribute off

template <typename... KArgs, typename... Args>
inline cudaError_t launch_chain(void (*k)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st, Args... args) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = pdl_enabled() ? 1 : 0;
    return cudaLaunchKernelEx(&cfg, k, args...);
}

// ------------------------------------------------------------ event timing (host)
// Pairs of events recorded around kernel groups; summed on read (which syncs).
struct EventTimer {
    bool on = false;
    std::vector<cudaEvent_t> pool;
    std::vector<std::pair<int, int>> pairs;   // indices into pool
    int used = 0;
    cudaEvent_t next() {
        if (used == (int)pool.size()) {
            cudaEvent_t e;
            cudaEventCreate(&e);
            pool.push_back(e);
        }
        return pool[used++];
    }
    void reset() { used = 0; pairs.clear(); }
    // Create the events of `n` more pairs now, outside the timed region: creating them on demand
    // inside it put ~12 cudaEventCreate calls per batch on the caller's thread, which contend for
    // the driver with the staged path's host-function callbacks (200-step papers100m: the device-
    // timed region ran 15-25% below the untimed e2e region on the same box).
    void reserve(int n_pairs) {
        while ((int)pool.size() < used + 2 * n_pairs) {
            cudaEvent_t e;
            if (cudaEventCreate(&e) != cudaSuccess) break;
            pool.push_back(e);
        }
    }
    // record the start of a group on `s`; returns the pair slot
    int begin(cudaStream_t s) {
        const int a = used;
        cudaEventRecord(next(), s);
        pairs.push_back({a, -1});
        return (int)pairs.size() - 1;
    }
    void end(int slot, cudaStream_t s) {
        pairs[slot].second = used;
        cudaEventRecord(next(), s);
    }
    double total_ms(int stride, int which) {   // sum the pairs with index % stride == which
        double t = 0;
        for (size_t i = which; i < pairs.size(); i += stride) {
            if (pairs[i].second < 0) continue;
            float ms = 0;
            cudaEventSynchronize(pool[pairs[i].second]);
            cudaEventElapsedTime(&ms, pool[pairs[i].first], pool[pairs[i].second]);
            t += ms;
        }
        return t;
    }
    void destroy() {
        for (auto e : pool) cudaEventDestroy(e);
        pool.clear();
        reset();
    }
};

// --------------------------------------------------------- scan tile states (host)
// Decoupled look-back needs one 64-bit status word per tile, zero before a launch.
// Two arrays alternate: each scan launch uses one and clears the other for the next
// launch on the same stream, so no memset node is needed between launches.
struct ScanState {
    unsigned long long* buf[2] = {nullptr, nullptr};
    int64_t cap = 0;     // tiles per array
    int parity = 0;
    gd_status ensure(int64_t tiles);
    void release();
    unsigned long long* use() const { return buf[parity]; }
    unsigned long long* other() const { return buf[parity ^ 1]; }
    void flip() { parity ^= 1; }
    // Tiles each array's last launch may have written, tracked on the host: a launch whose tile
    // count is known clears only what the previous launch on the other array dirtied (clearing
    // the whole array from a small grid -- the 8-block first-hop relabel of products -- cost
    // ~16 us of stores).  Launches that do not know their tile count record the whole array.
    int64_t dirty[2] = {0, 0};
    int64_t clear_n() const { return dirty[parity ^ 1]; }
    void launched(int64_t tiles) {
        dirty[parity] = tiles < cap ? tiles : cap;
        dirty[parity ^ 1] = 0;
        flip();
    }
};

// ----------------------------------------------------------------- device side
constexpr unsigned long long kFlagA = 1ull << 62;   // tile aggregate published
constexpr unsigned long long kFlagP = 2ull << 62;   // tile inclusive prefix published
constexpr unsigned long long kValMask = (1ull << 62) - 1;
constexpr uint32_t kEmpty = 0xFFFFFFFFu;            // empty hash key
constexpr uint32_t kPending = 0x80000000u;          // hash value tag: first position this hop

__device__ __forceinline__ void st_relaxed_u64(unsigned long long* p, unsigned long long v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long ld_relaxed_u64(const unsigned long long* p) {
    unsigned long long v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_relaxed_u32(uint32_t* p, uint32_t v) {
    asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t ld_relaxed_u32(const uint32_t* p) {
    uint32_t v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ void clear_tile_state(unsigned long long* p, int64_t n) {
    if (p == nullptr) return;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
         i += (int64_t)gridDim.x * blockDim.x)
        p[i] = 0ull;
}

template <typename T>
__device__ __forceinline__ T warp_inclusive_sum(T v) {
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        T n = __shfl_up_sync(0xffffffffu, v, o);
        if (lane >= o) v += n;
    }
    return v;
}
template <typename T>
__device__ __forceinline__ T warp_sum(T v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

// Decoupled look-back (Merrill & Garland 2016).  Called by all 32 lanes of ONE warp
// of the block owning `tile`, after the block computed its aggregate `agg`.  Tiles
// are processed by blocks that start in tile order (blockIdx order or a ticket), so
// every predecessor is running or done.  `base` is added to tile 0's prefix.
// Returns the exclusive prefix of `tile` (same value in every lane).
__device__ __forceinline__ long long lookback_exclusive(unsigned long long* st, long long tile,
                                                        long long agg, long long base) {
    const int lane = threadIdx.x & 31;
    if (tile == 0) {
        if (lane == 0) st_relaxed_u64(st, kFlagP | (unsigned long long)(base + agg));
        return base;
    }
    if (lane == 0) st_relaxed_u64(st + tile, kFlagA | (unsigned long long)agg);
    long long excl = 0;
    long long t = tile - 1 - lane;
    while (true) {
        unsigned long long w;
        int spins = 0;
        while (true) {
            w = (t >= 0) ? ld_relaxed_u64(st + t) : kFlagP;
            if (__all_sync(0xffffffffu, (w >> 62) != 0)) break;
            if (++spins > 8) __nanosleep(64);
        }
        const unsigned pmask = __ballot_sync(0xffffffffu, (w >> 62) == 2);
        const int first_p = pmask ? (__ffs(pmask) - 1) : 32;
        long long v = (lane <= first_p) ? (long long)(w & kValMask) : 0;
        excl += warp_sum(v);
        if (pmask) break;
        t -= 32;
    }
    if (lane == 0) st_relaxed_u64(st + tile, kFlagP | (unsigned long long)(excl + agg));
    return excl;
}

// Philox4x32-10 (Salmon et al., SC'11), the counter-based generator of reading R1.
__device__ __forceinline__ void philox4x32_10(uint32_t c[4], uint32_t k0, uint32_t k1) {
#pragma unroll
    for (int r = 0; r < 10; ++r) {
        const uint32_t lo0 = 0xD2511F53u * c[0];
        const uint32_t hi0 = __umulhi(0xD2511F53u, c[0]);
        const uint32_t lo1 = 0xCD9E8D57u * c[2];
        const uint32_t hi1 = __umulhi(0xCD9E8D57u, c[2]);
        const uint32_t n0 = hi1 ^ c[1] ^ k0;
        const uint32_t n2 = hi0 ^ c[3] ^ k1;
        c[0] = n0;
        c[1] = lo1;
        c[2] = n2;
        c[3] = lo0;
        k0 += 0x9E3779B9u;
        k1 += 0xBB67AE85u;
    }
}

// Draw t for node v at 0-based hop h of batch b, mapped to [0, j] (reading R2):
// u = y << 32 | x of Philox(ctr=(t, v, h, b), key=(lo, hi of seed)); floor(u (j+1) / 2^64).
__device__ __forceinline__ uint64_t draw_uniform(uint32_t t, uint32_t v, uint32_t h, uint32_t b,
                                                 uint64_t seed, uint64_t j) {
    uint32_t c[4] = {t, v, h, b};
    philox4x32_10(c, (uint32_t)seed, (uint32_t)(seed >> 32));
    const uint64_t u = ((uint64_t)c[1] << 32) | (uint64_t)c[0];
    return __umul64hi(u, j + 1);
}

__device__ __forceinline__ uint32_t fmix32(uint32_t h) {   // MurmurHash3 finaliser
    h ^= h >> 16;
    h *= 0x85EBCA6Bu;
    h ^= h >> 13;
    h *= 0xC2B2AE35u;
    h ^= h >> 16;
    return h;
}

}  // namespace gd
