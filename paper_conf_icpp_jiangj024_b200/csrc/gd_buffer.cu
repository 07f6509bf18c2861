// gd_buffer.cu — the slot-managed feature buffer and extraction (rows a5-a9).
//
// gd_extract(b), all stream-ordered, no host sync:
//   caller stream:  k_lookup (Alg. 1 loop 1 + miss ranks) -> k_pop_assign (loop 2:
//                   LRU standby slots, eviction, map/reverse/alias) -> [L_b]
//   stream G:       wait L_b, X_{b-1}, Xs_{b-1} -> k_gather_hits (slots -> out) -> [G_b]
//   stream Z:       wait L_b -> k_miss_copy<zero-copy> misses [0, K0) -> [X_b]
//   stream H:       wait L_b -> host gather (thread pool) of misses [K0, M) -> [E_b]
//   stream P:       wait E_b -> k_miss_copy<staged> pull of the staging slot -> [Xs_b]
//   stream J:       wait X_b, Xs_b, G_b -> [done]
// gd_buffer_release(b): k_compact (only when the ring is nearly full; exits at once
//   otherwise) -> k_release (refcount--, became-zero slots appended at the tail).
//
// Standby list: a ring of slot ids in LRU order with lazy deletion.  A slot's
// live entry is the one at pos_of_slot[slot]; removing a slot (a hit whose refcount was
// 0, Alg. 1 line 11) just sets pos_of_slot = -1.  Popping takes the first M live entries
// from head (a ticketed look-back scan that stops at the M-th), pushing appends at tail.
#include <algorithm>
#include <cstring>
#include <string>
#include <vector>
#include <cstdlib>
#include <thread>

#include <cuda.h>
#include <cudaTypedefs.h>

#include "gd_common.cuh"
#include "gd_handles.cuh"

namespace gd {

constexpr int kBThreads = 256;
#ifndef GD_BOOK_ITEMS
#define GD_BOOK_ITEMS 8   // entries per thread of the bookkeeping scans (macro for same-box A/B builds)
#endif
constexpr int kBItems = GD_BOOK_ITEMS;
constexpr int kBTile = kBThreads * kBItems;    // 2048 entries per scan tile
constexpr int kBWarps = kBThreads / 32;
constexpr int kStageRingMax = 16; // pinned chunk buffers of the copy-engine staging ring (max)
constexpr int kJobRing = 1024;   // host-function argument slots of the staged chunks
constexpr int kTimedPairs = 5;
constexpr double kZeroCopyCapCE = 0.15;   // adaptive zero-copy share cap with copy-engine staging   // per gd_extract: bookkeeping, gather, zero-copy, pull/scatter, CE copy

static int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }

// Block-wide ordered scan of per-item 0/1 flags in striped arrangement
// (item k of thread t = element k*256 + t).  ball[k] = warp ballot of round k.
// Fills s_cnt[k*8+warp] with the exclusive block offset of (round k, warp) and
// returns the block aggregate in every thread of warp 0 (others: unspecified).
__device__ __forceinline__ int block_flag_offsets(const unsigned (&ball)[kBItems], int* s_cnt) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
#pragma unroll
    for (int k = 0; k < kBItems; ++k)
        if (lane == 0) s_cnt[k * kBWarps + warp] = __popc(ball[k]);
    __syncthreads();
    int agg = 0;
    if (warp == 0) {
        constexpr int kPer = kBItems * kBWarps / 32;   // consecutive (round, warp) counts per lane
        static_assert(kPer >= 1 && kBItems * kBWarps % 32 == 0, "bookkeeping scan layout");
        int c[kPer], sum = 0;
#pragma unroll
        for (int q = 0; q < kPer; ++q) {
            c[q] = s_cnt[kPer * lane + q];
            sum += c[q];
        }
        const int inc = warp_inclusive_sum(sum);
        agg = __shfl_sync(0xffffffffu, inc, 31);
        __syncwarp();
        int run = inc - sum;
#pragma unroll
        for (int q = 0; q < kPer; ++q) {
            s_cnt[kPer * lane + q] = run;
            run += c[q];
        }
    }
    return agg;
}

// ------------------------------------------------------------------ a5: lookup
struct LookupArgs {
    const int32_t* ids;
    const int64_t* n_dev;
    int64_t N;
    int2* map;
    int32_t* pos_of_slot;
    int32_t* alias;
    int2* hitlist;                   // [n - M]: {batch position, slot} of the non-misses, list order
    int64_t* hcount;                 // n - M
    int2* misslist;                  // [M]: {batch position, node} of the misses, list order
    int64_t* mcount;
    int64_t* stats;
    unsigned long long* st;
    unsigned long long* st_clear;
    int64_t st_clear_n;
    unsigned int* status;
};

__global__ void __launch_bounds__(kBThreads) k_lookup(LookupArgs a) {
    GD_PDL_ENTRY();
    clear_tile_state(a.st_clear, a.st_clear_n);
    const int64_t n = *a.n_dev;
    const int64_t tile = blockIdx.x;
    const int64_t i0 = tile * kBTile;
    if (i0 >= n && tile != 0) return;
    __shared__ int s_cnt[kBItems * kBWarps];
    __shared__ long long s_base;
    const int t = threadIdx.x, lane = t & 31;
    unsigned ball[kBItems];
    int32_t alv[kBItems];
    // all loads of the thread's items first (ids, then their map entries), stores after: the
    // stores to map / pos_of_slot / alias could alias `ids` for the compiler, which otherwise
    // serialises the items' dependent round trips (node ids are distinct within a batch, so no
    // item reads an entry another item writes)
    int32_t vv[kBItems];
    int2 mm[kBItems];
#pragma unroll
    for (int k = 0; k < kBItems; ++k) {
        const int64_t i = i0 + (int64_t)k * kBThreads + t;
        vv[k] = (i < n) ? __ldg(a.ids + i) : -1;
    }
#pragma unroll
    for (int k = 0; k < kBItems; ++k)
        mm[k] = (vv[k] >= 0 && (int64_t)vv[k] < a.N) ? a.map[vv[k]] : make_int2(-1, 0);
#pragma unroll
    for (int k = 0; k < kBItems; ++k) {
        const int64_t i = i0 + (int64_t)k * kBThreads + t;
        bool miss = false;
        int32_t al = -1;
        if (i < n) {
            const int32_t v = vv[k];
            if (v < 0 || (int64_t)v >= a.N) {
                atomicOr(a.status, GD_DEV_BAD_ID);
            } else {
                const int2 m = mm[k];
                const int valid = m.y & 1;
                const int rc = m.y >> 1;
                if (valid) {                                   // Alg. 1 lines 8-13
                    al = m.x;
                    if (rc == 0) a.pos_of_slot[m.x] = -1;      // line 11: leave the standby list
                } else if (rc > 0) {                           // lines 14-17 (R8: not reachable
                    al = m.x;                                  // on the GPU, valid is set at alloc)
                } else {
                    miss = true;
                }
                a.map[v].y = ((rc + 1) << 1) | valid;           // line 19
            }
            a.alias[i] = al;
        }
        alv[k] = al;
        ball[k] = __ballot_sync(0xffffffffu, miss);
    }
    const int agg = block_flag_offsets(ball, s_cnt);
    if ((t >> 5) == 0) {
        const long long base = lookback_exclusive(a.st, tile, agg, 0);
        if (lane == 0) {
            s_base = base;
            const bool last = (n == 0) ? (tile == 0) : (tile == (n - 1) / kBTile);
            if (last) {
                const long long M = base + agg;
                *a.mcount = M;
                *a.hcount = n - M;
                if (a.stats) {
                    a.stats[0] = n - M;
                    a.stats[1] = M;
                }
            }
        }
    }
    __syncthreads();
    const long long base = s_base;
    const int warp = t >> 5;
    const unsigned lt = (1u << lane) - 1u;
#pragma unroll
    for (int k = 0; k < kBItems; ++k) {
        const int64_t i = i0 + (int64_t)k * kBThreads + t;
        const long long mrank = base + s_cnt[k * kBWarps + warp] + __popc(ball[k] & lt);   // misses before i
        if (ball[k] & (1u << lane))
            a.misslist[mrank] = make_int2((int32_t)i, vv[k]);
        else if (i < n)
            a.hitlist[i - mrank] = make_int2((int32_t)i, alv[k]);
    }
}

// ------------------------------------------------------- a6: pop + assign (loop 2)
struct PopArgs {
    const int32_t* ring;
    const GdCtl* ctl_in;
    GdCtl* ctl_out;
    int32_t* pos_of_slot;
    int2* map;
    int32_t* reverse;
    const int32_t* ids;
    const int2* misslist;
    const int64_t* mcount;
    int32_t* alias;
    int4* trip;
    int64_t* trip_count;
    int64_t* trip_split;            // K0 = floor(M * alpha_q16 / 2^16): first staged rank
    uint32_t alpha_q16;
    long long staged_cap;           // >= 0 (copy-engine staging): K0 = max(0, M - staged_cap)
    unsigned long long* ready;      // [S] publication tags: a reassigned slot is unpublished
    int32_t* h_nodes;               // mapped host: node ids of ranks [K0, M) (staged share)
    int64_t* h_meta;                // mapped host: {M, K0, M - K0}
    int64_t* stats;                 // caller's stats or null: [2] = K0, [3] = M - K0
    unsigned long long* ticket;     // [2]: next tile, blocks finished
    unsigned long long* done_word;
    unsigned long long epoch;
    unsigned long long* st;
    unsigned long long* st_clear;
    int64_t st_clear_n;
    unsigned int* status;
};

__device__ __forceinline__ void ticket_finish(unsigned long long* ticket) {
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence();
        const unsigned long long old = atomicAdd(ticket + 1, 1ull);
        if (old == gridDim.x - 1) {   // last block out resets the counters for the next launch
            ticket[0] = 0;
            ticket[1] = 0;
            __threadfence();
        }
    }
}

// The staged share's counts, published to mapped host memory: {M, K0, M - K0} for the host
// gather of this batch, and the word h_meta[4] = (epoch << 32 | M) (one 8-byte store): the
// host takes the newest epoch over the D slots as the latest miss count and sizes the next
// copy-engine staging share from it without querying an event or synchronising, however far
// ahead of the device it runs.
__device__ __forceinline__ void publish_meta(int64_t* h_meta, long long M, long long K0, unsigned long long epoch) {
    volatile int64_t* hm = h_meta;
    hm[0] = M;
    hm[1] = K0;
    hm[2] = M - K0;
    volatile unsigned long long* latest = (volatile unsigned long long*)(h_meta + 4);
    *latest = (epoch << 32) | (unsigned long long)(M & 0xffffffffll);
}

__global__ void __launch_bounds__(kBThreads) k_pop_assign(PopArgs a) {
    GD_PDL_ENTRY();
    clear_tile_state(a.st_clear, a.st_clear_n);
    const long long M = *a.mcount;
    const GdCtl c = *a.ctl_in;
    __shared__ long long s_tile;
    __shared__ int s_stop;
    __shared__ int s_cnt[kBItems * kBWarps];
    __shared__ long long s_base;
    const int t = threadIdx.x, lane = t & 31, warp = t >> 5;
    const long long K0 = a.staged_cap >= 0 ? (M > a.staged_cap ? M - a.staged_cap : 0)
                                           : (long long)(((unsigned long long)M * a.alpha_q16) >> 16);
    if (M == 0) {
        if (blockIdx.x == 0 && t == 0) {
            *a.ctl_out = c;
            *a.trip_count = 0;
            *a.trip_split = 0;
            if (a.h_meta) publish_meta(a.h_meta, 0, 0, a.epoch);
            if (a.stats) {
                a.stats[2] = 0;
                a.stats[3] = 0;
            }
        }
        ticket_finish(a.ticket);
        return;
    }
    while (true) {
        if (t == 0) {
            // Check `done` BEFORE taking a ticket: every ticket taken must be processed and
            // published, or the block holding the next ticket would spin on it forever.
            if (ld_relaxed_u64(a.done_word) == a.epoch) {
                s_stop = 1;
            } else {
                const long long tl = (long long)atomicAdd(a.ticket, 1ull);
                s_tile = tl;
                s_stop = (c.head + tl * kBTile >= c.tail && tl > 0);   // monotone in tl
            }
        }
        __syncthreads();
        if (s_stop) break;
        const long long tl = s_tile;
        const long long p0 = c.head + tl * kBTile;
        unsigned ball[kBItems];
        int32_t slot[kBItems];
#pragma unroll
        for (int k = 0; k < kBItems; ++k) {
            const long long p = p0 + (long long)k * kBThreads + t;
            bool live = false;
            slot[k] = -1;
            if (p < c.tail) {
                slot[k] = a.ring[p];
                live = (a.pos_of_slot[slot[k]] == (int32_t)p);
            }
            ball[k] = __ballot_sync(0xffffffffu, live);
        }
        const int agg = block_flag_offsets(ball, s_cnt);
        if (warp == 0) {
            const long long base = lookback_exclusive(a.st, tl, agg, 0);
            if (lane == 0) {
                s_base = base;
                const bool last_tile = (p0 + kBTile >= c.tail);
                if (last_tile && base + agg < M) {       // standby list ran dry (capacity rule)
                    atomicOr(a.status, GD_DEV_STANDBY_DRY);
                    GdCtl o = c;
                    o.head = c.tail;
                    *a.ctl_out = o;
                    const long long Mx = base + agg, K0x = K0 < Mx ? K0 : Mx;
                    *a.trip_count = Mx;
                    *a.trip_split = K0x;
                    if (a.h_meta) publish_meta(a.h_meta, Mx, K0x, a.epoch);
                    if (a.stats) {
                        a.stats[2] = K0x;
                        a.stats[3] = Mx - K0x;
                    }
                    __threadfence();
                    st_relaxed_u64(a.done_word, a.epoch);
                }
            }
        }
        __syncthreads();
        const long long base = s_base;
        if (base < M) {
            const unsigned lt = (1u << lane) - 1u;
            // loads of every item first ({position, node} of the miss, the slot's old node), then
            // the stores: an evicted node sits in the standby list (valid, refcount 0), so k_lookup
            // made it a hit of this batch if it is in it -- no store below aliases a load above
            long long rk[kBItems];
            int2 mi[kBItems];
            int32_t oldv[kBItems];
#pragma unroll
            for (int k = 0; k < kBItems; ++k) {
                rk[k] = -1;
                if (!(ball[k] & (1u << lane))) continue;
                const long long rank = base + s_cnt[k * kBWarps + warp] + __popc(ball[k] & lt);
                if (rank >= M) continue;
                rk[k] = rank;
                mi[k] = __ldg(a.misslist + rank);
                oldv[k] = a.reverse[slot[k]];
            }
#pragma unroll
            for (int k = 0; k < kBItems; ++k) {
                const long long rank = rk[k];
                if (rank < 0) continue;
                const int32_t s = slot[k];
                const int32_t i = mi[k].x;
                const int32_t v = mi[k].y;
                const int32_t old = oldv[k];
                if (old >= 0) a.map[old] = make_int2(-1, 0);   // invalidate (R9)
                // lines 27, 37: slot s, valid; a miss had refcount 0 before k_lookup's
                // increment (line 19), so its refcount is 1
                a.map[v] = make_int2(s, (1 << 1) | 1);
                a.reverse[s] = v;                               // line 28
                a.alias[i] = s;                                 // line 29
                a.pos_of_slot[s] = -1;
                if (a.ready) a.ready[s] = kReadyNone;           // peers stop reading it (f2)
                a.trip[rank] = make_int4(v, s, i, 0);
                if (rank >= K0 && a.h_nodes) a.h_nodes[rank - K0] = v;
                if (rank == M - 1) {
                    const long long p = p0 + (long long)k * kBThreads + t;
                    GdCtl o = c;
                    o.head = p + 1;
                    *a.ctl_out = o;
                    *a.trip_count = M;
                    *a.trip_split = K0;
                    if (a.h_meta) publish_meta(a.h_meta, M, K0, a.epoch);
                    if (a.stats) {
                        a.stats[2] = K0;
                        a.stats[3] = M - K0;
                    }
                    __threadfence();
                    st_relaxed_u64(a.done_word, a.epoch);
                }
            }
        }
        __syncthreads();
    }
    ticket_finish(a.ticket);
}

// ------------------------------------------------------------ a7: miss stream
// Copies miss ranks k in [*begin, *end) (begin == nullptr: 0) into their slot and
// their `out` row.  STAGED = false: source row = pinned host table row trip[k].x
// (zero-copy over the host link).  STAGED = true: source row = staging row k - begin
// (the contiguous phase-2 pull of rows the host gathered in phase 1).
// One 16-byte chunk per thread-iteration, UNROLL chunks in flight per thread.
template <int UNROLL, bool STAGED>
__global__ void __launch_bounds__(1024, 1) k_miss_copy(const int4* __restrict__ trip, const int64_t* __restrict__ begin,
                                                   const int64_t* __restrict__ end, const uint8_t* __restrict__ src,
                                                   uint8_t* __restrict__ slots, uint8_t* __restrict__ out, int64_t R,
                                                   int64_t P) {
    const int64_t k0 = begin ? *begin : 0;
    const int64_t M = *end - k0;
    const int64_t cpr = R >> 4;                     // 16-byte chunks per row
    const int64_t total = M * cpr;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; base < total; base += stride * UNROLL) {
        uint4 val[UNROLL];
        int64_t dsl[UNROLL], dout[UNROLL];
#pragma unroll
        for (int u = 0; u < UNROLL; ++u) {
            const int64_t idx = base + (int64_t)u * stride;
            dsl[u] = -1;
            if (idx < total) {
                const int64_t r = idx / cpr, c = idx - r * cpr;
                const int4 tr = __ldg(trip + k0 + r);
                const int64_t row = (int64_t)tr.x < P ? (int64_t)tr.x : (int64_t)tr.x % P;   // table row of node
                const uint4* sp = STAGED ? (const uint4*)(src + r * R) + c : (const uint4*)(src + row * R) + c;
                asm volatile("ld.global.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                             : "=r"(val[u].x), "=r"(val[u].y), "=r"(val[u].z), "=r"(val[u].w)
                             : "l"(sp));
                dsl[u] = (int64_t)tr.y * R + c * 16;
                dout[u] = (int64_t)tr.z * R + c * 16;
            }
        }
#pragma unroll
        for (int u = 0; u < UNROLL; ++u) {
            if (dsl[u] >= 0) {
                *(uint4*)(slots + dsl[u]) = val[u];
                *(uint4*)(out + dout[u]) = val[u];
            }
        }
    }
}

// 4-byte fallback for rows that are not a multiple of 16 bytes
template <bool STAGED>
__global__ void k_miss_copy_w4(const int4* __restrict__ trip, const int64_t* __restrict__ begin,
                               const int64_t* __restrict__ end, const uint8_t* __restrict__ src,
                               uint8_t* __restrict__ slots, uint8_t* __restrict__ out, int64_t R, int64_t P) {
    const int64_t k0 = begin ? *begin : 0;
    const int64_t M = *end - k0;
    const int64_t cpr = R >> 2;
    const int64_t total = M * cpr;
    for (int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; idx < total;
         idx += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = idx / cpr, c = idx - r * cpr;
        const int4 tr = trip[k0 + r];
        const int64_t row = (int64_t)tr.x % P;
        const uint32_t v = STAGED ? ((const uint32_t*)(src + r * R))[c] : ((const uint32_t*)(src + row * R))[c];
        ((uint32_t*)(slots + (int64_t)tr.y * R))[c] = v;
        ((uint32_t*)(out + (int64_t)tr.z * R))[c] = v;
    }
}

// ------------------------------------------------------- f2: NVLink peer buffers
// One warp per miss: look the node up in each peer's mapping table (a hint), check the
// peer slot's publication tag, copy the row over NVLink into the local slot and `out`,
// then re-read the tag (seqlock): unchanged = the copy is the node's row (a slot is
// unpublished before it is refilled, and a tag (epoch, node) never repeats); otherwise
// the miss goes to the host paths, which rewrite slot and `out`.  Unserved misses are
// compacted into trip2 (order irrelevant: every path writes the same bytes).
__global__ void __launch_bounds__(256) k_peer_probe(const int4* __restrict__ trip, const int64_t* __restrict__ tcount,
                                                    PeerView pv, int npeers, uint8_t* __restrict__ slots,
                                                    uint8_t* __restrict__ out, int64_t R, int4* __restrict__ trip2,
                                                    int64_t* __restrict__ t2count, unsigned long long* ctr) {
    // A warp takes 32 misses: every lane looks its miss up in the peers (the round trips
    // overlap), the warp copies the found rows one after another (16 B per lane), then
    // every finder re-checks its tag; the unserved misses are appended with one atomic.
    const int lane = threadIdx.x & 31;
    const int64_t M = *tcount;
    const int64_t gw = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
    const int64_t cpr = R >> 4;
    unsigned long long served = 0;
    for (int64_t k0 = gw * 32; k0 < M; k0 += warps * 32) {
        const int64_t k = k0 + lane;
        const bool have = k < M;
        int4 tr = make_int4(0, 0, 0, 0);
        int p_hit = -1, ps = -1;
        unsigned long long t1 = kReadyNone;
        if (have) {
            tr = trip[k];
            for (int p = 0; p < npeers && p_hit < 0; ++p) {
                int2 m;
                asm volatile("ld.relaxed.sys.global.v2.s32 {%0,%1}, [%2];" : "=r"(m.x), "=r"(m.y) : "l"(pv.map[p] + tr.x));
                if (m.x < 0 || !(m.y & 1)) continue;
                unsigned long long t;
                asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(t) : "l"(pv.ready[p] + m.x) : "memory");
                if (t != kReadyNone && (uint32_t)t == (uint32_t)tr.x) {
                    p_hit = p;
                    ps = m.x;
                    t1 = t;
                }
            }
        }
        unsigned found = __ballot_sync(0xffffffffu, p_hit >= 0);
        for (unsigned f = found; f; f &= f - 1) {
            const int src_lane = __ffs(f) - 1;
            const int pp = __shfl_sync(0xffffffffu, p_hit, src_lane);
            const int sps = __shfl_sync(0xffffffffu, ps, src_lane);
            const int dsl = __shfl_sync(0xffffffffu, tr.y, src_lane);
            const int dpos = __shfl_sync(0xffffffffu, tr.z, src_lane);
            const uint4* src = (const uint4*)(pv.slots[pp] + (int64_t)sps * R);
            uint4* ds = (uint4*)(slots + (int64_t)dsl * R);
            uint4* dout = (uint4*)(out + (int64_t)dpos * R);
            for (int64_t c = lane; c < cpr; c += 32) {
                uint4 v;
                asm volatile("ld.volatile.global.v4.u32 {%0,%1,%2,%3}, [%4];"
                             : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(src + c));
                ds[c] = v;
                dout[c] = v;
            }
        }
        bool ok = false;
        if (found) {
            __syncwarp();
            // load-load ordering (seqlock read side): the rows' loads before the tag re-reads
            asm volatile("fence.acq_rel.sys;" ::: "memory");
            if (p_hit >= 0) {
                unsigned long long t2;
                asm volatile("ld.relaxed.sys.global.u64 %0, [%1];" : "=l"(t2) : "l"(pv.ready[p_hit] + ps) : "memory");
                ok = t2 == t1;
            }
        }
        served += __popc(__ballot_sync(0xffffffffu, ok));
        const unsigned rest = __ballot_sync(0xffffffffu, have && !ok);
        if (rest) {
            unsigned long long base = 0;
            if (lane == 0) base = atomicAdd((unsigned long long*)t2count, (unsigned long long)__popc(rest));
            base = __shfl_sync(0xffffffffu, base, 0);
            if (have && !ok) trip2[base + __popc(rest & ((1u << lane) - 1u))] = tr;
        }
    }
    if (lane == 0 && served) atomicAdd(ctr, served);
    if (threadIdx.x == 0 && blockIdx.x == 0) atomicAdd(ctr + 1, (unsigned long long)M);
}

// After k_peer_probe: split the unserved misses between zero-copy [0, K0) and staged
// [K0, M2) (the rule k_pop_assign applies without peers) and publish the staged share's
// node list and counts to the host gather.
__global__ void k_peer_split(const int4* __restrict__ trip2, const int64_t* __restrict__ t2count,
                             int64_t* __restrict__ t2split, uint32_t alpha_q16, long long staged_cap,
                             int32_t* __restrict__ h_nodes, int64_t* __restrict__ h_meta, int64_t* __restrict__ stats,
                             unsigned long long epoch) {
    const long long M = *t2count;
    const long long K0 = staged_cap >= 0 ? (M > staged_cap ? M - staged_cap : 0)
                                         : (long long)(((unsigned long long)M * alpha_q16) >> 16);
    if (h_nodes)
        for (long long k = K0 + (long long)blockIdx.x * blockDim.x + threadIdx.x; k < M;
             k += (long long)gridDim.x * blockDim.x)
            h_nodes[k - K0] = trip2[k].x;
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        *t2split = K0;
        if (h_meta) publish_meta(h_meta, M, K0, epoch);
        if (stats) {
            stats[2] = K0;
            stats[3] = M - K0;
        }
    }
}

// Publish the batch's newly filled slots to peers once every copy into them is done.
__global__ void k_publish(const int4* __restrict__ trip, const int64_t* __restrict__ tcount,
                          unsigned long long* __restrict__ ready, unsigned long long epoch) {
    const int64_t M = *tcount;
    for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < M; k += (int64_t)gridDim.x * blockDim.x) {
        const int4 tr = trip[k];
        ready[tr.y] = (epoch << 32) | (uint32_t)tr.x;
    }
}

__global__ void k_init_ready(unsigned long long* ready, int64_t S, int64_t N, int preload) {
    for (int64_t s = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; s < S; s += (int64_t)gridDim.x * blockDim.x)
        ready[s] = (preload && s < N) ? (unsigned long long)(uint32_t)s : kReadyNone;
}

// ------------------------------------------------------------- a8: hit gather
// out[i] = slots[s] for every (i, s) of the compacted hit list (only hits are visited).
template <int UNROLL>
__global__ void __launch_bounds__(256) k_gather_hits(const int2* __restrict__ hitlist, const int64_t* __restrict__ hcount,
                                                     const uint8_t* __restrict__ slots, uint8_t* __restrict__ out, int64_t R) {
    const int64_t H = *hcount;
    const int64_t cpr = R >> 4;
    const int64_t total = H * cpr;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; base < total; base += stride * UNROLL) {
        uint4 val[UNROLL];
        int64_t dst[UNROLL];
#pragma unroll
        for (int u = 0; u < UNROLL; ++u) {
            const int64_t idx = base + (int64_t)u * stride;
            dst[u] = -1;
            if (idx < total) {
                const int64_t r = idx / cpr, c = idx - r * cpr;
                const int2 h = __ldg(hitlist + r);
                if (h.y >= 0) {
                    const uint4* src = (const uint4*)(slots + (int64_t)h.y * R) + c;
                    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                                 : "=r"(val[u].x), "=r"(val[u].y), "=r"(val[u].z), "=r"(val[u].w)
                                 : "l"(src));
                    dst[u] = (int64_t)h.x * R + c * 16;
                }
            }
        }
#pragma unroll
        for (int u = 0; u < UNROLL; ++u)
            if (dst[u] >= 0) *(uint4*)(out + dst[u]) = val[u];
    }
}

// Warp per row, U rows in flight per warp, CPL 16-byte chunks per lane (R <= 512 * CPL):
// all loads of U rows are issued before any store (measured 5.0 TB/s = 78% of the HBM
// copy peak on 512-byte rows vs 4.1 TB/s for the flat chunk loop, tools/gather_bench.cu).
// ctr != nullptr: dynamic assignment, each warp takes the next G = 8U rows from a per-launch
// counter (the last block out re-zeroes it).  Live, the gather shares the GPU with the next
// batch's sampling and with the miss copies, whose microsecond host loads clog the memory
// pipeline of the SMs they run on; with a static row partition the blocks landing on those
// SMs (or scheduled late, behind other kernels) set the kernel's duration, with dynamic
// assignment they just take fewer rows.  ctr == nullptr: static grid-stride partition.
template <int U, int CPL>
__device__ __forceinline__ void gather_rows_span(const int2* __restrict__ hitlist, int64_t r0, int64_t rend,
                                                 const uint8_t* __restrict__ slots, uint8_t* __restrict__ out,
                                                 int64_t R, int cpr, int lane) {
    int2 h[U];
    uint4 v[U][CPL];
#pragma unroll
    for (int u = 0; u < U; ++u) h[u] = (r0 + u < rend) ? __ldg(hitlist + r0 + u) : make_int2(-1, -1);
#pragma unroll
    for (int u = 0; u < U; ++u)
#pragma unroll
        for (int q = 0; q < CPL; ++q)
            if (h[u].y >= 0 && lane + 32 * q < cpr)
                asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                             : "=r"(v[u][q].x), "=r"(v[u][q].y), "=r"(v[u][q].z), "=r"(v[u][q].w)
                             : "l"((const uint4*)(slots + (int64_t)h[u].y * R) + lane + 32 * q));
#pragma unroll
    for (int u = 0; u < U; ++u)
#pragma unroll
        for (int q = 0; q < CPL; ++q)
            if (h[u].y >= 0 && lane + 32 * q < cpr) ((uint4*)(out + (int64_t)h[u].x * R))[lane + 32 * q] = v[u][q];
}

template <int U, int CPL>
__global__ void __launch_bounds__(256) k_gather_rows(const int2* __restrict__ hitlist, const int64_t* __restrict__ hcount,
                                                     const uint8_t* __restrict__ slots, uint8_t* __restrict__ out, int64_t R,
                                                     unsigned long long* __restrict__ ctr) {
    const int64_t H = *hcount;
    const int lane = threadIdx.x & 31;
    const int cpr = (int)(R >> 4);
    if (ctr == nullptr) {
        const int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
        const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
        for (int64_t r0 = w * U; r0 < H; r0 += nw * U) gather_rows_span<U, CPL>(hitlist, r0, H, slots, out, R, cpr, lane);
        return;
    }
    constexpr int G = 8 * U;
    while (true) {
        unsigned long long g0 = 0;
        if (lane == 0) g0 = atomicAdd(ctr, (unsigned long long)G);
        g0 = __shfl_sync(0xffffffffu, g0, 0);
        if ((int64_t)g0 >= H) break;
        const int64_t gend = (int64_t)g0 + G < H ? (int64_t)g0 + G : H;
        for (int64_t r0 = (int64_t)g0; r0 < gend; r0 += U) gather_rows_span<U, CPL>(hitlist, r0, gend, slots, out, R, cpr, lane);
    }
    ticket_finish(ctr);
}

// a8 variant: TMA gather.  One warp per CTA, one elected thread: a 2-D tensor map
// over the slots ([S rows x R bytes], box = one row), `cp.async.bulk.tensor.2d.tile::gather4`
// brings 4 hit rows (4 slot indices) into a shared-memory stage, and 4 bulk stores
// (`cp.async.bulk.global.shared::cta`) write them to their `out` rows.  L gathers in flight per
// CTA over P = 2L stages; a stage is reloaded once the store group that last read it is done
// (`cp.async.bulk.wait_group.read P - L`).  Rows are taken dynamically from a per-launch counter
// (G = 32 per grab; the last CTA out re-zeroes it).  Address generation and the data movement
// are the TMA unit's, so the SM issues ~2 instructions per row instead of one load + one store
// per 16 bytes per lane.  R % 16 == 0, R <= 2048 (box of R / 4 uint32 or R / 8 uint64 <= 256).
__device__ __forceinline__ uint32_t gsm_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void gsm_mbar_wait(uint32_t addr, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "GWAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra GWAIT_%=;\n}\n" ::"r"(addr),
        "r"(parity)
        : "memory");
}

template <int L>
__global__ void __launch_bounds__(32) k_gather_tma(const __grid_constant__ CUtensorMap tm, const int2* __restrict__ hitlist,
                                                   const int64_t* __restrict__ hcount, uint8_t* __restrict__ out, int64_t R,
                                                   int64_t stage_stride, unsigned long long* __restrict__ ctr) {
    constexpr int P = 2 * L;
    constexpr int G = 32;
    extern __shared__ __align__(128) uint8_t gsm[];
    __shared__ __align__(8) unsigned long long full[P];
    __shared__ int32_t spos[P][4];
    __shared__ int32_t s_n[P];
    if (threadIdx.x == 0) {
        const int64_t H = *hcount;
        for (int st = 0; st < P; ++st) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;\n" ::"r"(gsm_u32(&full[st])));
        asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
        const uint32_t stage_bytes = (uint32_t)(4 * R);
        int64_t g0 = 0, gend = 0, issued = 0, done = 0;
        bool exhausted = false;
        while (true) {
            while (!exhausted && issued - done < L) {
                if (g0 >= gend) {
                    const unsigned long long t = atomicAdd(ctr, (unsigned long long)G);
                    if ((int64_t)t >= H) {
                        exhausted = true;
                        break;
                    }
                    g0 = (int64_t)t;
                    gend = g0 + G < H ? g0 + G : H;
                }
                const int nq = gend - g0 < 4 ? (int)(gend - g0) : 4;
                const int st = (int)(issued % P);
                int32_t rows[4];
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int2 h = __ldg(hitlist + g0 + (q < nq ? q : nq - 1));
                    rows[q] = h.y;
                    if (q < nq) spos[st][q] = h.x;
                }
                s_n[st] = nq;
                g0 += nq;
                // the store group that last read stage st (iteration issued - P) has finished reading
                asm volatile("cp.async.bulk.wait_group.read %0;\n" ::"n"(P - L) : "memory");
                const uint32_t bar = gsm_u32(&full[st]);
                asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(bar), "r"(stage_bytes) : "memory");
                asm volatile(
                    "cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes"
                    " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];\n" ::"r"(gsm_u32(gsm + st * stage_stride)),
                    "l"((uint64_t)&tm), "r"(0), "r"(rows[0]), "r"(rows[1]), "r"(rows[2]), "r"(rows[3]), "r"(bar)
                    : "memory");
                ++issued;
            }
            if (done == issued) break;
            const int st = (int)(done % P);
            gsm_mbar_wait(gsm_u32(&full[st]), (uint32_t)((done / P) & 1));
            asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");
            for (int q = 0; q < s_n[st]; ++q)
                asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;\n" ::"l"(out + (int64_t)spos[st][q] * R),
                             "r"(gsm_u32(gsm + st * stage_stride + q * R)), "r"((uint32_t)R)
                             : "memory");
            asm volatile("cp.async.bulk.commit_group;\n" ::: "memory");
            ++done;
        }
        asm volatile("cp.async.bulk.wait_group 0;\n" ::: "memory");
    }
    ticket_finish(ctr);
}

// Tensor map over the slots for k_gather_tma: dims {R / e, S}, row stride R, box {R / e, 1}
// (e = 4 or 8 bytes), no swizzle.  Returns false when R does not fit one box.
static bool make_slot_map(CUtensorMap* m, const void* slots, int64_t S, int64_t R) {
    static PFN_cuTensorMapEncodeTiled_v12000 encode = nullptr;
    if (!encode) {
        cudaDriverEntryPointQueryResult q;
        cudaError_t e = cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&encode, cudaEnableDefault, &q);
        if (e != cudaSuccess || q != cudaDriverEntryPointSuccess || !encode) {
            cudaGetLastError();
            encode = nullptr;
            return false;
        }
    }
    if (R % 16 != 0 || S < 1 || S > (1ll << 31) - 1) return false;
    const int64_t e = R / 4 <= 256 ? 4 : (R / 8 <= 256 ? 8 : 0);
    if (!e) return false;
    const cuuint64_t dims[2] = {(cuuint64_t)(R / e), (cuuint64_t)S};
    const cuuint64_t strides[1] = {(cuuint64_t)R};
    const cuuint32_t box[2] = {(cuuint32_t)(R / e), 1};
    const cuuint32_t es[2] = {1, 1};
    const CUresult r = encode(m, e == 4 ? CU_TENSOR_MAP_DATA_TYPE_UINT32 : CU_TENSOR_MAP_DATA_TYPE_INT64, 2,
                              const_cast<void*>(slots), dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                              CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS;
}

__global__ void k_gather_hits_w4(const int2* __restrict__ hitlist, const int64_t* __restrict__ hcount,
                                 const uint8_t* __restrict__ slots, uint8_t* __restrict__ out, int64_t R) {
    const int64_t H = *hcount;
    const int64_t cpr = R >> 2;
    const int64_t total = H * cpr;
    for (int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; idx < total;
         idx += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = idx / cpr, c = idx - r * cpr;
        const int2 h = hitlist[r];
        if (h.y < 0) continue;
        ((uint32_t*)(out + (int64_t)h.x * R))[c] = ((const uint32_t*)(slots + (int64_t)h.y * R))[c];
    }
}

// ------------------------------------------------------------ a9: release
struct ReleaseArgs {
    const int32_t* ids;
    const int64_t* n_dev;
    int64_t N;
    int2* map;
    int32_t* ring;
    int32_t* pos_of_slot;
    const GdCtl* ctl_in;
    GdCtl* ctl_out;
    unsigned long long* st;
    unsigned long long* st_clear;
    int64_t st_clear_n;
    unsigned int* status;
};

__global__ void __launch_bounds__(kBThreads) k_release(ReleaseArgs a) {
    GD_PDL_ENTRY();
    clear_tile_state(a.st_clear, a.st_clear_n);
    const int64_t n = *a.n_dev;
    const int64_t tile = blockIdx.x;
    const int64_t i0 = tile * kBTile;
    const GdCtl c = *a.ctl_in;
    if (i0 >= n && tile != 0) return;
    __shared__ int s_cnt[kBItems * kBWarps];
    __shared__ long long s_base;
    const int t = threadIdx.x, lane = t & 31, warp = t >> 5;
    unsigned ball[kBItems];
    int32_t slot[kBItems];
    int32_t vv[kBItems];
    int2 mm[kBItems];
#pragma unroll
    for (int k = 0; k < kBItems; ++k) {   // loads first (as in k_lookup)
        const int64_t i = i0 + (int64_t)k * kBThreads + t;
        vv[k] = (i < n) ? __ldg(a.ids + i) : -1;
    }
#pragma unroll
    for (int k = 0; k < kBItems; ++k)
        mm[k] = (vv[k] >= 0 && (int64_t)vv[k] < a.N) ? a.map[vv[k]] : make_int2(-1, 0);
#pragma unroll
    for (int k = 0; k < kBItems; ++k) {
        const int64_t i = i0 + (int64_t)k * kBThreads + t;
        bool zero = false;
        slot[k] = -1;
        if (i < n) {
            const int32_t v = vv[k];
            if (v < 0 || (int64_t)v >= a.N) {
                atomicOr(a.status, GD_DEV_BAD_ID);
            } else {
                const int2 m = mm[k];
                const int rc = m.y >> 1;
                if (rc <= 0) {
                    atomicOr(a.status, GD_DEV_UNDERFLOW);
                } else {
                    a.map[v].y = ((rc - 1) << 1) | (m.y & 1);
                    zero = (rc == 1) && m.x >= 0;
                    slot[k] = m.x;
                }
            }
        }
        ball[k] = __ballot_sync(0xffffffffu, zero);
    }
    const int agg = block_flag_offsets(ball, s_cnt);
    if (warp == 0) {
        const long long base = lookback_exclusive(a.st, tile, agg, 0);
        if (lane == 0) {
            s_base = base;
            const bool last = (n == 0) ? (tile == 0) : (tile == (n - 1) / kBTile);
            if (last) {
                GdCtl o = c;
                o.tail = c.tail + base + agg;
                *a.ctl_out = o;
            }
        }
    }
    __syncthreads();
    const long long base = s_base;
    const unsigned lt = (1u << lane) - 1u;
#pragma unroll
    for (int k = 0; k < kBItems; ++k) {
        if (!(ball[k] & (1u << lane))) continue;
        const long long p = c.tail + base + s_cnt[k * kBWarps + warp] + __popc(ball[k] & lt);
        a.ring[p] = slot[k];                 // append at the tail of the standby list
        a.pos_of_slot[slot[k]] = (int32_t)p;
    }
}

// ------------------------------------------- ring compaction (rare, before a release)
struct CompactArgs {
    int32_t* ring;
    int32_t* pos_of_slot;
    const GdCtl* ctl_in;
    GdCtl* ctl_out;
    int64_t C;
    int64_t n_max;
    unsigned long long* ticket;
    unsigned long long* st;
    unsigned long long* st_clear;
    int64_t st_clear_n;
};

__global__ void __launch_bounds__(kBThreads) k_compact(CompactArgs a) {
    GD_PDL_ENTRY();
    clear_tile_state(a.st_clear, a.st_clear_n);
    const GdCtl c = *a.ctl_in;
    const bool need = (c.tail + a.n_max > c.base + a.C);
    if (!need) {
        if (blockIdx.x == 0 && threadIdx.x == 0) *a.ctl_out = c;
        return;
    }
    const long long nbase = (c.base == 0) ? a.C : 0;
    __shared__ long long s_tile;
    __shared__ int s_cnt[kBItems * kBWarps];
    __shared__ long long s_base;
    const int t = threadIdx.x, lane = t & 31, warp = t >> 5;
    const long long ntiles = (c.tail - c.head + kBTile - 1) / kBTile;
    while (true) {
        if (t == 0) s_tile = (long long)atomicAdd(a.ticket, 1ull);
        __syncthreads();
        const long long tl = s_tile;
        if (tl >= ntiles && !(tl == 0)) break;
        const long long p0 = c.head + tl * kBTile;
        unsigned ball[kBItems];
        int32_t slot[kBItems];
#pragma unroll
        for (int k = 0; k < kBItems; ++k) {
            const long long p = p0 + (long long)k * kBThreads + t;
            bool live = false;
            slot[k] = -1;
            if (p < c.tail) {
                slot[k] = a.ring[p];
                live = (a.pos_of_slot[slot[k]] == (int32_t)p);
            }
            ball[k] = __ballot_sync(0xffffffffu, live);
        }
        const int agg = block_flag_offsets(ball, s_cnt);
        if (warp == 0) {
            const long long base = lookback_exclusive(a.st, tl, agg, 0);
            if (lane == 0) {
                s_base = base;
                if (tl == (ntiles > 0 ? ntiles - 1 : 0)) {
                    GdCtl o;
                    o.base = nbase;
                    o.head = nbase;
                    o.tail = nbase + base + agg;
                    *a.ctl_out = o;
                }
            }
        }
        __syncthreads();
        const long long base = s_base;
        const unsigned lt = (1u << lane) - 1u;
#pragma unroll
        for (int k = 0; k < kBItems; ++k) {
            if (!(ball[k] & (1u << lane))) continue;
            const long long q = nbase + base + s_cnt[k * kBWarps + warp] + __popc(ball[k] & lt);
            a.ring[q] = slot[k];
            a.pos_of_slot[slot[k]] = (int32_t)q;
        }
        __syncthreads();
        if (tl >= ntiles - 1) break;
    }
    ticket_finish(a.ticket);
}

// ------------------------------------------------------------------- init
__global__ void k_init_map(int2* map, int64_t N, int preload) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < N; v += (int64_t)gridDim.x * blockDim.x)
        map[v] = preload ? make_int2((int32_t)v, 1) : make_int2(-1, 0);
}
__global__ void k_init_slots(int32_t* reverse, int32_t* pos_of_slot, int32_t* ring, int64_t S, int64_t N,
                             int preload) {
    for (int64_t s = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; s < S; s += (int64_t)gridDim.x * blockDim.x) {
        reverse[s] = (preload && s < N) ? (int32_t)s : -1;
        pos_of_slot[s] = (int32_t)s;
        ring[s] = (int32_t)s;
    }
}

}  // namespace gd

using namespace gd;

extern "C" {
static gd_status calibrate_link(gd_buffer* b);
}

static void buffer_free(gd_buffer* b) {
    if (!b) return;
    DeviceGuard guard(b->hdr.device);
    if (b->side) cudaStreamSynchronize(b->side);
    for (cudaStream_t s : {b->side, b->side_h, b->side_p, b->side_j, b->side_g, b->side_c})
        if (s) cudaStreamSynchronize(s);
    void* ptrs[] = {b->slots, b->map, b->reverse, b->pos_of_slot, b->ring, b->ctl, b->misslist, b->hitlist, b->hcount,
                    b->alias_ws, b->mcount, b->trip, b->trip_count, b->trip_split, b->tickets, b->done_word,
                    b->hdr.dev_status, b->dstage, b->ready, b->trip2, b->trip2_count, b->trip2_split, b->peer_ctr};
    for (void* p : ptrs)
        if (p) cudaFree(p);
    for (void* p : {(void*)b->stage_mem, (void*)b->hnodes_mem, (void*)b->hmeta_mem, (void*)b->ring_mem})
        if (p) cudaFreeHost(p);
    for (void* p : b->ipc_opened) cudaIpcCloseMemHandle(p);
    delete b->pool;
    b->scan.release();
    b->timer.destroy();
    for (auto* v : {&b->ev_trip, &b->ev_E, &b->ev_P, &b->ev_z0, &b->ev_z1, &b->ev_H, &b->ev_ring, &b->ev_job, &b->ev_fin})
        for (cudaEvent_t e : *v)
            if (e) cudaEventDestroy(e);
    for (cudaEvent_t e : {b->ev_L, b->ev_X, b->ev_Xs, b->ev_G, b->ev_chunk, b->ev_S, b->ev_ref})
        if (e) cudaEventDestroy(e);
    for (cudaStream_t s : {b->side, b->side_h, b->side_p, b->side_j, b->side_g, b->side_c})
        if (s) cudaStreamDestroy(s);
    if (b->registered) cudaHostUnregister((void*)b->host_feat);
    b->hdr.magic = 0;
    delete b;
}

extern "C" {

gd_status gd_buffer_init(const void* host_feat, int64_t num_nodes, int64_t row_bytes, int64_t capacity_slots,
                         int32_t max_inflight, int64_t max_nodes_per_batch, int preload, int device,
                         gd_buffer** out) {
    return gd_buffer_init_mod(host_feat, num_nodes, num_nodes, row_bytes, capacity_slots, max_inflight,
                              max_nodes_per_batch, preload, device, out);
}

gd_status gd_buffer_init_mod(const void* host_feat, int64_t table_rows, int64_t num_nodes, int64_t row_bytes,
                             int64_t capacity_slots, int32_t max_inflight, int64_t max_nodes_per_batch, int preload,
                             int device, gd_buffer** out) {
    if (!host_feat || !out) return set_error(GD_ERR_INVALID, "gd_buffer_init: null pointer");
    if (table_rows < 1 || table_rows > num_nodes)
        return set_error(GD_ERR_INVALID, "gd_buffer_init_mod: need 1 <= table_rows <= num_nodes");
    if (num_nodes < 1 || num_nodes > 0x7FFFFFFFLL || row_bytes < 4 || (row_bytes & 3) ||
        capacity_slots < 1 || max_inflight < 1 || max_nodes_per_batch < 1)
        return set_error(GD_ERR_INVALID, "gd_buffer_init: bad size (row_bytes must be a positive multiple of 4)");
    if (preload && capacity_slots < num_nodes)
        return set_error(GD_ERR_INVALID, "gd_buffer_init: preload needs capacity_slots >= num_nodes");
    const int64_t need = std::min<int64_t>(num_nodes, (int64_t)max_inflight * max_nodes_per_batch);
    if (capacity_slots < need)
        return set_error(GD_ERR_CAPACITY, "gd_buffer_init: capacity_slots < min(N, max_inflight * max_nodes_per_batch)"
                                          " (the N_e x M_b reservation, P:122)");
    const int64_t C = 2 * capacity_slots + max_nodes_per_batch;
    if (2 * C >= 0x7FFFFFFFLL) return set_error(GD_ERR_INVALID, "gd_buffer_init: capacity too large");
    DeviceGuard guard(device);
    GD_CUDA(cudaSetDevice(device));
    gd_buffer* b = new gd_buffer();
    b->hdr.magic = kMagicBuffer;
    b->hdr.device = device;
    b->N = num_nodes;
    b->R = row_bytes;
    b->S = capacity_slots;
    b->C = C;
    b->n_max = max_nodes_per_batch;
    b->Q = max_inflight;
    b->preload = preload;
    b->host_feat = host_feat;
    b->P = table_rows;
    b->D = max_inflight + 2;
    auto fail = [&](gd_status s) {
        buffer_free(b);
        return s;
    };
    // map the pinned host table (the SSD stand-in) into the device address space
    cudaPointerAttributes pa;
    bool pinned = (cudaPointerGetAttributes(&pa, host_feat) == cudaSuccess && pa.type == cudaMemoryTypeHost);
    cudaGetLastError();
    if (!pinned) {
        cudaError_t e = cudaHostRegister((void*)host_feat, (size_t)table_rows * row_bytes,
                                         cudaHostRegisterMapped | cudaHostRegisterPortable);
        if (e != cudaSuccess) return fail(cuda_error(e, "cudaHostRegister(host_feat)"));
        b->registered = true;
    }
    void* dptr = nullptr;
    {
        cudaError_t e = cudaHostGetDevicePointer(&dptr, (void*)host_feat, 0);
        if (e != cudaSuccess) return fail(cuda_error(e, "cudaHostGetDevicePointer(host_feat)"));
    }
    b->feat_dev = (const uint8_t*)dptr;

    const int64_t nm = max_nodes_per_batch;
#define GD_ALLOC(ptr, bytes)                                                          \
    do {                                                                              \
        cudaError_t e_ = cudaMalloc((void**)&(ptr), (size_t)(bytes));                 \
        if (e_ != cudaSuccess) return fail(cuda_error(e_, "cudaMalloc " #ptr));       \
    } while (0)
    GD_ALLOC(b->hdr.dev_status, sizeof(unsigned int));
    GD_ALLOC(b->slots, capacity_slots * row_bytes);
    GD_ALLOC(b->map, num_nodes * sizeof(int2));
    GD_ALLOC(b->reverse, capacity_slots * sizeof(int32_t));
    GD_ALLOC(b->pos_of_slot, capacity_slots * sizeof(int32_t));
    GD_ALLOC(b->ring, 2 * C * sizeof(int32_t));
    GD_ALLOC(b->ctl, 2 * sizeof(GdCtl));
    GD_ALLOC(b->misslist, nm * sizeof(int2));
    GD_ALLOC(b->hitlist, (int64_t)b->D * nm * sizeof(int2));
    GD_ALLOC(b->hcount, (int64_t)b->D * sizeof(int64_t));
    GD_ALLOC(b->alias_ws, (int64_t)b->D * nm * sizeof(int32_t));
    GD_ALLOC(b->mcount, sizeof(int64_t));
    GD_ALLOC(b->trip, (int64_t)b->D * nm * sizeof(int4));
    GD_ALLOC(b->trip_count, b->D * sizeof(int64_t));
    GD_ALLOC(b->trip_split, b->D * sizeof(int64_t));
    GD_ALLOC(b->tickets, 6 * sizeof(unsigned long long));
    GD_ALLOC(b->done_word, sizeof(unsigned long long));
    GD_ALLOC(b->ready, capacity_slots * sizeof(unsigned long long));
    GD_ALLOC(b->trip2, (int64_t)b->D * nm * sizeof(int4));
    GD_ALLOC(b->trip2_count, b->D * sizeof(int64_t));
    GD_ALLOC(b->trip2_split, b->D * sizeof(int64_t));
    GD_ALLOC(b->peer_ctr, 2 * sizeof(unsigned long long));
#undef GD_ALLOC
    gd_status s = b->scan.ensure(std::max(cdiv(nm, kBTile), cdiv(C, kBTile)) + 1);
    if (s != GD_OK) return fail(s);
    GdCtl c0[2];
    c0[0].head = 0;
    c0[0].tail = capacity_slots;
    c0[0].base = 0;
    c0[1] = c0[0];
    if (cudaMemcpy(b->ctl, c0, sizeof(c0), cudaMemcpyHostToDevice) != cudaSuccess ||
        cudaMemset(b->hdr.dev_status, 0, sizeof(unsigned int)) != cudaSuccess ||
        cudaMemset(b->tickets, 0, 6 * sizeof(unsigned long long)) != cudaSuccess ||
        cudaMemset(b->done_word, 0, sizeof(unsigned long long)) != cudaSuccess ||
        cudaMemset(b->trip_count, 0, b->D * sizeof(int64_t)) != cudaSuccess ||
        cudaMemset(b->trip_split, 0, b->D * sizeof(int64_t)) != cudaSuccess ||
        cudaMemset(b->trip2_count, 0, b->D * sizeof(int64_t)) != cudaSuccess ||
        cudaMemset(b->trip2_split, 0, b->D * sizeof(int64_t)) != cudaSuccess ||
        cudaMemset(b->peer_ctr, 0, 2 * sizeof(unsigned long long)) != cudaSuccess)
        return fail(cuda_error(cudaGetLastError(), "gd_buffer_init: init copies"));
    k_init_map<<<148 * 8, 256>>>(b->map, num_nodes, preload);
    k_init_slots<<<148 * 8, 256>>>(b->reverse, b->pos_of_slot, b->ring, capacity_slots, num_nodes, preload);
    k_init_ready<<<148 * 8, 256>>>(b->ready, capacity_slots, num_nodes, preload);
    if (preload) {
        for (int64_t v0 = 0; v0 < num_nodes; v0 += table_rows) {   // slot v holds row v mod P
            const int64_t nr = std::min(table_rows, num_nodes - v0);
            cudaError_t e = cudaMemcpy(b->slots + v0 * row_bytes, host_feat, (size_t)nr * row_bytes,
                                       cudaMemcpyHostToDevice);
            if (e != cudaSuccess) return fail(cuda_error(e, "gd_buffer_init: preload copy"));
        }
    }
    {
        cudaError_t e = cudaDeviceSynchronize();
        if (e != cudaSuccess) return fail(cuda_error(e, "gd_buffer_init: init kernels"));
    }
    for (cudaStream_t* sp : {&b->side, &b->side_h, &b->side_p, &b->side_j, &b->side_c})
        if (cudaStreamCreateWithFlags(sp, cudaStreamNonBlocking) != cudaSuccess)
            return fail(cuda_error(cudaGetLastError(), "gd_buffer_init: stream"));
    {   // the hit gather (stream G) at the highest stream priority: when SMs free up, the block
        // scheduler starts its blocks before those of the sampling / miss-copy kernels beside it
        // (env GD_GATHER_PRIORITY=0: default priority); GD_GATHER_DYNAMIC=0: static row partition
        int lo = 0, hi = 0;
        cudaDeviceGetStreamPriorityRange(&lo, &hi);
        const char* e = std::getenv("GD_GATHER_PRIORITY");
        if (cudaStreamCreateWithPriority(&b->side_g, cudaStreamNonBlocking, (e && e[0] == '0') ? lo : hi) != cudaSuccess)
            return fail(cuda_error(cudaGetLastError(), "gd_buffer_init: stream"));
        const char* d = std::getenv("GD_GATHER_DYNAMIC");
        b->gather_dynamic = !(d && d[0] == '0');
        if (const char* e2 = std::getenv("GD_GATHER_BPS")) b->gather_bps = std::max(1, std::min(8, std::atoi(e2)));
        if (const char* e2 = std::getenv("GD_GATHER_U")) b->gather_u = std::atoi(e2) == 8 ? 8 : 4;
        if (const char* e2 = std::getenv("GD_ZC_AFTER_GATHER")) b->zc_after_gather = e2[0] != '0';
        // GD_GATHER_TMA=1: the TMA gather4 variant of a8 (rows <= 2048 B, multiples of 16)
        const char* t = std::getenv("GD_GATHER_TMA");
        if (t && t[0] == '1' && make_slot_map(&b->slot_map, b->slots, capacity_slots, row_bytes)) {
            const int64_t stride = (4 * row_bytes + 127) / 128 * 128;
            if (cudaFuncSetAttribute(k_gather_tma<4>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)(8 * stride)) == cudaSuccess)
                b->gather_tma = true;
            cudaGetLastError();
        }
    }
    for (cudaEvent_t* ep : {&b->ev_L, &b->ev_X, &b->ev_Xs, &b->ev_G, &b->ev_S})
        if (cudaEventCreateWithFlags(ep, cudaEventDisableTiming) != cudaSuccess)
            return fail(cuda_error(cudaGetLastError(), "gd_buffer_init: event"));
    // Only the events an elapsed time is read from carry timing (recording a timing event between
    // chained kernels / copies costs throughput: per-kernel pairs in bench's timed region cost ~18%):
    // ev_z0 / ev_z1 (zero-copy rate, recorded on every 8th batch) and ev_fin (share tuner only).
    for (auto* v : {&b->ev_trip, &b->ev_E, &b->ev_P, &b->ev_z0, &b->ev_z1, &b->ev_H, &b->ev_fin}) {
        const bool timing = (v == &b->ev_z0 || v == &b->ev_z1 || v == &b->ev_fin);
        v->assign(b->D, nullptr);
        for (int d = 0; d < b->D; ++d)
            if (cudaEventCreateWithFlags(&(*v)[d], timing ? cudaEventDefault : cudaEventDisableTiming) != cudaSuccess)
                return fail(cuda_error(cudaGetLastError(), "gd_buffer_init: event"));
    }
    // staged miss path (phase 1 host gather + phase 2 contiguous pull): on by default
    // unless every row is resident from the start; GD_HOST_THREADS overrides the width.
    const int hw = (int)std::thread::hardware_concurrency();
    int threads = preload ? 0 : std::min(13, std::max(1, hw - 3));
    if (const char* e = std::getenv("GD_HOST_THREADS")) threads = std::max(0, std::atoi(e));
    double share = -1.0;
    if (const char* e = std::getenv("GD_ZERO_COPY_SHARE")) share = std::atof(e);
    int zcb = 0, plb = 0;
    if (const char* e = std::getenv("GD_ZC_BLOCKS")) zcb = std::atoi(e);
    if (const char* e = std::getenv("GD_PULL_BLOCKS")) plb = std::atoi(e);
    if (const char* e = std::getenv("GD_STAGE_COPY_ENGINE")) b->ce_mode = e[0] != '0';
    s = gd_buffer_config(b, threads, share, zcb, plb);
    if (s != GD_OK) return fail(s);
    *out = b;
    return GD_OK;
}

gd_status gd_buffer_destroy(gd_buffer* b) {
    if (!b) return GD_OK;
    if (b->hdr.magic != kMagicBuffer) return set_error(GD_ERR_INVALID, "gd_buffer_destroy: bad handle");
    buffer_free(b);
    return GD_OK;
}

gd_status gd_buffer_config(gd_buffer* b, int host_threads, double zero_copy_share, int zc_blocks, int pull_blocks) {
    if (!b || b->hdr.magic != kMagicBuffer) return set_error(GD_ERR_INVALID, "gd_buffer_config: bad handle");
    if (host_threads < 0 || host_threads > 256 || zero_copy_share > 1.0 || zc_blocks > 4096 || pull_blocks > 4096)
        return set_error(GD_ERR_INVALID, "gd_buffer_config: host_threads in [0, 256], zero_copy_share <= 1, blocks <= 4096");
    if (zc_blocks > 0) b->zc_blocks = zc_blocks;
    if (pull_blocks > 0) b->pull_blocks = pull_blocks;
    DeviceGuard guard(b->hdr.device);
    for (cudaStream_t s : {b->side, b->side_h, b->side_p, b->side_j, b->side_g, b->side_c})
        if (s) GD_CUDA(cudaStreamSynchronize(s));
    if (host_threads > 0 && !b->stage_mem) {
        const int D = b->D;
        const int64_t nm = b->n_max;
        GD_CUDA(cudaHostAlloc((void**)&b->stage_mem, (size_t)D * nm * b->R, cudaHostAllocMapped | cudaHostAllocPortable));
        GD_CUDA(cudaHostAlloc((void**)&b->hnodes_mem, (size_t)D * nm * sizeof(int32_t), cudaHostAllocMapped | cudaHostAllocPortable));
        GD_CUDA(cudaHostAlloc((void**)&b->hmeta_mem, (size_t)D * 8 * sizeof(int64_t), cudaHostAllocMapped | cudaHostAllocPortable));
        std::memset(b->hmeta_mem, 0, (size_t)D * 8 * sizeof(int64_t));
        b->stg.assign(D, StagedSlot());
        for (int d = 0; d < D; ++d) {
            b->stg[d].owner = b;
            b->stg[d].d = d;
            b->stg[d].staging = b->stage_mem + (size_t)d * nm * b->R;
            b->stg[d].h_nodes = b->hnodes_mem + (size_t)d * nm;
            b->stg[d].h_meta = b->hmeta_mem + 8 * d;
        }
    }
    if (b->pool && (host_threads == 0 || b->pool->threads() != host_threads)) {
        delete b->pool;
        b->pool = nullptr;
    }
    if (host_threads > 0 && !b->pool) b->pool = new HostGatherPool(host_threads);
    if (host_threads > 0 && b->ce_mode && !b->dstage)
        GD_CUDA(cudaMalloc(&b->dstage, (size_t)b->D * b->n_max * b->R));
    if ((host_threads == 0 || !b->ce_mode) && b->dstage) {
        GD_CUDA(cudaFree(b->dstage));
        b->dstage = nullptr;
    }
    // chunked staging ring (copy-engine mode): env GD_STAGE_CHUNK_KB, default 8 MB chunks;
    // 0 = one chunk per batch into the batch's full pinned staging slot
    // chunked staging ring: env GD_STAGE_CHUNK_KB fixes the chunk size (0 = one chunk per batch
    // into the batch's full pinned staging slot); by default the ring holds 16 MB chunks and each
    // batch uses a sixth of its staged share, clamped to [8, 16] MB (measured, papers100m 8 / 12 /
    // 16 / 24 / 32 MB: 496 / 528 / 524 / 509 / 485 batches/s; mag240m, ~33 MB staged per batch,
    // 8 MB 1087 vs 16 MB 979; friendster 8 MB 98.1 vs 16 MB 103.3): enough chunks that the copy
    // engine starts early in a batch, few enough that per-chunk callback costs stay small
    int64_t chunk_kb = 16384;
    b->chunk_adaptive = true;
    if (const char* e = std::getenv("GD_STAGE_CHUNK_KB")) {
        chunk_kb = std::max<int64_t>(0, std::atoll(e));
        b->chunk_adaptive = false;
    }
    const int64_t rows = (host_threads > 0 && b->ce_mode && chunk_kb > 0)
                             ? std::min<int64_t>(b->n_max, std::max<int64_t>(1, (chunk_kb << 10) / b->R)) : 0;
    if (rows != b->stage_chunk_rows) {
        if (b->ring_mem) GD_CUDA(cudaFreeHost(b->ring_mem));
        b->ring_mem = nullptr;
        b->stage_chunk_rows = rows;
        if (rows > 0) {
            b->stage_ring = 4;
            if (const char* e = std::getenv("GD_STAGE_RING")) b->stage_ring = std::max(2, std::min(kStageRingMax, std::atoi(e)));
            GD_CUDA(cudaHostAlloc((void**)&b->ring_mem, (size_t)b->stage_ring * rows * b->R, cudaHostAllocPortable));
            if (b->ev_ring.empty()) {
                b->ev_ring.assign(kStageRingMax, nullptr);
                for (auto& e : b->ev_ring) GD_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
                GD_CUDA(cudaEventCreateWithFlags(&b->ev_chunk, cudaEventDisableTiming));
            }
            if (b->ev_job.empty()) {
                b->ev_job.assign(kJobRing, nullptr);
                for (auto& e : b->ev_job) GD_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
            }
            b->jobs.assign((size_t)kJobRing, ChunkJob());
        }
    }
    b->host_threads = host_threads;
    b->m_est = 0;
    b->alpha_fixed = zero_copy_share >= 0;
    b->alpha = host_threads == 0 ? 1.0 : (zero_copy_share >= 0 ? zero_copy_share : 0.2);
    b->r_host = 0;
    b->r_zc = 0;
    b->rate_samples = 0;
    b->rated_batch = b->batch_counter - 1;
    b->tune = ShareTuner();
    {
        const char* e = std::getenv("GD_SHARE_TUNER");
        // off by default: measured no better than the model share on a fast-host box (papers100m
        // 511 vs 519, mag240m 923 vs 1014 batches/s) and its probes of large shares can hit the
        // copy-engine collapse inside a short timed region; GD_SHARE_TUNER=1 enables
        b->tune.on = host_threads > 0 && !b->alpha_fixed && b->ce_mode && (e && e[0] == '1');
        for (int k = 0; k < 64; ++k) b->tune.mb[k] = -1;
        b->tune.change_batch = b->batch_counter;
        if (!b->ev_ref) GD_CUDA(cudaEventCreate(&b->ev_ref));
        GD_CUDA(cudaEventRecord(b->ev_ref, b->side_j));
    }
    if (host_threads > 0 && !b->alpha_fixed) {
        gd_status st = calibrate_link(b);
        if (st != GD_OK) return st;
    }
    return GD_OK;
}

gd_status gd_buffer_stage_mode(gd_buffer* b, int copy_engine) {
    if (!b || b->hdr.magic != kMagicBuffer) return set_error(GD_ERR_INVALID, "gd_buffer_stage_mode: bad handle");
    if (copy_engine != 0 && copy_engine != 1) return set_error(GD_ERR_INVALID, "gd_buffer_stage_mode: 0 or 1");
    if ((copy_engine == 1) == b->ce_mode) return GD_OK;
    b->ce_mode = copy_engine == 1;
    return gd_buffer_config(b, b->host_threads, b->alpha_fixed ? b->alpha : -1.0, 0, 0);
}

// ------------------------------------------------------------------ f2: peers
static gd_status drain_streams(gd_buffer* b) {
    for (cudaStream_t s : {b->side, b->side_h, b->side_p, b->side_j, b->side_g, b->side_c})
        if (s) GD_CUDA(cudaStreamSynchronize(s));
    return GD_OK;
}

static gd_status set_peers(gd_buffer* b, int n, const int2* const* maps, const unsigned long long* const* readys,
                           const uint8_t* const* slots) {
    if (n < 0 || n > kMaxPeers) return set_error(GD_ERR_INVALID, "gd_buffer_peer_attach: 0..7 peers");
    for (int p = 0; p < kMaxPeers; ++p) {
        b->peers.map[p] = p < n ? maps[p] : nullptr;
        b->peers.ready[p] = p < n ? readys[p] : nullptr;
        b->peers.slots[p] = p < n ? slots[p] : nullptr;
    }
    b->npeers = n;
    return GD_OK;
}

// A buffer maintains its f2 publication tags (cleared by k_pop_assign on reassignment, set by
// k_publish) only from the moment another buffer can read them: in-process attach as someone's
// peer, or an IPC export.  Until then it skips both (a random 8-byte write per miss, twice).
// Switching on rebuilds every tag from the mapping table once the buffer's streams are idle
// (so every valid node's row is in its slot): slot s of valid node v gets (epoch << 32 | v)
// with the current epoch, every other slot none; a tag left from before can never vouch for
// a slot's current row.
__global__ void k_republish(const int2* __restrict__ map, int64_t N, unsigned long long* __restrict__ ready,
                            unsigned long long epoch) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < N; v += (int64_t)gridDim.x * blockDim.x) {
        const int2 m = map[v];
        if ((m.y & 1) && m.x >= 0) ready[m.x] = (epoch << 32) | (uint32_t)v;
    }
}

static gd_status ensure_publishing(gd_buffer* q) {
    if (q->publish) return GD_OK;
    DeviceGuard guard(q->hdr.device);
    gd_status s = drain_streams(q);
    if (s != GD_OK) return s;
    k_init_ready<<<148 * 8, 256, 0, q->side_j>>>(q->ready, q->S, q->N, 0);
    k_republish<<<148 * 8, 256, 0, q->side_j>>>(q->map, q->N, q->ready, (unsigned long long)q->epoch);
    GD_CUDA(cudaStreamSynchronize(q->side_j));
    q->publish = true;
    return GD_OK;
}

gd_status gd_buffer_peer_attach(gd_buffer* b, int npeers, gd_buffer* const* peers) {
    if (!b || b->hdr.magic != kMagicBuffer) return set_error(GD_ERR_INVALID, "gd_buffer_peer_attach: bad handle");
    if (npeers < 0 || npeers > kMaxPeers || (npeers > 0 && !peers))
        return set_error(GD_ERR_INVALID, "gd_buffer_peer_attach: 0..7 peers");
    const int2* maps[kMaxPeers];
    const unsigned long long* readys[kMaxPeers];
    const uint8_t* slots[kMaxPeers];
    DeviceGuard guard(b->hdr.device);
    for (int p = 0; p < npeers; ++p) {
        gd_buffer* q = peers[p];
        if (!q || q->hdr.magic != kMagicBuffer || q == b)
            return set_error(GD_ERR_INVALID, "gd_buffer_peer_attach: bad peer handle");
        if (q->N != b->N || q->R != b->R || q->P != b->P)
            return set_error(GD_ERR_INVALID, "gd_buffer_peer_attach: peer has another graph size / row size / table");
        if (q->hdr.device != b->hdr.device) {
            int can = 0;
            GD_CUDA(cudaDeviceCanAccessPeer(&can, b->hdr.device, q->hdr.device));
            if (!can) return set_error(GD_ERR_INVALID, "gd_buffer_peer_attach: no P2P path between the devices");
            cudaError_t e = cudaDeviceEnablePeerAccess(q->hdr.device, 0);
            if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) return cuda_error(e, "cudaDeviceEnablePeerAccess");
            cudaGetLastError();
        }
        maps[p] = q->map;
        readys[p] = q->ready;
        slots[p] = q->slots;
    }
    for (int p = 0; p < npeers; ++p) {
        gd_status st = ensure_publishing(peers[p]);
        if (st != GD_OK) return st;
    }
    gd_status s = drain_streams(b);
    if (s != GD_OK) return s;
    return set_peers(b, npeers, maps, readys, slots);
}

// blob layout: int64 {magic, N, R, P, S}, then 3 cudaIpcMemHandle_t (map, ready, slots)
static constexpr int64_t kBlobMagic = 0x4744504545520001ll;   // "GDPEER" v1

gd_status gd_buffer_peer_export_ipc(gd_buffer* b, void* blob, int64_t blob_bytes) {
    if (!b || b->hdr.magic != kMagicBuffer) return set_error(GD_ERR_INVALID, "gd_buffer_peer_export_ipc: bad handle");
    if (!blob || blob_bytes < GD_PEER_BLOB_BYTES) return set_error(GD_ERR_INVALID, "gd_buffer_peer_export_ipc: blob too small");
    DeviceGuard guard(b->hdr.device);
    {
        gd_status st = ensure_publishing(b);
        if (st != GD_OK) return st;
    }
    std::memset(blob, 0, GD_PEER_BLOB_BYTES);
    int64_t* h = (int64_t*)blob;
    h[0] = kBlobMagic;
    h[1] = b->N;
    h[2] = b->R;
    h[3] = b->P;
    h[4] = b->S;
    cudaIpcMemHandle_t* mh = (cudaIpcMemHandle_t*)(h + 5);
    GD_CUDA(cudaIpcGetMemHandle(&mh[0], b->map));
    GD_CUDA(cudaIpcGetMemHandle(&mh[1], b->ready));
    GD_CUDA(cudaIpcGetMemHandle(&mh[2], b->slots));
    return GD_OK;
}

gd_status gd_buffer_peer_attach_ipc(gd_buffer* b, int npeers, const void* blobs) {
    if (!b || b->hdr.magic != kMagicBuffer) return set_error(GD_ERR_INVALID, "gd_buffer_peer_attach_ipc: bad handle");
    if (npeers < 0 || npeers > kMaxPeers || (npeers > 0 && !blobs))
        return set_error(GD_ERR_INVALID, "gd_buffer_peer_attach_ipc: 0..7 peers");
    DeviceGuard guard(b->hdr.device);
    gd_status s = drain_streams(b);
    if (s != GD_OK) return s;
    set_peers(b, 0, nullptr, nullptr, nullptr);
    for (void* p : b->ipc_opened) cudaIpcCloseMemHandle(p);
    b->ipc_opened.clear();
    const int2* maps[kMaxPeers];
    const unsigned long long* readys[kMaxPeers];
    const uint8_t* slots[kMaxPeers];
    for (int p = 0; p < npeers; ++p) {
        const int64_t* h = (const int64_t*)((const uint8_t*)blobs + (int64_t)p * GD_PEER_BLOB_BYTES);
        if (h[0] != kBlobMagic) return set_error(GD_ERR_INVALID, "gd_buffer_peer_attach_ipc: not a peer blob");
        if (h[1] != b->N || h[2] != b->R || h[3] != b->P)
            return set_error(GD_ERR_INVALID, "gd_buffer_peer_attach_ipc: peer has another graph size / row size / table");
        const cudaIpcMemHandle_t* mh = (const cudaIpcMemHandle_t*)(h + 5);
        void* ptr[3];
        for (int k = 0; k < 3; ++k) {
            cudaError_t e = cudaIpcOpenMemHandle(&ptr[k], mh[k], cudaIpcMemLazyEnablePeerAccess);
            if (e != cudaSuccess) return cuda_error(e, "gd_buffer_peer_attach_ipc: cudaIpcOpenMemHandle");
            b->ipc_opened.push_back(ptr[k]);
        }
        maps[p] = (const int2*)ptr[0];
        readys[p] = (const unsigned long long*)ptr[1];
        slots[p] = (const uint8_t*)ptr[2];
    }
    return set_peers(b, npeers, maps, readys, slots);
}

gd_status gd_buffer_peer_stats(gd_buffer* b, int64_t* served, int64_t* probed) {
    if (!b || b->hdr.magic != kMagicBuffer) return set_error(GD_ERR_INVALID, "gd_buffer_peer_stats: bad handle");
    DeviceGuard guard(b->hdr.device);
    gd_status s = drain_streams(b);
    if (s != GD_OK) return s;
    GD_CUDA(cudaDeviceSynchronize());
    unsigned long long c[2];
    GD_CUDA(cudaMemcpy(c, b->peer_ctr, sizeof(c), cudaMemcpyDeviceToHost));
    if (served) *served = (int64_t)c[0];
    if (probed) *probed = (int64_t)c[1];
    return GD_OK;
}

gd_status gd_buffer_timing(gd_buffer* b, int enable) {
    if (!b || b->hdr.magic != kMagicBuffer) return set_error(GD_ERR_INVALID, "gd_buffer_timing: bad handle");
    DeviceGuard guard(b->hdr.device);
    if (enable) {
        for (cudaStream_t s : {b->side, b->side_h, b->side_p, b->side_j, b->side_g, b->side_c}) GD_CUDA(cudaStreamSynchronize(s));
        b->timer.reset();
        b->timer.reserve(kTimedPairs * 4096);   // events for 4096 batches, created before the timed region
        b->timer_host_ms = 0;
    }
    b->timer.on = enable != 0;
    return GD_OK;
}

gd_status gd_buffer_timing_read(gd_buffer* b, double* ms, int64_t* batches) {
    if (!b || b->hdr.magic != kMagicBuffer) return set_error(GD_ERR_INVALID, "gd_buffer_timing_read: bad handle");
    DeviceGuard guard(b->hdr.device);
    for (cudaStream_t s : {b->side, b->side_h, b->side_p, b->side_j, b->side_g, b->side_c}) GD_CUDA(cudaStreamSynchronize(s));
    if (ms) {
        // pair order per batch (begin() order in gd_extract): bookkeeping, gather,
        // zero-copy, copy-engine H2D, pull / scatter
        for (int k = 0; k < 3; ++k) ms[k] = b->timer.total_ms(kTimedPairs, k);
        ms[3] = b->timer.total_ms(kTimedPairs, 4);
        ms[4] = b->timer_host_ms;
        ms[6] = b->timer.total_ms(kTimedPairs, 3);
        ms[5] = b->alpha;
    }
    if (batches) *batches = (int64_t)b->timer.pairs.size() / kTimedPairs;
    GD_CUDA(cudaGetLastError());
    return GD_OK;
}

void* gd_buffer_side_stream(gd_buffer* b) { return (b && b->hdr.magic == kMagicBuffer) ? (void*)b->side : nullptr; }

// Phase 1 of the staged share, run by the CUDA callback thread of stream H once the
// pop kernel has written the node list and counts to mapped host memory.
static void CUDART_CB host_gather_cb(void* arg) {
    StagedSlot* ss = (StagedSlot*)arg;
    gd_buffer* b = ss->owner;
    const int64_t n = ((volatile int64_t*)ss->h_meta)[2];
    ss->cpu_ms = b->pool->gather((const uint8_t*)b->host_feat, ss->h_nodes, n, b->R, ss->staging, b->P);
    if (b->timer.on) b->timer_host_ms += ss->cpu_ms;   // serialised on stream H
}

// One chunk of the staged share (copy-engine mode): ranks [lo, min(hi, n)) into a ring
// buffer with ordinary stores (it is read by DMA right after, while still cached).
static void CUDART_CB chunk_gather_cb(void* arg) {
    ChunkJob* j = (ChunkJob*)arg;
    StagedSlot* ss = j->ss;
    gd_buffer* b = ss->owner;
    const int64_t staged = ((volatile int64_t*)ss->h_meta)[2];
    const int64_t n = std::min<int64_t>(staged, j->hi);
    if (j->first) ss->cpu_ms = 0;
    const double ms = n > j->lo ? b->pool->gather((const uint8_t*)b->host_feat, ss->h_nodes + j->lo, n - j->lo, b->R,
                                                  j->buf, b->P, false)
                                : 0.0;
    ss->cpu_ms += ms;
    if (b->timer.on) b->timer_host_ms += ms;   // serialised on stream H
}

// Zero-copy share alpha.  Both miss paths have their own cap: the zero-copy copy the
// host's random-translation rate (r_zc; a row rate, so small rows move few bytes), the
// staged path the host gather rate r_host; both share the host link r_link.  Minimising
// max(alpha B / r_zc, (1 - alpha) B / r_host, B / r_link):
//   r_zc + r_host <= r_link: balance the paths, alpha = r_zc / (r_zc + r_host);
//   otherwise the link binds and the smallest zero-copy share that keeps the staged path
//   within it is best (zero-copy loads also slow the SMs they run on):
//   alpha = 1 - r_host / r_link.
static void adapt_alpha(gd_buffer* b) {
    const int64_t bc = b->batch_counter;   // the batch being enqueued; slots of bc-1 .. bc-D+1 are intact
    // (1) misses per batch, for the copy-engine staging size: the newest batch whose loop 2
    // has run, from the word every slot's publication also writes (no event, no sync)
    int64_t newest_epoch = 0;
    for (int d = 0; d < b->D; ++d) {
        const unsigned long long w = *(volatile const unsigned long long*)(b->stg[d].h_meta + 4);
        if ((int64_t)(w >> 32) > newest_epoch) {
            newest_epoch = (int64_t)(w >> 32);
            b->m_est = (double)(w & 0xffffffffull);
        }
    }
    if (b->alpha_fixed || b->r_link <= 0) return;
    // (2) path rates from the newest batch whose miss paths have finished and that has not
    // been used yet (a caller Q + 1 batches ahead still finds batch bc - Q - 1 complete)
    for (int k = 1; k < b->D && bc - k > b->rated_batch; ++k) {
        const int d = (int)((bc - k) % b->D);
        StagedSlot& ss = b->stg[d];
        if (ss.batch != bc - k) break;
        if (cudaEventQuery(b->ev_trip[d]) != cudaSuccess) {   // the batch has joined (both miss paths done)
            cudaGetLastError();                     // still in flight: try an older one
            continue;
        }
        // (Balancing the two paths' concurrently measured durations instead was tried and
        // measured worse: the zero-copy share is translation-bound and its SM loads slow the
        // copy engine's transfers, so the smallest share that keeps the link busy wins.)
        const volatile int64_t* hm = ss.h_meta;
        const double staged_rows = (double)hm[2], zc_rows = (double)hm[1];
        if (staged_rows >= 2048 && ss.cpu_ms > 0) {
            const double r = staged_rows * (double)b->R / ss.cpu_ms;
            b->r_host = b->r_host > 0 ? 0.7 * b->r_host + 0.3 * r : r;
            b->rate_samples++;
        }
        float tz = 0;
        if (ss.zc_timed && zc_rows >= 2048 && cudaEventElapsedTime(&tz, b->ev_z0[d], b->ev_z1[d]) == cudaSuccess && tz > 0) {
            const double r = zc_rows * (double)b->R / tz;
            b->r_zc = b->r_zc > 0 ? 0.7 * b->r_zc + 0.3 * r : r;
        }
        cudaGetLastError();
        b->rated_batch = bc - k;
        break;
    }
    if (b->r_host <= 0) return;
    double a;
    if (b->r_zc > 0 && b->r_zc + b->r_host <= b->r_link)
        a = b->r_zc / (b->r_zc + b->r_host);
    else
        a = 1.0 - b->r_host / b->r_link;
    // With copy-engine staging the zero-copy share also costs the DMA engine: its random
    // 4 KB-page reads contend with the copy engine for the host's DMA translation, and past a
    // box-dependent threshold the copy rate collapses (r01: ~17 GB/s at 0.4; r02, a slow-host
    // box, papers100m: share 0.1 / 0.15 / 0.2 / 0.3 -> 450 / 500 / 197 / 319 batches/s, the copy
    // engine 2.0 ms per batch at 0.15 and 5.1 ms at 0.2).  The model's share is clamped to
    // [0.05, 0.15], below every collapse measured; with the tuner on, it is only the start.
    const double hi = (b->ce_mode && b->dstage) ? kZeroCopyCapCE : 0.9;
    const double model = std::min(hi, std::max(0.05, a));
    if (!b->tune.on) {
        b->alpha = model;
        return;
    }
    ShareTuner& T = b->tune;
    if (!T.have_best && T.windows == 0 && T.phase == 0 && T.w_b0 < 0) {
        T.alpha = T.best_alpha = model;                     // start from the model
        b->alpha = model;
    }
}

// (3) The share tuner (ShareTuner in gd_handles.cuh).  Called at every gd_extract after the
// estimates; reads only events that have completed and mapped host words.
static void tune_share(gd_buffer* b) {
    ShareTuner& T = b->tune;
    if (!T.on || T.frozen || b->r_host <= 0) return;
    const int64_t bc = b->batch_counter;
    // per-batch miss counts: a slot's word belongs to its current batch once the epochs match
    for (int d = 0; d < b->D; ++d) {
        const StagedSlot& ss = b->stg[d];
        if (ss.batch < 0) continue;
        const unsigned long long w = *(volatile const unsigned long long*)(ss.h_meta + 4);
        if ((w >> 32) == (ss.epoch & 0xffffffffull) && T.mb[ss.batch & 63] != ss.batch) {
            T.mb[ss.batch & 63] = ss.batch;
            T.mc[ss.batch & 63] = (int64_t)(w & 0xffffffffull);
        }
    }
    // newest completed batch and its completion time
    int64_t nb = -1;
    float tnb = 0;
    for (int k = 1; k < b->D && bc - k >= 0; ++k) {
        const int d = (int)((bc - k) % b->D);
        if (b->stg[d].batch != bc - k) break;
        if (cudaEventQuery(b->ev_fin[d]) == cudaSuccess && cudaEventElapsedTime(&tnb, b->ev_ref, b->ev_fin[d]) == cudaSuccess) {
            nb = bc - k;
            break;
        }
        cudaGetLastError();
    }
    cudaGetLastError();
    if (nb < 0) return;
    if (T.phase == 0) {                    // settling: the window starts at the first new-share batch
        if (nb >= T.change_batch) {
            T.w_b0 = nb;
            T.w_t0 = tnb;
            T.phase = 1;
        }
        return;
    }
    constexpr int kWindow = 6;
    if (nb - T.w_b0 < kWindow) return;
    int64_t misses = 0;
    bool known = true;
    for (int64_t x = T.w_b0 + 1; x <= nb; ++x) {
        if (T.mb[x & 63] != x) { known = false; break; }
        misses += T.mc[x & 63];
    }
    if (!known || misses <= 0) {           // a count was missed (the host ran far ahead): re-measure
        T.w_b0 = nb;
        T.w_t0 = tnb;
        return;
    }
    const double cost = (double)(tnb - T.w_t0) / (double)misses;
    T.windows++;
    double next;
    if (!T.have_best || cost < T.best_cost * 0.985) {            // better: keep going this way
        T.have_best = true;
        T.best_alpha = T.alpha;
        T.best_cost = cost;
        T.fails = 0;
        next = T.alpha + T.dir * T.step;
    } else if (T.alpha == T.best_alpha) {                        // re-measured the best
        T.best_cost = cost;
        next = T.alpha + T.dir * T.step;
    } else {                                                     // worse: try the other side
        T.dir = -T.dir;
        if (++T.fails >= 2) {
            T.fails = 0;
            T.step *= 0.5;
        }
        next = T.best_alpha + T.dir * T.step;
    }
    constexpr double kLo = 0.0, kHi = 0.4;
    if (next < kLo || next > kHi) {                              // at a bound: the other side
        T.dir = -T.dir;
        next = T.best_alpha + T.dir * T.step;
    }
    if (T.step < 0.0124 || next < kLo || next > kHi) {
        T.frozen = true;
        next = T.best_alpha;
    }
    T.alpha = next;
    b->alpha = next;
    T.change_batch = bc;
    T.phase = 0;
}

gd_status gd_buffer_policy_read(gd_buffer* b, double* out, int32_t n) {
    if (!b || b->hdr.magic != kMagicBuffer) return set_error(GD_ERR_INVALID, "gd_buffer_policy_read: bad handle");
    if (!out || n < 0) return set_error(GD_ERR_INVALID, "gd_buffer_policy_read: null output");
    const ShareTuner& T = b->tune;
    const double v[12] = {b->alpha, b->r_host * 1e-6, b->r_zc * 1e-6, b->r_link * 1e-6, b->m_est,
                          (double)b->rate_samples, (b->ce_mode && b->dstage) ? kZeroCopyCapCE : 0.9,
                          (double)b->rated_batch, T.on ? 1.0 : 0.0, (double)T.windows, T.frozen ? 1.0 : 0.0,
                          T.best_cost * 1e6};
    for (int k = 0; k < n && k < 12; ++k) out[k] = v[k];
    return GD_OK;
}

// Contiguous host-link pull rate (bytes/ms), measured once on the staging memory.
__global__ void __launch_bounds__(1024, 1) k_link_calib(const uint4* __restrict__ src, uint4* __restrict__ dst, int64_t n16) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n16; i += (int64_t)gridDim.x * blockDim.x) {
        uint4 v;
        asm volatile("ld.global.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                     : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(src + i));
        dst[i] = v;
    }
}

static gd_status calibrate_link(gd_buffer* b) {
    const int64_t bytes = std::min<int64_t>(64ll << 20, (int64_t)b->n_max * b->R) & ~(int64_t)15;
    if (bytes < (1 << 20)) return GD_OK;
    const uint8_t* src = nullptr;
    GD_CUDA(cudaHostGetDevicePointer((void**)&src, b->stage_mem, 0));
    uint8_t* dst = nullptr;
    GD_CUDA(cudaMalloc(&dst, bytes));
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    float best = 1e30f;
    for (int rep = 0; rep < 4; ++rep) {
        cudaEventRecord(e0, b->side_p);
        if (b->ce_mode)   // the staged share crosses the link by copy engine
            cudaMemcpyAsync(dst, b->stage_mem, bytes, cudaMemcpyHostToDevice, b->side_p);
        else
            k_link_calib<<<b->pull_blocks, 1024, 0, b->side_p>>>((const uint4*)src, (uint4*)dst, bytes / 16);
        cudaEventRecord(e1, b->side_p);
        cudaEventSynchronize(e1);
        float ms = 0;
        cudaEventElapsedTime(&ms, e0, e1);
        if (rep > 0 && ms > 0 && ms < best) best = ms;
    }
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFree(dst);
    GD_CUDA(cudaGetLastError());
    b->r_link = (double)bytes / best;
    return GD_OK;
}

gd_status gd_extract(gd_buffer* b, const int32_t* node_ids, const int64_t* n_dev, int64_t n_max, void* out,
                     int32_t* alias, int64_t* stats, void* stream_v, void* done_v) {
    if (!b || b->hdr.magic != kMagicBuffer) return set_error(GD_ERR_INVALID, "gd_extract: bad buffer handle");
    if (!node_ids || !n_dev || !out) return set_error(GD_ERR_INVALID, "gd_extract: null pointer");
    if (n_max < 0 || n_max > b->n_max)
        return set_error(GD_ERR_INVALID, "gd_extract: n_max exceeds max_nodes_per_batch");
    if (b->inflight >= b->Q)
        return set_error(GD_ERR_CAPACITY, "gd_extract: max_inflight unreleased batches already extracted");
    if (((uintptr_t)out & 15) && (b->R % 16 == 0)) return set_error(GD_ERR_INVALID, "gd_extract: out must be 16-byte aligned");
    DeviceGuard guard(b->hdr.device);
    cudaStream_t st = (cudaStream_t)stream_v;
    const int d = (int)(b->batch_counter % b->D);
    int32_t* al = alias ? alias : b->alias_ws + (int64_t)d * b->n_max;
    int2* hlist = b->hitlist + (int64_t)d * b->n_max;
    int64_t* hcnt = b->hcount + d;
    int4* trip = b->trip + (int64_t)d * b->n_max;
    int64_t* tcount = b->trip_count + d;
    int64_t* tsplit = b->trip_split + d;
    const int64_t lt = std::max<int64_t>(1, cdiv(n_max, kBTile));
    const bool staged = b->host_threads > 0;
    StagedSlot* ss = staged ? &b->stg[d] : nullptr;

    // every stream is done with trip / host-list slot d (batch - D)
    GD_CUDA(cudaStreamWaitEvent(st, b->ev_trip[d], 0));
    if (staged) {
        adapt_alpha(b);
        tune_share(b);
        ss->batch = b->batch_counter;
    }
    const uint32_t alpha_q16 = staged ? (uint32_t)std::lround(b->alpha * 65536.0) : 65536u;
    // Copy-engine staging: the H2D copy is enqueued now, so its size must be known now;
    // the staged share is the first `cap` misses (cap from the recent misses per batch),
    // the zero-copy share takes the rest.  A batch with fewer misses copies some unused
    // staging rows (bounded by the estimate's error).
    const bool ce = staged && b->ce_mode && b->dstage;
    const long long cap = ce ? std::min<long long>(b->n_max, (long long)((1.0 - b->alpha) * b->m_est * 0.97)) : -1;
    const bool timed = b->timer.on;
    const int t_book = timed ? b->timer.begin(st) : -1;

    LookupArgs la;
    la.ids = node_ids;
    la.n_dev = n_dev;
    la.N = b->N;
    la.map = b->map;
    la.pos_of_slot = b->pos_of_slot;
    la.alias = al;
    la.hitlist = hlist;
    la.hcount = hcnt;
    la.misslist = b->misslist;
    la.mcount = b->mcount;
    la.stats = stats;
    la.st = b->scan.use();
    la.st_clear = b->scan.other();
    la.st_clear_n = b->scan.cap;
    la.status = b->hdr.dev_status;
    GD_CUDA(launch_chain(k_lookup, dim3((unsigned)lt), dim3(kBThreads), 0, st, la));
    GD_DEBUG_AFTER("k_lookup", st);
    b->scan.flip();

    PopArgs pa;
    pa.ring = b->ring;
    pa.ctl_in = b->ctl + b->ctl_parity;
    pa.ctl_out = b->ctl + (b->ctl_parity ^ 1);
    pa.pos_of_slot = b->pos_of_slot;
    pa.map = b->map;
    pa.reverse = b->reverse;
    pa.ids = node_ids;
    pa.misslist = b->misslist;
    pa.mcount = b->mcount;
    pa.alias = al;
    pa.trip = trip;
    pa.trip_count = tcount;
    pa.trip_split = tsplit;
    pa.alpha_q16 = alpha_q16;
    pa.staged_cap = cap;
    pa.ready = b->publish ? b->ready : nullptr;   // f2 tags only once a peer can read them
    pa.h_nodes = nullptr;
    pa.h_meta = nullptr;
    int32_t* h_nodes_dev = nullptr;
    int64_t* h_meta_dev = nullptr;
    if (staged) {
        GD_CUDA(cudaHostGetDevicePointer((void**)&h_nodes_dev, ss->h_nodes, 0));
        GD_CUDA(cudaHostGetDevicePointer((void**)&h_meta_dev, ss->h_meta, 0));
    }
    const bool peer = b->npeers > 0 && !b->preload;
    if (!peer) {   // with peers, k_peer_split publishes the host share instead
        pa.h_nodes = h_nodes_dev;
        pa.h_meta = h_meta_dev;
    }
    pa.stats = peer ? nullptr : stats;   // with peers, k_peer_split writes stats[2..3] (final at `done`)
    pa.ticket = b->tickets;
    pa.done_word = b->done_word;
    pa.epoch = ++b->epoch;
    if (staged) ss->epoch = pa.epoch;
    pa.st = b->scan.use();
    pa.st_clear = b->scan.other();
    pa.st_clear_n = b->scan.cap;
    pa.status = b->hdr.dev_status;
    GD_CUDA(launch_chain(k_pop_assign, dim3(148 * 2), dim3(kBThreads), 0, st, pa));
    GD_DEBUG_AFTER("k_pop_assign", st);
    b->scan.flip();
    b->ctl_parity ^= 1;
    if (timed) b->timer.end(t_book, st);
    // f2: peers first; the host paths copy what no peer served (trip2)
    int4* mtrip = trip;
    int64_t* mcount_d = tcount;
    int64_t* msplit = tsplit;
    if (peer) {
        mtrip = b->trip2 + (int64_t)d * b->n_max;
        mcount_d = b->trip2_count + d;
        msplit = b->trip2_split + d;
    }
    GD_CUDA(cudaEventRecord(b->ev_L, st));

    // Stream order (the host enqueue order below matters: each wait captures the event's
    // latest record):  G(b) waits X/Xs of b-1 (hits may sit in slots the previous
    // batch's misses are still filling); Z(b)/P(b) wait G(b-1) (their slots were freed
    // by releases of batches whose gathers are <= b-1, so no live gather reads them).
    GD_CUDA(cudaStreamWaitEvent(b->side_g, b->ev_L, 0));
    GD_CUDA(cudaStreamWaitEvent(b->side_g, b->ev_X, 0));
    GD_CUDA(cudaStreamWaitEvent(b->side_g, b->ev_Xs, 0));
    GD_CUDA(cudaStreamWaitEvent(b->side, b->ev_L, 0));
    GD_CUDA(cudaStreamWaitEvent(b->side, b->ev_G, 0));   // (before the probe: it writes slots too)
    if (peer) {
        // f2 on stream Z (off the caller's stream, so the next batch's sampling does not
        // wait for NVLink round trips): peers serve what they hold, the rest is split
        // between the host paths.  H waits for the split (its node list).
        GD_CUDA(cudaMemsetAsync(mcount_d, 0, sizeof(int64_t), b->side));
        k_peer_probe<<<148 * 2, 256, 0, b->side>>>(trip, tcount, b->peers, b->npeers, b->slots, (uint8_t*)out, b->R,
                                                  mtrip, mcount_d, b->peer_ctr);
        GD_DEBUG_AFTER("k_peer_probe", b->side);
        k_peer_split<<<148, 256, 0, b->side>>>(mtrip, mcount_d, msplit, alpha_q16, cap, h_nodes_dev, h_meta_dev, stats,
                                              pa.epoch);
        GD_DEBUG_AFTER("k_peer_split", b->side);
        GD_CUDA(cudaEventRecord(b->ev_S, b->side));
    }
    if (staged) {
        GD_CUDA(cudaStreamWaitEvent(b->side_h, peer ? b->ev_S : b->ev_L, 0));
        GD_CUDA(cudaStreamWaitEvent(b->side_h, b->ev_P[d], 0));   // pull of batch - D left slot d
        GD_CUDA(cudaStreamWaitEvent(b->side_p, b->ev_G, 0));
    }

    // a8: hits, slots -> out (stream G)
    const int t_gat = timed ? b->timer.begin(b->side_g) : -1;
    unsigned long long* gctr = b->gather_dynamic ? b->tickets + 4 : nullptr;
    if (b->gather_tma) {
        const int64_t stride = (4 * b->R + 127) / 128 * 128, smem = 8 * stride;   // P = 8 stages
        const int per_sm = (int)std::max<int64_t>(1, std::min<int64_t>(16, (200 << 10) / (smem + 256)));
        k_gather_tma<4><<<148 * per_sm, 32, smem, b->side_g>>>(b->slot_map, hlist, hcnt, (uint8_t*)out, b->R, stride,
                                                                 b->tickets + 4);
    } else if (b->R % 16 == 0 && b->R <= 512 && b->gather_u == 8)
        k_gather_rows<8, 1><<<148 * b->gather_bps, 256, 0, b->side_g>>>(hlist, hcnt, b->slots, (uint8_t*)out, b->R, gctr);
    else if (b->R % 16 == 0 && b->R <= 512)
        k_gather_rows<4, 1><<<148 * b->gather_bps, 256, 0, b->side_g>>>(hlist, hcnt, b->slots, (uint8_t*)out, b->R, gctr);
    else if (b->R % 16 == 0 && b->R <= 1024)
        k_gather_rows<4, 2><<<148 * b->gather_bps, 256, 0, b->side_g>>>(hlist, hcnt, b->slots, (uint8_t*)out, b->R, gctr);
    else if (b->R % 16 == 0 && b->R <= 2048)
        k_gather_rows<2, 4><<<148 * b->gather_bps, 256, 0, b->side_g>>>(hlist, hcnt, b->slots, (uint8_t*)out, b->R, gctr);
    else if (b->R % 16 == 0)
        k_gather_hits<4><<<148 * 8, 256, 0, b->side_g>>>(hlist, hcnt, b->slots, (uint8_t*)out, b->R);
    else
        k_gather_hits_w4<<<148 * 8, 256, 0, b->side_g>>>(hlist, hcnt, b->slots, (uint8_t*)out, b->R);
    GD_DEBUG_AFTER("k_gather_hits", b->side_g);
    if (timed) b->timer.end(t_gat, b->side_g);
    GD_CUDA(cudaEventRecord(b->ev_G, b->side_g));
    // zc_after_gather: the zero-copy kernel of this batch also waits for this batch's hit gather,
    // so the two never overlap (microsecond host loads clog the memory pipeline of the SMs the
    // gather shares with them); the gather already waits for the previous batch's copies
    if (b->zc_after_gather && !peer) GD_CUDA(cudaStreamWaitEvent(b->side, b->ev_G, 0));

    // a7, zero-copy share: misses [0, K0) straight from the pinned host table (stream Z).
    // With preload every node is valid from the start and never evicted: no misses, no copy.
    const int t_zc = timed ? b->timer.begin(b->side) : -1;
    const bool zc_timed = staged && (b->batch_counter % 8) == 0;   // the zero-copy rate, every 8th batch
    if (staged) ss->zc_timed = zc_timed;
    if (zc_timed) GD_CUDA(cudaEventRecord(b->ev_z0[d], b->side));
    if (b->preload) {
    } else if (b->R % 16 == 0)
        k_miss_copy<4, false><<<b->zc_blocks, 1024, 0, b->side>>>(mtrip, nullptr, msplit, b->feat_dev, b->slots, (uint8_t*)out, b->R, b->P);
    else
        k_miss_copy_w4<false><<<b->zc_blocks, 1024, 0, b->side>>>(mtrip, nullptr, msplit, b->feat_dev, b->slots, (uint8_t*)out, b->R, b->P);
    GD_DEBUG_AFTER("k_miss_copy", b->side);
    if (zc_timed) GD_CUDA(cudaEventRecord(b->ev_z1[d], b->side));
    if (timed) b->timer.end(t_zc, b->side);
    GD_CUDA(cudaEventRecord(b->ev_X, b->side));

    // a7, staged share: misses [K0, M).  Phase 1 on stream H (host gather into pinned
    // staging slot d), phase 2 on stream P (contiguous pull into slots + out).
    if (staged) {
        const uint8_t* stage_dev = nullptr;
        if (ce && b->stage_chunk_rows > 0) {
            // chunk c: H waits until the copy out of ring buffer r (chunk k - stage_ring)
            // is done, gathers into it; C copies it to dstage[d] at rank offset lo
            stage_dev = b->dstage + (int64_t)d * b->n_max * b->R;
            int64_t ch = b->stage_chunk_rows;
            if (b->chunk_adaptive) {
                const int64_t want = std::min<int64_t>(16ll << 20, std::max<int64_t>(8ll << 20, cap * b->R / 6));
                ch = std::max<int64_t>(1, std::min<int64_t>(ch, want / b->R));
            }
            const int64_t nch = cap > 0 ? cdiv(cap, ch) : 0;
            const int t_ce = timed ? b->timer.begin(b->side_c) : -1;
            if (nch == 0) ss->cpu_ms = 0;
            for (int64_t c = 0; c < nch; ++c) {
                const int r = (int)(b->chunk_counter++ % b->stage_ring);
                // The callback reads its arguments when stream H reaches it, possibly many
                // batches after this enqueue: each chunk gets its own argument slot, reused
                // only after its previous callback ran (a host wait that needs the caller to
                // be kJobRing chunks ahead of the host gather).
                const uint64_t jk = b->job_counter++;
                const size_t js = (size_t)(jk % kJobRing);
                if (jk >= (uint64_t)kJobRing) GD_CUDA(cudaEventSynchronize(b->ev_job[js]));
                ChunkJob* j = &b->jobs[js];
                j->ss = ss;
                j->lo = c * ch;
                j->hi = std::min<int64_t>(cap, (c + 1) * ch);
                j->buf = b->ring_mem + (int64_t)r * b->stage_chunk_rows * b->R;   // ring stride = max chunk
                j->first = c == 0;
                GD_CUDA(cudaStreamWaitEvent(b->side_h, b->ev_ring[r], 0));
                GD_CUDA(cudaLaunchHostFunc(b->side_h, chunk_gather_cb, j));
                GD_CUDA(cudaEventRecord(b->ev_job[js], b->side_h));
                GD_CUDA(cudaStreamWaitEvent(b->side_c, b->ev_job[js], 0));
                GD_CUDA(cudaMemcpyAsync((void*)(stage_dev + j->lo * b->R), j->buf, (size_t)(j->hi - j->lo) * b->R,
                                        cudaMemcpyHostToDevice, b->side_c));
                GD_CUDA(cudaEventRecord(b->ev_ring[r], b->side_c));
            }
            if (timed) b->timer.end(t_ce, b->side_c);
            GD_CUDA(cudaEventRecord(b->ev_H[d], b->side_h));     // every chunk gathered
            GD_CUDA(cudaStreamWaitEvent(b->side_c, b->ev_H[d], 0));
            GD_CUDA(cudaEventRecord(b->ev_E[d], b->side_c));
        } else if (ce) {
            GD_CUDA(cudaLaunchHostFunc(b->side_h, host_gather_cb, ss));
            // phase 2 by the copy engine on stream C, so that the host gather of the next
            // batch (stream H) overlaps this copy: pinned slot d -> dstage[d].  dstage[d]
            // is free: H waited for the scatter of batch - D before this gather.
            stage_dev = b->dstage + (int64_t)d * b->n_max * b->R;
            GD_CUDA(cudaEventRecord(b->ev_H[d], b->side_h));
            GD_CUDA(cudaStreamWaitEvent(b->side_c, b->ev_H[d], 0));
            const int t_ce = timed ? b->timer.begin(b->side_c) : -1;
            if (cap > 0)
                GD_CUDA(cudaMemcpyAsync((void*)stage_dev, ss->staging, (size_t)cap * b->R, cudaMemcpyHostToDevice, b->side_c));
            if (timed) b->timer.end(t_ce, b->side_c);
            GD_CUDA(cudaEventRecord(b->ev_E[d], b->side_c));
        } else {
            GD_CUDA(cudaLaunchHostFunc(b->side_h, host_gather_cb, ss));
            GD_CUDA(cudaHostGetDevicePointer((void**)&stage_dev, ss->staging, 0));
            if (timed) b->timer.end(b->timer.begin(b->side_h), b->side_h);
            GD_CUDA(cudaEventRecord(b->ev_E[d], b->side_h));
        }
        GD_CUDA(cudaStreamWaitEvent(b->side_p, b->ev_E[d], 0));
        const int t_pl = timed ? b->timer.begin(b->side_p) : -1;
        if (b->R % 16 == 0)
            k_miss_copy<4, true><<<ce ? 64 : b->pull_blocks, 1024, 0, b->side_p>>>(mtrip, msplit, mcount_d, stage_dev, b->slots, (uint8_t*)out, b->R, b->P);
        else
            k_miss_copy_w4<true><<<b->pull_blocks, 1024, 0, b->side_p>>>(mtrip, msplit, mcount_d, stage_dev, b->slots, (uint8_t*)out, b->R, b->P);
        GD_DEBUG_AFTER("k_stage_copy", b->side_p);
        if (timed) b->timer.end(t_pl, b->side_p);
        GD_CUDA(cudaEventRecord(b->ev_P[d], b->side_p));
        GD_CUDA(cudaEventRecord(b->ev_Xs, b->side_p));
    } else if (timed) {
        b->timer.end(b->timer.begin(b->side), b->side);   // keep kTimedPairs timing pairs per batch
        b->timer.end(b->timer.begin(b->side), b->side);
    }

    // join: out complete, trip slot d free
    GD_CUDA(cudaStreamWaitEvent(b->side_j, b->ev_X, 0));
    if (staged) GD_CUDA(cudaStreamWaitEvent(b->side_j, b->ev_Xs, 0));
    GD_CUDA(cudaStreamWaitEvent(b->side_j, b->ev_G, 0));
    // f2: the batch's new slots are complete: publish them to peers (before `done`, so a
    // release, and with it any reuse of these slots, is ordered after the publication)
    if (!b->preload && b->publish) k_publish<<<148, 256, 0, b->side_j>>>(trip, tcount, b->ready, pa.epoch);
    GD_CUDA(cudaEventRecord(b->ev_trip[d], b->side_j));
    if (b->tune.on) GD_CUDA(cudaEventRecord(b->ev_fin[d], b->side_j));
    if (done_v) GD_CUDA(cudaEventRecord((cudaEvent_t)done_v, b->side_j));
    GD_CUDA(cudaGetLastError());
    b->inflight++;
    b->batch_counter++;
    return GD_OK;
}

gd_status gd_buffer_release(gd_buffer* b, const int32_t* node_ids, const int64_t* n_dev, int64_t n_max,
                            void* stream_v) {
    if (!b || b->hdr.magic != kMagicBuffer) return set_error(GD_ERR_INVALID, "gd_buffer_release: bad buffer handle");
    if (!node_ids || !n_dev) return set_error(GD_ERR_INVALID, "gd_buffer_release: null pointer");
    if (n_max < 0 || n_max > b->n_max)
        return set_error(GD_ERR_INVALID, "gd_buffer_release: n_max exceeds max_nodes_per_batch");
    if (b->inflight <= 0) return set_error(GD_ERR_INVALID, "gd_buffer_release: no extracted batch to release");
    DeviceGuard guard(b->hdr.device);
    cudaStream_t st = (cudaStream_t)stream_v;

    CompactArgs ca;
    ca.ring = b->ring;
    ca.pos_of_slot = b->pos_of_slot;
    ca.ctl_in = b->ctl + b->ctl_parity;
    ca.ctl_out = b->ctl + (b->ctl_parity ^ 1);
    ca.C = b->C;
    ca.n_max = b->n_max;
    ca.ticket = b->tickets + 2;
    ca.st = b->scan.use();
    ca.st_clear = b->scan.other();
    ca.st_clear_n = b->scan.cap;
    GD_CUDA(launch_chain(k_compact, dim3(148 * 2), dim3(kBThreads), 0, st, ca));
    GD_DEBUG_AFTER("k_compact", st);
    b->scan.flip();
    b->ctl_parity ^= 1;

    ReleaseArgs ra;
    ra.ids = node_ids;
    ra.n_dev = n_dev;
    ra.N = b->N;
    ra.map = b->map;
    ra.ring = b->ring;
    ra.pos_of_slot = b->pos_of_slot;
    ra.ctl_in = b->ctl + b->ctl_parity;
    ra.ctl_out = b->ctl + (b->ctl_parity ^ 1);
    ra.st = b->scan.use();
    ra.st_clear = b->scan.other();
    ra.st_clear_n = b->scan.cap;
    ra.status = b->hdr.dev_status;
    GD_CUDA(launch_chain(k_release, dim3((unsigned)std::max<int64_t>(1, cdiv(n_max, kBTile))), dim3(kBThreads), 0, st, ra));
    GD_DEBUG_AFTER("k_release", st);
    b->scan.flip();
    b->ctl_parity ^= 1;
    GD_CUDA(cudaGetLastError());
    b->inflight--;
    return GD_OK;
}

gd_status gd_buffer_snapshot(gd_buffer* b, int32_t* map_slot, int32_t* map_rc, uint8_t* map_valid, int32_t* reverse,
                             int32_t* standby, int64_t* standby_len) {
    if (!b || b->hdr.magic != kMagicBuffer) return set_error(GD_ERR_INVALID, "gd_buffer_snapshot: bad handle");
    DeviceGuard guard(b->hdr.device);
    GD_CUDA(cudaDeviceSynchronize());
    if (map_slot || map_rc || map_valid) {
        std::vector<int2> m(b->N);
        GD_CUDA(cudaMemcpy(m.data(), b->map, b->N * sizeof(int2), cudaMemcpyDeviceToHost));
        for (int64_t v = 0; v < b->N; ++v) {
            if (map_slot) map_slot[v] = m[v].x;
            if (map_rc) map_rc[v] = m[v].y >> 1;
            if (map_valid) map_valid[v] = (uint8_t)(m[v].y & 1);
        }
    }
    if (reverse) GD_CUDA(cudaMemcpy(reverse, b->reverse, b->S * sizeof(int32_t), cudaMemcpyDeviceToHost));
    if (standby || standby_len) {
        GdCtl c;
        GD_CUDA(cudaMemcpy(&c, b->ctl + b->ctl_parity, sizeof(c), cudaMemcpyDeviceToHost));
        std::vector<int32_t> pos(b->S), ring(std::max<long long>(1, c.tail - c.head));
        GD_CUDA(cudaMemcpy(pos.data(), b->pos_of_slot, b->S * sizeof(int32_t), cudaMemcpyDeviceToHost));
        if (c.tail > c.head)
            GD_CUDA(cudaMemcpy(ring.data(), b->ring + c.head, (c.tail - c.head) * sizeof(int32_t), cudaMemcpyDeviceToHost));
        int64_t k = 0;
        for (long long p = c.head; p < c.tail; ++p) {
            const int32_t s = ring[p - c.head];
            if (pos[s] == (int32_t)p) {
                if (standby) standby[k] = s;
                ++k;
            }
        }
        if (standby_len) *standby_len = k;
    }
    return GD_OK;
}

gd_status gd_buffer_set_state(gd_buffer* b, const int32_t* map_slot, const int32_t* map_rc, const uint8_t* map_valid,
                              const int32_t* reverse, const int32_t* standby, int64_t standby_len) {
    if (!b || b->hdr.magic != kMagicBuffer) return set_error(GD_ERR_INVALID, "gd_buffer_set_state: bad handle");
    if (!map_slot || !map_rc || !map_valid || !reverse || (standby_len > 0 && !standby) || standby_len > b->S)
        return set_error(GD_ERR_INVALID, "gd_buffer_set_state: bad arguments");
    DeviceGuard guard(b->hdr.device);
    GD_CUDA(cudaDeviceSynchronize());
    std::vector<int2> m(b->N);
    for (int64_t v = 0; v < b->N; ++v) m[v] = make_int2(map_slot[v], (map_rc[v] << 1) | (map_valid[v] & 1));
    GD_CUDA(cudaMemcpy(b->map, m.data(), b->N * sizeof(int2), cudaMemcpyHostToDevice));
    GD_CUDA(cudaMemcpy(b->reverse, reverse, b->S * sizeof(int32_t), cudaMemcpyHostToDevice));
    std::vector<int32_t> pos(b->S, -1);
    for (int64_t k = 0; k < standby_len; ++k) pos[standby[k]] = (int32_t)k;
    GD_CUDA(cudaMemcpy(b->pos_of_slot, pos.data(), b->S * sizeof(int32_t), cudaMemcpyHostToDevice));
    if (standby_len > 0) GD_CUDA(cudaMemcpy(b->ring, standby, standby_len * sizeof(int32_t), cudaMemcpyHostToDevice));
    GdCtl c[2];
    c[0].head = 0;
    c[0].tail = standby_len;
    c[0].base = 0;
    c[1] = c[0];
    GD_CUDA(cudaMemcpy(b->ctl, c, sizeof(c), cudaMemcpyHostToDevice));
    std::vector<unsigned long long> tags(b->S, kReadyNone);
    for (int64_t v = 0; v < b->N; ++v)
        if ((map_valid[v] & 1) && map_slot[v] >= 0) {
            GD_CUDA(cudaMemcpy(b->slots + (int64_t)map_slot[v] * b->R, (const uint8_t*)b->host_feat + (v % b->P) * b->R, b->R,
                               cudaMemcpyHostToDevice));
            tags[map_slot[v]] = (unsigned long long)(uint32_t)v;
        }
    GD_CUDA(cudaMemcpy(b->ready, tags.data(), b->S * sizeof(unsigned long long), cudaMemcpyHostToDevice));
    return GD_OK;
}

}  // extern "C"
