// gd_sample.cu — topology replica and the multi-hop sampler (rows a1-a4 of the hot path).
//
// One gd_sample call = 1 + 2K launches on the caller's stream (hops with 1 <= f <= 32), no host
// sync:   k_seed_intake ; K x { k_sample_pad ; k_relabel_pad }
//
// k_sample_pad  (S1, a2+a3): G = pow2 >= f lanes per frontier node, no tiles, no scan: Floyd
//   positions by Philox (lane t = draw t, resolution by ballots, rank sort by shuffles); the
//   draw of rank r of node i goes to padded position q = i f + r, its neighbour into the global
//   open-addressing hash with atomicMin(PENDING | q) (first occurrence), its hash slot to
//   pslot[q], min(f, deg) to pcnt[i].
// k_relabel_pad (S2, a2+a4): one pass over the padded positions, one decoupled look-back over
//   (edges, new nodes): rowptr, compacted col / eid, new nodes' local ids n_{h-1} + rank
//   (warp-aggregated compaction), appended to n_id and finalised in the hash; then every edge's
//   final col (waiting for the store of a node first seen in an earlier tile).  The last hop's
//   pass also empties the slots the previous call used in the workspace's other hash table.
// Hops with f = -1 or f > 32 (or gd_graph_sampler(g, 0)) take the count-scan form:
// k_sample_hop (counts + look-back -> rowptr, sampling writes col at rowptr + rank),
// k_relabel_hop (first-occurrence flags, look-back ranks) and one k_col_resolve pass over those
// hops' edges (+ k_hash_clear when the last hop has this form).
#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <string>

#include "gd_common.cuh"
#include "gd_handles.cuh"

namespace gd {

constexpr int kThreads = 256;
constexpr int kWarps = kThreads / 32;
constexpr int kRelabelItems = 8;    // (16 measured slower: products 4345 vs 4534 batches/s)
constexpr int kEdgesPerTile = kThreads * kRelabelItems;   // 2048 edges per relabel block
static_assert((kRelabelItems * kWarps) % 32 == 0, "relabel scan layout");
constexpr int kMaxFanSmem = GD_MAX_FANOUT;
// k_relabel_pad: padded positions per thread (<= kRelabelItems) and the launch-bounds block
// minimum (the defaults were measured; the macros exist for same-box A/B builds)
#ifndef GD_PAD_ITEMS
#define GD_PAD_ITEMS 4
#endif
#ifndef GD_PAD_MINB
#define GD_PAD_MINB 1
#endif
constexpr int kPadItems = GD_PAD_ITEMS;
constexpr int kPadPerTile = kThreads * kPadItems;
static_assert(kPadItems <= kRelabelItems && (kPadItems * kWarps) % 32 == 0, "relabel_pad scan layout");

struct SampleHopArgs {
    const int64_t* indptr;
    const int32_t* indices;
    int64_t N;
    int32_t* n_id;
    int64_t* sizes;
    int hop;          // 1-based
    int K;
    int fanout;
    uint32_t batch;
    uint64_t seed;
    int64_t* rowptr;
    int32_t* col;
    int64_t* eid;
    uint32_t* hkeys;
    uint32_t* hvals;
    uint32_t mask;
    unsigned long long* st;
    unsigned long long* st_clear;
    int64_t st_clear_n;
    unsigned int* status;
};

// Insert neighbour u seen at flat position e of this hop; returns its hash slot.
// (A CAS-first probe -- one atomic per probe instead of a load then a CAS for a new key -- was
// measured no faster: products 4463 vs 4482 batches/s.)
__device__ __forceinline__ uint32_t hash_insert(uint32_t* __restrict__ hk, uint32_t* __restrict__ hv,
                                                uint32_t mask, uint32_t u, uint32_t e) {
    uint32_t h = fmix32(u) & mask;
    const uint32_t tag = kPending | e;
    while (true) {
        const uint32_t k = ld_relaxed_u32(hk + h);
        if (k == u) break;
        if (k == kEmpty) {
            const uint32_t old = atomicCAS(hk + h, kEmpty, u);
            if (old == kEmpty) {           // claimed: the value is empty (> any tag), no load first
                atomicMin(hv + h, tag);
                return h;
            }
            if (old == u) break;
        }
        h = (h + 1) & mask;
    }
    if (ld_relaxed_u32(hv + h) > tag) atomicMin(hv + h, tag);
    return h;
}

__global__ void __launch_bounds__(kThreads) k_seed_intake(const int32_t* __restrict__ seeds, int64_t B,
                                                          int64_t N, uint32_t* hk, uint32_t* hv,
                                                          uint32_t mask, int32_t* n_id, int64_t* sizes,
                                                          int32_t* slot_of, unsigned int* status) {
    GD_PDL_ENTRY();
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i == 0) sizes[0] = B;
    if (i >= B) return;
    const int32_t v = seeds[i];
    n_id[i] = v;
    if (v < 0 || (int64_t)v >= N) {
        atomicOr(status, GD_DEV_BAD_ID);
        return;
    }
    uint32_t h = fmix32((uint32_t)v) & mask;
    while (true) {
        const uint32_t old = atomicCAS(hk + h, kEmpty, (uint32_t)v);
        if (old == kEmpty) {
            hv[h] = (uint32_t)i;   // finalised local id = position
            slot_of[i] = (int32_t)h;
            return;
        }
        if (old == (uint32_t)v) {
            atomicOr(status, GD_DEV_DUP_SEED);
            return;
        }
        h = (h + 1) & mask;
    }
}

// Emit neighbour at CSR position p of node (start) as flat edge e.
__device__ __forceinline__ void emit_edge(const SampleHopArgs& a, int64_t start, int64_t p, int64_t e) {
    const uint32_t u = (uint32_t)__ldg(a.indices + start + p);
    const uint32_t slot = hash_insert(a.hkeys, a.hvals, a.mask, u, (uint32_t)e);
    a.col[e] = (int32_t)slot;
    if (a.eid) a.eid[e] = start + p;
}

// G = lanes per frontier node (a power of two >= fanout, or 32 for the generic paths);
// NPB = frontier nodes per 256-thread block (8 node-iterations per warp).
template <int G, int NPB>
__global__ void __launch_bounds__(kThreads) k_sample_hop(SampleHopArgs a) {
    static_assert(NPB <= kThreads && (32 % G) == 0, "tile shape");
    GD_PDL_ENTRY();
    clear_tile_state(a.st_clear, a.st_clear_n);
    const int64_t n_prev = a.sizes[a.hop - 1];
    const int64_t tile = blockIdx.x;
    const int64_t i0 = tile * NPB;
    if (i0 >= n_prev && tile != 0) return;

    __shared__ int64_t s_start[NPB];
    __shared__ int64_t s_deg[NPB];
    __shared__ int64_t s_off[NPB];
    __shared__ int32_t s_v[NPB];
    __shared__ long long s_wtot[kWarps];
    __shared__ long long s_base;
    __shared__ int64_t s_sel[G == 32 ? kWarps : 1][G == 32 ? kMaxFanSmem : 1];   // f > 32 path only

    const int t = threadIdx.x;
    const int lane = t & 31;
    const int warp = t >> 5;
    const int f = a.fanout;

    // ---- a2: counts (one frontier node per thread) and their exclusive scan (rowptr)
    long long cnt = 0;
    if (t < NPB) {
        const int64_t i = i0 + t;
        int64_t start = 0, d = 0;
        int32_t v = 0;
        if (i < n_prev) {
            v = a.n_id[i];
            if (v >= 0 && (int64_t)v < a.N) {
                start = a.indptr[v];
                d = a.indptr[v + 1] - start;
            }
            cnt = (f < 0) ? d : (d < f ? d : f);
        }
        s_v[t] = v;
        s_start[t] = start;
        s_deg[t] = d;
    }
    const long long incl = warp_inclusive_sum(cnt);
    if (lane == 31) s_wtot[warp] = incl;
    __syncthreads();
    if (warp == 0) {
        const long long wt = lane < kWarps ? s_wtot[lane] : 0;
        const long long winc = warp_inclusive_sum(wt);
        const long long agg = __shfl_sync(0xffffffffu, winc, kWarps - 1);
        __syncwarp();
        if (lane < kWarps) s_wtot[lane] = winc - wt;          // exclusive warp offsets
        const long long base = lookback_exclusive(a.st, tile, agg, 0);
        if (lane == 0) s_base = base;
    }
    __syncthreads();
    if (t < NPB) {
        const long long excl = s_base + s_wtot[warp] + incl - cnt;
        s_off[t] = excl;
        const int64_t i = i0 + t;
        if (i < n_prev) a.rowptr[i] = excl;
        const bool last = (n_prev == 0) ? (tile == 0 && t == 0) : (i == n_prev - 1);
        if (last) {
            const long long total = (n_prev == 0) ? 0 : excl + cnt;
            a.rowptr[n_prev] = total;
            a.sizes[a.K + a.hop] = total;
        }
    }
    __syncthreads();

    // ---- a3: Floyd sampling, G lanes per frontier node
    const uint32_t hidx = (uint32_t)(a.hop - 1);
    if constexpr (G < 32) {
        // 0 <= f <= G: lane gl of the group holds draw gl; groups are independent nodes
        constexpr int P = 32 / G;
        const int gl = lane & (G - 1);
        const int gbase = lane & ~(G - 1);
        const unsigned gmask = ((G == 32) ? 0xffffffffu : ((1u << G) - 1u)) << gbase;
        for (int ln0 = warp * P; ln0 < NPB; ln0 += kWarps * P) {
            const int ln = ln0 + lane / G;
            const int64_t i = i0 + ln;
            const bool active = (ln < NPB) && (i < n_prev);
            int64_t d = 0, start = 0, off = 0;
            uint32_t v = 0;
            if (active) {
                d = s_deg[ln];
                start = s_start[ln];
                off = s_off[ln];
                v = (uint32_t)s_v[ln];
            }
            const bool fl = active && d > f;           // Floyd; otherwise the row verbatim
            int64_t sel = INT64_MAX;
            if (fl) {
                if (gl < f) sel = (int64_t)draw_uniform((uint32_t)gl, v, hidx, a.batch, a.seed, (uint64_t)(d - f + gl));
            } else if (active && gl < d) {
                sel = gl;
            }
            for (int s = 1; s < f; ++s) {
                const int64_t rs = __shfl_sync(0xffffffffu, sel, gbase + s);
                const unsigned bl = __ballot_sync(0xffffffffu, fl && gl < s && sel == rs);
                if (fl && gl == s && (bl & gmask)) sel = d - f + s;
            }
            int rank = gl;
            if (f > 1) {
                int r = 0;
                for (int s = 0; s < f; ++s) {
                    const int64_t o = __shfl_sync(0xffffffffu, sel, gbase + s);
                    r += (o < sel);
                }
                if (fl) rank = r;
            }
            if (sel != INT64_MAX) emit_edge(a, start, sel, off + rank);
        }
    } else {
        for (int ln = warp; ln < NPB; ln += kWarps) {
            const int64_t i = i0 + ln;
            if (i >= n_prev) break;
            const int64_t start = s_start[ln];
            const int64_t d = s_deg[ln];
            const int64_t off = s_off[ln];
            const uint32_t v = (uint32_t)s_v[ln];
            if (f < 0 || d <= f) {
                // the row verbatim (reading R5): coalesced copy
                for (int64_t p = lane; p < d; p += 32) emit_edge(a, start, p, off + p);
            } else if (f <= 32) {
                // Floyd: lane t holds draw t in [0, d-f+t]
                int64_t sel = INT64_MAX;
                if (lane < f) {
                    const uint64_t j = (uint64_t)(d - f + lane);
                    sel = (int64_t)draw_uniform((uint32_t)lane, v, hidx, a.batch, a.seed, j);
                }
                for (int s = 1; s < f; ++s) {
                    const int64_t rs = __shfl_sync(0xffffffffu, sel, s);
                    const bool present = __ballot_sync(0xffffffffu, lane < s && sel == rs) != 0;
                    if (lane == s && present) sel = d - f + s;
                }
                int rank = 0;
                for (int s = 0; s < f; ++s) {
                    const int64_t o = __shfl_sync(0xffffffffu, sel, s);
                    rank += (o < sel);
                }
                if (lane < f) emit_edge(a, start, sel, off + rank);
            } else {
                // f in (32, 256]: resolution in shared memory, O(f^2/32) per node
                int64_t* ss = s_sel[warp];
                for (int c = 0; c < f; c += 32) {
                    const int tt = c + lane;
                    int64_t r = 0;
                    if (tt < f) {
                        const uint64_t j = (uint64_t)(d - f + tt);
                        r = (int64_t)draw_uniform((uint32_t)tt, v, hidx, a.batch, a.seed, j);
                    }
                    const int cend = min(32, f - c);
                    for (int s = 0; s < cend; ++s) {
                        const int step = c + s;
                        const int64_t rs = __shfl_sync(0xffffffffu, r, s);
                        bool hit = false;
                        for (int q = lane; q < step; q += 32) hit |= (ss[q] == rs);
                        const bool present = __ballot_sync(0xffffffffu, hit) != 0;
                        if (lane == 0) ss[step] = present ? (d - f + step) : rs;
                        __syncwarp();
                    }
                }
                __syncwarp();
                for (int q = lane; q < f; q += 32) {
                    const int64_t me = ss[q];
                    int rank = 0;
                    for (int x = 0; x < f; ++x) rank += (ss[x] < me);
                    emit_edge(a, start, me, off + rank);
                }
                __syncwarp();
            }
        }
    }
}

// Tile shape: G lanes per node (pow2 >= fanout; 32 for f > 16 or f < 0), ITERS node
// iterations per warp, NPB = 8 warps x ITERS x (32 / G) nodes per block (<= 256, one per
// thread in the count phase).  ITERS is chosen from the frontier bound so that small
// frontiers get many short warps (latency) and large ones still fill every SM.
static int sampler_group(int f) {
    if (f < 0 || f > 16) return 32;
    int g = 1;
    while (g < f) g *= 2;
    return g;
}

template <int G, int ITERS>
static void launch_hop_t(const SampleHopArgs& a, int64_t n_frontier_max, cudaStream_t st) {
    constexpr int NPB = kWarps * ITERS * (32 / G);
    const unsigned nt = (unsigned)std::max<int64_t>(1, (n_frontier_max + NPB - 1) / NPB);
    launch_chain(k_sample_hop<G, NPB>, dim3(nt), dim3(kThreads), 0, st, a);
}

template <int G>
static void launch_hop_g(const SampleHopArgs& a, int64_t n_frontier_max, cudaStream_t st) {
    constexpr int P = 32 / G;
    constexpr int CAP = (256 / (kWarps * P)) < 8 ? (256 / (kWarps * P)) : 8;   // max ITERS
    const int64_t warp_iters = (n_frontier_max + P - 1) / P;
    int iters = 1;
    while (iters < CAP && warp_iters / (iters * 2) >= 8192) iters *= 2;      // keep >= 8k warps
    if constexpr (CAP >= 8) { if (iters == 8) return launch_hop_t<G, 8>(a, n_frontier_max, st); }
    if constexpr (CAP >= 4) { if (iters == 4) return launch_hop_t<G, 4>(a, n_frontier_max, st); }
    if constexpr (CAP >= 2) { if (iters == 2) return launch_hop_t<G, 2>(a, n_frontier_max, st); }
    launch_hop_t<G, 1>(a, n_frontier_max, st);
}

static void launch_sample_hop(const SampleHopArgs& a, int64_t n_frontier_max, cudaStream_t st) {
    switch (sampler_group(a.fanout)) {
        case 1: launch_hop_g<1>(a, n_frontier_max, st); break;
        case 2: launch_hop_g<2>(a, n_frontier_max, st); break;
        case 4: launch_hop_g<4>(a, n_frontier_max, st); break;
        case 8: launch_hop_g<8>(a, n_frontier_max, st); break;
        case 16: launch_hop_g<16>(a, n_frontier_max, st); break;
        default: launch_hop_g<32>(a, n_frontier_max, st); break;
    }
}

// ---------------------------------------------------------------- padded hop (default, 1 <= f <= 32)
// The hop is split where its only grid-wide dependency lies.  k_sample_pad draws every frontier
// node's neighbours into a padded layout (node i's draw of rank r at q = i f + r) with no scan:
// first occurrence over (frontier index, ascending position) is first occurrence over q, so the
// hash tag kPending | q decides it exactly as the flat position did (reading R5).  k_relabel_pad
// then makes one pass over the padded positions and one decoupled look-back over the pair
// (edges, new nodes): it writes rowptr, the compacted col / eid, and the new nodes' local ids.
// Compared with k_sample_hop + k_relabel_hop, the look-back chain of the sampling kernel (one
// tile per 64-256 frontier nodes: the longest dependency chain of the hop) is gone, and the
// relabel tiles cover ~2048 padded positions each.
struct PadHopArgs {
    const int64_t* indptr;
    const int32_t* indices;
    int64_t N;
    const int32_t* n_id;
    const int64_t* sizes;
    int hop;          // 1-based
    int fanout;       // 1..32
    uint32_t batch;
    uint64_t seed;
    int32_t* pslot;   // [n_{h-1} f] hash slot of the draw at q
    int64_t* ppos;    // [n_{h-1} f] CSR position (eid) of the draw at q, or null
    int32_t* pcnt;    // [n_{h-1}] min(f, deg)
    uint32_t* hkeys;
    uint32_t* hvals;
    uint32_t mask;
};

template <int G>
__global__ void __launch_bounds__(kThreads) k_sample_pad(PadHopArgs a) {
    GD_PDL_ENTRY();
    const int64_t n_prev = a.sizes[a.hop - 1];
    const int lane = threadIdx.x & 31;
    const int64_t gt = (int64_t)blockIdx.x * kThreads + threadIdx.x;
    if ((gt - lane) / G >= n_prev) return;      // the whole warp is past the frontier (warp-uniform)
    const int64_t i = gt / G;
    const int gl = lane & (G - 1);
    const int gbase = lane & ~(G - 1);
    const unsigned gmask = ((G == 32) ? 0xffffffffu : ((1u << G) - 1u)) << gbase;
    const int f = a.fanout;
    const bool active = i < n_prev;
    int64_t d = 0, start = 0;
    uint32_t v = 0;
    if (active) {
        v = (uint32_t)a.n_id[i];
        if ((int32_t)v >= 0 && (int64_t)v < a.N) {
            start = a.indptr[v];
            d = a.indptr[v + 1] - start;
        }
        if (gl == 0) a.pcnt[i] = (int32_t)(d < f ? d : f);
    }
    const bool fl = active && d > f;           // Floyd; otherwise the row verbatim
    int64_t sel = INT64_MAX;
    if (fl) {
        if (gl < f) sel = (int64_t)draw_uniform((uint32_t)gl, v, (uint32_t)(a.hop - 1), a.batch, a.seed, (uint64_t)(d - f + gl));
    } else if (active && gl < d) {
        sel = gl;
    }
    for (int s = 1; s < f; ++s) {
        const int64_t rs = __shfl_sync(0xffffffffu, sel, gbase + s);
        const unsigned bl = __ballot_sync(0xffffffffu, fl && gl < s && sel == rs);
        if (fl && gl == s && (bl & gmask)) sel = d - f + s;
    }
    int rank = gl;
    if (f > 1) {
        int r = 0;
        for (int s = 0; s < f; ++s) {
            const int64_t o = __shfl_sync(0xffffffffu, sel, gbase + s);
            r += (o < sel);
        }
        if (fl) rank = r;
    }
    if (sel != INT64_MAX) {
        const uint32_t q = (uint32_t)(i * f + rank);
        const uint32_t u = (uint32_t)__ldg(a.indices + start + sel);
        a.pslot[q] = (int32_t)hash_insert(a.hkeys, a.hvals, a.mask, u, q);
        if (a.ppos) a.ppos[q] = start + sel;
    }
}

struct PadRelabelArgs {
    const int32_t* pslot;
    const int64_t* ppos;
    const int32_t* pcnt;
    int64_t* rowptr;
    int32_t* col;
    int64_t* eid;
    int32_t* n_id;
    int64_t* sizes;
    int hop;
    int K;
    int fanout;
    int nt;           // frontier nodes per tile (nt f <= kPadPerTile)
    uint32_t* hkeys;
    uint32_t* hvals;
    int32_t* slot_of;
    unsigned long long* st;
    unsigned long long* st_clear;
    int64_t st_clear_n;
    // last hop only (else null): empty the slots the previous call used in the other table
    // (clr_slot_of[0, *clr_count)), and record this call's node count (*rec_used = n_K)
    const int32_t* clr_slot_of;
    const int64_t* clr_count;
    uint32_t* clr_hk;
    uint32_t* clr_hv;
    int64_t* rec_used;
};

constexpr unsigned long long kPairShift = 31;

// Stores only (no result is read back in this call): the other table is not touched by any
// kernel of this call, and the next call on it is stream-ordered after this one.
__device__ __forceinline__ void clear_previous_table(const PadRelabelArgs& a) {
    if (a.clr_slot_of == nullptr) return;
    const int64_t n = *a.clr_count;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
        const int32_t sl = __ldg(a.clr_slot_of + i);
        a.clr_hk[sl] = kEmpty;
        a.clr_hv[sl] = kEmpty;
    }
}   // look-back value = edges << 31 | new nodes

__global__ void __launch_bounds__(kThreads, GD_PAD_MINB) k_relabel_pad(PadRelabelArgs a) {
    GD_PDL_ENTRY();
    clear_tile_state(a.st_clear, a.st_clear_n);
    const int64_t n_prev = a.sizes[a.hop - 1];
    const int64_t tile = blockIdx.x;
    const int64_t i0 = tile * a.nt;
    if (i0 >= n_prev && tile != 0) {
        clear_previous_table(a);
        return;
    }
    const uint32_t f = (uint32_t)a.fanout;
    const uint32_t q0 = (uint32_t)(i0 * f);
    const uint32_t qend = (uint32_t)((i0 + a.nt < n_prev ? i0 + a.nt : n_prev) * f);

    __shared__ uint32_t s_cnt[kPadItems * kWarps];   // (valid << 16 | new) per (round, warp)
    __shared__ unsigned long long s_base;
    const int t = threadIdx.x, lane = t & 31, warp = t >> 5;

    uint32_t slot[kPadItems];
    bool valid[kPadItems];
#pragma unroll
    for (int k = 0; k < kPadItems; ++k) {
        const uint32_t q = q0 + (uint32_t)(k * kThreads + t);
        valid[k] = false;
        slot[k] = 0;
        if (q < qend) {   // both loads at once (pslot past a node's count is stale but in bounds)
            const uint32_t i = q / f;
            const int32_t c = __ldg(a.pcnt + i);
            slot[k] = (uint32_t)__ldg(a.pslot + q);
            valid[k] = q - i * f < (uint32_t)c;
        }
    }
    uint32_t hv0[kPadItems];
    unsigned bv[kPadItems], bn[kPadItems];
#pragma unroll
    for (int k = 0; k < kPadItems; ++k) {
        const uint32_t q = q0 + (uint32_t)(k * kThreads + t);
        hv0[k] = valid[k] ? ld_relaxed_u32(a.hvals + slot[k]) : 0u;
        const bool isnew = valid[k] && hv0[k] == (kPending | q);
        bv[k] = __ballot_sync(0xffffffffu, valid[k]);
        bn[k] = __ballot_sync(0xffffffffu, isnew);
        if (lane == 0) s_cnt[k * kWarps + warp] = ((uint32_t)__popc(bv[k]) << 16) | (uint32_t)__popc(bn[k]);
    }
    __syncthreads();
    if (warp == 0) {
        constexpr int kPer = kPadItems * kWarps / 32;
        uint32_t c[kPer];
        uint32_t sum = 0;
#pragma unroll
        for (int q = 0; q < kPer; ++q) {
            c[q] = s_cnt[kPer * lane + q];
            sum += c[q];
        }
        const uint32_t inc = warp_inclusive_sum(sum);
        const uint32_t agg = __shfl_sync(0xffffffffu, inc, 31);
        __syncwarp();
        uint32_t run = inc - sum;
#pragma unroll
        for (int q = 0; q < kPer; ++q) {
            s_cnt[kPer * lane + q] = run;
            run += c[q];
        }
        const unsigned long long agg64 = ((unsigned long long)(agg >> 16) << kPairShift) | (agg & 0xFFFFu);
        const unsigned long long base = (unsigned long long)lookback_exclusive(a.st, tile, (long long)agg64, 0);
        if (lane == 0) {
            s_base = base;
            const bool last = (n_prev == 0) ? (tile == 0) : (tile == (n_prev - 1) / a.nt);
            if (last) {
                const unsigned long long tot = base + agg64;
                const int64_t edges = (int64_t)(tot >> kPairShift);
                a.rowptr[n_prev] = edges;
                a.sizes[a.K + a.hop] = edges;
                a.sizes[a.hop] = n_prev + (int64_t)(tot & ((1ull << kPairShift) - 1));
                if (a.rec_used) *a.rec_used = a.sizes[a.hop];
            }
        }
    }
    __syncthreads();
    const int64_t ebase = (int64_t)(s_base >> kPairShift);
    const int64_t nbase = (int64_t)(s_base & ((1ull << kPairShift) - 1));
    const unsigned lt = (1u << lane) - 1u;
    // first occurrences take their local ids (n_prev + rank) and finalise the hash value
#pragma unroll
    for (int k = 0; k < kPadItems; ++k) {
        if (bn[k] & (1u << lane)) {
            const uint32_t ex = s_cnt[k * kWarps + warp];
            const int64_t local = n_prev + nbase + (ex & 0xFFFFu) + __popc(bn[k] & lt);
            a.n_id[local] = (int32_t)a.hkeys[slot[k]];
            st_relaxed_u32(a.hvals + slot[k], (uint32_t)local);
            a.slot_of[local] = (int32_t)slot[k];
            hv0[k] = (uint32_t)local;
        }
    }
    // every edge's final col (no k_col_resolve for this hop): a node first seen at an earlier
    // position q' < q of this hop is finalised by the tile owning q' (this one or an earlier one,
    // resident or done, as the look-back already requires): wait for that store
#pragma unroll
    for (int k = 0; k < kPadItems; ++k) {
        const uint32_t q = q0 + (uint32_t)(k * kThreads + t);
        if (q >= qend) continue;
        const uint32_t ex = s_cnt[k * kWarps + warp];
        const int64_t e = ebase + (ex >> 16) + __popc(bv[k] & lt);
        const uint32_t i = q / f;
        if (q == i * f) a.rowptr[i] = e;
        if (valid[k]) {
            uint32_t v = hv0[k];
            int spins = 0;
            while (v >= kPending) {
                if (++spins > 4) __nanosleep(32);
                v = ld_relaxed_u32(a.hvals + slot[k]);
            }
            a.col[e] = (int32_t)v;
            if (a.eid) a.eid[e] = __ldg(a.ppos + q);
        }
    }
    clear_previous_table(a);
}

struct RelabelArgs {
    int32_t* col;
    int32_t* n_id;
    int64_t* sizes;
    int hop;
    int K;
    uint32_t* hkeys;
    uint32_t* hvals;
    int32_t* slot_of;
    unsigned long long* st;
    unsigned long long* st_clear;
    int64_t st_clear_n;
};

__global__ void __launch_bounds__(kThreads) k_relabel_hop(RelabelArgs a) {
    GD_PDL_ENTRY();
    clear_tile_state(a.st_clear, a.st_clear_n);
    const int64_t e_h = a.sizes[a.K + a.hop];
    const int64_t n_prev = a.sizes[a.hop - 1];
    const int64_t tile = blockIdx.x;
    const int64_t e0 = tile * kEdgesPerTile;
    if (e0 >= e_h && tile != 0) return;

    __shared__ int s_cnt[kRelabelItems * kWarps];
    __shared__ long long s_base;
    const int t = threadIdx.x, lane = t & 31, warp = t >> 5;

    uint32_t slot[kRelabelItems];
    unsigned ball[kRelabelItems];
#pragma unroll
    for (int k = 0; k < kRelabelItems; ++k) {
        const int64_t e = e0 + (int64_t)k * kThreads + t;
        bool flag = false;
        slot[k] = 0;
        if (e < e_h) {
            slot[k] = (uint32_t)a.col[e];
            flag = (ld_relaxed_u32(a.hvals + slot[k]) == (kPending | (uint32_t)e));
        }
        ball[k] = __ballot_sync(0xffffffffu, flag);
        if (lane == 0) s_cnt[k * kWarps + warp] = __popc(ball[k]);
    }
    __syncthreads();
    if (warp == 0) {
        // exclusive scan over the kRelabelItems x kWarps (round, warp) counts in edge order,
        // kPer consecutive counts per lane
        constexpr int kPer = kRelabelItems * kWarps / 32;
        int c[kPer];
        int sum = 0;
#pragma unroll
        for (int q = 0; q < kPer; ++q) {
            c[q] = s_cnt[kPer * lane + q];
            sum += c[q];
        }
        const int inc = warp_inclusive_sum(sum);
        const int agg = __shfl_sync(0xffffffffu, inc, 31);
        __syncwarp();
        int run = inc - sum;
#pragma unroll
        for (int q = 0; q < kPer; ++q) {
            s_cnt[kPer * lane + q] = run;
            run += c[q];
        }
        const long long base = lookback_exclusive(a.st, tile, agg, 0);
        if (lane == 0) {
            s_base = base;
            const bool last = (e_h == 0) ? (tile == 0) : (tile == (e_h - 1) / kEdgesPerTile);
            if (last) a.sizes[a.hop] = n_prev + base + agg;
        }
    }
    __syncthreads();
    const long long base = s_base;
    const unsigned lt = (1u << lane) - 1u;
#pragma unroll
    for (int k = 0; k < kRelabelItems; ++k) {
        if (ball[k] & (1u << lane)) {
            const long long rank = base + s_cnt[k * kWarps + warp] + __popc(ball[k] & lt);
            const int64_t local = n_prev + rank;
            a.n_id[local] = (int32_t)a.hkeys[slot[k]];
            a.hvals[slot[k]] = (uint32_t)local;
            a.slot_of[local] = (int32_t)slot[k];
        }
    }
}

struct ColResolveArgs {
    int32_t* col[GD_MAX_HOPS];
    const int64_t* sizes;
    int K;
    const uint32_t* hvals;
};

// One flat pass over the concatenated edges of all hops (hop boundaries from the device sizes),
// 4 edges per thread in flight: each edge is a dependent pair of loads (col, then the hash
// value it names), so the loads of 4 edges are issued before any result is stored.  (A 2-D
// grid with one row of blocks per hop left most blocks of the small hops idle: 18.5 us warm.)
constexpr int kResolveItems = 4;
__global__ void __launch_bounds__(kThreads) k_col_resolve(ColResolveArgs a) {
    GD_PDL_ENTRY();
    int64_t cum[GD_MAX_HOPS + 1];
    cum[0] = 0;
    for (int h = 0; h < a.K; ++h) cum[h + 1] = cum[h] + (a.col[h] ? a.sizes[a.K + 1 + h] : 0);   // null: resolved
    const int64_t total = cum[a.K];
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; base < total; base += stride * kResolveItems) {
        int32_t* ptr[kResolveItems];
        uint32_t slot[kResolveItems];
#pragma unroll
        for (int u = 0; u < kResolveItems; ++u) {
            const int64_t e = base + (int64_t)u * stride;
            ptr[u] = nullptr;
            if (e < total) {
                int h = 0;
                while (e >= cum[h + 1]) ++h;
                ptr[u] = a.col[h] + (e - cum[h]);
                slot[u] = (uint32_t)*ptr[u];
            }
        }
        uint32_t v[kResolveItems];
#pragma unroll
        for (int u = 0; u < kResolveItems; ++u)
            if (ptr[u]) v[u] = __ldg(a.hvals + slot[u]);
#pragma unroll
        for (int u = 0; u < kResolveItems; ++u)
            if (ptr[u]) *ptr[u] = (int32_t)v[u];
    }
}

// Empties exactly the hash slots this call used: every claimed key is a node of n_id (a seed
// or a neighbour, appended at its first occurrence), whose slot k_seed_intake /
// k_relabel_hop recorded.  Replaces a memset of the whole table per call.
__global__ void __launch_bounds__(kThreads) k_hash_clear(const int32_t* __restrict__ slot_of, const int64_t* __restrict__ n_p,
                                                         uint32_t* hk, uint32_t* hv, const int64_t* rec_src, int64_t* rec_dst) {
    GD_PDL_ENTRY();
    const int64_t n = *n_p;
    if (rec_dst && blockIdx.x == 0 && threadIdx.x == 0) *rec_dst = *rec_src;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const int32_t s = slot_of[i];
        hk[s] = kEmpty;
        hv[s] = kEmpty;
    }
}

__global__ void k_validate_csr(const int64_t* indptr, const int32_t* indices, int64_t N, int64_t E,
                               unsigned int* bad) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t t0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    for (int64_t v = t0; v < N; v += stride)
        if (indptr[v + 1] < indptr[v]) atomicOr(bad, 1u);
    if (t0 == 0 && (indptr[0] != 0 || indptr[N] != E)) atomicOr(bad, 2u);
    for (int64_t e = t0; e < E; e += stride) {
        const int32_t u = indices[e];
        if (u < 0 || (int64_t)u >= N) atomicOr(bad, 4u);
    }
}

static int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

static gd_status copy_in(void* dst, const void* src, size_t bytes) {
    GD_CUDA(cudaMemcpy(dst, src, bytes, cudaMemcpyDefault));
    return GD_OK;
}

template <int G>
static void launch_pad_g(const PadHopArgs& a, int64_t n_frontier_max, cudaStream_t st) {
    const unsigned nb = (unsigned)std::max<int64_t>(1, ceil_div(n_frontier_max * G, kThreads));
    launch_chain(k_sample_pad<G>, dim3(nb), dim3(kThreads), 0, st, a);
}

static void launch_sample_pad(const PadHopArgs& a, int64_t n_frontier_max, cudaStream_t st) {
    switch (sampler_group(a.fanout)) {
        case 1: launch_pad_g<1>(a, n_frontier_max, st); break;
        case 2: launch_pad_g<2>(a, n_frontier_max, st); break;
        case 4: launch_pad_g<4>(a, n_frontier_max, st); break;
        case 8: launch_pad_g<8>(a, n_frontier_max, st); break;
        case 16: launch_pad_g<16>(a, n_frontier_max, st); break;
        default: launch_pad_g<32>(a, n_frontier_max, st); break;
    }
}

// grow-only device array (the workspace's steady state never reallocates)
template <typename T>
static gd_status grow(T*& p, int64_t& cap, int64_t want) {
    if (want <= cap) return GD_OK;
    if (p) cudaFree(p);
    p = nullptr;
    cap = 0;
    GD_CUDA(cudaMalloc(&p, std::max<int64_t>(1, want) * sizeof(T)));
    cap = want;
    return GD_OK;
}

}  // namespace gd

void gd_workspace::release_padded() {
    if (pslot) cudaFree(pslot);
    if (ppos) cudaFree(ppos);
    if (pcnt) cudaFree(pcnt);
    pslot = nullptr;
    ppos = nullptr;
    pcnt = nullptr;
    pcap = ppos_cap = pcnt_cap = 0;
}

using namespace gd;

extern "C" {

gd_status gd_sample_bounds(int64_t num_seeds, const int32_t* fanouts, int32_t num_hops, int64_t num_nodes,
                           int64_t num_edges, int64_t* max_nodes, int64_t* max_edges) {
    if (!fanouts || !max_nodes || !max_edges)
        return set_error(GD_ERR_INVALID, "gd_sample_bounds: null pointer");
    if (num_hops < 1 || num_hops > GD_MAX_HOPS)
        return set_error(GD_ERR_INVALID, "gd_sample_bounds: num_hops must be in [1, GD_MAX_HOPS]");
    if (num_seeds < 0 || num_nodes < 0 || num_edges < 0)
        return set_error(GD_ERR_INVALID, "gd_sample_bounds: negative size");
    max_nodes[0] = num_seeds;
    for (int h = 1; h <= num_hops; ++h) {
        const int32_t f = fanouts[h - 1];
        if (f < -1 || f > GD_MAX_FANOUT)
            return set_error(GD_ERR_INVALID, "gd_sample_bounds: fanout must be -1 or in [0, 256]");
        int64_t e;
        if (f < 0) {
            e = num_edges;
        } else {
            const int64_t prev = max_nodes[h - 1];
            e = (f == 0 || prev <= num_edges / f) ? std::min<int64_t>(num_edges, prev * f) : num_edges;
        }
        max_edges[h - 1] = e;
        max_nodes[h] = std::min<int64_t>(num_nodes, max_nodes[h - 1] + e);
    }
    return GD_OK;
}

gd_status gd_graph_create(const int64_t* indptr, const int32_t* indices, int64_t num_nodes, int64_t num_edges,
                          int device, int validate, gd_graph** out) {
    if (!indptr || !out || (num_edges > 0 && !indices))
        return set_error(GD_ERR_INVALID, "gd_graph_create: null pointer");
    if (num_nodes < 1 || num_nodes > 0x7FFFFFFFLL || num_edges < 0)
        return set_error(GD_ERR_INVALID, "gd_graph_create: need 1 <= num_nodes <= 2^31-1, num_edges >= 0");
    DeviceGuard guard(device);
    GD_CUDA(cudaSetDevice(device));
    gd_graph* g = new gd_graph();
    g->hdr.magic = kMagicGraph;
    g->hdr.device = device;
    g->N = num_nodes;
    g->E = num_edges;
    if (const char* e = std::getenv("GD_SAMPLE_PAD")) g->sample_padded = e[0] != '0';
    if (const char* e = std::getenv("GD_HASH_CLEAR_KERNEL")) g->fold_clear = e[0] != '1';
    auto fail = [&](gd_status s) {
        gd_graph_destroy(g);
        return s;
    };
    if (cudaMalloc(&g->hdr.dev_status, sizeof(unsigned int)) != cudaSuccess ||
        cudaMalloc(&g->indptr, (num_nodes + 1) * sizeof(int64_t)) != cudaSuccess ||
        cudaMalloc(&g->indices, std::max<int64_t>(1, num_edges) * sizeof(int32_t)) != cudaSuccess) {
        cudaGetLastError();
        return fail(set_error(GD_ERR_OOM, "gd_graph_create: cudaMalloc failed for the topology replica"));
    }
    gd_status s;
    if ((s = copy_in(g->indptr, indptr, (num_nodes + 1) * sizeof(int64_t))) != GD_OK) return fail(s);
    if (num_edges > 0 && (s = copy_in(g->indices, indices, num_edges * sizeof(int32_t))) != GD_OK) return fail(s);
    if (cudaMemset(g->hdr.dev_status, 0, sizeof(unsigned int)) != cudaSuccess)
        return fail(cuda_error(cudaGetLastError(), "cudaMemset"));
    if (validate) {
        unsigned int* bad = nullptr;
        if (cudaMalloc(&bad, sizeof(unsigned int)) != cudaSuccess) return fail(cuda_error(cudaGetLastError(), "cudaMalloc"));
        cudaMemset(bad, 0, sizeof(unsigned int));
        k_validate_csr<<<148 * 8, 256>>>(g->indptr, g->indices, num_nodes, num_edges, bad);
        unsigned int hb = 0;
        cudaError_t e = cudaMemcpy(&hb, bad, sizeof(hb), cudaMemcpyDeviceToHost);
        cudaFree(bad);
        if (e != cudaSuccess) return fail(cuda_error(e, "k_validate_csr"));
        if (hb)
            return fail(set_error(GD_ERR_INVALID, std::string("gd_graph_create: invalid CSR (") +
                                                      ((hb & 1) ? "indptr not monotone " : "") +
                                                      ((hb & 2) ? "indptr[0]!=0 or indptr[N]!=E " : "") +
                                                      ((hb & 4) ? "index out of range" : "") + ")"));
    }
    *out = g;
    return GD_OK;
}

gd_status gd_graph_destroy(gd_graph* g) {
    if (!g) return GD_OK;
    DeviceGuard guard(g->hdr.device);
    if (g->indptr) cudaFree(g->indptr);
    if (g->indices) cudaFree(g->indices);
    if (g->ws.hash) cudaFree(g->ws.hash);
    if (g->ws.slot_of) cudaFree(g->ws.slot_of);
    if (g->ws.used) cudaFree(g->ws.used);
    if (g->ws.seeds_ws) cudaFree(g->ws.seeds_ws);
    g->ws.release_padded();
    if (g->hdr.dev_status) cudaFree(g->hdr.dev_status);
    g->ws.scan.release();
    g->timer.destroy();
    g->hdr.magic = 0;
    delete g;
    return GD_OK;
}

gd_status gd_workspace_create(gd_graph* g, gd_workspace** out) {
    if (!g || g->hdr.magic != kMagicGraph || !out) return set_error(GD_ERR_INVALID, "gd_workspace_create: bad argument");
    gd_workspace* w = new gd_workspace();
    w->device = g->hdr.device;
    *out = w;
    return GD_OK;
}

gd_status gd_workspace_destroy(gd_workspace* w) {
    if (!w) return GD_OK;
    if (w->magic != 0x47445753u) return set_error(GD_ERR_INVALID, "gd_workspace_destroy: bad handle");
    DeviceGuard guard(w->device);
    if (w->hash) cudaFree(w->hash);
    if (w->slot_of) cudaFree(w->slot_of);
    if (w->used) cudaFree(w->used);
    if (w->seeds_ws) cudaFree(w->seeds_ws);
    w->release_padded();
    w->scan.release();
    w->magic = 0;
    delete w;
    return GD_OK;
}

gd_status gd_sample(gd_graph* g, const int32_t* seeds, int64_t num_seeds, const int32_t* fanouts, int32_t num_hops,
                    uint64_t rng_seed, uint32_t batch_id, gd_sample_out* out, void* stream_v) {
    return gd_sample_ws(g, nullptr, seeds, num_seeds, fanouts, num_hops, rng_seed, batch_id, out, stream_v);
}

gd_status gd_sample_ws(gd_graph* g, gd_workspace* wsp, const int32_t* seeds, int64_t num_seeds,
                       const int32_t* fanouts, int32_t num_hops, uint64_t rng_seed, uint32_t batch_id,
                       gd_sample_out* out, void* stream_v) {
    if (!g || g->hdr.magic != kMagicGraph) return set_error(GD_ERR_INVALID, "gd_sample: bad graph handle");
    if (wsp && (wsp->magic != 0x47445753u || wsp->device != g->hdr.device))
        return set_error(GD_ERR_INVALID, "gd_sample_ws: bad workspace handle");
    gd_workspace& w = wsp ? *wsp : g->ws;
    if (!out || !fanouts || (num_seeds > 0 && !seeds) || !out->n_id || !out->sizes)
        return set_error(GD_ERR_INVALID, "gd_sample: null pointer");
    int64_t nmax[GD_MAX_HOPS + 1], emax[GD_MAX_HOPS];
    gd_status s = gd_sample_bounds(num_seeds, fanouts, num_hops, g->N, g->E, nmax, emax);
    if (s != GD_OK) return s;
    if (num_seeds > g->N) return set_error(GD_ERR_INVALID, "gd_sample: more seeds than nodes");
    for (int h = 0; h < num_hops; ++h) {
        if (!out->rowptr[h] || (!out->col[h] && emax[h] > 0))
            return set_error(GD_ERR_INVALID, "gd_sample: null rowptr/col for a hop");
        if (emax[h] >= (int64_t)kPending)
            return set_error(GD_ERR_INVALID, "gd_sample: a hop may sample >= 2^31 edges");
    }
    DeviceGuard guard(g->hdr.device);
    cudaStream_t st = (cudaStream_t)stream_v;

    // workspace (grows on first use of a larger shape; not on the steady-state path)
    // capacity: power of two >= 1.25 x the worst-case node count (load <= 0.8 at the bound;
    // real batches reach 30-70% of the bound), so the per-batch clear stays small
    int64_t want = 1024;
    while (want < std::max<int64_t>(nmax[num_hops], 1) * 5 / 4 + 1) want *= 2;
    if (want > w.hcap || nmax[num_hops] > w.slot_cap || !w.used) {
        // (re)allocate; both tables start empty and no call's slots are pending
        if (want > w.hcap) {
            if (w.hash) cudaFree(w.hash);
            w.hash = nullptr;
            w.hcap = 0;
            GD_CUDA(cudaMalloc(&w.hash, 4 * want * sizeof(uint32_t)));
            w.hcap = want;
        }
        if (nmax[num_hops] > w.slot_cap) {
            if (w.slot_of) cudaFree(w.slot_of);
            w.slot_of = nullptr;
            w.slot_cap = 0;
            GD_CUDA(cudaMalloc(&w.slot_of, 2 * std::max<int64_t>(1, nmax[num_hops]) * sizeof(int32_t)));
            GD_CUDA(cudaMemsetAsync(w.slot_of, 0, 2 * std::max<int64_t>(1, nmax[num_hops]) * sizeof(int32_t), st));
            w.slot_cap = std::max<int64_t>(1, nmax[num_hops]);
        }
        if (!w.used) GD_CUDA(cudaMalloc(&w.used, 2 * sizeof(int64_t)));
        GD_CUDA(cudaMemsetAsync(w.hash, 0xFF, 4 * w.hcap * sizeof(uint32_t), st));
        GD_CUDA(cudaMemsetAsync(w.used, 0, 2 * sizeof(int64_t), st));
    }
    int64_t tiles = 1;
    for (int h = 0; h < num_hops; ++h) {
        tiles = std::max(tiles, ceil_div(nmax[h], 8));   // smallest sampler tile: 8 nodes
        tiles = std::max(tiles, ceil_div(emax[h], kEdgesPerTile));
    }
    if ((s = w.scan.ensure(tiles)) != GD_OK) return s;

    const int32_t* seeds_d = seeds;
    // pinned host seeds are read by k_seed_intake through the mapping (a few KB): a copy-engine
    // transfer would queue behind the miss stream's bulk H2D copies and stall this stream
    const int32_t* mapped = (num_seeds > 0 && !is_device_pointer(seeds)) ? (const int32_t*)mapped_host_pointer(seeds) : nullptr;
    if (mapped) {
        seeds_d = mapped;
    } else if (num_seeds > 0 && !is_device_pointer(seeds)) {   // pageable host memory: staged copy
        if (num_seeds > w.seeds_cap) {
            if (w.seeds_ws) cudaFree(w.seeds_ws);
            w.seeds_ws = nullptr;
            w.seeds_cap = 0;
            GD_CUDA(cudaMalloc(&w.seeds_ws, num_seeds * sizeof(int32_t)));
            w.seeds_cap = num_seeds;
        }
        GD_CUDA(cudaMemcpyAsync(w.seeds_ws, seeds, num_seeds * sizeof(int32_t), cudaMemcpyHostToDevice, st));
        seeds_d = w.seeds_ws;
    }

    const int tb = w.tsel, tp = tb ^ 1;     // this call's table, the previous call's
    w.tsel = tp;
    uint32_t* hk = w.hash + 2 * tb * w.hcap;
    uint32_t* hv = hk + w.hcap;
    int32_t* slot_of = w.slot_of + tb * w.slot_cap;
    const uint32_t mask = (uint32_t)(w.hcap - 1);
    const int tslot = g->timer.on ? g->timer.begin(st) : -1;
    GD_CUDA(launch_chain(k_seed_intake, dim3((unsigned)std::max<int64_t>(1, ceil_div(num_seeds, kThreads))), dim3(kThreads),
                         0, st, seeds_d, num_seeds, g->N, hk, hv, mask, out->n_id, out->sizes, slot_of, g->hdr.dev_status));

    bool resolved[GD_MAX_HOPS] = {};
    bool cleared_prev = false;   // the last hop's relabel emptied the previous call's table
    for (int h = 1; h <= num_hops; ++h) {
        const int f = fanouts[h - 1];
        if (g->sample_padded && f >= 1 && f <= 32 && nmax[h - 1] * f < (int64_t)kPending) {
            const int64_t np = nmax[h - 1] * f;
            if ((s = grow(w.pslot, w.pcap, np)) != GD_OK) return s;
            if ((s = grow(w.pcnt, w.pcnt_cap, nmax[h - 1])) != GD_OK) return s;
            if (out->eid[h - 1] && (s = grow(w.ppos, w.ppos_cap, np)) != GD_OK) return s;
            PadHopArgs a;
            a.indptr = g->indptr;
            a.indices = g->indices;
            a.N = g->N;
            a.n_id = out->n_id;
            a.sizes = out->sizes;
            a.hop = h;
            a.fanout = f;
            a.batch = batch_id;
            a.seed = rng_seed;
            a.pslot = w.pslot;
            a.ppos = out->eid[h - 1] ? w.ppos : nullptr;
            a.pcnt = w.pcnt;
            a.hkeys = hk;
            a.hvals = hv;
            a.mask = mask;
            launch_sample_pad(a, nmax[h - 1], st);
            GD_DEBUG_AFTER("k_sample_pad", st);

            PadRelabelArgs r;
            r.pslot = w.pslot;
            r.ppos = a.ppos;
            r.pcnt = w.pcnt;
            r.rowptr = out->rowptr[h - 1];
            r.col = out->col[h - 1];
            r.eid = out->eid[h - 1];
            r.n_id = out->n_id;
            r.sizes = out->sizes;
            r.hop = h;
            r.K = num_hops;
            r.fanout = f;
            r.nt = kPadPerTile / f;
            r.hkeys = hk;
            r.hvals = hv;
            r.slot_of = slot_of;
            const bool last_hop = h == num_hops && g->fold_clear;
            r.clr_slot_of = last_hop ? w.slot_of + tp * w.slot_cap : nullptr;
            r.clr_count = w.used + tp;
            r.clr_hk = w.hash + 2 * tp * w.hcap;
            r.clr_hv = r.clr_hk + w.hcap;
            r.rec_used = last_hop ? w.used + tb : nullptr;
            cleared_prev = cleared_prev || last_hop;
            r.st = w.scan.use();
            r.st_clear = w.scan.other();
            r.st_clear_n = w.scan.clear_n();
            const int64_t et = std::max<int64_t>(1, ceil_div(nmax[h - 1], r.nt));
            GD_CUDA(launch_chain(k_relabel_pad, dim3((unsigned)et), dim3(kThreads), 0, st, r));
            GD_DEBUG_AFTER("k_relabel_pad", st);
            w.scan.launched(et);
            resolved[h - 1] = true;
            continue;
        }
        SampleHopArgs a;
        a.indptr = g->indptr;
        a.indices = g->indices;
        a.N = g->N;
        a.n_id = out->n_id;
        a.sizes = out->sizes;
        a.hop = h;
        a.K = num_hops;
        a.fanout = fanouts[h - 1];
        a.batch = batch_id;
        a.seed = rng_seed;
        a.rowptr = out->rowptr[h - 1];
        a.col = out->col[h - 1];
        a.eid = out->eid[h - 1];
        a.hkeys = hk;
        a.hvals = hv;
        a.mask = mask;
        a.st = w.scan.use();
        a.st_clear = w.scan.other();
        a.st_clear_n = w.scan.clear_n();
        a.status = g->hdr.dev_status;
        launch_sample_hop(a, nmax[h - 1], st);
        GD_DEBUG_AFTER("k_sample_hop", st);
        w.scan.launched(w.scan.cap);

        RelabelArgs r;
        r.col = out->col[h - 1];
        r.n_id = out->n_id;
        r.sizes = out->sizes;
        r.hop = h;
        r.K = num_hops;
        r.hkeys = hk;
        r.hvals = hv;
        r.slot_of = slot_of;
        r.st = w.scan.use();
        r.st_clear = w.scan.other();
        r.st_clear_n = w.scan.clear_n();
        const int64_t et = std::max<int64_t>(1, ceil_div(emax[h - 1], kEdgesPerTile));
        GD_CUDA(launch_chain(k_relabel_hop, dim3((unsigned)et), dim3(kThreads), 0, st, r));
        GD_DEBUG_AFTER("k_relabel_hop", st);
        w.scan.launched(et);
    }
    ColResolveArgs c;
    int64_t esum = 0;
    for (int h = 0; h < num_hops; ++h) {
        c.col[h] = resolved[h] ? nullptr : out->col[h];
        if (!resolved[h]) esum += emax[h];
    }
    c.sizes = out->sizes;
    c.K = num_hops;
    c.hvals = hv;
    if (esum > 0) {   // hops of the count-scan form only (padded hops wrote their final col)
        dim3 grid((unsigned)std::min<int64_t>(148 * 8, std::max<int64_t>(1, ceil_div(esum, kThreads * kResolveItems))));
        GD_CUDA(launch_chain(k_col_resolve, grid, dim3(kThreads), 0, st, c));
    }
    if (!cleared_prev) {   // last hop of the count-scan form: empty the previous call's table here
        uint32_t* phk = w.hash + 2 * tp * w.hcap;
        GD_CUDA(launch_chain(k_hash_clear, dim3((unsigned)std::min<int64_t>(148 * 8, std::max<int64_t>(1, ceil_div(nmax[num_hops], kThreads)))),
                             dim3(kThreads), 0, st, (const int32_t*)(w.slot_of + tp * w.slot_cap), (const int64_t*)(w.used + tp),
                             phk, phk + w.hcap, (const int64_t*)(out->sizes + num_hops), w.used + tb));
    }
        GD_DEBUG_AFTER("k_col_resolve", st);
    if (tslot >= 0) g->timer.end(tslot, st);
    GD_CUDA(cudaGetLastError());
    return GD_OK;
}

gd_status gd_graph_sampler(gd_graph* g, int padded) {
    if (!g || g->hdr.magic != kMagicGraph) return set_error(GD_ERR_INVALID, "gd_graph_sampler: bad handle");
    g->sample_padded = padded != 0;
    return GD_OK;
}

gd_status gd_graph_timing(gd_graph* g, int enable) {
    if (!g || g->hdr.magic != kMagicGraph) return set_error(GD_ERR_INVALID, "gd_graph_timing: bad handle");
    DeviceGuard guard(g->hdr.device);
    if (enable) {
        g->timer.reset();
        g->timer.reserve(4096);      // events for 4096 calls, created before the timed region
    }
    g->timer.on = enable != 0;
    return GD_OK;
}

gd_status gd_graph_timing_read(gd_graph* g, double* sample_ms, int64_t* calls) {
    if (!g || g->hdr.magic != kMagicGraph) return set_error(GD_ERR_INVALID, "gd_graph_timing_read: bad handle");
    DeviceGuard guard(g->hdr.device);
    if (sample_ms) *sample_ms = g->timer.total_ms(1, 0);
    if (calls) *calls = (int64_t)g->timer.pairs.size();
    GD_CUDA(cudaGetLastError());
    return GD_OK;
}

}  // extern "C"
