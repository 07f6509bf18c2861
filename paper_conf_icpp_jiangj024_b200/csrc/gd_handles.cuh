// gd_handles.cuh — layouts of the two opaque handles of libgd.so.
#pragma once

#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include <vector>

#include "gd_common.cuh"
#include "gd_hostpool.h"

// Per-call sampling workspace; one per concurrently sampling stream.
struct gd_workspace {
    uint32_t magic = 0x47445753u;   // "GDWS"
    int device = 0;
    uint32_t* hash = nullptr;       // two tables, table t at hash + 2 t hcap: keys [hcap] then
                                    // values [hcap] (L2-resident).  Calls alternate tables; a call
                                    // empties the slots the previous call used in the other table
                                    // (inside its last relabel pass), so a table is empty when used
    int64_t hcap = 0;               // power of two >= 1.25 x max_nodes[K]
    int32_t* slot_of = nullptr;     // [2 slot_cap] hash slot of n_id[i], table t at slot_of + t slot_cap
    int64_t slot_cap = 0;
    int64_t* used = nullptr;        // device [2]: entries of slot_of of the last call on table t
    int tsel = 0;                   // table of the next call
    int32_t* seeds_ws = nullptr;    // staging for host seed arrays
    int64_t seeds_cap = 0;
    int32_t* pslot = nullptr;       // padded hop: [pcap] hash slot of draw q = i f + r
    int64_t* ppos = nullptr;        // padded hop: [ppos_cap] CSR position of draw q (eid requested)
    int32_t* pcnt = nullptr;        // padded hop: [pcnt_cap] min(f, deg) of frontier node i
    int64_t pcap = 0, ppos_cap = 0, pcnt_cap = 0;
    gd::ScanState scan;
    void release_padded();
};

// Topology replica + its default workspace.
struct gd_graph {
    gd::HandleHdr hdr;
    int64_t N = 0, E = 0;
    int64_t* indptr = nullptr;      // HBM int64[N+1]
    int32_t* indices = nullptr;     // HBM int32[E]
    gd_workspace ws;                // used by gd_sample
    int fold_clear = 1;             // padded last hop empties the previous table (GD_HASH_CLEAR_KERNEL=1: k_hash_clear)
    int sample_padded = 1;          // padded hops for 1 <= f <= 32 (GD_SAMPLE_PAD=0 / gd_graph_sampler)
    gd::EventTimer timer;           // one pair per gd_sample call
};

// Control block of the standby ring.  Kernels that move head/tail read ctl[p] and
// write ctl[p^1]; the host flips p after each such launch (no in-kernel RAW race).
// The ring is one array of 2C positions: the live window [head, tail) lies in the
// half starting at `base` (0 or C); compaction copies the live entries to the other
// half, so a new position can never equal a stale one.
struct GdCtl {
    long long head;       // first ring position that may hold a live entry
    long long tail;       // next free ring position
    long long base;       // start of the current half (0 or C)
};

struct gd_buffer;

namespace gd {
constexpr int kMaxPeers = 7;
constexpr unsigned long long kReadyNone = ~0ull;
struct PeerView {
    const int2* map[kMaxPeers];
    const unsigned long long* ready[kMaxPeers];
    const uint8_t* slots[kMaxPeers];
};
}  // namespace gd

// One slot of the staged miss path (phase 1 host gather -> phase 2 contiguous pull).
struct ChunkJob {
    struct StagedSlot* ss = nullptr;
    int64_t lo = 0, hi = 0;   // staged ranks [lo, hi) of this chunk
    uint8_t* buf = nullptr;   // pinned ring buffer the chunk is gathered into
    bool first = false;       // first chunk of the batch (resets the batch's cpu_ms)
};

struct StagedSlot {
    gd_buffer* owner = nullptr;
    int d = 0;
    int32_t* h_nodes = nullptr;   // pinned, mapped [n_max]: node ids of the staged share
    int64_t* h_meta = nullptr;    // pinned, mapped [8]: M, K0, staged rows, -, (epoch << 32 | M) of the
                                  // newest batch that used this slot (read for the staging size)
    uint8_t* staging = nullptr;   // pinned, mapped [n_max x R]
    double cpu_ms = 0;            // duration of the last host gather into this slot
    int64_t batch = -1;           // batch that last used this slot
    uint64_t epoch = 0;           // that batch's epoch (its published miss-count word carries it)
    bool zc_timed = false;        // its zero-copy kernel was bracketed by ev_z0 / ev_z1
};

// Hill-climbing tuner of the zero-copy share: the cost of a share is the
// extraction period per miss over a window of completed batches (done-to-done event time /
// their misses); the tuner moves the share by `step` while that improves, turns back when it
// gets worse, halves the step after failing on both sides, and freezes at the best share.
struct ShareTuner {
    bool on = false;
    bool frozen = false;
    int phase = 0;                 // 0: settling after a change, 1: measuring
    int64_t change_batch = 0;      // first batch enqueued with the current share
    int64_t w_b0 = -1;             // window start: batch, its completion time (ms since ev_ref)
    double w_t0 = 0;
    double alpha = 0.1;            // share under test
    double best_alpha = 0.1, best_cost = 0;
    bool have_best = false;
    int dir = +1, fails = 0, windows = 0;
    double step = 0.05;
    int64_t mb[64];                // per-batch miss counts seen so far: batch id and count, ring
    int64_t mc[64];
};

// Feature buffer + extraction workspace.
struct gd_buffer {
    gd::HandleHdr hdr;
    int64_t N = 0, R = 0, S = 0;     // nodes, row bytes, slots
    int64_t P = 0;                   // host table rows: node v's row is v mod P (P = N normally)
    int64_t C = 0;                   // ring capacity per half
    int64_t n_max = 0;               // max nodes per batch
    int32_t Q = 0;                   // max in-flight (extracted, unreleased) batches
    int preload = 0;
    const void* host_feat = nullptr;
    const uint8_t* feat_dev = nullptr;   // device alias of the pinned host table
    bool registered = false;             // we registered host_feat ourselves
    uint8_t* slots = nullptr;            // HBM [S x R]
    int2* map = nullptr;                 // HBM [N]: {slot, rc << 1 | valid}
    int32_t* reverse = nullptr;          // HBM [S]
    int32_t* pos_of_slot = nullptr;      // HBM [S]: ring position of a slot's live entry, or -1
    int32_t* ring = nullptr;             // HBM [2C]: slots in LRU order, lazy deletion
    GdCtl* ctl = nullptr;                // HBM [2]
    int ctl_parity = 0;
    // per-batch workspace used on the caller's stream
    int2* misslist = nullptr;            // [n_max] {batch position, node} of the misses, list order
    int2* hitlist = nullptr;             // [D][n_max] {position, slot} of the hits (read on stream G)
    int64_t* hcount = nullptr;           // [D] number of hits
    int32_t* alias_ws = nullptr;         // [D][n_max] used when the caller passes alias = NULL
    int64_t* mcount = nullptr;           // [1] misses of the current batch
    // miss triples for the side stream, a ring of D batches
    int D = 0;
    int4* trip = nullptr;                // [D][n_max] {node, slot, batch position, 0}
    int64_t* trip_count = nullptr;       // [D]
    unsigned long long* tickets = nullptr;   // [6] {ticket, finished} x 3 kernels (pop, compact, gather)
    bool gather_dynamic = true;          // hit gather: dynamic row assignment (GD_GATHER_DYNAMIC)
    bool gather_tma = false;             // hit gather by TMA gather4 (GD_GATHER_TMA=1)
    int gather_bps = 4;                  // hit gather: 256-thread blocks per SM (GD_GATHER_BPS)
    bool zc_after_gather = false;        // zero-copy kernel of batch b after the hit gather of b (GD_ZC_AFTER_GATHER)
    int gather_u = 4;                    // hit gather, rows <= 512 B: rows in flight per warp (GD_GATHER_U: 4 | 8)
    CUtensorMap slot_map;                // tensor map over the slots for the TMA gather
    unsigned long long* done_word = nullptr; // [1] epoch-tagged early-exit word of the pop scan
    gd::ScanState scan;
    cudaStream_t side = nullptr;         // Z: zero-copy share of the misses
    cudaStream_t side_h = nullptr;       // H: host gather (phase 1) of the staged share
    cudaStream_t side_p = nullptr;       // P: contiguous pull (phase 2) of the staged share
    cudaStream_t side_j = nullptr;       // J: joins Z, P and the hit gather into `done`
    cudaStream_t side_g = nullptr;       // G: hit gather (slots -> out)
    cudaEvent_t ev_L = nullptr, ev_X = nullptr, ev_Xs = nullptr, ev_G = nullptr;
    cudaEvent_t ev_S = nullptr;          // f2: peer probe + split done (stream Z)
    std::vector<cudaEvent_t> ev_trip;    // [D] every stream finished with trip ring slot d
    std::vector<cudaEvent_t> ev_E, ev_P; // [D] staging slot d ready in HBM or pinned / staged pull done
    std::vector<cudaEvent_t> ev_H;       // [D] host gather of slot d done (copy-engine mode)
    cudaStream_t side_c = nullptr;       // C: copy-engine H2D of the staged share
    std::vector<cudaEvent_t> ev_z0, ev_z1;   // [D] timing of the zero-copy path (every 8th batch)
    int64_t* trip_split = nullptr;       // [D] K0: misses [0, K0) zero-copy, [K0, M) staged
    int host_threads = 0;                // 0: staged path off (all misses zero-copy)
    int zc_blocks = 16;                  // 1024-thread blocks (~whole SMs) of the zero-copy copy
    int pull_blocks = 8;                 // 1024-thread blocks of the staged pull
    double alpha = 1.0;                  // zero-copy share of the misses (adapted)
    double r_host = 0;                   // EMA of the host gather rate (bytes/ms)
    double r_zc = 0;                     // EMA of the zero-copy copy rate (bytes/ms)
    double r_link = 0;                   // contiguous pull rate of the host link (bytes/ms), calibrated
    bool alpha_fixed = false;
    int64_t rate_samples = 0;            // host-gather rate samples since the last config
    int64_t rated_batch = -1;            // newest batch whose path rates entered the estimates
    ShareTuner tune;                     // GD_SHARE_TUNER=0: model-based share only
    std::vector<cudaEvent_t> ev_fin;     // [D] timing: batch d's extraction complete (stream J join)
    cudaEvent_t ev_ref = nullptr;        // timing reference of ev_fin
    gd::HostGatherPool* pool = nullptr;
    // phase 2 of the staged share: copy engine (cudaMemcpyAsync pinned slot -> dstage[d]
    // on stream H, then a scatter kernel on P) or an SM pull kernel reading the pinned slot
    bool ce_mode = true;
    uint8_t* dstage = nullptr;           // HBM [D][n_max x R] (copy-engine mode)
    double m_est = 0;                    // misses of a recently completed batch
    // chunked copy-engine staging (stage_chunk_rows > 0): the host gathers chunk c of the
    // staged share into ring buffer (k mod stage_ring) of a small pinned ring that stays
    // in the CPU caches, and the copy engine moves each chunk as soon as it is gathered
    int64_t stage_chunk_rows = 0;        // ring buffer stride (max chunk) in rows
    bool chunk_adaptive = true;          // per-batch chunk = staged share / 6, in [8, 16] MB
    uint8_t* ring_mem = nullptr;         // pinned [stage_ring x stage_chunk_rows x R]
    int stage_ring = 4;                  // ring buffers (env GD_STAGE_RING)
    uint64_t chunk_counter = 0;
    // host-function arguments of the staged chunks: a ring indexed by a global job counter, so
    // a pending callback's arguments are never rewritten by a later batch's enqueue (slot k is
    // reused only after ev_job[k], recorded after its callback, has fired)
    std::vector<cudaEvent_t> ev_job;
    uint64_t job_counter = 0;
    std::vector<cudaEvent_t> ev_ring;    // [kStageRingMax] copy out of ring buffer r done
    cudaEvent_t ev_chunk = nullptr;      // chunk gathered (re-recorded per chunk)
    std::vector<struct ChunkJob> jobs;   // [kJobRing] host-function arguments (see ev_job)
    // f2: NVLink peer feature buffers (subprocesses reuse rows another has loaded).
    // ready[s] = (epoch << 32) | node once slot s holds that node's row (published after
    // the batch's copies joined), kReadyNone from the moment the slot is reassigned.
    unsigned long long* ready = nullptr; // HBM [S]
    int npeers = 0;
    bool publish = false;                // tags maintained (someone can read them as a peer)
    gd::PeerView peers;                  // device pointers of the peers' map / ready / slots
    std::vector<void*> ipc_opened;       // pointers opened with cudaIpcOpenMemHandle (closed at destroy)
    int4* trip2 = nullptr;               // [D][n_max] misses no peer served (compacted)
    int64_t* trip2_count = nullptr;      // [D]
    int64_t* trip2_split = nullptr;      // [D]
    unsigned long long* peer_ctr = nullptr;   // [2] rows served by peers, misses probed
    std::vector<StagedSlot> stg;
    uint8_t* stage_mem = nullptr;        // pinned allocations behind stg
    int32_t* hnodes_mem = nullptr;
    int64_t* hmeta_mem = nullptr;
    gd::EventTimer timer;                // 4 pairs per gd_extract: bookkeeping, gather, zero-copy, pull
    double timer_host_ms = 0;            // host gather time while timing is on
    int64_t batch_counter = 0;
    int64_t inflight = 0;
    unsigned long long epoch = 1;
};
