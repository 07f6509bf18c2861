/*
 * gd.h — C ABI of the B200-native GNNDrive sample + extract hot path.
 *
 * Paper: Jiang, Jia, Wang, "Reducing Memory Contention and I/O Congestion for
 * Disk-based GNN Training" (ICPP'24, "GNNDrive").  "P:NNN" cites line NNN of the
 * paper text (reference PAPER.md); "Alg. 1" is its Algorithm 1;
 * readings R<k> are listed in DESIGN.md §3.
 *
 * Conventions for every entry point
 *   - Returns a gd_status; no exception crosses the ABI.  On a non-OK status
 *     gd_last_error() gives a thread-local message and no library state changed.
 *   - "device" pointers are CUDA device (or managed) pointers on the handle's
 *     device; "host or device" pointers are detected with cudaPointerGetAttributes.
 *   - Every array argument is caller-owned; the library never frees it.  Library
 *     state (HBM topology copy, hash workspace, mapping table, reverse map,
 *     standby ring, slots, internal side stream and events) is owned by the handle
 *     and released by the matching *_destroy.
 *   - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).
 *     Every call is stream-ordered on it and does NOT synchronise the host on the
 *     hot path (gd_sample / gd_extract / gd_buffer_release).  Calls on one handle
 *     must be externally serialised and ordered on one stream.
 *   - Device-side precondition violations (duplicate / out-of-range seed or node
 *     id, refcount underflow, exhausted standby list) cannot be detected on the
 *     host without a sync; they set a sticky status word on the handle, reported
 *     by gd_check_device_status().  Outputs of such a call are unspecified but all
 *     memory accesses stay in bounds.
 */
#ifndef GD_H_
#define GD_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define GD_MAX_HOPS 8
#define GD_MAX_FANOUT 256   /* largest sampled fanout; -1 (= whole row) is also allowed */

typedef enum {
    GD_OK = 0,
    GD_ERR_INVALID = 1,     /* bad argument (null pointer, size, hop count, fanout, CSR) */
    GD_ERR_OOM = 2,         /* device or pinned allocation failed */
    GD_ERR_CUDA = 3,        /* a CUDA runtime call failed */
    GD_ERR_CAPACITY = 4,    /* buffer capacity / in-flight rule violated */
    GD_ERR_DEVICE = 5       /* a device-side precondition check tripped (sticky) */
} gd_status;

/* device status bits (gd_check_device_status sets *bits) */
#define GD_DEV_BAD_ID       0x1u   /* seed or node id outside [0, N) */
#define GD_DEV_DUP_SEED     0x2u   /* a seed appears twice in one gd_sample call */
#define GD_DEV_UNDERFLOW    0x4u   /* gd_buffer_release of a node with refcount 0 */
#define GD_DEV_STANDBY_DRY  0x8u   /* fewer standby slots than misses (capacity rule broken) */

typedef struct gd_graph gd_graph;
typedef struct gd_buffer gd_buffer;

/* Thread-local message describing the last non-OK status ("" if none). */
const char* gd_last_error(void);

/* Library version (major*10000 + minor*100 + patch). */
int gd_version(void);

/* ----------------------------------------------------------------------------
 * Topology.  GNNDrive "forms the topological data of a graph as an adjacency
 * matrix for efficient sampling" in compressed form (indptr / indices,
 * P:146).  Reading R6: row v lists the nodes v samples from (pass the CSC
 * of A, i.e. the CSR of A^T, to sample in-neighbours as P:41 does).
 *
 *   indptr   host or device int64[num_nodes+1], indptr[0] = 0, non-decreasing,
 *            indptr[num_nodes] = num_edges.
 *   indices  host or device int32[num_edges], each in [0, num_nodes).
 *   validate nonzero: check the CSR on the device once (GD_ERR_INVALID on failure).
 * The library copies both arrays into HBM on `device` (a replica per GPU)
 * and keeps no reference to the caller's arrays.  num_nodes <= 2^31-1.
 * ------------------------------------------------------------------------- */
gd_status gd_graph_create(const int64_t* indptr, const int32_t* indices, int64_t num_nodes,
                          int64_t num_edges, int device, int validate, gd_graph** out);
gd_status gd_graph_destroy(gd_graph* g);

/* Host-only worst-case sizes of one gd_sample call (no device work).  The last entry,
 * max_nodes[K], is the paper's M_b, "the maximum number of nodes in a mini-batch" that sizes
 * the feature buffer's N_e x M_b reservation; the rest size gd_sample_out.
 *   max_nodes[0] = num_seeds,
 *   max_edges[h-1] = f_h < 0 ? num_edges : min(num_edges, max_nodes[h-1] * f_h),
 *   max_nodes[h]   = min(num_nodes, max_nodes[h-1] + max_edges[h-1]),  h = 1..num_hops.
 * max_nodes has num_hops+1 entries, max_edges num_hops. */
gd_status gd_sample_bounds(int64_t num_seeds, const int32_t* fanouts, int32_t num_hops,
                           int64_t num_nodes, int64_t num_edges, int64_t* max_nodes,
                           int64_t* max_edges);

/* Caller-allocated device outputs of gd_sample, sized from gd_sample_bounds. */
typedef struct {
    int32_t* n_id;                    /* [max_nodes[K]] sampled node ids, seeds first       */
    int64_t* rowptr[GD_MAX_HOPS];     /* hop h: [max_nodes[h-1]+1] row offsets of block h   */
    int32_t* col[GD_MAX_HOPS];        /* hop h: [max_edges[h-1]] local (relabelled) src ids */
    int64_t* eid[GD_MAX_HOPS];        /* hop h: [max_edges[h-1]] CSR edge offsets, or NULL  */
    int64_t* sizes;                   /* [2K+1]: n_0..n_K, e_1..e_K (device-resident)       */
} gd_sample_out;

/* ----------------------------------------------------------------------------
 * Multi-hop neighbour sampling + relabel of one mini-batch (the sampler stage,
 * "each sampler generates a subgraph for a mini-batch from which a list of
 * sampled node IDs is made"; "3-hop random neighborhood sampling").
 *
 *   seeds      host or device int32[num_seeds], distinct, in [0, N) (the
 *              mini-batch's training nodes).  n_id[0:num_seeds] = seeds.  Pinned
 *              host memory is read by the kernel through its mapping (no copy-engine
 *              transfer to queue behind the miss stream's H2D copies); pageable host
 *              memory is copied first.
 *   fanouts    host int32[num_hops]; f in [0, GD_MAX_FANOUT] or -1 (whole row).
 *   rng_seed   64-bit key of the counter-based Philox4x32-10 stream (R1).
 *   batch_id   global mini-batch index; part of the Philox counter, so results
 *              do not depend on the GPU count or call order (R2).
 * Semantics (R3-R5): hop h expands every node of n_id[0:n_{h-1}] (cumulative
 * frontier).  Node v of degree d gets min(f, d) distinct CSR positions (all of
 * them if f < 0 or d <= f), drawn by Floyd's algorithm with draw t =
 * floor(u_t * (j+1) / 2^64), u_t = Philox(ctr=(t, v, h-1, batch_id), key=rng_seed)
 * words (y<<32|x), and listed in ascending position order.  Unseen neighbours
 * get the next local ids in first-occurrence order and are appended to n_id.
 * Block h = (rowptr[h], col[h], eid[h]) has dst = n_id[0:n_{h-1}], src =
 * n_id[0:n_h].  sizes is written on the device; nothing is copied to the host.
 * ------------------------------------------------------------------------- */
gd_status gd_sample(gd_graph* g, const int32_t* seeds, int64_t num_seeds, const int32_t* fanouts,
                    int32_t num_hops, uint64_t rng_seed, uint32_t batch_id, gd_sample_out* out,
                    void* stream);

/* Sampling workspaces.  gd_sample uses the graph's default workspace, so calls on
 * one graph are stream-ordered on one stream.  Several samplers ("a pool of
 * threads as samplers") may run concurrently on different streams, each with its own
 * workspace (relabel hash, scan tile states, seed staging), via gd_sample_ws.  A
 * workspace must not be used by two calls that may overlap in time. */
typedef struct gd_workspace gd_workspace;
gd_status gd_workspace_create(gd_graph* g, gd_workspace** out);
gd_status gd_workspace_destroy(gd_workspace* w);
/* gd_sample with an explicit workspace (w = NULL: the graph's default). */
gd_status gd_sample_ws(gd_graph* g, gd_workspace* w, const int32_t* seeds, int64_t num_seeds,
                       const int32_t* fanouts, int32_t num_hops, uint64_t rng_seed, uint32_t batch_id,
                       gd_sample_out* out, void* stream);

/* ----------------------------------------------------------------------------
 * Feature buffer: `capacity_slots` rows of `row_bytes` in HBM, a
 * mapping table {slot, reference count, valid bit} per node, a reverse
 * mapping array and an LRU standby list of slots with refcount 0
 * (P:109).  The feature table (ascending node id) lives in
 * pinned host memory, the SSD stand-in:
 *
 *   host_feat        host pointer to num_nodes*row_bytes bytes.  If not already
 *                    page-locked it is registered (cudaHostRegisterMapped |
 *                    Portable) and unregistered at destroy.  It must stay alive
 *                    and unmodified until gd_buffer_destroy.
 *   row_bytes        bytes per row, a multiple of 4 (16 for the vector path).
 *   capacity_slots   S.  Must be >= min(N, max_inflight * max_nodes_per_batch):
 *                    the paper's N_e x M_b reservation as a check
 *                    (GD_ERR_CAPACITY), since a caller-driven API cannot wait
 *                    for a releaser (R12).
 *   max_inflight     most extracted-but-unreleased batches at any time (Q).
 *   preload          nonzero: S >= N, node v resident in slot v from the start.
 * Initial state: map = {-1, 0, 0}, reverse = -1, standby = [0, 1, .., S-1] (R10).
 * ------------------------------------------------------------------------- */
gd_status gd_buffer_init(const void* host_feat, int64_t num_nodes, int64_t row_bytes,
                         int64_t capacity_slots, int32_t max_inflight,
                         int64_t max_nodes_per_batch, int preload, int device, gd_buffer** out);
/* As gd_buffer_init, but the host table holds only `table_rows` rows (1 <= table_rows <=
 * num_nodes) and node v's feature row is table row (v mod table_rows): a bounded physical
 * table for workloads whose full table exceeds host memory (the mag240m config: 375 GB
 * logical).  The same bytes cross the host link per miss. */
gd_status gd_buffer_init_mod(const void* host_feat, int64_t table_rows, int64_t num_nodes, int64_t row_bytes,
                             int64_t capacity_slots, int32_t max_inflight, int64_t max_nodes_per_batch,
                             int preload, int device, gd_buffer** out);
gd_status gd_buffer_destroy(gd_buffer* b);

/* ----------------------------------------------------------------------------
 * Extraction of one mini-batch (Alg. 1):
 *   loop 1: hits (valid) take their slot, leaving the standby list if their
 *           refcount was 0; every node's refcount++;
 *   loop 2: misses, in list order, take successive LRU standby slots; a slot's
 *           previous node is invalidated (R9); map / reverse / alias updated;
 *   the missed rows stream from the pinned host table into their slots and into
 *   `out` on the library's side streams (asynchronous extraction),
 *   overlapping the caller's next gd_sample; hit rows are gathered from the slots
 *   into `out` on a side stream too (the trainer's alias indexing, P:96,
 *   materialised).  Only the bookkeeping (loops 1 and 2) runs on `stream`.
 *
 *   node_ids  device int32[n], distinct, in [0, N) (normally gd_sample's n_id).
 *   n_dev     device int64*: n (normally &sizes[K]); n <= n_max.
 *   n_max     host bound on n (grid sizing); must be <= max_nodes_per_batch.
 *   out       device [n_max * row_bytes] (16-byte aligned): out[i] = feat[node_ids[i]].
 *   alias     device int32[n_max] or NULL: slot of node_ids[i] (Alg. 1 ids_r).
 *   stats     device int64[4] or NULL: {hits, misses, misses copied zero-copy,
 *             misses copied through the staged path} of this batch.
 *   done      cudaEvent_t (void*) or NULL: recorded when `out` is complete.
 *             `out` is valid only after `done`; `stream` itself does NOT wait
 *             for the misses or the hit gather.  node_ids, *n_dev and alias
 *             must stay unmodified until `done`.
 * GD_ERR_CAPACITY if this would exceed max_inflight unreleased batches.
 * stats[0..1] are written on `stream` (after loop 1); stats[2..3] are final only at
 * `done` (with peers attached they are written on a side stream after the peer probe; rows
 * served by peers count in neither, see gd_buffer_peer_stats).
 * The call does not synchronise the device; it blocks the calling thread only when
 * 1024 staged chunk jobs (8-16 MB each by default) enqueued by earlier calls are still
 * waiting for their host-gather callbacks (their argument slots are then reused).
 * ------------------------------------------------------------------------- */
gd_status gd_extract(gd_buffer* b, const int32_t* node_ids, const int64_t* n_dev, int64_t n_max,
                     void* out, int32_t* alias, int64_t* stats, void* stream, void* done);

/* ----------------------------------------------------------------------------
 * Miss-stream configuration.  The misses of a batch are split in list order: ranks
 * [0, K0) are copied zero-copy from the pinned table by SM loads; ranks [K0, M) take
 * the paper's two-phase path: phase 1, `host_threads` library-owned
 * CPU threads gather the rows into a pinned staging slot (run from a CUDA host
 * function, so still stream-ordered, no caller sync); phase 2, a kernel pulls the
 * slot contiguously over the host link.  K0 = floor(M * zero_copy_share).
 *   host_threads     0 disables the staged path (all misses zero-copy).
 *   zero_copy_share  in [0, 1]; < 0 = adaptive, from the measured zero-copy rate r_zc
 *                    and host gather rate r_host and the contiguous pull rate r_link of
 *                    the host link (calibrated when this call enables adaptation):
 *                    r_zc / (r_zc + r_host) if r_zc + r_host <= r_link, else
 *                    1 - r_host / r_link; clamped to [0.05, 0.9] ([0.05, 0.15] with
 *                    copy-engine staging: a larger zero-copy share collapses the copy
 *                    engine's rate on some hosts); GD_SHARE_TUNER=1 refines
 *                    it by measurement (gd_buffer_policy_read).
 *   zc_blocks, pull_blocks  grid (1024-thread blocks, about one SM each) of the two
 *                    copy kernels; <= 0 keeps the current value (defaults 16 and 8).
 *                    Few whole-SM blocks keep long-latency host loads off the SMs
 *                    that run sampling / bookkeeping / the hit gather.
 * Default at init: host_threads = min(13, cores - 3) (0 with preload),
 * adaptive share; env GD_HOST_THREADS / GD_ZERO_COPY_SHARE / GD_ZC_BLOCKS /
 * GD_PULL_BLOCKS override.  Further knobs, read here: GD_STAGE_CHUNK_KB (fixed staging chunk;
 * default a sixth of the batch's staged share in [8, 16] MB), GD_STAGE_RING (pinned chunk
 * buffers, default 4), GD_POOL_SPIN (host-gather pool spin before sleeping), GD_GATHER_PF
 * (host prefetch distance in rows), GD_SHARE_TUNER=1 (see gd_buffer_policy_read); at init:
 * GD_GATHER_DYNAMIC / GD_GATHER_PRIORITY / GD_GATHER_TMA (hit-gather variants).  Synchronises
 * the buffer's internal streams; call between batches.
 * ------------------------------------------------------------------------- */
gd_status gd_buffer_config(gd_buffer* b, int host_threads, double zero_copy_share, int zc_blocks,
                           int pull_blocks);

/* The miss-path split policy (gd_buffer_config, adaptive share), for reports: out[0..n) of
 * {zero-copy share, r_host, r_zc, r_link (GB/s), misses-per-batch estimate (the copy-engine
 * staging size), host-rate samples, the model share's upper clamp, newest batch rated,
 * tuner on (0/1), tuner windows measured, tuner frozen (0/1), tuner's best cost (ns per miss)}.
 * The estimates come from the newest completed batch at each gd_extract (events queried, never
 * waited on) and the miss count from the newest batch whose loop 2 ran (an epoch-tagged count
 * the device writes to mapped host memory).  Optionally (env GD_SHARE_TUNER=1, copy-engine
 * staging, adaptive share) a hill-climbing tuner owns the share: it starts at the model's value,
 * measures the extraction period per miss over windows of 6 completed batches, moves the share
 * in steps (0.05, halved after failing on both sides) while that improves, and freezes at the
 * best share in [0, 0.4].  Host-only, no sync; n <= 12. */
gd_status gd_buffer_policy_read(gd_buffer* b, double* out, int32_t n);

/* ----------------------------------------------------------------------------
 * Phase 2 of the staged share ("CUDA async copy" of the staging buffer).
 *   copy_engine = 1 (default; env GD_STAGE_COPY_ENGINE=0 at init selects 0): the
 *     staged share is the FIRST `cap` misses of the batch, cap = (1 - share) x the
 *     misses of a recently completed batch (the copy size must be known when it is
 *     enqueued, and nothing may synchronise the host); after the host gather, stream
 *     H copies cap rows pinned -> HBM staging with cudaMemcpyAsync (DMA, no SM
 *     loads over the link) and a kernel scatters them into slots + out.  The other
 *     misses go zero-copy.  HBM cost: D x max_nodes_per_batch x row_bytes.
 *   copy_engine = 0: ranks [K0, M) are staged and a kernel pulls the pinned slot.
 * Either way the results (out, alias, buffer state) are identical.  Synchronises the
 * internal streams (re-runs gd_buffer_config); call between batches.
 * ------------------------------------------------------------------------- */
gd_status gd_buffer_stage_mode(gd_buffer* b, int copy_engine);

/* ----------------------------------------------------------------------------
 * f2: NVLink peer feature buffers.  P:142: "each subprocess ... may
 * reuse feature data that have been loaded [by] other subprocesses" (the paper shares
 * the host staging buffer; on B200 the peers' HBM buffers are one NVLink/NVSwitch hop
 * away).  With peers attached, every miss of gd_extract first looks its node up in
 * each peer's mapping table and, if the peer slot is published (see below),
 * copies the row over NVLink into the local slot and `out`; only the misses no peer
 * served go to the host paths.  Alg. 1 is unchanged (a peer-served node is still a
 * miss that takes a local LRU slot): out, alias, hits/misses and the buffer state are
 * identical with or without peers.
 * Consistency (seqlock, no locks): a buffer tags slot s with (batch epoch << 32 | node)
 * after every copy into it has finished and clears the tag when the slot is
 * reassigned (before it is refilled); a reader checks the tag, copies, re-reads the
 * tag and falls back to the host when it changed.  Tags never repeat, so a stale copy
 * is always detected.  A buffer maintains its tags only from the moment another buffer can
 * read them (it is attached as someone's peer, or exported): that switch rebuilds every tag
 * from its mapping table (its streams idle, so every valid node's row is in its slot), and
 * until then its extractions skip the tag writes.
 *   gd_buffer_peer_attach     in-process peers (same or other device; P2P access is
 *                             enabled here).  npeers = 0 detaches.  <= 7 peers; they
 *                             must have the same num_nodes, row_bytes and table rows.
 *   gd_buffer_peer_export_ipc writes GD_PEER_BLOB_BYTES describing b (sizes + CUDA IPC
 *                             handles of its map, tags and slots) for other processes.
 *   gd_buffer_peer_attach_ipc attaches npeers blobs (consecutive) from other processes;
 *                             the handles are opened here and closed at destroy.
 *   gd_buffer_peer_stats      synchronises; rows served by peers and misses probed since init.
 * Peers stay alive (not destroyed) while attached.  Synchronise b's streams; call
 * between batches.
 * ------------------------------------------------------------------------- */
#define GD_PEER_BLOB_BYTES 256
gd_status gd_buffer_peer_attach(gd_buffer* b, int npeers, gd_buffer* const* peers);
gd_status gd_buffer_peer_export_ipc(gd_buffer* b, void* blob, int64_t blob_bytes);
gd_status gd_buffer_peer_attach_ipc(gd_buffer* b, int npeers, const void* blobs);
gd_status gd_buffer_peer_stats(gd_buffer* b, int64_t* served, int64_t* probed);

/* ----------------------------------------------------------------------------
 * f4: the train stage on the extracted mini-batch.  GraphSAGE
 * (three layers, hidden 256; mean aggregator with root weight, PyG SAGEConv,
 * P:146) on the blocks of gd_sample, features = the rows gd_extract wrote (fp32).
 * Layer j = 0..L-1 consumes hop h = L - j: a_i = [x_i | mean_{e in row i} x_col[e]],
 * z = a W_j + b_j, relu between layers; loss = mean softmax cross entropy of the n_0
 * seeds.  bf16 tensor-core GEMMs (hand-written tcgen05, csrc/gd_umma.cuh) over the
 * device-resident row counts, fp32 accumulation, fp32 master parameters.
 *   gd_sage_create   dims[0..L] widths (dims[0] = feature dim, multiples of 4 for the
 *                    inputs); init_w[j] host fp32 row-major [2 dims[j] x dims[j+1]] (rows
 *                    0..dims[j]-1 multiply x_i, the rest the neighbour mean), init_b[j]
 *                    [dims[j+1]]; max_nodes[0..L] = gd_sample_bounds of the blocks (buffers
 *                    are sized by them; kernels read the actual counts on the device: no
 *                    host sync).
 *   gd_sage_step     forward + loss + backward for one batch, stream-ordered: rowptr[h-1]
 *                    / col[h-1] the device block arrays of hop h (gd_sample_out), sizes the
 *                    device sizes array, feats device fp32 [n_L x dims[0]], labels device
 *                    int32 [n_0], loss a device float.  Writes the gradients.
 *   gd_sage_grads    device pointer + length of the flat fp32 gradient buffer (layout
 *                    [W_0 b_0 W_1 b_1 ...]) for a data-parallel all-reduce.
 *   gd_sage_apply_sgd  p -= lr * grad_scale * g (grad_scale = 1/world after a SUM
 *                    all-reduce), then refreshes the bf16 copies; stream-ordered.
 *   gd_sage_get      synchronising debug copy of one layer's item (GD_SAGE_*) to host.
 *                    Activation items are valid for the rows of the last step's device
 *                    count; the rows up to the next multiple of 64 are zero, rows past that
 *                    hold earlier steps' data.
 * Environment: GD_SAGE_TIMING=1 records one event pair per phase of every step on the
 * train stream and prints the mean live time per phase at gd_sage_destroy.
 * ------------------------------------------------------------------------- */
typedef struct gd_sage gd_sage;
#define GD_SAGE_W 0     /* fp32 [2 d_in x d_out] */
#define GD_SAGE_B 1     /* fp32 [d_out] */
#define GD_SAGE_DW 2
#define GD_SAGE_DB 3
#define GD_SAGE_A16 4   /* bf16 [n_dst bound x 2 d_in], last forward */
#define GD_SAGE_Z 5     /* fp32 [n_dst bound x d_out], last forward logits z + b (top layer only) */
#define GD_SAGE_H 6     /* bf16 [n_dst bound x d_out], last forward relu(z + b) (hidden layers only) */
gd_status gd_sage_create(int32_t num_layers, const int32_t* dims, const float* const* init_w,
                         const float* const* init_b, const int64_t* max_nodes, int device, gd_sage** out);
gd_status gd_sage_destroy(gd_sage* s);
gd_status gd_sage_step(gd_sage* s, const int64_t* const* rowptr, const int32_t* const* col,
                       const int64_t* sizes, const float* feats, const int32_t* labels, float* loss,
                       void* stream);
gd_status gd_sage_grads(gd_sage* s, float** grads, int64_t* count);
gd_status gd_sage_apply_sgd(gd_sage* s, float lr, float grad_scale, void* stream);
gd_status gd_sage_get(gd_sage* s, int32_t what, int32_t layer, void* host_out, int64_t bytes);

/* Test surface of the train stage's tensor-core GEMM (csrc/gd_umma.cuh; tcgen05.mma with
 * the accumulator in TMEM), all pointers device, bf16 operands, stream-ordered:
 *   mode 0 FWD  C[i, n] = f(sum_k A[i*lda + k] B[k*ldb + n] + bias[n]), f = relu if `relu`
 *   mode 1 DA   C[i, n] = sum_k A[i*lda + k] B[n*ldb + k]
 *   for i < *rows_dev (<= rows_max), k < k_valid (multiple of 8), n < n_store; C is bf16 if
 *   c_bf16 else fp32, row stride ldc; bias nullable; B is valid (and read) for n < n_valid
 *   (multiple of 8), zero beyond.
 *   mode 2 DW   C[m, n] += sum_{i < *rows_dev} A[i*lda + m] B[i*ldb + n] for m < m_valid
 *   (multiple of 8), n < n_store, C fp32, the reduction split over `splits` CTAs per tile
 *   (fp32 red.add into C: the caller zeroes it); rows [*rows_dev, round_up(*rows_dev, 64))
 *   of A and B (below rows_max) must be zero (64-row blocks are reduced whole).
 * Row strides are multiples of 8 elements, base pointers 16-byte aligned (GD_ERR_INVALID). */
gd_status gd_debug_umma_gemm(int32_t mode, const void* A, int64_t lda, const void* B, int64_t ldb,
                             void* C, int64_t ldc, int32_t c_bf16, int32_t relu, const float* bias,
                             const int64_t* rows_dev, int64_t rows_max, int64_t m_valid, int32_t k_valid,
                             int32_t n_valid, int32_t n_store, int32_t splits, void* stream);

/* ----------------------------------------------------------------------------
 * Release stage: for node_ids in list order decrement the refcount; a
 * slot whose count reaches zero is appended at the tail (MRU end) of the standby
 * list.  The node stays valid until its slot is reused (delayed invalidation).
 * Arguments as in gd_extract.  Stream-ordered; no host sync.  It does not wait for the
 * batch's `done`: a slot it frees is refilled only by a later batch's miss copies, which
 * wait for every earlier batch's hit gather.  Issue it after the gd_extract calls it must
 * follow in Alg. 1 order, on `stream` or on a stream ordered after them by events.
 * ------------------------------------------------------------------------- */
gd_status gd_buffer_release(gd_buffer* b, const int32_t* node_ids, const int64_t* n_dev,
                            int64_t n_max, void* stream);

/* Error reporting of the device-side preconditions (no paper passage: the paper's
 * extractor threads check on the host; here the checks run inside the kernels and
 * cannot return a status without a sync, so they set a sticky word, CUDA sticky-error style).
 * Synchronises the handle's device and returns GD_ERR_DEVICE (and the sticky
 * GD_DEV_* bits in *bits, if non-NULL) if a device-side check tripped since the
 * handle was created.  `handle` is a gd_graph* or a gd_buffer*. */
gd_status gd_check_device_status(void* handle, uint32_t* bits);

/* ----------------------------------------------------------------------------
 * Debug / test surface (synchronising; not for the hot path).
 * ------------------------------------------------------------------------- */
/* Copy the buffer state to host arrays (any may be NULL): map_slot/map_rc/
 * map_valid [N], reverse [S], standby [S] in LRU order (head first); the number
 * of standby slots is stored in *standby_len. */
gd_status gd_buffer_snapshot(gd_buffer* b, int32_t* map_slot, int32_t* map_rc, uint8_t* map_valid,
                             int32_t* reverse, int32_t* standby, int64_t* standby_len);
/* Install an explicit state from host arrays (used for the Fig. 6 example,
 * P:131); slot contents of valid nodes are loaded from the host table. */
gd_status gd_buffer_set_state(gd_buffer* b, const int32_t* map_slot, const int32_t* map_rc,
                              const uint8_t* map_valid, const int32_t* reverse,
                              const int32_t* standby, int64_t standby_len);
/* The internal side stream (cudaStream_t as void*) misses are copied on. */
void* gd_buffer_side_stream(gd_buffer* b);

/* Per-kernel timing with CUDA events recorded on the streams the kernels run on
 * (the caller's stream for bookkeeping / gather / sampling, the side stream for
 * misses).  enable != 0 starts collecting (and clears what was collected);
 * enable == 0 stops.  *_timing_read synchronises and sums the collected
 * durations in milliseconds.  Used by bench.py for the roofline fractions. */
gd_status gd_buffer_timing(gd_buffer* b, int enable);
/* ms[7] = {bookkeeping (lookup + pop/assign), hit gather, zero-copy miss copy,
 *          staged miss pull (SM pull mode) or scatter (copy-engine mode), host gather
 *          (phase 1, summed), current zero-copy share, copy-engine H2D of the staged
 *          share (copy-engine mode; 0 otherwise)}. */
gd_status gd_buffer_timing_read(gd_buffer* b, double* ms, int64_t* batches);
/* Sampler variant of the hops with 1 <= f <= 32 (test / A-B surface, readings R4-R5
 * in DESIGN.md): padded = 1 (default; GD_SAMPLE_PAD=0 in the environment at gd_graph_create turns
 * it off) draws each frontier node's neighbours into a padded [n_{h-1} x f] layout with no scan
 * (k_sample_pad), then one pass with one decoupled look-back over (edges, new nodes) writes rowptr,
 * the compacted col / eid and the new nodes (k_relabel_pad); padded = 0 scans the counts inside
 * the sampling kernel (k_sample_hop + k_relabel_hop).  Outputs are identical (bit for bit) either
 * way; hops with f = -1 or f > 32 always take the second form.  Host-only, not stream-ordered:
 * call it between gd_sample calls.  GD_ERR_INVALID on a bad handle. */
gd_status gd_graph_sampler(gd_graph* g, int padded);
gd_status gd_graph_timing(gd_graph* g, int enable);
gd_status gd_graph_timing_read(gd_graph* g, double* sample_ms, int64_t* calls);

#ifdef __cplusplus
}
#endif
#endif /* GD_H_ */
