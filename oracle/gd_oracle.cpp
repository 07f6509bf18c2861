/*
 * gd_oracle.cpp — the CPU ORACLE for the GNNDrive sample + extract hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Nothing on the product path may link, load or call
 * this file.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * `--impl reference` leg use it.  It shares no code, header, table or constant
 * generator with the CUDA library under paper_conf_icpp_jiangj024_b200/csrc/.
 *
 * It is deliberately plain and slow: one sequential pass per step, in the order
 * the paper (and DESIGN.md's readings) state, with std::unordered_map for the
 * relabel map and std::list for the LRU standby list.  No blocking, no fusion,
 * no reordering.
 *
 * Citations: "P:NNN" = line NNN of the paper text (reference PAPER.md,
 * Jiang, Jia, Wang, "Reducing Memory Contention and I/O Congestion for
 * Disk-based GNN Training", ICPP'24).  "C<k>" = reading k of SURVEY.md §8(c),
 * restated in DESIGN.md §3.
 *
 * Pins (tests/test_oracle_*.py, -m "not gpu"):
 *   philox4x32_10     -> Random123 known-answer vectors + curand_Philox4x32_10
 *   randint           -> Python big-int (u*(j+1))>>64
 *   floyd             -> exhaustive enumeration of draw sequences (uniform f-subsets)
 *   sample / relabel  -> invariants, textbook BFS special case, brute force K-hop ball
 *   extract / release -> Fig. 6 worked example, batch-LRU model at Q=1,
 *                        closed-form compulsory misses, out == feat[ids] bytewise
 * No function here is "parity unpinned".
 */
#include <cstdint>
#include <cstring>
#include <cstdio>
#include <list>
#include <unordered_map>
#include <vector>
#include <algorithm>

extern "C" {

/* ------------------------------------------------------------------------- */
/* C1: Philox4x32-10 (Salmon et al., SC'11; Random123).  The paper does not  */
/* name an RNG (P:173 says only "random neighborhood sampling")   */
/* reading R1 fixes this counter-based generator.                            */
/* ------------------------------------------------------------------------- */
static void philox_round(uint32_t c[4], const uint32_t k[2]) {
    const uint64_t p0 = (uint64_t)0xD2511F53u * (uint64_t)c[0];
    const uint64_t p1 = (uint64_t)0xCD9E8D57u * (uint64_t)c[2];
    const uint32_t hi0 = (uint32_t)(p0 >> 32), lo0 = (uint32_t)p0;
    const uint32_t hi1 = (uint32_t)(p1 >> 32), lo1 = (uint32_t)p1;
    const uint32_t n0 = hi1 ^ c[1] ^ k[0];
    const uint32_t n1 = lo1;
    const uint32_t n2 = hi0 ^ c[3] ^ k[1];
    const uint32_t n3 = lo0;
    c[0] = n0; c[1] = n1; c[2] = n2; c[3] = n3;
}

void oracle_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]) {
    uint32_t c[4] = {ctr[0], ctr[1], ctr[2], ctr[3]};
    uint32_t k[2] = {key[0], key[1]};
    for (int round = 0; round < 10; ++round) {
        if (round > 0) { k[0] += 0x9E3779B9u; k[1] += 0xBB67AE85u; }
        philox_round(c, k);
    }
    out[0] = c[0]; out[1] = c[1]; out[2] = c[2]; out[3] = c[3];
}

/* Batch form of the above over n records of (ctr[4], key[2]) -> out[4] (test helper). */
void oracle_philox4x32_10_many(int64_t n, const uint32_t* ctr_key, uint32_t* out) {
    for (int64_t i = 0; i < n; ++i) oracle_philox4x32_10(ctr_key + 6 * i, ctr_key + 6 * i + 4, out + 4 * i);
}

/* C2: uniform integer on [0, j] from a 64-bit word u: floor(u * (j+1) / 2^64). */
uint64_t oracle_randint(uint64_t u, uint64_t j) {
    unsigned __int128 prod = (unsigned __int128)u * (unsigned __int128)(j + 1);
    return (uint64_t)(prod >> 64);
}

/* C2: draw number t for frontier node v at 0-based hop index h of global
 * mini-batch b:  (x, y, ., .) = Philox(ctr = (t, v, h, b), key = (lo, hi of seed)),
 * u = y << 32 | x. */
uint64_t oracle_draw_word(uint32_t t, uint32_t v, uint32_t h, uint32_t b, uint64_t rng_seed) {
    uint32_t ctr[4] = {t, v, h, b};
    uint32_t key[2] = {(uint32_t)rng_seed, (uint32_t)(rng_seed >> 32)};
    uint32_t r[4];
    oracle_philox4x32_10(ctr, key, r);
    return ((uint64_t)r[1] << 32) | (uint64_t)r[0];
}

/* C4: Floyd's subset algorithm (Bentley & Floyd, CACM 1987) given the draws
 * r[t] in [0, d-f+t].  S = {}; for t in 0..f-1: j = d-f+t; if r[t] in S add j
 * else add r[t].  Writes the f positions sorted ascending into pos. */
void oracle_floyd(int64_t d, int32_t f, const uint64_t* r, int64_t* pos) {
    std::vector<int64_t> S;
    for (int32_t t = 0; t < f; ++t) {
        const int64_t j = d - f + t;
        const int64_t rt = (int64_t)r[t];
        bool present = false;
        for (int64_t s : S) if (s == rt) { present = true; break; }
        S.push_back(present ? j : rt);
    }
    std::sort(S.begin(), S.end());
    for (int32_t t = 0; t < f; ++t) pos[t] = S[t];
}

/* C4: the CSR positions sampled for node v (degree d) at hop index h, batch b.
 * fanout f < 0 or d <= f: all positions 0..d-1 (the row verbatim, C11).
 * Otherwise Floyd with draws r_t = randint(draw_word(t, v, h, b), d-f+t).
 * Returns |P| = min(f, d) (or d when f < 0). */
int64_t oracle_sample_positions(int64_t v, int64_t d, int32_t f, uint32_t h, uint32_t b,
                                uint64_t rng_seed, int64_t* pos) {
    if (f < 0 || d <= f) {
        for (int64_t p = 0; p < d; ++p) pos[p] = p;
        return d;
    }
    std::vector<uint64_t> r(f);
    for (int32_t t = 0; t < f; ++t) {
        const uint64_t j = (uint64_t)(d - f + t);
        r[t] = oracle_randint(oracle_draw_word((uint32_t)t, (uint32_t)v, h, b, rng_seed), j);
    }
    oracle_floyd(d, f, r.data(), pos);
    return f;
}

/* ------------------------------------------------------------------------- */
/* Multi-hop neighbour sampling with relabel ("each sampler generates a */
/* subgraph for a mini-batch from which a list of sampled node IDs is made"; */
/* P:173 "3-hop random neighborhood sampling"; readings C3, C5, C9-C11).     */
/*                                                                           */
/* n_id starts as the seeds (local id = position).  Hop h = 1..K expands    */
/* every node of n_id[0:n_{h-1}] (cumulative frontier, C3) with fanout       */
/* fanouts[h-1]; for frontier index i in order and each sampled position p   */
/* in ascending order, neighbour u = indices[indptr[v]+p]; an unseen u gets  */
/* the next local id and is appended to n_id (first occurrence, C5); col     */
/* gets u's local id, eid gets the CSR offset indptr[v]+p.                   */
/* sizes = [n_0..n_K, e_1..e_K].  Returns 0, or -1 on a precondition         */
/* violation (duplicate or out-of-range seed).                              */
/* ------------------------------------------------------------------------- */
int oracle_sample(const int64_t* indptr, const int32_t* indices, int64_t num_nodes,
                  const int32_t* seeds, int64_t num_seeds,
                  const int32_t* fanouts, int32_t num_hops,
                  uint64_t rng_seed, uint32_t batch_id,
                  int32_t* n_id, int64_t** rowptr, int32_t** col, int64_t** eid,
                  int64_t* sizes) {
    std::unordered_map<int32_t, int32_t> local;   /* global id -> local id */
    std::vector<int32_t> nid;
    for (int64_t i = 0; i < num_seeds; ++i) {
        const int32_t s = seeds[i];
        if (s < 0 || s >= num_nodes) return -1;
        if (local.count(s)) return -1;
        local[s] = (int32_t)nid.size();
        nid.push_back(s);
    }
    sizes[0] = (int64_t)nid.size();
    std::vector<int64_t> pos;
    for (int32_t hop = 1; hop <= num_hops; ++hop) {
        const int32_t f = fanouts[hop - 1];
        const int64_t n_prev = (int64_t)nid.size();
        int64_t e = 0;
        rowptr[hop - 1][0] = 0;
        for (int64_t i = 0; i < n_prev; ++i) {
            const int32_t v = nid[i];
            const int64_t start = indptr[v];
            const int64_t d = indptr[v + 1] - start;
            pos.resize(d > 0 ? d : 1);
            const int64_t cnt = oracle_sample_positions(v, d, f, (uint32_t)(hop - 1), batch_id,
                                                        rng_seed, pos.data());
            for (int64_t k = 0; k < cnt; ++k) {
                const int32_t u = indices[start + pos[k]];
                auto it = local.find(u);
                int32_t lu;
                if (it == local.end()) {
                    lu = (int32_t)nid.size();
                    local[u] = lu;
                    nid.push_back(u);
                } else {
                    lu = it->second;
                }
                col[hop - 1][e] = lu;
                if (eid && eid[hop - 1]) eid[hop - 1][e] = start + pos[k];
                ++e;
            }
            rowptr[hop - 1][i + 1] = e;
        }
        sizes[hop] = (int64_t)nid.size();
        sizes[num_hops + hop] = e;
    }
    std::memcpy(n_id, nid.data(), nid.size() * sizeof(int32_t));
    return 0;
}

/* ------------------------------------------------------------------------- */
/* Feature buffer management and extraction: Algorithm 1 with    */
/* the mapping table entry {slot index, reference count, valid bit}, */
/* the reverse mapping array, the LRU standby list (P:109,    */
/* P:126) and the release stage.  Sequential: the wait list of       */
/* Alg. 1 line 5/16/38 stays empty because one extraction completes before   */
/* the next starts (reading C12).                                            */
/* ------------------------------------------------------------------------- */
struct MapEntry { int32_t slot; int32_t rc; uint8_t valid; };

struct OracleBuffer {
    const uint8_t* feat;      /* host table [P x R]; node v's row is row v mod P (P = N normally) */
    int64_t N, R, S, P;
    std::vector<MapEntry> map;             /* mapping table */
    std::vector<int32_t> reverse;          /* reverse mapping array */
    std::list<int32_t> standby;            /* LRU order: head = least recently used */
    std::vector<std::list<int32_t>::iterator> where;   /* slot -> list node (the "hash table") */
    std::vector<uint8_t> in_standby;
    std::vector<uint8_t> slots;            /* the feature buffer, S x R bytes */
    int keep_rows;                         /* 0: bookkeeping only, no slot contents (see below) */
    int64_t hits, misses;                  /* cumulative */
};

static void standby_push_back(OracleBuffer* B, int32_t s) {
    B->standby.push_back(s);
    B->where[s] = std::prev(B->standby.end());
    B->in_standby[s] = 1;
}

static void standby_remove(OracleBuffer* B, int32_t s) {   /* Alg. 1 line 11 */
    B->standby.erase(B->where[s]);
    B->in_standby[s] = 0;
}

/* Initial state (C6, C14): every map entry {-1, 0, 0}, reverse = -1, standby =
 * [0, 1, ..., S-1] (ascending; "slot 2 is the first available free slot").
 * preload (requires S >= N): node v resident in slot v, valid, rc 0. */
/* Feature row of node v: the table holds P rows, node v's features are row (v mod P)
 * (P = N is the paper's layout; P < N is the bounded table of the mag240m config). */
static const uint8_t* feat_row(const OracleBuffer* B, int64_t v) { return B->feat + (size_t)(v % B->P) * B->R; }

/* keep_rows = 0 builds the same buffer without the S x R slot contents: Alg. 1's
 * bookkeeping (map, reverse, standby list, alias, hits / misses) is unchanged, lines 30-36's
 * row copy is skipped and extract refuses `out` (-2).  Storage only, no arithmetic: it lets
 * full-size replays (37.5 GB of slots at mag240m, one replay per GPU) fit in host memory; the
 * rows themselves are checked by the closed form out[i] = feat[ids[i] mod P] (P5). */
void* oracle_buffer_create2(const uint8_t* host_feat, int64_t num_nodes, int64_t row_bytes,
                            int64_t capacity_slots, int preload, int64_t table_rows, int keep_rows) {
    if (preload && capacity_slots < num_nodes) return nullptr;
    if (table_rows < 1 || table_rows > num_nodes) return nullptr;
    OracleBuffer* B = new OracleBuffer();
    B->feat = host_feat; B->N = num_nodes; B->R = row_bytes; B->S = capacity_slots; B->P = table_rows;
    B->map.assign(num_nodes, MapEntry{-1, 0, 0});
    B->reverse.assign(capacity_slots, -1);
    B->where.resize(capacity_slots);
    B->in_standby.assign(capacity_slots, 0);
    B->keep_rows = keep_rows != 0;
    if (B->keep_rows) B->slots.assign((size_t)capacity_slots * (size_t)row_bytes, 0);
    B->hits = B->misses = 0;
    for (int64_t s = 0; s < capacity_slots; ++s) standby_push_back(B, (int32_t)s);
    if (preload) {
        for (int64_t v = 0; v < num_nodes; ++v) {
            B->map[v] = MapEntry{(int32_t)v, 0, 1};
            B->reverse[v] = (int32_t)v;
            if (B->keep_rows) std::memcpy(&B->slots[(size_t)v * row_bytes], feat_row(B, v), row_bytes);
        }
    }
    return B;
}

void* oracle_buffer_create(const uint8_t* host_feat, int64_t num_nodes, int64_t row_bytes,
                           int64_t capacity_slots, int preload, int64_t table_rows) {
    return oracle_buffer_create2(host_feat, num_nodes, row_bytes, capacity_slots, preload, table_rows, 1);
}

void oracle_buffer_destroy(void* h) { delete (OracleBuffer*)h; }

/* Algorithm 1 for one mini-batch ids[0:n] (distinct node ids).
 * alias[i] = slot of ids[i]; out[i] = slots[alias[i]] (the trainer's alias
 * indexing, materialised); stats = {hits, misses} of this batch.
 * Returns 0, or -1 if the standby list runs dry (P:122 would wait for the
 * releaser; the API instead rejects the configuration, reading C16). */
int oracle_extract(void* h, const int32_t* ids, int64_t n, uint8_t* out, int32_t* alias,
                   int64_t* stats) {
    OracleBuffer* B = (OracleBuffer*)h;
    if (out && !B->keep_rows) return -2;
    std::vector<int32_t> ids_r(n, -1);                       /* lines 3-4 */
    int64_t hits = 0, misses = 0;
    for (int64_t i = 0; i < n; ++i) {                         /* lines 6-20 */
        const int32_t id = ids[i];
        MapEntry& m = B->map[id];
        if (m.valid == 1) {                                   /* line 8 */
            if (m.rc == 0) standby_remove(B, m.slot);         /* lines 10-11 */
            ids_r[i] = m.slot;                                /* line 13 */
            ++hits;
        } else if (m.rc > 0) {                                /* line 14: being loaded */
            ids_r[i] = m.slot;                                /* lines 16-17 (wait list) */
            ++hits;
        }
        m.rc++;                                               /* line 19 */
    }
    for (int64_t i = 0; i < n; ++i) {                         /* lines 21-31 */
        const int32_t id = ids[i];
        if (ids_r[i] >= 0) continue;                          /* lines 23-24 */
        if (B->standby.empty()) return -1;
        const int32_t index = B->standby.front();             /* line 26: LRU standby slot */
        standby_remove(B, index);
        const int32_t old = B->reverse[index];
        if (old >= 0) {                                       /* P:122 invalidate previous node */
            B->map[old].valid = 0;
            B->map[old].slot = -1;                            /* reading C13 ("absent") */
        }
        B->map[id].slot = index;                              /* line 27 */
        B->reverse[index] = id;                               /* line 28 */
        ids_r[i] = index;                                     /* line 29 */
        /* lines 30-36: load from the table (the SSD stand-in) into the slot */
        if (B->keep_rows) std::memcpy(&B->slots[(size_t)index * B->R], feat_row(B, id), B->R);
        B->map[id].valid = 1;                                 /* line 37 */
        ++misses;
    }
    for (int64_t i = 0; i < n; ++i) {
        if (alias) alias[i] = ids_r[i];
        if (out) std::memcpy(out + (size_t)i * B->R, &B->slots[(size_t)ids_r[i] * B->R], B->R);
    }
    B->hits += hits; B->misses += misses;
    if (stats) { stats[0] = hits; stats[1] = misses; }
    return 0;                                                 /* line 39 */
}

/* Release stage: for each node in list order decrement its reference
 * count; when it reaches zero add its slot at the tail of the standby list.
 * Invalidation is deferred until the slot is reused.  Returns -1 on a
 * reference-count underflow. */
int oracle_release(void* h, const int32_t* ids, int64_t n) {
    OracleBuffer* B = (OracleBuffer*)h;
    for (int64_t i = 0; i < n; ++i) {
        MapEntry& m = B->map[ids[i]];
        if (m.rc <= 0) return -1;
        m.rc--;
        if (m.rc == 0) standby_push_back(B, m.slot);
    }
    return 0;
}

/* The CPU variant's data path (every feature row host-resident, no device buffer):
 * out[i] = feat[ids[i] mod P], row by row in list order (the closed form of C6's out). */
void oracle_gather_rows(const uint8_t* feat, int64_t P, int64_t R, const int32_t* ids, int64_t n, uint8_t* out) {
    for (int64_t i = 0; i < n; ++i)
        std::memcpy(out + (size_t)i * R, feat + (size_t)((int64_t)ids[i] % P) * R, R);
}

/* Debug snapshot of the whole state (C8).  Any pointer may be null. */
int64_t oracle_buffer_state(void* h, int32_t* map_slot, int32_t* map_rc, uint8_t* map_valid,
                            int32_t* reverse, int32_t* standby) {
    OracleBuffer* B = (OracleBuffer*)h;
    for (int64_t v = 0; v < B->N; ++v) {
        if (map_slot) map_slot[v] = B->map[v].slot;
        if (map_rc) map_rc[v] = B->map[v].rc;
        if (map_valid) map_valid[v] = B->map[v].valid;
    }
    if (reverse) for (int64_t s = 0; s < B->S; ++s) reverse[s] = B->reverse[s];
    int64_t k = 0;
    for (int32_t s : B->standby) { if (standby) standby[k] = s; ++k; }
    return k;
}

/* Install an explicit state (used to reconstruct the Fig. 6 example).
 * Slot contents are loaded from the table for every valid mapped node. */
int oracle_buffer_set_state(void* h, const int32_t* map_slot, const int32_t* map_rc,
                            const uint8_t* map_valid, const int32_t* reverse,
                            const int32_t* standby, int64_t standby_len) {
    OracleBuffer* B = (OracleBuffer*)h;
    for (int64_t v = 0; v < B->N; ++v) B->map[v] = MapEntry{map_slot[v], map_rc[v], map_valid[v]};
    for (int64_t s = 0; s < B->S; ++s) B->reverse[s] = reverse[s];
    B->standby.clear();
    std::fill(B->in_standby.begin(), B->in_standby.end(), 0);
    for (int64_t k = 0; k < standby_len; ++k) standby_push_back(B, standby[k]);
    for (int64_t v = 0; B->keep_rows && v < B->N; ++v)
        if (B->map[v].valid && B->map[v].slot >= 0)
            std::memcpy(&B->slots[(size_t)B->map[v].slot * B->R], feat_row(B, v), B->R);
    return 0;
}

}  /* extern "C" */
