// gd_umma.cuh — hand-written sm_100a tensor-core GEMM (tcgen05.mma, accumulator in TMEM) for
// the f4 train stage.  The three GEMMs of a GraphSAGE layer are
//   FWD  Z[i, n]  = sum_k A16[i, k] W16[k, n] (+ b[n]; H = relu(Z))    i < n_dst (device count)
//   DA   dA[i, n] = sum_k dZ16[i, k] W16[n, k]                          i < n_dst
//   DW   dW[m, n] += sum_i A16[i, m] dZ16[i, n]                         i < n_dst, split over i
// all with bf16 operands and fp32 accumulation.  The row count lives in device memory (it is
// the sampled block size), so tiles past it exit before touching memory: unlike a library
// GEMM run at the host-side bound, no padded rows are read, multiplied or written.
//
// Tile: UMMA M = 128 rows (one TMEM lane per output row), N = BN <= 256 columns (TMEM columns),
// K = 64 per pipeline stage (4 MMAs of K = 16).  CTAs are persistent over the tiles.  The 128
// threads of a CTA stage operands with cp.async (16-byte chunks, zero-filled past the valid
// range) into the no-swizzle canonical UMMA layouts, 4 stages deep and across tile
// boundaries; thread 0 issues the MMAs and tcgen05.commit's them to the stage's mbarrier,
// which releases the stage for the next load.  The epilogue reads the
// accumulator with tcgen05.ld (warp w owns TMEM lanes 32w..32w+31 = rows, 32 columns per
// load), adds the bias and applies relu (FWD), transposes the 32 x 32 block through shared
// memory (the drained stage buffers) and writes whole rows per instruction: fp32 or bf16
// stores, or fp32 red.add of the split-K partial (DW).
//
// Shared-memory image of one operand tile (R rows of the M/N dimension x 64 of K), both majors:
//   K-major  (row-major global, K contiguous):  byte(r, k8) = (r / 8) * 1024 + k8 * 128 + (r % 8) * 16
//   MN-major (M/N contiguous):                 byte(r8, k) = r8 * 1024 + (k / 8) * 128 + (k % 8) * 16
// i.e. 8 x 16-byte core matrices, K-adjacent ones 128 B apart (LBO), M/N-adjacent 8-groups
// 1024 B apart (SBO); one MMA (K = 16) covers two K groups, so the k-th MMA of a stage starts
// 256 B further.
#pragma once
#include <cuda_bf16.h>
#include <stdint.h>

#include <algorithm>

namespace gd {
namespace umma {

constexpr int BM = 128;
constexpr int BK = 64;
constexpr int STAGES = 4;
constexpr int A_STAGE = BM * BK * 2;   // 16 KB

enum Mode { FWD = 0, DA = 1, DW = 2 };

struct Args {
    const __nv_bfloat16* A; int64_t lda;
    const __nv_bfloat16* B; int64_t ldb;
    void* C; int64_t ldc;        // fp32, or bf16 when c_bf16 (FWD / DA); fp32 for DW
    int c_bf16;
    int relu;                    // FWD: C = relu(acc + bias)
    const float* bias;           // FWD: [n_store] (nullable)
    const int64_t* rows_dev;     // device row count: M (FWD, DA) or the reduction length (DW)
    int64_t m_valid;             // DW: output rows (A's contiguous width); FWD/DA: unused
    int k_valid;                 // FWD/DA: reduction length (multiple of 8)
    int n_valid;                 // B's valid extent along N (multiple of 8; zero-filled past it)
    int n_store;                 // output columns written
    int bn;                      // N tile (multiple of 16, <= 256)
};

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void cp_async16(uint32_t dst, const void* src, bool valid) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(dst), "l"(src), "r"(valid ? 16 : 0) : "memory");
}

__device__ __forceinline__ void mbar_wait(uint32_t addr, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra WAIT_%=;\n}\n" ::"r"(addr),
        "r"(parity)
        : "memory");
}

__device__ __forceinline__ uint64_t smem_desc(uint32_t addr) {
    uint64_t d = 0;
    d |= (uint64_t)((addr >> 4) & 0x3FFF);            // start address
    d |= (uint64_t)(128 >> 4) << 16;                   // LBO: K-adjacent core matrices
    d |= (uint64_t)(1024 >> 4) << 32;                  // SBO: M/N-adjacent 8-row groups
    d |= (uint64_t)1 << 46;                            // descriptor version (sm_100)
    return d;                                          // base offset 0, layout SWIZZLE_NONE
}

template <bool A_MN, bool B_MN>
__host__ __device__ constexpr uint32_t instr_desc(int bn) {
    return (1u << 4)                      // D format f32
           | (1u << 7) | (1u << 10)       // A, B bf16
           | ((A_MN ? 1u : 0u) << 15) | ((B_MN ? 1u : 0u) << 16)
           | ((uint32_t)(bn >> 3) << 17)  // N / 8
           | ((uint32_t)(BM >> 4) << 24); // M / 16
}

// Stage one operand tile (R rows along M/N starting at r0, BK along K starting at k0).  Chunks
// are assigned so that every 8 consecutive lanes write 8 distinct 16-byte bank slots (the low
// 7 address bits are (r % 8) * 16, resp. (k % 8) * 16: conflict-free cp.async writes) while
// each warp still reads whole 32-byte sectors of global memory:
//   K-major:  idx = (r / 8) * 64 + k8 * 8 + r % 8            (8 rows x 4 chunks of 16 B per warp)
//   MN-major: idx = (r8 / 2) * 128 + (k / 8) * 16 + (r8 % 2) * 8 + k % 8
//                                                          (8 K-rows x 2 adjacent chunks per 16 lanes)
template <bool MN_MAJOR>
__device__ __forceinline__ void load_tile(uint32_t s, const __nv_bfloat16* __restrict__ g, int64_t ld, int R, int64_t r0,
                                          int64_t r_valid, int64_t k0, int64_t k_end) {
    const int total = R * 8;   // 16-byte chunks in an R x 64 bf16 tile
    for (int idx = threadIdx.x; idx < total; idx += blockDim.x) {
        int r, k;              // K-major: row r, chunk k (of 8 elements); MN-major: 8-group r, K-row k
        uint32_t off;
        if (!MN_MAJOR) {
            r = ((idx >> 6) << 3) + (idx & 7);
            k = (idx >> 3) & 7;
            off = (uint32_t)idx * 16;   // (r / 8) * 1024 + k * 128 + (r % 8) * 16
        } else {
            r = ((idx >> 7) << 1) | ((idx >> 3) & 1);
            k = (((idx >> 4) & 7) << 3) + (idx & 7);
            off = (uint32_t)(r * 1024 + (k >> 3) * 128 + (k & 7) * 16);
        }
        const int64_t gr = r0 + (MN_MAJOR ? r * 8 : r), gk = k0 + (MN_MAJOR ? k : k * 8);
        const bool v = gr < r_valid && gk < k_end;
        cp_async16(s + off, v ? (MN_MAJOR ? g + gk * ld + gr : g + gr * ld + gk) : g, v);
    }
}

// Epilogue of one unit: warp w reads TMEM lanes 32w.. (= tile rows rbase..rbase+31), 32
// columns per load (bn is a multiple of 16 and the allocation a power of two >= 32, so a load
// past bn stays inside it; those columns are not stored), transposes the 32 x 32 block
// through its 4 KB of shared memory and writes (or red.adds) one 32-column row segment per
// instruction.
template <int MODE>
__device__ __forceinline__ void epilogue(const Args& a, uint32_t tmem, float* st, int64_t rbase, int64_t n0, int64_t m_valid,
                                         int bn, int warp, int lane) {
    for (int c0 = 0; c0 < bn; c0 += 32) {
        uint32_t r[32];
        const uint32_t taddr = tmem + ((uint32_t)(warp * 32) << 16) + (uint32_t)c0;
        asm volatile(
            "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
            "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];\n"
            : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
              "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
              "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
              "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
            : "r"(taddr));
        asm volatile("tcgen05.wait::ld.sync.aligned;\n" ::: "memory");
#pragma unroll
        for (int j = 0; j < 32; ++j) st[lane * 33 + j] = __uint_as_float(r[j]);
        __syncwarp();
        const int64_t cg = n0 + c0 + lane;              // this lane's output column
        const bool col_ok = c0 + lane < bn && cg < a.n_store;
        const float b = (MODE == FWD && a.bias && col_ok) ? __ldg(a.bias + cg) : 0.f;
        for (int rr = 0; rr < 32; ++rr) {
            const int64_t row = rbase + rr;
            if (row >= m_valid) break;
            float v = st[rr * 33 + lane];
            if (!col_ok) continue;
            if (MODE == DW) {
                atomicAdd((float*)a.C + row * a.ldc + cg, v);
            } else {
                v += b;
                if (MODE == FWD && a.relu) v = fmaxf(v, 0.f);
                if (a.c_bf16) ((__nv_bfloat16*)a.C)[row * a.ldc + cg] = __float2bfloat16_rn(v);
                else ((float*)a.C)[row * a.ldc + cg] = v;
            }
        }
        __syncwarp();
    }
}

// One unit of work: an output tile (m0, n0) and its reduction range [k_begin, k_end).
struct Unit {
    int64_t u, m0, n0, k_begin, k_end;
    int nkb, kb;
};

// Units: FWD / DA: (m-tile, n-tile) over the device row count, full K.  DW: (m-tile, n-tile,
// split) with split z taking a BK-aligned slice of the device row count (empty slices skipped).
template <int MODE>
__device__ __forceinline__ bool unit_at(Unit& c, int64_t u, const Args& a, int64_t rows, int nt, int splits) {
    for (;; u += gridDim.x) {
        if (MODE == DW) {
            const int64_t mt = (a.m_valid + BM - 1) / BM;
            if (u >= mt * nt * splits) return false;
            const int64_t z = u % splits, rest = u / splits;
            c.n0 = (rest % nt) * a.bn;
            c.m0 = (rest / nt) * BM;
            int64_t per = (rows + splits - 1) / splits;
            per = (per + BK - 1) / BK * BK;
            c.k_begin = z * per;
            c.k_end = c.k_begin + per < rows ? c.k_begin + per : rows;
            if (c.k_begin >= c.k_end) continue;
        } else {
            if (u >= (rows + BM - 1) / BM * nt) return false;
            c.m0 = (u / nt) * BM;
            c.n0 = (u % nt) * a.bn;
            c.k_begin = 0;
            c.k_end = a.k_valid;
        }
        c.u = u;
        c.kb = 0;
        c.nkb = (int)((c.k_end - c.k_begin + BK - 1) / BK);
        return true;
    }
}

// Persistent CTAs (grid <= resident CTAs); the load cursor runs STAGES-1 k-blocks ahead of the
// MMA cursor across unit boundaries, so the next unit's operands stream in during a unit's
// epilogue.
template <int MODE>
__global__ void __launch_bounds__(128) k_umma_gemm(Args a, int nt, int splits) {
    constexpr bool A_MN = MODE == DW;
    constexpr bool B_MN = MODE != DA;
    extern __shared__ __align__(1024) uint8_t smem[];
    const int bn = a.bn;
    const int b_stage = bn * BK * 2;
    uint8_t* sA = smem;
    uint8_t* sB = smem + STAGES * A_STAGE;
    float* stage_out = (float*)(sB + STAGES * b_stage);          // 4 warps x 32 x 33 fp32
    uint64_t* mbar = (uint64_t*)(stage_out + 4 * 32 * 33);
    uint32_t* tmem_slot = (uint32_t*)(mbar + STAGES);

    const int64_t rows = *a.rows_dev;   // device-resident size
    Unit cm, ld;
    if (!unit_at<MODE>(cm, blockIdx.x, a, rows, nt, splits)) return;
    ld = cm;
    const int64_t m_valid = MODE == DW ? a.m_valid : rows;
    uint32_t ncols = 32;
    while ((int)ncols < bn) ncols <<= 1;

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;\n" ::"r"(smem_u32(tmem_slot)),
                     "r"(ncols));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;\n");
    }
    if (threadIdx.x == 0) {
        for (int s = 0; s < STAGES; ++s)
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;\n" ::"r"(smem_u32(mbar + s)));
        asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;\n" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;\n" ::: "memory");
    const uint32_t tmem = *tmem_slot;
    const uint32_t idesc = instr_desc<A_MN, B_MN>(bn);

    bool ld_ok = true;
    auto issue_load = [&](uint32_t it) {
        const int s = (int)(it % STAGES);
        const int64_t k0 = ld.k_begin + (int64_t)ld.kb * BK;
        load_tile<A_MN>(smem_u32(sA + s * A_STAGE), a.A, a.lda, BM, ld.m0, m_valid, k0, ld.k_end);
        load_tile<B_MN>(smem_u32(sB + s * b_stage), a.B, a.ldb, bn, ld.n0, a.n_valid, k0, ld.k_end);
        if (++ld.kb == ld.nkb) ld_ok = unit_at<MODE>(ld, ld.u + gridDim.x, a, rows, nt, splits);
    };
    uint32_t it_ld = 0, it_cm = 0;
    for (int s = 0; s < STAGES - 1; ++s) {
        if (ld_ok) issue_load(it_ld++);
        asm volatile("cp.async.commit_group;\n" ::: "memory");
    }
    for (;;) {
        if (ld_ok) {
            if (it_ld >= STAGES)   // the stage's previous occupant (item it_ld - STAGES) was multiplied
                mbar_wait(smem_u32(mbar + it_ld % STAGES), ((it_ld / STAGES) - 1) & 1);
            issue_load(it_ld++);
        }
        asm volatile("cp.async.commit_group;\n" ::: "memory");
        asm volatile("cp.async.wait_group %0;\n" ::"n"(STAGES - 1) : "memory");   // item it_cm landed
        asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");            // generic writes -> tensor core
        __syncthreads();
        const int s = (int)(it_cm % STAGES);
        if (threadIdx.x == 0) {
            asm volatile("tcgen05.fence::after_thread_sync;\n" ::: "memory");
            const uint32_t a0 = smem_u32(sA + s * A_STAGE), b0 = smem_u32(sB + s * b_stage);
#pragma unroll
            for (int ks = 0; ks < BK / 16; ++ks) {
                const uint64_t ad = smem_desc(a0 + ks * 256), bd = smem_desc(b0 + ks * 256);
                const uint32_t acc = (cm.kb > 0 || ks > 0) ? 1u : 0u;
                asm volatile(
                    "{\n\t.reg .pred p;\n\t"
                    "setp.ne.b32 p, %4, 0;\n\t"
                    "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(tmem),
                    "l"(ad), "l"(bd), "r"(idesc), "r"(acc)
                    : "memory");
            }
            asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n" ::"r"(
                             smem_u32(mbar + s))
                         : "memory");
        }
        if (cm.kb == cm.nkb - 1) {
            mbar_wait(smem_u32(mbar + s), (it_cm / STAGES) & 1);   // the unit's accumulator is complete
            asm volatile("tcgen05.fence::after_thread_sync;\n" ::: "memory");
            epilogue<MODE>(a, tmem, stage_out + warp * (32 * 33), cm.m0 + warp * 32, cm.n0, m_valid, bn, warp, lane);
            asm volatile("tcgen05.fence::before_thread_sync;\n" ::: "memory");
        }
        ++it_cm;
        if (++cm.kb == cm.nkb && !unit_at<MODE>(cm, cm.u + gridDim.x, a, rows, nt, splits)) break;
    }
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;\n" ::"r"(tmem), "r"(ncols));
}

inline int smem_bytes(int bn) { return STAGES * (A_STAGE + bn * BK * 2) + 4 * 32 * 33 * 4 + 64; }

// Host launcher.  rows_max: host bound of *rows_dev (grid sizing).  n_total: output columns
// (split into <= 256-wide tiles).  splits: DW reduction slices per tile.
inline cudaError_t launch(int mode, const Args& a0, int64_t rows_max, int n_total, int splits, cudaStream_t st) {
    Args a = a0;
    const int nt = (n_total + 255) / 256;
    int bn = (n_total + nt - 1) / nt;
    bn = (bn + 15) / 16 * 16;
    a.bn = bn;
    if (splits < 1) splits = 1;
    const int smem = smem_bytes(bn);
    int ncols = 32;
    while (ncols < bn) ncols <<= 1;
    const int per_sm = std::max(1, std::min(227 * 1024 / smem, 512 / ncols));
    const int64_t units = mode == DW ? (a.m_valid + BM - 1) / BM * nt * splits : (rows_max + BM - 1) / BM * nt;
    if (units <= 0) return cudaSuccess;
    const unsigned grid = (unsigned)std::min<int64_t>(units, (int64_t)148 * per_sm);
    cudaError_t e = cudaSuccess;
    switch (mode) {
        case FWD:
            e = cudaFuncSetAttribute(k_umma_gemm<FWD>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
            if (e == cudaSuccess) k_umma_gemm<FWD><<<grid, 128, smem, st>>>(a, nt, splits);
            break;
        case DA:
            e = cudaFuncSetAttribute(k_umma_gemm<DA>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
            if (e == cudaSuccess) k_umma_gemm<DA><<<grid, 128, smem, st>>>(a, nt, splits);
            break;
        default:
            e = cudaFuncSetAttribute(k_umma_gemm<DW>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
            if (e == cudaSuccess) k_umma_gemm<DW><<<grid, 128, smem, st>>>(a, nt, splits);
            break;
    }
    return e != cudaSuccess ? e : cudaGetLastError();
}

}  // namespace umma
}  // namespace gd
