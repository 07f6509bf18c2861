// gd_umma.cuh — hand-written sm_100a tensor-core GEMM (TMA -> shared memory -> tcgen05.mma,
// accumulator in TMEM) for the f4 train stage.  The three GEMMs of a GraphSAGE layer:
//   FWD  H[i, n]  = f(sum_k A16[i, k] W16[k, n] + b[n])   f = relu (hidden, bf16 out) or id (logits)
//   DA   dA[i, n] = sum_k dZ16[i, k] W16[n, k]
//   DW   dW[m, n] += sum_i A16[i, m] dZ16[i, n]           (split over i, fp32 red.add)
// for i < n_dst, all with bf16 operands and fp32 accumulation.  The row count n_dst lives in
// device memory (it is the sampled block size), so work past it is skipped on the device:
// unlike a library GEMM run at the host-side bound, no padded rows are multiplied or written.
//
// Tile: UMMA M = 128 rows (one TMEM lane per output row), N = bn <= 256 columns (TMEM
// columns), K = 64 per pipeline stage (4 MMAs of K = 16).  CTAs are persistent over the tiles
// ("units"; DW units are (tile, row slice) pairs), fetched from a per-launch atomic counter
// (a CTA that only gets an SM after the others finished finds no work and leaves, so SMs held
// by concurrent kernels of the SET pipeline do not stretch the grid), and warp-specialised
// (288 threads):
//   warp 0, lane 0: producer + MMA issuer.  It keeps STAGES-1 k-blocks of TMA loads in flight
//     ahead of the MMAs, across unit boundaries (TMA completes a stage's "full" mbarrier with
//     its byte count; the tcgen05.commit of the MMAs that read a stage arrives on its "empty"
//     mbarrier, which lets the stage be refilled), and accumulates unit u into TMEM buffer
//     u % 2, committing the unit's last k-block to acc_full[u % 2].
//   warps 1-8: epilogue.  Warp w drains TMEM lanes 32 (w % 4).. (one output row per thread)
//     of the finished buffer, alternate 32-column chunks per warp pair (tcgen05.ld, 32
//     columns per load), adds the bias / applies relu and writes 16-byte vectors of its row
//     (fp32 / bf16 stores, or fp32 vector red.add for DW), then arrives on acc_empty[u % 2].
//     The next unit's MMAs run meanwhile in the other buffer.
//
// Operand tiles use the 128-byte-swizzled canonical UMMA layouts that TMA writes directly
// (SWIZZLE_128B, tile bases 1024-byte aligned):
//   K-major  (K contiguous in global):  box {64 (K), R rows}: row r at r * 128 B, 8-row groups
//            1024 B apart (SBO); the k-th MMA (K = 16) of a stage starts 32 B further.
//   MN-major (M/N contiguous in global): boxes {64 (M/N), 64 (K)}: K-row k at k * 128 B, 8-row
//            K groups 1024 B apart (SBO), 64-wide M/N blocks 8 KB apart (LBO); the k-th MMA
//            starts 2048 B further.
// Out-of-bounds box elements (past the tensor extents) are zero-filled by TMA.  Rows between
// the device count and the host bound hold stale data: FWD / DA never store those rows, and
// DW (which reduces over rows) requires the producers of A16 / dZ16 to zero rows
// [n, round_up(n, 64)) (k_sage_agg, k_xent and k_relu_grad do).
#pragma once
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>

#include "gd_common.cuh"   // GD_PDL_ENTRY, launch_chain

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
    int n_valid;                 // B's extent along N (multiple of 8; zero-filled past it)
    int n_store;                 // output columns written
    int bn;                      // N tile (multiple of 16, <= 256; multiple of 64 when B is MN-major)
    unsigned int* counter;       // device words {work, exits}: zero at launch; the last CTA to
                                 // leave re-zeroes them, so back-to-back launches need no memset
};

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_wait(uint32_t addr, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra WAIT_%=;\n}\n" ::"r"(addr),
        "r"(parity)
        : "memory");
}

__device__ __forceinline__ void tma2d(uint32_t dst, const CUtensorMap* map, int32_t c0, int32_t c1, uint32_t bar) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];\n" ::"r"(dst),
        "l"((uint64_t)map), "r"(c0), "r"(c1), "r"(bar)
        : "memory");
}

// UMMA shared-memory descriptor, SWIZZLE_128B (layout type 2), version 1 (sm_100).
__device__ __forceinline__ uint64_t smem_desc_sw128(uint32_t addr, uint32_t lbo, uint32_t sbo) {
    return (uint64_t)((addr >> 4) & 0x3FFF) | ((uint64_t)((lbo >> 4) & 0x3FFF) << 16) |
           ((uint64_t)((sbo >> 4) & 0x3FFF) << 32) | ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
}

template <bool A_MN, bool B_MN>
__host__ __device__ constexpr uint32_t instr_desc(int bn) {
    return (1u << 4)                      // D format f32
           | (1u << 7) | (1u << 10)       // A, B bf16
           | ((A_MN ? 1u : 0u) << 15) | ((B_MN ? 1u : 0u) << 16)
           | ((uint32_t)(bn >> 3) << 17)  // N / 8
           | ((uint32_t)(BM >> 4) << 24); // M / 16
}

// Epilogue of one unit for one epilogue warp: TMEM lanes 32q.. (q = CTA warp % 4, the
// tcgen05.ld lane rule) are tile rows rbase..rbase+31, one row per thread; the warp takes the
// 32-column chunks c0 = 32 h, 32 h + 64, ... (h = which of the two warps of the quarter).  A
// thread holds 32 consecutive columns of its row after one tcgen05.ld and writes them as
// 16-byte vectors (bf16: 4 stores, fp32: 8) or vector red.adds (DW), scalar at a ragged edge.
template <int MODE, bool OUT_BF16, bool RELU>
__device__ __forceinline__ void epilogue(const Args& a, uint32_t tacc, int64_t rbase, int64_t n0, int64_t m_valid, int bn,
                                         int h, int lane, bool vec_ok) {
    const int64_t row = rbase + lane;
    const bool row_ok = row < m_valid;
    for (int c0 = 32 * h; c0 < bn; c0 += 64) {
        uint32_t r[32];
        asm volatile(
            "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
            "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];\n"
            : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
              "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
              "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
              "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
            : "r"(tacc + (uint32_t)c0));
        asm volatile("tcgen05.wait::ld.sync.aligned;\n" ::: "memory");
        const int64_t cg = n0 + c0;
        if (!row_ok || cg >= a.n_store) continue;
        float v[32];
#pragma unroll
        for (int j = 0; j < 32; ++j) {
            v[j] = __uint_as_float(r[j]);
            if (MODE == FWD) {
                if (a.bias) v[j] += cg + j < a.n_store ? __ldg(a.bias + cg + j) : 0.f;
                if (RELU) v[j] = fmaxf(v[j], 0.f);
            }
        }
        const bool full = vec_ok && cg + 32 <= a.n_store;
        if (MODE == DW) {
            float* dst = (float*)a.C + row * a.ldc + cg;
            if (full) {
#pragma unroll
                for (int j = 0; j < 32; j += 4) atomicAdd((float4*)(dst + j), make_float4(v[j], v[j + 1], v[j + 2], v[j + 3]));
            } else {
                for (int j = 0; j < 32 && cg + j < a.n_store; ++j) atomicAdd(dst + j, v[j]);
            }
        } else if (OUT_BF16) {
            __nv_bfloat16* dst = (__nv_bfloat16*)a.C + row * a.ldc + cg;
            if (full) {
#pragma unroll
                for (int j = 0; j < 32; j += 8) {
                    uint4 w;
                    __nv_bfloat162 p0 = __floats2bfloat162_rn(v[j], v[j + 1]), p1 = __floats2bfloat162_rn(v[j + 2], v[j + 3]);
                    __nv_bfloat162 p2 = __floats2bfloat162_rn(v[j + 4], v[j + 5]), p3 = __floats2bfloat162_rn(v[j + 6], v[j + 7]);
                    w.x = *(uint32_t*)&p0; w.y = *(uint32_t*)&p1; w.z = *(uint32_t*)&p2; w.w = *(uint32_t*)&p3;
                    *(uint4*)(dst + j) = w;
                }
            } else {
                for (int j = 0; j < 32 && cg + j < a.n_store; ++j) dst[j] = __float2bfloat16_rn(v[j]);
            }
        } else {
            float* dst = (float*)a.C + row * a.ldc + cg;
            if (full) {
#pragma unroll
                for (int j = 0; j < 32; j += 4) *(float4*)(dst + j) = make_float4(v[j], v[j + 1], v[j + 2], v[j + 3]);
            } else {
                for (int j = 0; j < 32 && cg + j < a.n_store; ++j) dst[j] = v[j];
            }
        }
    }
}

// One unit of work: an output tile (m0, n0) and its reduction range [k_begin, k_end).
struct Unit {
    int64_t u, m0, n0, k_begin, k_end;
    int nkb, kb;
};

// Units: FWD / DA: (m-tile, n-tile) over the device row count, full K.  DW: (m-tile, n-tile,
// split) with split z taking a BK-aligned slice of the device row count.  decode: 1 = a unit
// with work, 0 = an empty DW slice, -1 = past the last unit.
template <int MODE>
__device__ __forceinline__ int decode_unit(Unit& c, int64_t u, const Args& a, int64_t rows, int nt, int splits) {
    if (MODE == DW) {
        const int64_t mt = (a.m_valid + BM - 1) / BM;
        if (u >= mt * nt * splits) return -1;
        const int64_t z = u % splits, rest = u / splits;
        c.n0 = (rest % nt) * a.bn;
        c.m0 = (rest / nt) * BM;
        int64_t per = (rows + splits - 1) / splits;
        per = (per + BK - 1) / BK * BK;
        c.k_begin = z * per;
        c.k_end = c.k_begin + per < rows ? c.k_begin + per : rows;
        if (c.k_begin >= c.k_end) return 0;
    } else {
        if (u >= (rows + BM - 1) / BM * nt) return -1;
        c.m0 = (u / nt) * BM;
        c.n0 = (u % nt) * a.bn;
        c.k_begin = 0;
        c.k_end = a.k_valid;
    }
    c.u = u;
    c.kb = 0;
    c.nkb = (int)((c.k_end - c.k_begin + BK - 1) / BK);
    return 1;
}

// Next unit with work from the launch's shared counter (CTAs that start late, e.g. on SMs
// other streams' kernels held, find the work taken and leave instead of delaying the grid).
template <int MODE>
__device__ __forceinline__ bool fetch_unit(Unit& c, const Args& a, int64_t rows, int nt, int splits) {
    for (;;) {
        const int r = decode_unit<MODE>(c, (int64_t)atomicAdd(a.counter, 1u), a, rows, nt, splits);
        if (r != 0) return r > 0;
    }
}

// The last CTA of the grid to leave re-zeroes the work counter (every CTA has fetched its
// last unit by then), so the next launch starts from zero without a memset between kernels.
__device__ __forceinline__ void cta_exit(unsigned int* counter) {
    __threadfence();
    if (atomicAdd(counter + 1, 1u) == gridDim.x - 1) {
        counter[0] = 0u;
        counter[1] = 0u;
        __threadfence();
    }
}

template <int MODE, bool OUT_BF16, bool RELU>
__global__ void __launch_bounds__(288) k_umma_gemm(const __grid_constant__ CUtensorMap tmA,
                                                   const __grid_constant__ CUtensorMap tmB, Args a, int nt, int splits,
                                                   int vec_ok) {
    constexpr bool A_MN = MODE == DW;
    constexpr bool B_MN = MODE != DA;
    GD_PDL_ENTRY();   // the operands are the previous kernel's outputs
    extern __shared__ uint8_t smem_raw[];
    // SWIZZLE_128B tiles need 1024-byte aligned bases
    uint8_t* smem = smem_raw + ((1024 - (smem_u32(smem_raw) & 1023)) & 1023);
    const int bn = a.bn;
    const int b_stage = bn * BK * 2;
    uint8_t* sA = smem;
    uint8_t* sB = smem + STAGES * A_STAGE;
    uint64_t* full = (uint64_t*)(sB + STAGES * b_stage);
    uint64_t* empty = full + STAGES;
    uint64_t* acc_full = empty + STAGES;                          // [2] accumulator buffer ready
    uint64_t* acc_empty = acc_full + 2;                           // [2] accumulator buffer drained
    uint32_t* tmem_slot = (uint32_t*)(acc_empty + 2);
    int64_t* ep_unit = (int64_t*)(tmem_slot + 2);                 // [2] unit id of each accumulator buffer (-1: end)

    const int64_t rows = *a.rows_dev;   // device-resident size
    Unit cm;
    __shared__ int64_t first_unit;
    if (threadIdx.x == 0) first_unit = fetch_unit<MODE>(cm, a, rows, nt, splits) ? cm.u : -1;
    __syncthreads();
    if (first_unit < 0) {               // no work left for this CTA
        if (threadIdx.x == 0) cta_exit(a.counter);
        return;
    }
    decode_unit<MODE>(cm, first_unit, a, rows, nt, splits);
    const int64_t m_valid = MODE == DW ? a.m_valid : rows;
    uint32_t nc = 32;                   // columns of one accumulator buffer
    while ((int)nc < bn) nc <<= 1;

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;\n" ::"r"(smem_u32(tmem_slot)),
                     "r"(2 * nc));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;\n");
    }
    if (threadIdx.x == 0) {
        asm volatile("prefetch.tensormap [%0];\n" ::"l"((uint64_t)&tmA) : "memory");
        asm volatile("prefetch.tensormap [%0];\n" ::"l"((uint64_t)&tmB) : "memory");
        for (int s = 0; s < 2 * STAGES; ++s)
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;\n" ::"r"(smem_u32(full + s)));
        for (int s = 0; s < 2; ++s)   // tcgen05.commit + the issuer's arrive after publishing the unit id
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 2;\n" ::"r"(smem_u32(acc_full + s)));
        for (int s = 0; s < 2; ++s)
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 8;\n" ::"r"(smem_u32(acc_empty + s)));   // one per epilogue warp
        asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;\n" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;\n" ::: "memory");
    const uint32_t tmem = *tmem_slot;

    if (warp == 0) {
        if (lane == 0) {
            // ===== producer (TMA) + MMA issuer
            const uint32_t idesc = instr_desc<A_MN, B_MN>(bn);
            const uint32_t stage_bytes = (uint32_t)(A_STAGE + b_stage);
            Unit ld = cm;
            bool ld_ok = true;
            // the next unit id is fetched one unit ahead, so the atomic's round trip hides
            // behind the current unit's loads instead of stalling the producer
            unsigned int next_u = atomicAdd(a.counter, 1u);
            int64_t uq[8];                 // units fetched by the load cursor, not yet reached by the MMAs
            uint32_t uq_head = 0, uq_tail = 0;
            uint32_t it_ld = 0, it_cm = 0, u_local = 0;
            auto issue_load = [&]() {
                const int s = (int)(it_ld % STAGES);
                if (it_ld >= STAGES) mbar_wait(smem_u32(empty + s), ((it_ld / STAGES) - 1) & 1);   // stage's MMAs done
                const uint32_t fb = smem_u32(full + s);
                asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(fb), "r"(stage_bytes) : "memory");
                const int32_t k0 = (int32_t)(ld.k_begin + (int64_t)ld.kb * BK);
                const uint32_t a0 = smem_u32(sA + s * A_STAGE), b0 = smem_u32(sB + s * b_stage);
                if (!A_MN) tma2d(a0, &tmA, k0, (int32_t)ld.m0, fb);
                else
                    for (int j = 0; j < BM / 64; ++j) tma2d(a0 + j * 8192, &tmA, (int32_t)ld.m0 + 64 * j, k0, fb);
                if (!B_MN) tma2d(b0, &tmB, k0, (int32_t)ld.n0, fb);
                else
                    for (int j = 0; j < bn / 64; ++j) tma2d(b0 + j * 8192, &tmB, (int32_t)ld.n0 + 64 * j, k0, fb);
                ++it_ld;
                if (++ld.kb == ld.nkb) {
                    int r;
                    while ((r = decode_unit<MODE>(ld, (int64_t)next_u, a, rows, nt, splits)) == 0)   // empty DW slice
                        next_u = atomicAdd(a.counter, 1u);
                    ld_ok = r > 0;
                    if (ld_ok) {
                        uq[uq_tail++ & 7] = ld.u;
                        next_u = atomicAdd(a.counter, 1u);
                    }
                }
            };
            for (int s = 0; s < STAGES - 1 && ld_ok; ++s) issue_load();
            for (;;) {
                const int s = (int)(it_cm % STAGES);
                const uint32_t buf = u_local & 1;
                if (cm.kb == 0 && u_local >= 2)   // the epilogue of unit u_local - 2 drained this buffer
                    mbar_wait(smem_u32(acc_empty + buf), ((u_local >> 1) - 1) & 1);
                mbar_wait(smem_u32(full + s), (it_cm / STAGES) & 1);            // operands landed
                asm volatile("tcgen05.fence::after_thread_sync;\n" ::: "memory");
                const uint32_t a0 = smem_u32(sA + s * A_STAGE), b0 = smem_u32(sB + s * b_stage);
#pragma unroll
                for (int ks = 0; ks < BK / 16; ++ks) {
                    const uint64_t ad = A_MN ? smem_desc_sw128(a0 + ks * 2048, 8192, 1024) : smem_desc_sw128(a0 + ks * 32, 16, 1024);
                    const uint64_t bd = B_MN ? smem_desc_sw128(b0 + ks * 2048, 8192, 1024) : smem_desc_sw128(b0 + ks * 32, 16, 1024);
                    const uint32_t acc = (cm.kb > 0 || ks > 0) ? 1u : 0u;
                    asm volatile(
                        "{\n\t.reg .pred p;\n\t"
                        "setp.ne.b32 p, %4, 0;\n\t"
                        "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(tmem + buf * nc),
                        "l"(ad), "l"(bd), "r"(idesc), "r"(acc)
                        : "memory");
                }
                asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n" ::"r"(
                                 smem_u32(empty + s))
                             : "memory");
                const bool last = cm.kb == cm.nkb - 1;
                if (last) {
                    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n" ::"r"(
                                     smem_u32(acc_full + buf))
                                 : "memory");
                    ep_unit[buf] = cm.u;   // published by the release-arrive below
                    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];\n" ::"r"(smem_u32(acc_full + buf)) : "memory");
                }
                if (ld_ok) issue_load();   // refill the stage the previous k-block used (MMAs stay queued)
                ++it_cm;
                if (last) ++u_local;
                if (++cm.kb == cm.nkb) {
                    if (uq_head == uq_tail) break;
                    decode_unit<MODE>(cm, uq[uq_head++ & 7], a, rows, nt, splits);
                }
            }
            // end marker for the epilogue warps in the next buffer
            const uint32_t buf = u_local & 1;
            if (u_local >= 2) mbar_wait(smem_u32(acc_empty + buf), ((u_local >> 1) - 1) & 1);
            ep_unit[buf] = -1;
            asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];\n" ::"r"(smem_u32(acc_full + buf)) : "memory");
            asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];\n" ::"r"(smem_u32(acc_full + buf)) : "memory");
        }
    } else {
        // ===== epilogue warps 1..8: TMEM lane quarter q = warp % 4 (tcgen05.ld lane rule),
        // column half h = (warp - 1) / 4
        const int q = warp & 3, h = (warp - 1) >> 2;
        for (uint32_t u_local = 0;; ++u_local) {
            const uint32_t buf = u_local & 1;
            mbar_wait(smem_u32(acc_full + buf), (u_local >> 1) & 1);
            const int64_t u = *(volatile int64_t*)(ep_unit + buf);
            if (u < 0) break;
            decode_unit<MODE>(cm, u, a, rows, nt, splits);
            asm volatile("tcgen05.fence::after_thread_sync;\n" ::: "memory");
            epilogue<MODE, OUT_BF16, RELU>(a, tmem + buf * nc + ((uint32_t)(q * 32) << 16), cm.m0 + q * 32, cm.n0, m_valid, bn,
                                           h, lane, vec_ok != 0);
            asm volatile("tcgen05.fence::before_thread_sync;\n" ::: "memory");
            __syncwarp();
            if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];\n" ::"r"(smem_u32(acc_empty + buf)) : "memory");
        }
    }
    __syncthreads();
    if (warp == 0) {
        asm volatile("tcgen05.fence::after_thread_sync;\n" ::: "memory");
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;\n" ::"r"(tmem), "r"(2 * nc));
    }
    if (threadIdx.x == 0) cta_exit(a.counter);
}

inline int smem_bytes(int bn) { return 1024 + STAGES * (A_STAGE + bn * BK * 2) + (2 * STAGES + 4) * 8 + 8 + 16; }

// 2-D bf16 tensor map, SWIZZLE_128B, box {64, box_outer}; inner = contiguous extent, outer =
// rows, ld = row stride in elements.  Out-of-bounds box elements read as zero.
inline cudaError_t make_map(CUtensorMap* m, const void* base, uint64_t inner, uint64_t outer, uint64_t ld, uint32_t box_outer) {
    static PFN_cuTensorMapEncodeTiled_v12000 encode = nullptr;
    if (!encode) {
        cudaDriverEntryPointQueryResult q;
        cudaError_t e = cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&encode, cudaEnableDefault, &q);
        if (e != cudaSuccess || q != cudaDriverEntryPointSuccess || !encode) return e != cudaSuccess ? e : cudaErrorNotSupported;
    }
    const cuuint64_t dims[2] = {inner, outer < 1 ? 1 : outer};
    const cuuint64_t strides[1] = {ld * 2};
    const cuuint32_t box[2] = {64, box_outer};
    const cuuint32_t es[2] = {1, 1};
    const CUresult r = encode(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims, strides, box, es,
                              CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                              CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS ? cudaSuccess : cudaErrorInvalidValue;
}

// Host launcher.  rows_max: host bound of *rows_dev (grid sizing, tensor extents).  n_total:
// output columns (split into <= 256-wide tiles).  splits: DW reduction slices per tile.
// a.counter: two device words, zero before the first launch (each launch leaves them zero).
inline cudaError_t launch(int mode, const Args& a0, int64_t rows_max, int n_total, int splits, cudaStream_t st) {
    Args a = a0;
    const bool b_mn = mode != DA;
    const int nt = (n_total + 255) / 256;
    int bn = (n_total + nt - 1) / nt;
    bn = b_mn ? (bn + 63) / 64 * 64 : (bn + 15) / 16 * 16;
    a.bn = bn;
    if (splits < 1) splits = 1;
    CUtensorMap tmA, tmB;
    cudaError_t e;
    if (mode == FWD) {
        e = make_map(&tmA, a.A, a.k_valid, rows_max, a.lda, BM);
        if (e == cudaSuccess) e = make_map(&tmB, a.B, a.n_valid, a.k_valid, a.ldb, 64);
    } else if (mode == DA) {
        e = make_map(&tmA, a.A, a.k_valid, rows_max, a.lda, BM);
        if (e == cudaSuccess) e = make_map(&tmB, a.B, a.k_valid, a.n_valid, a.ldb, bn);
    } else {
        e = make_map(&tmA, a.A, a.m_valid, rows_max, a.lda, 64);
        if (e == cudaSuccess) e = make_map(&tmB, a.B, a.n_valid, rows_max, a.ldb, 64);
    }
    if (e != cudaSuccess) return e;
    const int smem = smem_bytes(bn);
    int ncols = 32;
    while (ncols < bn) ncols <<= 1;
    const int per_sm = std::max(1, std::min(227 * 1024 / smem, 512 / (2 * ncols)));   // two accumulator buffers
    const int64_t units = mode == DW ? (a.m_valid + BM - 1) / BM * nt * splits : (rows_max + BM - 1) / BM * nt;
    if (units <= 0) return cudaSuccess;
    if (!a.counter) return cudaErrorInvalidValue;
    const unsigned grid = (unsigned)std::min<int64_t>(units, (int64_t)148 * per_sm);
    const int vec_ok = mode == FWD && a.c_bf16 ? (a.ldc % 8 == 0) : (a.ldc % 4 == 0);
#define GD_UMMA_LAUNCH(M, BF, RL)                                                                     \
    do {                                                                                              \
        e = cudaFuncSetAttribute(k_umma_gemm<M, BF, RL>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem); \
        if (e == cudaSuccess) e = launch_chain(k_umma_gemm<M, BF, RL>, dim3(grid), dim3(288), smem, st, tmA, tmB, a, nt, splits, vec_ok); \
    } while (0)
    if (mode == FWD) {
        if (a.c_bf16 && a.relu) GD_UMMA_LAUNCH(FWD, true, true);
        else if (a.c_bf16) GD_UMMA_LAUNCH(FWD, true, false);
        else if (a.relu) GD_UMMA_LAUNCH(FWD, false, true);
        else GD_UMMA_LAUNCH(FWD, false, false);
    } else if (mode == DA) {
        if (a.c_bf16) GD_UMMA_LAUNCH(DA, true, false);
        else GD_UMMA_LAUNCH(DA, false, false);
    } else {
        GD_UMMA_LAUNCH(DW, false, false);
    }
#undef GD_UMMA_LAUNCH
    return e != cudaSuccess ? e : cudaGetLastError();
}

}  // namespace umma
}  // namespace gd
