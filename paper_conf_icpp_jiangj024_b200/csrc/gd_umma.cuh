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
// K = 64 per pipeline stage (4 MMAs of K = 16).  The 128 threads of the CTA stage operands with
// cp.async (16-byte chunks, zero-filled past the valid range) into the no-swizzle canonical
// UMMA layouts, 2 stages deep; thread 0 issues the MMAs and tcgen05.commit's them to the
// stage's mbarrier, which releases the stage for the next load.  The epilogue reads the
// accumulator with tcgen05.ld (warp w owns TMEM lanes 32w..32w+31 = rows), adds the bias,
// stores fp32 (FWD: also relu into H) or red.adds the split-K partial (DW).
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

namespace gd {
namespace umma {

constexpr int BM = 128;
constexpr int BK = 64;
constexpr int STAGES = 2;
constexpr int A_STAGE = BM * BK * 2;   // 16 KB

enum Mode { FWD = 0, DA = 1, DW = 2 };

struct Args {
    const __nv_bfloat16* A; int64_t lda;
    const __nv_bfloat16* B; int64_t ldb;
    float* C; int64_t ldc;
    float* H;                    // FWD: relu(C) (nullable)
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

// Stage one operand tile (R rows along M/N starting at r0, BK along K starting at k0).
template <bool MN_MAJOR>
__device__ __forceinline__ void load_tile(uint32_t s, const __nv_bfloat16* __restrict__ g, int64_t ld, int R, int64_t r0,
                                          int64_t r_valid, int64_t k0, int64_t k_end) {
    if (!MN_MAJOR) {
        const int total = R * 8;
        for (int idx = threadIdx.x; idx < total; idx += blockDim.x) {
            const int r = idx >> 3, k8 = idx & 7;
            const int64_t gr = r0 + r, gk = k0 + k8 * 8;
            const bool v = gr < r_valid && gk < k_end;
            cp_async16(s + (r >> 3) * 1024 + k8 * 128 + (r & 7) * 16, v ? g + gr * ld + gk : g, v);
        }
    } else {
        const int r8n = R >> 3;
        const int total = r8n * BK;
        for (int idx = threadIdx.x; idx < total; idx += blockDim.x) {
            const int r8 = idx % r8n, k = idx / r8n;
            const int64_t gr = r0 + r8 * 8, gk = k0 + k;
            const bool v = gr < r_valid && gk < k_end;
            cp_async16(s + r8 * 1024 + (k >> 3) * 128 + (k & 7) * 16, v ? g + gk * ld + gr : g, v);
        }
    }
}

template <int MODE>
__global__ void __launch_bounds__(128) k_umma_gemm(Args a) {
    constexpr bool A_MN = MODE == DW;
    constexpr bool B_MN = MODE != DA;
    extern __shared__ __align__(1024) uint8_t smem[];
    const int bn = a.bn;
    const int b_stage = bn * BK * 2;
    uint8_t* sA = smem;
    uint8_t* sB = smem + STAGES * A_STAGE;
    uint64_t* mbar = (uint64_t*)(sB + STAGES * b_stage);
    uint32_t* tmem_slot = (uint32_t*)(mbar + STAGES);

    // ---- work range (device-resident sizes: tiles past them leave at once)
    const int64_t rows = *a.rows_dev;
    int64_t m0, m_valid, k_begin, k_end;
    if (MODE == DW) {
        m0 = (int64_t)blockIdx.x * BM;
        m_valid = a.m_valid;
        int64_t per = (rows + gridDim.z - 1) / gridDim.z;
        per = (per + BK - 1) / BK * BK;
        k_begin = (int64_t)blockIdx.z * per;
        k_end = k_begin + per < rows ? k_begin + per : rows;
        if (k_begin >= k_end) return;
    } else {
        m0 = (int64_t)blockIdx.x * BM;
        m_valid = rows;
        k_begin = 0;
        k_end = a.k_valid;
        if (m0 >= rows) return;
    }
    const int64_t n0 = (int64_t)blockIdx.y * bn;
    const int nkb = (int)((k_end - k_begin + BK - 1) / BK);
    uint32_t ncols = 32;
    while ((int)ncols < bn) ncols <<= 1;

    // ---- setup: TMEM accumulator (warp 0), stage barriers (thread 0)
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

    auto load_stage = [&](int kb) {
        const int s = kb % STAGES;
        const int64_t k0 = k_begin + (int64_t)kb * BK;
        load_tile<A_MN>(smem_u32(sA + s * A_STAGE), a.A, a.lda, BM, m0, m_valid, k0, k_end);
        load_tile<B_MN>(smem_u32(sB + s * b_stage), a.B, a.ldb, bn, n0, a.n_valid, k0, k_end);
    };

    // ---- main loop: loads of stage kb+1 overlap the MMAs of stage kb
    for (int s = 0; s < STAGES - 1; ++s) {
        if (s < nkb) load_stage(s);
        asm volatile("cp.async.commit_group;\n" ::: "memory");
    }
    for (int kb = 0; kb < nkb; ++kb) {
        const int pf = kb + STAGES - 1;
        if (pf < nkb) {
            if (kb >= 1) mbar_wait(smem_u32(mbar + (kb - 1) % STAGES), ((kb - 1) / STAGES) & 1);  // MMAs of kb-1 done
            load_stage(pf);
        }
        asm volatile("cp.async.commit_group;\n" ::: "memory");
        asm volatile("cp.async.wait_group %0;\n" ::"n"(STAGES - 1) : "memory");
        asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");   // generic-proxy writes -> tensor core
        __syncthreads();
        if (threadIdx.x == 0) {
            asm volatile("tcgen05.fence::after_thread_sync;\n" ::: "memory");
            const int s = kb % STAGES;
            const uint32_t a0 = smem_u32(sA + s * A_STAGE), b0 = smem_u32(sB + s * b_stage);
#pragma unroll
            for (int ks = 0; ks < BK / 16; ++ks) {
                const uint64_t ad = smem_desc(a0 + ks * 256), bd = smem_desc(b0 + ks * 256);
                const uint32_t acc = (kb > 0 || ks > 0) ? 1u : 0u;
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
    }
    mbar_wait(smem_u32(mbar + (nkb - 1) % STAGES), ((nkb - 1) / STAGES) & 1);
    asm volatile("tcgen05.fence::after_thread_sync;\n" ::: "memory");

    // ---- epilogue: warp w reads TMEM lanes 32w.. (= tile rows), 16 columns per load
    const int64_t row = m0 + warp * 32 + lane;
    const bool row_ok = row < m_valid;
    for (int c0 = 0; c0 < bn; c0 += 16) {
        uint32_t r[16];
        const uint32_t taddr = tmem + ((uint32_t)(warp * 32) << 16) + (uint32_t)c0;
        asm volatile(
            "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];\n"
            : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
              "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
            : "r"(taddr));
        asm volatile("tcgen05.wait::ld.sync.aligned;\n" ::: "memory");
        const int64_t cg = n0 + c0;
        if (!row_ok || cg >= a.n_store) continue;
        float v[16];
#pragma unroll
        for (int j = 0; j < 16; ++j) v[j] = __uint_as_float(r[j]);
        const bool full = cg + 16 <= a.n_store && (a.ldc & 3) == 0;
        if (MODE == DW) {
            float* dst = a.C + row * a.ldc + cg;
            if (full) {
#pragma unroll
                for (int j = 0; j < 16; j += 4) atomicAdd((float4*)(dst + j), make_float4(v[j], v[j + 1], v[j + 2], v[j + 3]));
            } else {
                for (int j = 0; j < 16 && cg + j < a.n_store; ++j) atomicAdd(dst + j, v[j]);
            }
        } else {
            if (a.bias) {
#pragma unroll
                for (int j = 0; j < 16; ++j) v[j] += cg + j < a.n_store ? __ldg(a.bias + cg + j) : 0.f;
            }
            float* dst = a.C + row * a.ldc + cg;
            float* hdst = a.H ? a.H + row * a.ldc + cg : nullptr;
            if (full) {
#pragma unroll
                for (int j = 0; j < 16; j += 4) {
                    *(float4*)(dst + j) = make_float4(v[j], v[j + 1], v[j + 2], v[j + 3]);
                    if (hdst)
                        *(float4*)(hdst + j) = make_float4(fmaxf(v[j], 0.f), fmaxf(v[j + 1], 0.f), fmaxf(v[j + 2], 0.f),
                                                           fmaxf(v[j + 3], 0.f));
                }
            } else {
                for (int j = 0; j < 16 && cg + j < a.n_store; ++j) {
                    dst[j] = v[j];
                    if (hdst) hdst[j] = fmaxf(v[j], 0.f);
                }
            }
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;\n" ::: "memory");
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;\n" ::"r"(tmem), "r"(ncols));
}

inline int smem_bytes(int bn) { return STAGES * (A_STAGE + bn * BK * 2) + 64; }

// Host launcher.  rows_max: host bound of *rows_dev (grid sizing).  n_total: output columns
// to cover (FWD/DA: n_store rounded up; DW: n_store).  splits: DW reduction CTAs per tile.
inline cudaError_t launch(int mode, const Args& a0, int64_t rows_max, int n_total, int splits, cudaStream_t st) {
    Args a = a0;
    const int nt = (n_total + 255) / 256;                        // N tiles of <= 256 columns
    int bn = (n_total + nt - 1) / nt;
    bn = (bn + 15) / 16 * 16;
    a.bn = bn;
    const int smem = smem_bytes(bn);
    dim3 grid;
    if (mode == DW) grid = dim3((unsigned)((a.m_valid + BM - 1) / BM), (unsigned)nt, (unsigned)(splits < 1 ? 1 : splits));
    else grid = dim3((unsigned)((rows_max + BM - 1) / BM), (unsigned)nt, 1);
    if (grid.x == 0) return cudaSuccess;
    cudaError_t e = cudaSuccess;
    switch (mode) {
        case FWD:
            e = cudaFuncSetAttribute(k_umma_gemm<FWD>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
            if (e == cudaSuccess) k_umma_gemm<FWD><<<grid, 128, smem, st>>>(a);
            break;
        case DA:
            e = cudaFuncSetAttribute(k_umma_gemm<DA>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
            if (e == cudaSuccess) k_umma_gemm<DA><<<grid, 128, smem, st>>>(a);
            break;
        default:
            e = cudaFuncSetAttribute(k_umma_gemm<DW>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
            if (e == cudaSuccess) k_umma_gemm<DW><<<grid, 128, smem, st>>>(a);
            break;
    }
    return e != cudaSuccess ? e : cudaGetLastError();
}

}  // namespace umma
}  // namespace gd
