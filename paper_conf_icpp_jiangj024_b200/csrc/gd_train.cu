// gd_train.cu — f4: the train stage of the SET pipeline on B200.
//
// One GraphSAGE training step on the blocks gd_sample produced and the rows gd_extract
// gathered (the trainer "adopts the node alias list to index required feature data
// in device memory"; GraphSAGE, 3 layers, hidden 256; DDP gradient sync).
// Layer j (j = 0..L-1) consumes hop h = L - j (outermost block first):
//   a_i = [x_i | mean_{e in row i} x_col[e]]  (k_sage_agg: warp per dst row, fp32 sums, bf16 out)
//   z   = a W + b, h = relu(z)                (gd_umma.cuh FWD: tcgen05 GEMM, TMEM accumulator,
//                                              bias + relu in the epilogue)
//   loss = mean softmax cross entropy of the seeds' logits (k_xent + k_loss_sum)
// backward: dW = a^T dz (umma DW, split over rows, red.add), da = dz W^T (umma DA), db =
// column sums of dz (k_colsum_*, deterministic), k_scatter_init + k_sage_scatter spread da to
// the layer's inputs (own row by plain stores, neighbour mean by fp32 red.add), k_relu_grad
// masks by the previous layer's activation.  Every kernel, the GEMMs included, reads the
// block sizes from device memory (gd_sample's `sizes`) and stops there: buffers are sized by
// the host-side bounds (gd_sample_bounds), nothing synchronises the host, and no padded row
// is read, multiplied or written.  Widths dout are stored at a stride dp = round_up(dout, 16)
// (the MMA N granularity; pad columns of W16 and dZ16 are zero).
// Gradients live in one flat fp32 buffer (layout [W0 b0 W1 b1 ...]) that the caller may
// all-reduce (NCCL) between gd_sage_step and gd_sage_apply_sgd.
#include <cuda_bf16.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>

#include "gd_common.cuh"
#include "gd_umma.cuh"

namespace gd {

constexpr uint32_t kMagicSage = 0x47445341u;   // "GDSA"

struct SageLayer {
    int din = 0, dout = 0, dp = 0, hop = 0;     // dp = round_up(dout, 16): row stride of Z, H, dZ16, W16
    int64_t n_dst_max = 0, n_src_max = 0;
    int64_t w_off = 0, b_off = 0, w16_off = 0;   // offsets into params / grads / W16
    __nv_bfloat16* A16 = nullptr;   // [n_dst_max, 2 din]  (saved for backward)
    float* Z = nullptr;             // [n_dst_max, dp]     logits z + b (top layer)
    __nv_bfloat16* H16 = nullptr;   // [n_dst_max, dp]     relu(z + b) (hidden layers: the next layer's input)
    __nv_bfloat16* dZ16 = nullptr;  // [n_dst_max, dp]
    float* dA = nullptr;            // [n_dst_max, 2 din]  (j >= 1)
    float* dX = nullptr;            // [n_src_max, din]    gradient wrt this layer's input (j >= 1)
};

}  // namespace gd

struct gd_sage {
    gd::HandleHdr hdr;
    int L = 0;
    std::vector<int> dims;
    std::vector<int64_t> max_nodes;
    std::vector<gd::SageLayer> layers;
    float* params = nullptr;        // flat fp32 master parameters [W0 b0 W1 b1 ...]
    float* grads = nullptr;         // same layout
    __nv_bfloat16* W16 = nullptr;   // bf16 copies of the W's, [2 din x dp] each (pad columns 0)
    int64_t nparams = 0, nw16 = 0;
    float* loss_rows = nullptr;     // [n0_max]
    float* colsum_part = nullptr;   // [kColsumChunks x max dout] partial column sums (db)
    unsigned int* gemm_counter = nullptr;   // work counter of the (stream-ordered) GEMM launches
    gd::EventTimer timer;                   // GD_SAGE_TIMING=1: per-phase stream times, printed at destroy
    std::vector<const char*> phase;         // name of each timer pair
};

namespace gd {

// ------------------------------------------------------------------ kernels
// rows [n, round_up(n, 64)) of the GEMM operands A16 / dZ16 are zeroed by their producers
// (gd_umma.cuh: the DW GEMM reduces over whole 64-row blocks)
__device__ __forceinline__ int64_t pad64(int64_t n, int64_t n_alloc) {
    const int64_t p = (n + 63) / 64 * 64;
    return p < n_alloc ? p : n_alloc;
}

// a_i = [x_i | mean x_col] for i < n_dst (x fp32 features or bf16 activations, rows at stride ldx).  Warp per row; each lane
// owns 4-column groups (float4) g = lane, lane + 32, ...; neighbour ids are loaded 32 at a
// time and broadcast with shuffles, 4 neighbour rows in flight per lane.
__device__ __forceinline__ float4 load4(const float* __restrict__ row, int g) { return __ldg((const float4*)row + g); }
__device__ __forceinline__ float4 load4(const __nv_bfloat16* __restrict__ row, int g) {
    const uint2 u = __ldg((const uint2*)row + g);
    const float2 a = __bfloat1622float2(*(const __nv_bfloat162*)&u.x), b = __bfloat1622float2(*(const __nv_bfloat162*)&u.y);
    return make_float4(a.x, a.y, b.x, b.y);
}

template <typename T>
__global__ void __launch_bounds__(256) k_sage_agg(const T* __restrict__ x, int64_t ldx, int din,
                                                  const int64_t* __restrict__ rowptr, const int32_t* __restrict__ col,
                                                  const int64_t* __restrict__ n_dst_p, int64_t n_alloc,
                                                  __nv_bfloat16* __restrict__ A16) {
    GD_PDL_ENTRY();
    const int lane = threadIdx.x & 31;
    const int64_t n_dst = *n_dst_p;
    const int64_t n_end = pad64(n_dst, n_alloc);
    const int groups = din >> 2;
    const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
    for (int64_t i = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); i < n_end; i += warps) {
        __nv_bfloat162* arow = (__nv_bfloat162*)(A16 + i * 2 * din);
        if (i >= n_dst) {   // zero pad rows up to a multiple of 64 (the DW GEMM reduces whole 64-row blocks)
            for (int c = lane; c < din; c += 32) arow[c] = __floats2bfloat162_rn(0.f, 0.f);
            continue;
        }
        const int64_t lo = rowptr[i], hi = rowptr[i + 1];
        const float inv = hi > lo ? 1.0f / (float)(hi - lo) : 0.0f;
        for (int g0 = 0; g0 < groups; g0 += 64) {          // up to 2 float4 per lane per pass
            const int ga = g0 + lane, gb = g0 + 32 + lane;
            float4 sa = make_float4(0.f, 0.f, 0.f, 0.f), sb = sa;
            for (int64_t e0 = lo; e0 < hi; e0 += 32) {
                const int m = (int)(hi - e0 < 32 ? hi - e0 : 32);
                const int32_t c = lane < m ? col[e0 + lane] : 0;
                int t = 0;
                for (; t + 4 <= m; t += 4) {      // 4 neighbour rows in flight per lane
                    const T* xr[4];
#pragma unroll
                    for (int q = 0; q < 4; ++q) xr[q] = x + (int64_t)__shfl_sync(0xffffffffu, c, t + q) * ldx;
                    if (ga < groups) {
                        float4 v[4];
#pragma unroll
                        for (int q = 0; q < 4; ++q) v[q] = load4(xr[q], ga);
#pragma unroll
                        for (int q = 0; q < 4; ++q) { sa.x += v[q].x; sa.y += v[q].y; sa.z += v[q].z; sa.w += v[q].w; }
                    }
                    if (gb < groups) {
                        float4 v[4];
#pragma unroll
                        for (int q = 0; q < 4; ++q) v[q] = load4(xr[q], gb);
#pragma unroll
                        for (int q = 0; q < 4; ++q) { sb.x += v[q].x; sb.y += v[q].y; sb.z += v[q].z; sb.w += v[q].w; }
                    }
                }
                for (; t < m; ++t) {
                    const int64_t u = __shfl_sync(0xffffffffu, c, t);
                    const T* xr = x + u * ldx;
                    if (ga < groups) {
                        const float4 v = load4(xr, ga);
                        sa.x += v.x; sa.y += v.y; sa.z += v.z; sa.w += v.w;
                    }
                    if (gb < groups) {
                        const float4 v = load4(xr, gb);
                        sb.x += v.x; sb.y += v.y; sb.z += v.z; sb.w += v.w;
                    }
                }
            }
            const T* xi = x + i * ldx;
            if (ga < groups) {
                const float4 s = load4(xi, ga);
                arow[2 * ga] = __floats2bfloat162_rn(s.x, s.y);
                arow[2 * ga + 1] = __floats2bfloat162_rn(s.z, s.w);
                arow[(din >> 1) + 2 * ga] = __floats2bfloat162_rn(sa.x * inv, sa.y * inv);
                arow[(din >> 1) + 2 * ga + 1] = __floats2bfloat162_rn(sa.z * inv, sa.w * inv);
            }
            if (gb < groups) {
                const float4 s = load4(xi, gb);
                arow[2 * gb] = __floats2bfloat162_rn(s.x, s.y);
                arow[2 * gb + 1] = __floats2bfloat162_rn(s.z, s.w);
                arow[(din >> 1) + 2 * gb] = __floats2bfloat162_rn(sb.x * inv, sb.y * inv);
                arow[(din >> 1) + 2 * gb + 1] = __floats2bfloat162_rn(sb.z * inv, sb.w * inv);
            }
        }
    }
}

// Softmax cross entropy of the logits (z + b, from the FWD epilogue, row stride dp), warp
// per seed row: loss_rows[i] = lse - z[label]; dZ16[i] = (softmax - onehot) / n0 for the C
// classes, 0 in the pad columns [C, dp).  Also zeroes the gradient buffer (the DW GEMMs
// red.add into it), so no memset breaks the train stream's dependent-launch chain.
__global__ void __launch_bounds__(256) k_xent(const float* __restrict__ Z, int C, int dp, const int32_t* __restrict__ labels,
                                              const int64_t* __restrict__ n_p, int64_t n_alloc,
                                              __nv_bfloat16* __restrict__ dZ16, float* __restrict__ loss_rows,
                                              float* __restrict__ grads, int64_t nparams) {
    GD_PDL_ENTRY();
    for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < nparams; k += (int64_t)gridDim.x * blockDim.x)
        grads[k] = 0.f;
    const int lane = threadIdx.x & 31;
    const int64_t n = *n_p;
    const int64_t n_end = pad64(n, n_alloc);
    const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
    for (int64_t i = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); i < n_end; i += warps) {
        const float* z = Z + i * dp;
        __nv_bfloat16* dz = dZ16 + i * dp;
        if (i >= n) {
            for (int c = lane; c < dp; c += 32) dz[c] = __float2bfloat16_rn(0.f);
            continue;
        }
        float m = -INFINITY;
        for (int c = lane; c < C; c += 32) m = fmaxf(m, z[c]);
        for (int o = 16; o; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
        float s = 0.f;
        for (int c = lane; c < C; c += 32) s += __expf(z[c] - m);
        for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
        const int y = labels[i];
        const float inv_n = 1.0f / (float)n;
        for (int c = lane; c < dp; c += 32) {
            const float p = c < C ? __expf(z[c] - m) / s : 0.f;
            dz[c] = __float2bfloat16_rn(c < C ? (p - (c == y ? 1.f : 0.f)) * inv_n : 0.f);
        }
        if (lane == 0) loss_rows[i] = m + __logf(s) - z[y];
    }
}

// loss = mean of loss_rows[0:n] (one block, fixed reduction order: deterministic).
__global__ void k_loss_sum(const float* __restrict__ loss_rows, const int64_t* __restrict__ n_p, float* __restrict__ loss) {
    GD_PDL_ENTRY();
    __shared__ float sh[256];
    const int64_t n = *n_p;
    float s = 0.f;
    for (int64_t i = threadIdx.x; i < n; i += blockDim.x) s += loss_rows[i];
    sh[threadIdx.x] = s;
    __syncthreads();
    for (int w = blockDim.x / 2; w; w >>= 1) {
        if ((int)threadIdx.x < w) sh[threadIdx.x] += sh[threadIdx.x + w];
        __syncthreads();
    }
    if (threadIdx.x == 0) *loss = n > 0 ? sh[0] / (float)n : 0.f;
}

// dX[i] = own-row part of da (first din columns) for i < n_dst, 0 for n_dst <= i < n_src:
// plain stores, so neither a bound-sized memset nor atomics for the own rows.
__global__ void __launch_bounds__(256) k_scatter_init(const float* __restrict__ dA, int din, const int64_t* __restrict__ n_dst_p,
                                                      const int64_t* __restrict__ n_src_p, float* __restrict__ dX) {
    GD_PDL_ENTRY();
    const int64_t n_dst = *n_dst_p, n_src = *n_src_p;
    const int dv = din >> 2;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.y + threadIdx.y; i < n_src; i += (int64_t)gridDim.x * blockDim.y) {
        float4* d4 = (float4*)(dX + i * din);
        const float4* a4 = (const float4*)(dA + i * 2 * din);
        for (int c = threadIdx.x; c < dv; c += blockDim.x) d4[c] = i < n_dst ? a4[c] : make_float4(0.f, 0.f, 0.f, 0.f);
    }
}

// dX += neighbour-mean contributions of da (last din columns / deg), warp per dst row,
// vector red.add (fp32; the summation order of a row's contributions is not fixed).
__global__ void __launch_bounds__(256) k_sage_scatter(const float* __restrict__ dA, int din,
                                                      const int64_t* __restrict__ rowptr, const int32_t* __restrict__ col,
                                                      const int64_t* __restrict__ n_dst_p, float* __restrict__ dX) {
    GD_PDL_ENTRY();
    const int lane = threadIdx.x & 31;
    const int64_t n_dst = *n_dst_p;
    const int groups = din >> 2;
    const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
    for (int64_t i = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); i < n_dst; i += warps) {
        const int64_t lo = rowptr[i], hi = rowptr[i + 1];
        if (hi == lo) continue;
        const float inv = 1.0f / (float)(hi - lo);
        const float4* da = (const float4*)(dA + i * 2 * din) + groups;
        for (int g0 = 0; g0 < groups; g0 += 32) {
            const int g = g0 + lane;
            float4 nb = g < groups ? da[g] : make_float4(0.f, 0.f, 0.f, 0.f);
            nb.x *= inv; nb.y *= inv; nb.z *= inv; nb.w *= inv;
            for (int64_t e0 = lo; e0 < hi; e0 += 32) {
                const int m = (int)(hi - e0 < 32 ? hi - e0 : 32);
                const int32_t c = lane < m ? col[e0 + lane] : 0;
                for (int t = 0; t < m; ++t) {
                    const int64_t u = __shfl_sync(0xffffffffu, c, t);
                    if (g < groups) atomicAdd((float4*)(dX + u * din) + g, nb);
                }
            }
        }
    }
}

// dZ16 = bf16(dX * (H > 0)) for rows < n (dX at stride d, H16 and dZ16 at stride dp; pad
// columns stay zero).  Block (32, 8): threadIdx.x walks a row's float4 columns, threadIdx.y
// rows; no index division.
__global__ void __launch_bounds__(256) k_relu_grad(const float* __restrict__ dX, const __nv_bfloat16* __restrict__ H16, int d, int dp,
                                                   const int64_t* __restrict__ n_p, int64_t n_alloc,
                                                   __nv_bfloat16* __restrict__ dZ16) {
    GD_PDL_ENTRY();
    const int64_t n = *n_p;
    const int64_t n_end = pad64(n, n_alloc);
    const int dv = d >> 2;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.y + threadIdx.y; i < n_end; i += (int64_t)gridDim.x * blockDim.y) {
        const float4* x4 = (const float4*)(dX + i * d);
        const __nv_bfloat16* hrow = H16 + i * dp;
        __nv_bfloat162* o2 = (__nv_bfloat162*)(dZ16 + i * dp);
        if (i >= n) {
            for (int c = threadIdx.x; c < dv; c += blockDim.x)
                o2[2 * c] = o2[2 * c + 1] = __floats2bfloat162_rn(0.f, 0.f);
            continue;
        }
        for (int c = threadIdx.x; c < dv; c += blockDim.x) {
            const float4 x = x4[c], h = load4(hrow, c);
            o2[2 * c] = __floats2bfloat162_rn(h.x > 0.f ? x.x : 0.f, h.y > 0.f ? x.y : 0.f);
            o2[2 * c + 1] = __floats2bfloat162_rn(h.z > 0.f ? x.z : 0.f, h.w > 0.f ? x.w : 0.f);
        }
    }
}

// db = column sums of dZ16 rows < n, deterministic (fixed assignment and reduction order).
// Pass 1: block (32, 8) sums a 32-column strip over row chunk blockIdx.y (thread (x, y) takes
// rows y, y + 8, ... of the chunk), reduces the 8 row lanes in shared memory and writes
// part[chunk][col].  Pass 2 does the same over the kColsumChunks partials.
constexpr int kColsumChunks = 256;
__global__ void __launch_bounds__(256) k_colsum_part(const __nv_bfloat16* __restrict__ dZ16, int d, int ld,
                                                     const int64_t* __restrict__ n_p, float* __restrict__ part) {
    GD_PDL_ENTRY();
    __shared__ float sh[8][33];
    const int64_t n = *n_p;
    const int64_t per = (n + gridDim.y - 1) / gridDim.y;
    const int64_t r0 = (int64_t)blockIdx.y * per, r1 = r0 + per < n ? r0 + per : n;
    const int c = blockIdx.x * 32 + threadIdx.x;
    float s = 0.f;
    if (c < d) {
        int64_t i = r0 + threadIdx.y;
#pragma unroll 4
        for (; i < r1; i += 8) s += __bfloat162float(dZ16[i * ld + c]);
    }
    sh[threadIdx.y][threadIdx.x] = s;
    __syncthreads();
    if (threadIdx.y == 0 && c < d) {
        float t = 0.f;
        for (int y = 0; y < 8; ++y) t += sh[y][threadIdx.x];
        part[(int64_t)blockIdx.y * d + c] = t;
    }
}

__global__ void __launch_bounds__(256) k_colsum_final(const float* __restrict__ part, int d, int nchunk,
                                                      float* __restrict__ out) {
    GD_PDL_ENTRY();
    __shared__ float sh[8][33];
    const int c = blockIdx.x * 32 + threadIdx.x;
    float s = 0.f;
    if (c < d)
        for (int k = threadIdx.y; k < nchunk; k += 8) s += part[(int64_t)k * d + c];
    sh[threadIdx.y][threadIdx.x] = s;
    __syncthreads();
    if (threadIdx.y == 0 && c < d) {
        float t = 0.f;
        for (int y = 0; y < 8; ++y) t += sh[y][threadIdx.x];
        out[c] = t;
    }
}

__global__ void k_sgd(float* __restrict__ p, const float* __restrict__ g, int64_t n, float step) {
    GD_PDL_ENTRY();
    for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < n; k += (int64_t)gridDim.x * blockDim.x)
        p[k] = fmaf(-step, g[k], p[k]);
}

// W16[r, c] = bf16(W[r, c]) for c < d, 0 for d <= c < dp (rows of W at stride d).
__global__ void k_to_bf16(const float* __restrict__ src, __nv_bfloat16* __restrict__ dst, int64_t rows, int d, int dp) {
    GD_PDL_ENTRY();
    for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < rows * dp; k += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = k / dp;
        const int c = (int)(k - r * dp);
        dst[k] = __float2bfloat16_rn(c < d ? src[r * d + c] : 0.f);
    }
}

// ------------------------------------------------------------------ GEMMs (gd_umma.cuh)
static umma::Args gemm_args(const __nv_bfloat16* A, int64_t lda, const __nv_bfloat16* B, int64_t ldb, void* C, int64_t ldc,
                            const int64_t* rows_dev, unsigned int* counter) {
    umma::Args a{};
    a.A = A; a.lda = lda; a.B = B; a.ldb = ldb; a.C = C; a.ldc = ldc; a.rows_dev = rows_dev; a.counter = counter;
    return a;
}

static unsigned grid_for(int64_t n, int per_block = 256) {
    return (unsigned)std::max<int64_t>(1, std::min<int64_t>((n + per_block - 1) / per_block, 148 * 16));
}

static void sage_free(gd_sage* s) {
    if (!s) return;
    DeviceGuard guard(s->hdr.device);
    cudaDeviceSynchronize();
    if (s->timer.on && !s->phase.empty()) {   // summary of the per-phase live times on the train stream
        std::vector<std::pair<const char*, double>> acc;
        int steps = 0;
        for (size_t i = 0; i < s->phase.size(); ++i) {
            float ms = 0;
            const auto pr = s->timer.pairs[i];
            if (pr.second < 0) continue;
            cudaEventElapsedTime(&ms, s->timer.pool[pr.first], s->timer.pool[pr.second]);
            size_t k = 0;
            while (k < acc.size() && std::strcmp(acc[k].first, s->phase[i]) != 0) ++k;
            if (k == acc.size()) acc.push_back({s->phase[i], 0.0});
            acc[k].second += ms;
            if (std::strcmp(s->phase[i], "agg0") == 0) ++steps;
        }
        std::fprintf(stderr, "[gd_sage] live ms per step over %d steps:", steps);
        for (auto& p : acc) std::fprintf(stderr, " %s %.4f", p.first, p.second / std::max(1, steps));
        std::fprintf(stderr, "\n");
    }
    s->timer.destroy();
    for (auto& l : s->layers)
        for (void* p : {(void*)l.A16, (void*)l.Z, (void*)l.H16, (void*)l.dZ16, (void*)l.dA, (void*)l.dX})
            if (p) cudaFree(p);
    for (void* p : {(void*)s->params, (void*)s->grads, (void*)s->W16, (void*)s->loss_rows, (void*)s->colsum_part, (void*)s->gemm_counter})
        if (p) cudaFree(p);
    s->hdr.magic = 0;
    delete s;
}

}  // namespace gd

using namespace gd;

extern "C" {

gd_status gd_sage_create(int32_t num_layers, const int32_t* dims, const float* const* init_w,
                         const float* const* init_b, const int64_t* max_nodes, int device, gd_sage** out) {
    if (!out || !dims || !init_w || !init_b || !max_nodes || num_layers < 1 || num_layers > GD_MAX_HOPS)
        return set_error(GD_ERR_INVALID, "gd_sage_create: null pointer or num_layers outside 1..GD_MAX_HOPS");
    for (int l = 0; l <= num_layers; ++l)
        if (dims[l] <= 0 || dims[l] > 4096 || (l < num_layers && dims[l] % 4 != 0))
            return set_error(GD_ERR_INVALID, "gd_sage_create: widths in 1..4096, input widths multiples of 4");
    for (int l = 0; l <= num_layers; ++l)
        if (max_nodes[l] < 1 || (l > 0 && max_nodes[l] < max_nodes[l - 1]))
            return set_error(GD_ERR_INVALID, "gd_sage_create: max_nodes must be the gd_sample_bounds of the blocks");
    *out = nullptr;
    DeviceGuard guard(device);
    gd_sage* s = new gd_sage();
    s->hdr.magic = kMagicSage;
    s->hdr.device = device;
    s->hdr.dev_status = nullptr;
    s->L = num_layers;
    s->dims.assign(dims, dims + num_layers + 1);
    s->max_nodes.assign(max_nodes, max_nodes + num_layers + 1);
    auto fail = [&](gd_status st) { sage_free(s); return st; };
    int64_t off = 0, off16 = 0;
    s->layers.resize(num_layers);
    for (int j = 0; j < num_layers; ++j) {
        SageLayer& l = s->layers[j];
        l.din = dims[j];
        l.dout = dims[j + 1];
        l.dp = (l.dout + 15) / 16 * 16;
        l.hop = num_layers - j;
        l.n_dst_max = max_nodes[l.hop - 1];
        l.n_src_max = max_nodes[l.hop];
        l.w_off = off;
        off += (int64_t)2 * l.din * l.dout;
        l.b_off = off;
        off += l.dout;
        l.w16_off = off16;
        off16 += (int64_t)2 * l.din * l.dp;
    }
    s->nparams = off;
    s->nw16 = off16;
#define SA(ptr, bytes)                                                                    \
    do {                                                                                  \
        cudaError_t e_ = cudaMalloc(&(ptr), (size_t)(bytes));                             \
        if (e_ != cudaSuccess) return fail(cuda_error(e_, "gd_sage_create: cudaMalloc")); \
    } while (0)
    SA(s->params, off * sizeof(float));
    SA(s->grads, off * sizeof(float));
    SA(s->W16, off16 * sizeof(__nv_bfloat16));
    SA(s->loss_rows, max_nodes[0] * sizeof(float));
    int max_dout = 1;
    for (int j = 0; j < num_layers; ++j) {
        SageLayer& l = s->layers[j];
        SA(l.A16, l.n_dst_max * 2 * l.din * sizeof(__nv_bfloat16));
        if (j == num_layers - 1) SA(l.Z, l.n_dst_max * l.dp * sizeof(float));
        else SA(l.H16, l.n_dst_max * l.dp * sizeof(__nv_bfloat16));
        SA(l.dZ16, l.n_dst_max * l.dp * sizeof(__nv_bfloat16));
        if (j > 0) {
            SA(l.dA, l.n_dst_max * 2 * l.din * sizeof(float));
            SA(l.dX, l.n_src_max * l.din * sizeof(float));
        }
        max_dout = std::max(max_dout, l.dout);
    }
    SA(s->colsum_part, (size_t)kColsumChunks * max_dout * sizeof(float));
    SA(s->gemm_counter, 2 * sizeof(unsigned int));
    if (const char* e = std::getenv("GD_SAGE_TIMING")) s->timer.on = std::atoi(e) != 0;
#undef SA
    if (cudaMemset(s->gemm_counter, 0, 2 * sizeof(unsigned int)) != cudaSuccess)
        return fail(cuda_error(cudaGetLastError(), "gd_sage_create: memset"));
    for (int j = 0; j < num_layers; ++j) {      // pad columns of dZ16 (the DA GEMM's K) start and stay zero
        const SageLayer& l = s->layers[j];
        cudaError_t e = cudaMemset(l.dZ16, 0, l.n_dst_max * l.dp * sizeof(__nv_bfloat16));
        if (e != cudaSuccess) return fail(cuda_error(e, "gd_sage_create: memset"));
    }
    for (int j = 0; j < num_layers; ++j) {
        const SageLayer& l = s->layers[j];
        if (!init_w[j] || !init_b[j]) return fail(set_error(GD_ERR_INVALID, "gd_sage_create: null initial parameter"));
        cudaError_t e = cudaMemcpy(s->params + l.w_off, init_w[j], (size_t)2 * l.din * l.dout * sizeof(float),
                                   cudaMemcpyHostToDevice);
        if (e == cudaSuccess)
            e = cudaMemcpy(s->params + l.b_off, init_b[j], (size_t)l.dout * sizeof(float), cudaMemcpyHostToDevice);
        if (e != cudaSuccess) return fail(cuda_error(e, "gd_sage_create: parameter copy"));
        k_to_bf16<<<grid_for(2 * l.din * l.dp), 256>>>(s->params + l.w_off, s->W16 + l.w16_off, 2 * l.din, l.dout, l.dp);
    }
    if (cudaMemset(s->grads, 0, off * sizeof(float)) != cudaSuccess)
        return fail(cuda_error(cudaGetLastError(), "gd_sage_create: memset"));
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) return fail(cuda_error(e, "gd_sage_create: init kernels"));
    *out = s;
    return GD_OK;
}

gd_status gd_sage_destroy(gd_sage* s) {
    if (!s) return GD_OK;
    if (s->hdr.magic != kMagicSage) return set_error(GD_ERR_INVALID, "gd_sage_destroy: bad handle");
    sage_free(s);
    return GD_OK;
}

gd_status gd_sage_step(gd_sage* s, const int64_t* const* rowptr, const int32_t* const* col, const int64_t* sizes,
                       const float* feats, const int32_t* labels, float* loss, void* stream_v) {
    if (!s || s->hdr.magic != kMagicSage) return set_error(GD_ERR_INVALID, "gd_sage_step: bad handle");
    if (!rowptr || !col || !sizes || !feats || !labels || !loss)
        return set_error(GD_ERR_INVALID, "gd_sage_step: null pointer");
    for (int h = 0; h < s->L; ++h)
        if (!rowptr[h] || !col[h]) return set_error(GD_ERR_INVALID, "gd_sage_step: null block pointer");
    DeviceGuard guard(s->hdr.device);
    cudaStream_t st = (cudaStream_t)stream_v;
    const int L = s->L;
    const dim3 rows_blk(32, 8);          // (float4 column, row) blocks of the row-wise kernels
    int tph = -1;                        // GD_SAGE_TIMING: one event pair per phase
    auto ph_begin = [&]() { tph = s->timer.on ? s->timer.begin(st) : -1; };
    auto ph_end = [&](const char* name) {
        if (tph >= 0) {
            s->timer.end(tph, st);
            s->phase.push_back(name);
        }
    };
    static const char* kAgg[] = {"agg0", "agg1", "agg2", "agg3", "agg4", "agg5", "agg6", "agg7"};
    static const char* kFwd[] = {"fwd0", "fwd1", "fwd2", "fwd3", "fwd4", "fwd5", "fwd6", "fwd7"};
    static const char* kDw[] = {"dw0", "dw1", "dw2", "dw3", "dw4", "dw5", "dw6", "dw7"};
    static const char* kDa[] = {"da0", "da1", "da2", "da3", "da4", "da5", "da6", "da7"};
    static const char* kSc[] = {"scatter0", "scatter1", "scatter2", "scatter3", "scatter4", "scatter5", "scatter6", "scatter7"};
    // ---- forward
    const void* x = feats;
    int64_t ldx = s->dims[0];
    for (int j = 0; j < L; ++j) {
        SageLayer& l = s->layers[j];
        const int h = l.hop;
        const int64_t* n_dst = sizes + (h - 1);
        ph_begin();
        if (j == 0)
            GD_CUDA(launch_chain(k_sage_agg<float>, dim3(grid_for(l.n_dst_max * 32)), dim3(256), 0, st, (const float*)x, ldx, l.din, rowptr[h - 1],
                                                                          col[h - 1], n_dst, l.n_dst_max, l.A16));
        else
            GD_CUDA(launch_chain(k_sage_agg<__nv_bfloat16>, dim3(grid_for(l.n_dst_max * 32)), dim3(256), 0, st, (const __nv_bfloat16*)x, ldx, l.din,
                                                                                  rowptr[h - 1], col[h - 1], n_dst,
                                                                                  l.n_dst_max, l.A16));
        GD_DEBUG_AFTER("k_sage_agg", st);
        ph_end(kAgg[j]);
        ph_begin();
        const bool hidden = j < L - 1;   // hidden: h = relu(z + b) in bf16 (the next layer's input); top: logits
        umma::Args a = gemm_args(l.A16, 2 * l.din, s->W16 + l.w16_off, l.dp, hidden ? (void*)l.H16 : (void*)l.Z, l.dp, n_dst,
                                 s->gemm_counter);
        a.c_bf16 = hidden;
        a.relu = hidden;
        a.bias = s->params + l.b_off;
        a.k_valid = 2 * l.din;
        a.n_valid = l.dp;
        a.n_store = l.dout;
        GD_CUDA(umma::launch(umma::FWD, a, l.n_dst_max, l.dout, 1, st));
        GD_DEBUG_AFTER("k_umma_gemm<FWD>", st);
        ph_end(kFwd[j]);
        x = l.H16;
        ldx = l.dp;
    }
    // ---- loss
    SageLayer& top = s->layers[L - 1];
    ph_begin();
    GD_CUDA(launch_chain(k_xent, dim3(grid_for(top.n_dst_max * 32)), dim3(256), 0, st, top.Z, top.dout, top.dp, labels, sizes,
                         top.n_dst_max, top.dZ16, s->loss_rows, s->grads, s->nparams));
    GD_CUDA(launch_chain(k_loss_sum, dim3(1), dim3(256), 0, st, s->loss_rows, sizes, loss));
    GD_DEBUG_AFTER("k_xent", st);
    ph_end("loss");
    // ---- backward
    for (int j = L - 1; j >= 0; --j) {
        SageLayer& l = s->layers[j];
        const int h = l.hop;
        const int64_t* n_dst = sizes + (h - 1);
        ph_begin();
        {   // dW = a^T dz, the rows split over ~1 CTA per SM
            umma::Args a = gemm_args(l.A16, 2 * l.din, l.dZ16, l.dp, s->grads + l.w_off, l.dout, n_dst, s->gemm_counter);
            a.m_valid = 2 * l.din;
            a.n_valid = l.dp;
            a.n_store = l.dout;
            const int64_t tiles = ((2 * l.din + umma::BM - 1) / umma::BM) * ((l.dout + 255) / 256);
            const int64_t kblocks = (l.n_dst_max + umma::BK - 1) / umma::BK;
            const int splits = (int)std::max<int64_t>(1, std::min<int64_t>(kblocks, 148 / tiles));
            GD_CUDA(umma::launch(umma::DW, a, l.n_dst_max, l.dout, splits, st));
            GD_DEBUG_AFTER("k_umma_gemm<DW>", st);
        }
        const unsigned strips = (unsigned)((l.dout + 31) / 32);
        GD_CUDA(launch_chain(k_colsum_part, dim3(dim3(strips, kColsumChunks)), dim3(rows_blk), 0, st, l.dZ16, l.dout, l.dp, n_dst, s->colsum_part));
        GD_CUDA(launch_chain(k_colsum_final, dim3(strips), dim3(rows_blk), 0, st, s->colsum_part, l.dout, kColsumChunks, s->grads + l.b_off));
        GD_DEBUG_AFTER("k_colsum", st);
        ph_end(kDw[j]);
        if (j == 0) break;
        ph_begin();
        {   // da = dz W^T
            umma::Args a = gemm_args(l.dZ16, l.dp, s->W16 + l.w16_off, l.dp, l.dA, 2 * l.din, n_dst, s->gemm_counter);
            a.k_valid = l.dp;
            a.n_valid = 2 * l.din;
            a.n_store = 2 * l.din;
            GD_CUDA(umma::launch(umma::DA, a, l.n_dst_max, 2 * l.din, 1, st));
            GD_DEBUG_AFTER("k_umma_gemm<DA>", st);
        }
        ph_end(kDa[j]);
        ph_begin();
        GD_CUDA(launch_chain(k_scatter_init, dim3(grid_for(l.n_src_max * 8)), dim3(rows_blk), 0, st, l.dA, l.din, n_dst, sizes + h, l.dX));
        GD_CUDA(launch_chain(k_sage_scatter, dim3(grid_for(l.n_dst_max * 32)), dim3(256), 0, st, l.dA, l.din, rowptr[h - 1], col[h - 1], n_dst, l.dX));
        GD_DEBUG_AFTER("k_sage_scatter", st);
        SageLayer& prev = s->layers[j - 1];   // its output (H16) is this layer's input
        GD_CUDA(launch_chain(k_relu_grad, dim3(grid_for(prev.n_dst_max * 8)), dim3(rows_blk), 0, st, l.dX, prev.H16, prev.dout, prev.dp, sizes + h,
                                                                       prev.n_dst_max, prev.dZ16));
        GD_DEBUG_AFTER("k_relu_grad", st);
        ph_end(kSc[j]);
    }
    GD_CUDA(cudaGetLastError());
    return GD_OK;
}

gd_status gd_sage_grads(gd_sage* s, float** grads, int64_t* count) {
    if (!s || s->hdr.magic != kMagicSage || !grads || !count) return set_error(GD_ERR_INVALID, "gd_sage_grads: bad argument");
    *grads = s->grads;
    *count = s->nparams;
    return GD_OK;
}

gd_status gd_sage_apply_sgd(gd_sage* s, float lr, float grad_scale, void* stream_v) {
    if (!s || s->hdr.magic != kMagicSage) return set_error(GD_ERR_INVALID, "gd_sage_apply_sgd: bad handle");
    DeviceGuard guard(s->hdr.device);
    cudaStream_t st = (cudaStream_t)stream_v;
    GD_CUDA(launch_chain(k_sgd, dim3(grid_for(s->nparams)), dim3(256), 0, st, s->params, s->grads, s->nparams, lr * grad_scale));
    for (const SageLayer& l : s->layers)
        GD_CUDA(launch_chain(k_to_bf16, dim3(grid_for(2 * l.din * l.dp)), dim3(256), 0, st, s->params + l.w_off, s->W16 + l.w16_off, 2 * l.din, l.dout,
                                                              l.dp));
    GD_CUDA(cudaGetLastError());
    return GD_OK;
}

gd_status gd_sage_get(gd_sage* s, int32_t what, int32_t layer, void* host_out, int64_t bytes) {
    if (!s || s->hdr.magic != kMagicSage || !host_out || layer < 0 || layer >= s->L)
        return set_error(GD_ERR_INVALID, "gd_sage_get: bad argument");
    DeviceGuard guard(s->hdr.device);
    const SageLayer& l = s->layers[layer];
    const void* src = nullptr;
    int64_t n = 0;
    switch (what) {
        case GD_SAGE_W: src = s->params + l.w_off; n = (int64_t)2 * l.din * l.dout * 4; break;
        case GD_SAGE_B: src = s->params + l.b_off; n = (int64_t)l.dout * 4; break;
        case GD_SAGE_DW: src = s->grads + l.w_off; n = (int64_t)2 * l.din * l.dout * 4; break;
        case GD_SAGE_DB: src = s->grads + l.b_off; n = (int64_t)l.dout * 4; break;
        case GD_SAGE_A16: src = l.A16; n = l.n_dst_max * 2 * l.din * 2; break;
        case GD_SAGE_Z: src = l.Z; n = l.n_dst_max * l.dout * 4; break;
        case GD_SAGE_H: src = l.H16; n = l.n_dst_max * l.dout * 2; break;
        default: return set_error(GD_ERR_INVALID, "gd_sage_get: unknown item");
    }
    if (!src) return set_error(GD_ERR_INVALID, "gd_sage_get: Z exists for the top layer, H for hidden layers");
    if (bytes < n) return set_error(GD_ERR_INVALID, "gd_sage_get: host buffer too small");
    GD_CUDA(cudaDeviceSynchronize());
    if (what == GD_SAGE_Z || what == GD_SAGE_H) {   // stored at row stride dp
        const size_t e = what == GD_SAGE_Z ? 4 : 2;
        GD_CUDA(cudaMemcpy2D(host_out, (size_t)l.dout * e, src, (size_t)l.dp * e, (size_t)l.dout * e, (size_t)l.n_dst_max,
                             cudaMemcpyDeviceToHost));
    }
    else
        GD_CUDA(cudaMemcpy(host_out, src, (size_t)n, cudaMemcpyDeviceToHost));
    return GD_OK;
}

gd_status gd_debug_umma_gemm(int32_t mode, const void* A, int64_t lda, const void* B, int64_t ldb, void* C, int64_t ldc,
                             int32_t c_bf16, int32_t relu, const float* bias, const int64_t* rows_dev, int64_t rows_max,
                             int64_t m_valid, int32_t k_valid, int32_t n_valid, int32_t n_store, int32_t splits,
                             void* stream) {
    if (mode < 0 || mode > 2 || !A || !B || !C || !rows_dev || n_store < 1 || n_valid < 1 || (mode == 2 && c_bf16))
        return set_error(GD_ERR_INVALID, "gd_debug_umma_gemm: bad argument");
    if ((lda | ldb) & 7 || (k_valid & 7) || (n_valid & 7) || (m_valid & 7) || ((uintptr_t)A | (uintptr_t)B) & 15)
        return set_error(GD_ERR_INVALID, "gd_debug_umma_gemm: strides / extents must be multiples of 8, bases 16-byte aligned");
    cudaStream_t st = (cudaStream_t)stream;
    unsigned int* counter = nullptr;
    GD_CUDA(cudaMallocAsync((void**)&counter, 2 * sizeof(unsigned int), st));
    GD_CUDA(cudaMemsetAsync(counter, 0, 2 * sizeof(unsigned int), st));
    umma::Args a = gemm_args((const __nv_bfloat16*)A, lda, (const __nv_bfloat16*)B, ldb, C, ldc, rows_dev, counter);
    a.c_bf16 = c_bf16;
    a.relu = relu;
    a.bias = bias;
    a.m_valid = m_valid; a.k_valid = k_valid; a.n_valid = n_valid; a.n_store = n_store;
    const cudaError_t e = umma::launch(mode, a, rows_max, n_store, splits, st);
    cudaFreeAsync(counter, st);
    GD_CUDA(e);
    return GD_OK;
}

}  // extern "C"
