// gather_bench.cu — HBM row gather out[i] = src[idx[i]] (R-byte rows): LDG/STG v4 with
// unroll U vs TMA bulk copies (cp.async.bulk global->shared, shared->global).  Tooling.
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o gb tools/gather_bench.cu
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <random>
#include <vector>

#define CK(x)                                                                              \
    do {                                                                                   \
        cudaError_t e = (x);                                                               \
        if (e != cudaSuccess) { printf("CUDA %s line %d\n", cudaGetErrorString(e), __LINE__); return 1; } \
    } while (0)

template <int U>
__global__ void __launch_bounds__(256) k_ldg(const int2* __restrict__ hl, int64_t H, const uint8_t* __restrict__ src,
                                             uint8_t* __restrict__ out, int64_t R) {
    const int64_t cpr = R >> 4, total = H * cpr, stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; base < total; base += stride * U) {
        uint4 v[U];
        int64_t d[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t idx = base + u * stride;
            d[u] = -1;
            if (idx < total) {
                const int64_t r = idx / cpr, c = idx - r * cpr;
                const int2 h = __ldg(hl + r);
                asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                             : "=r"(v[u].x), "=r"(v[u].y), "=r"(v[u].z), "=r"(v[u].w)
                             : "l"((const uint4*)(src + (int64_t)h.y * R) + c));
                d[u] = (int64_t)h.x * R + c * 16;
            }
        }
#pragma unroll
        for (int u = 0; u < U; ++u)
            if (d[u] >= 0) *(uint4*)(out + d[u]) = v[u];
    }
}

// warp-per-row variant: lane covers 16B chunks of one row, U rows per warp in flight
template <int U>
__global__ void __launch_bounds__(256) k_warp(const int2* __restrict__ hl, int64_t H, const uint8_t* __restrict__ src,
                                              uint8_t* __restrict__ out, int64_t R) {
    const int lane = threadIdx.x & 31;
    const int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int cpr = (int)(R >> 4);
    for (int64_t r0 = w * U; r0 < H; r0 += nw * U) {
        uint4 v[U][2];
        int2 h[U];
#pragma unroll
        for (int u = 0; u < U; ++u) h[u] = (r0 + u < H) ? __ldg(hl + r0 + u) : make_int2(-1, -1);
#pragma unroll
        for (int u = 0; u < U; ++u)
#pragma unroll
            for (int q = 0; q < 2; ++q)
                if (h[u].x >= 0 && lane + 32 * q < cpr)
                    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                                 : "=r"(v[u][q].x), "=r"(v[u][q].y), "=r"(v[u][q].z), "=r"(v[u][q].w)
                                 : "l"((const uint4*)(src + (int64_t)h[u].y * R) + lane + 32 * q));
#pragma unroll
        for (int u = 0; u < U; ++u)
#pragma unroll
            for (int q = 0; q < 2; ++q)
                if (h[u].x >= 0 && lane + 32 * q < cpr) ((uint4*)(out + (int64_t)h[u].x * R))[lane + 32 * q] = v[u][q];
    }
}

// TMA bulk: each thread owns a pipeline of ST smem row buffers
template <int ST>
__global__ void __launch_bounds__(128) k_tma(const int2* __restrict__ hl, int64_t H, const uint8_t* __restrict__ src,
                                             uint8_t* __restrict__ out, int64_t R) {
    extern __shared__ __align__(128) uint8_t smem[];
    __shared__ __align__(8) uint64_t bar[128 * ST];
    const int t = threadIdx.x;
    const int64_t gt = (int64_t)blockIdx.x * blockDim.x + t, nt = (int64_t)gridDim.x * blockDim.x;
    uint8_t* buf = smem + (size_t)t * ST * R;
    for (int s = 0; s < ST; ++s) {
        uint32_t a = (uint32_t)__cvta_generic_to_shared(&bar[t * ST + s]);
        asm volatile("mbarrier.init.shared.b64 [%0], 1;" ::"r"(a));
    }
    asm volatile("fence.mbarrier_init.release.cluster;");
    uint32_t ph = 0;   // phase bits per stage
    auto issue = [&](int s, int64_t r) {
        const int2 h = __ldg(hl + r);
        uint32_t b = (uint32_t)__cvta_generic_to_shared(&bar[t * ST + s]);
        uint32_t d = (uint32_t)__cvta_generic_to_shared(buf + s * R);
        asm volatile("mbarrier.arrive.expect_tx.shared.b64 _, [%0], %1;" ::"r"(b), "r"((uint32_t)R));
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                     ::"r"(d), "l"(src + (int64_t)h.y * R), "r"((uint32_t)R), "r"(b) : "memory");
    };
    int64_t r = gt;
    for (int s = 0; s < ST; ++s)
        if (r + s * nt < H) issue(s, r + s * nt);
    int s = 0;
    for (; r < H; r += nt) {
        uint32_t b = (uint32_t)__cvta_generic_to_shared(&bar[t * ST + s]);
        const uint32_t p = (ph >> s) & 1;
        asm volatile("{ .reg .pred q; W: mbarrier.try_wait.parity.shared.b64 q, [%0], %1; @!q bra W; }" ::"r"(b), "r"(p));
        ph ^= (1u << s);
        const int2 h = __ldg(hl + r);
        uint32_t d = (uint32_t)__cvta_generic_to_shared(buf + s * R);
        asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(out + (int64_t)h.x * R), "r"(d),
                     "r"((uint32_t)R) : "memory");
        asm volatile("cp.async.bulk.commit_group;");
        const int64_t rn = r + (int64_t)ST * nt;
        if (rn < H) {
            asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(ST - 1) : "memory");  // oldest store read smem
            asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
            issue(s, rn);
        }
        s = (s + 1) % ST;
    }
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

template <typename F>
float timeit(F f) {
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    float best = 1e30f;
    f();
    cudaDeviceSynchronize();
    for (int i = 0; i < 10; ++i) {
        cudaEventRecord(a);
        f();
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        best = std::min(best, ms);
    }
    return best;
}

int main() {
    const int64_t S = 11100000, R = 512, H = 337000;
    uint8_t *src, *out;
    int2* hl;
    CK(cudaMalloc(&src, S * R));
    CK(cudaMalloc(&out, 1000000 * R));
    CK(cudaMemset(src, 1, S * R));
    std::vector<int2> h(H);
    std::mt19937_64 g(3);
    std::vector<int> pos(1000000);
    for (int i = 0; i < 1000000; ++i) pos[i] = i;
    std::shuffle(pos.begin(), pos.end(), g);
    std::sort(pos.begin(), pos.begin() + H);
    for (int64_t i = 0; i < H; ++i) h[i] = make_int2(pos[i], (int)(g() % S));
    CK(cudaMalloc(&hl, H * sizeof(int2)));
    CK(cudaMemcpy(hl, h.data(), H * sizeof(int2), cudaMemcpyHostToDevice));
    // flush L2 buffer
    uint8_t* fl;
    CK(cudaMalloc(&fl, 256 << 20));
    const double bytes = 2.0 * H * R;
    auto rep = [&](const char* name, auto launch) {
        float ms = timeit([&] { cudaMemsetAsync(fl, 0, 256 << 20); launch(); });
        float m0 = timeit([&] { cudaMemsetAsync(fl, 0, 256 << 20); });
        cudaError_t e = cudaGetLastError();
        printf("%-28s %.1f us  %.0f GB/s (%s)\n", name, (ms - m0) * 1e3, bytes / ((ms - m0) * 1e6), cudaGetErrorString(e));
    };
    rep("ldg u4 g1184x256", [&] { k_ldg<4><<<1184, 256>>>(hl, H, src, out, R); });
    rep("ldg u8 g1184x256", [&] { k_ldg<8><<<1184, 256>>>(hl, H, src, out, R); });
    rep("ldg u4 g2368x256", [&] { k_ldg<4><<<2368, 256>>>(hl, H, src, out, R); });
    rep("ldg u2 g4736x256", [&] { k_ldg<2><<<4736, 256>>>(hl, H, src, out, R); });
    rep("warp u2 g1184x256", [&] { k_warp<2><<<1184, 256>>>(hl, H, src, out, R); });
    rep("warp u4 g1184x256", [&] { k_warp<4><<<1184, 256>>>(hl, H, src, out, R); });
    rep("warp u4 g592x256", [&] { k_warp<4><<<592, 256>>>(hl, H, src, out, R); });
    rep("warp u8 g592x256", [&] { k_warp<8><<<592, 256>>>(hl, H, src, out, R); });
    rep("warp u8 g1184x256", [&] { k_warp<8><<<1184, 256>>>(hl, H, src, out, R); });
    rep("warp u4 g2368x256", [&] { k_warp<4><<<2368, 256>>>(hl, H, src, out, R); });
    rep("warp u2 g2368x256", [&] { k_warp<2><<<2368, 256>>>(hl, H, src, out, R); });
    for (int st : {2, 4}) {
        for (int G : {148, 296, 592}) {
            size_t sm = (size_t)128 * st * R;
            if (st == 2) cudaFuncSetAttribute(k_tma<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
            else cudaFuncSetAttribute(k_tma<4>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
            char nm[64];
            snprintf(nm, 64, "tma st%d g%dx128", st, G);
            if (st == 2) rep(nm, [&] { k_tma<2><<<G, 128, sm>>>(hl, H, src, out, R); });
            else rep(nm, [&] { k_tma<4><<<G, 128, sm>>>(hl, H, src, out, R); });
        }
    }
    return 0;
}
