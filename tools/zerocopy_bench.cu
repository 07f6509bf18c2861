// zerocopy_bench.cu — how fast can SMs gather random R-byte rows from pinned host memory?
// Sweeps load flavour (plain / L2::128B / L2::256B hint / cp.async.bulk via TMA),
// unroll, grid size and host allocation (cudaHostAlloc / malloc+register / THP+register).
// Tooling for DESIGN.md §6, not part of the product.
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o zc tools/zerocopy_bench.cu
//   ./zc <table_GB> <row_bytes> <rows_per_launch>
#include <cuda.h>
#include <cuda_runtime.h>
#include <sys/mman.h>
#include <linux/mman.h>

#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <algorithm>
#include <random>
#include <vector>

#define CK(x)                                                                         \
    do {                                                                              \
        cudaError_t e = (x);                                                          \
        if (e != cudaSuccess) {                                                       \
            printf("CUDA %s at %s:%d\n", cudaGetErrorString(e), __FILE__, __LINE__); \
            exit(1);                                                                  \
        }                                                                             \
    } while (0)

template <int MODE>
__device__ __forceinline__ uint4 ld16(const uint4* p) {
    uint4 v;
    if (MODE == 0)
        asm volatile("ld.global.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
    else if (MODE == 1)
        asm volatile("ld.global.L1::no_allocate.L2::128B.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
    else if (MODE == 2)
        asm volatile("ld.global.L1::no_allocate.L2::256B.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
    else
        asm volatile("ld.global.nc.L1::no_allocate.L2::256B.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
    return v;
}

// flat (row, 16B chunk) decomposition, UNROLL chunks in flight per thread
template <int MODE, int UNROLL>
__global__ void k_flat(const int32_t* __restrict__ rows, int64_t n, const uint8_t* __restrict__ src,
                       uint8_t* __restrict__ dst, int64_t R) {
    const int64_t cpr = R >> 4, total = n * cpr, stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; base < total; base += stride * UNROLL) {
        uint4 v[UNROLL];
        int64_t d[UNROLL];
#pragma unroll
        for (int u = 0; u < UNROLL; ++u) {
            const int64_t idx = base + u * stride;
            d[u] = -1;
            if (idx < total) {
                const int64_t r = idx / cpr, c = idx - r * cpr;
                v[u] = ld16<MODE>((const uint4*)(src + (int64_t)__ldg(rows + r) * R) + c);
                d[u] = idx * 16;
            }
        }
#pragma unroll
        for (int u = 0; u < UNROLL; ++u)
            if (d[u] >= 0) *(uint4*)(dst + d[u]) = v[u];
    }
}

// warp per row group: each warp copies ROWS consecutive list entries, all loads first
template <int MODE, int ROWS>
__global__ void k_warp_rows(const int32_t* __restrict__ rows, int64_t n, const uint8_t* __restrict__ src,
                            uint8_t* __restrict__ dst, int64_t R) {
    const int lane = threadIdx.x & 31;
    const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int cpr = (int)(R >> 4);   // assume cpr <= 32 * 4
    for (int64_t r0 = warp * ROWS; r0 < n; r0 += nwarps * ROWS) {
        uint4 v[ROWS][4];
#pragma unroll
        for (int k = 0; k < ROWS; ++k) {
            const int64_t r = r0 + k;
            if (r < n) {
                const uint4* s = (const uint4*)(src + (int64_t)__ldg(rows + r) * R);
#pragma unroll
                for (int q = 0; q < 4; ++q)
                    if (lane + 32 * q < cpr) v[k][q] = ld16<MODE>(s + lane + 32 * q);
            }
        }
#pragma unroll
        for (int k = 0; k < ROWS; ++k) {
            const int64_t r = r0 + k;
            if (r < n) {
                uint4* d = (uint4*)(dst + r * R);
#pragma unroll
                for (int q = 0; q < 4; ++q)
                    if (lane + 32 * q < cpr) d[lane + 32 * q] = v[k][q];
            }
        }
    }
}

// TMA bulk (cp.async.bulk global -> shared), one row per bulk op, STAGES rows in flight per warp
template <int STAGES>
__global__ void k_bulk(const int32_t* __restrict__ rows, int64_t n, const uint8_t* __restrict__ src,
                       uint8_t* __restrict__ dst, int64_t R) {
    extern __shared__ __align__(128) uint8_t smem[];
    __shared__ __align__(8) uint64_t bar[8][STAGES];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    uint8_t* buf = smem + (size_t)w * STAGES * R;
    if (lane == 0)
        for (int s = 0; s < STAGES; ++s) {
            uint32_t a = (uint32_t)__cvta_generic_to_shared(&bar[w][s]);
            asm volatile("mbarrier.init.shared.b64 [%0], 1;" ::"r"(a));
        }
    asm volatile("fence.mbarrier_init.release.cluster;");
    __syncwarp();
    uint32_t phase[STAGES] = {0};
    int64_t r = gw;
    // prologue
    for (int s = 0; s < STAGES; ++s) {
        const int64_t rr = gw + (int64_t)s * nw;
        if (lane == 0 && rr < n) {
            uint32_t b = (uint32_t)__cvta_generic_to_shared(&bar[w][s]);
            uint32_t d = (uint32_t)__cvta_generic_to_shared(buf + s * R);
            asm volatile("mbarrier.arrive.expect_tx.shared.b64 _, [%0], %1;" ::"r"(b), "r"((uint32_t)R));
            asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                         ::"r"(d), "l"(src + (int64_t)__ldg(rows + rr) * R), "r"((uint32_t)R), "r"(b) : "memory");
        }
    }
    int s = 0;
    for (; r < n; r += nw) {
        uint32_t b = (uint32_t)__cvta_generic_to_shared(&bar[w][s]);
        asm volatile("{ .reg .pred p; W: mbarrier.try_wait.parity.shared.b64 p, [%0], %1; @!p bra W; }" ::"r"(b), "r"(phase[s]));
        phase[s] ^= 1;
        const uint4* sv = (const uint4*)(buf + s * R);
        uint4* d = (uint4*)(dst + r * R);
        for (int q = lane; q < (int)(R >> 4); q += 32) d[q] = sv[q];
        __syncwarp();
        const int64_t rn = r + (int64_t)STAGES * nw;
        if (lane == 0 && rn < n) {
            uint32_t dd = (uint32_t)__cvta_generic_to_shared(buf + s * R);
            asm volatile("mbarrier.arrive.expect_tx.shared.b64 _, [%0], %1;" ::"r"(b), "r"((uint32_t)R));
            asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                         ::"r"(dd), "l"(src + (int64_t)__ldg(rows + rn) * R), "r"((uint32_t)R), "r"(b) : "memory");
        }
        s = (s + 1) % STAGES;
    }
}

template <typename F>
float timeit(F f, int reps = 5) {
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    float best = 1e30f;
    f();
    CK(cudaDeviceSynchronize());
    for (int i = 0; i < reps; ++i) {
        cudaEventRecord(a);
        f();
        cudaEventRecord(b);
        CK(cudaEventSynchronize(b));
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        if (ms < best) best = ms;
    }
    return best;
}

int main(int argc, char** argv) {
    const double GB = argc > 1 ? atof(argv[1]) : 16;
    const int64_t R = argc > 2 ? atoll(argv[2]) : 512;
    const int64_t n = argc > 3 ? atoll(argv[3]) : 200000;
    const int64_t N = (int64_t)(GB * 1e9) / R;
    const size_t bytes = (size_t)N * R;
    std::vector<int32_t> rows(n);
    std::mt19937_64 rng(7);
    for (auto& r : rows) r = (int32_t)(rng() % N);
    int32_t* d_rows;
    uint8_t* d_dst;
    CK(cudaMalloc(&d_rows, n * 4));
    CK(cudaMalloc(&d_dst, n * R));
    CK(cudaMemcpy(d_rows, rows.data(), n * 4, cudaMemcpyHostToDevice));
    // sorted variant
    std::vector<int32_t> srt = rows;
    std::sort(srt.begin(), srt.end());
    int32_t* d_srt;
    CK(cudaMalloc(&d_srt, n * 4));
    CK(cudaMemcpy(d_srt, srt.data(), n * 4, cudaMemcpyHostToDevice));

    // H2D memcpy reference
    {
        uint8_t* h;
        CK(cudaHostAlloc(&h, 1 << 30, cudaHostAllocDefault));
        memset(h, 1, 1 << 30);
        uint8_t* d;
        CK(cudaMalloc(&d, 1 << 30));
        float ms = timeit([&] { cudaMemcpyAsync(d, h, 1 << 30, cudaMemcpyHostToDevice); });
        printf("memcpy H2D 1GiB: %.1f GB/s\n", (1 << 30) / ms / 1e6);
        cudaFree(d);
        cudaFreeHost(h);
    }
    const double mb = (double)n * R;
    if (getenv("ZC_QUICK")) {   // one allocation, random vs contiguous rows, flat kernel
        uint8_t* h = nullptr;
        uint8_t* src = nullptr;
        const int am = getenv("ZC_ALLOC") ? atoi(getenv("ZC_ALLOC")) : 0;
        size_t abytes = bytes;
        if (am == 0) {
            CK(cudaHostAlloc(&h, bytes, cudaHostAllocMapped | cudaHostAllocPortable));
        } else if (am == 3 || am == 5) {   // hugetlbfs 2MB / 1GB pages
            const size_t pg = am == 3 ? (2ull << 20) : (1ull << 30);
            abytes = (bytes + pg - 1) / pg * pg;
            h = (uint8_t*)mmap(nullptr, abytes, PROT_READ | PROT_WRITE,
                               MAP_PRIVATE | MAP_ANONYMOUS | MAP_HUGETLB | (am == 3 ? MAP_HUGE_2MB : MAP_HUGE_1GB), -1, 0);
            if (h == MAP_FAILED) { printf("hugetlb mmap failed (mode %d)\n", am); return 0; }
            memset(h, 3, abytes);
            CK(cudaHostRegister(h, abytes, cudaHostRegisterMapped | cudaHostRegisterPortable));
        } else if (am == 4) {              // driver VMM allocation on the host NUMA node
            cuInit(0);
            CUmemAllocationProp prop = {};
            prop.type = CU_MEM_ALLOCATION_TYPE_PINNED;
            prop.location.type = CU_MEM_LOCATION_TYPE_HOST_NUMA;
            prop.location.id = 0;
            size_t gran = 0;
            CUresult r = cuMemGetAllocationGranularity(&gran, &prop, CU_MEM_ALLOC_GRANULARITY_RECOMMENDED);
            printf("vmm host granularity %zu (r=%d)\n", gran, (int)r);
            abytes = (bytes + gran - 1) / gran * gran;
            CUmemGenericAllocationHandle hd;
            r = cuMemCreate(&hd, abytes, &prop, 0);
            if (r != CUDA_SUCCESS) { printf("cuMemCreate host failed %d\n", (int)r); return 0; }
            CUdeviceptr va;
            r = cuMemAddressReserve(&va, abytes, gran, 0, 0);
            r = cuMemMap(va, abytes, 0, hd, 0);
            CUmemAccessDesc ad[2] = {};
            ad[0].location.type = CU_MEM_LOCATION_TYPE_DEVICE; ad[0].location.id = 0; ad[0].flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
            ad[1].location.type = CU_MEM_LOCATION_TYPE_HOST_NUMA; ad[1].location.id = 0; ad[1].flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
            r = cuMemSetAccess(va, abytes, ad, 2);
            printf("vmm map/access r=%d\n", (int)r);
            h = (uint8_t*)va;
        } else {
            h = (uint8_t*)mmap(nullptr, bytes, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
            madvise(h, bytes, MADV_HUGEPAGE);
            memset(h, 3, bytes);
            CK(cudaHostRegister(h, bytes, cudaHostRegisterMapped | cudaHostRegisterPortable));
        }
        if (am == 0 || am == 4) memset(h, 3, bytes);
        if (am == 4) src = h;
        else CK(cudaHostGetDevicePointer((void**)&src, h, 0));
        std::vector<int32_t> seq(n);
        for (int64_t i = 0; i < n; ++i) seq[i] = (int32_t)(i % N);
        int32_t* d_seq;
        CK(cudaMalloc(&d_seq, n * 4));
        CK(cudaMemcpy(d_seq, seq.data(), n * 4, cudaMemcpyHostToDevice));
        if (getenv("ZC_SMS")) {   // few whole-SM blocks (1024 threads)
            for (int G : {2, 4, 8, 12, 16, 24, 32, 48}) {
                float a1 = timeit([&] { k_flat<0, 4><<<G, 1024>>>(d_rows, n, src, d_dst, R); });
                float a2 = timeit([&] { k_flat<0, 8><<<G, 1024>>>(d_rows, n, src, d_dst, R); });
                float c1 = timeit([&] { k_flat<0, 4><<<G, 1024>>>(d_seq, n, src, d_dst, R); });
                float c2 = timeit([&] { k_flat<0, 8><<<G, 1024>>>(d_seq, n, src, d_dst, R); });
                printf("SMs=%2d x1024thr: random u4 %.1f u8 %.1f | contiguous u4 %.1f u8 %.1f GB/s\n", G, mb / a1 / 1e6,
                       mb / a2 / 1e6, mb / c1 / 1e6, mb / c2 / 1e6);
            }
            return 0;
        }
        float a = timeit([&] { k_flat<0, 4><<<296, 256>>>(d_rows, n, src, d_dst, R); });
        float b = timeit([&] { k_flat<0, 4><<<296, 256>>>(d_srt, n, src, d_dst, R); });
        float c = timeit([&] { k_flat<0, 4><<<296, 256>>>(d_seq, n, src, d_dst, R); });
        float c2 = timeit([&] { k_flat<0, 8><<<1184, 256>>>(d_seq, n, src, d_dst, R); });
        printf("alloc %d table %.1f GB R=%lld n=%lld: random %.1f  sorted %.1f  contiguous %.1f / %.1f GB/s\n", am, bytes / 1e9,
               (long long)R, (long long)n, mb / a / 1e6, mb / b / 1e6, mb / c / 1e6, mb / c2 / 1e6);
        return 0;
    }
    for (int mode_alloc = 0; mode_alloc < 3; ++mode_alloc) {
        uint8_t* h = nullptr;
        const char* an[] = {"cudaHostAlloc", "malloc+register", "THP mmap+register"};
        if (mode_alloc == 0) {
            CK(cudaHostAlloc(&h, bytes, cudaHostAllocMapped | cudaHostAllocPortable));
            memset(h, 3, bytes);
        } else if (mode_alloc == 1) {
            h = (uint8_t*)malloc(bytes);
            memset(h, 3, bytes);
            CK(cudaHostRegister(h, bytes, cudaHostRegisterMapped | cudaHostRegisterPortable));
        } else {
            h = (uint8_t*)mmap(nullptr, bytes, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
            if (h == MAP_FAILED) { printf("mmap failed\n"); continue; }
            int mr = madvise(h, bytes, MADV_HUGEPAGE);
            memset(h, 3, bytes);
            CK(cudaHostRegister(h, bytes, cudaHostRegisterMapped | cudaHostRegisterPortable));
            printf("(madvise rc=%d)\n", mr);
        }
        uint8_t* src;
        CK(cudaHostGetDevicePointer((void**)&src, h, 0));
        printf("== %s, table %.1f GB, R=%lld, rows=%lld\n", an[mode_alloc], bytes / 1e9, (long long)R, (long long)n);
#define RUNF(MODE, U, G, T, ROWS_PTR, NAME)                                                            \
    {                                                                                                  \
        float ms = timeit([&] { k_flat<MODE, U><<<G, T>>>(ROWS_PTR, n, src, d_dst, R); });             \
        CK(cudaGetLastError());                                                                        \
        printf("  flat mode=%d unroll=%d grid=%d thr=%d %s: %.1f GB/s\n", MODE, U, G, T, NAME, mb / ms / 1e6); \
    }
        for (int G : {148, 296, 592, 1184}) {
            RUNF(0, 4, G, 256, d_rows, "rand");
            RUNF(2, 4, G, 256, d_rows, "rand");
        }
        RUNF(0, 1, 148, 256, d_rows, "rand");
        RUNF(0, 2, 148, 256, d_rows, "rand");
        RUNF(0, 8, 148, 256, d_rows, "rand");
        RUNF(1, 4, 296, 256, d_rows, "rand");
        RUNF(3, 4, 296, 256, d_rows, "rand");
        RUNF(0, 4, 296, 256, d_srt, "sorted");
        RUNF(2, 4, 296, 256, d_srt, "sorted");
#define RUNW(MODE, ROWS, G, T)                                                                         \
    {                                                                                                  \
        float ms = timeit([&] { k_warp_rows<MODE, ROWS><<<G, T>>>(d_rows, n, src, d_dst, R); });       \
        CK(cudaGetLastError());                                                                        \
        printf("  warp_rows mode=%d rows=%d grid=%d thr=%d: %.1f GB/s\n", MODE, ROWS, G, T, mb / ms / 1e6); \
    }
        RUNW(0, 1, 296, 256);
        RUNW(0, 2, 296, 256);
        RUNW(0, 4, 296, 256);
        RUNW(2, 2, 296, 256);
        RUNW(2, 4, 148, 256);
        RUNW(2, 4, 296, 128);
#define RUNB(ST, G, T)                                                                                 \
    {                                                                                                  \
        size_t sm = (size_t)(T / 32) * ST * R;                                                         \
        cudaFuncSetAttribute(k_bulk<ST>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);        \
        float ms = timeit([&] { k_bulk<ST><<<G, T, sm>>>(d_rows, n, src, d_dst, R); });                \
        cudaError_t e = cudaGetLastError();                                                            \
        printf("  bulk stages=%d grid=%d thr=%d: %.1f GB/s (%s)\n", ST, G, T, mb / ms / 1e6, cudaGetErrorString(e)); \
    }
        RUNB(4, 148, 256);
        RUNB(8, 148, 256);
        RUNB(8, 296, 128);
        RUNB(16, 148, 256);
        if (mode_alloc == 0) cudaFreeHost(h);
        else {
            cudaHostUnregister(h);
            if (mode_alloc == 1) free(h);
            else munmap(h, bytes);
        }
    }
    return 0;
}
