// gd_api.cu — host plumbing shared by the C ABI: thread-local errors, pointer
// classification, scan-state allocation, sticky device status.
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>

#include "gd_common.cuh"
#include "gd_handles.cuh"

namespace gd {

static thread_local std::string g_last_error;

gd_status set_error(gd_status s, const std::string& msg) {
    g_last_error = msg;
    return s;
}

gd_status cuda_error(cudaError_t e, const char* what) {
    std::string m = std::string(what) + ": " + cudaGetErrorString(e);
    cudaGetLastError();   // clear non-sticky errors
    return set_error(e == cudaErrorMemoryAllocation ? GD_ERR_OOM : GD_ERR_CUDA, m);
}

bool debug_kernels() {
    static const bool on = [] {
        const char* e = std::getenv("GD_DEBUG_KERNELS");
        return e && e[0] == '1';
    }();
    return on;
}

void debug_after(const char* what, cudaStream_t s) {
    cudaError_t e = cudaStreamSynchronize(s);
    std::fprintf(stderr, "[gd] %s -> %s\n", what, cudaGetErrorString(e));
    std::fflush(stderr);
}

bool is_device_pointer(const void* p) {
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

bool pdl_enabled() {
    static const bool on = [] {
        const char* e = std::getenv("GD_PDL");
        return !(e && e[0] == '0');
    }();
    return on;
}

const void* mapped_host_pointer(const void* p) {
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();
        return nullptr;
    }
    return a.type == cudaMemoryTypeHost ? a.devicePointer : nullptr;
}

gd_status ScanState::ensure(int64_t tiles) {
    if (tiles <= cap) return GD_OK;
    int64_t ncap = 1024;
    while (ncap < tiles) ncap *= 2;
    release();
    unsigned long long* b = nullptr;
    GD_CUDA(cudaMalloc(&b, 2 * ncap * sizeof(unsigned long long)));
    GD_CUDA(cudaMemset(b, 0, 2 * ncap * sizeof(unsigned long long)));
    buf[0] = b;
    buf[1] = b + ncap;
    cap = ncap;
    parity = 0;
    dirty[0] = dirty[1] = 0;
    return GD_OK;
}

void ScanState::release() {
    if (buf[0]) cudaFree(buf[0]);
    buf[0] = buf[1] = nullptr;
    cap = 0;
}

}  // namespace gd

extern "C" {

const char* gd_last_error(void) { return gd::g_last_error.c_str(); }

int gd_version(void) { return 10000; }

gd_status gd_check_device_status(void* handle, uint32_t* bits) {
    if (!handle) return gd::set_error(GD_ERR_INVALID, "gd_check_device_status: null handle");
    gd::HandleHdr* h = (gd::HandleHdr*)handle;
    if (h->magic != gd::kMagicGraph && h->magic != gd::kMagicBuffer)
        return gd::set_error(GD_ERR_INVALID, "gd_check_device_status: not a gd handle");
    gd::DeviceGuard guard(h->device);
    GD_CUDA(cudaDeviceSynchronize());
    unsigned int v = 0;
    GD_CUDA(cudaMemcpy(&v, h->dev_status, sizeof(v), cudaMemcpyDeviceToHost));
    if (bits) *bits = v;
    if (v) {
        char msg[160];
        std::snprintf(msg, sizeof(msg), "device-side check tripped: bits=0x%x (%s%s%s%s)", v,
                      (v & GD_DEV_BAD_ID) ? "bad-id " : "", (v & GD_DEV_DUP_SEED) ? "dup-seed " : "",
                      (v & GD_DEV_UNDERFLOW) ? "refcount-underflow " : "",
                      (v & GD_DEV_STANDBY_DRY) ? "standby-dry" : "");
        return gd::set_error(GD_ERR_DEVICE, msg);
    }
    return GD_OK;
}

}  // extern "C"
