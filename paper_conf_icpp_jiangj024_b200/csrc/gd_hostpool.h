// gd_hostpool.h — host worker pool for the staged miss path (see gd_hostpool.cu).
#pragma once

#include <stdint.h>

namespace gd {

class HostGatherPool {
   public:
    explicit HostGatherPool(int threads);
    ~HostGatherPool();
    int threads() const;
    // dst[j*R : (j+1)*R] = src[(rows[j] mod P)*R : ...] for j < n, on all threads; returns elapsed ms.
    // nt = true: non-temporal stores (the destination is read later, from DRAM); false:
    // ordinary stores (the destination is a small cache-resident ring read at once by DMA).
    double gather(const uint8_t* src, const int32_t* rows, int64_t n, int64_t R, uint8_t* dst, int64_t P,
                  bool nt = true);

   private:
    struct Impl;
    Impl* impl_;
};

}  // namespace gd
