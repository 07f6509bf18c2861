// Host-side re-execution of the CUDA library's Philox4x32-10 (curand_Philox4x32_10,
// /usr/local/cuda/include/curand_philox4x32_x.h) — an implementation independent of
// oracle/gd_oracle.cpp, used only to pin the oracle's Philox (pin P1).
// stdin: n records of 6 x uint32 (ctr[4], key[2]); stdout: n records of 4 x uint32.
#define QUALIFIERS static __host__ __device__ inline
#include <curand_philox4x32_x.h>
#include <cstdio>
#include <cstdint>
int main() {
  uint32_t in[6];
  while (fread(in, sizeof(uint32_t), 6, stdin) == 6) {
    uint4 c = make_uint4(in[0], in[1], in[2], in[3]);
    uint2 k = make_uint2(in[4], in[5]);
    uint4 r = curand_Philox4x32_10(c, k);
    uint32_t o[4] = {r.x, r.y, r.z, r.w};
    fwrite(o, sizeof(uint32_t), 4, stdout);
  }
  return 0;
}
