// common.cuh — device helpers of the CUDA path (sm_100a).  Written
// independently of oracle/ (which has its own C versions); the two sides only
// agree through DESIGN.md and the published KAT vectors.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "convgpu.h"

namespace convgpu {

constexpr uint32_t kFull = 0xFFFFFFFFu;
constexpr uint32_t kKeyNone = 0xFFFFFFFFu;  // "no pending event" key
constexpr uint32_t kSizeMask = 0x3FFFFFFFu;

// Philox4x32-10 (Salmon et al., SC'11).  R6 (Random-Fit draws) and the
// synthetic generator.  mul.hi / mul.lo via __umulhi and 32-bit multiply.
struct U4 {
  uint32_t x, y, z, w;
};

__device__ __forceinline__ U4 philox4x32_10(uint32_t c0, uint32_t c1, uint32_t c2,
                                            uint32_t c3, uint32_t k0, uint32_t k1) {
#pragma unroll
  for (int r = 0; r < 10; ++r) {
    const uint32_t hi0 = __umulhi(0xD2511F53u, c0), lo0 = 0xD2511F53u * c0;
    const uint32_t hi1 = __umulhi(0xCD9E8D57u, c2), lo1 = 0xCD9E8D57u * c2;
    const uint32_t n0 = hi1 ^ c1 ^ k0, n2 = hi0 ^ c3 ^ k1;
    c0 = n0; c1 = lo1; c2 = n2; c3 = lo0;
    k0 += 0x9E3779B9u;
    k1 += 0xBB67AE85u;
  }
  return U4{c0, c1, c2, c3};
}

// splitmix64 finalizer — R20 digest.
__device__ __forceinline__ uint64_t mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

__device__ __forceinline__ uint64_t warp_sum_u64(uint64_t v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(kFull, v, o);
  return v;
}

}  // namespace convgpu
