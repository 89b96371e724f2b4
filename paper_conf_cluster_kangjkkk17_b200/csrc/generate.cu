// generate.cu — synthetic workload generator on the device (§8(a) row a0,
// DESIGN.md §Input recipe; P:179 random Table III types every 5 s,
// P:181-187 sizes, durations "from 5 seconds to 45 seconds" by size).
// Counter-based: trace id g, container c -> Philox4x32-10(ctr = (lo g, hi g,
// c, 0), key = gen_seed), so any shard / range regenerates identically.
// One warp per trace; stores are coalesced along c.
#include <cuda_runtime.h>
#include <stdint.h>

#include "common.cuh"
#include "internal.h"

namespace convgpu {

// One warp per trace (grid-stride), lanes over containers: every row of the
// SoA layout is written by consecutive lanes (coalesced), no 64-bit division.
__global__ void __launch_bounds__(256) generate_kernel(const GenArgs a) {
  const uint32_t n = a.p.n_containers, K = a.p.n_ops;
  const uint32_t k0 = (uint32_t)a.p.gen_seed, k1 = (uint32_t)(a.p.gen_seed >> 32);
  const uint32_t lane = threadIdx.x & 31u;
  const uint64_t W = (uint64_t)gridDim.x * (blockDim.x >> 5);
  for (uint64_t i = (uint64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); i < a.count;
       i += W) {
    const uint64_t g = a.tid_base + i;
    for (uint32_t c = lane; c < n; c += 32) {
      const U4 x = philox4x32_10((uint32_t)g, (uint32_t)(g >> 32), c, 0u, k0, k1);
      const uint32_t cls = __umulhi(x.x, a.p.n_classes);
      const uint32_t L = (uint32_t)((uint64_t)a.p.class_mib[cls] * a.p.num / a.p.den);
      const uint32_t jit = (uint32_t)(((uint64_t)x.y * ((uint64_t)a.p.dur_jit + 1ull)) >> 32);
      const uint32_t dur = a.p.dur_base + a.p.dur_step * (cls + a.p.dur_class_offset) + jit;
      const uint32_t e = L > a.p.ctx_overhead_mib ? L - a.p.ctx_overhead_mib : 0u;
      const uint64_t idx = i * n + c;
      a.arrival[idx] = c * a.p.iat;
      a.limit[idx] = L;
      const uint64_t o = i * (uint64_t)K * n + c;
      if (K == 4) {
        const uint32_t s1 = e / 2, d1 = dur / 4, d2 = dur / 2;
        a.delta[o] = 0;                     a.arg[o] = (CONVGPU_OP_ALLOC << 30) | s1;
        a.delta[o + n] = d1;                a.arg[o + n] = (CONVGPU_OP_ALLOC << 30) | (e - s1);
        a.delta[o + 2 * n] = d2;            a.arg[o + 2 * n] = (CONVGPU_OP_FREE << 30) | s1;
        a.delta[o + 3 * n] = dur - d1 - d2; a.arg[o + 3 * n] = (uint32_t)CONVGPU_OP_FINISH << 30;
      } else {
        a.delta[o] = 0;       a.arg[o] = (CONVGPU_OP_ALLOC << 30) | e;
        a.delta[o + n] = dur; a.arg[o + n] = (uint32_t)CONVGPU_OP_FINISH << 30;
      }
    }
  }
}

cudaError_t launch_generate(const GenArgs& a, cudaStream_t stream) {
  int dev = 0, sms = 0;
  cudaError_t e;
  if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
  if ((e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess) return e;
  uint64_t blocks = (a.count + 7) / 8;  // 8 warps (traces) per block
  const uint64_t cap = (uint64_t)sms * 8;
  if (blocks > cap) blocks = cap;
  if (blocks < 1) blocks = 1;
  generate_kernel<<<(unsigned)blocks, 256, 0, stream>>>(a);
  return cudaGetLastError();
}

}  // namespace convgpu
