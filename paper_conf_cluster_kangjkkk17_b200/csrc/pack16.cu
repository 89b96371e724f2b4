// pack16.cu — the compact 16-bit trace format of include/convgpu.h
// (convgpu_traces16_t) to and from the 32-bit SoA layout of convgpu_traces_t.
//
// The host end-to-end path (convgpu_replay_host16) is bound by the PCIe copy
// of the traces (~51 GB/s host-to-device), not by the replay;
// the compact format carries the same traces in 21 B per container instead of
// 40 (n_ops = 4), and unpack16_kernel restores the 32-bit layout on the
// device, next to the replay, at HBM speed.  Pure data movement: no scheduler
// arithmetic (the replay kernels consume the unpacked arrays unchanged).
//
// One thread per (trace, container) column: every SoA row is read and written
// by consecutive threads (coalesced), the K ops of a column in registers.
#include <cuda_runtime.h>
#include <stdint.h>

#include "common.cuh"
#include "internal.h"

namespace convgpu {

__global__ void __launch_bounds__(256) pack16_kernel(const Pack16Args a) {
  const uint64_t cols = a.count * a.n;
  uint32_t bad = 0;
  for (uint64_t x = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; x < cols;
       x += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t i = (cols >> 32) ? x / a.n : (uint64_t)((uint32_t)x / a.n), c = x - i * a.n;
    const uint32_t arr = __ldg(a.arrival + x), L = __ldg(a.limit + x);
    bad += (arr > 0xFFFFu) + (L > 0xFFFFu);
    a.arrival16[x] = (uint16_t)arr;
    a.limit16[x] = (uint16_t)L;
    uint32_t kinds = 0;
    for (uint32_t k = 0; k < a.K; ++k) {
      const uint64_t o = (i * a.K + k) * a.n + c;
      const uint32_t w = __ldg(a.arg + o), d = __ldg(a.delta + o);
      const uint32_t sz = w & kSizeMask;
      bad += (sz > 0xFFFFu) + (d > 0xFFFFu);
      a.size16[o] = (uint16_t)sz;
      a.delta16[o] = (uint16_t)d;
      kinds |= (w >> 30) << (2 * k);
    }
    a.kinds8[x] = (uint8_t)kinds;
  }
  if (a.out_of_range) {
    bad = __reduce_add_sync(kFull, bad);
    if ((threadIdx.x & 31u) == 0 && bad) atomicAdd((unsigned long long*)a.out_of_range, bad);
  }
}

__global__ void __launch_bounds__(256) unpack16_kernel(const Pack16Args a) {
  const uint64_t cols = a.count * a.n;
  for (uint64_t x = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; x < cols;
       x += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t i = (cols >> 32) ? x / a.n : (uint64_t)((uint32_t)x / a.n), c = x - i * a.n;
    a.w_arrival[x] = __ldg(a.r_arrival16 + x);
    a.w_limit[x] = __ldg(a.r_limit16 + x);
    const uint32_t kinds = __ldg(a.r_kinds8 + x);
    for (uint32_t k = 0; k < a.K; ++k) {
      const uint64_t o = (i * a.K + k) * a.n + c;
      a.w_delta[o] = __ldg(a.r_delta16 + o);
      a.w_arg[o] = (((kinds >> (2 * k)) & 3u) << 30) | __ldg(a.r_size16 + o);
    }
  }
}

static unsigned grid_for(uint64_t cols) {
  int dev = 0, sms = 148;
  if (cudaGetDevice(&dev) == cudaSuccess) cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  uint64_t g = (cols + 255) / 256;
  const uint64_t cap = (uint64_t)sms * 8;  // 8 x 256 threads per SM, grid-stride beyond
  if (g > cap) g = cap;
  return (unsigned)(g < 1 ? 1 : g);
}

cudaError_t launch_pack16(const Pack16Args& a, cudaStream_t stream) {
  pack16_kernel<<<grid_for(a.count * a.n), 256, 0, stream>>>(a);
  return cudaGetLastError();
}

cudaError_t launch_unpack16(const Pack16Args& a, cudaStream_t stream) {
  unpack16_kernel<<<grid_for(a.count * a.n), 256, 0, stream>>>(a);
  return cudaGetLastError();
}

}  // namespace convgpu
