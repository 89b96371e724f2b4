// wrap.cu — NEXT-3: the wrapper module's size semantics on the
// device.  The wrapper "calculates adjusted allocate size before checking
// available memory size" for the APIs of Table II
// (P:118-131); this kernel maps API-level program records to the scheduler's
// op words (kind << 30 | MiB), the step just before the replay:
//   cudaMalloc(b)              -> ALLOC ceil(b / 2^20)
//   cudaMallocManaged(b)       -> ALLOC of b rounded up to 128 MiB
//   cudaMallocPitch(w, h)      -> ALLOC of roundup(w, pitch) * h
//   cudaMalloc3D(w, h, d)      -> ALLOC of roundup(w, pitch) * h * d (Table II)
//   cudaFree(op j)             -> FREE of op j's size (the scheduler's hash of
//                                 address -> size); anything but
//                                 an earlier, unfreed allocation -> FREE 2^30-1
//   cudaMemGetInfo / compute   -> NOP (answered from the ledger)
//   __cudaUnregisterFatBinary  -> FINISH
//   unknown code               -> FINISH before the last op, NOP as the last
//                                 (the replay flags BAD_PROGRAM either way)
// DESIGN.md R13' fixes the unit (MiB, rounded up, saturated at 2^30 - 1).
//
// Bandwidth kernel: one thread per (trace, container) column, its K records
// (16 B each) loaded at once with streaming loads (read once), K 4-byte
// stores; consecutive threads take consecutive containers, so every load
// and store instruction of a warp covers contiguous memory.  Persistent
// grid-stride loop, grid = SMs x resident blocks.
#include <cuda_runtime.h>
#include <stdint.h>

#include "internal.h"

namespace convgpu {

namespace {

constexpr uint32_t kSat = 0x3FFFFFFFu;
constexpr unsigned long long kMiB = 1ull << 20;

__device__ __forceinline__ uint32_t to_mib(unsigned long long b) {
  const unsigned long long m = (b >> 20) + ((b & (kMiB - 1)) != 0);
  return m > kSat ? kSat : (uint32_t)m;
}
__device__ __forceinline__ unsigned long long sat_mul(unsigned long long a, unsigned long long b) {
  return __umul64hi(a, b) ? ~0ull : a * b;  // a * b, saturating at 2^64 - 1
}
// roundup(width, pitch) for a 32-bit width: a mask for a power-of-two granule
// (512 on B200), else one 32-bit division; exact in 64 bits either way
__device__ __forceinline__ unsigned long long pitch_of(uint32_t w, uint32_t pitch) {
  if (pitch == 0) return w;
  if ((pitch & (pitch - 1)) == 0)
    return ((unsigned long long)w + pitch - 1) & ~((unsigned long long)pitch - 1);
  const uint32_t q = w / pitch + (w % pitch != 0);
  return (unsigned long long)q * pitch;
}
// MiB charged for an allocation record (0 for any other API), branch-free:
// every candidate size is computed and one is selected, so lanes holding
// different API codes do not diverge.
__device__ __forceinline__ uint32_t alloc_mib(const uint4 r, uint32_t pitch) {
  const unsigned long long b64 = (unsigned long long)r.y | ((unsigned long long)r.z << 32);
  // managed: least multiple of 128 MiB = 2^27 bytes (saturating)
  const unsigned long long q = (b64 >> 27) + ((b64 & ((1ull << 27) - 1)) != 0);
  const unsigned long long managed = (q >> 37) ? ~0ull : (q << 27);
  const unsigned long long p2 = sat_mul(pitch_of(r.y, pitch), r.z);
  const unsigned long long p3 = sat_mul(p2, r.w);
  unsigned long long b = 0;
  b = r.x == CONVGPU_API_MALLOC ? b64 : b;
  b = r.x == CONVGPU_API_MALLOC_MANAGED ? managed : b;
  b = r.x == CONVGPU_API_MALLOC_PITCH ? p2 : b;
  b = r.x == CONVGPU_API_MALLOC_3D ? p3 : b;
  return to_mib(b);
}

// One (trace i, container c) column: K records in, K op words out (selects
// only; the FREE lookup compares against every earlier op).
template <int KF>
__device__ __forceinline__ void wrap_column(uint32_t* __restrict__ arg, uint64_t base, uint32_t n,
                                            uint32_t K, uint32_t pitch,
                                            const uint4 (&r)[KF ? KF : CONVGPU_MAX_OPS]) {
  constexpr int KM = KF ? KF : CONVGPU_MAX_OPS;
  uint32_t mib[KM];
  uint32_t live = 0;  // allocations not yet freed
#pragma unroll
  for (int k = 0; k < KM; ++k) {
    if (k >= (int)K) break;
    const uint32_t a = r[k].x;
    mib[k] = alloc_mib(r[k], pitch);
    const bool is_alloc = a <= CONVGPU_API_MALLOC_3D;
    // FREE: the named allocation, an earlier op of this container, not yet freed
    const uint32_t j = r[k].y;
    const bool hit = a == CONVGPU_API_FREE && j < (uint32_t)k && ((live >> (j & 31u)) & 1u);
    uint32_t fsz = kSat;
#pragma unroll
    for (int q = 0; q < KM; ++q)
      if (q < k) fsz = (hit && j == (uint32_t)q) ? mib[q] : fsz;
    live &= hit ? ~(1u << (j & 31u)) : ~0u;
    live |= is_alloc ? (1u << k) : 0u;
    const uint32_t bad = ((uint32_t)k + 1 < K) ? ((uint32_t)CONVGPU_OP_FINISH << 30)
                                                : ((uint32_t)CONVGPU_OP_NOP << 30);
    uint32_t w = bad;  // unknown code
    w = is_alloc ? (((uint32_t)CONVGPU_OP_ALLOC << 30) | mib[k]) : w;
    w = a == CONVGPU_API_FREE ? (((uint32_t)CONVGPU_OP_FREE << 30) | fsz) : w;
    w = (a == CONVGPU_API_MEM_GET_INFO || a == CONVGPU_API_COMPUTE) ? ((uint32_t)CONVGPU_OP_NOP << 30) : w;
    w = a == CONVGPU_API_EXIT ? ((uint32_t)CONVGPU_OP_FINISH << 30) : w;
    __stcs(arg + base + (uint64_t)k * n, w);
  }
}

// Generic shapes: grid-stride over the count * n columns.
template <int KF>
__global__ void __launch_bounds__(256) wrap_kernel(const uint4* __restrict__ api, uint64_t count,
                                                   uint32_t n, uint32_t K_rt, uint32_t pitch,
                                                   uint32_t* __restrict__ arg) {
  constexpr int KM = KF ? KF : CONVGPU_MAX_OPS;
  const uint32_t K = KF ? (uint32_t)KF : K_rt;
  const uint64_t cols = count * n;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; t < cols; t += stride) {
    const uint64_t i = t / n, c = t - i * n;
    const uint64_t base = i * K * n + c;  // record (i, k, c) at base + k * n
    uint4 r[KM];
#pragma unroll
    for (int k = 0; k < KM; ++k)
      if (k < (int)K) r[k] = __ldcs(api + base + (uint64_t)k * n);
    wrap_column<KF>(arg, base, n, K, pitch, r);
  }
}

// n = 64, K = 4 (the configs): a thread keeps its container c = tid % 64 and
// steps over traces (no division), two traces per iteration so that eight
// 16-byte loads per thread are in flight before any compute.
__global__ void __launch_bounds__(256) wrap_kernel_n64k4(const uint4* __restrict__ api, uint64_t count,
                                                         uint32_t pitch, uint32_t* __restrict__ arg) {
  constexpr uint32_t n = 64, K = 4, TPB = 256 / n;
  const uint32_t c = threadIdx.x % n;
  const uint64_t step = (uint64_t)gridDim.x * TPB;
  uint64_t i = (uint64_t)blockIdx.x * TPB + threadIdx.x / n;
  for (; i + step < count; i += 2 * step) {
    const uint64_t b0 = i * K * n + c, b1 = (i + step) * K * n + c;
    uint4 r0[4], r1[4];
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      r0[k] = __ldcs(api + b0 + (uint64_t)k * n);
      r1[k] = __ldcs(api + b1 + (uint64_t)k * n);
    }
    wrap_column<4>(arg, b0, n, K, pitch, r0);
    wrap_column<4>(arg, b1, n, K, pitch, r1);
  }
  if (i < count) {
    const uint64_t b0 = i * K * n + c;
    uint4 r0[4];
#pragma unroll
    for (int k = 0; k < 4; ++k) r0[k] = __ldcs(api + b0 + (uint64_t)k * n);
    wrap_column<4>(arg, b0, n, K, pitch, r0);
  }
}

}  // namespace

cudaError_t launch_wrap(const uint4* api, uint64_t count, uint32_t n, uint32_t K, uint32_t pitch,
                        uint32_t* arg, cudaStream_t stream) {
  int dev = 0, sms = 0, per_sm = 0;
  cudaError_t e;
  if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
  if ((e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess) return e;
  const bool fast = n == 64 && K == 4;
  const void* kern = fast ? (const void*)wrap_kernel_n64k4
                          : (K == 4 ? (const void*)wrap_kernel<4> : (const void*)wrap_kernel<0>);
  if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, 256, 0)) != cudaSuccess) return e;
  const uint64_t cap = (uint64_t)sms * (per_sm > 0 ? per_sm : 1);
  uint64_t grid = fast ? (count + 3) / 4 : (count * n + 255) / 256;
  if (grid > cap) grid = cap;
  if (grid < 1) grid = 1;
  if (fast)
    wrap_kernel_n64k4<<<(unsigned)grid, 256, 0, stream>>>(api, count, pitch, arg);
  else if (K == 4)
    wrap_kernel<4><<<(unsigned)grid, 256, 0, stream>>>(api, count, n, K, pitch, arg);
  else
    wrap_kernel<0><<<(unsigned)grid, 256, 0, stream>>>(api, count, n, K, pitch, arg);
  return cudaGetLastError();
}

}  // namespace convgpu
