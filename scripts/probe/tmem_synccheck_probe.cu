#include <cstdio>
#include <cstdint>
__device__ __forceinline__ uint32_t sa(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
template <int MODE>
__global__ void k(uint32_t* out) {
  __shared__ uint32_t s_tmem;
  const uint32_t wib = threadIdx.x >> 5;
  if (wib == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(sa(&s_tmem)), "r"(128u) : "memory");
    if (MODE != 1) asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  uint32_t t = s_tmem;
  uint32_t v = threadIdx.x * 7, r = 0;
  if (MODE != 2) {
    asm volatile("tcgen05.st.sync.aligned.32x32b.x1.b32 [%0], {%1};" ::"r"(t + ((32u * (wib & 3)) << 16)), "r"(v) : "memory");
    asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x1.b32 {%0}, [%1];" : "=r"(r) : "r"(t + ((32u * (wib & 3)) << 16)) : "memory");
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = r;
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  if (wib == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(t), "r"(128u) : "memory");
}
int main() {
  uint32_t* d; cudaMalloc(&d, 4 * 1024 * 4);
  k<0><<<4, 32>>>(d); printf("m0 %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
  k<0><<<4, 128>>>(d); printf("m0b %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
  k<1><<<4, 32>>>(d); printf("m1 %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
  k<2><<<4, 32>>>(d); printf("m2 %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
  uint32_t h[32]; cudaMemcpy(h, d, 128, cudaMemcpyDeviceToHost); printf("h[5]=%u\n", h[5]);
}
