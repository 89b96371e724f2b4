// internal.h — launch structs shared by the CUDA translation units of
// libconvgpu.so (not part of the public ABI; see include/convgpu.h).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "convgpu.h"

namespace convgpu {

constexpr int kReplayThreads = 128;  // warp-per-trace: 4 warps, one trace each at a time
constexpr int kLptThreads = 64;      // lane-per-trace: 2 warps, 64 traces at a time

struct ReplayArgs {
  const uint32_t *arrival, *limit, *delta, *arg;
  uint32_t n, K;
  uint64_t tid_base, seed;
  uint32_t ovh, cap;
  uint64_t count;
  uint32_t* admit_tick;
  uint8_t* admit_rank;
  uint32_t *wait, *finish;
  convgpu_summary_t* summary;
  convgpu_stats_t* stats;
  uint64_t* range_digest;
  uint64_t range_size;
  uint64_t grid_override;  // 0 = occupancy-sized persistent grid
  uint32_t per_sm_cap;     // tuning knob (env CONVGPU_PER_SM_CAP): at most this many CTAs per SM
  uint32_t aligned16;      // all trace arrays and per-container outputs 16-B aligned, n % 4 == 0
  uint32_t aligned32;      // the four trace arrays 32-B aligned and n % 8 == 0 (32-byte loads)
  uint32_t only_marked;    // 0, or a mark: replay only traces with adm_buf()[i*n] == only_marked
  uint32_t* adm_scratch;   // compact kernel: admissions during the replay when admit_tick == NULL
  uint32_t no_wide;        // compact kernel: no 17-bit pass (16-bit host format: limits <= 0xFFFF)

  // where the compact kernel keeps admissions (and its fallback marks)
  __host__ __device__ uint32_t* adm_buf() const { return admit_tick ? admit_tick : adm_scratch; }
};

// admit_tick[i*n] (container 0's admission slot, above every admission
// value) of a trace the compact kernel left to the next pass: the 16-bit
// layout's to the 17-bit one (R1-LIT: to the warp-per-trace kernel), the
// 17-bit layout's to the 32-bit lane kernel
constexpr uint32_t kLpt16Mark = 0xFFFFFFFEu;
constexpr uint32_t kLpt16Mark2 = 0xFFFFFFFDu;

cudaError_t launch_replay(const ReplayArgs& a, int policy, bool bulk, cudaStream_t stream);
cudaError_t launch_replay_lpt(const ReplayArgs& a, int policy, cudaStream_t stream);
bool lpt16_supported(const ReplayArgs& a);
cudaError_t launch_replay_lpt16(const ReplayArgs& a, int policy, cudaStream_t stream,
                                bool wide_first = false);

struct GenArgs {
  convgpu_gen_params_t p;
  uint64_t tid_base, count;
  uint32_t *arrival, *limit, *delta, *arg;
};

cudaError_t launch_generate(const GenArgs& a, cudaStream_t stream);

// pack16.cu: 32-bit SoA <-> compact 16-bit trace format (convgpu_traces16_t)
struct Pack16Args {
  uint64_t count;
  uint32_t n, K;
  // pack: read 32-bit, write 16-bit
  const uint32_t *arrival, *limit, *delta, *arg;
  uint16_t *arrival16, *limit16, *size16, *delta16;
  uint8_t* kinds8;
  unsigned long long* out_of_range;  // values that do not fit (accumulated), or NULL
  // unpack: read 16-bit, write 32-bit
  const uint16_t *r_arrival16, *r_limit16, *r_size16, *r_delta16;
  const uint8_t* r_kinds8;
  uint32_t *w_arrival, *w_limit, *w_delta, *w_arg;
};

cudaError_t launch_pack16(const Pack16Args& a, cudaStream_t stream);
cudaError_t launch_unpack16(const Pack16Args& a, cudaStream_t stream);

cudaError_t launch_wrap(const uint4* api, uint64_t count, uint32_t n, uint32_t K, uint32_t pitch,
                        uint32_t* arg, cudaStream_t stream);

}  // namespace convgpu
