// replay_lpt16.cu — lane-per-trace replay of ConVGPU's GPU-memory scheduler
// (§III-D, Fig. 3) with COMPACT per-container
// state, so that two warps per scheduler (8 per SM) fit in shared memory.
//
// Same algorithm and the same branch-free micro-step structure as
// replay_lpt.cu; what differs is the state layout:
//  * 14 bytes per container instead of 24 (n = 64: 896 B per trace, 28 KB per
//    warp): key (u32), ust (u32: used 16 | op index 2 | FIRST | PAUSED |
//    ADMITTED | op kinds 2 x K), sd (u32: size of the current op, saturated
//    to 16 bits | delta of the next op 16), L (u16, [container][lane]);
//  * no admission word: an admission is stored straight to admit_tick, or to
//    the caller's admission scratch when admit_tick is not requested (as
//    tick << 6 | rank), and read back by the epilogue; the finish tick lives
//    in the container's key after FINISH (0x80000000 | tick) and a paused
//    container's key is 0xC0000000 (Recent-Fit: | the next container down the
//    suspension stack, which is thereby a linked list needing no extra
//    memory), both above every event key (ticks < 2^25 here);
//  * Best-Fit keeps the trace's distinct limits (at most 8, sorted) and one
//    64-bit member mask per limit in registers (no shared-memory tables, so
//    it runs 8 warps per SM too); traces with more distinct limits are left
//    to the fallback pass;
//  * arrival + sum of deltas of every container (for R17's wait) is parked
//    in the thread's tensor-memory lane between init and epilogue (16 at a
//    time: init and epilogue run converged for every lane of the warp);
//  * init reads the trace and the epilogue its admissions with 32-byte loads
//    (LDG.256, one whole DRAM sector of the lane's own row per instruction)
//    and writes the outputs with 32-byte streaming stores, when the arrays
//    are 32-B aligned (else 16-byte operations);
//  * under R1-LIT (policy | CONVGPU_DISPATCH_LITERAL, NEXT-1) each
//    container's partial assignment is a u16 at [container][lane] (7 warps
//    per SM) and the fallback pass is the warp-per-trace kernel;
//  * an arrival whose first op has delta 0 is applied together with that op
//    in one step (see the EVENT step);
//  * the one-op-ahead fetch (raw op word + next delta, cp.async) lands in a
//    2-word staging slot and is packed into the container's sd word at the
//    end of the NEXT iteration, so the copy has a whole iteration to land
//    (a register destination would make the compiler wait for it at the loop
//    head); an event of the container fetched in the previous iteration
//    (rare) waits one iteration, until the retire has landed its op.
// A trace qualifies when every limit is <= 0xFFFE MiB, every delta <= 0xFFFF
// ticks and its horizon (R19) < 2^25 (BASELINE configs [1]-[3] and [4] up to
// rho = 7 do; the 16-bit fields are then exact: a saturated size is above
// every limit, so it is rejected / flagged exactly as the full size would
// be).  Other traces are marked (admissions[trace][0] = kLpt16Mark) and
// replayed by a second launch of this kernel with 17-bit limits / used memory
// (WIDE, R1; exact while every ALLOC / FREE size is <= 0xFFFE), which marks
// what it cannot hold (kLpt16Mark2) for a third, 32-bit lane-per-trace
// launch; each launch skips unmarked traces.
// Semantics are identical to replay_lpt.cu / replay.cu; every
// GPU parity test runs this kernel against the oracle too.
#include <cuda_runtime.h>
#include <stdint.h>

#include "common.cuh"
#include "internal.h"
#include "lpt_util.cuh"

namespace convgpu {
namespace lpt16 {

using lpt::ffs64;
using lpt::shl_c;
using lpt::sts_if;

constexpr uint32_t N = 64, KOPS = 4;  // compile-time shape (configs [2]-[4])
// ust word: used (16 bits; WIDE: 17) | op index 2 (K = 4: 0..3, FINISH is op
// 3) | FIRST | PAUSED | ADMITTED | op kinds 2 x K | WIDE: bit 16 of the
// declared limit, whose bits 0-15 are in the u16 limit array
#ifndef LPT16_V8
#define LPT16_V8 1
#endif
template <bool WIDE>
struct Lay {
  static constexpr uint32_t kUsedBits = WIDE ? 17u : 16u;
  static constexpr uint32_t kUsedMask = (1u << kUsedBits) - 1u;
  static constexpr uint32_t kKShift = kUsedBits;
  static constexpr uint32_t kFirst = 1u << (kUsedBits + 2);
  static constexpr uint32_t kPaused = 1u << (kUsedBits + 3);
  static constexpr uint32_t kAdmitted = 1u << (kUsedBits + 4);
  static constexpr uint32_t kKindShift = kUsedBits + 5;
  static constexpr uint32_t kLimHi = WIDE ? 1u << 31 : 0u;
};
// keys
constexpr uint32_t kDone = 0x80000000u;    // | finish tick
constexpr uint32_t kPausedKey = 0xC0000000u;  // | suspension number
constexpr uint32_t kNoC = 64u;
constexpr uint32_t kTickLimit = CONVGPU_TICK_LIMIT;
constexpr uint32_t kCompactHorizon = 1u << 25;
constexpr uint32_t kStopMask = ~(uint32_t)CONVGPU_FLAG_OVERCOMMIT;
// TMEM per warp: 64 columns of per-container sums + 32 of statistics
// accumulators (20 used); warps w and w + 4 share a lane quarter
constexpr uint32_t kTmemCols = 256;
constexpr uint32_t kWarpCols = 128;
 // 64 per warp, warps w and w + 4 share a lane quarter

// bytes per lane (= per trace) and warps per CTA (one CTA per SM)
// policy may carry CONVGPU_DISPATCH_LITERAL (R1-LIT, NEXT-1): several
// containers then hold partial assignments, kept as u16 per container
__host__ __device__ constexpr bool is_lit(int policy) {
  return (policy & CONVGPU_DISPATCH_LITERAL) != 0;
}
__host__ __device__ constexpr uint32_t extra_bytes(int policy) {
  return is_lit(policy) ? N * 2u : 0u;  // R1: every policy's extra state lives in registers
}
__host__ __device__ constexpr uint32_t lane_bytes(int policy) {
  return N * 14u + extra_bytes(policy) + 8u;  // + 2-word fetch staging slot
}
__host__ __device__ constexpr int warps_per_cta(int policy) {
  return is_lit(policy) ? 7 : 8;  // 1,032 B per trace under R1-LIT
}
// Best-Fit keeps the trace's distinct declared limits ("classes") in
// registers; a trace with more distinct limits than this is left to the
// 32-bit kernel (marked), like one whose values exceed the 16-bit fields.
constexpr int kBfClasses = 8;

__device__ __forceinline__ uint32_t comp(const uint4& v, int j) {
  return j == 0 ? v.x : (j == 1 ? v.y : (j == 2 ? v.z : v.w));
}
__device__ __forceinline__ void stg_if(uint32_t* p, uint32_t v, bool on) {
  asm volatile("{ .reg .pred q; setp.ne.u32 q, %2, 0; @q st.global.u32 [%0], %1; }"
               ::"l"(p), "r"(v), "r"((uint32_t)on) : "memory");
}
__device__ __forceinline__ uint32_t pack_sd(uint32_t cw, uint32_t d) {
  return min(cw & kSizeMask, 0xFFFFu) | (d << 16);
}

// WIDE: the second pass over the traces the 16-bit layout could not hold
// (marked kLpt16Mark by the first): 17-bit limits and used memory; traces it
// cannot hold either are re-marked kLpt16Mark2 for the 32-bit kernel.
template <int POLICY, bool WIDE>
__global__ void __launch_bounds__(32 * warps_per_cta(POLICY), 1) replay_lpt16_kernel(const ReplayArgs p) {
  extern __shared__ __align__(16) uint32_t smem_w[];
  using Ly = Lay<WIDE>;
  constexpr uint32_t kUsedMask = Ly::kUsedMask, kKShift = Ly::kKShift, kKOne = 1u << kKShift;
  constexpr uint32_t kFirst = Ly::kFirst, kPaused = Ly::kPaused, kAdmitted = Ly::kAdmitted;
  constexpr uint32_t kNotArrived = kPaused | kAdmitted;
  constexpr uint32_t kKindShift = Ly::kKindShift, kKindsMask = 0xFFu << kKindShift;
  constexpr uint32_t kLimHi = Ly::kLimHi;
  // the declared limit of a container whose ust word is u
#define FULL_L(c, u) (WIDE ? (uint32_t)LIM(c) | (((u) >> 31) << 16) : (uint32_t)LIM(c))
  constexpr bool LIT = is_lit(POLICY);     // R1-LIT (NEXT-1) instead of R1
  constexpr int P = POLICY & 0xFF;         // convgpu_policy_t
  const uint32_t lane = threadIdx.x & 31u, wib = threadIdx.x >> 5;
  constexpr uint32_t n = N, K = KOPS;
  const uint32_t cap = p.cap, ovh = p.ovh;
  uint32_t* const W0 = smem_w + wib * (32u * lane_bytes(POLICY) / 4u);
  // word w of container c of this lane at W0[(w*n + c)*32 + lane]; limits as
  // u16 pairs (containers 2j, 2j+1 in word j); then the policy's extra state
  uint32_t* const s_key = W0 + lane;
  uint32_t* const s_ust = W0 + 1 * n * 32 + lane;
  uint32_t* const s_sd = W0 + 2 * n * 32 + lane;
  // limits: u16 of container c of this lane at [c * 32 + lane] (one IMAD per
  // address; at most 2-way bank conflicts, between lanes 2j and 2j + 1)
  uint16_t* const s_L = reinterpret_cast<uint16_t*>(W0 + 3 * n * 32) + lane;
  // staging slot of the one-op-ahead fetch: {op word, delta of the op after}
  // R1-LIT: assignment a of container c (u16, at most its limit), [c][lane]
  uint16_t* const s_A = reinterpret_cast<uint16_t*>(W0 + (3 * n + n / 2) * 32) + lane;
  uint32_t* const s_stg = W0 + (3 * n + n / 2 + extra_bytes(POLICY) / 4) * 32 + lane;
#define AT(arr, c) (arr)[(c) * 32u]
#define LIM(c) s_L[(c) * 32u]
#define ASG(c) s_A[(c) * 32u]

  // A warp replays 32 consecutive traces per round; round-robin warp slots
  // run SM-first (slot = wib * gridDim + block), so the last, partial round
  // spreads over every SM instead of filling the first CTAs.
  const uint64_t T = (uint64_t)gridDim.x * blockDim.x;
  // only_marked (the WIDE pass): the next trace from j on whose container-0
  // admission slot holds the mark (8 markers probed per step, all in flight)
  auto next = [&](uint64_t j) -> uint64_t {
    if (!WIDE || !p.only_marked) return j;
    while (j < p.count) {
      uint32_t m[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const uint64_t jj = j + (uint64_t)u * T;
        m[u] = jj < p.count ? p.adm_buf()[jj * N] : 0u;
      }
#pragma unroll
      for (int u = 0; u < 8; ++u)
        if (m[u] == p.only_marked) return j + (uint64_t)u * T;
      j += 8 * T;
    }
    return j;
  };
  uint64_t i = next(((uint64_t)wib * gridDim.x + blockIdx.x) * 32u + lane);

  unsigned long long st_traces = 0, st_events = 0, st_mk = 0, st_wait = 0, st_rej = 0,
                     st_sel = 0, st_dig = 0;
  uint32_t st_maxmk = 0, st_maxpk = 0;
  unsigned long long racc_r = ~0ull, racc = 0;

  uint32_t gmin[8];
  // arrival + sum of deltas per container (R17's wait = finish - base is then
  // computed without re-reading the trace in the epilogue).  Computed in
  // registers by init, parked in this thread's TMEM lane for the whole event
  // loop (64 columns), read back for the epilogue: the loop does not carry 64
  // registers for it.  The thread's statistics accumulators (only touched by
  // the epilogue) are parked the same way (20 more columns).
  __shared__ uint32_t s_tmem;
  if (wib == 0) lpt::tmem_alloc(&s_tmem, kTmemCols);
  lpt::tmem_fence_before_sync();
  __syncthreads();
  lpt::tmem_fence_after_sync();
  const uint32_t t_base = s_tmem + ((32u * (wib & 3u)) << 16) + (wib >> 2) * kWarpCols;
  // init parks the sums 16 containers at a time and the epilogue loads them
  // the same way (both run converged, for every lane of the warp), so at
  // most 16 of them are ever live in registers
  auto park_state = [&]() {  // whole warp, converged
    __syncwarp();
    uint32_t sr[32];
    const unsigned long long u[9] = {st_traces, st_events, st_mk, st_wait, st_rej, st_sel, st_dig,
                                     racc_r, racc};
#pragma unroll
    for (int j = 0; j < 9; ++j) { sr[2 * j] = (uint32_t)u[j]; sr[2 * j + 1] = (uint32_t)(u[j] >> 32); }
    sr[18] = st_maxmk; sr[19] = st_maxpk;
#pragma unroll
    for (int j = 20; j < 32; ++j) sr[j] = 0;
    lpt::tmem_st16(t_base + 64u, sr);
    lpt::tmem_st16(t_base + 80u, sr + 16);
  };
  auto fetch_state = [&]() {  // whole warp, converged
    __syncwarp();
    lpt::tmem_wait_st();
    uint32_t sr[32];
    lpt::tmem_ld16(t_base + 64u, sr);
    lpt::tmem_ld16(t_base + 80u, sr + 16);
    lpt::tmem_wait_ld();
    auto u64 = [&](int j) { return (unsigned long long)sr[2 * j] | ((unsigned long long)sr[2 * j + 1] << 32); };
    st_traces = u64(0); st_events = u64(1); st_mk = u64(2); st_wait = u64(3); st_rej = u64(4);
    st_sel = u64(5); st_dig = u64(6); racc_r = u64(7); racc = u64(8);
    st_maxmk = sr[18]; st_maxpk = sr[19];
  };
  uint32_t arr0 = 0;
  // Best-Fit (R3, R4): the trace's distinct limits in ascending order (unused
  // slots 0xFFFFFFFF, above every free amount) and, per class, the mask of
  // containers declaring that limit.  A paused non-target container has no
  // memory assigned (R1: only the fill target is ever partial), so its
  // shortfall is its limit: the Best-Fit choice is the lowest-index paused
  // member of the highest class whose limit fits the free memory, else of
  // the lowest class with a paused member.
  uint32_t bl[kBfClasses], bm_lo[kBfClasses], bm_hi[kBfClasses];
  uint32_t free_mem = 0, target = kNoC, a_tg = 0, used_total = 0, rank = 0, draws = 0,
           n_rej = 0, n_sel = 0, peak_res = 0, peak_used = 0, flags = 0, live = 0, events = 0;
  uint32_t pm_lo = 0, pm_hi = 0;
  uint32_t ru_head = kNoC;        // Recent-Fit: top of the suspension stack (linked
                                  // through the paused containers' keys)
  // the op fetched in the previous iteration: container, op word, delta
  uint32_t pre_c = kNoC;
  bool skip = false;
#ifdef LPT16_DEBUG
  uint32_t dbg0 = 0, dbg1 = 0, dbg2 = 0, dbg3 = 0, dbg4 = 0;
#endif
#ifdef LPT16_COUNT  // experiment only: micro-step counters in the summary
  uint32_t cnt_ev = 0, cnt_ds = 0, cnt_hz = 0, cnt_it = 0;
#endif
  const uint32_t* trace_delta = nullptr;
  const uint32_t* trace_arg = nullptr;
  uint32_t* adm_out = nullptr;

  auto regroup = [&](uint32_t c) {
    const uint32_t g = c >> 3, b = g << 3;
    uint32_t v[8];
#pragma unroll
    for (uint32_t j = 0; j < 8; ++j) v[j] = AT(s_key, b + j);
    const uint32_t m =
        min(min(min(v[0], v[1]), min(v[2], v[3])), min(min(v[4], v[5]), min(v[6], v[7])));
#pragma unroll
    for (uint32_t j = 0; j < 8; ++j) gmin[j] = (j == g) ? m : gmin[j];
  };

  // Called by every lane of the warp (converged: it parks to TMEM); a lane
  // without a trace (act = false) replays trace 0's loads with no global side
  // effect and its state is never used.
  auto init = [&](uint64_t ti, bool act) {
    uint32_t base[16];
    const uint4* A4 = reinterpret_cast<const uint4*>(p.arrival + ti * n);
    const uint4* L4 = reinterpret_cast<const uint4*>(p.limit + ti * n);
    trace_delta = p.delta + ti * (uint64_t)K * n;
    trace_arg = p.arg + ti * (uint64_t)K * n;
    adm_out = p.adm_buf() + ti * n;
    const uint4* D4 = reinterpret_cast<const uint4*>(trace_delta);
    const uint4* R4 = reinterpret_cast<const uint4*>(trace_arg);
    uint32_t bad = 0, lsum = 0, amax = 0, prev = 0, lmax = 0, dmax = 0, smax = 0;
#pragma unroll
    for (int j = 0; j < 8; ++j) gmin[j] = kKeyNone;
    // two-stage software pipeline: the loads of containers 4q+4..4q+7 are in
    // flight while 4q..4q+3 are processed (one warp's 32 traces are 32
    // separate rows per load)
    uint4 a4b[2], l4b[2], d4b[2][4], w4b[2][4];
    auto ld_q = [&](uint32_t q, int s) {
      a4b[s] = lpt::ldg4_cg(A4 + q);
      l4b[s] = lpt::ldg4_cg(L4 + q);
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        d4b[s][k] = lpt::ldg4_cg(D4 + k * 16 + q);
        w4b[s][k] = lpt::ldg4_cg(R4 + k * 16 + q);
      }
    };
    // one container's values: validation, derived state, shared-memory words
    auto proc = [&](uint32_t c, uint32_t a, uint32_t L, const uint32_t (&d)[4], const uint32_t (&w)[4]) {
      if (L > cap) bad |= CONVGPU_FLAG_INVALID_LIMIT;
      if (c > 0 && a < prev) bad |= CONVGPU_FLAG_UNSORTED_ARRIVAL;
      prev = a;
      amax = max(amax, a);
      lmax = max(lmax, L);
      uint32_t kinds = 0, bsum = a;
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        bsum += d[k];
        lsum = min(lsum + min(d[k], kTickLimit), kTickLimit);
        dmax = max(dmax, d[k]);
        if (((w[k] >> 30) == CONVGPU_OP_FINISH) != (k == 3)) bad |= CONVGPU_FLAG_BAD_PROGRAM;
        if (WIDE && ((w[k] >> 30) == CONVGPU_OP_ALLOC || (w[k] >> 30) == CONVGPU_OP_FREE))
          smax = max(smax, w[k] & kSizeMask);
        kinds |= (w[k] >> 30) << (2 * k);
      }
      const uint32_t key = (min(a, kTickLimit - 1) << 6) | c;
      AT(s_key, c) = key;
      AT(s_ust, c) = kNotArrived | (kinds << kKindShift) | min(d[0], 0xFFFFu) |
                     (WIDE ? ((L >> 16) & 1u) << 31 : 0u);
      AT(s_sd, c) = pack_sd(w[0], min(d[1], 0xFFFFu));
      LIM(c) = (uint16_t)(WIDE ? L : min(L, 0xFFFFu));  // WIDE: bit 16 in the ust word
      if (LIT) ASG(c) = 0;
      gmin[c >> 3] = min(gmin[c >> 3], key);
      base[c & 15] = bsum;
      if (c == 0) arr0 = a;
    };
    if (LPT16_V8 && p.aligned32) {
    // 32-byte loads (LDG.256: one full sector per lane), 8 containers a step
    // (the four trace arrays 32-B aligned; warp-uniform)
#pragma unroll
    for (uint32_t q = 0; q < 8; ++q) {
      uint32_t av[8], lv[8], dv[4][8], wv[4][8];
      lpt::ldg8_cg(av, p.arrival + ti * n + 8 * q);
      lpt::ldg8_cg(lv, p.limit + ti * n + 8 * q);
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        lpt::ldg8_cg(dv[k], trace_delta + k * n + 8 * q);
        lpt::ldg8_cg(wv[k], trace_arg + k * n + 8 * q);
      }
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        const uint32_t d[4] = {dv[0][j], dv[1][j], dv[2][j], dv[3][j]};
        const uint32_t w[4] = {wv[0][j], wv[1][j], wv[2][j], wv[3][j]};
        proc(8 * q + j, av[j], lv[j], d, w);
      }
      if ((q & 1) == 1) {  // park 16 sums (R17's wait) in this thread's TMEM lane
        __syncwarp();
        lpt::tmem_st16(t_base + 8u * (q & ~1u), base);
      }
    }
    } else {
    ld_q(0, 0);
#pragma unroll
    for (uint32_t q = 0; q < 16; ++q) {
      if (q + 1 < 16) ld_q(q + 1, (q + 1) & 1);
      const uint4 a4 = a4b[q & 1], l4 = l4b[q & 1];
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const uint32_t d[4] = {comp(d4b[q & 1][0], j), comp(d4b[q & 1][1], j), comp(d4b[q & 1][2], j),
                               comp(d4b[q & 1][3], j)};
        const uint32_t w[4] = {comp(w4b[q & 1][0], j), comp(w4b[q & 1][1], j), comp(w4b[q & 1][2], j),
                               comp(w4b[q & 1][3], j)};
        proc(4 * q + j, comp(a4, j), comp(l4, j), d, w);
      }
      if ((q & 3) == 3) {  // park 16 sums (R17's wait) in this thread's TMEM lane
        __syncwarp();
        lpt::tmem_st16(t_base + 4u * (q & ~3u), base);
      }
    }
    }
    if (amax >= kTickLimit || amax + lsum >= kTickLimit) bad |= CONVGPU_FLAG_TICK_RANGE;
    // not representable in the 16-bit fields: the 32-bit kernel replays it
    // Op sizes are saturated at 0xFFFF, which is exact while every limit is
    // <= 0xFFFE (a saturated size is above every limit, so rejected or
    // flagged as the full size would be).  WIDE: limits and used memory have
    // 17 bits and the sizes must fit exactly.
    const bool lim_ok = WIDE ? (lmax <= 0x1FFFFu && smax <= 0xFFFEu) : lmax <= 0xFFFEu;
    skip = bad == 0 && (!lim_ok || dmax > 0xFFFFu || amax + lsum >= kCompactHorizon);
    // container 0's slot doubles as the fallback mark; clear a stale mark a
    // previous call may have left in caller scratch (admissions of container
    // 0 are only read back when it was admitted, so 0 is harmless)
    if (act) adm_out[0] = skip ? (WIDE ? kLpt16Mark2 : kLpt16Mark) : 0u;
    if (P == CONVGPU_BEST_FIT && !LIT) {
      // distinct limits (unsorted while collected), with member masks
      uint32_t ncls = 0;
#pragma unroll
      for (int j = 0; j < kBfClasses; ++j) { bl[j] = 0xFFFFFFFFu; bm_lo[j] = 0; bm_hi[j] = 0; }
#pragma unroll
      for (int c = 0; c < 64; ++c) {
        const uint32_t Lc = FULL_L(c, AT(s_ust, c)), bit = 1u << (c & 31);
        bool hit = false;
#pragma unroll
        for (int j = 0; j < kBfClasses; ++j) {
          const bool e = bl[j] == Lc;
          hit |= e;
          if (c < 32) bm_lo[j] |= e ? bit : 0u; else bm_hi[j] |= e ? bit : 0u;
        }
        if (!hit) {  // a new class (at most kBfClasses + 1 times per trace)
#pragma unroll
          for (int j = 0; j < kBfClasses; ++j) {
            const bool e = (uint32_t)j == ncls;
            bl[j] = e ? Lc : bl[j];
            if (c < 32) bm_lo[j] |= e ? bit : 0u; else bm_hi[j] |= e ? bit : 0u;
          }
          ++ncls;
        }
      }
      // sort the classes by limit (Batcher's network for 8 keys, 19 exchanges)
#define BF_CE(a, b)                                                              \
  {                                                                              \
    const bool sw = bl[a] > bl[b];                                               \
    const uint32_t x = bl[a], y = bm_lo[a], z = bm_hi[a];                        \
    bl[a] = sw ? bl[b] : x; bm_lo[a] = sw ? bm_lo[b] : y; bm_hi[a] = sw ? bm_hi[b] : z; \
    bl[b] = sw ? x : bl[b]; bm_lo[b] = sw ? y : bm_lo[b]; bm_hi[b] = sw ? z : bm_hi[b]; \
  }
      BF_CE(0, 1) BF_CE(2, 3) BF_CE(4, 5) BF_CE(6, 7)
      BF_CE(0, 2) BF_CE(1, 3) BF_CE(4, 6) BF_CE(5, 7)
      BF_CE(1, 2) BF_CE(5, 6) BF_CE(0, 4) BF_CE(3, 7)
      BF_CE(1, 5) BF_CE(2, 6)
      BF_CE(1, 4) BF_CE(3, 6)
      BF_CE(2, 4) BF_CE(3, 5)
      BF_CE(3, 4)
#undef BF_CE
      // more distinct limits than classes: the 32-bit kernel replays it
      if (bad == 0 && ncls > (uint32_t)kBfClasses && !skip) {
        skip = true;
        if (act) adm_out[0] = WIDE ? kLpt16Mark2 : kLpt16Mark;
      }
    }
    flags = bad;
    free_mem = cap; target = kNoC; a_tg = 0; used_total = 0; rank = 0; draws = 0;
    n_rej = 0; n_sel = 0; peak_res = 0; peak_used = 0; live = n; events = 0;
    pm_lo = pm_hi = 0;
    pre_c = kNoC;
    ru_head = kNoC;
  };

  // Called by every lane of the warp (converged: it loads from TMEM); only
  // lanes with act = true store or count anything.
  auto epilogue = [&](uint64_t ti, bool act) {
    lpt::cp_wait0();
    uint32_t base[16];
    const bool stopped = (flags & kStopMask) != 0;
    if (stopped) { peak_res = 0; peak_used = 0; n_rej = 0; n_sel = 0; }
    uint64_t dig = 0, swait = 0;
    uint32_t mfin = 0;
    const uint64_t ob = ti * n;
    // one container's outputs and its digest terms
    auto epi_c = [&](uint32_t c, uint32_t adm, uint32_t bs, uint32_t& at, uint32_t& ar, uint32_t& wt,
                     uint32_t& fn) {
      at = kKeyNone; ar = 0xFFu; wt = 0; fn = 0;
      if (!stopped) {
        if (AT(s_ust, c) & kAdmitted) {
          at = adm >> 6;
          ar = adm & 63u;
        }
        fn = AT(s_key, c) & ~kDone;
        wt = fn - bs;  // R17: wait = finish - arrival - sum of deltas
      }
      const uint64_t h1 = mix64(((uint64_t)c << 56) ^ ((uint64_t)ar << 48) ^ (uint64_t)at);
      dig += mix64(h1 ^ (((uint64_t)wt << 32) | fn));
      mfin = max(mfin, fn);
      swait += wt;
    };
    if (LPT16_V8 && p.aligned32) {
      // 32-byte admission loads (all in flight) and 32-byte streaming stores
      uint32_t m8[8][8];
#pragma unroll
      for (uint32_t g = 0; g < 8; ++g) lpt::ldg8_cg(m8[g], adm_out + 8 * g);
#pragma unroll
      for (uint32_t g = 0; g < 8; ++g) {
        if ((g & 1) == 0) {  // the next 16 parked sums
          __syncwarp();
          lpt::tmem_ld16(t_base + 8u * g, base);
          lpt::tmem_wait_ld();
        }
        uint32_t at[8], ar[8], wt[8], fn[8];
#pragma unroll
        for (int j = 0; j < 8; ++j)
          epi_c(8 * g + j, m8[g][j], base[(8 * g + j) & 15], at[j], ar[j], wt[j], fn[j]);
        if (act && p.admit_tick) lpt::stg8_cs(p.admit_tick + ob + 8 * g, at);
        if (act && p.admit_rank)
          lpt::stg2_cs(p.admit_rank + ob + 8 * g, ar[0] | (ar[1] << 8) | (ar[2] << 16) | (ar[3] << 24),
                       ar[4] | (ar[5] << 8) | (ar[6] << 16) | (ar[7] << 24));
        if (act && p.wait) lpt::stg8_cs(p.wait + ob + 8 * g, wt);
        if (act && p.finish) lpt::stg8_cs(p.finish + ob + 8 * g, fn);
      }
    } else {
    const uint4* M4 = reinterpret_cast<const uint4*>(adm_out);
    // all 16 admission loads in flight at once (this thread stored them during
    // the replay: read at L2), then the parked sums
    uint4 m4a[16];
#pragma unroll
    for (uint32_t q = 0; q < 16; ++q) m4a[q] = lpt::ldg4_cg(M4 + q);
#pragma unroll
    for (uint32_t q = 0; q < 16; ++q) {
      if ((q & 3) == 0) {  // the next 16 parked sums
        __syncwarp();
        lpt::tmem_ld16(t_base + 4u * q, base);
        lpt::tmem_wait_ld();
      }
      // admissions this thread stored during the replay (coherent load)
      const uint4 m4 = stopped ? make_uint4(0, 0, 0, 0) : m4a[q];
      uint32_t at[4], ar[4], wt[4], fn[4];
#pragma unroll
      for (int j = 0; j < 4; ++j) epi_c(4 * q + j, comp(m4, j), base[(4 * q + j) & 15], at[j], ar[j], wt[j], fn[j]);
      // streaming stores (evict-first): outputs are not re-read, inputs of the
      // traces in flight should stay in L2
      if (act && p.admit_tick)
        __stcs(reinterpret_cast<uint4*>(p.admit_tick + ob) + q, make_uint4(at[0], at[1], at[2], at[3]));
      if (act && p.admit_rank)
        __stcs(reinterpret_cast<unsigned int*>(p.admit_rank + ob) + q,
               ar[0] | (ar[1] << 8) | (ar[2] << 16) | (ar[3] << 24));
      if (act && p.wait)
        __stcs(reinterpret_cast<uint4*>(p.wait + ob) + q, make_uint4(wt[0], wt[1], wt[2], wt[3]));
      if (act && p.finish)
        __stcs(reinterpret_cast<uint4*>(p.finish + ob) + q, make_uint4(fn[0], fn[1], fn[2], fn[3]));
    }
    }
    const uint32_t makespan = stopped ? 0u : mfin - arr0;
    dig += mix64(((uint64_t)makespan << 32) | peak_res);
    dig += mix64(((uint64_t)peak_used << 32) | flags);
    dig += mix64(swait);
    dig += mix64(((uint64_t)n_rej << 32) | n_sel);
    if (!act) return;
    if (p.summary) {
      convgpu_summary_t sm;
      sm.makespan = makespan; sm.peak_reserved = peak_res; sm.peak_used = peak_used;
      sm.flags = flags; sm.sum_wait = swait; sm.n_rejected = n_rej; sm.n_select = n_sel;
      sm.digest = dig;
#ifdef LPT16_DEBUG
      if (flags & CONVGPU_FLAG_INVALID_FREE) {
        sm.makespan = dbg0; sm.peak_reserved = dbg1; sm.peak_used = dbg2; sm.n_rejected = dbg3;
        sm.n_select = dbg4; sm.sum_wait = events;
      }
#endif
#ifdef LPT16_COUNT
      sm.makespan = cnt_ev; sm.peak_reserved = cnt_ds; sm.peak_used = cnt_hz; sm.n_rejected = cnt_it;
      cnt_ev = cnt_ds = cnt_hz = cnt_it = 0;
#endif
      p.summary[ti] = sm;
    }
    st_traces += 1; st_events += events; st_mk += makespan; st_wait += swait; st_rej += n_rej;
    st_sel += n_sel; st_dig += dig;
    st_maxmk = max(st_maxmk, makespan);
    st_maxpk = max(st_maxpk, peak_res);
    if (flags && p.stats)
      for (int b = 0; b < 8; ++b)
        if ((flags >> b) & 1u) atomicAdd(&p.stats->flag_count[b], 1u);
    if (p.range_digest) {
      const unsigned long long r = (p.tid_base + ti) / p.range_size;
      if (r != racc_r) {
        if (racc_r != ~0ull) atomicAdd((unsigned long long*)&p.range_digest[racc_r], racc);
        racc_r = r;
        racc = 0;
      }
      racc += dig;
    }
  };

  // SELECT (R3-R7): a new fill target when there is none (FIFO:
  // computed unconditionally, taken by lanes with `on`)
  auto select_target = [&](bool on) {
    if (P == CONVGPU_FIFO) {
      const bool ns = on && target == kNoC;  // (always under R1-LIT: no sticky target)
      const uint32_t sel = ffs64(pm_lo, pm_hi);
      target = ns ? sel : target;
      a_tg = ns ? (LIT ? (uint32_t)ASG(sel & 63u) : 0u) : a_tg;  // R1-LIT: its partial hold
      n_sel += ns ? 1u : 0u;
    } else if (on && target == kNoC) {
      uint32_t sel;
      if (P == CONVGPU_BEST_FIT && LIT) {  // R3, R4 with partial holds: shortfall L - a
        uint32_t best = kNoC, bneed = 0, mn = kNoC, mneed = 0xFFFFFFFFu;
        uint32_t wl = pm_lo, wh = pm_hi;
        while (wl | wh) {  // ascending index: strict comparisons keep the lowest
          const uint32_t c = ffs64(wl, wh);
          wl &= ~shl_c(1u, c);
          wh &= ~shl_c(1u, c - 32u);
          const uint32_t need = (uint32_t)LIM(c) - (uint32_t)ASG(c);
          const bool f = need <= free_mem && (best == kNoC || need > bneed);
          best = f ? c : best;
          bneed = f ? need : bneed;
          const bool m = need < mneed;
          mn = m ? c : mn;
          mneed = m ? need : mneed;
        }
        sel = best != kNoC ? best : mn;
      } else if (P == CONVGPU_BEST_FIT) {  // R3, R4 (classes: see bl above)
        // ascending classes: the last fitting class with a paused
        // member wins; descending: the last class with one is the lowest
        uint32_t fl = 0, fh = 0, ml = 0, mh = 0;
#pragma unroll
        for (int j = 0; j < kBfClasses; ++j) {
          const uint32_t a = pm_lo & bm_lo[j], b = pm_hi & bm_hi[j];
          const bool on = ((a | b) != 0u) && bl[j] <= free_mem;
          fl = on ? a : fl;
          fh = on ? b : fh;
        }
#pragma unroll
        for (int j = kBfClasses - 1; j >= 0; --j) {
          const uint32_t a = pm_lo & bm_lo[j], b = pm_hi & bm_hi[j];
          const bool on = (a | b) != 0u;
          ml = on ? a : ml;
          mh = on ? b : mh;
        }
        const bool fit = (fl | fh) != 0u;
        sel = ffs64(fit ? fl : ml, fit ? fh : mh);
      } else if (P == CONVGPU_RECENT_FIT) {  // R5
        // pop the suspension stack: paused containers leave the paused
        // set only by resuming, and only the target resumes, so popping
        // at selection keeps the stack exactly the paused set in
        // suspension order.  R1-LIT: the selected container may stay
        // paused (partially filled), so it is popped when it resumes
        sel = ru_head;
        if (!LIT) ru_head = AT(s_key, sel) & 127u;
      } else {  // RANDOM_FIT (R6)
        const uint64_t tid = p.tid_base + i;
        const uint32_t clo = __popc(pm_lo), m = clo + __popc(pm_hi);
        const U4 x = philox4x32_10((uint32_t)tid, (uint32_t)(tid >> 32), draws, 1u,
                                   (uint32_t)p.seed, (uint32_t)(p.seed >> 32));
        ++draws;
        const uint32_t jj = __umulhi(x.x, m);
        sel = lpt::nth_set64(pm_lo, pm_hi, jj);
      }
      target = sel;
      a_tg = LIT ? (uint32_t)ASG(sel) : 0u;  // R1-LIT: its partial hold
      ++n_sel;
    }
  };

  bool have = i < p.count, tdone = false, dmode = false;
  uint32_t cur_t = 0;
#ifdef LPT16_NOLOOP  // experiment: init + epilogue only
#define LPT16_TD true
#else
#define LPT16_TD (flags != 0 || skip)
#endif
  if (__any_sync(kFull, have)) { init(have ? i : 0, have); tdone = LPT16_TD; }
  park_state();
  while (__any_sync(kFull, have)) {
    do {
      if (have && !tdone) {
        uint32_t kc = kNoC, nkc = kKeyNone, pfk = 0xFFu;
        // next event (a2).  If it belongs to the container whose next op was
        // fetched in the previous iteration (rare), this lane idles for one
        // iteration: the tail below retires that fetch into the container's
        // sd word, so the event block never handles an op still in flight.
        const uint32_t m01 = min(gmin[0], gmin[1]), m23 = min(gmin[2], gmin[3]);
        const uint32_t m45 = min(gmin[4], gmin[5]), m67 = min(gmin[6], gmin[7]);
        const uint32_t kmin = min(min(m01, m23), min(m45, m67));
        const bool hz = (kmin & 63u) == pre_c && kmin < kDone;
#ifdef LPT16_COUNT
        cnt_it++; cnt_ev += (!dmode && !hz) ? 1u : 0u; cnt_ds += dmode ? 1u : 0u; cnt_hz += (!dmode && hz) ? 1u : 0u;
#endif
        if (!dmode && !hz) {
          // ================= EVENT step (a2 + a3), branch-free =================
          if (kmin >= kDone) {
            if (live) flags |= CONVGPU_FLAG_DEADLOCK;  // P:7
            tdone = true;
          } else {
            const uint32_t t = kmin >> 6, c = kmin & 63u;
            cur_t = t;
            ++events;
            const uint32_t ust = AT(s_ust, c), sd = AT(s_sd, c), L = FULL_L(c, ust);
            const bool arr = (ust & kNotArrived) == kNotArrived;
            // ARRIVE (Fig. 3b/3c; R2)
            // R1-LIT: every newcomer takes what is free (no fill target)
            const uint32_t g = (arr && (LIT || target == kNoC)) ? min(L, free_mem) : 0u;
            const bool vadm = arr && g == L;
            const bool vtgt = !LIT && arr && !vadm && g > 0;
            // An arrival whose first op has delta 0 (before arrival the used
            // field holds d_0) is followed by that op at the same tick: the
            // DISPATCH after an ARRIVE is empty (with a target free = 0 and the
            // target's resume test is unchanged; without one nothing is paused)
            // and (t, c) stays the least key, so both events are applied in
            // this step, the op on the post-ARRIVE state.  The peaks need no
            // intermediate sample: the ARRIVE changes no used memory, and
            // cap - free only falls after it.
            const bool fz = arr && (ust & kUsedMask) == 0u;
            const bool op = !arr || fz;
            events += fz ? 1u : 0u;
            const uint32_t ust1 = arr ? ((vadm ? kAdmitted : 0u) | (ust & (kKindsMask | kLimHi))) : ust;
            const uint32_t tg1 = vtgt ? c : target;
            const uint32_t k = (ust1 >> kKShift) & 3u;
            const uint32_t kind = (ust1 >> (kKindShift + 2 * k)) & 3u;
            const uint32_t r = sd & 0xFFFFu, used = ust1 & kUsedMask;
            const uint32_t nd = (arr && !fz) ? (ust & kUsedMask) : (sd >> 16);  // d_0 / d_{k+1}
            const bool isA = op && kind == CONVGPU_OP_ALLOC;
            const bool isF = op && kind == CONVGPU_OP_FREE;
            const bool isX = op && kind == CONVGPU_OP_FINISH;
            const bool tnone = tg1 == kNoC, ctg = c == tg1;
            const uint32_t a_c =
                (ust1 & kAdmitted) ? L
                                   : (LIT ? (arr ? g : (uint32_t)ASG(c)) : (vtgt ? g : (ctg ? a_tg : 0u)));
            if (LIT && arr) ASG(c) = (uint16_t)g;
            // ALLOC
            const uint32_t need = used + r + ((ust1 & kFirst) ? 0u : ovh);
            const bool rej = isA && need > L;                // R10
            const bool grant = isA && !rej && need <= a_c;
            const bool pause = isA && !rej && !grant;       // reply withheld
            // FREE (R11)
            const bool badfree = isF && r > used;
            const uint32_t free1 = free_mem - g;
            peak_res = max(peak_res, cap - free1);
            free_mem = free1 + (isX ? a_c : 0u);
            used_total = used_total + (grant ? need - used : 0u) - ((isF && !badfree) ? r : 0u) -
                         (isX ? used : 0u);
            peak_used = max(peak_used, used_total);
            if (used_total > cap - free_mem) flags |= CONVGPU_FLAG_OVERCOMMIT;
            const bool clear_tg = isX && ctg;               // R20
            target = clear_tg ? kNoC : tg1;
            a_tg = clear_tg ? 0u : (vtgt ? g : a_tg);
            stg_if(adm_out + c, (t << 6) | rank, vadm);     // admission at arrival
            rank += vadm ? 1u : 0u;
            n_rej += rej ? 1u : 0u;
            live -= isX ? 1u : 0u;
            const uint32_t pmask = pause ? 0xFFFFFFFFu : 0u;
            pm_lo |= shl_c(1u, c) & pmask;
            pm_hi |= shl_c(1u, c - 32u) & pmask;
            // Recent-Fit: push c on the suspension stack (its key links the old
            // top) unless it is the fill target, which resumes without a
            // selection (R1) and so must never be popped
            const uint32_t plink = (P == CONVGPU_RECENT_FIT) ? ru_head : 0u;
            if (P == CONVGPU_RECENT_FIT) ru_head = (pause && !ctg) ? c : ru_head;
            // R1-LIT dispatches whenever memory is free and someone is paused
            dmode = LIT ? (free_mem != 0u && (pm_lo | pm_hi) != 0u)
                        : (pause & tnone) | (isX & ((target != kNoC) | ((pm_lo | pm_hi) != 0u)));
            if (badfree) { flags |= CONVGPU_FLAG_INVALID_FREE; tdone = true;
#ifdef LPT16_DEBUG
              dbg0 = c | (k << 8) | ((uint32_t)(pre_c) << 16); dbg1 = r; dbg2 = used; dbg3 = ust; dbg4 = sd;
#endif
            }
            const bool adv = !isX && !pause && !badfree;
            uint32_t nu = ust1;
            nu = grant ? ((ust1 & ~kUsedMask) | need | kFirst) : nu;
            nu = (isF && !badfree) ? ust1 - r : nu;
            nu = isX ? (ust1 & ~kUsedMask) : nu;
            nu = pause ? (ust1 | kPaused) : nu;
            nu = (adv && op) ? nu + kKOne : nu;
            kc = badfree ? kNoC : c;
            nkc = adv ? (((t + nd) << 6) | c) : (isX ? (kDone | t) : (kPausedKey | plink));
            pfk = (adv && op) ? k + 1u : 0xFFu;
            AT(s_ust, c) = nu;
          }
        } else if (dmode) {
          // ====== one DISPATCH step at the triggering tick (R1, R9) ======
          const uint32_t t = cur_t;
          select_target(true);
          {
            // the target was not fetched in the previous iteration: a dispatch
            // step follows a pause / FINISH (no fetch) or an admission, after
            // which the resumed container is no longer paused
            const uint32_t tg = target;
            const uint32_t ut = AT(s_ust, tg), sdt = AT(s_sd, tg), Lt = FULL_L(tg, ut);
            const uint32_t g = min(free_mem, Lt - a_tg);
            a_tg += g;
            free_mem -= g;
            const uint32_t pend = (sdt & 0xFFFFu) + ((ut & kFirst) ? 0u : ovh);
            const uint32_t uu = ut & kUsedMask;
            const bool res = (ut & kPaused) && uu + pend <= a_tg;  // RESUME (R9)
            const bool full = a_tg == Lt;                          // admit, cascade
            used_total += res ? pend : 0u;
            peak_res = max(peak_res, cap - free_mem);
            peak_used = max(peak_used, used_total);
            if (used_total > cap - free_mem) flags |= CONVGPU_FLAG_OVERCOMMIT;
            uint32_t nu = res ? (((ut & ~(kUsedMask | kPaused)) | (uu + pend) | kFirst) + kKOne) : ut;
            nu |= full ? kAdmitted : 0u;
            nkc = ((t + (sdt >> 16)) << 6) | tg;
            pfk = res ? ((nu >> kKShift) & 3u) : 0xFFu;
            AT(s_ust, tg) = nu;
            const uint32_t rmask = res ? 0xFFFFFFFFu : 0u;
            pm_lo &= ~(shl_c(1u, tg) & rmask);
            pm_hi &= ~(shl_c(1u, tg - 32u) & rmask);
            stg_if(adm_out + tg, (t << 6) | rank, full);
            rank += full ? 1u : 0u;
            if (LIT) {  // no sticky target: select again while memory is free
              ASG(tg) = (uint16_t)a_tg;
              if (P == CONVGPU_RECENT_FIT) ru_head = res ? (AT(s_key, tg) & 127u) : ru_head;
              target = kNoC;
              a_tg = 0;
              dmode = free_mem != 0u && (pm_lo | pm_hi) != 0u;
            } else {
              target = full ? kNoC : target;
              a_tg = full ? 0u : a_tg;
              dmode = full && (pm_lo | pm_hi) != 0u;
            }
            kc = res ? tg : kNoC;
          }
        }
        // ---- shared tail: key update, group re-min, retire the previous
        // iteration's fetch, issue this iteration's ----
        {
          const uint32_t kcs = kc & 63u;
          sts_if(&AT(s_key, kcs), nkc, kc != kNoC);
          regroup(kcs);
          // retire last iteration's fetch (issued one iteration ago)
          lpt::cp_wait0();  // nothing pending if nothing was fetched: no branch needed
          sts_if(&AT(s_sd, pre_c & 63u), pack_sd(AT(s_stg, 0), AT(s_stg, 1)), pre_c != kNoC);
          // op k word and the delta of op k+1 (clamped: FINISH never reads it)
          const bool f = pfk < K;
          const uint32_t off = pfk * n + kcs;
          lpt::cp_async4_if(&AT(s_stg, 0), trace_arg + off, f);
          lpt::cp_async4_if(&AT(s_stg, 1), trace_delta + min(pfk + 1u, K - 1u) * n + kcs, f);
          lpt::cp_commit();
          pre_c = f ? kcs : kNoC;
        }
      }
    } while (!__all_sync(kFull, !have || tdone));
    fetch_state();
    epilogue(have ? i : 0, have && !skip);
    if (have) {
      i = next(i + T);
      have = i < p.count;
    }
#ifdef LPT16_INIT2  // experiment: init twice (its cost in the running kernel)
    if (__any_sync(kFull, have)) { init(have ? i : 0, have); }
#endif
    if (__any_sync(kFull, have)) { init(have ? i : 0, have); tdone = LPT16_TD; dmode = false; }
    park_state();
  }
  fetch_state();  // the statistics accumulators, for the final reduction
#undef FULL_L
#undef ASG
#undef LIM
#undef AT

  if (p.range_digest && racc_r != ~0ull)
    atomicAdd((unsigned long long*)&p.range_digest[racc_r], racc);
  if (p.stats) {
    __syncwarp();
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      st_traces += __shfl_xor_sync(kFull, st_traces, o);
      st_events += __shfl_xor_sync(kFull, st_events, o);
      st_mk += __shfl_xor_sync(kFull, st_mk, o);
      st_wait += __shfl_xor_sync(kFull, st_wait, o);
      st_rej += __shfl_xor_sync(kFull, st_rej, o);
      st_sel += __shfl_xor_sync(kFull, st_sel, o);
      st_dig += __shfl_xor_sync(kFull, st_dig, o);
      st_maxmk = max(st_maxmk, __shfl_xor_sync(kFull, st_maxmk, o));
      st_maxpk = max(st_maxpk, __shfl_xor_sync(kFull, st_maxpk, o));
    }
    if (lane == 0 && st_traces) {
      convgpu_stats_t* Sg = p.stats;
      atomicAdd((unsigned long long*)&Sg->traces, st_traces);
      atomicAdd((unsigned long long*)&Sg->events, st_events);
      atomicAdd((unsigned long long*)&Sg->sum_makespan, st_mk);
      atomicAdd((unsigned long long*)&Sg->sum_wait, st_wait);
      atomicAdd((unsigned long long*)&Sg->n_rejected, st_rej);
      atomicAdd((unsigned long long*)&Sg->n_select, st_sel);
      atomicAdd((unsigned long long*)&Sg->digest_sum, st_dig);
      atomicMax(&Sg->max_makespan, st_maxmk);
      atomicMax(&Sg->max_peak_reserved, st_maxpk);
    }
  }
  lpt::tmem_fence_before_sync();
  __syncthreads();
  lpt::tmem_fence_after_sync();
  if (wib == 0) lpt::tmem_dealloc(s_tmem, kTmemCols);
}

template <int POLICY, bool WIDE = false>
static cudaError_t launch_t(const ReplayArgs& a, cudaStream_t stream) {
  auto kern = replay_lpt16_kernel<POLICY, WIDE>;
  int dev = 0, sms = 0;
  cudaError_t e;
  if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
  if ((e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess) return e;
  // one persistent CTA per SM; a batch smaller than one trace per lane of a
  // full grid gets smaller CTAs, so that it still spreads over every SM
  uint64_t warps = (uint64_t)warps_per_cta(POLICY);
  if (!a.grid_override) {
    const uint64_t w = (a.count + 32ull * sms - 1) / (32ull * sms);
    warps = w < 1 ? 1 : (w < warps ? w : warps);
  }
  const int threads = (int)(32 * warps);
  const size_t smem = (size_t)threads * lane_bytes(POLICY);
  if ((e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)((size_t)32 * warps_per_cta(POLICY) * lane_bytes(POLICY)))) != cudaSuccess)
    return e;
  const uint64_t need = (a.count + threads - 1) / threads;
  uint64_t grid = (uint64_t)sms;  // one CTA per SM, persistent
  if (a.grid_override) grid = a.grid_override;
  if (grid > need) grid = need;
  if (grid < 1) grid = 1;
  kern<<<(unsigned)grid, threads, smem, stream>>>(a);
  return cudaGetLastError();
}

}  // namespace lpt16

bool lpt16_supported(const ReplayArgs& a) {
  return a.n == lpt16::N && a.K == lpt16::KOPS && a.adm_buf() != nullptr && a.aligned16;
}

cudaError_t launch_replay_lpt16(const ReplayArgs& a, int policy, cudaStream_t stream,
                                bool wide_first) {
  cudaError_t e;
  const bool lit = (policy & CONVGPU_DISPATCH_LITERAL) != 0;
  constexpr int L = CONVGPU_DISPATCH_LITERAL;
  ReplayArgs b = a;
  if (wide_first && !lit) {
    // CONVGPU_KERNEL_LANE_COMPACT_WIDE: the 17-bit layout over every trace,
    // what it cannot hold (kLpt16Mark2) to the 32-bit lane kernel
    switch (policy & 0xFF) {
      case CONVGPU_FIFO: e = lpt16::launch_t<CONVGPU_FIFO, true>(a, stream); break;
      case CONVGPU_BEST_FIT: e = lpt16::launch_t<CONVGPU_BEST_FIT, true>(a, stream); break;
      case CONVGPU_RECENT_FIT: e = lpt16::launch_t<CONVGPU_RECENT_FIT, true>(a, stream); break;
      case CONVGPU_RANDOM_FIT: e = lpt16::launch_t<CONVGPU_RANDOM_FIT, true>(a, stream); break;
      default: return cudaErrorInvalidValue;
    }
    if (e != cudaSuccess) return e;
    b.only_marked = kLpt16Mark2;
    return launch_replay_lpt(b, policy, stream);
  }
  switch ((policy & 0xFF) | (lit ? L : 0)) {
    case CONVGPU_FIFO: e = lpt16::launch_t<CONVGPU_FIFO>(a, stream); break;
    case CONVGPU_BEST_FIT: e = lpt16::launch_t<CONVGPU_BEST_FIT>(a, stream); break;
    case CONVGPU_RECENT_FIT: e = lpt16::launch_t<CONVGPU_RECENT_FIT>(a, stream); break;
    case CONVGPU_RANDOM_FIT: e = lpt16::launch_t<CONVGPU_RANDOM_FIT>(a, stream); break;
    case CONVGPU_FIFO | L: e = lpt16::launch_t<CONVGPU_FIFO | L>(a, stream); break;
    case CONVGPU_BEST_FIT | L: e = lpt16::launch_t<CONVGPU_BEST_FIT | L>(a, stream); break;
    case CONVGPU_RECENT_FIT | L: e = lpt16::launch_t<CONVGPU_RECENT_FIT | L>(a, stream); break;
    case CONVGPU_RANDOM_FIT | L: e = lpt16::launch_t<CONVGPU_RANDOM_FIT | L>(a, stream); break;
    default: return cudaErrorInvalidValue;
  }
  if (e != cudaSuccess) return e;
  b.only_marked = kLpt16Mark;
  // R1-LIT: the traces the 16-bit layout cannot hold go to the warp-per-trace
  // kernel (which implements that reading), marked only
  if (lit) return launch_replay(b, policy, false, stream);
  // 16-bit host format (limits <= 0xFFFF): the 17-bit pass could only take
  // limits of exactly 0xFFFF; the 32-bit kernel does, one launch fewer
  if (a.no_wide) return launch_replay_lpt(b, policy, stream);
  // R1: to the 17-bit layout (WIDE), marked only; what that cannot hold
  // either (re-marked kLpt16Mark2) to the 32-bit lane kernel
#ifdef LPT16_NO_WIDE
  return launch_replay_lpt(b, policy, stream);
#endif
  switch (policy & 0xFF) {
    case CONVGPU_FIFO: e = lpt16::launch_t<CONVGPU_FIFO, true>(b, stream); break;
    case CONVGPU_BEST_FIT: e = lpt16::launch_t<CONVGPU_BEST_FIT, true>(b, stream); break;
    case CONVGPU_RECENT_FIT: e = lpt16::launch_t<CONVGPU_RECENT_FIT, true>(b, stream); break;
    case CONVGPU_RANDOM_FIT: e = lpt16::launch_t<CONVGPU_RANDOM_FIT, true>(b, stream); break;
    default: return cudaErrorInvalidValue;
  }
  if (e != cudaSuccess) return e;
  b.only_marked = kLpt16Mark2;
  return launch_replay_lpt(b, policy, stream);
}

}  // namespace convgpu
