// replay_lpt.cu — lane-per-trace replay of ConVGPU's GPU-memory scheduler
// (§III-D, Fig. 3) on sm_100a.
//
// The warp-per-trace kernel (replay.cu) spends ~85 warp instructions per
// event because one trace's event loop is inherently serial and all 32 lanes
// execute it.  Here every LANE owns a trace, so each warp instruction
// advances 32 independent traces:
//  * per-container state lives in shared memory in a lane-interleaved layout
//    (word w of container c of lane l at [(w*n + c)*32 + l]) — every access
//    with an arbitrary per-lane container index is bank-conflict-free;
//  * the next event is found with a two-level min: 8 group minima (8
//    containers each) in registers, the 64 keys in shared memory; a key
//    change re-mins one group (8 LDS + 7 IMNMX);
//  * the op words of a container are fetched one op ahead with cp.async
//    (global -> shared, no registers), one commit group per iteration; an
//    event waits only for the group that can still be in flight for it;
//  * outputs and the digest are produced in a per-trace epilogue, which all
//    lanes run together (valid traces have exactly n*(1+K) events), and the
//    statistics are reduced warp -> grid at the end.
// Semantics are identical to replay.cu; parity is tested
// against the oracle on both.
#include <cuda_runtime.h>
#include <stdint.h>

#include "common.cuh"
#include "internal.h"

namespace convgpu {
namespace lpt {

// ust word: used (26 bits) | k << 26 (3 bits) | FIRST | PAUSED | ADMITTED.
// PAUSED|ADMITTED together (impossible for a live container) = not arrived.
constexpr uint32_t kUsedMask = (1u << 26) - 1;
constexpr uint32_t kKShift = 26;
constexpr uint32_t kKMask = 7u << kKShift;
constexpr uint32_t kFirst = 1u << 29;
constexpr uint32_t kPaused = 1u << 30;
constexpr uint32_t kAdmitted = 1u << 31;
constexpr uint32_t kNotArrived = kPaused | kAdmitted;
constexpr uint32_t kTargetNone = 64u;
constexpr uint32_t kTickLimit = CONVGPU_TICK_LIMIT;
constexpr uint32_t kStopMask = ~(uint32_t)CONVGPU_FLAG_OVERCOMMIT;
constexpr int kWords = 7;  // key, L, ust, wait, adm, cw, nd
enum { W_KEY = 0, W_L = 1, W_UST = 2, W_WAIT = 3, W_ADM = 4, W_CW = 5, W_ND = 6 };
// Before arrival W_WAIT holds delta_0 and W_ADM delta_1 (K > 1).  While a
// container is paused W_ADM holds its suspension number (Recent-Fit).  After
// FINISH W_ND holds its finish tick.

__host__ __device__ inline size_t warp_bytes(uint32_t n) { return (size_t)kWords * n * 32 * 4; }

__device__ __forceinline__ uint32_t smem_addr(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void cp_async4(uint32_t* dst, const uint32_t* src) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_addr(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_wait1() { asm volatile("cp.async.wait_group 1;" ::: "memory"); }
__device__ __forceinline__ void cp_wait0() { asm volatile("cp.async.wait_group 0;" ::: "memory"); }

template <int POLICY, int MODE>
__global__ void __launch_bounds__(kLptThreads) replay_lpt_kernel(const ReplayArgs p) {
  extern __shared__ __align__(16) uint32_t smem_w[];
  const uint32_t lane = threadIdx.x & 31u, wib = threadIdx.x >> 5;
  const uint32_t n = p.n, K = p.K, cap = p.cap, ovh = p.ovh;
  uint32_t* const S = smem_w + (size_t)wib * kWords * n * 32 + lane;
  uint32_t* const s_key = S + (size_t)W_KEY * n * 32;
  uint32_t* const s_L = S + (size_t)W_L * n * 32;
  uint32_t* const s_ust = S + (size_t)W_UST * n * 32;
  uint32_t* const s_wait = S + (size_t)W_WAIT * n * 32;
  uint32_t* const s_adm = S + (size_t)W_ADM * n * 32;
  uint32_t* const s_cw = S + (size_t)W_CW * n * 32;
  uint32_t* const s_nd = S + (size_t)W_ND * n * 32;
#define AT(arr, c) (arr)[(c) * 32u]

  const uint64_t T = (uint64_t)gridDim.x * blockDim.x;
  uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;

  // per-thread statistics
  unsigned long long st_traces = 0, st_events = 0, st_mk = 0, st_wait = 0, st_rej = 0,
                     st_sel = 0, st_dig = 0;
  uint32_t st_maxmk = 0, st_maxpk = 0;
  unsigned long long racc_r = ~0ull, racc = 0;

  // per-trace scheduler ledger
  uint32_t gmin[8];
  uint32_t free_mem = 0, target = kTargetNone, a_tg = 0, used_total = 0, seq = 0, rank = 0,
           draws = 0, n_rej = 0, n_sel = 0, peak_res = 0, peak_used = 0, flags = 0, live = 0,
           events = 0, a0 = 0;
  uint32_t pm_lo = 0, pm_hi = 0, pfc_lo = 0, pfc_hi = 0;
  const uint32_t* trace_delta = nullptr;
  const uint32_t* trace_arg = nullptr;

  auto regroup = [&](uint32_t c) {  // re-min the group of container c
    const uint32_t g = c >> 3, b = g << 3;
    uint32_t m = kKeyNone;
#pragma unroll
    for (uint32_t j = 0; j < 8; ++j)
      if (b + j < n) m = min(m, AT(s_key, b + j));
#pragma unroll
    for (uint32_t j = 0; j < 8; ++j) gmin[j] = (j == g) ? m : gmin[j];
  };
  auto prefetch = [&](uint32_t c, uint32_t k) {  // op k word, delta of op k+1
    if (MODE == 2) {
      if (k < K) AT(s_cw, c) = __ldg(trace_arg + (size_t)k * n + c);
      if (k + 1 < K) AT(s_nd, c) = __ldg(trace_delta + (size_t)(k + 1) * n + c);
      return;
    }
    if (k < K) cp_async4(&AT(s_cw, c), trace_arg + (size_t)k * n + c);
    if (k + 1 < K) cp_async4(&AT(s_nd, c), trace_delta + (size_t)(k + 1) * n + c);
    if (c < 32) pfc_lo |= 1u << c; else pfc_hi |= 1u << (c - 32);
  };
  auto init = [&](uint64_t ti) {
    const uint32_t* A = p.arrival + ti * n;
    const uint32_t* Lg = p.limit + ti * n;
    trace_delta = p.delta + ti * (uint64_t)K * n;
    trace_arg = p.arg + ti * (uint64_t)K * n;
    uint32_t bad = 0, lsum = 0, amax = 0, prev = 0;
#pragma unroll
    for (int j = 0; j < 8; ++j) gmin[j] = kKeyNone;
    for (uint32_t c = 0; c < n; ++c) {
      const uint32_t a = __ldg(A + c), L = __ldg(Lg + c);
      if (L > cap) bad |= CONVGPU_FLAG_INVALID_LIMIT;
      if (c > 0 && a < prev) bad |= CONVGPU_FLAG_UNSORTED_ARRIVAL;
      prev = a;
      amax = max(amax, a);
      uint32_t d0 = 0, d1 = 0, w0 = 0;
      for (uint32_t k = 0; k < K; ++k) {
        const uint32_t d = __ldg(trace_delta + (size_t)k * n + c);
        const uint32_t w = __ldg(trace_arg + (size_t)k * n + c);
        lsum = min(lsum + min(d, kTickLimit), kTickLimit);
        if (((w >> 30) == CONVGPU_OP_FINISH) != (k + 1 == K)) bad |= CONVGPU_FLAG_BAD_PROGRAM;
        if (k == 0) { d0 = d; w0 = w; }
        if (k == 1) d1 = d;
      }
      const uint32_t key = (min(a, kTickLimit - 1) << 6) | c;
      AT(s_key, c) = key;
      AT(s_L, c) = L;
      AT(s_ust, c) = kNotArrived;
      AT(s_wait, c) = d0;
      AT(s_adm, c) = d1;
      AT(s_cw, c) = w0;
      const uint32_t g = c >> 3;
#pragma unroll
      for (uint32_t j = 0; j < 8; ++j) gmin[j] = (j == g) ? min(gmin[j], key) : gmin[j];
    }
    if (amax >= kTickLimit || amax + lsum >= kTickLimit) bad |= CONVGPU_FLAG_TICK_RANGE;
    flags = bad;
    free_mem = cap; target = kTargetNone; a_tg = 0; used_total = 0; seq = 0; rank = 0;
    draws = 0; n_rej = 0; n_sel = 0; peak_res = 0; peak_used = 0; live = n; events = 0;
    a0 = __ldg(A);
    pm_lo = pm_hi = pfc_lo = pfc_hi = 0;
  };
  auto epilogue = [&](uint64_t ti) {
    cp_wait0();
    const bool stopped = (flags & kStopMask) != 0;
    if (stopped) { peak_res = 0; peak_used = 0; n_rej = 0; n_sel = 0; }
    uint64_t dig = 0, swait = 0;
    uint32_t mfin = 0;
    const uint64_t ob = ti * n;
    for (uint32_t c = 0; c < n; ++c) {
      uint32_t at = kKeyNone, ar = 0xFFu, wt = 0, fn = 0;
      if (!stopped) {
        const uint32_t u = AT(s_ust, c);
        if (u & kAdmitted) {
          const uint32_t adm = AT(s_adm, c);
          at = adm >> 6;
          ar = adm & 63u;
        }
        wt = AT(s_wait, c);
        fn = AT(s_nd, c);
      }
      if (p.admit_tick) p.admit_tick[ob + c] = at;
      if (p.admit_rank) p.admit_rank[ob + c] = (uint8_t)ar;
      if (p.wait) p.wait[ob + c] = wt;
      if (p.finish) p.finish[ob + c] = fn;
      const uint64_t h1 = mix64(((uint64_t)c << 56) ^ ((uint64_t)ar << 48) ^ (uint64_t)at);
      dig += mix64(h1 ^ (((uint64_t)wt << 32) | fn));
      mfin = max(mfin, fn);
      swait += wt;
    }
    const uint32_t makespan = stopped ? 0u : mfin - a0;
    dig += mix64(((uint64_t)makespan << 32) | peak_res);
    dig += mix64(((uint64_t)peak_used << 32) | flags);
    dig += mix64(swait);
    dig += mix64(((uint64_t)n_rej << 32) | n_sel);
    if (p.summary) {
      convgpu_summary_t sm;
      sm.makespan = makespan; sm.peak_reserved = peak_res; sm.peak_used = peak_used;
      sm.flags = flags; sm.sum_wait = swait; sm.n_rejected = n_rej; sm.n_select = n_sel;
      sm.digest = dig;
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

  bool have = i < p.count, halted = false;
  if (have) { init(i); halted = flags != 0; }  // static flags stop before the first event
  while (have) {
    bool done = halted;
    if (!done) {
      // ---- next event: two-level min (a2) ----
      const uint32_t m01 = min(gmin[0], gmin[1]), m23 = min(gmin[2], gmin[3]);
      const uint32_t m45 = min(gmin[4], gmin[5]), m67 = min(gmin[6], gmin[7]);
      const uint32_t kmin = min(min(m01, m23), min(m45, m67));
      if (kmin == kKeyNone) {
        if (live) flags |= CONVGPU_FLAG_DEADLOCK;  // P:7
        done = true;
      } else {
        const uint32_t t = kmin >> 6, c = kmin & 63u;
        // the op data of c may still be in flight from the previous iteration
        // groups older than the previous iteration's are complete after
        // wait_group 1; the previous iteration's group (containers in pfc)
        // may still be in flight
        cp_wait1();
        if (MODE == 1 || ((c < 32 ? (pfc_lo >> c) : (pfc_hi >> (c - 32))) & 1u)) cp_wait0();
        pfc_lo = 0; pfc_hi = 0;
        ++events;
        uint32_t ust = AT(s_ust, c);
        const uint32_t L = AT(s_L, c);
        uint32_t nk = kKeyNone;
        bool disp = false;
        if ((ust & kNotArrived) == kNotArrived) {
          // ARRIVE (Fig. 3b/3c; R2)
          const uint32_t d0 = AT(s_wait, c), d1 = AT(s_adm, c);
          const uint32_t g = (target == kTargetNone) ? min(L, free_mem) : 0u;
          free_mem -= g;
          uint32_t adm = kKeyNone;
          ust = 0;
          if (g == L) {
            adm = (t << 6) | rank; ++rank; ust = kAdmitted;
          } else if (g > 0) {
            target = c; a_tg = g;
          }
          AT(s_adm, c) = adm;
          AT(s_wait, c) = 0;
          AT(s_nd, c) = d1;
          peak_res = max(peak_res, cap - free_mem);
          nk = ((t + d0) << 6) | c;
        } else {
          const uint32_t cw = AT(s_cw, c);
          const uint32_t kind = cw >> 30, r = cw & kSizeMask, used = ust & kUsedMask;
          bool adv = true;
          if (kind == CONVGPU_OP_ALLOC) {
            const uint32_t need = used + r + ((ust & kFirst) ? 0u : ovh);
            const uint32_t a = (ust & kAdmitted) ? L : (c == target ? a_tg : 0u);
            if (need > L) {
              ++n_rej;  // R10
            } else if (need <= a) {
              used_total += need - used;
              peak_used = max(peak_used, used_total);
              ust = (ust & ~kUsedMask) | need | kFirst;
            } else {  // pause: reply withheld
              ust |= kPaused;
              AT(s_wait, c) -= t;
              if (POLICY == CONVGPU_RECENT_FIT) AT(s_adm, c) = seq;
              ++seq;
              if (c < 32) pm_lo |= 1u << c; else pm_hi |= 1u << (c - 32);
              adv = false;
              disp = (target == kTargetNone);
            }
          } else if (kind == CONVGPU_OP_FREE) {  // P:110, R11
            if (r > used) {
              flags |= CONVGPU_FLAG_INVALID_FREE;
              adv = false;
              done = true;
            } else {
              ust -= r;
              used_total -= r;
            }
          } else if (kind == CONVGPU_OP_FINISH) {  // P:110, R18
            const uint32_t a = (ust & kAdmitted) ? L : (c == target ? a_tg : 0u);
            free_mem += a;
            used_total -= used;
            ust &= ~kUsedMask;
            AT(s_nd, c) = t;  // finish tick
            --live;
            if (c == target) { target = kTargetNone; a_tg = 0; }  // R20
            adv = false;
            disp = true;
          }
          if (adv) {
            const uint32_t k = ((ust >> kKShift) & 7u) + 1u;
            nk = ((t + AT(s_nd, c)) << 6) | c;
            ust = (ust & ~kKMask) | (k << kKShift);
            prefetch(c, k);
          }
        }
        if (!done) {
          AT(s_ust, c) = ust;
          AT(s_key, c) = nk;
          regroup(c);
          // ---- DISPATCH (Fig. 3d; R1, R9) ----
          if (disp) {
            for (;;) {
              if (target != kTargetNone) {
                const uint32_t tg = target, Lt = AT(s_L, tg);
                const uint32_t g = min(free_mem, Lt - a_tg);
                a_tg += g;
                free_mem -= g;
                peak_res = max(peak_res, cap - free_mem);
                uint32_t ut = AT(s_ust, tg);
                if (ut & kPaused) {
                  const uint32_t cwt = AT(s_cw, tg);
                  const uint32_t pend = (cwt & kSizeMask) + ((ut & kFirst) ? 0u : ovh);
                  const uint32_t uu = ut & kUsedMask;
                  if (uu + pend <= a_tg) {  // RESUME (R9)
                    used_total += pend;
                    peak_used = max(peak_used, used_total);
                    AT(s_wait, tg) += t;
                    AT(s_adm, tg) = kKeyNone;
                    if (tg < 32) pm_lo &= ~(1u << tg); else pm_hi &= ~(1u << (tg - 32));
                    const uint32_t k = ((ut >> kKShift) & 7u) + 1u;
                    ut = (ut & ~(kUsedMask | kKMask | kPaused)) | (uu + pend) | kFirst | (k << kKShift);
                    AT(s_key, tg) = ((t + AT(s_nd, tg)) << 6) | tg;
                    regroup(tg);
                    prefetch(tg, k);
                  }
                }
                if (a_tg == Lt) {  // fully guaranteed: admit, cascade leftover
                  AT(s_adm, tg) = (t << 6) | rank; ++rank;
                  AT(s_ust, tg) = ut | kAdmitted;
                  target = kTargetNone;
                  a_tg = 0;
                  continue;
                }
                AT(s_ust, tg) = ut;
                break;
              }
              if ((pm_lo | pm_hi) == 0u) break;
              // ---- SELECT among paused ----
              uint32_t sel;
              if (POLICY == CONVGPU_FIFO) {  // oldest created (R7)
                sel = pm_lo ? (uint32_t)(__ffs(pm_lo) - 1) : 32u + (uint32_t)(__ffs(pm_hi) - 1);
              } else if (POLICY == CONVGPU_BEST_FIT) {  // R3, R4: shortfall L - 0
                uint32_t bf = kTargetNone, bfL = 0, bm = kTargetNone, bmL = 0;
#pragma unroll
                for (uint32_t h = 0; h < 2; ++h) {
                  uint32_t m = h ? pm_hi : pm_lo;
                  while (m) {
                    const uint32_t b = (uint32_t)(__ffs(m) - 1);
                    m &= m - 1;
                    const uint32_t cc = b + 32u * h;
                    const uint32_t Lc = AT(s_L, cc);
                    if (Lc <= free_mem && (bf == kTargetNone || Lc > bfL)) { bf = cc; bfL = Lc; }
                    if (bm == kTargetNone || Lc < bmL) { bm = cc; bmL = Lc; }
                  }
                }
                sel = (bf != kTargetNone) ? bf : bm;
              } else if (POLICY == CONVGPU_RECENT_FIT) {  // R5
                uint32_t best = 0, bs = 0;
#pragma unroll
                for (uint32_t h = 0; h < 2; ++h) {
                  uint32_t m = h ? pm_hi : pm_lo;
                  while (m) {
                    const uint32_t b = (uint32_t)(__ffs(m) - 1);
                    m &= m - 1;
                    const uint32_t cc = b + 32u * h;
                    const uint32_t sq = AT(s_adm, cc) + 1u;
                    if (sq > bs) { bs = sq; best = cc; }
                  }
                }
                sel = best;
              } else {  // RANDOM_FIT (R6)
                const uint64_t tid = p.tid_base + i;
                const uint32_t clo = __popc(pm_lo), m = clo + __popc(pm_hi);
                const U4 x = philox4x32_10((uint32_t)tid, (uint32_t)(tid >> 32), draws, 1u,
                                           (uint32_t)p.seed, (uint32_t)(p.seed >> 32));
                ++draws;
                const uint32_t jj = __umulhi(x.x, m);
                sel = (jj < clo) ? __fns(pm_lo, 0, jj + 1) : 32u + __fns(pm_hi, 0, jj - clo + 1);
              }
              target = sel;
              a_tg = 0;
              ++n_sel;
            }
          }
          if (used_total > cap - free_mem || free_mem > cap) flags |= CONVGPU_FLAG_OVERCOMMIT;
        }
        cp_commit();
      }
    }
    if (done) {
      epilogue(i);
      i += T;
      have = i < p.count;
      if (have) { init(i); halted = flags != 0; }
    }
  }
#undef AT

  // ---- statistics: warp -> grid (a6) ----
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
}

template <int POLICY, int MODE>
static cudaError_t launch_m(const ReplayArgs& a, cudaStream_t stream) {
  const size_t smem = (size_t)(kLptThreads / 32) * warp_bytes(a.n);
  auto kern = replay_lpt_kernel<POLICY, MODE>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  int dev = 0, sms = 0, per_sm = 0;
  if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
  if ((e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess) return e;
  if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, kLptThreads, smem)) !=
      cudaSuccess)
    return e;
  if (per_sm < 1) return cudaErrorInvalidConfiguration;
  const uint64_t need = (a.count + kLptThreads - 1) / kLptThreads;
  uint64_t grid = (uint64_t)sms * (uint64_t)per_sm;
  if (a.grid_override) grid = a.grid_override;
  if (grid > need) grid = need;
  if (grid < 1) grid = 1;
  kern<<<(unsigned)grid, kLptThreads, smem, stream>>>(a);
  return cudaGetLastError();
}

template <int POLICY>
static cudaError_t launch_t(const ReplayArgs& a, cudaStream_t stream) {
  return launch_m<POLICY, 0>(a, stream);
}

}  // namespace lpt

cudaError_t launch_replay_lpt(const ReplayArgs& a, int policy, cudaStream_t stream) {
  switch (policy) {
    case CONVGPU_FIFO: return lpt::launch_t<CONVGPU_FIFO>(a, stream);
    case CONVGPU_BEST_FIT: return lpt::launch_t<CONVGPU_BEST_FIT>(a, stream);
    case CONVGPU_RECENT_FIT: return lpt::launch_t<CONVGPU_RECENT_FIT>(a, stream);
    case CONVGPU_RANDOM_FIT: return lpt::launch_t<CONVGPU_RANDOM_FIT>(a, stream);
  }
  return cudaErrorInvalidValue;
}

}  // namespace convgpu
