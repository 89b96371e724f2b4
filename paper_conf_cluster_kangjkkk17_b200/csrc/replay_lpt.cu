// replay_lpt.cu — lane-per-trace replay of ConVGPU's GPU-memory scheduler
// (§III-D, Fig. 3) on sm_100a.
//
// The warp-per-trace kernel (replay.cu) spends ~70 warp instructions per
// event because one trace's event loop is inherently serial and all 32 lanes
// execute it.  Here every LANE owns a trace, so one warp instruction advances
// 32 independent traces:
//  * per-container state lives in shared memory in a lane-interleaved layout
//    (word w of container c of lane l at [(w*n + c)*32 + l]) — every access
//    with an arbitrary per-lane container index is bank-conflict-free;
//  * the next event comes from a two-level min: 8 group minima (8 containers
//    each) in registers, the keys in shared memory; a key change re-mins one
//    group (8 LDS + 7 IMNMX);
//  * each iteration is ONE micro-step per lane — an event, or one step of the
//    DISPATCH loop that an event started — written branch-free (selects and
//    predicated stores), so the 32 lanes stay converged whatever event kind
//    each of them processes; one shared tail does the key update, group
//    re-min and op prefetch;
//  * a container's next op word / delta are fetched one op ahead with
//    cp.async (global -> shared), one commit group per iteration; an event
//    waits only when its container was prefetched in the previous iteration;
//  * selection is O(1): FIFO = ffs of the paused mask, Random-Fit = Philox +
//    popc + fns, Recent-Fit = a lazily-deleted suspension stack, Best-Fit =
//    per-trace ranks of (limit, index) + a paused mask in rank order + a
//    binary search of the free memory over the sorted limits;
//  * suspended time is not tracked per event: wait = finish - arrival -
//    sum(deltas) (R17) is recovered in the per-trace epilogue, which all
//    lanes run together (they start and finish traces in lockstep).
// Semantics are identical to replay.cu; parity is tested
// against the oracle for both kernels.
#include <cuda_runtime.h>
#include <stdint.h>

#include "common.cuh"
#include "internal.h"
#include "lpt_util.cuh"

namespace convgpu {
namespace lpt {

// ust word: used (26 bits) | k << 26 (3 bits) | FIRST | PAUSED | ADMITTED.
// PAUSED|ADMITTED together (impossible for a live container) = not arrived.
constexpr uint32_t kUsedMask = (1u << 26) - 1;
constexpr uint32_t kKShift = 26;
constexpr uint32_t kKOne = 1u << kKShift;
constexpr uint32_t kFirst = 1u << 29;
constexpr uint32_t kPaused = 1u << 30;
constexpr uint32_t kAdmitted = 1u << 31;
constexpr uint32_t kNotArrived = kPaused | kAdmitted;
constexpr uint32_t kNoC = 64u;  // "no container" / no fill target
constexpr uint32_t kTickLimit = CONVGPU_TICK_LIMIT;
constexpr uint32_t kStopMask = ~(uint32_t)CONVGPU_FLAG_OVERCOMMIT;
constexpr uint32_t kStack = 128;  // Recent-Fit suspension stack entries

// shared-memory words per container
enum { W_KEY = 0, W_L = 1, W_UST = 2, W_ADM = 3, W_CW = 4, W_ND = 5, W_BASE_WORDS = 6 };
// W_ADM: d_1 before arrival; admission (tick << 6 | rank) once admitted;
//        the suspension number while paused (Recent-Fit scan fallback).
// W_ND:  delta to add at the container's next scheduling (d_0 before
//        arrival, then d_{k+1}); the finish tick after FINISH.
// Best-Fit adds W_RK (byte0 rank_of[j], byte1 gs[j], byte2 pi[j]: rank of
// container j in (L, index) order, first rank of rank j's limit, container
// of rank j); Recent-Fit adds a kStack-byte stack.
__host__ __device__ constexpr int extra_words(int policy) { return policy == CONVGPU_BEST_FIT ? 1 : 0; }

__host__ __device__ inline size_t warp_bytes(int policy, uint32_t n) {
  size_t b = (size_t)(W_BASE_WORDS + extra_words(policy)) * n * 32 * 4;
  if (policy == CONVGPU_RECENT_FIT) b += kStack * 32;
  return b;
}

// NF, KF: compile-time container / op counts (64, 4 for the configs) or 0.
__device__ __forceinline__ uint32_t comp(const uint4& v, int j) {
  return j == 0 ? v.x : (j == 1 ? v.y : (j == 2 ? v.z : v.w));
}

template <int POLICY, int NF, int KF>
__global__ void __launch_bounds__(kLptThreads) replay_lpt_kernel(const ReplayArgs p) {
  extern __shared__ __align__(16) uint32_t smem_w[];
  const uint32_t lane = threadIdx.x & 31u, wib = threadIdx.x >> 5;
  const uint32_t n = NF ? (uint32_t)NF : p.n, K = KF ? (uint32_t)KF : p.K;
  const uint32_t cap = p.cap, ovh = p.ovh;
  uint32_t* const W0 = smem_w + (wib * warp_bytes(POLICY, n)) / 4;
  uint32_t* const S = W0 + lane;
  uint32_t* const s_key = S + (size_t)W_KEY * n * 32;
  uint32_t* const s_L = S + (size_t)W_L * n * 32;
  uint32_t* const s_ust = S + (size_t)W_UST * n * 32;
  uint32_t* const s_adm = S + (size_t)W_ADM * n * 32;
  uint32_t* const s_cw = S + (size_t)W_CW * n * 32;
  uint32_t* const s_nd = S + (size_t)W_ND * n * 32;
  uint32_t* const s_rk = S + (size_t)(W_BASE_WORDS + 0) * n * 32;  // Best-Fit only
  uint8_t* const s_stk = reinterpret_cast<uint8_t*>(W0 + (size_t)W_BASE_WORDS * n * 32) + lane * 4;
#define AT(arr, c) (arr)[(c) * 32u]
#define RKB(j, b) reinterpret_cast<uint8_t*>(&AT(s_rk, (j)))[b]
#define STK(e) s_stk[((e) >> 2) * 128u + ((e) & 3u)]

  const uint64_t T = (uint64_t)gridDim.x * blockDim.x;
  uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;

  // per-thread statistics
  unsigned long long st_traces = 0, st_events = 0, st_mk = 0, st_wait = 0, st_rej = 0,
                     st_sel = 0, st_dig = 0;
  uint32_t st_maxmk = 0, st_maxpk = 0;
  unsigned long long racc_r = ~0ull, racc = 0;

  // per-trace scheduler ledger (all in registers)
  uint32_t gmin[8];
  uint32_t piv[8];  // Best-Fit, n = 64: limit at ranks 7, 15, ..., 63 (group maxima)
  uint32_t free_mem = 0, target = kNoC, a_tg = 0, used_total = 0, seq = 0, rank = 0, draws = 0,
           n_rej = 0, n_sel = 0, peak_res = 0, peak_used = 0, flags = 0, live = 0, events = 0;
  uint32_t pm_lo = 0, pm_hi = 0, pr_lo = 0, pr_hi = 0, sp = 0;
  uint32_t pfc = kNoC;  // container whose op words were prefetched in the last iteration
  bool ru_scan = false;
  const uint32_t* trace_delta = nullptr;
  const uint32_t* trace_arg = nullptr;

  auto regroup = [&](uint32_t c) {  // re-min the group of container c
    const uint32_t g = c >> 3, b = g << 3;
    uint32_t m = kKeyNone;
    if (NF != 0 && NF % 8 == 0) {  // whole groups: 8 loads in flight, min tree
      uint32_t v[8];
#pragma unroll
      for (uint32_t j = 0; j < 8; ++j) v[j] = AT(s_key, b + j);
      m = min(min(min(v[0], v[1]), min(v[2], v[3])), min(min(v[4], v[5]), min(v[6], v[7])));
    } else {
#pragma unroll
      for (uint32_t j = 0; j < 8; ++j)
        if (b + j < n) m = min(m, AT(s_key, b + j));
    }
#pragma unroll
    for (uint32_t j = 0; j < 8; ++j) gmin[j] = (j == g) ? m : gmin[j];
  };

  auto init = [&](uint64_t ti) {
    const uint32_t* A = p.arrival + ti * n;
    const uint32_t* Lg = p.limit + ti * n;
    trace_delta = p.delta + ti * (uint64_t)K * n;
    trace_arg = p.arg + ti * (uint64_t)K * n;
    uint32_t bad = 0, lsum = 0, amax = 0, prev = 0;
#pragma unroll
    for (int j = 0; j < 8; ++j) gmin[j] = kKeyNone;
    if (NF == 64 && KF == 4 && p.aligned16) {
      // 16-byte loads, 4 containers per step, every load of a step in flight
      const uint4* A4 = reinterpret_cast<const uint4*>(A);
      const uint4* L4 = reinterpret_cast<const uint4*>(Lg);
      const uint4* D4 = reinterpret_cast<const uint4*>(trace_delta);
      const uint4* R4 = reinterpret_cast<const uint4*>(trace_arg);
#pragma unroll
      for (uint32_t q = 0; q < 16; ++q) {
        const uint4 a4 = __ldg(A4 + q), l4 = __ldg(L4 + q);
        uint4 d4[4], w4[4];
#pragma unroll
        for (int k = 0; k < 4; ++k) { d4[k] = __ldg(D4 + k * 16 + q); w4[k] = __ldg(R4 + k * 16 + q); }
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          const uint32_t c = 4 * q + j, a = comp(a4, j), L = comp(l4, j);
          if (L > cap) bad |= CONVGPU_FLAG_INVALID_LIMIT;
          if (c > 0 && a < prev) bad |= CONVGPU_FLAG_UNSORTED_ARRIVAL;
          prev = a;
          amax = max(amax, a);
#pragma unroll
          for (int k = 0; k < 4; ++k) {
            lsum = min(lsum + min(comp(d4[k], j), kTickLimit), kTickLimit);
            if (((comp(w4[k], j) >> 30) == CONVGPU_OP_FINISH) != (k == 3)) bad |= CONVGPU_FLAG_BAD_PROGRAM;
          }
          const uint32_t key = (min(a, kTickLimit - 1) << 6) | c;
          AT(s_key, c) = key;
          AT(s_L, c) = L;
          AT(s_ust, c) = kNotArrived;
          AT(s_adm, c) = comp(d4[1], j);
          AT(s_cw, c) = comp(w4[0], j);
          AT(s_nd, c) = comp(d4[0], j);
          gmin[c >> 3] = min(gmin[c >> 3], key);
        }
      }
    } else {
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
        AT(s_adm, c) = d1;
        AT(s_cw, c) = w0;
        AT(s_nd, c) = d0;
        const uint32_t g = c >> 3;
  #pragma unroll
        for (uint32_t j = 0; j < 8; ++j) gmin[j] = (j == g) ? min(gmin[j], key) : gmin[j];
      }
    }
    if (amax >= kTickLimit || amax + lsum >= kTickLimit) bad |= CONVGPU_FLAG_TICK_RANGE;
    if (POLICY == CONVGPU_BEST_FIT) {
      // ranks of (L, index) ascending; gs = first rank with the same L
      if (NF == 64) {
        // bitonic sort network over the 64 packed keys L << 6 | c (L < 2^26)
        uint32_t v[64];
#pragma unroll
        for (int c = 0; c < 64; ++c) v[c] = (AT(s_L, c) << 6) | (uint32_t)c;
#pragma unroll
        for (int k = 2; k <= 64; k <<= 1) {
#pragma unroll
          for (int j = k >> 1; j > 0; j >>= 1) {
#pragma unroll
            for (int x = 0; x < 64; ++x) {
              const int y = x ^ j;
              if (y > x) {
                const uint32_t a = v[x], b = v[y];
                const bool up = (x & k) == 0;
                v[x] = up ? min(a, b) : max(a, b);
                v[y] = up ? max(a, b) : min(a, b);
              }
            }
          }
        }
#pragma unroll
        for (int j = 0; j < 8; ++j) piv[j] = v[8 * j + 7] >> 6;
        uint32_t gsr = 0, prevL = 0xFFFFFFFFu;
#pragma unroll
        for (int r = 0; r < 64; ++r) {
          const uint32_t c = v[r] & 63u, Lc = v[r] >> 6;
          gsr = (Lc == prevL) ? gsr : (uint32_t)r;
          prevL = Lc;
          RKB(c, 0) = (uint8_t)r;
          RKB(r, 1) = (uint8_t)gsr;
          RKB(r, 2) = (uint8_t)c;
        }
      } else {
        for (uint32_t c = 0; c < n; ++c) {
          const uint32_t Lc = AT(s_L, c);
          uint32_t lt = 0, eq = 0;
          for (uint32_t d = 0; d < n; ++d) {
            const uint32_t Ld = AT(s_L, d);
            lt += (Ld < Lc) ? 1u : 0u;
            eq += (Ld == Lc && d < c) ? 1u : 0u;
          }
          const uint32_t r = lt + eq;
          RKB(c, 0) = (uint8_t)r;
          RKB(r, 1) = (uint8_t)lt;
          RKB(r, 2) = (uint8_t)c;
        }
      }
    }
    flags = bad;
    free_mem = cap; target = kNoC; a_tg = 0; used_total = 0; seq = 0; rank = 0; draws = 0;
    n_rej = 0; n_sel = 0; peak_res = 0; peak_used = 0; live = n; events = 0;
    pm_lo = pm_hi = pr_lo = pr_hi = 0;
    pfc = kNoC;
    sp = 0;
    ru_scan = false;
  };

  auto epilogue = [&](uint64_t ti) {
    cp_wait0();
    const bool stopped = (flags & kStopMask) != 0;
    if (stopped) { peak_res = 0; peak_used = 0; n_rej = 0; n_sel = 0; }
    const uint32_t* A = p.arrival + ti * n;
    uint64_t dig = 0, swait = 0;
    uint32_t mfin = 0;
    const uint64_t ob = ti * n;
    if (NF == 64 && KF == 4 && p.aligned16) {
      const uint4* A4 = reinterpret_cast<const uint4*>(A);
      const uint4* D4 = reinterpret_cast<const uint4*>(trace_delta);
#pragma unroll 4
      for (uint32_t q = 0; q < 16; ++q) {
        uint4 a4 = make_uint4(0, 0, 0, 0), d4[4];
        if (!stopped) {
          a4 = __ldg(A4 + q);
#pragma unroll
          for (int k = 0; k < 4; ++k) d4[k] = __ldg(D4 + k * 16 + q);
        }
        uint32_t at[4], ar[4], wt[4], fn[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          const uint32_t c = 4 * q + j;
          at[j] = kKeyNone; ar[j] = 0xFFu; wt[j] = 0; fn[j] = 0;
          if (!stopped) {
            const uint32_t u = AT(s_ust, c);
            if (u & kAdmitted) {
              const uint32_t adm = AT(s_adm, c);
              at[j] = adm >> 6;
              ar[j] = adm & 63u;
            }
            fn[j] = AT(s_nd, c);
            // R17: wait = finish - arrival - sum of deltas
            wt[j] = fn[j] - comp(a4, j) - comp(d4[0], j) - comp(d4[1], j) - comp(d4[2], j) -
                    comp(d4[3], j);
          }
          const uint64_t h1 = mix64(((uint64_t)c << 56) ^ ((uint64_t)ar[j] << 48) ^ (uint64_t)at[j]);
          dig += mix64(h1 ^ (((uint64_t)wt[j] << 32) | fn[j]));
          mfin = max(mfin, fn[j]);
          swait += wt[j];
        }
        if (p.admit_tick) reinterpret_cast<uint4*>(p.admit_tick + ob)[q] = make_uint4(at[0], at[1], at[2], at[3]);
        if (p.admit_rank)
          reinterpret_cast<uint32_t*>(p.admit_rank + ob)[q] = ar[0] | (ar[1] << 8) | (ar[2] << 16) | (ar[3] << 24);
        if (p.wait) reinterpret_cast<uint4*>(p.wait + ob)[q] = make_uint4(wt[0], wt[1], wt[2], wt[3]);
        if (p.finish) reinterpret_cast<uint4*>(p.finish + ob)[q] = make_uint4(fn[0], fn[1], fn[2], fn[3]);
      }
    } else {
      for (uint32_t c = 0; c < n; ++c) {
        uint32_t at = kKeyNone, ar = 0xFFu, wt = 0, fn = 0;
        if (!stopped) {
          const uint32_t u = AT(s_ust, c);
          if (u & kAdmitted) {
            const uint32_t adm = AT(s_adm, c);
            at = adm >> 6;
            ar = adm & 63u;
          }
          fn = AT(s_nd, c);
          uint32_t sd = __ldg(A + c);  // R17: wait = finish - arrival - sum of deltas
          for (uint32_t k = 0; k < K; ++k) sd += __ldg(trace_delta + (size_t)k * n + c);
          wt = fn - sd;
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
    }
    const uint32_t makespan = stopped ? 0u : mfin - __ldg(A);
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

  // only_marked: the traces replay_lpt16.cu left to this kernel (8 markers
  // probed per step, all loads in flight)
  auto next = [&](uint64_t j) -> uint64_t {
    if (!p.only_marked) return j;
    while (j < p.count) {
      uint32_t m[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const uint64_t jj = j + (uint64_t)u * T;
        m[u] = jj < p.count ? p.adm_buf()[jj * n] : 0u;
      }
#pragma unroll
      for (int u = 0; u < 8; ++u)
        if (m[u] == p.only_marked) return j + (uint64_t)u * T;
      j += 8 * T;
    }
    return j;
  };
  i = next(i);
  bool have = i < p.count, tdone = false, dmode = false;
  uint32_t cur_t = 0;
  if (have) { init(i); tdone = flags != 0; dmode = false; }  // static flags: no events
  // Lanes advance through their traces independently but start and finish
  // them together (warp vote below), so init/epilogue run converged.
  while (__any_sync(kFull, have)) {
    // inner loop: one micro-step per lane until every lane's trace is done
    do {
      if (have && !tdone) {
        uint32_t kc = kNoC, nkc = kKeyNone, pfk = 0xFFu;
        const uint32_t pf = pfc;  // previous iteration's group
        pfc = kNoC;
        // next event (a2).  If it belongs to the container whose op words were
        // fetched in the previous iteration (rare), this lane idles for one
        // iteration; the cp.async.wait_group 1 of its next event step then
        // covers that fetch (as in replay_lpt16.cu).
        const uint32_t m01 = min(gmin[0], gmin[1]), m23 = min(gmin[2], gmin[3]);
        const uint32_t m45 = min(gmin[4], gmin[5]), m67 = min(gmin[6], gmin[7]);
        const uint32_t kmin = min(min(m01, m23), min(m45, m67));
        const bool hz = (kmin & 63u) == pf && kmin != kKeyNone;
        if (!dmode && !hz) {
          // ================= EVENT step (a2 + a3), branch-free =================
          if (kmin == kKeyNone) {
            if (live) flags |= CONVGPU_FLAG_DEADLOCK;  // P:7
            tdone = true;
          } else {
            const uint32_t t = kmin >> 6, c = kmin & 63u;
            cur_t = t;
            cp_wait1();  // every group but the previous iteration's is complete
            ++events;
            const uint32_t ust = AT(s_ust, c), L = AT(s_L, c), cw = AT(s_cw, c);
            const uint32_t nd = AT(s_nd, c), am = AT(s_adm, c);
            const bool arr = (ust & kNotArrived) == kNotArrived;
            const uint32_t kind = cw >> 30, r = cw & kSizeMask, used = ust & kUsedMask;
            const bool isA = !arr && kind == CONVGPU_OP_ALLOC;
            const bool isF = !arr && kind == CONVGPU_OP_FREE;
            const bool isX = !arr && kind == CONVGPU_OP_FINISH;
            const bool tnone = target == kNoC, ctg = c == target;
            const uint32_t a_c = (ust & kAdmitted) ? L : (ctg ? a_tg : 0u);
            // ARRIVE (Fig. 3b/3c; R2)
            const uint32_t g = (arr && tnone) ? min(L, free_mem) : 0u;
            const bool vadm = arr && g == L;
            const bool vtgt = arr && !vadm && g > 0;
            // ALLOC
            const uint32_t need = used + r + ((ust & kFirst) ? 0u : ovh);
            const bool rej = isA && need > L;                // R10
            const bool grant = isA && !rej && need <= a_c;
            const bool pause = isA && !rej && !grant;       // reply withheld
            // FREE (R11)
            const bool badfree = isF && r > used;
            // ledger
            free_mem = free_mem - g + (isX ? a_c : 0u);
            used_total = used_total + (grant ? need - used : 0u) - ((isF && !badfree) ? r : 0u) -
                         (isX ? used : 0u);
            peak_res = max(peak_res, cap - free_mem);
            peak_used = max(peak_used, used_total);
            if (used_total > cap - free_mem) flags |= CONVGPU_FLAG_OVERCOMMIT;
            const bool clear_tg = isX && ctg;               // R20
            target = vtgt ? c : (clear_tg ? kNoC : target);
            a_tg = vtgt ? g : (clear_tg ? 0u : a_tg);
            const uint32_t admv = (t << 6) | rank;
            rank += vadm ? 1u : 0u;
            n_rej += rej ? 1u : 0u;
            live -= isX ? 1u : 0u;
            // pause: mark c paused (branch-free: all-ones / zero mask)
            const uint32_t pmask = pause ? 0xFFFFFFFFu : 0u;
            pm_lo |= shl_c(1u, c) & pmask;
            pm_hi |= shl_c(1u, c - 32u) & pmask;
            if (POLICY == CONVGPU_BEST_FIT) {
              const uint32_t rc = RKB(c, 0);
              pr_lo |= shl_c(1u, rc) & pmask;
              pr_hi |= shl_c(1u, rc - 32u) & pmask;
            }
            const uint32_t seq0 = seq;
            if (POLICY == CONVGPU_RECENT_FIT) {
              if (pause && sp < kStack) STK(sp) = (uint8_t)c;
              sp += pause ? 1u : 0u;
              ru_scan = ru_scan || sp > kStack;
            }
            seq += pause ? 1u : 0u;
            // DISPATCH has work after a pause with no target (select) or a
            // FINISH that leaves a target to fill or paused containers
            dmode = (pause & tnone) | (isX & ((target != kNoC) | ((pm_lo | pm_hi) != 0u)));
            if (badfree) { flags |= CONVGPU_FLAG_INVALID_FREE; tdone = true; }
            const bool adv = !isX && !pause && !badfree;
            // new state word
            uint32_t nu = ust;
            nu = grant ? ((ust & ~kUsedMask) | need | kFirst) : nu;
            nu = (isF && !badfree) ? ust - r : nu;
            nu = isX ? (ust & ~kUsedMask) : nu;
            nu = pause ? (ust | kPaused) : nu;
            nu = arr ? (vadm ? kAdmitted : 0u) : nu;
            nu = (adv && !arr) ? nu + kKOne : nu;
            AT(s_ust, c) = nu;
            // admission at arrival; the suspension number (Recent-Fit scan fallback)
            sts_if(&AT(s_adm, c), arr ? (vadm ? admv : kKeyNone) : seq0,
                   arr | (POLICY == CONVGPU_RECENT_FIT && pause));
            sts_if(&AT(s_nd, c), arr ? am : t, arr | isX);  // d_1 / finish tick
            kc = badfree ? kNoC : c;
            nkc = adv ? (((t + nd) << 6) | c) : kKeyNone;
            pfk = (adv && !arr) ? ((nu >> kKShift) & 7u) : 0xFFu;
          }
        } else if (dmode) {
          // ====== one DISPATCH step at the triggering tick (R1, R9) ======
          // A step = [SELECT if there is no fill target] + fill / resume / admit
          // of the target; an admit keeps the lane in dispatch mode (the
          // leftover cascades to the next selection, Fig. 3d).
          const uint32_t t = cur_t;
          if (POLICY == CONVGPU_FIFO) {
            // ---- SELECT: oldest created paused container (R7);
            // cheap enough to compute always and keep only with no target ----
            const bool ns = target == kNoC;
            const uint32_t sel = ffs64(pm_lo, pm_hi);
            target = ns ? sel : target;
            a_tg = ns ? 0u : a_tg;
            n_sel += ns ? 1u : 0u;
          } else if (target == kNoC) {
            // ---- SELECT among paused; pm != 0 here ----
            uint32_t sel;
            if (POLICY == CONVGPU_BEST_FIT) {  // R3, R4: shortfall L - 0
              // R = #ranks with L <= free (limits sorted by (L, index)); a
              // branch-free binary search (mid clamped once lo == hi)
              uint32_t lo = 0, hi = n;
              if (NF == 64) {
                // groups of 8 ranks whose maximum fits, then the 8 ranks of the
                // first group that does not (all 8 loads in flight)
                uint32_t gc = 0;
#pragma unroll
                for (int j = 0; j < 8; ++j) gc += (piv[j] <= free_mem) ? 1u : 0u;
                const uint32_t rb = min(gc, 7u) * 8u;
                uint32_t in = 0;
#pragma unroll
                for (uint32_t j = 0; j < 8; ++j) in += (AT(s_L, RKB(rb + j, 2)) <= free_mem) ? 1u : 0u;
                lo = (gc == 8u) ? 64u : rb + in;
              } else {
#pragma unroll
                for (int it = 0; it < 7; ++it) {
                  const uint32_t mid = min((lo + hi) >> 1, n - 1u);
                  const bool go = lo < hi, le = AT(s_L, RKB(mid, 2)) <= free_mem;
                  lo = (go & le) ? mid + 1u : lo;
                  hi = (go & !le) ? mid : hi;
                }
              }
              uint32_t ml, mh;
              lowmask64(lo, ml, mh);
              const uint32_t fl = pr_lo & ml, fh = pr_hi & mh;
              // largest fitting limit, lowest index among equals; else the
              // smallest limit, lowest index (both computed, one kept)
              const uint32_t h = min(fls64(fl, fh), n - 1u);  // in range when nothing fits
              uint32_t gl, gh;
              lowmask64(RKB(h, 1), gl, gh);
              const uint32_t r_fit = ffs64(pr_lo & ~gl, pr_hi & ~gh);
              const uint32_t r_min = ffs64(pr_lo, pr_hi);
              sel = RKB((fl | fh) ? r_fit : r_min, 2);
            } else if (POLICY == CONVGPU_RECENT_FIT) {  // R5: most recent suspension
              if (!ru_scan) {
                while (sp > 0 && !bit64(pm_lo, pm_hi, STK(sp - 1))) --sp;  // lazy deletion
                sel = STK(sp - 1);
              } else {
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
              }
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
            a_tg = 0;
            ++n_sel;
          }
          {
            const uint32_t tg = target;
            const uint32_t Lt = AT(s_L, tg), ut = AT(s_ust, tg), cwt = AT(s_cw, tg),
                           ndt = AT(s_nd, tg);
            const uint32_t g = min(free_mem, Lt - a_tg);
            a_tg += g;
            free_mem -= g;
            const uint32_t pend = (cwt & kSizeMask) + ((ut & kFirst) ? 0u : ovh);
            const uint32_t uu = ut & kUsedMask;
            const bool res = (ut & kPaused) && uu + pend <= a_tg;  // RESUME (R9)
            const bool full = a_tg == Lt;                          // admit, cascade
            used_total += res ? pend : 0u;
            peak_res = max(peak_res, cap - free_mem);
            peak_used = max(peak_used, used_total);
            if (used_total > cap - free_mem) flags |= CONVGPU_FLAG_OVERCOMMIT;
            uint32_t nu = res ? (((ut & ~(kUsedMask | kPaused)) | (uu + pend) | kFirst) + kKOne) : ut;
            nu |= full ? kAdmitted : 0u;
            AT(s_ust, tg) = nu;
            const uint32_t rmask = res ? 0xFFFFFFFFu : 0u;  // resumed: no longer paused
            pm_lo &= ~(shl_c(1u, tg) & rmask);
            pm_hi &= ~(shl_c(1u, tg - 32u) & rmask);
            if (POLICY == CONVGPU_BEST_FIT) {
              const uint32_t rt = RKB(tg, 0);
              pr_lo &= ~(shl_c(1u, rt) & rmask);
              pr_hi &= ~(shl_c(1u, rt - 32u) & rmask);
            }
            sts_if(&AT(s_adm, tg), (t << 6) | rank, full);
            rank += full ? 1u : 0u;
            target = full ? kNoC : target;
            a_tg = full ? 0u : a_tg;
            dmode = full && (pm_lo | pm_hi) != 0u;  // another selection follows
            kc = res ? tg : kNoC;
            nkc = ((t + ndt) << 6) | tg;
            pfk = res ? ((nu >> kKShift) & 7u) : 0xFFu;
          }
        }
        // ---- shared tail: key update, group re-min, op prefetch (branch-free:
        // with no key change the store is off and group 0 is re-min'ed as is) ----
        {
          const uint32_t kcs = kc & 63u;
          sts_if(&AT(s_key, kcs), nkc, kc != kNoC);
          regroup(kcs);
          // op k word, delta of op k+1 (pfk = 0xFF: nothing to fetch)
          const uint32_t off = pfk * n + kcs;  // < 2^32: K * n per trace
          cp_async4_if(&AT(s_cw, kcs), trace_arg + off, pfk < K);
          cp_async4_if(&AT(s_nd, kcs), trace_delta + off + n, pfk + 1 < K);
          pfc = (pfk != 0xFFu) ? kcs : kNoC;
        }
        cp_commit();
      }
    } while (!__all_sync(kFull, !have || tdone));
    if (have) {
      epilogue(i);
      i = next(i + T);
      have = i < p.count;
      if (have) { init(i); tdone = flags != 0; dmode = false; }
    }
  }
#undef STK
#undef RKB
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

template <int POLICY, int NF, int KF>
static cudaError_t launch_t(const ReplayArgs& a, cudaStream_t stream) {
  // two 2-warp CTAs (four warps) per SM for every policy
  const int threads = kLptThreads;
  const size_t smem = (size_t)(threads / 32) * warp_bytes(POLICY, a.n);
  auto kern = replay_lpt_kernel<POLICY, NF, KF>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  int dev = 0, sms = 0, per_sm = 0;
  if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
  if ((e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess) return e;
  if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, threads, smem)) !=
      cudaSuccess)
    return e;
  if (per_sm < 1) return cudaErrorInvalidConfiguration;
  if (a.per_sm_cap && (uint32_t)per_sm > a.per_sm_cap) per_sm = (int)a.per_sm_cap;
  const uint64_t need = (a.count + threads - 1) / threads;
  uint64_t grid = (uint64_t)sms * (uint64_t)per_sm;
  if (a.grid_override) grid = a.grid_override;
  if (grid > need) grid = need;
  if (grid < 1) grid = 1;
  kern<<<(unsigned)grid, threads, smem, stream>>>(a);
  return cudaGetLastError();
}

}  // namespace lpt

template <int POLICY>
static cudaError_t launch_p(const ReplayArgs& a, cudaStream_t stream) {
  if (a.n == 64 && a.K == 4) return lpt::launch_t<POLICY, 64, 4>(a, stream);
  return lpt::launch_t<POLICY, 0, 0>(a, stream);
}

cudaError_t launch_replay_lpt(const ReplayArgs& a, int policy, cudaStream_t stream) {
  switch (policy) {
    case CONVGPU_FIFO: return launch_p<CONVGPU_FIFO>(a, stream);
    case CONVGPU_BEST_FIT: return launch_p<CONVGPU_BEST_FIT>(a, stream);
    case CONVGPU_RECENT_FIT: return launch_p<CONVGPU_RECENT_FIT>(a, stream);
    case CONVGPU_RANDOM_FIT: return launch_p<CONVGPU_RANDOM_FIT>(a, stream);
  }
  return cudaErrorInvalidValue;
}

}  // namespace convgpu
