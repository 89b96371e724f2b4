// replay.cu — the hot path: batched replay of ConVGPU's GPU-memory scheduler
// (§III-D, Fig. 3) on sm_100a, one warp per
// trace.
//
// Design:
//  * persistent grid-stride loop over traces, one trace per warp at a time;
//  * the next trace's SoA arrays are prefetched into a per-warp shared-memory
//    double buffer by the bulk-copy (TMA) engine — cp.async.bulk completing
//    on an mbarrier — while the warp replays the current trace;
//  * event keys (tick << 6 | container) live in registers, two containers
//    per lane; the next event is one redux.sync.min;
//  * each container's hot state is one 16-byte record {state, current op
//    word, delta to its next op, limit} in shared memory: an event is one
//    broadcast LDS.128, an advance one STS.128 (the next op's word/delta come
//    from the staged trace); the scheduler ledger (free memory, fill target,
//    counters, the 64-bit paused mask) is warp-uniform in registers, so the
//    event loop never diverges;
//  * policy selection is lane-parallel: FIFO = find-first-set of
//    the paused mask, Best-Fit = two packed redux (max fitting shortfall,
//    else min shortfall), Recent-Fit = redux.max over packed suspension
//    numbers, Random-Fit = Philox draw + popc + fns;
//  * outputs, the R20 digest and a warp -> block -> grid statistics reduction
//    are fused into the trace epilogue / kernel tail.
#include <cuda_runtime.h>
#include <stdint.h>

#include "common.cuh"
#include "internal.h"

namespace convgpu {
namespace wpt {

// state word: used (26 bits) | k << 26 (3 bits) | FIRST | PAUSED | ADMITTED;
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

struct WarpStats {  // 96 B, per warp, shared memory
  unsigned long long traces, events, sum_makespan, sum_wait, n_rejected, n_select, digest_sum;
  uint32_t max_makespan, max_peak_reserved;
  uint32_t flag_count[8];
};
static_assert(sizeof(WarpStats) == 96, "WarpStats layout");

// Per-warp shared memory: header (2 mbarriers, WarpStats, range accumulator)
// | cs[64] {state, cw, nd, L} | cx[64] {wait, adm} | 2 x staged trace.
// cs.nd: delta to add at the container's next scheduling (d_0 before
//        arrival, then d_{k+1}); after FINISH it holds the finish tick.
// cx.wait: d_1 before arrival, then the suspended-time accumulator.
// cx.adm: admission (tick << 6 | rank); suspension number while paused.
constexpr uint32_t kHeaderBytes = 128;
// ca[64]: explicit assignment a per container, used only by the literal
// reading R1-LIT (partial holds are kept, so a is not derivable).
constexpr uint32_t kCsBytes = 64 * 16, kCxBytes = 64 * 8, kCaBytes = 64 * 4;

__host__ __device__ inline uint32_t in_words(uint32_t n, uint32_t K) { return (2 + 2 * K) * n; }
__host__ __device__ inline uint32_t warp_region_bytes(uint32_t n, uint32_t K) {
  uint32_t b = kHeaderBytes + kCsBytes + kCxBytes + kCaBytes + 2 * in_words(n, K) * 4;
  return (b + 15u) & ~15u;
}

// ---------------------------------------------------------------- TMA bits
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(bar)));
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("{\n\t.reg .b64 st;\n\tmbarrier.arrive.expect_tx.shared::cta.b64 st, [%0], %1;\n\t}" ::"r"(
                   smem_u32(bar)),
               "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra WAIT_%=;\n\t}" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ uint32_t redux_min(uint32_t v) {
  uint32_t r;
  asm volatile("redux.sync.min.u32 %0, %1, 0xffffffff;" : "=r"(r) : "r"(v));
  return r;
}
__device__ __forceinline__ uint32_t redux_max(uint32_t v) {
  uint32_t r;
  asm volatile("redux.sync.max.u32 %0, %1, 0xffffffff;" : "=r"(r) : "r"(v));
  return r;
}

// ---------------------------------------------------------------- kernel
// A write to the per-warp scheduler state (the warp runs one trace with
// warp-uniform control flow, so every lane holds the same value): the warp
// syncs so every lane's earlier read of the location is done, one lane
// stores, and the warp syncs again so every later read sees the store.
#define WSTORE(lhs, val)                  \
  do {                                    \
    const auto wstore_v_ = (val);         \
    __syncwarp();                         \
    if (lane == 0) (lhs) = wstore_v_;     \
    __syncwarp();                         \
  } while (0)
// two writes with no read of either location between them: one sync pair
#define WSTORE2(l1, v1, l2, v2)           \
  do {                                    \
    const auto wstore_v1_ = (v1);         \
    const auto wstore_v2_ = (v2);         \
    __syncwarp();                         \
    if (lane == 0) {                      \
      (l1) = wstore_v1_;                  \
      (l2) = wstore_v2_;                  \
    }                                     \
    __syncwarp();                         \
  } while (0)

// NF: compile-time container count (64) or 0 = runtime p.n.
// LIT: the literal re-select-on-every-release reading R1-LIT (NEXT-1).
template <int POLICY, bool BULK, int NF, bool LIT>
__global__ void __launch_bounds__(kReplayThreads, 8) replay_kernel(const ReplayArgs p) {
  extern __shared__ __align__(16) unsigned char smem[];
  const uint32_t lane = threadIdx.x & 31u, lane32 = lane + 32u;
  const uint32_t wib = threadIdx.x >> 5;
  const uint32_t n = NF ? (uint32_t)NF : p.n;
  const uint32_t K = p.K, cap = p.cap, ovh = p.ovh;
  const uint32_t IN = in_words(n, K);
  unsigned char* base = smem + wib * warp_region_bytes(n, K);
  uint64_t* mbar = reinterpret_cast<uint64_t*>(base);
  WarpStats* ws = reinterpret_cast<WarpStats*>(base + 16);
  unsigned long long* racc = reinterpret_cast<unsigned long long*>(base + 112);  // [cur, acc]
  uint4* cs = reinterpret_cast<uint4*>(base + kHeaderBytes);
  uint2* cx = reinterpret_cast<uint2*>(base + kHeaderBytes + kCsBytes);
  uint32_t* ca = reinterpret_cast<uint32_t*>(base + kHeaderBytes + kCsBytes + kCxBytes);
  uint32_t* inbuf = reinterpret_cast<uint32_t*>(base + kHeaderBytes + kCsBytes + kCxBytes + kCaBytes);

  const uint64_t warps_per_block = blockDim.x >> 5;
  const uint64_t gw = (uint64_t)blockIdx.x * warps_per_block + wib;
  const uint64_t W = (uint64_t)gridDim.x * warps_per_block;

  if (lane == 0) {
    unsigned long long* z = reinterpret_cast<unsigned long long*>(ws);
#pragma unroll
    for (int j = 0; j < 12; ++j) z[j] = 0ull;
    racc[0] = ~0ull;
    racc[1] = 0ull;
    if (BULK) {
      mbar_init(&mbar[0]);
      mbar_init(&mbar[1]);
      asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
  }
  __syncwarp();

  auto prefetch = [&](uint64_t i, uint32_t b) {
    uint32_t* dst = inbuf + b * IN;
    if (BULK) {
      if (lane == 0) {
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        const uint32_t nb = n * 4u, knb = K * n * 4u;
        mbar_expect_tx(&mbar[b], 2u * nb + 2u * knb);
        bulk_g2s(dst, p.arrival + i * n, nb, &mbar[b]);
        bulk_g2s(dst + n, p.limit + i * n, nb, &mbar[b]);
        bulk_g2s(dst + 2 * n, p.delta + i * (uint64_t)K * n, knb, &mbar[b]);
        bulk_g2s(dst + 2 * n + K * n, p.arg + i * (uint64_t)K * n, knb, &mbar[b]);
      }
    } else {
      for (uint32_t j = lane; j < n; j += 32) {
        dst[j] = __ldg(p.arrival + i * n + j);
        dst[n + j] = __ldg(p.limit + i * n + j);
      }
      const uint64_t ob = i * (uint64_t)K * n;
      for (uint32_t j = lane; j < K * n; j += 32) {
        dst[2 * n + j] = __ldg(p.delta + ob + j);
        dst[2 * n + K * n + j] = __ldg(p.arg + ob + j);
      }
    }
  };

  uint32_t phase = 0;  // bit b = parity to wait for on buffer b
  if (BULK && gw < p.count) prefetch(gw, 0);

  uint64_t j = 0;
  for (uint64_t i = gw; i < p.count; i += W, ++j) {
    const uint32_t b = (uint32_t)(j & 1);
    if (BULK) {
      if (i + W < p.count) prefetch(i + W, b ^ 1u);
      mbar_wait(&mbar[b], (phase >> b) & 1u);
      phase ^= 1u << b;
    } else {
      // fallback pass of the compact kernel (R1-LIT): only the traces it marked
      if (p.only_marked && p.adm_buf()[i * n] != p.only_marked) continue;
      __syncwarp();
      prefetch(i, 0);
      __syncwarp();
    }
    const uint32_t* A = inbuf + (BULK ? b * IN : 0);
    const uint32_t* Lm = A + n;
    const uint32_t* D = A + 2 * n;
    const uint32_t* R = A + 2 * n + K * n;
    const uint64_t tid = p.tid_base + i;

    // ---- per-trace init + static validation (DESIGN.md §2 Flags) ----
    uint32_t key0 = kKeyNone, key1 = kKeyNone;
    uint32_t bad = 0, lsum = 0, lmax = 0;
#pragma unroll
    for (uint32_t s = 0; s < 2; ++s) {
      const uint32_t c = lane + 32u * s;
      if (c < n) {
        const uint32_t a = A[c], L = Lm[c];
        if (L > cap) bad |= CONVGPU_FLAG_INVALID_LIMIT;
        if (c > 0 && a < A[c - 1]) bad |= CONVGPU_FLAG_UNSORTED_ARRIVAL;
        lmax = max(lmax, a);
        for (uint32_t k = 0; k < K; ++k) {
          lsum = min(lsum + min(D[k * n + c], kTickLimit), kTickLimit);
          const bool fin = (R[k * n + c] >> 30) == CONVGPU_OP_FINISH;
          if (fin != (k + 1 == K)) bad |= CONVGPU_FLAG_BAD_PROGRAM;
        }
        cs[c] = make_uint4(kNotArrived, R[c], D[c], L);
        cx[c] = make_uint2(K > 1 ? D[n + c] : 0u, kKeyNone);
        if (LIT) ca[c] = 0;
        const uint32_t key = (min(a, kTickLimit - 1) << 6) | c;
        if (s == 0) key0 = key; else key1 = key;
      }
    }
    uint32_t flags = __reduce_or_sync(kFull, bad);
    {
      const uint32_t tot = __reduce_add_sync(kFull, lsum);
      const uint32_t amax = __reduce_max_sync(kFull, lmax);
      if (amax >= kTickLimit || amax + tot >= kTickLimit) flags |= CONVGPU_FLAG_TICK_RANGE;
    }
    __syncwarp();

    // ---- uniform scheduler ledger (D4, D1 target, counters) ----
    uint32_t free_mem = cap, target = kTargetNone, a_tg = 0, used_total = 0;
    uint32_t seq = 0, rank = 0, draws = 0, n_rej = 0, n_sel = 0;
    uint32_t peak_res = 0, peak_used = 0, live = n, events = 0;
    uint32_t pm_lo = 0, pm_hi = 0;  // paused set (D3) as a 64-bit mask

    if (flags == 0) {
      for (;;) {
        const uint32_t kmin = redux_min(min(key0, key1));
        if (kmin == kKeyNone) {
          if (live) flags |= CONVGPU_FLAG_DEADLOCK;  // P:7
          break;
        }
        const uint32_t t = kmin >> 6, c = kmin & 63u;
        ++events;
        const uint4 s = cs[c];
        uint32_t ust = s.x;
        const uint32_t L = s.w;
        uint32_t nk = kKeyNone;
        bool disp = false;
        if ((ust & kNotArrived) == kNotArrived) {
          // ARRIVE (Fig. 3b/3c; R2)
          const uint32_t g = (LIT || target == kTargetNone) ? min(L, free_mem) : 0u;
          free_mem -= g;
          peak_res = max(peak_res, cap - free_mem);
          if (used_total > cap - free_mem) flags |= CONVGPU_FLAG_OVERCOMMIT;
          uint32_t adm = kKeyNone;
          ust = 0;
          if (LIT) WSTORE(ca[c], g);
          if (g == L) {
            adm = (t << 6) | rank; ++rank; ust = kAdmitted;
          } else if (g > 0 && !LIT) {
            target = c; a_tg = g;
          }
          const uint32_t d1 = cx[c].x;
          WSTORE2(cx[c], make_uint2(0u, adm), cs[c], make_uint4(ust, s.y, d1, L));
          nk = ((t + s.z) << 6) | c;
        } else {
          const uint32_t cw = s.y;
          const uint32_t kind = cw >> 30, r = cw & kSizeMask, used = ust & kUsedMask;
          bool adv = true;
          if (kind == CONVGPU_OP_ALLOC) {
            const uint32_t need = used + r + ((ust & kFirst) ? 0u : ovh);
            const uint32_t a = LIT ? ca[c] : ((ust & kAdmitted) ? L : (c == target ? a_tg : 0u));
            if (need > L) {
              ++n_rej;  // R10
            } else if (need <= a) {
              used_total += need - used;
              peak_used = max(peak_used, used_total);
              if (used_total > cap - free_mem) flags |= CONVGPU_FLAG_OVERCOMMIT;
              ust = (ust & ~kUsedMask) | need | kFirst;
            } else {  // pause: reply withheld
              ust |= kPaused;
              const uint32_t wv = cx[c].x - t;
              WSTORE2(cx[c], make_uint2(wv, POLICY == CONVGPU_RECENT_FIT ? seq : kKeyNone), cs[c].x, ust);
              ++seq;
              if (c < 32) pm_lo |= 1u << c; else pm_hi |= 1u << (c - 32);
              adv = false;
              disp = LIT || (target == kTargetNone);
            }
          } else if (kind == CONVGPU_OP_FREE) {  // P:110, R11
            if (r > used) { flags |= CONVGPU_FLAG_INVALID_FREE; break; }
            ust -= r;
            used_total -= r;
          } else if (kind == CONVGPU_OP_FINISH) {  // P:110, R18
            const uint32_t a = LIT ? ca[c] : ((ust & kAdmitted) ? L : (c == target ? a_tg : 0u));
            free_mem += a;
            used_total -= used;
            --live;
            if (c == target) { target = kTargetNone; a_tg = 0; }  // R20
            WSTORE(cs[c], make_uint4(ust & ~kUsedMask, cw, t, L));  // nd := finish tick
            adv = false;
            disp = true;
          }
          if (adv) {
            const uint32_t k = ((ust >> kKShift) & 7u) + 1u;
            nk = ((t + s.z) << 6) | c;
            ust = (ust & ~kKMask) | (k << kKShift);
            const uint32_t ncw = R[k * n + c];
            const uint32_t nnd = (k + 1 < K) ? D[(k + 1) * n + c] : 0u;
            WSTORE(cs[c], make_uint4(ust, ncw, nnd, L));
          }
        }
        key0 = (c == lane) ? nk : key0;
        key1 = (c == lane32) ? nk : key1;

        // ---- DISPATCH (Fig. 3d; R1, R9) ----
        // ---- SELECT among paused ----
        auto select_paused = [&]() -> uint32_t {
          uint32_t sel;
          if (POLICY == CONVGPU_FIFO) {  // oldest created (R7)
            sel = pm_lo ? (uint32_t)(__ffs(pm_lo) - 1) : 32u + (uint32_t)(__ffs(pm_hi) - 1);
          } else if (POLICY == CONVGPU_BEST_FIT) {  // R3, R4: shortfall L - a (a = 0 when selectable under R1)
            uint32_t vf = 0, vm = kKeyNone;
            if ((pm_lo >> lane) & 1u) {
              const uint32_t need = Lm[lane] - (LIT ? ca[lane] : 0u);
              if (need <= free_mem) vf = (need << 6) | (63u - lane);
              vm = (need << 6) | lane;
            }
            if (lane32 < n && ((pm_hi >> lane) & 1u)) {
              const uint32_t need = Lm[lane32] - (LIT ? ca[lane32] : 0u);
              if (need <= free_mem) vf = max(vf, (need << 6) | (63u - lane32));
              vm = min(vm, (need << 6) | lane32);
            }
            const uint32_t kf = redux_max(vf);
            sel = kf ? 63u - (kf & 63u) : (redux_min(vm) & 63u);
          } else if (POLICY == CONVGPU_RECENT_FIT) {  // R5
            uint32_t v = 0;
            if ((pm_lo >> lane) & 1u) v = ((cx[lane].y + 1u) << 6) | lane;
            if (lane32 < n && ((pm_hi >> lane) & 1u)) v = max(v, ((cx[lane32].y + 1u) << 6) | lane32);
            sel = redux_max(v) & 63u;
          } else {  // RANDOM_FIT (R6)
            const uint32_t clo = __popc(pm_lo);
            const uint32_t m = clo + __popc(pm_hi);
            const U4 x = philox4x32_10((uint32_t)tid, (uint32_t)(tid >> 32), draws, 1u,
                                       (uint32_t)p.seed, (uint32_t)(p.seed >> 32));
            ++draws;
            const uint32_t jj = __umulhi(x.x, m);
            sel = (jj < clo) ? __fns(pm_lo, 0, jj + 1) : 32u + __fns(pm_hi, 0, jj - clo + 1);
          }
          return sel;
        };
        if (disp && LIT) {
          // R1-LIT: while memory is free and someone is paused, the policy's
          // pick receives min(free, L - a); partial holds are kept.
          while (free_mem != 0 && (pm_lo | pm_hi) != 0u) {
            const uint32_t x = select_paused();
            ++n_sel;
            uint4 st = cs[x];
            const uint32_t Lx = st.w;
            const uint32_t g = min(free_mem, Lx - ca[x]);
            const uint32_t ax = ca[x] + g;
            WSTORE(ca[x], ax);
            free_mem -= g;
            peak_res = max(peak_res, cap - free_mem);
            uint32_t ut = st.x;
            if (ut & kPaused) {
              const uint32_t pend = (st.y & kSizeMask) + ((ut & kFirst) ? 0u : ovh);
              const uint32_t uu = ut & kUsedMask;
              if (uu + pend <= ax) {  // RESUME (R9)
                used_total += pend;
                peak_used = max(peak_used, used_total);
                WSTORE(cx[x], make_uint2(cx[x].x + t, kKeyNone));
                if (x < 32) pm_lo &= ~(1u << x); else pm_hi &= ~(1u << (x - 32));
                const uint32_t k = ((ut >> kKShift) & 7u) + 1u;
                ut = (ut & ~(kUsedMask | kKMask | kPaused)) | (uu + pend) | kFirst | (k << kKShift);
                const uint32_t nkx = ((t + st.z) << 6) | x;
                key0 = (x == lane) ? nkx : key0;
                key1 = (x == lane32) ? nkx : key1;
                st.y = R[k * n + x];
                st.z = (k + 1 < K) ? D[(k + 1) * n + x] : 0u;
              }
            }
            if (used_total > cap - free_mem) flags |= CONVGPU_FLAG_OVERCOMMIT;
            if (ax == Lx) { WSTORE(cx[x].y, (t << 6) | rank); ++rank; ut |= kAdmitted; }
            WSTORE(cs[x], make_uint4(ut, st.y, st.z, Lx));
          }
        } else if (disp) {
          for (;;) {
            if (target != kTargetNone) {
              const uint32_t tg = target;
              uint4 st = cs[tg];
              const uint32_t Lt = st.w;
              const uint32_t g = min(free_mem, Lt - a_tg);
              a_tg += g;
              free_mem -= g;
              peak_res = max(peak_res, cap - free_mem);
              if (used_total > cap - free_mem) flags |= CONVGPU_FLAG_OVERCOMMIT;
              uint32_t ut = st.x;
              if (ut & kPaused) {
                const uint32_t pend = (st.y & kSizeMask) + ((ut & kFirst) ? 0u : ovh);
                const uint32_t uu = ut & kUsedMask;
                if (uu + pend <= a_tg) {  // RESUME (R9)
                  used_total += pend;
                  peak_used = max(peak_used, used_total);
                  if (used_total > cap - free_mem) flags |= CONVGPU_FLAG_OVERCOMMIT;
                  WSTORE(cx[tg], make_uint2(cx[tg].x + t, kKeyNone));
                  if (tg < 32) pm_lo &= ~(1u << tg); else pm_hi &= ~(1u << (tg - 32));
                  const uint32_t k = ((ut >> kKShift) & 7u) + 1u;
                  ut = (ut & ~(kUsedMask | kKMask | kPaused)) | (uu + pend) | kFirst | (k << kKShift);
                  const uint32_t nkt = ((t + st.z) << 6) | tg;
                  key0 = (tg == lane) ? nkt : key0;
                  key1 = (tg == lane32) ? nkt : key1;
                  st.y = R[k * n + tg];
                  st.z = (k + 1 < K) ? D[(k + 1) * n + tg] : 0u;
                }
              }
              if (a_tg == Lt) {  // fully guaranteed: admit, cascade leftover
                WSTORE2(cx[tg].y, (t << 6) | rank, cs[tg], make_uint4(ut | kAdmitted, st.y, st.z, Lt));
                ++rank;
                target = kTargetNone;
                a_tg = 0;
                continue;
              }
              WSTORE(cs[tg], make_uint4(ut, st.y, st.z, Lt));
              break;
            }
            if ((pm_lo | pm_hi) == 0u) break;
            const uint32_t sel = select_paused();
            target = sel;
            a_tg = 0;
            ++n_sel;
          }
        }
      }
    }

    // ---- epilogue: outputs, digest (R20), statistics ----
    __syncwarp();
    const bool stopped = (flags & kStopMask) != 0;
    if (stopped) { peak_res = 0; peak_used = 0; n_rej = 0; n_sel = 0; }
    uint64_t dig = 0;
    uint32_t mfin = 0, wlo = 0, whi = 0;
#pragma unroll
    for (uint32_t s = 0; s < 2; ++s) {
      const uint32_t c = lane + 32u * s;
      if (c < n) {
        uint32_t at = kKeyNone, ar = 0xFFu, wt = 0, fn = 0;
        if (!stopped) {
          const uint4 st = cs[c];
          const uint2 sx = cx[c];
          if (st.x & kAdmitted) { at = sx.y >> 6; ar = sx.y & 63u; }
          wt = sx.x;
          fn = st.z;
        }
        const uint64_t gi = i * n + c;
        if (p.admit_tick) p.admit_tick[gi] = at;
        if (p.admit_rank) p.admit_rank[gi] = (uint8_t)ar;
        if (p.wait) p.wait[gi] = wt;
        if (p.finish) p.finish[gi] = fn;
        const uint64_t h1 = mix64(((uint64_t)c << 56) ^ ((uint64_t)ar << 48) ^ (uint64_t)at);
        dig += mix64(h1 ^ (((uint64_t)wt << 32) | fn));
        mfin = max(mfin, fn);
        wlo += wt & 0xFFFFu;
        whi += wt >> 16;
      }
    }
    dig = warp_sum_u64(dig);
    mfin = __reduce_max_sync(kFull, mfin);
    const uint64_t sum_wait =
        ((uint64_t)__reduce_add_sync(kFull, whi) << 16) + (uint64_t)__reduce_add_sync(kFull, wlo);
    const uint32_t makespan = stopped ? 0u : mfin - A[0];
    if (lane == 0) {
      dig += mix64(((uint64_t)makespan << 32) | peak_res);
      dig += mix64(((uint64_t)peak_used << 32) | flags);
      dig += mix64(sum_wait);
      dig += mix64(((uint64_t)n_rej << 32) | n_sel);
      if (p.summary) {
        convgpu_summary_t sm;
        sm.makespan = makespan; sm.peak_reserved = peak_res; sm.peak_used = peak_used;
        sm.flags = flags; sm.sum_wait = sum_wait; sm.n_rejected = n_rej; sm.n_select = n_sel;
        sm.digest = dig;
        p.summary[i] = sm;
      }
      ws->traces += 1; ws->events += events; ws->sum_makespan += makespan;
      ws->sum_wait += sum_wait; ws->n_rejected += n_rej; ws->n_select += n_sel;
      ws->digest_sum += dig;
      ws->max_makespan = max(ws->max_makespan, makespan);
      ws->max_peak_reserved = max(ws->max_peak_reserved, peak_res);
      for (int bit = 0; bit < 8; ++bit) ws->flag_count[bit] += (flags >> bit) & 1u;
      if (p.range_digest) {
        const unsigned long long r = tid / p.range_size;
        if (r != racc[0]) {
          if (racc[0] != ~0ull) atomicAdd((unsigned long long*)&p.range_digest[racc[0]], racc[1]);
          racc[0] = r;
          racc[1] = 0;
        }
        racc[1] += dig;
      }
    }
    __syncwarp();
  }

  // ---- tail: flush range digest, block -> grid statistics ----
  if (lane == 0 && p.range_digest && racc[0] != ~0ull)
    atomicAdd((unsigned long long*)&p.range_digest[racc[0]], racc[1]);
  __syncthreads();
  if (threadIdx.x == 0 && p.stats) {
    WarpStats tot = *reinterpret_cast<WarpStats*>(smem + 16);
    const uint32_t rb = warp_region_bytes(n, K);
    for (uint32_t w = 1; w < warps_per_block; ++w) {
      const WarpStats* o = reinterpret_cast<const WarpStats*>(smem + w * rb + 16);
      tot.traces += o->traces; tot.events += o->events; tot.sum_makespan += o->sum_makespan;
      tot.sum_wait += o->sum_wait; tot.n_rejected += o->n_rejected; tot.n_select += o->n_select;
      tot.digest_sum += o->digest_sum;
      tot.max_makespan = max(tot.max_makespan, o->max_makespan);
      tot.max_peak_reserved = max(tot.max_peak_reserved, o->max_peak_reserved);
      for (int bit = 0; bit < 8; ++bit) tot.flag_count[bit] += o->flag_count[bit];
    }
    if (tot.traces) {
      convgpu_stats_t* S = p.stats;
      atomicAdd((unsigned long long*)&S->traces, tot.traces);
      atomicAdd((unsigned long long*)&S->events, tot.events);
      atomicAdd((unsigned long long*)&S->sum_makespan, tot.sum_makespan);
      atomicAdd((unsigned long long*)&S->sum_wait, tot.sum_wait);
      atomicAdd((unsigned long long*)&S->n_rejected, tot.n_rejected);
      atomicAdd((unsigned long long*)&S->n_select, tot.n_select);
      atomicAdd((unsigned long long*)&S->digest_sum, tot.digest_sum);
      atomicMax(&S->max_makespan, tot.max_makespan);
      atomicMax(&S->max_peak_reserved, tot.max_peak_reserved);
      for (int bit = 0; bit < 8; ++bit)
        if (tot.flag_count[bit]) atomicAdd(&S->flag_count[bit], tot.flag_count[bit]);
    }
  }
}

// ---------------------------------------------------------------- launcher
template <int POLICY, bool BULK, int NF, bool LIT>
static cudaError_t launch_t(const ReplayArgs& a, cudaStream_t stream) {
  const uint32_t warps = kReplayThreads / 32;
  const size_t smem = (size_t)warps * warp_region_bytes(a.n, a.K);
  auto kern = replay_kernel<POLICY, BULK, NF, LIT>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  int dev = 0, sms = 0, per_sm = 0;
  if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
  if ((e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess) return e;
  if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, kReplayThreads, smem)) !=
      cudaSuccess)
    return e;
  if (per_sm < 1) per_sm = 1;
  const uint64_t need = (a.count + warps - 1) / warps;
  uint64_t grid = (uint64_t)sms * (uint64_t)per_sm;
  if (a.grid_override) grid = a.grid_override;
  if (grid > need) grid = need;
  if (grid < 1) grid = 1;
  kern<<<(unsigned)grid, kReplayThreads, smem, stream>>>(a);
  return cudaGetLastError();
}

template <int POLICY>
static cudaError_t launch_p(const ReplayArgs& a, bool bulk, bool lit, cudaStream_t stream) {
  if (lit) return bulk ? launch_t<POLICY, true, 0, true>(a, stream) : launch_t<POLICY, false, 0, true>(a, stream);
  if (a.n == 64)
    return bulk ? launch_t<POLICY, true, 64, false>(a, stream) : launch_t<POLICY, false, 64, false>(a, stream);
  return bulk ? launch_t<POLICY, true, 0, false>(a, stream) : launch_t<POLICY, false, 0, false>(a, stream);
}

#undef WSTORE2
#undef WSTORE
}  // namespace wpt

cudaError_t launch_replay(const ReplayArgs& a, int policy, bool bulk, cudaStream_t stream) {
  const bool lit = (policy & CONVGPU_DISPATCH_LITERAL) != 0;
  switch (policy & 0xFF) {
    case CONVGPU_FIFO: return wpt::launch_p<CONVGPU_FIFO>(a, bulk, lit, stream);
    case CONVGPU_BEST_FIT: return wpt::launch_p<CONVGPU_BEST_FIT>(a, bulk, lit, stream);
    case CONVGPU_RECENT_FIT: return wpt::launch_p<CONVGPU_RECENT_FIT>(a, bulk, lit, stream);
    case CONVGPU_RANDOM_FIT: return wpt::launch_p<CONVGPU_RANDOM_FIT>(a, bulk, lit, stream);
  }
  return cudaErrorInvalidValue;
}

}  // namespace convgpu
