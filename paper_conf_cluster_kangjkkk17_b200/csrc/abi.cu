// abi.cu — the extern "C" boundary of libconvgpu.so (include/convgpu.h):
// argument validation, device check, error mapping, launch configuration and
// the chunked host-memory end-to-end path.  Every computation runs in the
// kernels of replay.cu / generate.cu.
#include <cuda_runtime.h>
#include <errno.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include "convgpu.h"
#include "internal.h"

namespace {

thread_local char g_err[256];

int fail_cuda(cudaError_t e, const char* where) {
  snprintf(g_err, sizeof g_err, "%s: %s (%s)", where, cudaGetErrorString(e), cudaGetErrorName(e));
  cudaGetLastError();  // clear sticky-free errors
  return -EIO;
}

int check_device() {
  int dev = 0, major = 0, minor = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e == cudaErrorNoDevice ? -ENODEV : fail_cuda(e, "cudaGetDevice");
  if (cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev) != cudaSuccess ||
      cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, dev) != cudaSuccess)
    return -ENODEV;
  if (major != 10 || minor != 0) return -ENODEV;  // built for sm_100a only
  return 0;
}

// Device (or managed) memory on the current device.
bool is_device_ptr(const void* p) {
  if (!p) return false;
  cudaPointerAttributes at;
  if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return at.type == cudaMemoryTypeDevice || at.type == cudaMemoryTypeManaged;
}

bool opt_device_ptr(const void* p) { return p == nullptr || is_device_ptr(p); }

bool aligned16(const void* p) { return ((uintptr_t)p & 15u) == 0; }

int validate_shape(const convgpu_traces_t* t, uint32_t cap, int policy) {
  if (!t) return -EINVAL;
  if (t->n_containers < 1 || t->n_containers > CONVGPU_MAX_CONTAINERS) return -EINVAL;
  if (t->n_ops < 1 || t->n_ops > CONVGPU_MAX_OPS) return -EINVAL;
  if (policy < 0 || (policy & ~(0xFF | CONVGPU_DISPATCH_LITERAL)) || (policy & 0xFF) > 3)
    return -EINVAL;
  if ((policy & CONVGPU_DISPATCH_LITERAL) && t->kernel_variant == CONVGPU_KERNEL_LANE_PER_TRACE)
    return -EINVAL;
  if (cap == 0 || cap >= CONVGPU_CAPACITY_LIMIT) return -EINVAL;
  if (t->ctx_overhead_mib >= CONVGPU_OVERHEAD_LIMIT) return -EINVAL;
  if (t->kernel_variant > CONVGPU_KERNEL_LANE_COMPACT_WIDE) return -EINVAL;
  return 0;
}

int validate_arrays(const convgpu_traces_t* t) {
  if (!t->arrival || !t->limit || !t->op_delta || !t->op_arg) return -EINVAL;
  return 0;
}

convgpu::ReplayArgs make_args(const convgpu_traces_t* t, uint64_t n, uint32_t cap) {
  convgpu::ReplayArgs a;
  memset(&a, 0, sizeof a);
  a.arrival = t->arrival; a.limit = t->limit; a.delta = t->op_delta; a.arg = t->op_arg;
  a.n = t->n_containers; a.K = t->n_ops;
  a.tid_base = t->trace_id_base; a.seed = t->rand_seed;
  a.ovh = t->ctx_overhead_mib; a.cap = cap; a.count = n;
  if (const char* s = getenv("CONVGPU_PER_SM_CAP")) a.per_sm_cap = (uint32_t)strtoul(s, nullptr, 10);
  return a;
}

bool aligned32(const void* p) { return ((uintptr_t)p & 31u) == 0; }

bool use_bulk(const convgpu::ReplayArgs& a) {
  return (a.n % 4u) == 0 && aligned16(a.arrival) && aligned16(a.limit) && aligned16(a.delta) &&
         aligned16(a.arg);
}

// Kernel choice for CONVGPU_KERNEL_AUTO (measured on B200, config [2] traces,
// scripts/gpu_small.sh): a lane-per-trace launch costs one "round" (~0.17-
// 0.24 ms per policy) for any batch up to its 18,944 (32-bit) / 37,888
// (compact) lanes; warp-per-trace holds 4,736 traces in flight at ~0.16 ms
// per 4,736.  Crossover ~40 traces per SM: warp-per-trace at 1,000-4,736
// traces (0.09-0.16 vs 0.17-0.24 ms), lane kernels 2x faster from 9,472.
// (policy is accepted for per-policy tuning; all four currently agree.)
uint32_t auto_variant(uint64_t count, int policy) {
  (void)policy;
  int dev = 0, sms = 148;
  if (cudaGetDevice(&dev) == cudaSuccess) cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const bool big = count >= (uint64_t)sms * 40u;
  return big ? CONVGPU_KERNEL_LANE_PER_TRACE : CONVGPU_KERNEL_WARP_PER_TRACE;
}

cudaError_t launch_any(convgpu::ReplayArgs a, int policy, uint32_t variant, cudaStream_t s) {
  a.aligned16 = use_bulk(a) && aligned16(a.admit_tick) && aligned16(a.adm_scratch) &&
                aligned16(a.wait) && aligned16(a.finish) && ((uintptr_t)a.admit_rank & 3u) == 0;
  // 32-byte loads of the trace and the admissions, 32-byte output stores
  a.aligned32 = (a.n % 8u) == 0 && aligned32(a.arrival) && aligned32(a.limit) && aligned32(a.delta) &&
                aligned32(a.arg) && aligned32(a.admit_tick) && aligned32(a.adm_scratch) &&
                aligned32(a.wait) && aligned32(a.finish) && ((uintptr_t)a.admit_rank & 7u) == 0;
  if (variant == CONVGPU_KERNEL_AUTO) {
    variant = auto_variant(a.count, policy);
    if (variant == CONVGPU_KERNEL_LANE_PER_TRACE && convgpu::lpt16_supported(a))
      variant = CONVGPU_KERNEL_LANE_COMPACT;
  }
  // R1-LIT runs on the compact kernel or the warp-per-trace kernel
  if ((policy & CONVGPU_DISPATCH_LITERAL) && variant == CONVGPU_KERNEL_LANE_PER_TRACE)
    variant = CONVGPU_KERNEL_WARP_PER_TRACE;
  if (variant == CONVGPU_KERNEL_LANE_COMPACT || variant == CONVGPU_KERNEL_LANE_COMPACT_WIDE) {
    if (!convgpu::lpt16_supported(a)) return cudaErrorInvalidValue;  // -EINVAL, see convgpu_replay
    return convgpu::launch_replay_lpt16(a, policy, s, variant == CONVGPU_KERNEL_LANE_COMPACT_WIDE);
  }
  if (variant == CONVGPU_KERNEL_LANE_PER_TRACE) return convgpu::launch_replay_lpt(a, policy, s);
  return convgpu::launch_replay(a, policy, use_bulk(a), s);
}

}  // namespace

extern "C" {

int convgpu_abi_version(void) { return CONVGPU_ABI_VERSION; }

int convgpu_launches_per_call(void) { return 3; }  // compact lane kernel + its 17-bit and 32-bit fallback passes

const char* convgpu_strerror(int rc) {
  switch (rc) {
    case 0: return "success";
    case -EINVAL: return "invalid argument (see include/convgpu.h)";
    case -ENODEV: return "no sm_100 (B200-class) CUDA device is current";
    case -EIO: return g_err[0] ? g_err : "CUDA error";
    default: return "unknown error";
  }
}

int convgpu_replay(const convgpu_traces_t* traces, uint64_t n, uint32_t capacity_mib, int policy,
                   const convgpu_out_t* out) {
  int rc = validate_shape(traces, capacity_mib, policy);
  if (rc) return rc;
  if (!out) return -EINVAL;
  if (out->range_digest && out->range_size == 0) return -EINVAL;
  if ((traces->kernel_variant == CONVGPU_KERNEL_LANE_COMPACT ||
       traces->kernel_variant == CONVGPU_KERNEL_LANE_COMPACT_WIDE) &&
      (traces->n_containers != 64 || traces->n_ops != 4 || (!out->admit_tick && !out->admit_scratch)))
    return -EINVAL;
  if (n == 0) return 0;  // no-op: array pointers may be NULL
  if ((rc = validate_arrays(traces))) return rc;
  if ((rc = check_device())) return rc;
  if (!is_device_ptr(traces->arrival) || !is_device_ptr(traces->limit) ||
      !is_device_ptr(traces->op_delta) || !is_device_ptr(traces->op_arg))
    return -EINVAL;
  if (!opt_device_ptr(out->admit_tick) || !opt_device_ptr(out->admit_rank) ||
      !opt_device_ptr(out->wait) || !opt_device_ptr(out->finish) ||
      !opt_device_ptr(out->summary) || !opt_device_ptr(out->stats) ||
      !opt_device_ptr(out->range_digest) || !opt_device_ptr(out->admit_scratch))
    return -EINVAL;
  convgpu::ReplayArgs a = make_args(traces, n, capacity_mib);
  a.admit_tick = out->admit_tick; a.admit_rank = out->admit_rank;
  a.wait = out->wait; a.finish = out->finish;
  a.summary = out->summary; a.stats = out->stats;
  a.range_digest = out->range_digest; a.range_size = out->range_size;
  a.adm_scratch = out->admit_scratch;
  if (traces->kernel_variant == CONVGPU_KERNEL_LANE_COMPACT ||
      traces->kernel_variant == CONVGPU_KERNEL_LANE_COMPACT_WIDE) {
    a.aligned16 = use_bulk(a) && aligned16(a.admit_tick) && aligned16(a.adm_scratch) &&
                  aligned16(a.wait) && aligned16(a.finish) && ((uintptr_t)a.admit_rank & 3u) == 0;
    if (!convgpu::lpt16_supported(a)) return -EINVAL;
  }
  cudaError_t e = launch_any(a, policy, traces->kernel_variant, (cudaStream_t)out->stream);
  return e == cudaSuccess ? 0 : fail_cuda(e, "replay launch");
}

int convgpu_generate(const convgpu_gen_params_t* p, uint64_t trace_id_base, uint64_t n,
                     const convgpu_trace_buffers_t* dst, void* stream) {
  if (!p || !dst) return -EINVAL;
  if (p->n_containers < 1 || p->n_containers > CONVGPU_MAX_CONTAINERS) return -EINVAL;
  if (p->n_ops != 4 && p->n_ops != 2) return -EINVAL;
  if (p->n_classes < 1 || p->n_classes > 8 || p->den == 0) return -EINVAL;
  int rc = check_device();
  if (rc) return rc;
  if (n == 0) return 0;
  if (!is_device_ptr(dst->arrival) || !is_device_ptr(dst->limit) || !is_device_ptr(dst->op_delta) ||
      !is_device_ptr(dst->op_arg))
    return -EINVAL;
  convgpu::GenArgs a;
  a.p = *p; a.tid_base = trace_id_base; a.count = n;
  a.arrival = dst->arrival; a.limit = dst->limit; a.delta = dst->op_delta; a.arg = dst->op_arg;
  cudaError_t e = convgpu::launch_generate(a, (cudaStream_t)stream);
  return e == cudaSuccess ? 0 : fail_cuda(e, "generate launch");
}

int convgpu_wrap_ops(const convgpu_api_op_t* api, uint64_t n, uint32_t n_containers, uint32_t n_ops,
                     uint32_t pitch_align, uint32_t* op_arg, void* stream) {
  if (n_containers < 1 || n_containers > CONVGPU_MAX_CONTAINERS) return -EINVAL;
  if (n_ops < 1 || n_ops > CONVGPU_MAX_OPS) return -EINVAL;
  int rc = check_device();
  if (rc) return rc;
  if (n == 0) return 0;
  if (!is_device_ptr(api) || !is_device_ptr(op_arg) || !aligned16(api)) return -EINVAL;
  cudaError_t e = convgpu::launch_wrap(reinterpret_cast<const uint4*>(api), n, n_containers, n_ops,
                                       pitch_align, op_arg, (cudaStream_t)stream);
  return e == cudaSuccess ? 0 : fail_cuda(e, "wrap launch");
}

// ---------------------------------------------------------------- host e2e
// Workspace layout (256-B aligned pieces): 2 x {arrival, limit, delta, arg}
// 32-bit chunk sets (the copy-in target, or for the 16-bit format the unpack
// target, which is then copied into 2 x {arrival16, limit16, size16, delta16,
// kinds8}), 2 x n_policies summary chunks, n_policies stats structs and
// n_policies chunks of per-container admission scratch.
static size_t align256(size_t x) { return (x + 255) & ~(size_t)255; }

namespace {

struct HostLayout {
  size_t cn, ckn, c16n, ck16n, c8n;
};
HostLayout host_layout(uint32_t nc, uint32_t K, uint64_t chunk) {
  HostLayout l;
  l.cn = align256(chunk * nc * 4);
  l.ckn = align256(chunk * nc * K * 4);
  l.c16n = align256(chunk * nc * 2);
  l.ck16n = align256(chunk * nc * K * 2);
  l.c8n = align256(chunk * nc);
  return l;
}
size_t host_ws_bytes(bool packed, uint32_t nc, uint32_t K, uint64_t chunk, uint32_t np) {
  const HostLayout l = host_layout(nc, K, chunk);
  const size_t in32 = 2 * l.cn + 2 * l.ckn;
  const size_t in16 = 2 * l.c16n + 2 * l.ck16n + l.c8n;
  const size_t inputs = packed ? 2 * in16 + 2 * in32 : 2 * in32;
  return inputs + 2 * (size_t)np * align256(chunk * sizeof(convgpu_summary_t)) +
         (size_t)np * align256(sizeof(convgpu_stats_t)) +
         (size_t)np * l.cn;  // + admission scratch, one per policy (they run concurrently)
}

// One end-to-end replay from host memory; `t32` or `t16` names the format.
int host_replay(const convgpu_traces_t* t32, const convgpu_traces16_t* t16, uint64_t n, uint32_t cap,
                uint32_t policy_mask, convgpu_summary_t* host_summary, convgpu_stats_t* host_stats,
                void* ws, size_t ws_bytes, uint64_t chunk, void* stream_) {
  const bool packed = t16 != nullptr;
  if (policy_mask == 0 || policy_mask > 0xFu) return -EINVAL;
  convgpu_traces_t ht;  // shape / parameters (array pointers unused when packed)
  if (packed) {
    memset(&ht, 0, sizeof ht);
    ht.n_containers = t16->n_containers; ht.n_ops = t16->n_ops;
    ht.trace_id_base = t16->trace_id_base; ht.rand_seed = t16->rand_seed;
    ht.ctx_overhead_mib = t16->ctx_overhead_mib; ht.kernel_variant = t16->kernel_variant;
    if (ht.n_ops > 4) return -EINVAL;  // kinds are one byte per container
  } else {
    if (!t32) return -EINVAL;
    ht = *t32;
  }
  int rc = validate_shape(&ht, cap, 0);
  if (rc) return rc;
  if (!host_stats || !ws || chunk == 0) return -EINVAL;
  if (packed ? (!t16->arrival || !t16->limit || !t16->op_size || !t16->op_delta || !t16->op_kinds)
             : (rc = validate_arrays(&ht)) != 0)
    return -EINVAL;
  if ((rc = check_device())) return rc;
  int pols[4], np = 0;
  for (int q = 0; q < 4; ++q)
    if (policy_mask & (1u << q)) pols[np++] = q;
  const uint32_t nc = ht.n_containers, K = ht.n_ops;
  if (ws_bytes < host_ws_bytes(packed, nc, K, chunk, (uint32_t)np) || !is_device_ptr(ws))
    return -EINVAL;
  cudaStream_t cs = (cudaStream_t)stream_;
  const HostLayout l = host_layout(nc, K, chunk);
  const size_t sb = align256(chunk * sizeof(convgpu_summary_t));
  char* w = (char*)ws;
  // two 32-bit chunk sets (the copy-in target, or the unpack target of the
  // 16-bit format) and, for the 16-bit format, two 16-bit copy-in sets
  uint32_t *arr[2], *lim[2], *del[2], *arg[2];
  uint16_t *arr16[2] = {nullptr, nullptr}, *lim16[2] = {nullptr, nullptr};
  uint16_t *siz16[2] = {nullptr, nullptr}, *del16[2] = {nullptr, nullptr};
  uint8_t* kin8[2] = {nullptr, nullptr};
  for (int b = 0; b < 2; ++b) {
    arr[b] = (uint32_t*)w; w += l.cn;
    lim[b] = (uint32_t*)w; w += l.cn;
    del[b] = (uint32_t*)w; w += l.ckn;
    arg[b] = (uint32_t*)w; w += l.ckn;
  }
  if (packed)
    for (int b = 0; b < 2; ++b) {
      arr16[b] = (uint16_t*)w; w += l.c16n;
      lim16[b] = (uint16_t*)w; w += l.c16n;
      siz16[b] = (uint16_t*)w; w += l.ck16n;
      del16[b] = (uint16_t*)w; w += l.ck16n;
      kin8[b] = (uint8_t*)w; w += l.c8n;
    }
  convgpu_summary_t* sum[2][4];
  for (int b = 0; b < 2; ++b)
    for (int q = 0; q < np; ++q) { sum[b][q] = (convgpu_summary_t*)w; w += sb; }
  convgpu_stats_t* dstats = (convgpu_stats_t*)w;  // [np], 256-B apart
  const size_t stb = align256(sizeof(convgpu_stats_t));
  // per-container admissions, one plane per policy (each policy replays its
  // chunks in order on its own stream)
  uint32_t* adm_scratch = (uint32_t*)(w + (size_t)np * stb);

  // Pipeline (b = chunk j & 1):
  //   copy:  [in-buffer b free] H2D chunk j -> h2d[b]
  //   cs:    wait h2d[b] (16-bit: [32-bit set b free] unpack -> unp[b]) -> ready[b]
  //   ps[q]: wait ready[b] [summaries b read back] replay policy q -> pdone[q]
  //   back:  wait every pdone -> kdone[b] (set b free), D2H summaries -> d2h[b]
  // Every policy has its own stream, and a policy's chunk j + 1 does not wait
  // for the other policies' chunk j: the tail of one launch (its last, partly
  // filled round of lanes) overlaps the start of the next.  PCIe is full
  // duplex: read-backs overlap copy-ins.
  cudaStream_t copy = nullptr, back = nullptr;
  cudaStream_t ps[4] = {nullptr, nullptr, nullptr, nullptr};
  cudaEvent_t pdone[4] = {nullptr, nullptr, nullptr, nullptr};
  cudaEvent_t h2d[2] = {nullptr, nullptr}, kdone[2] = {nullptr, nullptr};
  cudaEvent_t d2h[2] = {nullptr, nullptr}, ready[2] = {nullptr, nullptr}, unp[2] = {nullptr, nullptr};
  cudaEvent_t start_ev = nullptr;
  cudaError_t e = cudaStreamCreateWithFlags(&copy, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&back, cudaStreamNonBlocking);
  auto mk = [&](cudaEvent_t* ev) {
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(ev, cudaEventDisableTiming);
  };
  for (int b = 0; b < 2; ++b) { mk(&h2d[b]); mk(&kdone[b]); mk(&d2h[b]); mk(&ready[b]); mk(&unp[b]); }
  for (int q = 0; q < np && e == cudaSuccess; ++q) {
    e = cudaStreamCreateWithFlags(&ps[q], cudaStreamNonBlocking);
    mk(&pdone[q]);
  }
  mk(&start_ev);
  const uint64_t nchunks = (n + chunk - 1) / chunk;
  auto enqueue_h2d = [&](uint64_t j) -> cudaError_t {
    const int b = (int)(j & 1);
    const uint64_t lo = j * chunk, cnt = (n - lo < chunk) ? n - lo : chunk;
    cudaError_t r = cudaSuccess;
    // copy-in buffer b is free again once chunk j - 2 is consumed: unpacked
    // (16-bit) or replayed by every policy (32-bit)
    if (j >= 2) r = cudaStreamWaitEvent(copy, packed ? unp[b] : kdone[b], 0);
    auto cp = [&](void* dst, const void* src, size_t bytes) {
      if (r == cudaSuccess) r = cudaMemcpyAsync(dst, src, bytes, cudaMemcpyHostToDevice, copy);
    };
    if (packed) {
      cp(arr16[b], t16->arrival + lo * nc, cnt * nc * 2);
      cp(lim16[b], t16->limit + lo * nc, cnt * nc * 2);
      cp(siz16[b], t16->op_size + lo * nc * K, cnt * nc * K * 2);
      cp(del16[b], t16->op_delta + lo * nc * K, cnt * nc * K * 2);
      cp(kin8[b], t16->op_kinds + lo * nc, cnt * nc);
    } else {
      cp(arr[b], ht.arrival + lo * nc, cnt * nc * 4);
      cp(lim[b], ht.limit + lo * nc, cnt * nc * 4);
      cp(del[b], ht.op_delta + lo * nc * K, cnt * nc * K * 4);
      cp(arg[b], ht.op_arg + lo * nc * K, cnt * nc * K * 4);
    }
    if (r == cudaSuccess) r = cudaEventRecord(h2d[b], copy);
    return r;
  };
  for (int q = 0; q < np && e == cudaSuccess; ++q)
    e = cudaMemsetAsync((char*)dstats + q * stb, 0, sizeof(convgpu_stats_t), cs);
  if (e == cudaSuccess) e = cudaEventRecord(start_ev, cs);  // stats zeroed; the call starts
  if (e == cudaSuccess) e = cudaStreamWaitEvent(copy, start_ev, 0);
  for (int q = 0; q < np && e == cudaSuccess; ++q) e = cudaStreamWaitEvent(ps[q], start_ev, 0);
  if (e == cudaSuccess) e = cudaStreamWaitEvent(back, start_ev, 0);
  if (e == cudaSuccess && nchunks) e = enqueue_h2d(0);
  for (uint64_t j = 0; j < nchunks && e == cudaSuccess; ++j) {
    const int b = (int)(j & 1);
    const uint64_t lo = j * chunk, cnt = (n - lo < chunk) ? n - lo : chunk;
    if (j + 1 < nchunks) e = enqueue_h2d(j + 1);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(cs, h2d[b], 0);
    if (packed && e == cudaSuccess) {  // 16-bit copy-in set b -> 32-bit set b
      if (j >= 2) e = cudaStreamWaitEvent(cs, kdone[b], 0);
      convgpu::Pack16Args u;
      memset(&u, 0, sizeof u);
      u.count = cnt; u.n = nc; u.K = K;
      u.r_arrival16 = arr16[b]; u.r_limit16 = lim16[b]; u.r_size16 = siz16[b];
      u.r_delta16 = del16[b]; u.r_kinds8 = kin8[b];
      u.w_arrival = arr[b]; u.w_limit = lim[b]; u.w_delta = del[b]; u.w_arg = arg[b];
      if (e == cudaSuccess) e = convgpu::launch_unpack16(u, cs);
      if (e == cudaSuccess) e = cudaEventRecord(unp[b], cs);
    }
    if (e == cudaSuccess) e = cudaEventRecord(ready[b], cs);
    if (e != cudaSuccess) break;
    convgpu_traces_t dt = ht;
    dt.arrival = arr[b]; dt.limit = lim[b]; dt.op_delta = del[b]; dt.op_arg = arg[b];
    dt.trace_id_base = ht.trace_id_base + lo;
    for (int q = 0; q < np && e == cudaSuccess; ++q) {  // every policy on the resident chunk
      e = cudaStreamWaitEvent(ps[q], ready[b], 0);
      // summary buffers b: read back (chunk j - 2) before they are rewritten
      if (e == cudaSuccess && host_summary && j >= 2) e = cudaStreamWaitEvent(ps[q], d2h[b], 0);
      convgpu::ReplayArgs a = make_args(&dt, cnt, cap);
      a.summary = host_summary ? sum[b][q] : nullptr;
      a.adm_scratch = adm_scratch + (size_t)q * l.cn / 4;  // admissions only
      a.no_wide = packed;  // 16-bit limits: no 17-bit pass (replay_lpt16.cu)
      a.stats = (convgpu_stats_t*)((char*)dstats + q * stb);
      if (e == cudaSuccess) e = launch_any(a, pols[q], ht.kernel_variant, ps[q]);
      if (e == cudaSuccess) e = cudaEventRecord(pdone[q], ps[q]);
      if (e == cudaSuccess) e = cudaStreamWaitEvent(back, pdone[q], 0);
    }
    if (e == cudaSuccess) e = cudaEventRecord(kdone[b], back);
    if (e == cudaSuccess && host_summary) {
      for (int q = 0; q < np && e == cudaSuccess; ++q)
        e = cudaMemcpyAsync(host_summary + (uint64_t)q * n + lo, sum[b][q],
                            cnt * sizeof(convgpu_summary_t), cudaMemcpyDeviceToHost, back);
      if (e == cudaSuccess) e = cudaEventRecord(d2h[b], back);
    }
  }
  // join every internal stream back into the caller's stream (events on
  // `stream` then bracket every copy and kernel of the call), then the stats
  for (int q = 0; q < np && e == cudaSuccess; ++q) {
    e = cudaEventRecord(pdone[q], ps[q]);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(cs, pdone[q], 0);
  }
  if (e == cudaSuccess) e = cudaEventRecord(h2d[0], copy);
  if (e == cudaSuccess) e = cudaStreamWaitEvent(cs, h2d[0], 0);
  if (e == cudaSuccess) e = cudaEventRecord(d2h[0], back);
  if (e == cudaSuccess) e = cudaStreamWaitEvent(cs, d2h[0], 0);
  for (int q = 0; q < np && e == cudaSuccess; ++q)
    e = cudaMemcpyAsync(host_stats + q, (char*)dstats + q * stb, sizeof(convgpu_stats_t),
                        cudaMemcpyDeviceToHost, cs);
  if (e == cudaSuccess) e = cudaStreamSynchronize(cs);
  if (e != cudaSuccess) {
    // an error mid-way: copies and kernels already enqueued may still read the
    // caller's pinned buffers and write its workspace, which the caller frees
    // or reuses once we return, so drain every stream before tearing down
    // (secondary errors ignored; the first one is reported)
    if (copy) cudaStreamSynchronize(copy);
    if (back) cudaStreamSynchronize(back);
    for (int q = 0; q < 4; ++q)
      if (ps[q]) cudaStreamSynchronize(ps[q]);
    cudaStreamSynchronize(cs);
  }
  for (int b = 0; b < 2; ++b) {
    cudaEvent_t* evs[] = {&h2d[b], &kdone[b], &d2h[b], &ready[b], &unp[b]};
    for (cudaEvent_t* ev : evs)
      if (*ev) cudaEventDestroy(*ev);
  }
  for (int q = 0; q < 4; ++q) {
    if (ps[q]) cudaStreamDestroy(ps[q]);
    if (pdone[q]) cudaEventDestroy(pdone[q]);
  }
  if (start_ev) cudaEventDestroy(start_ev);
  if (copy) cudaStreamDestroy(copy);
  if (back) cudaStreamDestroy(back);
  return e == cudaSuccess ? 0 : fail_cuda(e, "replay_host");
}

}  // namespace

size_t convgpu_replay_host_workspace(uint32_t n_containers, uint32_t n_ops, uint64_t chunk,
                                     uint32_t n_policies) {
  return host_ws_bytes(false, n_containers, n_ops, chunk, n_policies);
}

size_t convgpu_replay_host16_workspace(uint32_t n_containers, uint32_t n_ops, uint64_t chunk,
                                       uint32_t n_policies) {
  return host_ws_bytes(true, n_containers, n_ops, chunk, n_policies);
}

int convgpu_replay_host(const convgpu_traces_t* ht, uint64_t n, uint32_t cap, uint32_t policy_mask,
                        convgpu_summary_t* host_summary, convgpu_stats_t* host_stats,
                        void* ws, size_t ws_bytes, uint64_t chunk, void* stream_) {
  if (!ht) return -EINVAL;
  return host_replay(ht, nullptr, n, cap, policy_mask, host_summary, host_stats, ws, ws_bytes,
                     chunk, stream_);
}

int convgpu_replay_host16(const convgpu_traces16_t* ht, uint64_t n, uint32_t cap,
                          uint32_t policy_mask, convgpu_summary_t* host_summary,
                          convgpu_stats_t* host_stats, void* ws, size_t ws_bytes, uint64_t chunk,
                          void* stream_) {
  if (!ht) return -EINVAL;
  return host_replay(nullptr, ht, n, cap, policy_mask, host_summary, host_stats, ws, ws_bytes,
                     chunk, stream_);
}

int convgpu_pack16(const convgpu_traces_t* src, uint64_t n, const convgpu_trace16_buffers_t* dst,
                   uint64_t* out_of_range, void* stream) {
  if (!src || !dst) return -EINVAL;
  if (src->n_containers < 1 || src->n_containers > CONVGPU_MAX_CONTAINERS) return -EINVAL;
  if (src->n_ops < 1 || src->n_ops > 4) return -EINVAL;
  int rc = check_device();
  if (rc) return rc;
  if (n == 0) return 0;
  if (!is_device_ptr(src->arrival) || !is_device_ptr(src->limit) || !is_device_ptr(src->op_delta) ||
      !is_device_ptr(src->op_arg) || !is_device_ptr(dst->arrival) || !is_device_ptr(dst->limit) ||
      !is_device_ptr(dst->op_size) || !is_device_ptr(dst->op_delta) ||
      !is_device_ptr(dst->op_kinds) || !opt_device_ptr(out_of_range))
    return -EINVAL;
  convgpu::Pack16Args a;
  memset(&a, 0, sizeof a);
  a.count = n; a.n = src->n_containers; a.K = src->n_ops;
  a.arrival = src->arrival; a.limit = src->limit; a.delta = src->op_delta; a.arg = src->op_arg;
  a.arrival16 = dst->arrival; a.limit16 = dst->limit; a.size16 = dst->op_size;
  a.delta16 = dst->op_delta; a.kinds8 = dst->op_kinds;
  a.out_of_range = (unsigned long long*)out_of_range;
  cudaError_t e = convgpu::launch_pack16(a, (cudaStream_t)stream);
  return e == cudaSuccess ? 0 : fail_cuda(e, "pack16 launch");
}

}  // extern "C"
