/*
 * convgpu.h — C ABI of the B200-native batched replay of ConVGPU's
 * GPU-memory scheduler (Kang, Jun, Kim, Kim, Kim, "ConVGPU: GPU Management
 * Middleware in Container Based Virtualized Environment", IEEE CLUSTER 2017;
 * text in PAPER.md, cited "P:<line>").  DESIGN.md states the semantics and
 * every reading ("R<n>") of the paper that the kernels implement.
 *
 * Library: paper_conf_cluster_kangjkkk17_b200/libconvgpu.so (sm_100a only).
 *
 * Conventions for every entry point
 *  - Pointers named "device" must be caller-owned device (or managed)
 *    memory on the current CUDA device; the library never allocates, frees
 *    or retains them.  Host-side structs are read during the call only.
 *  - Work is enqueued on the caller's stream (`stream`, a cudaStream_t; NULL =
 *    the legacy default stream) and is asynchronous: results are valid after
 *    the caller synchronises that stream.
 *  - Return 0 on success or a negative errno-style code:
 *      -EINVAL (-22) invalid argument (NULL required pointer, host pointer
 *                    where device memory is required, size out of range),
 *      -ENODEV (-19) the current device is not an sm_100 B200-class GPU,
 *      -EIO    (-5)  a CUDA error; its text is kept per thread and returned
 *                    by convgpu_strerror(-EIO).
 *  - No global mutable state: calls are reentrant and thread-safe; calls on
 *    different streams / devices may run concurrently.
 *  - Data-level anomalies are never return codes: they are per-trace flag
 *    bits (CONVGPU_FLAG_*) in the outputs.
 */
#ifndef CONVGPU_H
#define CONVGPU_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define CONVGPU_ABI_VERSION 5  /* 5: CONVGPU_KERNEL_LANE_COMPACT_WIDE */
#define CONVGPU_MAX_CONTAINERS 64u   /* containers per trace */
#define CONVGPU_MAX_OPS 8u           /* ops per container (K) */
#define CONVGPU_CAPACITY_LIMIT (1u << 26) /* capacity_mib must be below this */
#define CONVGPU_OVERHEAD_LIMIT (1u << 30) /* ctx_overhead_mib must be below this */
#define CONVGPU_TICK_LIMIT (1u << 26)     /* R19: trace horizon bound */
#define CONVGPU_NONE32 0xFFFFFFFFu        /* admit_tick of a never-admitted container */
#define CONVGPU_NONE8 0xFFu               /* admit_rank of a never-admitted container */

/* The four scheduling policies of P:141-145 (R3-R7). */
typedef enum {
  CONVGPU_FIFO = 0,        /* oldest created paused container */
  CONVGPU_BEST_FIT = 1,    /* shortfall closest to, not above, free memory */
  CONVGPU_RECENT_FIT = 2,  /* most recently suspended ("Recent use") */
  CONVGPU_RANDOM_FIT = 3   /* uniform among paused ("Random"), Philox-keyed */
} convgpu_policy_t;

/* OR-ed into the policy argument of convgpu_replay: replay under the literal
 * re-select-on-every-release reading (R1-LIT, SURVEY §8(f)
 * NEXT-1) instead of R1's sticky fill target.  Partial holds are kept, so
 * deadlocks can occur and are reported by CONVGPU_FLAG_DEADLOCK.  Runs on the
 * compact lane kernel (AUTO picks it under the same conditions as for R1;
 * traces it cannot hold go to a marked-only pass of the warp-per-trace
 * kernel) or on the warp-per-trace kernel; LANE_PER_TRACE is -EINVAL. */
#define CONVGPU_DISPATCH_LITERAL 0x100

/* Op kinds: op_arg = kind << 30 | size_mib (size < 2^30).  The replay maps
 * the wrapper-module API classes of Table II: allocation APIs ->
 * ALLOC, cudaFree -> FREE, __cudaUnregisterFatBinary /
 * container stop -> FINISH; NOP = compute without memory calls. */
typedef enum {
  CONVGPU_OP_ALLOC = 0,
  CONVGPU_OP_FREE = 1,
  CONVGPU_OP_FINISH = 2,
  CONVGPU_OP_NOP = 3
} convgpu_op_t;

/* Per-trace flag bits (summary.flags, stats.flag_count[bit]).  Bit 1 is an
 * assertion and does not stop the trace; any other bit stops it, its
 * per-container outputs become (NONE32, NONE8, 0, 0) and every summary field
 * except flags is 0. */
enum {
  CONVGPU_FLAG_DEADLOCK = 1u << 0,         /* containers remain, none can run (P:7) */
  CONVGPU_FLAG_OVERCOMMIT = 1u << 1,       /* memory in use > memory reserved */
  CONVGPU_FLAG_INVALID_LIMIT = 1u << 2,    /* a declared limit > capacity (R15) */
  CONVGPU_FLAG_INVALID_FREE = 1u << 3,     /* FREE of more than the container uses */
  CONVGPU_FLAG_UNSORTED_ARRIVAL = 1u << 4, /* arrival[c] < arrival[c-1] */
  CONVGPU_FLAG_TICK_RANGE = 1u << 5,       /* max arrival + sum of deltas >= 2^26 */
  CONVGPU_FLAG_BAD_PROGRAM = 1u << 6       /* last op not FINISH or FINISH not last */
};

/* A batch of n independent traces, structure-of-arrays in DEVICE memory.
 * Trace i, container c (0 <= c < n_containers), op k (0 <= k < n_ops):
 *   arrival[i*n_containers + c]                 tick of container creation
 *   limit[i*n_containers + c]                   declared GPU-memory limit, MiB
 *   op_delta[(i*n_ops + k)*n_containers + c]    ticks after the previous op
 *                                               (after arrival for k = 0)
 *   op_arg[(i*n_ops + k)*n_containers + c]      kind << 30 | size_mib
 * Arrivals must be non-decreasing within a trace (index = creation order,
 * R7) and every container's last op must be its only FINISH.
 * Fastest path: n_containers % 4 == 0 and 16-byte aligned arrays (traces are
 * then staged into shared memory by the bulk-copy engine). */
typedef struct {
  const uint32_t *arrival, *limit, *op_delta, *op_arg; /* device */
  uint32_t n_containers;     /* 1..64 */
  uint32_t n_ops;            /* K, 1..8 */
  uint64_t trace_id_base;    /* global id of trace 0 (sharding; Random-Fit counter) */
  uint64_t rand_seed;        /* Random-Fit Philox key (R6) */
  uint32_t ctx_overhead_mib; /* charged at a container's first ALLOC (66) */
  uint32_t kernel_variant;   /* CONVGPU_KERNEL_*: 0 = auto (recommended) */
} convgpu_traces_t;

/* Replay kernel variants.  Results are bit-identical; only
 * speed differs.  AUTO picks lane-per-trace when the batch fills the GPU. */
enum {
  CONVGPU_KERNEL_AUTO = 0,
  CONVGPU_KERNEL_WARP_PER_TRACE = 1, /* one warp per trace, TMA-staged trace */
  CONVGPU_KERNEL_LANE_PER_TRACE = 2, /* one lane per trace, 32 traces per warp */
  CONVGPU_KERNEL_LANE_COMPACT = 3,   /* one lane per trace, 16-bit packed state, up to
                                        8 warps per SM; needs n_containers = 64, n_ops = 4,
                                        out->admit_tick or out->admit_scratch != NULL (it
                                        holds admissions during the replay) and 16-byte
                                        aligned arrays / outputs,
                                        else -EINVAL.  Traces whose limits exceed 0xFFFE
                                        MiB are replayed by a second launch of the same
                                        kernel with 17-bit limits / used memory (R1; if
                                        every ALLOC / FREE size is <= 0xFFFE and every
                                        limit <= 0x1FFFF), the rest, and traces whose
                                        deltas exceed 0xFFFF ticks or horizon 2^25, by a
                                        32-bit lane-per-trace launch (R1-LIT: the
                                        warp-per-trace kernel).
                                        AUTO picks it whenever the lane kernel would run
                                        and these conditions hold. */
  CONVGPU_KERNEL_LANE_COMPACT_WIDE = 4 /* the same with the 17-bit layout as the first
                                        pass (R1; R1-LIT: as LANE_COMPACT): for batches
                                        whose limits exceed 0xFFFE MiB (config [4] at
                                        rho = 8), which would all take the second pass;
                                        same requirements, same results */
};

/* Per-trace summary, 40 bytes. */
typedef struct {
  uint32_t makespan;      /* max finish - arrival[0] (Table IV "finished time") */
  uint32_t peak_reserved; /* max over events of capacity - free */
  uint32_t peak_used;     /* max over events of sum of used */
  uint32_t flags;         /* CONVGPU_FLAG_* */
  uint64_t sum_wait;      /* total suspended ticks (Table V numerator) */
  uint32_t n_rejected;    /* ALLOCs denied for exceeding the limit */
  uint32_t n_select;      /* policy selections made */
  uint64_t digest;        /* DESIGN.md R20 digest of all outputs of the trace */
} convgpu_summary_t;

/* Batch statistics, accumulated with device atomics into caller-zeroed
 * DEVICE memory (several calls may accumulate into one struct). */
typedef struct {
  uint64_t traces, events, sum_makespan, sum_wait, n_rejected, n_select, digest_sum;
  uint32_t max_makespan, max_peak_reserved;
  uint32_t flag_count[8];
} convgpu_stats_t;

/* Outputs; every pointer is DEVICE memory or NULL (= not produced). */
typedef struct {
  uint32_t *admit_tick;  /* [n][n_containers] tick the limit became fully assigned */
  uint8_t *admit_rank;   /* [n][n_containers] admission order, NONE8 if never */
  uint32_t *wait;        /* [n][n_containers] ticks spent suspended */
  uint32_t *finish;      /* [n][n_containers] tick of FINISH */
  convgpu_summary_t *summary; /* [n] */
  convgpu_stats_t *stats;     /* 1 struct, caller-zeroed, accumulated */
  uint64_t *range_digest;     /* optional: range_digest[gid / range_size] += digest */
  uint64_t range_size;        /* > 0 when range_digest != NULL */
  void *stream;               /* cudaStream_t */
  /* Optional caller-owned DEVICE scratch, [n][n_containers] u32, 16-byte
   * aligned (ABI 4).  The compact lane kernel keeps each container's
   * admission in its slot while the trace replays (admit_tick itself serves
   * when it is requested).  With admit_tick == NULL and this scratch given,
   * summary- / digest- / stats-only launches still run on the compact kernel;
   * without either, AUTO falls back to the 32-bit lane kernel.  Contents are
   * undefined after the call; NULL allowed. */
  uint32_t *admit_scratch;
} convgpu_out_t;

/*
 * convgpu_replay — replay n traces under one policy (the hot path).
 * Semantics: DESIGN.md §Semantics; P:78, P:98, P:104, P:110, P:133-145,
 * P:149.  One warp per trace; the event loop, policy selection, outputs,
 * digests and the statistics reduction all run in the kernel.
 * capacity_mib: GPU memory to share, 1 .. CONVGPU_CAPACITY_LIMIT-1.
 * policy: convgpu_policy_t, optionally | CONVGPU_DISPATCH_LITERAL.  n may be 0
 * (no-op).
 * Errors: -EINVAL for NULL traces/out/arrays, n_containers or n_ops out of
 * range, policy out of range, capacity out of range, overhead out of range,
 * kernel_variant > 3 (or 3 without its conditions), host pointers, range_digest without range_size; -ENODEV;
 * -EIO (launch failure).
 */
int convgpu_replay(const convgpu_traces_t *traces, uint64_t n, uint32_t capacity_mib,
                   int policy, const convgpu_out_t *out);

/* Synthetic workload generator (DESIGN.md §Input recipe; P:179 random
 * Table III types every 5 s, P:181-187 sizes, "5 to 45 seconds" by size).
 * Per trace id g and container c, Philox4x32-10 with counter
 * (lo32 g, hi32 g, c, 0) and key gen_seed gives (x0, x1):
 *   k = (x0 * n_classes) >> 32, L = class_mib[k] * num / den,
 *   arrival = c * iat, dur = dur_base + dur_step * (k + dur_class_offset)
 *         + ((x1 * (dur_jit + 1)) >> 32), e = max(L - ovh, 0);
 *   n_ops = 4: ALLOC e/2 @0, ALLOC e - e/2 @dur/4, FREE e/2 @dur/2,
 *              FINISH @dur - dur/4 - dur/2;
 *   n_ops = 2: ALLOC e @0, FINISH @dur (paper-mimic). */
typedef struct {
  uint64_t gen_seed;
  uint32_t n_containers, n_ops;  /* 1..64; 4 or 2 */
  uint32_t n_classes;            /* 1..8 */
  uint32_t class_mib[8];
  uint32_t num, den;             /* den > 0 */
  uint32_t iat;
  uint32_t dur_base, dur_step, dur_class_offset, dur_jit;
  uint32_t ctx_overhead_mib;
} convgpu_gen_params_t;

/* Writable DEVICE buffers for convgpu_generate, same layout as
 * convgpu_traces_t for the generated trace ids [trace_id_base, +n). */
typedef struct {
  uint32_t *arrival, *limit, *op_delta, *op_arg;
} convgpu_trace_buffers_t;

/* Generate n traces with global ids trace_id_base .. +n-1 into dst.
 * Errors: -EINVAL (NULL, bad params, host pointers), -ENODEV, -EIO. */
int convgpu_generate(const convgpu_gen_params_t *params, uint64_t trace_id_base,
                     uint64_t n, const convgpu_trace_buffers_t *dst, void *stream);

/* End-to-end replay from HOST memory (pinned for full speed): traces->arrays
 * are HOST pointers.  The batch is streamed through the caller's DEVICE
 * workspace in chunks of chunk_traces traces; the copy-in of chunk j+1 (on an
 * internal stream) overlaps the replay of chunk j (on `stream`), and every
 * policy whose bit is set in policy_mask (bit q = convgpu_policy_t q) is
 * replayed on the chunk while it is resident.  Outputs go back to HOST:
 *   host_summary: [n_policies][n] records (NULL = not produced),
 *   host_stats:   [n_policies] records, overwritten (not accumulated),
 * in increasing policy order.  workspace: DEVICE, at least
 * convgpu_replay_host_workspace(n_containers, n_ops, chunk_traces,
 * n_policies) bytes.  Synchronous: returns when the results are in host
 * memory; all work is joined into `stream`, so CUDA events recorded on
 * `stream` around the call bracket every copy and kernel.
 * Errors: -EINVAL (bad shape, empty mask, small workspace, host workspace),
 * -ENODEV, -EIO. */
size_t convgpu_replay_host_workspace(uint32_t n_containers, uint32_t n_ops,
                                     uint64_t chunk_traces, uint32_t n_policies);
int convgpu_replay_host(const convgpu_traces_t *host_traces, uint64_t n,
                        uint32_t capacity_mib, uint32_t policy_mask,
                        convgpu_summary_t *host_summary, convgpu_stats_t *host_stats,
                        void *device_workspace, size_t workspace_bytes,
                        uint64_t chunk_traces, void *stream);

/* ---- Compact 16-bit trace format (host end-to-end path) -------------------
 * The same traces as convgpu_traces_t with every field in 16 bits and the op
 * kinds in one byte per container: 21 B per container at n_ops = 4 instead of
 * 40.  convgpu_replay_host is bound by the host-to-device copy of the traces
 * (PCIe), not by the replay; convgpu_replay_host16 copies this format and
 * restores the 32-bit layout on the device (an unpack kernel next to the
 * replay), so the same replay reads about half the PCIe bytes.  Layout, trace
 * i, container c, op k (n_ops <= 4):
 *   arrival[i*n_containers + c], limit[i*n_containers + c]     u16
 *   op_size[(i*n_ops + k)*n_containers + c]                    u16 (op_arg & 0x3FFFFFFF)
 *   op_delta[(i*n_ops + k)*n_containers + c]                   u16
 *   op_kinds[i*n_containers + c]                               u8: kind of op k in bits 2k, 2k+1
 * A trace is representable when every arrival, limit, op size and delta is
 * <= 0xFFFF (BASELINE configs [2]-[4] are; config [1] and the paper-mimic
 * workload space containers 5,000 ticks apart, so their later arrivals are
 * not); convgpu_pack16 counts the values that are not. */
typedef struct {
  const uint16_t *arrival, *limit, *op_size, *op_delta; /* host (pinned for full speed) */
  const uint8_t *op_kinds;
  uint32_t n_containers;     /* 1..64 */
  uint32_t n_ops;            /* 1..4 */
  uint64_t trace_id_base, rand_seed;
  uint32_t ctx_overhead_mib, kernel_variant; /* as in convgpu_traces_t */
} convgpu_traces16_t;

/* Writable DEVICE buffers of the 16-bit format. */
typedef struct {
  uint16_t *arrival, *limit, *op_size, *op_delta;
  uint8_t *op_kinds;
} convgpu_trace16_buffers_t;

/* Pack n traces (DEVICE, 32-bit layout; the arrays of `src` are read, its other
 * fields are ignored except n_containers / n_ops) into the 16-bit format in
 * DEVICE buffers `dst`.  out_of_range (DEVICE u64, caller-zeroed, accumulated;
 * NULL allowed) counts the values above 0xFFFF, whose packed copies are
 * truncated: a batch is exact in the 16-bit format iff it stays 0.
 * Asynchronous on `stream`.  Errors: -EINVAL (NULL, n_ops > 4, n_containers out
 * of range, host pointers), -ENODEV, -EIO. */
int convgpu_pack16(const convgpu_traces_t *src, uint64_t n, const convgpu_trace16_buffers_t *dst,
                   uint64_t *out_of_range, void *stream);

/* convgpu_replay_host for 16-bit HOST traces: the same chunked copy-in /
 * replay-every-policy / summaries-back pipeline, plus one unpack kernel per
 * chunk.  Same outputs, conventions and errors (n_ops > 4 is -EINVAL). */
size_t convgpu_replay_host16_workspace(uint32_t n_containers, uint32_t n_ops,
                                       uint64_t chunk_traces, uint32_t n_policies);
int convgpu_replay_host16(const convgpu_traces16_t *host_traces, uint64_t n,
                          uint32_t capacity_mib, uint32_t policy_mask,
                          convgpu_summary_t *host_summary, convgpu_stats_t *host_stats,
                          void *device_workspace, size_t workspace_bytes,
                          uint64_t chunk_traces, void *stream);

/* ---- NEXT-3: the wrapper module's size semantics ----------
 * PAPER.md §III-C: the wrapper intercepts the allocation APIs of Table II
 * and "calculates adjusted allocate size before checking
 * available memory size".  convgpu_wrap_ops maps API-level
 * program records to the op words convgpu_replay consumes:
 *   MALLOC(bytes = a0 | a1 << 32)          -> ALLOC ceil(bytes / 2^20) MiB
 *   MALLOC_MANAGED(bytes = a0 | a1 << 32)  -> ALLOC of bytes rounded up to a
 *                                             multiple of 128 MiB
 *   MALLOC_PITCH(width a0, height a1)      -> ALLOC of roundup(a0, pitch_align) * a1
 *                                             bytes
 *   MALLOC_3D(width a0, height a1, depth a2) -> ALLOC of roundup(a0, pitch_align)
 *                                             * a1 * a2 bytes (Table II)
 *   FREE(a0 = op index j of this container) -> FREE of op j's MiB if op j < k is
 *                                             an allocation not freed before
 *                                             (the scheduler's address -> size
 *                                             hash), else FREE of
 *                                             2^30 - 1 MiB (-> INVALID_FREE)
 *   MEM_GET_INFO, COMPUTE                  -> NOP (answered from the ledger)
 *   EXIT (__cudaUnregisterFatBinary)       -> FINISH
 *   any other code                         -> FINISH if k < n_ops - 1, else NOP
 *                                             (the replay flags BAD_PROGRAM)
 * Byte counts become MiB rounded up, saturated at 2^30 - 1 (R13');
 * products saturate at 2^64 - 1 before rounding.  pitch_align is the device's
 * pitch granule in bytes (cudaDeviceProp.textureAlignment: 512 on B200, where
 * cudaMallocPitch returns roundup(width, 512)); 0 = no rounding. */
typedef enum {
  CONVGPU_API_MALLOC = 0,
  CONVGPU_API_MALLOC_MANAGED = 1,
  CONVGPU_API_MALLOC_PITCH = 2,
  CONVGPU_API_MALLOC_3D = 3,
  CONVGPU_API_FREE = 4,
  CONVGPU_API_MEM_GET_INFO = 5,
  CONVGPU_API_COMPUTE = 6,
  CONVGPU_API_EXIT = 7
} convgpu_api_t;

typedef struct {
  uint32_t api;        /* convgpu_api_t */
  uint32_t a0, a1, a2; /* arguments, above */
} convgpu_api_op_t;    /* 16 bytes */

/* api:    DEVICE, [n][n_ops][n_containers] records, 16-byte aligned (the op_arg
 *         layout of convgpu_traces_t with a record per op).
 * op_arg: DEVICE, [n][n_ops][n_containers] u32, written; may be the op_arg of
 *         a convgpu_traces_t whose other arrays the caller fills.
 * Caller-owned buffers; asynchronous on `stream` (cudaStream_t or NULL).
 * Returns 0, -EINVAL (n_containers outside 1..64, n_ops outside 1..8, a
 * pointer that is NULL, not device memory or api not 16-byte aligned when
 * n > 0), -ENODEV or -EIO.  n = 0 is a no-op. */
int convgpu_wrap_ops(const convgpu_api_op_t *api, uint64_t n, uint32_t n_containers,
                     uint32_t n_ops, uint32_t pitch_align, uint32_t *op_arg, void *stream);

/* Upper bound on the kernel launches convgpu_replay enqueues per call (the
 * compact lane kernel is followed by its 17-bit and 32-bit fallback passes,
 * which replay only the traces the previous pass marked; every other
 * variant launches once; convgpu_generate launches once;
 * convgpu_replay_host: this many per chunk and policy). */
int convgpu_launches_per_call(void);

/* Human-readable text for a return code (thread-local CUDA text for -EIO). */
const char *convgpu_strerror(int rc);

/* CONVGPU_ABI_VERSION of the loaded library. */
int convgpu_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* CONVGPU_H */
