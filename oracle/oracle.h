/*
 * oracle.h — TEST INFRASTRUCTURE ONLY (see oracle/README.md).
 *
 * Plain, slow, single-threaded CPU oracle of ConVGPU's GPU-memory scheduler
 * (Kang et al., IEEE CLUSTER 2017 — /root/reference/PAPER.md, cited "P:<line>").
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * `--impl reference` leg may load it.  It shares no code, header, table or
 * constant generator with the CUDA path under
 * paper_conf_cluster_kangjkkk17_b200/csrc/ and include/ — it is written
 * independently from the paper and DESIGN.md's readings.
 */
#ifndef CONVGPU_ORACLE_H
#define CONVGPU_ORACLE_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define ORC_MAX_N 64          /* containers per trace */
#define ORC_MAX_K 8           /* ops per container */

/* Scheduling policies. */
enum { ORC_FIFO = 0, ORC_BEST_FIT = 1, ORC_RECENT = 2, ORC_RANDOM = 3 };

/* Dispatch-reading flag OR-ed into the policy argument: the literal
 * re-select-on-every-release reading (R1-LIT). */
#define ORC_LITERAL 0x100

/* Op kinds carried in the top two bits of an op word; low 30 bits = MiB. */
enum { ORC_ALLOC = 0, ORC_FREE = 1, ORC_FINISH = 2, ORC_NOP = 3 };

/* Per-trace flag bits. */
enum {
  ORC_F_DEADLOCK = 1u << 0,
  ORC_F_OVERCOMMIT = 1u << 1,
  ORC_F_INVALID_LIMIT = 1u << 2,
  ORC_F_INVALID_FREE = 1u << 3,
  ORC_F_UNSORTED_ARRIVAL = 1u << 4,
  ORC_F_TICK_RANGE = 1u << 5,
  ORC_F_BAD_PROGRAM = 1u << 6,
};

#define ORC_NONE32 0xFFFFFFFFu
#define ORC_NONE8 0xFFu

/* One trace, structure-of-arrays, op-major: delta[k*n + c], arg[k*n + c]. */
typedef struct {
  uint32_t n, K;
  const uint32_t *arrival, *limit, *delta, *arg;
} orc_trace_t;

typedef struct {
  uint32_t admit_tick[ORC_MAX_N];
  uint32_t admit_rank[ORC_MAX_N];
  uint32_t wait[ORC_MAX_N];
  uint32_t finish[ORC_MAX_N];
  uint32_t makespan, peak_reserved, peak_used, flags;
  uint64_t sum_wait;
  uint32_t n_rejected, n_select;
  uint64_t digest;
  uint64_t events;
  /* invariant checker (check != 0): first violated invariant id, 0 = none */
  int32_t violation;
  uint64_t violation_event;
} orc_result_t;

typedef struct {
  uint64_t traces, events, sum_makespan, sum_wait, n_rejected, n_select, digest_sum;
  uint32_t max_makespan, max_peak_reserved;
  uint32_t flag_count[8];
} orc_stats_t;

/* Synthetic workload generator parameters (DESIGN.md §Input recipe). */
typedef struct {
  uint64_t gen_seed;
  uint32_t n, K;                 /* K = 4 split program, K = 2 paper-mimic */
  uint32_t n_classes;
  uint32_t class_mib[8];
  uint32_t num, den;             /* L = class_mib[k] * num / den */
  uint32_t iat;                  /* arrival = c * iat */
  uint32_t dur_base, dur_step, dur_class_offset, dur_jit;
  uint32_t ovh;                  /* overhead subtracted from the ALLOC sizes */
} orc_gen_params_t;

void orc_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]);
uint64_t orc_mix64(uint64_t z);

int orc_replay(const orc_trace_t *tr, uint32_t cap, int policy, uint64_t tid,
               uint64_t rand_seed, uint32_t ovh, int check, orc_result_t *res);

int orc_generate(const orc_gen_params_t *p, uint64_t tid, uint32_t *arrival,
                 uint32_t *limit, uint32_t *delta, uint32_t *arg);

/* Replay generated traces [tid_lo, tid_hi).  Any of stats / summary outputs
 * may be NULL.  range_digest[i] accumulates trace digests of global ids in
 * [i*range_size, (i+1)*range_size) relative to range_base. */
int orc_replay_range(const orc_gen_params_t *p, uint32_t cap, int policy,
                     uint64_t rand_seed, uint32_t ovh, uint64_t tid_lo,
                     uint64_t tid_hi, int check, orc_stats_t *stats,
                     uint32_t *sum_u32x4 /* [n][4] makespan,peak_res,peak_used,flags */,
                     uint64_t *sum_u64x2 /* [n][2] sum_wait, digest */,
                     uint32_t *cnt_u32x2 /* [n][2] n_rejected, n_select */,
                     uint32_t *admit_tick, uint8_t *admit_rank, uint32_t *wait,
                     uint32_t *finish /* [n][N] each, or NULL */);

/* Replay caller-provided traces laid out like the C-ABI batch:
 * arrival[i*n + c], limit[i*n + c], delta[(i*K + k)*n + c], arg[...]. */
int orc_replay_batch(uint32_t n, uint32_t K, uint64_t count,
                     const uint32_t *arrival, const uint32_t *limit,
                     const uint32_t *delta, const uint32_t *arg, uint32_t cap,
                     int policy, uint64_t tid_base, uint64_t rand_seed,
                     uint32_t ovh, int check, orc_stats_t *stats,
                     uint32_t *sum_u32x4, uint64_t *sum_u64x2,
                     uint32_t *cnt_u32x2, uint32_t *admit_tick,
                     uint8_t *admit_rank, uint32_t *wait, uint32_t *finish);

/* ---- NEXT-3: wrapper-side size semantics (oracle/wrapper.c) ------------
 * The wrapper module sees CUDA API calls and "calculates adjusted allocate
 * size before checking available memory size"; Table II
 * lists the covered APIs.  An API-level program record per
 * (container, op) is mapped to the scheduler's op word. */
enum {
  ORC_API_MALLOC = 0,         /* cudaMalloc / cuMemAlloc(bytes = a0 | a1 << 32) */
  ORC_API_MALLOC_MANAGED = 1, /* cudaMallocManaged(bytes): multiple of 128 MiB */
  ORC_API_MALLOC_PITCH = 2,   /* cudaMallocPitch(width a0, height a1): pitch * height */
  ORC_API_MALLOC_3D = 3,      /* cudaMalloc3D(width a0, height a1, depth a2) */
  ORC_API_FREE = 4,           /* cudaFree of the allocation made by op a0 of this container */
  ORC_API_MEM_GET_INFO = 5,   /* cudaMemGetInfo: answered from the ledger, no memory effect */
  ORC_API_COMPUTE = 6,        /* work without memory calls */
  ORC_API_EXIT = 7            /* __cudaUnregisterFatBinary */
};
typedef struct {
  uint32_t api, a0, a1, a2;
} orc_api_op_t;
/* Bytes an allocation API really takes (saturating at 2^64 - 1); 0 for a
 * non-allocation API.  pitch_align = the device's pitch granule in bytes. */
uint64_t orc_wrap_bytes(const orc_api_op_t *op, uint32_t pitch_align);
/* The scheduler's unit is MiB: ceil(bytes / 2^20), saturated to 2^30 - 1. */
uint32_t orc_wrap_mib(uint64_t bytes);
/* One container's program of K API records -> K op words. */
void orc_wrap_program(const orc_api_op_t *ops, uint32_t K, uint32_t pitch_align,
                      uint32_t *op_words);
/* A batch laid out like the C-ABI: api[(i*K + k)*n + c] -> arg[(i*K + k)*n + c]. */
void orc_wrap_batch(uint32_t n, uint32_t K, uint64_t count, const orc_api_op_t *api,
                    uint32_t pitch_align, uint32_t *arg);

#ifdef __cplusplus
}
#endif
#endif
