/*
 * wrapper.c — TEST INFRASTRUCTURE ONLY (see oracle/README.md).
 *
 * NEXT-3: the wrapper module's size semantics, written
 * sentence by sentence from PAPER.md §III-C and DESIGN.md R13':
 *
 *  P:104  "At the moment when user program tries allocation, wrapper module
 *          only knows the requested memory size.  This memory size
 *          information is sent to the scheduler" -> an allocation API becomes
 *          an ALLOC of the size the wrapper computes.
 *  P:106  "cudaMallocPitch API allocates pitched memory ... This pitched size
 *  P:108   varies among the GPU model ... the wrapper module retrieves the
 *          pitched size of current GPU using cudaGetDeviceProperties" ->
 *          size = roundup(width, pitch granule) * height (* depth for
 *          cudaMalloc3D, Table II "similar with cudaMallocPitch, but
 *          specialized in 3D array").  The granule is a parameter; on B200
 *          the runtime's pitch is roundup(width, 512) = textureAlignment
 *          (measured, tests/golden/b200_pitch_probe.json).
 *  P:108  "cudaMallocManaged API allocates memory size which is multiple of
 *          128MiB" -> size rounded up to a multiple of 128 MiB.
 *  P:110  "When user program tries to deallocate GPU memory, wrapper module
 *          knows the address of the memory" and the scheduler "tracks this
 *          information using hash structure" -> a FREE releases the
 *          size recorded for the allocation it names (op a0 of the same
 *          container); naming anything else (a later op, a non-allocation, an
 *          already freed allocation) is a free of memory the container does
 *          not hold: FREE of 2^30 - 1 MiB, which the replay flags
 *          INVALID_FREE (R11).
 *  P:110  "__cudaUnregisterFatBinary ... wrapper module captures this API and
 *          sends the information to the GPU memory scheduler to deallocate"
 *          -> FINISH.
 *  P:129, "cudaMemGetInfo ... ConVGPU already knows the return value of the
 *  P:203   API without using the original CUDA API" -> no memory effect: NOP.
 *  R13'   The scheduler counts MiB (the replay's unit): an allocation of b
 *          bytes is charged ceil(b / 2^20) MiB, saturated at 2^30 - 1 (an
 *          over-limit request).  An unknown API code makes the program
 *          invalid: it maps to a FINISH before the last op, or to a NOP as
 *          the last op, which the replay flags BAD_PROGRAM either way.
 */
#include "oracle.h"

#define MIB (1ull << 20)
#define SIZE_SAT 0x3FFFFFFFu

static uint64_t sat_mul(uint64_t a, uint64_t b) {  /* a * b, saturating */
  if (a != 0 && b > UINT64_MAX / a) return UINT64_MAX;
  return a * b;
}

static uint64_t round_up(uint64_t x, uint64_t g) {  /* smallest multiple of g >= x */
  if (g == 0) return x;
  uint64_t q = x / g + (x % g != 0);
  return sat_mul(q, g);
}

uint64_t orc_wrap_bytes(const orc_api_op_t *op, uint32_t pitch_align) {
  switch (op->api) {
    case ORC_API_MALLOC:
      return (uint64_t)op->a0 | ((uint64_t)op->a1 << 32);
    case ORC_API_MALLOC_MANAGED:
      return round_up((uint64_t)op->a0 | ((uint64_t)op->a1 << 32), 128 * MIB);
    case ORC_API_MALLOC_PITCH:
      return sat_mul(round_up(op->a0, pitch_align), op->a1);
    case ORC_API_MALLOC_3D:
      return sat_mul(sat_mul(round_up(op->a0, pitch_align), op->a1), op->a2);
    default:
      return 0;
  }
}

uint32_t orc_wrap_mib(uint64_t bytes) {
  uint64_t m = bytes / MIB + (bytes % MIB != 0);
  return m > SIZE_SAT ? SIZE_SAT : (uint32_t)m;
}

static int is_alloc_api(uint32_t api) { return api <= ORC_API_MALLOC_3D; }

void orc_wrap_program(const orc_api_op_t *ops, uint32_t K, uint32_t pitch_align,
                      uint32_t *op_words) {
  int freed[ORC_MAX_K] = {0};
  for (uint32_t k = 0; k < K; k++) {
    const orc_api_op_t *op = &ops[k];
    uint32_t w;
    if (is_alloc_api(op->api)) {
      w = ((uint32_t)ORC_ALLOC << 30) | orc_wrap_mib(orc_wrap_bytes(op, pitch_align));
    } else if (op->api == ORC_API_FREE) {
      uint32_t j = op->a0;
      if (j < k && is_alloc_api(ops[j].api) && !freed[j]) {
        freed[j] = 1;
        w = ((uint32_t)ORC_FREE << 30) | orc_wrap_mib(orc_wrap_bytes(&ops[j], pitch_align));
      } else {
        w = ((uint32_t)ORC_FREE << 30) | SIZE_SAT;
      }
    } else if (op->api == ORC_API_MEM_GET_INFO || op->api == ORC_API_COMPUTE) {
      w = (uint32_t)ORC_NOP << 30;
    } else if (op->api == ORC_API_EXIT) {
      w = (uint32_t)ORC_FINISH << 30;
    } else {
      w = (k + 1 < K) ? ((uint32_t)ORC_FINISH << 30) : ((uint32_t)ORC_NOP << 30);
    }
    op_words[k] = w;
  }
}

void orc_wrap_batch(uint32_t n, uint32_t K, uint64_t count, const orc_api_op_t *api,
                    uint32_t pitch_align, uint32_t *arg) {
  orc_api_op_t prog[ORC_MAX_K];
  uint32_t words[ORC_MAX_K];
  for (uint64_t i = 0; i < count; i++) {
    for (uint32_t c = 0; c < n; c++) {
      for (uint32_t k = 0; k < K; k++) prog[k] = api[(i * K + k) * n + c];
      orc_wrap_program(prog, K, pitch_align, words);
      for (uint32_t k = 0; k < K; k++) arg[(i * K + k) * n + c] = words[k];
    }
  }
}
