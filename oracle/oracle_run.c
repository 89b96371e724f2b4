/*
 * oracle_run — TEST INFRASTRUCTURE ONLY: command-line driver of the plain C
 * oracle (oracle.c).  Generates and replays global trace ids [lo, hi) of a
 * synthetic workload single-threaded and prints one JSON line with the
 * aggregate statistics and per-range digests (sum of trace digests mod 2^64
 * over consecutive blocks of --range-size ids).  Used for large-range parity
 * (config [3] digests) and as the CPU baseline; runs one process per core
 * when the caller launches several on disjoint ranges.
 *
 *   oracle_run --n 64 --K 4 --classes 128,256,512,1024,2048,4096 --num 30
 *              --den 7 --iat 100 --cap 184320 --policy 1 --lo 0 --hi 100000
 *              [--gen-seed S] [--rand-seed S] [--ovh M] [--dur-base B]
 *              [--dur-step S] [--dur-off O] [--dur-jit J] [--range-size R]
 */
#define _POSIX_C_SOURCE 199309L
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <time.h>

#include "oracle.h"

static uint64_t num(const char *s) { return strtoull(s, NULL, 0); }

int main(int argc, char **argv) {
  orc_gen_params_t p;
  memset(&p, 0, sizeof p);
  p.gen_seed = 0x00C0FFEE; p.n = 64; p.K = 4; p.num = 1; p.den = 1; p.iat = 5000;
  p.dur_base = 5000; p.dur_step = 8000;
  uint32_t defaults[6] = {128, 256, 512, 1024, 2048, 4096};
  p.n_classes = 6;
  memcpy(p.class_mib, defaults, sizeof defaults);
  uint32_t cap = 184320, ovh = 0;
  int policy = 0;
  uint64_t seed = 0, lo = 0, hi = 1000, rsize = 1u << 20;
  for (int i = 1; i + 1 < argc; i += 2) {
    const char *k = argv[i], *v = argv[i + 1];
    if (!strcmp(k, "--n")) p.n = (uint32_t)num(v);
    else if (!strcmp(k, "--K")) p.K = (uint32_t)num(v);
    else if (!strcmp(k, "--num")) p.num = (uint32_t)num(v);
    else if (!strcmp(k, "--den")) p.den = (uint32_t)num(v);
    else if (!strcmp(k, "--iat")) p.iat = (uint32_t)num(v);
    else if (!strcmp(k, "--gen-seed")) p.gen_seed = num(v);
    else if (!strcmp(k, "--dur-base")) p.dur_base = (uint32_t)num(v);
    else if (!strcmp(k, "--dur-step")) p.dur_step = (uint32_t)num(v);
    else if (!strcmp(k, "--dur-off")) p.dur_class_offset = (uint32_t)num(v);
    else if (!strcmp(k, "--dur-jit")) p.dur_jit = (uint32_t)num(v);
    else if (!strcmp(k, "--gen-ovh")) p.ovh = (uint32_t)num(v);
    else if (!strcmp(k, "--ovh")) ovh = (uint32_t)num(v);
    else if (!strcmp(k, "--cap")) cap = (uint32_t)num(v);
    else if (!strcmp(k, "--policy")) policy = (int)num(v);
    else if (!strcmp(k, "--rand-seed")) seed = num(v);
    else if (!strcmp(k, "--lo")) lo = num(v);
    else if (!strcmp(k, "--hi")) hi = num(v);
    else if (!strcmp(k, "--range-size")) rsize = num(v);
    else if (!strcmp(k, "--classes")) {
      p.n_classes = 0;
      char buf[256];
      strncpy(buf, v, sizeof buf - 1);
      buf[sizeof buf - 1] = 0;
      for (char *tok = strtok(buf, ","); tok && p.n_classes < 8; tok = strtok(NULL, ","))
        p.class_mib[p.n_classes++] = (uint32_t)num(tok);
    } else {
      fprintf(stderr, "unknown option %s\n", k);
      return 2;
    }
  }
  if (hi < lo || rsize == 0) return 2;
  uint64_t r_first = lo / rsize, r_last = hi ? (hi - 1) / rsize : 0;
  uint64_t nr = hi > lo ? r_last - r_first + 1 : 0;
  uint64_t *rd = (uint64_t *)calloc(nr ? nr : 1, sizeof(uint64_t));
  uint64_t *dg = (uint64_t *)malloc(sizeof(uint64_t) * 2 * 4096);
  orc_stats_t st;
  memset(&st, 0, sizeof st);
  struct timespec t0, t1;
  clock_gettime(CLOCK_MONOTONIC, &t0);
  for (uint64_t a = lo; a < hi; a += 4096) {
    uint64_t b = a + 4096 < hi ? a + 4096 : hi;
    int rc = orc_replay_range(&p, cap, policy, seed, ovh, a, b, 0, &st, NULL, dg, NULL,
                              NULL, NULL, NULL, NULL);
    if (rc) { fprintf(stderr, "oracle rc=%d\n", rc); return 1; }
    for (uint64_t t = a; t < b; ++t) rd[t / rsize - r_first] += dg[(t - a) * 2 + 1];
  }
  clock_gettime(CLOCK_MONOTONIC, &t1);
  double secs = (double)(t1.tv_sec - t0.tv_sec) + 1e-9 * (double)(t1.tv_nsec - t0.tv_nsec);
  printf("{\"lo\": %llu, \"hi\": %llu, \"policy\": %d, \"seconds\": %.6f, \"traces\": %llu, "
         "\"events\": %llu, \"sum_makespan\": %llu, \"sum_wait\": %llu, \"n_rejected\": %llu, "
         "\"n_select\": %llu, \"digest_sum\": %llu, \"max_makespan\": %u, "
         "\"max_peak_reserved\": %u, \"flag_count\": [",
         (unsigned long long)lo, (unsigned long long)hi, policy, secs,
         (unsigned long long)st.traces, (unsigned long long)st.events,
         (unsigned long long)st.sum_makespan, (unsigned long long)st.sum_wait,
         (unsigned long long)st.n_rejected, (unsigned long long)st.n_select,
         (unsigned long long)st.digest_sum, st.max_makespan, st.max_peak_reserved);
  for (int b = 0; b < 8; ++b) printf("%s%u", b ? ", " : "", st.flag_count[b]);
  printf("], \"range_size\": %llu, \"range_first\": %llu, \"range_digests\": [",
         (unsigned long long)rsize, (unsigned long long)r_first);
  for (uint64_t i = 0; i < nr; ++i) printf("%s\"%016llx\"", i ? ", " : "", (unsigned long long)rd[i]);
  printf("]}\n");
  free(rd);
  free(dg);
  return 0;
}
