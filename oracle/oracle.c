/*
 * oracle.c — TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke()
 * and bench.py's cpu_baseline / `--impl reference` leg may load this code.
 * The product path (paper_conf_cluster_kangjkkk17_b200/) never links it.
 *
 * A plain, slow, single-threaded, obviously-sequential replay of ConVGPU's
 * GPU-memory scheduler (§III-D, and the Fig. 3 example,
 * P:147-167), written straight from the paper in its order and notation.
 * Every step cites the passage it follows; where the paper is silent or
 * ambiguous the DESIGN.md reading ("R<n>") is named.  No blocking, fusion or
 * reordering: one event at a time, O(n) scans, explicit per-container state.
 *
 * Pins (tests/test_oracle_*.py): Philox KAT, splitmix64 published outputs,
 * the Fig. 3 narrative (tests/golden/fig3.json), the FIFO/Lindley closed
 * form, the no-contention closed form, policy equivalences, per-event
 * invariants, and an independent brute-force DFS (oracle/bruteforce.py) over
 * every selection choice and every same-tick interleaving on tiny traces.
 */
#include "oracle.h"

#include <stdlib.h>
#include <string.h>

#define TICK_LIMIT (1ull << 26) /* R19: packed (tick, index) horizon */

/* Fault injection, TEST-ONLY (tests/test_oracle_faults.py): a build with
 * -DORC_FAULT=<n> plants one deliberate bug so the tests can show that the
 * invariant checker fires on it.  The normal build defines nothing, and then
 * FAULT(n) is 0 everywhere, so the replay below is unchanged. */
#ifndef ORC_FAULT
#define ORC_FAULT 0
#endif
#define FAULT(n) (ORC_FAULT == (n))

/* ------------------------------------------------------------------ */
/* Philox4x32-10 (Salmon et al., SC'11; Random123 constants).  Used for
 * Random-Fit selection (R6) and the synthetic workload (DESIGN.md recipe). */
void orc_philox4x32_10(const uint32_t ctr_in[4], const uint32_t key_in[2],
                       uint32_t out[4]) {
  uint32_t c0 = ctr_in[0], c1 = ctr_in[1], c2 = ctr_in[2], c3 = ctr_in[3];
  uint32_t k0 = key_in[0], k1 = key_in[1];
  for (int r = 0; r < 10; ++r) {
    if (r > 0) {
      k0 += 0x9E3779B9u;
      k1 += 0xBB67AE85u;
    }
    uint64_t p0 = (uint64_t)0xD2511F53u * c0;
    uint64_t p1 = (uint64_t)0xCD9E8D57u * c2;
    uint32_t hi0 = (uint32_t)(p0 >> 32), lo0 = (uint32_t)p0;
    uint32_t hi1 = (uint32_t)(p1 >> 32), lo1 = (uint32_t)p1;
    uint32_t n0 = hi1 ^ c1 ^ k0;
    uint32_t n1 = lo1;
    uint32_t n2 = hi0 ^ c3 ^ k1;
    uint32_t n3 = lo0;
    c0 = n0; c1 = n1; c2 = n2; c3 = n3;
  }
  out[0] = c0; out[1] = c1; out[2] = c2; out[3] = c3;
}

/* splitmix64 finalizer (Steele, Lea, Flood 2014) — digest mixing (R20). */
uint64_t orc_mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

/* ------------------------------------------------------------------ */
/* Scheduler state.  D1 ledger per container, D3 paused set
 * (P:139-145), D4 global free memory, D5 first-allocation flag
 * (P:135). */
enum { ST_PENDING = 0, ST_LIVE = 1, ST_DONE = 2 };

typedef struct {
  int st;
  uint32_t a;         /* memory assigned (guaranteed) to the container */
  uint32_t used;      /* memory the container's program currently holds */
  uint32_t k;         /* index of the container's next op */
  uint32_t next_tick; /* tick of that op (valid when LIVE and not paused) */
  int paused;         /* allocation reply withheld */
  uint32_t pending;   /* MiB the withheld ALLOC still needs (incl. overhead) */
  uint32_t susp_tick, susp_seq;
  int first_done;     /* first allocation of this pid happened */
  int admitted;
  uint32_t wait, admit_tick, admit_rank, finish;
} cont_t;

typedef struct {
  const orc_trace_t *tr;
  uint32_t cap;
  int policy;
  uint64_t tid, seed;
  uint32_t ovh;
  cont_t c[ORC_MAX_N];
  uint32_t free_mem; /* capacity not assigned to any container */
  int target;        /* R1 sticky fill target, -1 = NONE */
  uint32_t seq, rank, draws;
  uint32_t n_rejected, n_select, peak_reserved, peak_used, flags;
  uint64_t events;
  int stop;
  int check;
  int lit; /* 1 = literal re-select-on-every-release reading (NEXT-1, R1-LIT) */
  int32_t violation;
  uint64_t violation_event;
} sim_t;

static uint32_t op_kind(uint32_t w) { return w >> 30; }
static uint32_t op_size(uint32_t w) { return w & 0x3FFFFFFFu; }
static uint32_t L_of(const sim_t *s, int c) { return s->tr->limit[c]; }
static uint32_t delta_of(const sim_t *s, int c, uint32_t k) {
  return s->tr->delta[(size_t)k * s->tr->n + c];
}
static uint32_t arg_of(const sim_t *s, int c, uint32_t k) {
  return s->tr->arg[(size_t)k * s->tr->n + c];
}

/* ADMIT: the container's declared limit is now fully guaranteed (P:141,
 * "until the assigned memory reaches the required memory size"; R2). */
static void admit(sim_t *s, int c, uint32_t t) {
  s->c[c].admitted = 1;
  s->c[c].admit_tick = t;
  s->c[c].admit_rank = s->rank++;
}

/* "Advance": the op completed at tick t; the next op runs delta later (R17). */
static void advance(sim_t *s, int c, uint32_t t) {
  cont_t *x = &s->c[c];
  x->k += 1;
  if (x->k < s->tr->K) x->next_tick = t + delta_of(s, c, x->k);
}

/* ARRIVE — container creation (the limit is sent to the scheduler
 * before the container is created; P:149 / Fig. 3b: "GPU memory is partially
 * assigned to Container C which is requested at creation time"; Fig. 3c:
 * D "does not have any GPU memory assigned to itself" while C is partial).
 * Reading R2: g = min(L, free) if there is no fill target, else 0. */
static void ev_arrive(sim_t *s, int c, uint32_t t) {
  cont_t *x = &s->c[c];
  uint32_t L = L_of(s, c);
  x->st = ST_LIVE;
  uint32_t g = 0;
  /* R1-LIT: without a sticky target every newcomer takes what is free */
  if (s->lit || s->target < 0) g = (L < s->free_mem) ? L : s->free_mem;
  x->a = g;
  s->free_mem -= g;
  if (g == L || (FAULT(6) && g > 0))
    admit(s, c, t);
  else if (g > 0 && !s->lit)
    s->target = c;
  x->next_tick = t + delta_of(s, c, 0);
}

/* ALLOC — P:104 (size sent, scheduler answers), P:78 (deny over the limit,
 * pause if needed), P:135 (+66 MiB at the pid's first allocation, R12),
 * P:139 (valid request but insufficient memory: reply withheld = pause). */
static void ev_alloc(sim_t *s, int c, uint32_t t, uint32_t r) {
  cont_t *x = &s->c[c];
  uint64_t need = (uint64_t)x->used + r + (x->first_done ? 0u : s->ovh);
  if (need > L_of(s, c)) {            /* over the declared limit: reject (R10) */
    s->n_rejected++;
    advance(s, c, t);
  } else if (need <= x->a || FAULT(3)) { /* within the assigned memory: grant */
    x->used = (uint32_t)need;
    x->first_done = 1;
    advance(s, c, t);
  } else {                            /* valid but not assigned yet: pause */
    x->paused = 1;
    x->pending = (uint32_t)(need - x->used);
    x->susp_tick = t;
    x->susp_seq = s->seq++;
  }
}

/* FREE — P:110: the memory is released by the real cudaFree and the address
 * is un-tracked.  R11: the assignment stays with the container. */
static void ev_free(sim_t *s, int c, uint32_t t, uint32_t r) {
  cont_t *x = &s->c[c];
  if (r > x->used) {
    s->flags |= ORC_F_INVALID_FREE;
    s->stop = 1;
    return;
  }
  x->used -= r;
  advance(s, c, t);
}

/* FINISH — P:110/P:137 (process exit: the pid's allocations are dropped even
 * if never freed, R18) and P:137/P:139 (container stop: its memory goes back
 * to the scheduler, which can assign it to other containers). */
static void ev_finish(sim_t *s, int c, uint32_t t) {
  cont_t *x = &s->c[c];
  if (!FAULT(1)) s->free_mem += x->a;
  x->a = 0;
  x->used = 0;
  x->st = ST_DONE;
  x->finish = t;
  if (s->target == c && !FAULT(5)) s->target = -1; /* R20: target left before it was full */
}

/* SELECT among paused containers. */
static int select_paused(sim_t *s) {
  const orc_trace_t *tr = s->tr;
  int best = -1;
  switch (s->policy) {
    case ORC_FIFO: /* P:141 "oldest created container among paused" (R7) */
      for (uint32_t c = 0; c < tr->n; ++c) {
        if (!s->c[c].paused) continue;
        if (best < 0 || tr->arrival[c] < tr->arrival[best]) best = (int)c;
      }
      return best;
    case ORC_BEST_FIT: { /* P:142; "insufficient memory" = L - a (R3, R4) */
      uint32_t best_need = 0;
      for (uint32_t c = 0; c < tr->n; ++c) {
        if (!s->c[c].paused) continue;
        uint32_t need = L_of(s, (int)c) - s->c[c].a;
        if (need > s->free_mem) continue;   /* must not exceed the remaining */
        if (best < 0 || need > best_need) { /* closest to the remaining */
          best = (int)c;
          best_need = need;
        }
      }
      if (best >= 0) return best;
      for (uint32_t c = 0; c < tr->n; ++c) { /* else least insufficient */
        if (!s->c[c].paused) continue;
        uint32_t need = L_of(s, (int)c) - s->c[c].a;
        if (best < 0 || need < best_need) {
          best = (int)c;
          best_need = need;
        }
      }
      return best;
    }
    case ORC_RECENT: /* P:143 "most recently suspended" (R5) */
      for (uint32_t c = 0; c < tr->n; ++c) {
        if (!s->c[c].paused) continue;
        if (best < 0 || s->c[c].susp_seq > s->c[best].susp_seq) best = (int)c;
      }
      return best;
    case ORC_RANDOM: { /* P:145 "selects randomly among paused" (R6) */
      uint32_t m = 0;
      for (uint32_t c = 0; c < tr->n; ++c) m += s->c[c].paused ? 1u : 0u;
      uint32_t ctr[4] = {(uint32_t)s->tid, (uint32_t)(s->tid >> 32), s->draws, 1u};
      uint32_t key[2] = {(uint32_t)s->seed, (uint32_t)(s->seed >> 32)};
      uint32_t x[4];
      orc_philox4x32_10(ctr, key, x);
      s->draws++;
      uint32_t j = (uint32_t)(((uint64_t)x[0] * m) >> 32);
      for (uint32_t c = 0; c < tr->n; ++c) {
        if (!s->c[c].paused) continue;
        if (j == 0) return (int)c;
        --j;
      }
      return -1;
    }
  }
  return -1;
}

/* DISPATCH — P:139 ("When some container finishes its execution, the
 * scheduler can assign its occupied GPU memory to other containers"),
 * P:141-145 (assign to the selected container "until the assigned memory
 * reaches the required memory size"), P:149 / Fig. 3d (C is guaranteed all
 * its memory and resumes; the remainder goes to D, which stays suspended).
 * Reading R1 (sticky fill target), R9 (resume as soon as the withheld
 * request is covered), R16 (runs after every event). */
static void resume_if_covered(sim_t *s, int c, uint32_t t);

/* DISPATCH under the literal reading R1-LIT: every
 * time memory is free and someone is paused, the policy picks a paused
 * container (shortfall L - a counting partial holds) and
 * assigns it min(free, L - a); partial assignments are kept; the loop goes
 * on while memory is left.  Nothing guarantees progress, so this reading
 * can deadlock (R1). */
static void dispatch_lit(sim_t *s, uint32_t t) {
  for (;;) {
    if (s->free_mem == 0) break;
    int any_paused = 0;
    for (uint32_t c = 0; c < s->tr->n; ++c) any_paused |= s->c[c].paused;
    if (!any_paused) break;
    int x = select_paused(s);
    s->n_select++;
    cont_t *y = &s->c[x];
    uint32_t room = L_of(s, x) - y->a;
    uint32_t g = (s->free_mem < room) ? s->free_mem : room;
    y->a += g;
    s->free_mem -= g;
    resume_if_covered(s, x, t);
    if (y->a == L_of(s, x)) admit(s, x, t);
  }
}

static void resume_if_covered(sim_t *s, int c, uint32_t t) {
  cont_t *x = &s->c[c];
  if (x->paused && (uint64_t)x->used + x->pending <= x->a) { /* RESUME (R9) */
    x->used += x->pending;
    x->first_done = 1;
    x->paused = 0;
    x->wait += t - x->susp_tick;
    advance(s, c, t);
  }
}

static void dispatch(sim_t *s, uint32_t t) {
  if (s->lit) {
    dispatch_lit(s, t);
    return;
  }
  for (;;) {
    if (s->target >= 0) {
      int tg = s->target;
      cont_t *x = &s->c[tg];
      uint32_t L = L_of(s, tg);
      uint32_t room = L - x->a;
      uint32_t g = (s->free_mem < room || FAULT(2)) ? s->free_mem : room;
      x->a += g;
      s->free_mem -= g;
      if (x->paused && (uint64_t)x->used + x->pending <= x->a) { /* RESUME */
        x->used += x->pending;
        x->first_done = 1;
        x->paused = 0;
        if (!FAULT(4)) x->wait += t - x->susp_tick;
        advance(s, tg, t);
      }
      if (x->a == L) {
        admit(s, tg, t);
        s->target = -1;
        continue; /* leftover cascades to the next one, Fig. 3d */
      }
      break;
    }
    int any_paused = 0;
    for (uint32_t c = 0; c < s->tr->n; ++c) any_paused |= s->c[c].paused;
    if (!any_paused) break;
    s->target = select_paused(s);
    s->n_select++;
  }
}

/* ------------------------------------------------------------------ */
/* Invariant checker (test mode).  Ids are reported in orc_result_t. */
static int check_invariants(const sim_t *s) {
  const orc_trace_t *tr = s->tr;
  uint64_t sum_a = 0;
  int partial = 0;
  for (uint32_t c = 0; c < tr->n; ++c) {
    const cont_t *x = &s->c[c];
    uint32_t L = tr->limit[c];
    sum_a += x->a;
    if (x->used > x->a) return 2;            /* used <= a */
    if (x->a > L) return 3;                  /* a <= L */
    if (x->st != ST_LIVE && (x->a || x->used)) return 4;
    if (x->st == ST_LIVE && x->admitted && x->a != L) return 5; /* admitted => full */
    if (x->st == ST_LIVE && x->a > 0 && x->a < L) {
      partial++;
      if (!s->lit && (int)c != s->target) return 6; /* partial => it is the target */
    }
    if (x->paused && x->st != ST_LIVE) return 7;
    if (!s->lit && x->paused && s->target < 0) return 8; /* NONE => none paused */
  }
  if (sum_a + s->free_mem != s->cap) return 1; /* ledger conserves capacity */
  if (s->lit) return 0;
  if (partial > 1) return 9;
  if (s->target >= 0 && s->free_mem != 0) return 10;
  if (s->target >= 0 && s->c[s->target].st != ST_LIVE) return 11;
  return 0;
}

/* ------------------------------------------------------------------ */
static void zero_outputs(sim_t *s) {
  for (uint32_t c = 0; c < ORC_MAX_N; ++c) {
    s->c[c].admit_tick = ORC_NONE32;
    s->c[c].admit_rank = ORC_NONE8;
    s->c[c].wait = 0;
    s->c[c].finish = 0;
  }
}

/* Static validation: bits 2, 4, 5, 6. */
static uint32_t static_flags(const orc_trace_t *tr, uint32_t cap) {
  uint32_t f = 0;
  uint64_t max_arr = 0, sum_delta = 0;
  for (uint32_t c = 0; c < tr->n; ++c) {
    if (tr->limit[c] > cap) f |= ORC_F_INVALID_LIMIT; /* R15 */
    if (c > 0 && tr->arrival[c] < tr->arrival[c - 1]) f |= ORC_F_UNSORTED_ARRIVAL;
    if (tr->arrival[c] > max_arr) max_arr = tr->arrival[c];
    for (uint32_t k = 0; k < tr->K; ++k) {
      sum_delta += tr->delta[(size_t)k * tr->n + c];
      uint32_t kind = op_kind(tr->arg[(size_t)k * tr->n + c]);
      if ((k + 1 == tr->K) != (kind == ORC_FINISH)) f |= ORC_F_BAD_PROGRAM;
    }
  }
  /* R19: every tick of a deadlock-free replay is <= max arrival + sum of all
   * deltas (DESIGN.md proof); flag traces whose horizon reaches 2^26. */
  if (max_arr + sum_delta >= TICK_LIMIT) f |= ORC_F_TICK_RANGE;
  return f;
}

int orc_replay(const orc_trace_t *tr, uint32_t cap, int policy_mode, uint64_t tid,
               uint64_t rand_seed, uint32_t ovh, int check, orc_result_t *res) {
  const int policy = policy_mode & 0xFF, lit = (policy_mode & ORC_LITERAL) != 0;
  if (!tr || !res || tr->n < 1 || tr->n > ORC_MAX_N || tr->K < 1 ||
      tr->K > ORC_MAX_K || policy < 0 || policy > 3 || (policy_mode & ~(0xFF | ORC_LITERAL)) ||
      cap == 0)
    return -1;
  sim_t *s = (sim_t *)calloc(1, sizeof(sim_t));
  if (!s) return -2;
  s->tr = tr;
  s->cap = cap;
  s->policy = policy;
  s->tid = tid;
  s->seed = rand_seed;
  s->ovh = ovh;
  s->free_mem = cap;
  s->target = -1;
  s->check = check;
  s->lit = lit;
  for (uint32_t c = 0; c < tr->n; ++c) {
    s->c[c].st = ST_PENDING;
    s->c[c].admit_tick = ORC_NONE32;
    s->c[c].admit_rank = ORC_NONE8;
  }
  s->flags = static_flags(tr, cap);
  if (s->flags) s->stop = 1;

  while (!s->stop) {
    int live = 0;
    for (uint32_t c = 0; c < tr->n; ++c) live |= (s->c[c].st != ST_DONE);
    if (!live) break;
    /* Candidate events, total order by (tick, index) — P:133 "each step is
     * protected by a mutex lock": one event at a time (R16). */
    int bc = -1;
    uint32_t bt = 0;
    for (uint32_t c = 0; c < tr->n; ++c) {
      uint32_t t;
      if (s->c[c].st == ST_PENDING)
        t = tr->arrival[c];
      else if (s->c[c].st == ST_LIVE && !s->c[c].paused)
        t = s->c[c].next_tick;
      else
        continue;
      if (bc < 0 || t < bt) { bc = (int)c; bt = t; }
    }
    if (bc < 0) { /* nothing can ever run again */
      s->flags |= ORC_F_DEADLOCK;
      s->stop = 1;
      break;
    }
    s->events++;
    cont_t *x = &s->c[bc];
    if (x->st == ST_PENDING) {
      ev_arrive(s, bc, bt);
    } else {
      uint32_t w = arg_of(s, bc, x->k);
      switch (op_kind(w)) {
        case ORC_ALLOC: ev_alloc(s, bc, bt, op_size(w)); break;
        case ORC_FREE: ev_free(s, bc, bt, op_size(w)); break;
        case ORC_FINISH: ev_finish(s, bc, bt); break;
        default: advance(s, bc, bt); break; /* NOP */
      }
    }
    if (s->stop) break;
    dispatch(s, bt);
    uint64_t sum_used = 0;
    for (uint32_t c = 0; c < tr->n; ++c) sum_used += s->c[c].used;
    uint32_t reserved = cap - s->free_mem;
    if (reserved > s->peak_reserved) s->peak_reserved = reserved;
    if (sum_used > s->peak_used) s->peak_used = (uint32_t)sum_used;
    /* OVERCOMMIT: memory in use exceeds the memory reserved. */
    if (s->free_mem > cap || sum_used > (uint64_t)reserved) s->flags |= ORC_F_OVERCOMMIT;
    if (check && !s->violation) {
      int v = check_invariants(s);
      if (v) { s->violation = v; s->violation_event = s->events; }
    }
  }

  memset(res, 0, sizeof(*res));
  res->flags = s->flags;
  res->events = s->events;
  if (s->flags & (ORC_F_DEADLOCK | ORC_F_INVALID_LIMIT | ORC_F_INVALID_FREE |
                  ORC_F_UNSORTED_ARRIVAL | ORC_F_TICK_RANGE | ORC_F_BAD_PROGRAM)) {
    zero_outputs(s);
    s->peak_reserved = s->peak_used = 0;
    s->n_rejected = s->n_select = 0;
  } else if (check && !s->violation) {
    /* R17: finish = arrival + sum of deltas + suspended time, exactly. */
    for (uint32_t c = 0; c < tr->n; ++c) {
      uint64_t sd = 0;
      for (uint32_t k = 0; k < tr->K; ++k) sd += delta_of(s, (int)c, k);
      if ((uint64_t)tr->arrival[c] + sd + s->c[c].wait != s->c[c].finish) {
        s->violation = 12;
        break;
      }
    }
  }
  /* Outputs (R21): per container admit tick/rank, wait, finish; per trace
   * makespan = max finish - first arrival (Table IV "finished time"),
   * sum of suspended time (Table V), peaks, counters, digest. */
  uint32_t maxfin = 0;
  uint64_t sum_wait = 0;
  for (uint32_t c = 0; c < tr->n; ++c) {
    res->admit_tick[c] = s->c[c].admit_tick;
    res->admit_rank[c] = s->c[c].admit_rank;
    res->wait[c] = s->c[c].wait;
    res->finish[c] = s->c[c].finish;
    if (s->c[c].finish > maxfin) maxfin = s->c[c].finish;
    sum_wait += s->c[c].wait;
  }
  int stopped = (s->flags & ~ORC_F_OVERCOMMIT) != 0;
  res->makespan = stopped ? 0 : maxfin - tr->arrival[0];
  res->peak_reserved = s->peak_reserved;
  res->peak_used = s->peak_used;
  res->sum_wait = sum_wait;
  res->n_rejected = s->n_rejected;
  res->n_select = s->n_select;
  res->violation = s->violation;
  res->violation_event = s->violation_event;
  /* Digest (R20): order-independent over containers, keyed by position. */
  uint64_t d = 0;
  for (uint32_t c = 0; c < tr->n; ++c) {
    uint64_t h1 = orc_mix64(((uint64_t)c << 56) ^ ((uint64_t)res->admit_rank[c] << 48) ^
                            (uint64_t)res->admit_tick[c]);
    d += orc_mix64(h1 ^ (((uint64_t)res->wait[c] << 32) | res->finish[c]));
  }
  d += orc_mix64(((uint64_t)res->makespan << 32) | res->peak_reserved);
  d += orc_mix64(((uint64_t)res->peak_used << 32) | res->flags);
  d += orc_mix64(res->sum_wait);
  d += orc_mix64(((uint64_t)res->n_rejected << 32) | res->n_select);
  res->digest = d;
  free(s);
  return 0;
}

/* ------------------------------------------------------------------ */
/* Synthetic workload (DESIGN.md §Input recipe; "choosing the type of
 * the containers randomly and running it every five seconds", Table III
 * classes P:181-187, durations "from 5 seconds to 45 seconds" by size R22). */
int orc_generate(const orc_gen_params_t *p, uint64_t tid, uint32_t *arrival,
                 uint32_t *limit, uint32_t *delta, uint32_t *arg) {
  if (!p || p->n < 1 || p->n > ORC_MAX_N || (p->K != 4 && p->K != 2) ||
      p->n_classes < 1 || p->n_classes > 8 || p->den == 0)
    return -1;
  uint32_t n = p->n;
  uint32_t key[2] = {(uint32_t)p->gen_seed, (uint32_t)(p->gen_seed >> 32)};
  for (uint32_t c = 0; c < n; ++c) {
    uint32_t ctr[4] = {(uint32_t)tid, (uint32_t)(tid >> 32), c, 0u};
    uint32_t x[4];
    orc_philox4x32_10(ctr, key, x);
    uint32_t k = (uint32_t)(((uint64_t)x[0] * p->n_classes) >> 32);
    uint32_t L = (uint32_t)((uint64_t)p->class_mib[k] * p->num / p->den);
    uint32_t jit = (uint32_t)(((uint64_t)x[1] * ((uint64_t)p->dur_jit + 1)) >> 32);
    uint32_t dur = p->dur_base + p->dur_step * (k + p->dur_class_offset) + jit;
    uint32_t eff = L > p->ovh ? L - p->ovh : 0;
    arrival[c] = c * p->iat;
    limit[c] = L;
    if (p->K == 4) { /* split program: two ALLOCs, one FREE, FINISH */
      uint32_t s1 = eff / 2, s2 = eff - s1;
      uint32_t d1 = dur / 4, d2 = dur / 2;
      delta[0 * n + c] = 0;            arg[0 * n + c] = (ORC_ALLOC << 30) | s1;
      delta[1 * n + c] = d1;           arg[1 * n + c] = (ORC_ALLOC << 30) | s2;
      delta[2 * n + c] = d2;           arg[2 * n + c] = (ORC_FREE << 30) | s1;
      delta[3 * n + c] = dur - d1 - d2; arg[3 * n + c] = (uint32_t)ORC_FINISH << 30;
    } else { /* paper-mimic: allocate the whole limit, run, exit */
      delta[0 * n + c] = 0;   arg[0 * n + c] = (ORC_ALLOC << 30) | eff;
      delta[1 * n + c] = dur; arg[1 * n + c] = (uint32_t)ORC_FINISH << 30;
    }
  }
  return 0;
}

/* ------------------------------------------------------------------ */
static void accumulate(orc_stats_t *st, const orc_result_t *r) {
  st->traces++;
  st->events += r->events;
  st->sum_makespan += r->makespan;
  st->sum_wait += r->sum_wait;
  st->n_rejected += r->n_rejected;
  st->n_select += r->n_select;
  st->digest_sum += r->digest;
  if (r->makespan > st->max_makespan) st->max_makespan = r->makespan;
  if (r->peak_reserved > st->max_peak_reserved) st->max_peak_reserved = r->peak_reserved;
  for (int b = 0; b < 8; ++b)
    if (r->flags & (1u << b)) st->flag_count[b]++;
}

static void store(uint64_t i, uint32_t n, const orc_result_t *r, uint32_t *sum_u32x4,
                  uint64_t *sum_u64x2, uint32_t *cnt_u32x2, uint32_t *admit_tick,
                  uint8_t *admit_rank, uint32_t *wait, uint32_t *finish) {
  if (sum_u32x4) {
    sum_u32x4[i * 4 + 0] = r->makespan;
    sum_u32x4[i * 4 + 1] = r->peak_reserved;
    sum_u32x4[i * 4 + 2] = r->peak_used;
    sum_u32x4[i * 4 + 3] = r->flags;
  }
  if (sum_u64x2) {
    sum_u64x2[i * 2 + 0] = r->sum_wait;
    sum_u64x2[i * 2 + 1] = r->digest;
  }
  if (cnt_u32x2) {
    cnt_u32x2[i * 2 + 0] = r->n_rejected;
    cnt_u32x2[i * 2 + 1] = r->n_select;
  }
  for (uint32_t c = 0; c < n; ++c) {
    if (admit_tick) admit_tick[i * n + c] = r->admit_tick[c];
    if (admit_rank) admit_rank[i * n + c] = (uint8_t)r->admit_rank[c];
    if (wait) wait[i * n + c] = r->wait[c];
    if (finish) finish[i * n + c] = r->finish[c];
  }
}

int orc_replay_range(const orc_gen_params_t *p, uint32_t cap, int policy,
                     uint64_t rand_seed, uint32_t ovh, uint64_t tid_lo,
                     uint64_t tid_hi, int check, orc_stats_t *stats,
                     uint32_t *sum_u32x4, uint64_t *sum_u64x2, uint32_t *cnt_u32x2,
                     uint32_t *admit_tick, uint8_t *admit_rank, uint32_t *wait,
                     uint32_t *finish) {
  uint32_t arrival[ORC_MAX_N], limit[ORC_MAX_N];
  uint32_t delta[ORC_MAX_N * ORC_MAX_K], arg[ORC_MAX_N * ORC_MAX_K];
  orc_result_t r;
  int worst = 0;
  for (uint64_t tid = tid_lo; tid < tid_hi; ++tid) {
    if (orc_generate(p, tid, arrival, limit, delta, arg)) return -1;
    orc_trace_t tr = {p->n, p->K, arrival, limit, delta, arg};
    if (orc_replay(&tr, cap, policy, tid, rand_seed, ovh, check, &r)) return -1;
    if (r.violation && !worst) worst = r.violation;
    if (stats) accumulate(stats, &r);
    store(tid - tid_lo, p->n, &r, sum_u32x4, sum_u64x2, cnt_u32x2, admit_tick,
          admit_rank, wait, finish);
  }
  return worst ? 1000 + worst : 0;
}

int orc_replay_batch(uint32_t n, uint32_t K, uint64_t count, const uint32_t *arrival,
                     const uint32_t *limit, const uint32_t *delta, const uint32_t *arg,
                     uint32_t cap, int policy, uint64_t tid_base, uint64_t rand_seed,
                     uint32_t ovh, int check, orc_stats_t *stats, uint32_t *sum_u32x4,
                     uint64_t *sum_u64x2, uint32_t *cnt_u32x2, uint32_t *admit_tick,
                     uint8_t *admit_rank, uint32_t *wait, uint32_t *finish) {
  orc_result_t r;
  int worst = 0;
  for (uint64_t i = 0; i < count; ++i) {
    orc_trace_t tr = {n, K, arrival + i * n, limit + i * n, delta + i * (uint64_t)K * n,
                      arg + i * (uint64_t)K * n};
    if (orc_replay(&tr, cap, policy, tid_base + i, rand_seed, ovh, check, &r)) return -1;
    if (r.violation && !worst) worst = r.violation;
    if (stats) accumulate(stats, &r);
    store(i, n, &r, sum_u32x4, sum_u64x2, cnt_u32x2, admit_tick, admit_rank, wait, finish);
  }
  return worst ? 1000 + worst : 0;
}
