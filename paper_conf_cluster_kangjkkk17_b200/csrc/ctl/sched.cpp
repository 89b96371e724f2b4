// sched.cpp — the scheduler state machine of sched.hpp.  Each public call is
// one serialised scheduler step ("Each step is protected by a mutex
// lock"); every step that can change free memory or the paused set ends with
// DISPATCH (R16).
#include "sched.hpp"

#include <algorithm>

namespace convgpud {

namespace {

// Philox4x32-10 (Salmon et al., SC'11), the Random-Fit draw of R6: counter
// (lo tid, hi tid, draws, 1), key = seed; the first output word is used.
uint32_t philox_x0(uint32_t c0, uint32_t c1, uint32_t c2, uint32_t c3, uint32_t k0, uint32_t k1) {
  for (int r = 0; r < 10; ++r) {
    const uint64_t p0 = (uint64_t)0xD2511F53u * c0, p1 = (uint64_t)0xCD9E8D57u * c2;
    const uint32_t n0 = (uint32_t)(p1 >> 32) ^ c1 ^ k0, n2 = (uint32_t)(p0 >> 32) ^ c3 ^ k1;
    c1 = (uint32_t)p1;
    c3 = (uint32_t)p0;
    c0 = n0;
    c2 = n2;
    k0 += 0x9E3779B9u;
    k1 += 0xBB67AE85u;
  }
  return c0;
}

}  // namespace

Scheduler::Scheduler(uint64_t cap, Policy policy, uint64_t ovh, uint64_t tid, uint64_t seed)
    : cap_(cap), free_(cap), ovh_(ovh), tid_(tid), seed_(seed), policy_(policy) {}

void Scheduler::admit(uint32_t c) {
  cs_[c].admitted = true;
  cs_[c].admit_rank = rank_++;
}

uint32_t Scheduler::arrive(uint64_t limit) {
  Container k;
  k.L = limit;
  k.index = (uint32_t)cs_.size();
  cs_.push_back(k);
  const uint32_t c = k.index;
  // R2: the new container takes min(L, free) unless a fill target is waiting
  const uint64_t g = target_ < 0 ? std::min(limit, free_) : 0;
  cs_[c].a = g;
  free_ -= g;
  if (g == limit)
    admit(c);
  else if (g > 0)
    target_ = (int)c;
  note_peak();
  return c;
}

AllocResult Scheduler::alloc(uint32_t c, uint64_t r, bool first) {
  Container& k = cs_[c];
  const uint64_t need = k.used + r + (first ? ovh_ : 0);
  if (need > k.L) {  // R10: over the declared limit
    ++n_reject_;
    return AllocResult::Reject;
  }
  if (need <= k.a) {
    k.used = need;
    return AllocResult::Grant;
  }
  k.paused = true;  // withhold the reply
  k.pend = need - k.used;
  k.seq = seq_++;
  dispatch();  // with no fill target, a selection starts now
  if (!k.paused) {  // resumed within the same step
    resumed_.erase(std::remove(resumed_.begin(), resumed_.end(), c), resumed_.end());
    return AllocResult::Grant;
  }
  return AllocResult::Pause;
}

void Scheduler::alloc_failed(uint32_t c, uint64_t r) {
  Container& k = cs_[c];
  k.used = k.used > r ? k.used - r : 0;
}

bool Scheduler::free_bytes(uint32_t c, uint64_t r) {
  Container& k = cs_[c];
  if (r > k.used) return false;  // R11 INVALID_FREE
  k.used -= r;                   // R11: cudaFree gives nothing back to the pool
  return true;
}

void Scheduler::finish(uint32_t c) {
  Container& k = cs_[c];
  if (k.done) return;
  free_ += k.a;  // R18: everything returns to the pool
  k.a = k.used = 0;
  k.done = true;
  k.paused = false;
  if (target_ == (int)c) target_ = -1;
  dispatch();
}

bool Scheduler::cancel_pause(uint32_t c) {
  Container& k = cs_[c];
  if (!k.paused) return false;
  k.paused = false;
  k.pend = 0;
  // a resume of c recorded in this step would now deliver a grant to the
  // next queued request without its own admission check
  resumed_.erase(std::remove(resumed_.begin(), resumed_.end(), c), resumed_.end());
  return true;
}

int Scheduler::select() {
  int best = -1;
  for (uint32_t c = 0; c < cs_.size(); ++c) {
    const Container& k = cs_[c];
    if (!k.paused) continue;
    if (best < 0) { best = (int)c; continue; }
    const Container& b = cs_[best];
    switch (policy_) {
      case FIFO:  // R7: oldest created (ids are in creation order)
        break;
      case BEST_FIT: {  // R3, R4: largest shortfall that fits, else the smallest
        const uint64_t sk = k.L - k.a, sb = b.L - b.a;
        const bool fk = sk <= free_, fb = sb <= free_;
        if (fk != fb) { if (fk) best = (int)c; }
        else if (fk ? sk > sb : sk < sb) best = (int)c;
        break;
      }
      case RECENT_FIT:  // R5: the most recent suspension
        if (k.seq > b.seq) best = (int)c;
        break;
      case RANDOM_FIT:
        break;
    }
  }
  if (policy_ == RANDOM_FIT && best >= 0) {  // R6: j-th paused container by index
    uint32_t m = 0;
    for (const Container& k : cs_) m += k.paused ? 1u : 0u;
    const uint32_t x = philox_x0((uint32_t)tid_, (uint32_t)(tid_ >> 32), (uint32_t)draws_, 1u,
                                 (uint32_t)seed_, (uint32_t)(seed_ >> 32));
    ++draws_;
    uint32_t j = (uint32_t)(((uint64_t)x * m) >> 32);
    for (uint32_t c = 0; c < cs_.size(); ++c)
      if (cs_[c].paused && j-- == 0) { best = (int)c; break; }
  }
  return best;
}

void Scheduler::dispatch() {
  for (;;) {
    if (target_ < 0) {
      const int s = select();
      if (s < 0) return;
      target_ = s;
      ++n_select_;
    }
    Container& k = cs_[target_];
    const uint64_t g = std::min(free_, k.L - k.a);  // R1: fill the target
    k.a += g;
    free_ -= g;
    note_peak();
    if (k.paused && k.used + k.pend <= k.a) {  // R9: resume when covered
      k.paused = false;
      k.used += k.pend;
      k.pend = 0;
      resumed_.push_back((uint32_t)target_);
    }
    if (k.a == k.L) {  // admitted: the leftover cascades (Fig. 3d)
      admit((uint32_t)target_);
      target_ = -1;
      continue;
    }
    return;
  }
}

std::vector<uint32_t> Scheduler::take_resumed() {
  std::vector<uint32_t> r;
  r.swap(resumed_);
  return r;
}

}  // namespace convgpud
