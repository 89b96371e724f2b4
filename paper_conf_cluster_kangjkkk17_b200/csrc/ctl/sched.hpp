// sched.hpp — NEXT-4: ConVGPU's GPU-memory scheduler as a live state machine
// (§III-D, Fig. 3), the rules of DESIGN.md §2
// (R1 sticky fill target, R2-R12, R16) applied one message at a time.
// Units are whatever the caller uses (bytes in convgpud, MiB in trace-driven
// tests); product code, independent of oracle/.
#pragma once
#include <cstdint>
#include <unordered_map>
#include <vector>

namespace convgpud {

enum Policy { FIFO = 0, BEST_FIT = 1, RECENT_FIT = 2, RANDOM_FIT = 3 };

enum class AllocResult { Grant, Reject, Pause };

struct Container {
  uint64_t L = 0;          // declared limit
  uint64_t a = 0;          // memory assigned to it (reserved)
  uint64_t used = 0;       // memory it uses (granted requests)
  uint64_t pend = 0;       // paused request: memory still needed beyond `used`
  uint32_t index = 0;      // creation order (FIFO, R7; tie-breaks)
  uint64_t seq = 0;        // suspension number of the current pause (Recent-Fit, R5)
  bool admitted = false;   // a == L
  bool paused = false;     // reply withheld
  bool done = false;       // finished
  uint32_t admit_rank = ~0u;
  std::unordered_map<uint64_t, uint64_t> addr;  // device address -> size
};

class Scheduler {
 public:
  // cap: capacity; ovh: context charged at a process's first granted
  // allocation; tid / seed: Random-Fit's Philox counter and key (R6).
  Scheduler(uint64_t cap, Policy policy, uint64_t ovh, uint64_t tid, uint64_t seed);

  // ARRIVE (R2): returns the container id (= creation index).
  uint32_t arrive(uint64_t limit);
  // ALLOC (R10, R12).  first: the calling process has not
  // had an allocation granted yet (its context is charged now).
  AllocResult alloc(uint32_t c, uint64_t r, bool first);
  // A granted request that the device then failed to allocate: undo it.
  void alloc_failed(uint32_t c, uint64_t r);
  // FREE (R11): false if r exceeds what the container uses.
  bool free_bytes(uint32_t c, uint64_t r);
  // FINISH (R18): release everything the container holds.
  void finish(uint32_t c);
  // The process whose ALLOC paused container c went away before the reply:
  // withdraw that request (c leaves the paused set; its assignment and, if it
  // is the fill target, its target role stay).  Returns true if c was paused.
  bool cancel_pause(uint32_t c);
  // Containers resumed by the last step, in resume order (their withheld
  // ALLOC replies are due).
  std::vector<uint32_t> take_resumed();

  const Container& get(uint32_t c) const { return cs_[c]; }
  Container& get(uint32_t c) { return cs_[c]; }
  uint64_t free_pool() const { return free_; }
  uint64_t selections() const { return n_select_; }
  uint64_t rejections() const { return n_reject_; }
  uint64_t peak_reserved() const { return peak_res_; }
  uint32_t size() const { return (uint32_t)cs_.size(); }

 private:
  void dispatch();                  // fill / resume / admit cascade (R1, R9)
  int select();                     // SELECT among paused (R3-R7)
  void admit(uint32_t c);
  void note_peak() { peak_res_ = cap_ - free_ > peak_res_ ? cap_ - free_ : peak_res_; }

  uint64_t cap_, free_, ovh_, tid_, seed_;
  Policy policy_;
  int target_ = -1;                 // sticky fill target (R1)
  uint64_t seq_ = 0, draws_ = 0, n_select_ = 0, n_reject_ = 0, peak_res_ = 0;
  uint32_t rank_ = 0;
  std::vector<Container> cs_;
  std::vector<uint32_t> resumed_;
};

}  // namespace convgpud
