// convgpud.cpp — NEXT-4: the host GPU-memory scheduler daemon of ConVGPU
// (§III-D) for B200 hosts, speaking include/convgpu_ctl.h
// over a UNIX socket.  One process per host; a single-threaded poll loop, so
// every message is one serialised scheduler step.
//
//   convgpud --socket PATH [--capacity-mib M | --capacity B] [--policy fifo|
//            best_fit|recent_fit|random_fit] [--overhead-mib 66 | --overhead B]
//            [--seed S] [--tid T]
//
// Units: bytes unless the -mib forms are used; a trace driver may speak in any
// unit as long as capacity / overhead use the same one.  Capacity defaults to
// the device memory of a B200 as cudaMemGetInfo reports it is NOT assumed:
// it must be given.  The daemon never touches the GPU itself.
#include <errno.h>
#include <poll.h>
#include <signal.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <sys/socket.h>
#include <sys/un.h>
#include <unistd.h>

#include <deque>
#include <string>
#include <unordered_map>
#include <vector>

#include "convgpu_ctl.h"
#include "sched.hpp"

namespace {

using convgpud::AllocResult;
using convgpud::Scheduler;

struct Conn {
  int fd = -1;
  int container = -1;  // scheduler id after HELLO
  uint32_t pid = 0;
  bool first = true;   // no allocation granted to this process yet
  bool exited = false;
  std::string in;      // partial message bytes
  // an ALLOC whose reply is withheld, or queued behind another
  // process of the same container that is paused
  bool waiting = false;
  uint64_t wait_bytes = 0;
};

struct ContainerInfo {
  int live_procs = 0;
  std::deque<int> queue;  // connections with an ALLOC waiting on this container
};

Scheduler* g_s = nullptr;
std::vector<Conn> g_conns;
std::unordered_map<uint64_t, int> g_key2c;  // container key -> scheduler id
std::vector<ContainerInfo> g_ci;
uint64_t g_handled = 0;  // messages handled so far (CONVGPU_MSG_SYNC)

void send_reply(Conn& k, int32_t status, uint32_t type, uint64_t a = 0, uint64_t b = 0,
                uint64_t c = 0) {
  convgpu_reply_t r{status, type, a, b, c};
  const char* p = reinterpret_cast<const char*>(&r);
  size_t left = sizeof r;
  while (left > 0) {
    const ssize_t w = send(k.fd, p, left, MSG_NOSIGNAL);
    if (w < 0) {
      if (errno == EINTR) continue;
      return;  // the peer is gone; its disconnect is handled by the poll loop
    }
    p += w;
    left -= (size_t)w;
  }
}

void deliver_resumed();

// Start the ALLOC at the head of container c's queue, if the container is
// not paused.  Replies to grants / rejects immediately.
void pump(int c) {
  ContainerInfo& ci = g_ci[c];
  while (!ci.queue.empty() && !g_s->get(c).paused) {
    Conn& k = g_conns[ci.queue.front()];
    const AllocResult res = g_s->alloc(c, k.wait_bytes, k.first);
    if (res == AllocResult::Pause) return;  // reply withheld until resumed
    ci.queue.pop_front();
    k.waiting = false;
    if (res == AllocResult::Grant) {
      k.first = false;
      send_reply(k, CONVGPU_ST_OK, CONVGPU_MSG_ALLOC);
    } else {
      send_reply(k, CONVGPU_ST_REJECT, CONVGPU_MSG_ALLOC);
    }
  }
}

void deliver_resumed() {
  for (;;) {
    std::vector<uint32_t> rs = g_s->take_resumed();
    if (rs.empty()) return;
    for (uint32_t c : rs) {
      ContainerInfo& ci = g_ci[c];
      if (ci.queue.empty()) continue;
      Conn& k = g_conns[ci.queue.front()];
      ci.queue.pop_front();
      k.waiting = false;
      k.first = false;
      send_reply(k, CONVGPU_ST_OK, CONVGPU_MSG_ALLOC);
      pump((int)c);
    }
  }
}

void process_exit(Conn& k) {
  if (k.exited || k.container < 0) return;
  k.exited = true;
  ContainerInfo& ci = g_ci[k.container];
  if (--ci.live_procs == 0) g_s->finish((uint32_t)k.container);
  deliver_resumed();
}

void handle_one(int idx, const convgpu_msg_t& m);

void handle(int idx, const convgpu_msg_t& m) {
  handle_one(idx, m);
  ++g_handled;
}

void handle_one(int idx, const convgpu_msg_t& m) {
  Conn& k = g_conns[idx];
  // queries that need no container (a driver's or operator's control connection)
  if (m.type == CONVGPU_MSG_SYNC) {
    send_reply(k, CONVGPU_ST_OK, m.type, g_handled);
    return;
  }
  if (m.type == CONVGPU_MSG_STATS) {
    send_reply(k, CONVGPU_ST_OK, m.type, g_s->free_pool(), g_s->selections(), g_s->rejections());
    return;
  }
  if (m.type == CONVGPU_MSG_INFO && m.a != ~0ull) {
    if (m.a >= g_s->size()) { send_reply(k, CONVGPU_ST_INVALID, m.type); return; }
    const auto& ct = g_s->get((uint32_t)m.a);
    send_reply(k, CONVGPU_ST_OK, m.type, ct.a, ct.used,
               ct.admit_rank == ~0u ? ~0ull : (uint64_t)ct.admit_rank);
    return;
  }
  if (m.type != CONVGPU_MSG_HELLO && k.container < 0) {
    send_reply(k, CONVGPU_ST_PROTOCOL, m.type);
    return;
  }
  const int c = k.container;
  // a process that said EXIT (or whose container finished) owns no memory any
  // more: an allocation or free from it would charge a finished container
  // whose memory has gone back to the pool, so it is refused
  if ((m.type == CONVGPU_MSG_ALLOC || m.type == CONVGPU_MSG_ALLOC_DONE ||
       m.type == CONVGPU_MSG_ALLOC_FAIL || m.type == CONVGPU_MSG_FREE ||
       m.type == CONVGPU_MSG_FREE_BYTES) &&
      (k.exited || g_s->get((uint32_t)c).done)) {
    send_reply(k, CONVGPU_ST_PROTOCOL, m.type);
    return;
  }
  switch (m.type) {
    case CONVGPU_MSG_HELLO: {
      if (k.container >= 0) { send_reply(k, CONVGPU_ST_PROTOCOL, m.type); return; }
      auto it = g_key2c.find(m.b);
      int id;
      if (it == g_key2c.end() || g_s->get(it->second).done) {
        id = (int)g_s->arrive(m.a);  // ARRIVE
        g_key2c[m.b] = id;
        g_ci.emplace_back();
      } else {
        id = it->second;
      }
      k.container = id;
      k.pid = m.pid;
      ++g_ci[id].live_procs;
      deliver_resumed();
      send_reply(k, CONVGPU_ST_OK, m.type, (uint64_t)id);
      return;
    }
    case CONVGPU_MSG_ALLOC: {
      k.waiting = true;
      k.wait_bytes = m.a;
      g_ci[c].queue.push_back(idx);
      const bool was_head = g_ci[c].queue.size() == 1;
      if (was_head) pump(c);
      deliver_resumed();
      return;  // replied by pump / deliver_resumed, or withheld
    }
    case CONVGPU_MSG_ALLOC_DONE:
      g_s->get(c).addr[m.a] = m.b;
      send_reply(k, CONVGPU_ST_OK, m.type);
      return;
    case CONVGPU_MSG_ALLOC_FAIL:
      g_s->alloc_failed((uint32_t)c, m.a);
      send_reply(k, CONVGPU_ST_OK, m.type);
      return;
    case CONVGPU_MSG_FREE: {
      auto& mp = g_s->get(c).addr;
      auto it = mp.find(m.a);
      if (it == mp.end()) { send_reply(k, CONVGPU_ST_INVALID, m.type); return; }
      const bool ok = g_s->free_bytes((uint32_t)c, it->second);
      mp.erase(it);
      send_reply(k, ok ? CONVGPU_ST_OK : CONVGPU_ST_INVALID, m.type);
      return;
    }
    case CONVGPU_MSG_FREE_BYTES: {
      const bool ok = g_s->free_bytes((uint32_t)c, m.a);
      send_reply(k, ok ? CONVGPU_ST_OK : CONVGPU_ST_INVALID, m.type);
      return;
    }
    case CONVGPU_MSG_MEMINFO: {  // answered from the ledger
      const auto& ct = g_s->get(c);
      send_reply(k, CONVGPU_ST_OK, m.type, ct.L - ct.used, ct.L);
      return;
    }
    case CONVGPU_MSG_EXIT:
      process_exit(k);
      send_reply(k, CONVGPU_ST_OK, m.type);
      return;
    case CONVGPU_MSG_INFO: {  // own container (a = ~0)
      const auto& ct = g_s->get((uint32_t)c);
      send_reply(k, CONVGPU_ST_OK, m.type, ct.a, ct.used,
                 ct.admit_rank == ~0u ? ~0ull : (uint64_t)ct.admit_rank);
      return;
    }
    default:
      send_reply(k, CONVGPU_ST_PROTOCOL, m.type);
  }
}

uint64_t parse_u64(const char* s) { return strtoull(s, nullptr, 0); }

int usage() {
  fprintf(stderr,
          "usage: convgpud --socket PATH (--capacity-mib M | --capacity BYTES) [--policy "
          "fifo|best_fit|recent_fit|random_fit] [--overhead-mib 66 | --overhead BYTES] "
          "[--seed S] [--tid T]\n");
  return 2;
}

}  // namespace

int main(int argc, char** argv) {
  std::string path;
  uint64_t cap = 0, ovh = 66ull << 20, seed = 0, tid = 0;
  convgpud::Policy pol = convgpud::FIFO;
  for (int i = 1; i < argc; ++i) {
    const std::string a = argv[i];
    const char* v = i + 1 < argc ? argv[i + 1] : nullptr;
    if (!v) return usage();
    if (a == "--socket") path = v;
    else if (a == "--capacity") cap = parse_u64(v);
    else if (a == "--capacity-mib") cap = parse_u64(v) << 20;
    else if (a == "--overhead") ovh = parse_u64(v);
    else if (a == "--overhead-mib") ovh = parse_u64(v) << 20;
    else if (a == "--seed") seed = parse_u64(v);
    else if (a == "--tid") tid = parse_u64(v);
    else if (a == "--policy") {
      const std::string p = v;
      if (p == "fifo") pol = convgpud::FIFO;
      else if (p == "best_fit") pol = convgpud::BEST_FIT;
      else if (p == "recent_fit") pol = convgpud::RECENT_FIT;
      else if (p == "random_fit") pol = convgpud::RANDOM_FIT;
      else return usage();
    } else {
      return usage();
    }
    ++i;
  }
  if (path.empty() || cap == 0) return usage();
  signal(SIGPIPE, SIG_IGN);
  Scheduler s(cap, pol, ovh, tid, seed);
  g_s = &s;

  const int lfd = socket(AF_UNIX, SOCK_STREAM, 0);
  sockaddr_un addr{};
  addr.sun_family = AF_UNIX;
  if (path.size() >= sizeof addr.sun_path) return usage();
  strcpy(addr.sun_path, path.c_str());
  unlink(path.c_str());
  if (lfd < 0 || bind(lfd, (sockaddr*)&addr, sizeof addr) < 0 || listen(lfd, 256) < 0) {
    perror("convgpud: socket");
    return 1;
  }
  fprintf(stdout, "convgpud ready %s\n", path.c_str());
  fflush(stdout);

  std::vector<pollfd> pfds;
  for (;;) {
    pfds.clear();
    pfds.push_back({lfd, POLLIN, 0});
    std::vector<int> idx;
    for (int i = 0; i < (int)g_conns.size(); ++i)
      if (g_conns[i].fd >= 0) { pfds.push_back({g_conns[i].fd, POLLIN, 0}); idx.push_back(i); }
    if (poll(pfds.data(), pfds.size(), -1) < 0) {
      if (errno == EINTR) continue;
      perror("convgpud: poll");
      return 1;
    }
    if (pfds[0].revents & POLLIN) {
      const int fd = accept(lfd, nullptr, nullptr);
      if (fd >= 0) { Conn k; k.fd = fd; g_conns.push_back(k); }
    }
    for (size_t j = 1; j < pfds.size(); ++j) {
      if (!(pfds[j].revents & (POLLIN | POLLHUP | POLLERR))) continue;
      const int i = idx[j - 1];
      char buf[4096];
      const ssize_t r = recv(g_conns[i].fd, buf, sizeof buf, 0);
      if (r <= 0) {  // disconnected: the process is gone
        close(g_conns[i].fd);
        g_conns[i].fd = -1;
        if (g_conns[i].container >= 0) {
          const int c = g_conns[i].container;
          ContainerInfo& ci = g_ci[c];
          const bool head = !ci.queue.empty() && ci.queue.front() == i;
          for (auto it = ci.queue.begin(); it != ci.queue.end(); ++it)
            if (*it == i) { ci.queue.erase(it); break; }
          // its ALLOC paused the container: withdraw that request, so the
          // next queued one goes through its own admission check (alloc())
          // instead of inheriting the dead request's grant on resume
          if (head) g_s->cancel_pause((uint32_t)c);
          process_exit(g_conns[i]);
          if (!g_s->get((uint32_t)c).done) pump(c);
          deliver_resumed();
        }
        continue;
      }
      g_conns[i].in.append(buf, (size_t)r);
      while (g_conns[i].in.size() >= sizeof(convgpu_msg_t)) {
        convgpu_msg_t m;
        memcpy(&m, g_conns[i].in.data(), sizeof m);
        g_conns[i].in.erase(0, sizeof m);
        handle(i, m);
      }
    }
  }
}
