// shim.cpp — NEXT-4: ConVGPU's wrapper module (§III-C P:100-110,
// Table II) as an LD_PRELOAD library for B200 hosts.
//
// It overrides the CUDA runtime and driver memory APIs; each allocation is
// first sent to the scheduler (convgpud, include/convgpu_ctl.h) with the size
// the wrapper computes (P:104, P:106-108 — the same rules as
// convgpu_wrap_ops / DESIGN.md R13', in bytes here), and only a granted
// request reaches the real API; the call blocks while the scheduler withholds
// its reply (the container is paused), and a rejection returns
// cudaErrorMemoryAllocation / CUDA_ERROR_OUT_OF_MEMORY.  After the real
// allocation the address and size are reported for later frees (P:129,
// P:133); cudaFree frees through the real API and then reports the address
// (P:110); cudaMemGetInfo is answered by the scheduler from its ledger
// without the original API; __cudaUnregisterFatBinary tells the
// scheduler the process is ending.  Texture allocations such as
// cudaMallocArray are not captured.
//
// The real entry points are resolved with dlsym(RTLD_NEXT); nothing here
// links against CUDA.  Without CONVGPU_SOCKET every call passes through.
#include <dlfcn.h>
#include <pthread.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <sys/socket.h>
#include <sys/un.h>
#include <unistd.h>


#include <cuda.h>
#include <cuda_runtime_api.h>

#include "convgpu_ctl.h"

namespace {

pthread_mutex_t g_mu = PTHREAD_MUTEX_INITIALIZER;  // one request in flight per process
// Scoped lock without the C++ runtime (the shim is preloaded into arbitrary
// processes, so it links no libstdc++ and exports only the CUDA entry points).
// A call made while this thread is already inside the shim (e.g. a runtime
// call that reaches a driver entry point we also wrap) passes straight
// through: it is part of the outer request, and g_mu is not recursive.
//
// Known limitation: g_mu is held across the blocking request, so while one
// thread's cudaMalloc is paused (reply withheld) every other thread of
// the process that calls into the shim (cudaFree, cudaMemGetInfo, the
// teardown's __cudaUnregisterFatBinary) waits until the scheduler resumes it.
// Replies carry no request id, so one connection cannot have two requests in
// flight; a process exiting while a worker thread is paused therefore blocks
// in teardown until resumed (or until the daemon drops the connection).
__thread int t_depth = 0;
struct Lock {
  const bool outer;
  Lock() : outer(t_depth++ == 0) { if (outer) pthread_mutex_lock(&g_mu); }
  ~Lock() { if (outer) pthread_mutex_unlock(&g_mu); --t_depth; }
};
int g_fd = -1;       // connection to convgpud
int g_state = 0;     // 0 = not tried, 1 = connected, -1 = disabled
uint64_t g_pitch = 0;  // pitch granule, read once

template <typename F>
F real(const char* name) {
  return reinterpret_cast<F>(dlsym(RTLD_NEXT, name));
}

bool io(void* p, size_t n, bool wr) {
  char* c = static_cast<char*>(p);
  while (n > 0) {
    const ssize_t r = wr ? send(g_fd, c, n, MSG_NOSIGNAL) : recv(g_fd, c, n, 0);
    if (r <= 0) return false;
    c += r;
    n -= (size_t)r;
  }
  return true;
}

// One request / reply with the scheduler (g_mu held).  false: no scheduler.
bool rpc(uint32_t type, uint64_t a, uint64_t b, convgpu_reply_t* rep) {
  if (g_state == 0) {
    g_state = -1;
    const char* path = getenv("CONVGPU_SOCKET");
    if (!path || strlen(path) >= sizeof(sockaddr_un::sun_path)) return false;
    const int fd = socket(AF_UNIX, SOCK_STREAM, 0);
    sockaddr_un ad{};
    ad.sun_family = AF_UNIX;
    strcpy(ad.sun_path, path);
    if (fd < 0 || connect(fd, reinterpret_cast<sockaddr*>(&ad), sizeof ad) != 0) {
      if (fd >= 0) close(fd);
      fprintf(stderr, "convgpu shim: cannot reach %s, passing calls through\n", path);
      return false;
    }
    g_fd = fd;
    const char* lim = getenv("CONVGPU_LIMIT_MIB");
    const char* key = getenv("CONVGPU_CONTAINER");
    const uint64_t limit = (lim ? strtoull(lim, nullptr, 10) : 1024ull) << 20;  // 1 GiB default
    const uint64_t k = key ? strtoull(key, nullptr, 10) : (uint64_t)getpid();
    convgpu_msg_t m{CONVGPU_MSG_HELLO, (uint32_t)getpid(), limit, k, CONVGPU_CTL_VERSION};
    convgpu_reply_t r;
    if (!io(&m, sizeof m, true) || !io(&r, sizeof r, false) || r.status != CONVGPU_ST_OK) {
      close(fd);
      g_fd = -1;
      return false;
    }
    g_state = 1;
  }
  if (g_state != 1) return false;
  convgpu_msg_t m{type, (uint32_t)getpid(), a, b, 0};
  if (!io(&m, sizeof m, true) || !io(rep, sizeof *rep, false)) {
    close(g_fd);
    g_fd = -1;
    g_state = -1;
    return false;
  }
  return true;
}

uint64_t round_up(uint64_t x, uint64_t g) { return g ? (x + g - 1) / g * g : x; }

// The wrapper's pitch granule: the device property it reads on the first
// pitched allocation; on B200 the runtime pitches rows to 512 B.
uint64_t pitch_granule() {
  if (g_pitch == 0) {
    int dev = 0;
    cudaDeviceProp prop;
    auto get_dev = real<cudaError_t (*)(int*)>("cudaGetDevice");
    auto get_prop = real<cudaError_t (*)(cudaDeviceProp*, int)>("cudaGetDeviceProperties");
    if (get_dev && get_prop && get_dev(&dev) == cudaSuccess && get_prop(&prop, dev) == cudaSuccess)
      g_pitch = prop.textureAlignment;
    if (g_pitch == 0) g_pitch = 512;
  }
  return g_pitch;
}

enum class Ask { Pass, Grant, Reject };

// Ask the scheduler for `bytes`; blocks while the container is paused.
Ask ask(uint64_t bytes) {
  convgpu_reply_t r;
  if (!rpc(CONVGPU_MSG_ALLOC, bytes, 0, &r)) return Ask::Pass;
  return r.status == CONVGPU_ST_OK ? Ask::Grant : Ask::Reject;
}

void done(bool ok, uint64_t addr, uint64_t bytes) {
  convgpu_reply_t r;
  if (ok)
    rpc(CONVGPU_MSG_ALLOC_DONE, addr, bytes, &r);
  else
    rpc(CONVGPU_MSG_ALLOC_FAIL, bytes, 0, &r);
}

void freed(uint64_t addr) {
  convgpu_reply_t r;
  if (addr) rpc(CONVGPU_MSG_FREE, addr, 0, &r);
}

}  // namespace

#define EXPORT __attribute__((visibility("default")))

extern "C" {

EXPORT cudaError_t cudaMalloc(void** p, size_t size) {
  static auto fn = real<cudaError_t (*)(void**, size_t)>("cudaMalloc");
  Lock lk;
  if (!lk.outer) return fn(p, size);
  const Ask a = ask(size);
  if (a == Ask::Reject) return cudaErrorMemoryAllocation;
  const cudaError_t e = fn(p, size);
  if (a == Ask::Grant) done(e == cudaSuccess, e == cudaSuccess ? (uint64_t)*p : 0, size);
  return e;
}

EXPORT cudaError_t cudaMallocManaged(void** p, size_t size, unsigned int flags) {
  static auto fn = real<cudaError_t (*)(void**, size_t, unsigned int)>("cudaMallocManaged");
  Lock lk;
  if (!lk.outer) return fn(p, size, flags);
  const uint64_t adj = round_up(size, 128ull << 20);  // multiple of 128 MiB
  const Ask a = ask(adj);
  if (a == Ask::Reject) return cudaErrorMemoryAllocation;
  const cudaError_t e = fn(p, size, flags);
  if (a == Ask::Grant) done(e == cudaSuccess, e == cudaSuccess ? (uint64_t)*p : 0, adj);
  return e;
}

EXPORT cudaError_t cudaMallocPitch(void** p, size_t* pitch, size_t width, size_t height) {
  static auto fn = real<cudaError_t (*)(void**, size_t*, size_t, size_t)>("cudaMallocPitch");
  Lock lk;
  if (!lk.outer) return fn(p, pitch, width, height);
  const uint64_t adj = round_up(width, pitch_granule()) * height;
  const Ask a = ask(adj);
  if (a == Ask::Reject) return cudaErrorMemoryAllocation;
  const cudaError_t e = fn(p, pitch, width, height);
  if (a == Ask::Grant) done(e == cudaSuccess, e == cudaSuccess ? (uint64_t)*p : 0, adj);
  return e;
}

EXPORT cudaError_t cudaMalloc3D(cudaPitchedPtr* pp, cudaExtent ext) {
  static auto fn = real<cudaError_t (*)(cudaPitchedPtr*, cudaExtent)>("cudaMalloc3D");
  Lock lk;
  if (!lk.outer) return fn(pp, ext);
  const uint64_t adj = round_up(ext.width, pitch_granule()) * ext.height * ext.depth;  // Table II
  const Ask a = ask(adj);
  if (a == Ask::Reject) return cudaErrorMemoryAllocation;
  const cudaError_t e = fn(pp, ext);
  if (a == Ask::Grant) done(e == cudaSuccess, e == cudaSuccess ? (uint64_t)pp->ptr : 0, adj);
  return e;
}

EXPORT cudaError_t cudaFree(void* p) {
  static auto fn = real<cudaError_t (*)(void*)>("cudaFree");
  Lock lk;
  if (!lk.outer) return fn(p);
  const cudaError_t e = fn(p);  // the original API first, then the address
  if (e == cudaSuccess && g_state == 1) freed((uint64_t)p);
  return e;
}

EXPORT cudaError_t cudaMemGetInfo(size_t* free_b, size_t* total_b) {
  static auto fn = real<cudaError_t (*)(size_t*, size_t*)>("cudaMemGetInfo");
  Lock lk;
  if (!lk.outer) return fn(free_b, total_b);
  convgpu_reply_t r;
  if (rpc(CONVGPU_MSG_MEMINFO, 0, 0, &r)) {  // the container's view
    if (free_b) *free_b = (size_t)r.a;
    if (total_b) *total_b = (size_t)r.b;
    return cudaSuccess;
  }
  return fn(free_b, total_b);
}

EXPORT CUresult cuMemAlloc_v2(CUdeviceptr* p, size_t size) {
  static auto fn = real<CUresult (*)(CUdeviceptr*, size_t)>("cuMemAlloc_v2");
  Lock lk;
  if (!lk.outer) return fn(p, size);
  const Ask a = ask(size);
  if (a == Ask::Reject) return CUDA_ERROR_OUT_OF_MEMORY;
  const CUresult e = fn(p, size);
  if (a == Ask::Grant) done(e == CUDA_SUCCESS, e == CUDA_SUCCESS ? (uint64_t)*p : 0, size);
  return e;
}

EXPORT CUresult cuMemFree_v2(CUdeviceptr p) {
  static auto fn = real<CUresult (*)(CUdeviceptr)>("cuMemFree_v2");
  Lock lk;
  if (!lk.outer) return fn(p);
  const CUresult e = fn(p);
  if (e == CUDA_SUCCESS && g_state == 1) freed((uint64_t)p);
  return e;
}

EXPORT void __cudaUnregisterFatBinary(void** handle) {
  static auto fn = real<void (*)(void**)>("__cudaUnregisterFatBinary");
  {
    Lock lk;
    convgpu_reply_t r;
    if (lk.outer && g_state == 1) {
      rpc(CONVGPU_MSG_EXIT, 0, 0, &r);  // the process is ending
      // the container's memory is being released: later calls (teardown
      // allocations, another fat binary's unregistration) pass straight
      // through instead of charging a finished container
      g_state = -1;
      close(g_fd);
      g_fd = -1;
    }
  }
  if (fn) fn(handle);
}

}  // extern "C"
