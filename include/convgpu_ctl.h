/*
 * convgpu_ctl.h — NEXT-4: the live control plane.
 *
 * PAPER.md §III-C/D: a wrapper module preloaded into every container
 * (LD_PRELOAD) intercepts the CUDA memory APIs of Table II
 * and asks a host GPU-memory scheduler, over a UNIX socket per
 * container, before every allocation; the scheduler
 * accepts, rejects, or pauses the container by withholding its reply
 * (P:139), tracks addresses and sizes in a hash, charges 66 MiB of
 * context at a process's first allocation, and on container exit
 * reassigns memory to paused containers by FIFO, Best-Fit, Recent-Fit or
 * Random-Fit.
 *
 * Here: `convgpud` (paper_conf_cluster_kangjkkk17_b200/csrc/ctl/convgpud.cpp) is
 * the scheduler, a single-threaded poll loop (every message is one
 * serialised scheduler step) running the same rules as the replay
 * (R1-R21) in byte units; `libconvgpu_shim.so`
 * (csrc/ctl/shim.cpp) is the wrapper module.  This header is their wire
 * protocol: fixed 32-byte messages and 32-byte replies, host byte order, on
 * a SOCK_STREAM UNIX socket.
 *
 * Connection = one process of one container.  Its first message is HELLO
 * (SYNC, STATS and INFO of a given container need none: control connections);
 * containers are created (ARRIVE) in the order of their first HELLO, and a
 * container FINISHes when its last process has sent EXIT or disconnected.
 * Every message gets exactly one reply, sent when the step completes; the
 * reply to an ALLOC that pauses the container is sent when a later step
 * resumes it (the "withheld reply").
 */
#ifndef CONVGPU_CTL_H
#define CONVGPU_CTL_H
#include <stdint.h>

#define CONVGPU_CTL_VERSION 1

typedef enum {
  CONVGPU_MSG_HELLO = 1,      /* a = limit bytes, b = container key, c = version */
  CONVGPU_MSG_ALLOC = 2,      /* a = bytes (already adjusted by the wrapper):
                                 status GRANT / REJECT, withheld while paused */
  CONVGPU_MSG_ALLOC_DONE = 3, /* a = device address, b = bytes: record for FREE */
  CONVGPU_MSG_ALLOC_FAIL = 4, /* a = bytes: the real allocation failed after a grant */
  CONVGPU_MSG_FREE = 5,       /* a = device address: release its recorded size */
  CONVGPU_MSG_FREE_BYTES = 6, /* a = bytes: release a size directly (trace drivers) */
  CONVGPU_MSG_MEMINFO = 7,    /* reply a = limit - used, b = limit (cudaMemGetInfo) */
  CONVGPU_MSG_EXIT = 8,       /* this process ends (__cudaUnregisterFatBinary) */
  CONVGPU_MSG_INFO = 9,       /* a = container id (~0: the caller's): reply a = assigned,
                                 b = used, c = admit rank (~0 if not admitted) */
  CONVGPU_MSG_STATS = 10,     /* reply a = unassigned pool, b = selections, c = rejections */
  CONVGPU_MSG_SYNC = 11       /* reply a = messages handled before this one (all connections):
                                 a driver's barrier, since a withheld reply is silent */
} convgpu_msg_type_t;

typedef enum {
  CONVGPU_ST_OK = 0,          /* granted / done */
  CONVGPU_ST_REJECT = 1,      /* over the container's limit */
  CONVGPU_ST_INVALID = 2,     /* FREE of memory the container does not hold, unknown address */
  CONVGPU_ST_PROTOCOL = 3     /* malformed message or message before HELLO */
} convgpu_status_t;

typedef struct {
  uint32_t type; /* convgpu_msg_type_t */
  uint32_t pid;
  uint64_t a, b, c;
} convgpu_msg_t; /* 32 bytes */

typedef struct {
  int32_t status; /* convgpu_status_t */
  uint32_t type;  /* echo of the request type */
  uint64_t a, b, c;
} convgpu_reply_t; /* 32 bytes */

/* Environment read by the wrapper module (libconvgpu_shim.so):
 *   CONVGPU_SOCKET      path of the scheduler's socket (required; without it
 *                       the shim passes every call through untouched)
 *   CONVGPU_CONTAINER   container key (decimal; processes with the same key
 *                       share one container), default: the process id
 *   CONVGPU_LIMIT_MIB   the container's declared limit in MiB (default 1024,
 *                       P:98) */

#endif /* CONVGPU_CTL_H */
