// shim_probe.cu — a CUDA program for the NEXT-4 wrapper-module tests
// (tests/test_gpu_shim.py), built with -cudart=shared so LD_PRELOAD can
// interpose the runtime (a statically linked runtime cannot be, the paper's
// caveat about nvcc's default linking).  Modes:
//   api                 the Table II calls in sequence, one JSON line per step
//   hold MIB SECONDS    allocate MIB, report how long the call blocked, hold, free
//   latency N           mean microseconds per API call over N calls (Fig. 4)
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <time.h>
#include <unistd.h>

static double now_us() {
  timespec t;
  clock_gettime(CLOCK_MONOTONIC, &t);
  return t.tv_sec * 1e6 + t.tv_nsec / 1e3;
}

static int cmp_d(const void* a, const void* b) {
  const double x = *(const double*)a, y = *(const double*)b;
  return x < y ? -1 : (x > y);
}
static cudaPitchedPtr pp_dummy;

static void info(const char* step, int rc) {
  size_t f = 0, t = 0;
  cudaMemGetInfo(&f, &t);
  printf("{\"step\": \"%s\", \"rc\": %d, \"free\": %zu, \"total\": %zu}\n", step, rc, f, t);
  fflush(stdout);
}

int main(int argc, char** argv) {
  if (argc < 2) return 2;
  cudaFree(0);  // create the context outside the measured calls
  const size_t MiB = 1ull << 20;
  if (!strcmp(argv[1], "api")) {
    info("start", 0);
    void *a = 0, *big = 0, *p = 0, *m = 0;
    info("malloc_100", (int)cudaMalloc(&a, 100 * MiB));
    info("malloc_over", (int)cudaMalloc(&big, 1024 * MiB));
    size_t pitch = 0;
    const int rp = (int)cudaMallocPitch(&p, &pitch, 513, 2048);
    printf("{\"pitch\": %zu}\n", pitch);
    info("pitch_513x2048", rp);
    info("managed_1", (int)cudaMallocManaged(&m, 1 * MiB));
    cudaPitchedPtr pp;
    info("malloc3d_1000x7x3", (int)cudaMalloc3D(&pp, make_cudaExtent(1000, 7, 3)));
    info("free_3d", (int)cudaFree(pp.ptr));
    info("free_managed", (int)cudaFree(m));
    info("free_pitch", (int)cudaFree(p));
    info("free_100", (int)cudaFree(a));
    CUdeviceptr d = 0;
    info("cuMemAlloc_50", (int)cuMemAlloc(&d, 50 * MiB));
    info("cuMemFree_50", (int)cuMemFree(d));
    return 0;
  }
  if (!strcmp(argv[1], "hold") && argc >= 4) {
    void* a = 0;
    const double t0 = now_us();
    const int rc = (int)cudaMalloc(&a, (size_t)atoll(argv[2]) * MiB);
    const double t1 = now_us();
    printf("{\"rc\": %d, \"blocked_s\": %.4f}\n", rc, (t1 - t0) / 1e6);
    fflush(stdout);
    usleep((useconds_t)(atof(argv[3]) * 1e6));
    cudaFree(a);
    return 0;
  }
  if (!strcmp(argv[1], "latency") && argc >= 3) {
    // medians over N calls after 20 warm-up rounds (Fig. 4 reports means of
    // repeated calls; medians are robust to the runtime's occasional slow call)
    const int n = atoi(argv[2]);
    double* s[6];
    for (int k = 0; k < 6; ++k) s[k] = (double*)malloc(sizeof(double) * n);
    void* p;
    size_t pitch, f, t;
    double t0 = now_us();
    cudaMallocPitch(&p, &pitch, 1000, 1000);  // the first pitched call reads the granule
    const double t_pitch_first = now_us() - t0;
    cudaFree(p);
    for (int i = -20; i < n; ++i) {
      double d[6];
      t0 = now_us(); cudaMalloc(&p, MiB); d[0] = now_us() - t0;
      t0 = now_us(); cudaFree(p); d[1] = now_us() - t0;
      t0 = now_us(); cudaMallocPitch(&p, &pitch, 1000, 1000); d[2] = now_us() - t0;
      cudaFree(p);
      t0 = now_us(); cudaMallocManaged(&p, MiB); d[3] = now_us() - t0;
      cudaFree(p);
      t0 = now_us(); cudaMemGetInfo(&f, &t); d[4] = now_us() - t0;
      t0 = now_us(); cudaMalloc3D(&pp_dummy, make_cudaExtent(1000, 100, 10)); d[5] = now_us() - t0;
      cudaFree(pp_dummy.ptr);
      if (i >= 0) for (int k = 0; k < 6; ++k) s[k][i] = d[k];
    }
    double med[6];
    for (int k = 0; k < 6; ++k) {
      qsort(s[k], n, sizeof(double), cmp_d);
      med[k] = s[k][n / 2];
    }
    printf("{\"n\": %d, \"stat\": \"median\", \"cudaMalloc_us\": %.2f, \"cudaFree_us\": %.2f, "
           "\"cudaMallocPitch_us\": %.2f, \"cudaMallocPitch_first_us\": %.2f, "
           "\"cudaMallocManaged_us\": %.2f, \"cudaMemGetInfo_us\": %.2f, \"cudaMalloc3D_us\": %.2f}\n",
           n, med[0], med[1], med[2], t_pitch_first, med[3], med[4], med[5]);
    return 0;
  }
  return 2;
}
