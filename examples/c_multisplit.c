/* examples/c_multisplit.c -- the C ABI (include/ms.h) used from plain C, no Python, no torch:
 * a stable key-value multisplit of n keys into m delta-range buckets on the GPU, checked with the
 * invariants that define it (Eq. (1)): the output is a permutation of the
 * input (values = input positions), bucket ids ascend, input order is kept inside a bucket, and the
 * offsets are the bucket boundaries.
 *
 * build:  gcc -O2 -I include -I /usr/local/cuda/include examples/c_multisplit.c \
 *             -L paper_conf_ppopp_ashkianidmo16_b200 -lms -L /usr/local/cuda/lib64 -lcudart \
 *             -Wl,-rpath,$PWD/paper_conf_ppopp_ashkianidmo16_b200 -o c_multisplit
 * run:    ./c_multisplit [n] [m]                                  (prints "C ABI OK" and exits 0) */
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

#include "ms.h"

#define CK(x)                                                                      \
  do {                                                                             \
    ms_status s_ = (x);                                                            \
    if (s_ != MS_OK) {                                                             \
      fprintf(stderr, "%s failed: %s (%d)\n", #x, ms_status_string(s_), (int)s_); \
      return 1;                                                                    \
    }                                                                              \
  } while (0)
#define CC(x)                                                                 \
  do {                                                                        \
    cudaError_t e_ = (x);                                                     \
    if (e_ != cudaSuccess) {                                                  \
      fprintf(stderr, "%s failed: %s\n", #x, cudaGetErrorString(e_));         \
      return 1;                                                               \
    }                                                                         \
  } while (0)

static uint32_t mix(uint64_t z) { /* splitmix64 finaliser, high word */
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return (uint32_t)((z ^ (z >> 31)) >> 32);
}

int main(int argc, char **argv) {
  const uint64_t n = argc > 1 ? strtoull(argv[1], 0, 10) : (1u << 24) + 77;
  const uint32_t m = argc > 2 ? (uint32_t)atoi(argv[2]) : 16;
  const uint32_t delta = (uint32_t)(0xFFFFFFFFull / m) + 1; /* buckets divide the 32-bit domain */
  uint32_t *k = malloc(n * 4), *v = malloc(n * 4), *ko = malloc(n * 4), *vo = malloc(n * 4);
  uint32_t *off = malloc((m + 1) * 4);
  for (uint64_t i = 0; i < n; ++i) {
    k[i] = mix(0x4D53C0DEull ^ ((i + 1) * 0x9E3779B97F4A7C15ull));
    v[i] = (uint32_t)i;
  }
  ms_bucket_spec spec = {MS_DELTA, m, 0, delta, NULL, 0};
  ms_plan_t plan;
  CK(ms_plan_create(&plan, &spec, n, 1, 0, 0));
  size_t wsb = 0;
  CK(ms_plan_workspace_size(plan, n, &wsb));
  uint32_t *dk, *dv, *dko, *dvo, *doff;
  void *ws;
  CC(cudaMalloc((void **)&dk, n * 4));
  CC(cudaMalloc((void **)&dv, n * 4));
  CC(cudaMalloc((void **)&dko, n * 4));
  CC(cudaMalloc((void **)&dvo, n * 4));
  CC(cudaMalloc((void **)&doff, (m + 1) * 4));
  CC(cudaMalloc(&ws, wsb));
  cudaStream_t s;
  CC(cudaStreamCreate(&s));
  CC(cudaMemcpyAsync(dk, k, n * 4, cudaMemcpyHostToDevice, s));
  CC(cudaMemcpyAsync(dv, v, n * 4, cudaMemcpyHostToDevice, s));
  CK(ms_run(plan, dk, dv, NULL, dko, dvo, n, doff, ws, wsb, s));
  CC(cudaMemcpyAsync(ko, dko, n * 4, cudaMemcpyDeviceToHost, s));
  CC(cudaMemcpyAsync(vo, dvo, n * 4, cudaMemcpyDeviceToHost, s));
  CC(cudaMemcpyAsync(off, doff, (m + 1) * 4, cudaMemcpyDeviceToHost, s));
  CC(cudaStreamSynchronize(s));
  /* invariants: permutation (values are positions), keys travel with values, ascending ids,
   * stable inside a bucket, offsets are the bucket boundaries */
  char *seen = calloc(n, 1);
  uint64_t bad = 0;
  for (uint64_t p = 0; p < n; ++p) {
    const uint32_t i = vo[p];
    if (i >= n || seen[i] || ko[p] != k[i]) { ++bad; continue; }
    seen[i] = 1;
    const uint32_t id = ko[p] / delta < m ? ko[p] / delta : m - 1;
    if (p < off[id] || p >= off[id + 1]) ++bad;
    if (p > 0) {
      const uint32_t pid = ko[p - 1] / delta < m ? ko[p - 1] / delta : m - 1;
      if (pid > id || (pid == id && vo[p - 1] >= i)) ++bad;
    }
  }
  if (off[0] != 0 || off[m] != n) ++bad;
  printf("n=%llu m=%u launches=%d violations=%llu\n", (unsigned long long)n, m, ms_plan_last_launches(plan),
         (unsigned long long)bad);
  ms_plan_destroy(plan);
  if (bad) return 1;
  printf("C ABI OK\n");
  return 0;
}
