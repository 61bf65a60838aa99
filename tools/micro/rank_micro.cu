// Microbenchmark: cost of warp peer-mask computation on sm_100a.
// (a) __match_any_sync  (b) ballot loop with compile-time LOGM  (c) ballot loop, runtime logm
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

template <int MODE, int LOGM>
__global__ void k(const uint32_t* __restrict__ in, uint32_t* out, int iters, uint32_t logm_rt) {
  uint32_t x = in[blockIdx.x * blockDim.x + threadIdx.x];
  uint32_t acc = 0;
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t lt = (1u << lane) - 1;
  for (int it = 0; it < iters; ++it) {
    x = x * 1664525u + 1013904223u;
    uint32_t id = x >> (32 - LOGM);
    uint32_t peers;
    if (MODE == 0) {
      peers = __match_any_sync(0xFFFFFFFFu, id);
    } else if (MODE == 1) {
      peers = 0xFFFFFFFFu;
#pragma unroll
      for (int b = 0; b < LOGM; ++b) {
        uint32_t bit = (id >> b) & 1u;
        uint32_t v = __ballot_sync(0xFFFFFFFFu, bit);
        peers &= bit ? v : ~v;
      }
    } else {
      peers = 0xFFFFFFFFu;
#pragma unroll
      for (int b = 0; b < 8; ++b) {
        if ((uint32_t)b < logm_rt) {
          uint32_t bit = (id >> b) & 1u;
          uint32_t v = __ballot_sync(0xFFFFFFFFu, bit);
          peers &= bit ? v : ~v;
        }
      }
    }
    acc += __popc(peers & lt);
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}

template <int MODE, int LOGM>
void run(const char* name, uint32_t* din, uint32_t* dout, int blocks) {
  int iters = 4096;
  k<MODE, LOGM><<<blocks, 256>>>(din, dout, iters, LOGM);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  cudaEventRecord(a);
  k<MODE, LOGM><<<blocks, 256>>>(din, dout, iters, LOGM);
  cudaEventRecord(b); cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b);
  double keys = (double)blocks * 256 * iters;
  printf("%-28s LOGM=%d  %8.1f G keys/s  (%.3f ns per key per SM)\n", name, LOGM, keys / ms / 1e6,
         ms * 1e6 / keys * 148);
}

int main() {
  int blocks = 148 * 8;
  uint32_t *din, *dout;
  cudaMalloc(&din, blocks * 256 * 4); cudaMalloc(&dout, blocks * 256 * 4);
  cudaMemset(din, 1, blocks * 256 * 4);
  run<0, 3>("match_any", din, dout, blocks);
  run<0, 5>("match_any", din, dout, blocks);
  run<0, 8>("match_any", din, dout, blocks);
  run<1, 1>("ballot constexpr", din, dout, blocks);
  run<1, 3>("ballot constexpr", din, dout, blocks);
  run<1, 5>("ballot constexpr", din, dout, blocks);
  run<1, 8>("ballot constexpr", din, dout, blocks);
  run<2, 3>("ballot runtime", din, dout, blocks);
  run<2, 5>("ballot runtime", din, dout, blocks);
  run<2, 8>("ballot runtime", din, dout, blocks);
  printf("%s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
