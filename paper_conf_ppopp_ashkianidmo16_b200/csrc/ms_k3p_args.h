// ms_k3p_args.h -- host-side entry points of the persistent K3 (m <= 32), one TU per bucket kind.
#pragma once
#include <cuda_runtime.h>

#include <cstdint>

#include "ms_device.cuh"

namespace ms {

struct K3pArgs {
  const uint32_t *keys, *vals;
  const void *ids;
  const uint32_t *G;
  uint32_t *keys_out, *vals_out;
  uint32_t n, L, m, id_bytes, kpt;
  uint32_t nt;              // K3p threads per CTA (128 or 256); tile = nt * 16 keys
  const BucketParams *bp;  // host copy, passed by value to the kernel
  int sms;
  cudaStream_t stream;
};

cudaError_t k3p_launch_lowbits(const K3pArgs &a);
cudaError_t k3p_launch_shiftc(const K3pArgs &a);
cudaError_t k3p_launch_shift(const K3pArgs &a);
cudaError_t k3p_launch_delta(const K3pArgs &a);
cudaError_t k3p_launch_splitters(const K3pArgs &a);
cudaError_t k3p_launch_ids(const K3pArgs &a);
// m > 32: warp-ballot K3 (ms_k3_warp.cuh); kpt carries the rounds per warp R (8 or 16)
cudaError_t k3w_launch_lowbits(const K3pArgs &a);
cudaError_t k3w_launch_shiftc(const K3pArgs &a);
cudaError_t k3w_launch_shift(const K3pArgs &a);
cudaError_t k3w_launch_delta(const K3pArgs &a);
cudaError_t k3w_launch_splitters(const K3pArgs &a);
cudaError_t k3w_launch_ids(const K3pArgs &a);

}  // namespace ms
