// ms_k3p_args.h -- host-side entry points of the persistent K3 (m <= 32), one TU per bucket kind.
#pragma once
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <utility>

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
  int ranged = 0;               // 1: CTA-range mode (G = GB[C][m], ms_ranged.cuh); m <= 32 only
  int pdl = 0;                  // 1: programmatic dependent launch after K2 (ms_device.cuh pdl_wait)
  uint32_t *grid_out = nullptr;  // non-null: only compute the grid C (no launch)
};

// Launch with cudaLaunchAttributeProgrammaticStreamSerialization when `pdl`:
// the kernel may begin while its stream predecessor finishes, and must call
// pdl_wait() before touching the predecessor's output.
template <typename... KArgs, typename... Args>
inline cudaError_t launch_ex(bool pdl, void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s,
                             Args &&...args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = pdl ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...);
}

constexpr uint32_t kMaxRanges = 1024;  // upper bound on the CTA-range count C (workspace sizing)

cudaError_t k3p_launch_lowbits(const K3pArgs &a);
cudaError_t k3p_launch_shiftc(const K3pArgs &a);
cudaError_t k3p_launch_shift(const K3pArgs &a);
cudaError_t k3p_launch_delta(const K3pArgs &a);
cudaError_t k3p_launch_splitters(const K3pArgs &a);
cudaError_t k3p_launch_ids(const K3pArgs &a);
// m <= 32, second generation (ms_k3_v2.cuh): TMA-tensor staging, keys in registers
cudaError_t k3v_launch_lowbits(const K3pArgs &a);
cudaError_t k3v_launch_shiftc(const K3pArgs &a);
cudaError_t k3v_launch_shift(const K3pArgs &a);
cudaError_t k3v_launch_delta(const K3pArgs &a);
cudaError_t k3v_launch_splitters(const K3pArgs &a);
// m > 32: warp-ballot K3 (ms_k3_warp.cuh); kpt carries the rounds per warp R (8 or 16)
cudaError_t k3w_launch_lowbits(const K3pArgs &a);
cudaError_t k3w_launch_shiftc(const K3pArgs &a);
cudaError_t k3w_launch_shift(const K3pArgs &a);
cudaError_t k3w_launch_delta(const K3pArgs &a);
cudaError_t k3w_launch_splitters(const K3pArgs &a);
cudaError_t k3w_launch_ids(const K3pArgs &a);

}  // namespace ms
