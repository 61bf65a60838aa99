// k3_shiftc_lo.cu -- instantiates the post-scan kernels for the kernel-level bucket kind SHIFTC_LO
// (the low digit of a clamped id: pass A of the two-pass multisplit for m > 256):
// K3 v2 (digit <= 32 buckets, ms_k3_v2.cuh) and the warp-ballot K3 (<= 256, ms_k3_warp.cuh).
#include "ms_k3_v2.cuh"
#include "ms_k3_warp.cuh"

namespace ms {
cudaError_t k3v_launch_shiftc_lo(const K3pArgs &a) { return k3v_launch<SHIFTC_LO>(a); }
cudaError_t k3w_launch_shiftc_lo(const K3pArgs &a) { return k3w_launch<SHIFTC_LO>(a); }
}  // namespace ms
