// k3_ids.cu -- instantiates the post-scan kernels for the kernel-level bucket kind IDS:
// K3 v2 (m <= 32, ms_k3_v2.cuh) and the warp-ballot K3 (32 < m <= 256, ms_k3_warp.cuh).
// One translation unit per kind so that nvcc compiles them in parallel.
#include "ms_k3_v2.cuh"
#include "ms_k3_warp.cuh"

namespace ms {
cudaError_t k3v_launch_ids(const K3pArgs &a) { return k3v_launch<IDS>(a); }
cudaError_t k3w_launch_ids(const K3pArgs &a) { return k3w_launch<IDS>(a); }
}  // namespace ms
