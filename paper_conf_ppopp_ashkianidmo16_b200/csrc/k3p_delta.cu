// k3p_delta.cu -- instantiates the K3 variants for whatBucket kind DELTA:
// persistent blocked-rank K3 (m <= 32, ms_k3_blocked.cuh) and warp-ballot K3 (m > 32, ms_k3_warp.cuh).
#include "ms_k3_blocked.cuh"
#include "ms_k3_warp.cuh"
#include "ms_k3_v2.cuh"
#include "ms_k3_lsd.cuh"

namespace ms {
cudaError_t k3p_launch_delta(const K3pArgs &a) { return k3p_launch<DELTA>(a); }
cudaError_t k3w_launch_delta(const K3pArgs &a) { return k3w_launch<DELTA>(a); }
cudaError_t k3v_launch_delta(const K3pArgs &a) { return k3v_launch<DELTA>(a); }
cudaError_t k3h_launch_delta(const K3pArgs &a) { return k3h_launch<DELTA>(a); }
}  // namespace ms
