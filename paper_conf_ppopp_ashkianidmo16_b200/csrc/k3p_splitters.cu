// k3p_splitters.cu -- instantiates the K3 variants for whatBucket kind SPLITTERS:
// persistent blocked-rank K3 (m <= 32, ms_k3_blocked.cuh) and warp-ballot K3 (m > 32, ms_k3_warp.cuh).
#include "ms_k3_blocked.cuh"
#include "ms_k3_warp.cuh"
#include "ms_k3_v2.cuh"
#include "ms_k3_lsd.cuh"

namespace ms {
cudaError_t k3p_launch_splitters(const K3pArgs &a) { return k3p_launch<SPLITTERS>(a); }
cudaError_t k3w_launch_splitters(const K3pArgs &a) { return k3w_launch<SPLITTERS>(a); }
cudaError_t k3v_launch_splitters(const K3pArgs &a) { return k3v_launch<SPLITTERS>(a); }
cudaError_t k3h_launch_splitters(const K3pArgs &a) { return k3h_launch<SPLITTERS>(a); }
}  // namespace ms
