// k3p_delta.cu -- instantiates the persistent K3 (ms_k3_blocked.cuh) for whatBucket kind DELTA.
#include "ms_k3_blocked.cuh"

namespace ms {
cudaError_t k3p_launch_delta(const K3pArgs &a) { return k3p_launch<DELTA>(a); }
}  // namespace ms
