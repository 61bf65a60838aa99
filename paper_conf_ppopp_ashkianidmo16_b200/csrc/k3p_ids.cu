// k3p_ids.cu -- instantiates the persistent K3 (ms_k3_blocked.cuh) for whatBucket kind IDS.
#include "ms_k3_blocked.cuh"

namespace ms {
cudaError_t k3p_launch_ids(const K3pArgs &a) { return k3p_launch<IDS>(a); }
}  // namespace ms
