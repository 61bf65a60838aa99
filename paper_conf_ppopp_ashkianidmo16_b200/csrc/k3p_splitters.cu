// k3p_splitters.cu -- instantiates the persistent K3 (ms_k3_blocked.cuh) for whatBucket kind SPLITTERS.
#include "ms_k3_blocked.cuh"

namespace ms {
cudaError_t k3p_launch_splitters(const K3pArgs &a) { return k3p_launch<SPLITTERS>(a); }
}  // namespace ms
