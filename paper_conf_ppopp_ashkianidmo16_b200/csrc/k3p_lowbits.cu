// k3p_lowbits.cu -- instantiates the persistent K3 (ms_k3_blocked.cuh) for whatBucket kind LOWBITS.
#include "ms_k3_blocked.cuh"

namespace ms {
cudaError_t k3p_launch_lowbits(const K3pArgs &a) { return k3p_launch<LOWBITS>(a); }
}  // namespace ms
