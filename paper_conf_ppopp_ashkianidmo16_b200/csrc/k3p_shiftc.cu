// k3p_shiftc.cu -- instantiates the persistent K3 (ms_k3_blocked.cuh) for whatBucket kind SHIFTC.
#include "ms_k3_blocked.cuh"

namespace ms {
cudaError_t k3p_launch_shiftc(const K3pArgs &a) { return k3p_launch<SHIFTC>(a); }
}  // namespace ms
