// Instances of the TMA-staged multi-vector MV kernel (mmv_ring_kernel.cuh):
// fp32 K in {1, 2, 4, 8}; int32 (uint32 arithmetic, modulo 2^32) K = 1.
#include "mmv_ring_kernel.cuh"
#include "adaptic.h"

namespace adaptic {

void* mmv_ring_fn(int dt, int K) {
    if (dt == ADAPTIC_I32) return K == 1 ? reinterpret_cast<void*>(&mmv_ring_kernel<uint32_t, 1>) : nullptr;
    switch (K) {
        case 1: return reinterpret_cast<void*>(&mmv_ring_kernel<float, 1>);
        case 2: return reinterpret_cast<void*>(&mmv_ring_kernel<float, 2>);
        case 4: return reinterpret_cast<void*>(&mmv_ring_kernel<float, 4>);
        case 8: return reinterpret_cast<void*>(&mmv_ring_kernel<float, 8>);
        default: return nullptr;
    }
}

}  // namespace adaptic
