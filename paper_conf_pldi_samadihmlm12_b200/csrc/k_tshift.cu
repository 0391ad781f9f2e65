// Instances of the constant-shift misaligned TMV kernel (tmv_mis_kernel.cuh, round 2):
// fp32 and int32 (uint32 arithmetic), LR in {16, 32, 64} (c-lanes 16, 8, 4), U in {2, 4, 8},
// NT = 256.
#include "tmv_mis_kernel.cuh"
#include "adaptic.h"

namespace adaptic {

template <class T, int LR>
static void* ts_u(int U) {
    switch (U) {
        case 2: return reinterpret_cast<void*>(&tmv_shift_kernel<T, LR, 2, 256>);
        case 4: return reinterpret_cast<void*>(&tmv_shift_kernel<T, LR, 4, 256>);
        case 8: return reinterpret_cast<void*>(&tmv_shift_kernel<T, LR, 8, 256>);
        default: return nullptr;
    }
}

template <class T>
static void* ts_l(int LR, int U) {
    switch (LR) {
        case 16: return ts_u<T, 16>(U);
        case 32: return ts_u<T, 32>(U);
        case 64: return ts_u<T, 64>(U);
        default: return nullptr;
    }
}

void* tmv_shift_fn(int dt, int LR, int U) {
    return dt == ADAPTIC_I32 ? ts_l<uint32_t>(LR, U) : ts_l<float>(LR, U);
}

// sliding-window misaligned TMV (tmv_window_kernel): G8 groups of 4 rows in flight, NT = 256
void* tmv_window_fn(int dt, int G8) {
    if (dt == ADAPTIC_I32)
        return G8 == 1 ? reinterpret_cast<void*>(&tmv_window_kernel<uint32_t, 1, 256>)
             : G8 == 2 ? reinterpret_cast<void*>(&tmv_window_kernel<uint32_t, 2, 256>) : nullptr;
    return G8 == 1 ? reinterpret_cast<void*>(&tmv_window_kernel<float, 1, 256>)
         : G8 == 2 ? reinterpret_cast<void*>(&tmv_window_kernel<float, 2, 256>) : nullptr;
}

// warp-tile form (S = 1): register cap for 2 resident CTAs of 256 (8 rows in flight) or 3
// (4 rows; 8 rows at 3 CTAs spill)
template <class T>
static void* tww(int G8, int minb) {
    if (G8 == 2 && minb <= 2) return reinterpret_cast<void*>(&tmv_window_warp_kernel<T, 2, 256, 2>);
    if (G8 == 1 && minb <= 2) return reinterpret_cast<void*>(&tmv_window_warp_kernel<T, 1, 256, 2>);
    if (G8 == 1 && minb == 3) return reinterpret_cast<void*>(&tmv_window_warp_kernel<T, 1, 256, 3>);
    return nullptr;
}
void* tmv_window_warp_fn(int dt, int G8, int minb) {
    return dt == ADAPTIC_I32 ? tww<uint32_t>(G8, minb) : tww<float>(G8, minb);
}

}  // namespace adaptic
