// Instances of tmv_flat_kernel (TMV, R <= 256 and R % 4 != 0): NT = 256 (U 2/4/8) and
// NT = 1024 (U 2/4, for R > 64 so that floor(NT/R)*R keeps most threads busy), fp32 / int32.
#include "tmv_flat_kernel.cuh"

namespace adaptic {

template <class T, int NT>
static void* tf_u(int U) {
    switch (U) {
        case 2: return reinterpret_cast<void*>(&tmv_flat_kernel<T, NT, 2>);
        case 4: return reinterpret_cast<void*>(&tmv_flat_kernel<T, NT, 4>);
        case 8: if constexpr (NT <= 256) return reinterpret_cast<void*>(&tmv_flat_kernel<T, NT, 8>);
                else return nullptr;
        default: return nullptr;
    }
}

void* tmv_flat_fn(int dtype, int U, int NT) {
    if (NT == 1024) return dtype == DT_F32 ? tf_u<float, 1024>(U) : tf_u<uint32_t, 1024>(U);
    return dtype == DT_F32 ? tf_u<float, 256>(U) : tf_u<uint32_t, 256>(U);
}

}  // namespace adaptic
