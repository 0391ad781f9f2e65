// Instances of tmv_flat_kernel (TMV, R <= 64 and R % 4 != 0): NT = 256, U in {2, 4, 8}, fp32 / int32.
#include "tmv_flat_kernel.cuh"

namespace adaptic {

template <class T>
static void* tf_u(int U) {
    switch (U) {
        case 2: return reinterpret_cast<void*>(&tmv_flat_kernel<T, 256, 2>);
        case 4: return reinterpret_cast<void*>(&tmv_flat_kernel<T, 256, 4>);
        case 8: return reinterpret_cast<void*>(&tmv_flat_kernel<T, 256, 8>);
        default: return nullptr;
    }
}

void* tmv_flat_fn(int dtype, int U) { return dtype == DT_F32 ? tf_u<float>(U) : tf_u<uint32_t>(U); }

}  // namespace adaptic
