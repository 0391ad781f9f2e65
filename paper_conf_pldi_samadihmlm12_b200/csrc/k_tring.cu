// Instances of the TMA-ring TMV kernel (tmv_ring_kernel.cuh): fp32 K in {1, 2, 4, 8} x
// OPT (words per lane per row) in {1, 2, 4, 8} with K OPT <= 32; int32 (modulo 2^32) K = 1.
#include "tmv_ring_kernel.cuh"
#include "adaptic.h"

namespace adaptic {

template <class T, int K>
static void* tr_opt(int opt) {
    switch (opt) {
        case 1: return reinterpret_cast<void*>(&tmv_ring_kernel<T, K, 1>);
        case 2: return reinterpret_cast<void*>(&tmv_ring_kernel<T, K, 2>);
        case 4: return reinterpret_cast<void*>(&tmv_ring_kernel<T, K, 4>);
        case 8: if constexpr (K * 8 <= 32) return reinterpret_cast<void*>(&tmv_ring_kernel<T, K, 8>);
                else return nullptr;
        default: return nullptr;
    }
}

void* tmv_ring_fn(int dt, int K, int opt) {
    if (dt == ADAPTIC_I32) return K == 1 ? tr_opt<uint32_t, 1>(opt) : nullptr;
    switch (K) {
        case 1: return tr_opt<float, 1>(opt);
        case 2: return tr_opt<float, 2>(opt);
        case 4: return tr_opt<float, 4>(opt);
        case 8: return tr_opt<float, 8>(opt);
        default: return nullptr;
    }
}

int64_t tring_stage_words_h(int64_t R, int TW, int CR, int K) { return tring_stage_words(R, TW, CR, K); }

}  // namespace adaptic
