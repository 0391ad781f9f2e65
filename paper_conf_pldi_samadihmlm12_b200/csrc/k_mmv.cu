// Instances of the multi-vector kernels (mmv_kernels.cuh), fp32, K in {2, 4, 8}:
//   group: G in {1,2,4,8,16,32} x U in {1,2,4} (K*U <= 16) x VEC, RB = 2
//   cta  : NT = 256, U in {1, 2} x VEC x x-in-shared-memory
//   tmmv : LR in {1,...,256} x VEC x U in {2, 4} (4 only for K <= 4), NT = 256
#include "mmv_kernels.cuh"
#include "adaptic.h"

namespace adaptic {

template <int K, int G, bool VEC>
static void* mg_u(int U) {
    switch (U) {
        case 1: return reinterpret_cast<void*>(&mmv_group_kernel<K, G, 2, 1, VEC, GROUP_NT>);
        case 2: return reinterpret_cast<void*>(&mmv_group_kernel<K, G, 2, 2, VEC, GROUP_NT>);
        case 4: if constexpr (K * 4 <= 16) return reinterpret_cast<void*>(&mmv_group_kernel<K, G, 2, 4, VEC, GROUP_NT>);
                else return nullptr;
        default: return nullptr;
    }
}

template <int K, bool VEC>
static void* mg_g(int G, int U) {
    switch (G) {
        case 1: return mg_u<K, 1, VEC>(U);
        case 2: return mg_u<K, 2, VEC>(U);
        case 4: return mg_u<K, 4, VEC>(U);
        case 8: return mg_u<K, 8, VEC>(U);
        case 16: return mg_u<K, 16, VEC>(U);
        case 32: return mg_u<K, 32, VEC>(U);
        default: return nullptr;
    }
}

template <int K, bool VEC>
static void* mc_u(int U, bool xs) {
    switch (U * 2 + (xs ? 1 : 0)) {
        case 2: return reinterpret_cast<void*>(&mmv_cta_kernel<K, 256, 1, VEC, false>);
        case 3: return reinterpret_cast<void*>(&mmv_cta_kernel<K, 256, 1, VEC, true>);
        case 4: return reinterpret_cast<void*>(&mmv_cta_kernel<K, 256, 2, VEC, false>);
        case 5: return reinterpret_cast<void*>(&mmv_cta_kernel<K, 256, 2, VEC, true>);
        default: return nullptr;
    }
}

template <int K, int U, bool VEC>
static void* mt_lu(int LR) {
    switch (LR) {
        case 1: return reinterpret_cast<void*>(&tmmv_kernel<K, 1, U, VEC, 256>);
        case 2: return reinterpret_cast<void*>(&tmmv_kernel<K, 2, U, VEC, 256>);
        case 4: return reinterpret_cast<void*>(&tmmv_kernel<K, 4, U, VEC, 256>);
        case 8: return reinterpret_cast<void*>(&tmmv_kernel<K, 8, U, VEC, 256>);
        case 16: return reinterpret_cast<void*>(&tmmv_kernel<K, 16, U, VEC, 256>);
        case 32: return reinterpret_cast<void*>(&tmmv_kernel<K, 32, U, VEC, 256>);
        case 64: return reinterpret_cast<void*>(&tmmv_kernel<K, 64, U, VEC, 256>);
        case 128: return reinterpret_cast<void*>(&tmmv_kernel<K, 128, U, VEC, 256>);
        case 256: return reinterpret_cast<void*>(&tmmv_kernel<K, 256, U, VEC, 256>);
        default: return nullptr;
    }
}

template <int K, bool VEC>
static void* mt_l(int LR, int U) {
    if (U == 2) return mt_lu<K, 2, VEC>(LR);
    if constexpr (K <= 4) { if (U == 4) return mt_lu<K, 4, VEC>(LR); }
    return nullptr;
}

// warp-per-row kernel with x in shared memory: RB = 1, U = 2, NT = 256
void* mmv_warp_fn(int K) {
    switch (K) {
        case 2: return reinterpret_cast<void*>(&mmv_warp_kernel<2, 1, 2, 256>);
        case 4: return reinterpret_cast<void*>(&mmv_warp_kernel<4, 1, 2, 256>);
        case 8: return reinterpret_cast<void*>(&mmv_warp_kernel<8, 1, 2, 256>);
        default: return nullptr;
    }
}

// x-tiled stream-K kernel: RB = 4 rows per warp step (2 at K = 8), U = 2 (4 at K = 1), NT = 256;
// K = 1 also for int32 (dt = ADAPTIC_I32)
void* mmv_tile_fn(int dt, int K) {
    if (dt == ADAPTIC_I32) return K == 1 ? reinterpret_cast<void*>(&mmv_tile_kernel<uint32_t, 1, 4, 4, 256>) : nullptr;
    switch (K) {
        case 1: return reinterpret_cast<void*>(&mmv_tile_kernel<float, 1, 4, 4, 256>);
        case 2: return reinterpret_cast<void*>(&mmv_tile_kernel<float, 2, 4, 2, 256>);
        case 4: return reinterpret_cast<void*>(&mmv_tile_kernel<float, 4, 4, 2, 256>);
        case 8: return reinterpret_cast<void*>(&mmv_tile_kernel<float, 8, 2, 2, 256>);
        default: return nullptr;
    }
}

template <int K>
static void* tt_l(int LR) {
    switch (LR) {
        case 16: return reinterpret_cast<void*>(&tmmv_tma_kernel<K, 16, 256>);
        case 32: return reinterpret_cast<void*>(&tmmv_tma_kernel<K, 32, 256>);
        case 64: return reinterpret_cast<void*>(&tmmv_tma_kernel<K, 64, 256>);
        case 128: return reinterpret_cast<void*>(&tmmv_tma_kernel<K, 128, 256>);
        case 256: return reinterpret_cast<void*>(&tmmv_tma_kernel<K, 256, 256>);
        default: return nullptr;
    }
}

void* tmmv_tma_fn(int K, int LR) {
    switch (K) {
        case 2: return tt_l<2>(LR);
        case 4: return tt_l<4>(LR);
        case 8: return tt_l<8>(LR);
        default: return nullptr;
    }
}

// TMV groups of 4 rows, x as float4 (+ L2 prefetch PF groups ahead): LR in {16, 32, 64, 128,
// 256}, PF in {0, 2, 4}, NT = 256
template <int K, int PF>
static void* t4_l(int LR) {
    switch (LR) {
        case 16: return reinterpret_cast<void*>(&tmmv4_kernel<K, 16, PF, 256>);
        case 32: return reinterpret_cast<void*>(&tmmv4_kernel<K, 32, PF, 256>);
        case 64: return reinterpret_cast<void*>(&tmmv4_kernel<K, 64, PF, 256>);
        case 128: return reinterpret_cast<void*>(&tmmv4_kernel<K, 128, PF, 256>);
        case 256: return reinterpret_cast<void*>(&tmmv4_kernel<K, 256, PF, 256>);
        default: return nullptr;
    }
}
template <int K>
static void* t4_p(int LR, int PF) {
    switch (PF) {
        case 0: return t4_l<K, 0>(LR);
        case 2: return t4_l<K, 2>(LR);
        case 4: return t4_l<K, 4>(LR);
        default: return nullptr;
    }
}
void* tmmv4_fn(int K, int LR, int PF) {
    switch (K) {
        case 2: return t4_p<2>(LR, PF);
        case 4: return t4_p<4>(LR, PF);
        case 8: return t4_p<8>(LR, PF);
        default: return nullptr;
    }
}

#define ADAPTIC_K(FN, ...)                                                       \
    switch (K) {                                                                 \
        case 2: return vec ? FN<2, true>(__VA_ARGS__) : FN<2, false>(__VA_ARGS__); \
        case 4: return vec ? FN<4, true>(__VA_ARGS__) : FN<4, false>(__VA_ARGS__); \
        case 8: return vec ? FN<8, true>(__VA_ARGS__) : FN<8, false>(__VA_ARGS__); \
        default: return nullptr;                                                 \
    }

void* mmv_group_fn(int K, int G, int U, bool vec) { ADAPTIC_K(mg_g, G, U) }
void* mmv_cta_fn(int K, int U, bool vec, bool xs) { ADAPTIC_K(mc_u, U, xs) }
void* tmmv_fn(int K, int LR, int U, bool vec) { ADAPTIC_K(mt_l, LR, U) }
#undef ADAPTIC_K

}  // namespace adaptic
