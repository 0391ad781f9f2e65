// Instances of mv_cta_kernel (MV_CPR / MV_SPLIT) and mv_tpr_kernel (MV_TPR).
#include "mv_kernels.cuh"
#include "tpr_kernel.cuh"

namespace adaptic {

template <class T, int NT, int U, bool VEC, int PX>
static void* cfn() { return reinterpret_cast<void*>(&mv_cta_kernel<T, NT, U, VEC, PX>); }

template <class T, bool VEC, int PX>
static void* cpick(int NT, int U) {
#define ADAPTIC_U(N_)                                        \
    switch (U) {                                             \
        case 2: return cfn<T, N_, 2, VEC, PX>();             \
        case 4: return cfn<T, N_, 4, VEC, PX>();             \
        case 8: return cfn<T, N_, 8, VEC, PX>();             \
        default: return nullptr;                             \
    }
    switch (NT) {
        case 256: ADAPTIC_U(256)
        case 1024: ADAPTIC_U(1024)
        default: return nullptr;
    }
#undef ADAPTIC_U
}

template <class T>
static void* cta_fn_t(int NT, int U, bool vec, int xm) {
    switch (xm) {
        case XM_LDG: return vec ? cpick<T, true, XM_LDG>(NT, U) : cpick<T, false, XM_LDG>(NT, U);
        case XM_SMEM: return vec ? cpick<T, true, XM_SMEM>(NT, U) : cpick<T, false, XM_SMEM>(NT, U);
        case XM_ROW: return vec ? cpick<T, true, XM_ROW>(NT, U) : cpick<T, false, XM_ROW>(NT, U);
        default: return nullptr;
    }
}

void* cta_fn(int dtype, int NT, int U, bool vec, int xm) {
    return dtype == DT_F32 ? cta_fn_t<float>(NT, U, vec, xm) : cta_fn_t<uint32_t>(NT, U, vec, xm);
}

template <class T>
static void* tpr_fn_t(int NT, bool px) {
    switch (NT) {
        case 128: return px ? reinterpret_cast<void*>(&mv_tpr_kernel<T, 128, true>)
                            : reinterpret_cast<void*>(&mv_tpr_kernel<T, 128, false>);
        case 256: return px ? reinterpret_cast<void*>(&mv_tpr_kernel<T, 256, true>)
                            : reinterpret_cast<void*>(&mv_tpr_kernel<T, 256, false>);
        default: return nullptr;
    }
}

void* tpr_fn(int dtype, int NT, bool px) {
    return dtype == DT_F32 ? tpr_fn_t<float>(NT, px) : tpr_fn_t<uint32_t>(NT, px);
}

}  // namespace adaptic
