// Instances of mv_cta_kernel (MV_CPR / MV_SPLIT) and mv_tpr_kernel (MV_TPR).
#include "mv_kernels.cuh"
#include "tpr_kernel.cuh"

namespace adaptic {

// (RB, U) combinations: RB rows per CTA step x U loads per row.
template <class T, int NT, int RB, int U, bool VEC, int XM>
static void* cfn() {
    // 1024-thread CTAs have 64 registers per thread: at most 4 vector loads per step
    if constexpr (NT == 1024 && RB * U > 4) return nullptr;
    else return reinterpret_cast<void*>(&mv_cta_kernel<T, NT, RB, U, VEC, XM>);
}

template <class T, bool VEC, int XM, int NT>
static void* cpick_nt(int RB, int U) {
    switch (RB * 16 + U) {
        case 1 * 16 + 2: return cfn<T, NT, 1, 2, VEC, XM>();
        case 1 * 16 + 4: return cfn<T, NT, 1, 4, VEC, XM>();
        case 1 * 16 + 8: return cfn<T, NT, 1, 8, VEC, XM>();
        case 2 * 16 + 2: return cfn<T, NT, 2, 2, VEC, XM>();
        case 2 * 16 + 4: return cfn<T, NT, 2, 4, VEC, XM>();
        case 4 * 16 + 2: return cfn<T, NT, 4, 2, VEC, XM>();
        default: return nullptr;
    }
}

template <class T, bool VEC, int XM>
static void* cpick(int NT, int RB, int U) {
    switch (NT) {
        case 256: return cpick_nt<T, VEC, XM, 256>(RB, U);
        case 1024: return cpick_nt<T, VEC, XM, 1024>(RB, U);
        default: return nullptr;
    }
}

template <class T>
static void* cta_fn_t(int NT, int RB, int U, bool vec, int xm) {
    switch (xm) {
        case XM_LDG: return vec ? cpick<T, true, XM_LDG>(NT, RB, U) : cpick<T, false, XM_LDG>(NT, RB, U);
        case XM_SMEM: return vec ? cpick<T, true, XM_SMEM>(NT, RB, U) : cpick<T, false, XM_SMEM>(NT, RB, U);
        case XM_ROW: return vec ? cpick<T, true, XM_ROW>(NT, RB, U) : cpick<T, false, XM_ROW>(NT, RB, U);
        default: return nullptr;
    }
}

void* cta_fn(int dtype, int NT, int RB, int U, bool vec, int xm) {
    return dtype == DT_F32 ? cta_fn_t<float>(NT, RB, U, vec, xm) : cta_fn_t<uint32_t>(NT, RB, U, vec, xm);
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
