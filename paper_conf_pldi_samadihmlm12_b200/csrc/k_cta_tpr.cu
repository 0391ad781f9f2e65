// Instances of mv_cta_kernel (MV_CPR / MV_SPLIT) and mv_tpr_kernel (MV_TPR).
#include "mv_kernels.cuh"
#include "tpr_kernel.cuh"

namespace adaptic {

// (RB, U) combinations: RB rows per CTA step x U loads per row.
template <class T, int NT, int RB, int U, bool VEC, int XM, bool PIPE>
static void* cfn() {
    // 1024-thread CTAs have 64 registers per thread: at most 4 vector loads per
    // step and no register double buffering
    if constexpr (NT == 1024 && (RB * U > 4 || PIPE)) return nullptr;
    else return reinterpret_cast<void*>(&mv_cta_kernel<T, NT, RB, U, VEC, XM, PIPE>);
}

template <class T, bool VEC, int XM, int NT, bool PIPE>
static void* cpick_nt(int RB, int U) {
    switch (RB * 16 + U) {
        case 1 * 16 + 2: return cfn<T, NT, 1, 2, VEC, XM, PIPE>();
        case 1 * 16 + 4: return cfn<T, NT, 1, 4, VEC, XM, PIPE>();
        case 1 * 16 + 8: return cfn<T, NT, 1, 8, VEC, XM, PIPE>();
        case 2 * 16 + 2: return cfn<T, NT, 2, 2, VEC, XM, PIPE>();
        case 2 * 16 + 4: return cfn<T, NT, 2, 4, VEC, XM, PIPE>();
        case 4 * 16 + 2: return cfn<T, NT, 4, 2, VEC, XM, PIPE>();
        default: return nullptr;
    }
}

template <class T, bool VEC, int XM>
static void* cpick(int NT, int RB, int U, bool pipe) {
    switch (NT) {
        case 256: return pipe ? cpick_nt<T, VEC, XM, 256, true>(RB, U) : cpick_nt<T, VEC, XM, 256, false>(RB, U);
        case 1024: return pipe ? nullptr : cpick_nt<T, VEC, XM, 1024, false>(RB, U);
        default: return nullptr;
    }
}

template <class T>
static void* cta_fn_t(int NT, int RB, int U, bool vec, int xm, bool pipe) {
    switch (xm) {
        case XM_LDG: return vec ? cpick<T, true, XM_LDG>(NT, RB, U, pipe) : cpick<T, false, XM_LDG>(NT, RB, U, pipe);
        case XM_SMEM: return vec ? cpick<T, true, XM_SMEM>(NT, RB, U, pipe) : cpick<T, false, XM_SMEM>(NT, RB, U, pipe);
        case XM_ROW: return vec ? cpick<T, true, XM_ROW>(NT, RB, U, pipe) : cpick<T, false, XM_ROW>(NT, RB, U, pipe);
        default: return nullptr;
    }
}

void* cta_fn(int dtype, int NT, int RB, int U, bool vec, int xm, bool pipe) {
    return dtype == DT_F32 ? cta_fn_t<float>(NT, RB, U, vec, xm, pipe) : cta_fn_t<uint32_t>(NT, RB, U, vec, xm, pipe);
}

template <class T, bool SC>
static void* tpr_fn_s(int NT, bool px) {
    switch (NT) {
        case 128: return px ? reinterpret_cast<void*>(&mv_tpr_kernel<T, 128, true, SC>)
                            : reinterpret_cast<void*>(&mv_tpr_kernel<T, 128, false, SC>);
        case 256: return px ? reinterpret_cast<void*>(&mv_tpr_kernel<T, 256, true, SC>)
                            : reinterpret_cast<void*>(&mv_tpr_kernel<T, 256, false, SC>);
        default: return nullptr;
    }
}

void* tpr_fn(int dtype, int NT, bool px, bool scal) {
    if (dtype == DT_F32) return scal ? tpr_fn_s<float, true>(NT, px) : tpr_fn_s<float, false>(NT, px);
    return scal ? tpr_fn_s<uint32_t, true>(NT, px) : tpr_fn_s<uint32_t, false>(NT, px);
}

}  // namespace adaptic
