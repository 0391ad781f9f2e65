// Instances of the four-row-group misaligned TMV kernel (tmv_group_kernel.cuh, round 2):
// fp32 and int32 (uint32 arithmetic); (S slots per thread, U groups in flight, max threads)
// in {(1, 4, 1024), (1, 8, 512), (2, 4, 640), (3, 2, 640), (4, 2, 640)}.
#include "tmv_group_kernel.cuh"
#include "adaptic.h"

namespace adaptic {

static_assert(TG_GROUP == TG_GROUP_H, "four-row-group merge width: kernel vs planner");

template <class T>
static void* tg(int S, int U) {
    if (S == 1 && U == 4) return reinterpret_cast<void*>(&tmv_group_kernel<T, 1, 4, 1024>);
    if (S == 1 && U == 8) return reinterpret_cast<void*>(&tmv_group_kernel<T, 1, 8, 512>);
    if (S == 2 && U == 4) return reinterpret_cast<void*>(&tmv_group_kernel<T, 2, 4, 640>);
    if (S == 3 && U == 2) return reinterpret_cast<void*>(&tmv_group_kernel<T, 3, 2, 640>);
    if (S == 4 && U == 2) return reinterpret_cast<void*>(&tmv_group_kernel<T, 4, 2, 640>);
    return nullptr;
}

void* tmv_group_fn(int dt, int S, int U) {
    return dt == ADAPTIC_I32 ? tg<uint32_t>(S, U) : tg<float>(S, U);
}

int tmv_group_maxnt(int S, int U) { return S == 1 ? (U == 4 ? 1024 : 512) : 640; }

}  // namespace adaptic
