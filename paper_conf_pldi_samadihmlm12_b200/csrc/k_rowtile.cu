// Instances of mv_rowtile_kernel (MV_SUBWARP / MV_WPR with [ADAPTIC_P_XSMEM] = 4):
// G in {1, 2, 4, 8, 16, 32} lanes per row, 256 or 512 threads, fp32 / int32, MV / DOT.
#include "launch.h"
#include "rowtile_kernel.cuh"
#include "tmv_rowtile_kernel.cuh"

namespace adaptic {

// the planner (adaptic.cu) sizes rings with the launch.h constants
static_assert(RT_MAX_STAGES == RT_MAX_STAGES_H, "row-tile ring depth: kernel vs planner");
static_assert(TRT_MAX_STAGES == RT_MAX_STAGES_H, "TMV tile ring depth: kernel vs planner");

template <class T, int NT, bool PX>
static void* rt_g(int G) {
    switch (G) {
        case 1: return reinterpret_cast<void*>(&mv_rowtile_kernel<T, NT, 1, PX>);
        case 2: return reinterpret_cast<void*>(&mv_rowtile_kernel<T, NT, 2, PX>);
        case 4: return reinterpret_cast<void*>(&mv_rowtile_kernel<T, NT, 4, PX>);
        case 8: return reinterpret_cast<void*>(&mv_rowtile_kernel<T, NT, 8, PX>);
        case 16: return reinterpret_cast<void*>(&mv_rowtile_kernel<T, NT, 16, PX>);
        case 32: return reinterpret_cast<void*>(&mv_rowtile_kernel<T, NT, 32, PX>);
        default: return nullptr;
    }
}

template <class T>
static void* rt_t(int NT, int G, bool px) {
    if (NT == 256) return px ? rt_g<T, 256, true>(G) : rt_g<T, 256, false>(G);
    if (NT == 512) return px ? rt_g<T, 512, true>(G) : rt_g<T, 512, false>(G);
    return nullptr;
}

void* rowtile_fn(int dtype, int NT, int G, bool px) {
    return dtype == DT_F32 ? rt_t<float>(NT, G, px) : rt_t<uint32_t>(NT, G, px);
}

}  // namespace adaptic

namespace adaptic {
// words per operand tile (the kernel's tile_w): k*C plus up to 3 head and 3 tail words,
// rounded up to 16 bytes
size_t rowtile_tile_words(int64_t k, int64_t C) { return size_t((k * C + 6 + 3) / 4) * 4; }
}  // namespace adaptic

namespace adaptic {
// TMV on staged tiles of B (tmv_rowtile_kernel.cuh): 256, 512 or 1024 threads, 1, 2 or 4
// outputs per thread (rpt = the power of two >= R / NT)
template <class T>
static void* trt(int NT, int rpt) {
    switch (NT * 4 + rpt) {
        case 256 * 4 + 1: return reinterpret_cast<void*>(&tmv_rowtile_kernel<T, 256, 1>);
        case 512 * 4 + 1: return reinterpret_cast<void*>(&tmv_rowtile_kernel<T, 512, 1>);
        case 1024 * 4 + 1: return reinterpret_cast<void*>(&tmv_rowtile_kernel<T, 1024, 1>);
        case 256 * 4 + 2: return reinterpret_cast<void*>(&tmv_rowtile_kernel<T, 256, 2>);
        case 512 * 4 + 2: return reinterpret_cast<void*>(&tmv_rowtile_kernel<T, 512, 2>);
        case 1024 * 4 + 2: return reinterpret_cast<void*>(&tmv_rowtile_kernel<T, 1024, 2>);
        case 512 * 4 + 4: return reinterpret_cast<void*>(&tmv_rowtile_kernel<T, 512, 4>);
        case 1024 * 4 + 4: return reinterpret_cast<void*>(&tmv_rowtile_kernel<T, 1024, 4>);
        default: return nullptr;
    }
}
void* tmv_rowtile_fn(int dtype, int NT, int rpt) {
    return dtype == DT_F32 ? trt<float>(NT, rpt) : trt<uint32_t>(NT, rpt);
}
}  // namespace adaptic
