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

// whole-CTA reduction of k <= RTC_KMAX long rows per staged tile (MV_CPR, XSMEM 11): NT in
// {256, 512}, MX x values per thread in {4, 8, 16, 36} (C <= NT * MX), KR rows bound in
// {1, 2, 3, 4, 6, 8} (k <= KR)
template <class T, int NT, int MX>
static void* rtc_k(int KR) {
    switch (KR) {
        case 1: return reinterpret_cast<void*>(&mv_rowtile_cta_kernel<T, NT, MX, 1>);
        case 2: return reinterpret_cast<void*>(&mv_rowtile_cta_kernel<T, NT, MX, 2>);
        case 3: return reinterpret_cast<void*>(&mv_rowtile_cta_kernel<T, NT, MX, 3>);
        case 4: return reinterpret_cast<void*>(&mv_rowtile_cta_kernel<T, NT, MX, 4>);
        case 6: return reinterpret_cast<void*>(&mv_rowtile_cta_kernel<T, NT, MX, 6>);
        case 8: return reinterpret_cast<void*>(&mv_rowtile_cta_kernel<T, NT, MX, 8>);
        default: return nullptr;
    }
}
template <class T, int NT>
static void* rtc_m(int MX, int KR) {
    switch (MX) {
        case 4: return rtc_k<T, NT, 4>(KR);
        case 8: return rtc_k<T, NT, 8>(KR);
        case 16: return rtc_k<T, NT, 16>(KR);
        case 36: return rtc_k<T, NT, 36>(KR);
        default: return nullptr;
    }
}
template <class T>
static void* rtc_n(int NT, int MX, int KR) {
    return NT == 256 ? rtc_m<T, 256>(MX, KR) : NT == 512 ? rtc_m<T, 512>(MX, KR) : nullptr;
}
int rowtile_cta_kr(int k) { return k <= 4 ? k : k <= 6 ? 6 : 8; }
void* rowtile_cta_fn(int dtype, int NT, int MX, int k) {
    const int KR = rowtile_cta_kr(k);
    return dtype == DT_F32 ? rtc_n<float>(NT, MX, KR) : rtc_n<uint32_t>(NT, MX, KR);
}
static_assert(RTC_KMAX == RTC_KMAX_H, "long-row tile height: kernel vs planner");

// column-chunk form (mv_chunk_cta_kernel, XSMEM 13): NT in {256, 512}, MX in {8, 16, 36},
// KR in {1, 2, 4} (k <= KR row segments per tile)
template <class T, int NT, int MX>
static void* ck_k(int KR) {
    switch (KR) {
        case 1: return reinterpret_cast<void*>(&mv_chunk_cta_kernel<T, NT, MX, 1>);
        case 2: return reinterpret_cast<void*>(&mv_chunk_cta_kernel<T, NT, MX, 2>);
        case 4: return reinterpret_cast<void*>(&mv_chunk_cta_kernel<T, NT, MX, 4>);
        default: return nullptr;
    }
}
template <class T, int NT>
static void* ck_m(int MX, int KR) {
    switch (MX) {
        case 8: return ck_k<T, NT, 8>(KR);
        case 16: return ck_k<T, NT, 16>(KR);
        case 36: return ck_k<T, NT, 36>(KR);
        default: return nullptr;
    }
}
void* chunk_cta_fn(int dtype, int NT, int MX, int k) {
    const int KR = k <= 1 ? 1 : k <= 2 ? 2 : k <= 4 ? 4 : 0;
    if (KR == 0) return nullptr;
    if (NT == 256) return dtype == DT_F32 ? ck_m<float, 256>(MX, KR) : ck_m<uint32_t, 256>(MX, KR);
    if (NT == 512) return dtype == DT_F32 ? ck_m<float, 512>(MX, KR) : ck_m<uint32_t, 512>(MX, KR);
    return nullptr;
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
        case 544 * 4 + 1: return reinterpret_cast<void*>(&tmv_rowtile_kernel<T, 544, 1>);   // 17 warps: slices
        case 544 * 4 + 2: return reinterpret_cast<void*>(&tmv_rowtile_kernel<T, 544, 2>);   // of R + 1 rows
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
