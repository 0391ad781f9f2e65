// common.cuh -- element traits, 128-bit streaming loads and the warp/CTA
// combine used by every variant (sm_100a).
//
// The combine replaces the paper's Fig. 8 shared-memory tree: the
// L1 loop (halve active threads with a barrier per step) and the L2 loop (one
// warp, all 32 lanes active) become a __shfl_xor_sync butterfly inside
// each warp plus ONE shared-memory stage across warps.  Warp shuffles did not
// exist on the paper's sm_13/sm_20 targets.
#pragma once

#include <cstdint>
#include <cuda_runtime.h>

namespace adaptic {

// ---------------------------------------------------------------- element traits
// T = float (fp32, RNE, FMA allowed) or uint32_t (int32 semantics modulo 2^32).
template <class T> struct Vec4;
template <> struct Vec4<float> { using type = float4; };
template <> struct Vec4<uint32_t> { using type = uint4; };

template <class T> using vec4_t = typename Vec4<T>::type;

__device__ __forceinline__ float mac(float a, float b, float acc) { return fmaf(a, b, acc); }
__device__ __forceinline__ uint32_t mac(uint32_t a, uint32_t b, uint32_t acc) { return a * b + acc; }

template <class V> __device__ __forceinline__ V vzero() { V v; v.x = 0; v.y = 0; v.z = 0; v.w = 0; return v; }

template <class V> __device__ __forceinline__ V vadd(V a, V b) {
    a.x += b.x; a.y += b.y; a.z += b.z; a.w += b.w; return a;
}

// acc += a * b componentwise (MV/DOT: a = row chunk, b = x chunk)
template <class V> __device__ __forceinline__ void vmac(V& acc, const V& a, const V& b) {
    acc.x = mac(a.x, b.x, acc.x); acc.y = mac(a.y, b.y, acc.y);
    acc.z = mac(a.z, b.z, acc.z); acc.w = mac(a.w, b.w, acc.w);
}
// acc += a * s (TMV: a = 4 consecutive outputs' coefficients of one c, s = x[c])
template <class V, class T> __device__ __forceinline__ void vmacs(V& acc, const V& a, T s) {
    acc.x = mac(a.x, s, acc.x); acc.y = mac(a.y, s, acc.y);
    acc.z = mac(a.z, s, acc.z); acc.w = mac(a.w, s, acc.w);
}
// fixed pairwise order: (x + y) + (z + w)
template <class V> __device__ __forceinline__ auto vsum(const V& a) -> decltype(a.x) {
    return (a.x + a.y) + (a.z + a.w);
}

// elements s .. s+3 of the 8-element concatenation (lo, hi), s in 0..3 (a funnel shift
// of two aligned 128-bit vectors; the misaligned TMV and MV kernels)
template <class V> __device__ __forceinline__ V funnel4(const V& lo, const V& hi, int s) {
    V r;
    r.x = s == 0 ? lo.x : s == 1 ? lo.y : s == 2 ? lo.z : lo.w;
    r.y = s == 0 ? lo.y : s == 1 ? lo.z : s == 2 ? lo.w : hi.x;
    r.z = s == 0 ? lo.z : s == 1 ? lo.w : s == 2 ? hi.x : hi.y;
    r.w = s == 0 ? lo.w : s == 1 ? hi.x : s == 2 ? hi.y : hi.z;
    return r;
}

// ---------------------------------------------------------------- loads
// Matrix stream: read exactly once -> non-coherent path, no L1 allocation, and a
// 256-byte L2 fetch granule (each warp-wide 128-bit load covers 512 contiguous
// bytes, so the neighbouring sectors are always used).  Not volatile: ptxas may
// hoist/batch these loads, which is what the unrolled loops rely on.
__device__ __forceinline__ float4 ld_stream(const float4* p) {
    float4 v;
    asm("ld.global.nc.L1::no_allocate.L2::256B.v4.f32 {%0,%1,%2,%3}, [%4];"
        : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
    return v;
}
__device__ __forceinline__ uint4 ld_stream(const uint4* p) {
    uint4 v;
    asm("ld.global.nc.L1::no_allocate.L2::256B.v4.u32 {%0,%1,%2,%3}, [%4];"
        : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
    return v;
}
__device__ __forceinline__ float ld_stream(const float* p) {
    float v;
    asm("ld.global.nc.L1::no_allocate.L2::128B.f32 %0, [%1];" : "=f"(v) : "l"(p));
    return v;
}
__device__ __forceinline__ uint32_t ld_stream(const uint32_t* p) {
    uint32_t v;
    asm("ld.global.nc.L1::no_allocate.L2::128B.u32 %0, [%1];" : "=r"(v) : "l"(p));
    return v;
}
// Matrix stream whose 16-byte chunks are read twice by neighbouring lanes (the
// misaligned TMV funnel): allocate in L1 so the second read is an L1 hit.
__device__ __forceinline__ float4 ld_stream_l1(const float4* p) {
    float4 v;
    asm("ld.global.nc.L2::256B.v4.f32 {%0,%1,%2,%3}, [%4];"
        : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
    return v;
}
__device__ __forceinline__ uint4 ld_stream_l1(const uint4* p) {
    uint4 v;
    asm("ld.global.nc.L2::256B.v4.u32 {%0,%1,%2,%3}, [%4];"
        : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
    return v;
}
// x (re-read by many rows / CTAs): read-only path, cached in L1 and L2.
__device__ __forceinline__ float4 ld_x(const float4* p) { return __ldg(p); }
__device__ __forceinline__ uint4 ld_x(const uint4* p) { return __ldg(p); }
__device__ __forceinline__ float ld_x(const float* p) { return __ldg(p); }
__device__ __forceinline__ uint32_t ld_x(const uint32_t* p) { return __ldg(p); }
// Partials written by other CTAs of the same launch: bypass L1.
__device__ __forceinline__ float ld_partial(const float* p) { return __ldcg(p); }
__device__ __forceinline__ uint32_t ld_partial(const uint32_t* p) { return __ldcg(p); }
__device__ __forceinline__ float4 ld_partial(const float4* p) { return __ldcg(p); }
__device__ __forceinline__ uint4 ld_partial(const uint4* p) { return __ldcg(p); }
template <class T> __device__ __forceinline__ T ld_partial_any(const T* p) { return __ldcg(p); }

// ---------------------------------------------------------------- programmatic dependent launch
// Every kernel is launched with cudaLaunchAttributeProgrammaticStreamSerialization,
// so it may be scheduled while the previous kernel on the stream drains.  It must
// therefore wait for that grid (and its memory) before touching inputs, and it
// immediately allows the NEXT kernel to be scheduled into SMs its own CTAs free.
// Without PDL both instructions are no-ops.
#ifndef ADAPTIC_REFILL_FENCE
#define ADAPTIC_REFILL_FENCE 1
#endif
#ifndef ADAPTIC_PDL_EARLY_TRIGGER
#define ADAPTIC_PDL_EARLY_TRIGGER 0
#endif
__device__ __forceinline__ void pdl_prologue() {
    asm volatile("griddepcontrol.wait;" ::: "memory");
#if ADAPTIC_PDL_EARLY_TRIGGER
    asm volatile("griddepcontrol.launch_dependents;" :::);
#endif
}

// ---------------------------------------------------------------- TMA bulk copy + mbarrier
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
// Before a TMA refill of a ring stage the CTA has read through the generic proxy (after a
// __syncthreads).  A barrier alone orders the reads (CUTLASS's consumer-release pipelines issue
// no proxy fence), and dropping the fence measured no difference (the staged kernels' ~1 us
// per-tile cost is elsewhere), so the conservative fence stays on by default.
__device__ __forceinline__ void refill_fence() {
#if ADAPTIC_REFILL_FENCE
    fence_proxy_async();
#endif
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;"
                 :: "r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    asm volatile(
        "{\n"
        ".reg .pred p;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
        "@!p bra WAIT_%=;\n"
        "}\n" :: "r"(smem_u32(bar)), "r"(parity) : "memory");
}
// Ring position of a staged pipeline, advanced once per tile: the stage index and the
// mbarrier parity to wait for.  (Deriving them as i % stages and i / stages with a 64-bit
// tile counter costs two software 64-bit divisions per thread per tile -- ~1 us per tile
// per CTA measured on the staged kernels, the whole time of a small tile.)
__device__ __forceinline__ void ring_advance(int& st, uint32_t& ph, int stages) {
    if (++st == stages) { st = 0; ph ^= 1u; }
}

// 1-D bulk copy global -> shared, completion counted on the mbarrier (TMA engine;
// SASS UBLKCP).  dst, src 16-byte aligned; bytes a multiple of 16.
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;"
        :: "r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(0x12F0000000000000ull)  // EVICT_FIRST
        : "memory");
}
__device__ __forceinline__ void bulk_g2s_keep(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
        :: "r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}

// Stage `bytes` (multiple of 16, both pointers 16-byte aligned) of global memory
// into shared memory with the TMA engine; every thread of the CTA returns after
// the data has landed.  `bar` is a CTA-shared mbarrier used once (phase 0).
__device__ __forceinline__ void stage_to_smem(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
    if (threadIdx.x == 0) {
        mbar_init(bar, 1);
        fence_mbar_init();
        mbar_arrive_expect_tx(bar, bytes);
        constexpr uint32_t kPiece = 32768;
        for (uint32_t off = 0; off < bytes; off += kPiece)
            bulk_g2s_keep(static_cast<char*>(dst) + off, static_cast<const char*>(src) + off,
                          bytes - off < kPiece ? bytes - off : kPiece, bar);
    }
    __syncthreads();                       // barrier initialised before anyone waits
    mbar_wait(bar, 0);
}

// ---------------------------------------------------------------- combines
// Butterfly over the G lanes of an aligned lane group (G a power of two <= 32).
// Every lane of the group ends with the group total; the addition tree is fixed.
template <int G, class T> __device__ __forceinline__ T group_sum(T v) {
#pragma unroll
    for (int o = G / 2; o >= 1; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

// Sum over lanes that share (lane % STRIDE), i.e. xor offsets STRIDE..16.
template <int STRIDE, class T> __device__ __forceinline__ T strided_sum(T v) {
#pragma unroll
    for (int o = 16; o >= STRIDE; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

// Whole-CTA sum of one value per thread; result valid in thread 0.
// smem must hold NT/32 values.  Fixed tree: warp butterfly, then warp 0 sums
// the per-warp values with a butterfly.  Ends with a __syncthreads-free path
// for thread 0; callers that reuse smem must __syncthreads() first.
template <int NT, class T> __device__ __forceinline__ T cta_sum(T v, T* smem) {
    constexpr int NW = NT / 32;
    v = group_sum<32>(v);
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    if (NW == 1) return v;
    if (lane == 0) smem[warp] = v;
    __syncthreads();
    T w = T(0);
    if (warp == 0) {
        w = lane < NW ? smem[lane] : T(0);
        w = group_sum<32>(w);
    }
    return w;
}

// ---------------------------------------------------------------- ticket merge
// Phase 2 of the paper's two-kernel reduction (Fig. 7c), done in the
// same launch: each CTA publishes its partial, then takes a ticket; the CTA
// that draws the last ticket of its group merges all S partials in a FIXED
// order (independent of which CTA arrived last) and re-arms the counter.
__device__ __forceinline__ bool ticket_is_last(unsigned int* counter, unsigned int S, unsigned int* s_flag) {
    __threadfence();                       // partials visible device-wide before the ticket
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned int t = atomicAdd(counter, 1u);
        bool last = (t == S - 1);
        if (last) *counter = 0u;           // re-arm for the next run (no other CTA touches it now)
        *s_flag = last ? 1u : 0u;
    }
    __syncthreads();
    bool last = *s_flag != 0u;
    if (last) __threadfence();             // acquire side: see every partial
    return last;
}

}  // namespace adaptic
