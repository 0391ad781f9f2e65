// blas1_kernels.cuh -- BLAS-1 reductions on the same engine, sm_100a.
//
// The paper's Fig. 9 input-portability benchmarks include the CUBLAS routines
// Sasum, Snrm2 and Isamax/Isamin (Sec. 5.1): the same stream-reduction
// actor as MV -- N_arrays arrays of N_elements each, one output per array
// -- with a different associative/commutative operator.  Here
// rows = N vectors, cols = L elements, a row-major N x L, and the operator is a
// policy of the two kernels below:
//
//   ASUM  y_n = sum_e |a|          fp32 accumulators (4-wide, folded every FOLD
//                                  steps like MV: provable 1e-4 bound)
//   NRM2  y_n = sqrt(sum_e a^2)    squares of fp32 values are exact in fp64 and
//                                  cannot overflow or underflow there, so the
//                                  sum of squares is accumulated in fp64 (no
//                                  scaling pass; one rounding to fp32 at the end)
//   IAMAX smallest 1-based e with |a_e| maximal; IAMIN likewise for the minimum.
//                                  |a| of an fp32 value is exact, compared as its
//                                  IEEE bit pattern (monotone for |a| >= 0) packed
//                                  with the index into one uint64 so max/min
//                                  also resolves ties to the first index: the
//                                  result is exact and order independent.
//                                  NaN never wins (key 0 for max, ~0 for min)
//                                  unless it is a[0] (BLAS: the running maximum
//                                  starts at |a_1| and NaN compares false) -- a
//                                  leading NaN yields 1, checked at the end.
//
//   b1_group_kernel  G = 1..32 lanes per row (MV_SUBWARP / MV_WPR thread shapes)
//   b1_cta_kernel    one CTA per row (MV_CPR) or S CTAs per row + ticket merge
//                    in the same launch (MV_SPLIT, the two-kernel reduction of
//                    P:480 / Fig. 7c).
#pragma once

#include <type_traits>

#include "common.cuh"
#include "launch.h"

namespace adaptic {

enum B1Op { B1_ASUM = 0, B1_NRM2 = 1, B1_IAMAX = 2, B1_IAMIN = 3, B1_ALL = 4 };

// Per-op policy.  Acc<VEC> is a load slot's accumulator; P is what crosses
// lanes, warps and CTAs; comb() is the associative/commutative operator.
template <int OP> struct B1;

template <> struct B1<B1_ASUM> {
    using P = float;
    template <bool VEC> using Acc = typename std::conditional<VEC, float4, float>::type;
    static constexpr bool kFold = true;          // fp32 chains are folded (error bound)
    static constexpr bool kOneSlot = false;
    __device__ static P ident() { return 0.f; }
    __device__ static void zero(float& a) { a = 0.f; }
    __device__ static void zero(float4& a) { a = make_float4(0.f, 0.f, 0.f, 0.f); }
    __device__ static void elem(float& acc, float v, int64_t) { acc += fabsf(v); }
    __device__ static void elem(float4& acc, const float4& v, int64_t) {
        acc.x += fabsf(v.x); acc.y += fabsf(v.y); acc.z += fabsf(v.z); acc.w += fabsf(v.w);
    }
    __device__ static P fin(const float& a) { return a; }
    __device__ static P fin(const float4& a) { return (a.x + a.y) + (a.z + a.w); }
    __device__ static P comb(P a, P b) { return a + b; }
    __device__ static void add(float& a, const float& b) { a += b; }
    __device__ static void add(float4& a, const float4& b) { a.x += b.x; a.y += b.y; a.z += b.z; a.w += b.w; }
    __device__ static void store(void* y, int64_t r, P v, int64_t) { static_cast<float*>(y)[r] = v; }
};

template <> struct B1<B1_NRM2> {
    using P = double;
    template <bool VEC> using Acc = double;
    static constexpr bool kFold = false;         // fp64 sum of exact squares
    static constexpr bool kOneSlot = false;
    __device__ static P ident() { return 0.0; }
    __device__ static void zero(double& a) { a = 0.0; }
    __device__ static void elem(double& acc, float v, int64_t) { const double d = v; acc = fma(d, d, acc); }
    __device__ static void elem(double& acc, const float4& v, int64_t) {
        const double a = v.x, b = v.y, c = v.z, d = v.w;
        acc = fma(a, a, acc); acc = fma(b, b, acc); acc = fma(c, c, acc); acc = fma(d, d, acc);
    }
    __device__ static P fin(const double& a) { return a; }
    __device__ static P comb(P a, P b) { return a + b; }
    __device__ static void add(double& a, const double& b) { a += b; }
    __device__ static void store(void* y, int64_t r, P v, int64_t) {
        static_cast<float*>(y)[r] = float(sqrt(v));   // one rounding to fp32
    }
};

// IAMAX / IAMIN.  Hot loop: each load slot keeps (best, e) -- the extreme |a| it
// has seen and the FIRST element index reaching it (a slot visits indices in
// increasing order, so a strict compare keeps the first).  Per float4 that is a
// 4-way max/min plus one compare; the lane that attains it is resolved only when
// the best improves.  Across slots, lanes, warps and CTAs the pair travels as one
// uint64 (key << 32 | index bits) so that one unsigned max (min) compares the key
// first and breaks ties toward the smaller index.
//   IAMAX: best is a float, max via fmaxf (which ignores NaN: a NaN never wins)
//          starting from -1 (below every |a|); key = its bits (monotone for >= 0).
//   IAMIN: best is the key |a| bits as uint32 -- NaN keys exceed +inf's, so the
//          unsigned min never picks a NaN over a number; start 0xffffffff.
// A leading NaN is the BLAS special case (the running extreme starts at |a_1| and
// NaN compares false, so the answer is 1): element 0, when NaN, takes the extreme
// value (+inf for IAMAX, 0 for IAMIN) and so wins every tie by its index -- the
// check rides on data already in registers (a reload of a[0] at the store would
// put an L2 round trip at the end of every row).
__device__ __forceinline__ uint32_t abs_key(float v) { return __float_as_uint(v) & 0x7fffffffu; }

template <int OP> struct B1Arg {
    using P = unsigned long long;
    static constexpr bool kMax = (OP == B1_IAMAX);
    static constexpr bool kFold = false;
    static constexpr bool kOneSlot = false;
    using B = typename std::conditional<kMax, float, uint32_t>::type;
    struct Acc_ { B best; uint32_t e; };
    template <bool VEC> using Acc = Acc_;
    static constexpr uint32_t kNone = 0xffffffffu;
    __device__ static P ident() { return kMax ? 0ull : ~0ull; }
    __device__ static void zero(Acc_& a) {
        if constexpr (kMax) a.best = -1.f; else a.best = 0xffffffffu;
        a.e = kNone;
    }
    __device__ static B val(float v) {
        if constexpr (kMax) return fabsf(v); else return abs_key(v);
    }
    __device__ static B lead(float v, bool is0) {        // element 0: a NaN takes the extreme
        const B b = val(v);
        if (is0 && v != v) { if constexpr (kMax) return __int_as_float(0x7f800000); else return 0u; }
        return b;
    }
    __device__ static bool better(B a, B b) { return kMax ? (a > b) : (a < b); }   // NaN: false
    __device__ static B ext(B a, B b) {
        if constexpr (kMax) return fmaxf(a, b); else return a < b ? a : b;
    }
    __device__ static void elem(Acc_& acc, float v, int64_t e) {
        const B m = lead(v, e == 0);
        if (better(m, acc.best)) { acc.best = m; acc.e = uint32_t(e); }
    }
    __device__ static void elem(Acc_& acc, const float4& v, int64_t vi) {
        const B bx = lead(v.x, vi == 0), by = val(v.y), bz = val(v.z), bw = val(v.w);
        const B m = ext(ext(bx, by), ext(bz, bw));
        if (better(m, acc.best)) {
            acc.best = m;
            acc.e = uint32_t(vi) * 4u + (bx == m ? 0u : by == m ? 1u : bz == m ? 2u : 3u);
        }
    }
    __device__ static void add(Acc_& a, const Acc_& b) {
        if (better(b.best, a.best) || (b.best == a.best && b.e < a.e)) a = b;
    }
    __device__ static P fin(const Acc_& a) {
        if (a.e == kNone) return ident();
        const uint32_t key = kMax ? __float_as_uint(float(a.best)) : uint32_t(a.best);
        return (static_cast<P>(key) << 32) | (kMax ? 0xffffffffu - a.e : a.e);
    }
    __device__ static P comb(P a, P b) { return kMax ? (a > b ? a : b) : (a < b ? a : b); }
    __device__ static void store(void* y, int64_t r, P v, int64_t) {
        const uint32_t lo = uint32_t(v & 0xffffffffull);
        static_cast<int32_t*>(y)[r] = int32_t((kMax ? 0xffffffffu - lo : lo) + 1u);
    }
};
template <> struct B1<B1_IAMAX> : B1Arg<B1_IAMAX> {};
template <> struct B1<B1_IAMIN> : B1Arg<B1_IAMIN> {};

// ALL: horizontal actor integration ("assume there is a program that needs
// maximum and summation of all elements in an array. Instead of running two kernels
// ... Adaptic launches one kernel to compute both") -- the four BLAS-1 actors above
// share one pass over a.  y holds four N-vectors back to back:
// [asum (float) | nrm2 (float) | iamax (int32) | iamin (int32)].
// One accumulator per row (kOneSlot; 10 registers instead of 10 per load slot), so
// the fp32 asum chain takes U terms per step: it folds every FOLD/U steps.
struct B1AllP { double ssq; unsigned long long mx, mn; float asum; };
template <> struct B1<B1_ALL> {
    using MX = B1Arg<B1_IAMAX>;
    using MN = B1Arg<B1_IAMIN>;
    using P = B1AllP;
    template <bool VEC> struct Acc_ {
        typename B1<B1_ASUM>::template Acc<VEC> asum;
        double ssq;
        MX::Acc_ mx;
        MN::Acc_ mn;
    };
    template <bool VEC> using Acc = Acc_<VEC>;
    static constexpr bool kFold = true;
    static constexpr bool kOneSlot = true;
    __device__ static P ident() { P p; p.ssq = 0.0; p.mx = MX::ident(); p.mn = MN::ident(); p.asum = 0.f; return p; }
    template <bool VEC> __device__ static void zero(Acc_<VEC>& a) {
        B1<B1_ASUM>::zero(a.asum); a.ssq = 0.0; MX::zero(a.mx); MN::zero(a.mn);
    }
    template <bool VEC, class E> __device__ static void elem(Acc_<VEC>& a, const E& v, int64_t i) {
        B1<B1_ASUM>::elem(a.asum, v, i); B1<B1_NRM2>::elem(a.ssq, v, i); MX::elem(a.mx, v, i); MN::elem(a.mn, v, i);
    }
    template <bool VEC> __device__ static void add(Acc_<VEC>& a, const Acc_<VEC>& b) {
        B1<B1_ASUM>::add(a.asum, b.asum); a.ssq += b.ssq; MX::add(a.mx, b.mx); MN::add(a.mn, b.mn);
    }
    template <bool VEC> __device__ static P fin(const Acc_<VEC>& a) {
        P p; p.asum = B1<B1_ASUM>::fin(a.asum); p.ssq = a.ssq; p.mx = MX::fin(a.mx); p.mn = MN::fin(a.mn); return p;
    }
    __device__ static P comb(P a, const P& b) {
        a.asum += b.asum; a.ssq += b.ssq; a.mx = MX::comb(a.mx, b.mx); a.mn = MN::comb(a.mn, b.mn); return a;
    }
    __device__ static P shfl(P v, int o) {
        v.asum = __shfl_xor_sync(0xffffffffu, v.asum, o); v.ssq = __shfl_xor_sync(0xffffffffu, v.ssq, o);
        v.mx = __shfl_xor_sync(0xffffffffu, v.mx, o); v.mn = __shfl_xor_sync(0xffffffffu, v.mn, o);
        return v;
    }
    __device__ static void store(void* y, int64_t r, const P& v, int64_t R) {
        float* yf = static_cast<float*>(y);
        B1<B1_ASUM>::store(yf, r, v.asum, R);
        B1<B1_NRM2>::store(yf + R, r, v.ssq, R);
        MX::store(yf + 2 * R, r, v.mx, R);
        MN::store(yf + 3 * R, r, v.mn, R);
    }
};

// workspace partials of the fused op, read back by the merging CTA (bypass L1)
__device__ __forceinline__ B1AllP ld_partial_any(const B1AllP* p) {
    B1AllP v;
    v.ssq = __ldcg(&p->ssq); v.mx = __ldcg(&p->mx); v.mn = __ldcg(&p->mn); v.asum = __ldcg(&p->asum);
    return v;
}

// lane exchange: plain shuffle for scalar partials, the policy's own for structs
template <int OP, class P> __device__ __forceinline__ P b1_shfl(const P& v, int o) {
    if constexpr (std::is_arithmetic<P>::value) return __shfl_xor_sync(0xffffffffu, v, o);
    else return B1<OP>::shfl(v, o);
}

template <int OP, int G> __device__ __forceinline__ typename B1<OP>::P b1_group_comb(typename B1<OP>::P v) {
#pragma unroll
    for (int o = G / 2; o >= 1; o >>= 1) v = B1<OP>::comb(v, b1_shfl<OP>(v, o));
    return v;
}

// Fixed pairwise tree over the U load slots of one row.
template <int OP, int U, class A> __device__ __forceinline__ typename B1<OP>::P b1_slots(A* acc) {
#pragma unroll
    for (int w = U / 2; w >= 1; w >>= 1)
#pragma unroll
        for (int i = 0; i < w; ++i) B1<OP>::add(acc[i], acc[i + w]);
    return B1<OP>::fin(acc[0]);
}

// ------------------------------------------------------------------ lane group per row
// Warp w owns RB*(32/G) rows per step (row = base + i*(32/G) + g); lane li of a
// group reads vectors li, li+G, ... of its row -- in increasing index order, which
// IAMAX/IAMIN do not rely on (the packed key breaks ties by index).  Main loop
// unpredicated (rows past R read row 0 and are discarded), predicated tail.
template <int OP, int G, int RB, int U, bool VEC, int NT>
__global__ void __launch_bounds__(NT)
b1_group_kernel(const float* __restrict__ A, void* __restrict__ y, int64_t R, int64_t C)
{
    pdl_prologue();
    using Pol = B1<OP>;
    using E = typename std::conditional<VEC, float4, float>::type;
    using Acc = typename Pol::template Acc<VEC>;
    using P = typename Pol::P;
    constexpr int W = VEC ? 4 : 1;
    constexpr int NG = 32 / G;
    const int64_t nv = C / W;
    const E* __restrict__ Av = reinterpret_cast<const E*>(A);
    const int lane = threadIdx.x & 31;
    const int g = lane / G, li = lane % G;
    const int64_t warp = (int64_t(blockIdx.x) * NT + threadIdx.x) >> 5;
    const int64_t nwarps = (int64_t(gridDim.x) * NT) >> 5;
    const int64_t step = int64_t(RB) * NG;

    for (int64_t base = warp * step; base < R; base += nwarps * step) {
        Acc acc[RB][U];
        P outer[RB];
        int64_t rowoff[RB];
#pragma unroll
        for (int i = 0; i < RB; ++i) {
            outer[i] = Pol::ident();
#pragma unroll
            for (int u = 0; u < U; ++u) Pol::zero(acc[i][u]);
            const int64_t row = base + i * NG + g;
            rowoff[i] = (row < R ? row : 0) * nv;
        }
        int it = 0;
        int64_t j0 = li;
        for (; j0 + int64_t(G) * (U - 1) < nv; j0 += int64_t(G) * U) {
            E a[RB][U];
#pragma unroll
            for (int u = 0; u < U; ++u)
#pragma unroll
                for (int i = 0; i < RB; ++i) a[i][u] = ld_stream(Av + rowoff[i] + j0 + int64_t(G) * u);
#pragma unroll
            for (int i = 0; i < RB; ++i)
#pragma unroll
                for (int u = 0; u < U; ++u) Pol::elem(acc[i][Pol::kOneSlot ? 0 : u], a[i][u], j0 + int64_t(G) * u);
            if (Pol::kFold && ++it == (Pol::kOneSlot ? FOLD / U : FOLD)) {
                it = 0;
#pragma unroll
                for (int i = 0; i < RB; ++i) {
                    outer[i] = Pol::comb(outer[i], b1_slots<OP, U>(acc[i]));
#pragma unroll
                    for (int u = 0; u < U; ++u) Pol::zero(acc[i][u]);
                }
            }
        }
        for (; j0 < nv; j0 += G) {
#pragma unroll
            for (int i = 0; i < RB; ++i) Pol::elem(acc[i][0], ld_stream(Av + rowoff[i] + j0), j0);
        }
#pragma unroll
        for (int i = 0; i < RB; ++i) {
            P s = Pol::comb(outer[i], b1_slots<OP, U>(acc[i]));
            s = b1_group_comb<OP, G>(s);
            const int64_t row = base + i * NG + g;
            if (li == 0 && row < R) Pol::store(y, row, s, R);
        }
    }
}

// ------------------------------------------------------------------ CTA per row (+ splits)
template <int OP, int NT> __device__ __forceinline__ typename B1<OP>::P
b1_cta_comb(typename B1<OP>::P v, typename B1<OP>::P* red) {
    using P = typename B1<OP>::P;
    constexpr int NW = NT / 32;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    v = b1_group_comb<OP, 32>(v);
    if (NW == 1) return v;
    if (lane == 0) red[warp] = v;
    __syncthreads();
    P t = B1<OP>::ident();
    if (warp == 0) {                           // butterfly over the NW warp totals
        t = lane < NW ? red[lane] : B1<OP>::ident();
        t = b1_group_comb<OP, 32>(t);
    }
    return t;                                  // valid in thread 0
}

template <int OP, int NT, int U, bool VEC>
__global__ void __launch_bounds__(NT)
b1_cta_kernel(const float* __restrict__ A, void* __restrict__ y, int64_t R, int64_t C, int S,
              typename B1<OP>::P* __restrict__ ws_part, unsigned int* __restrict__ ws_cnt)
{
    pdl_prologue();
    using Pol = B1<OP>;
    using E = typename std::conditional<VEC, float4, float>::type;
    using Acc = typename Pol::template Acc<VEC>;
    using P = typename Pol::P;
    constexpr int W = VEC ? 4 : 1;
    constexpr int64_t BV = int64_t(NT) * U;
    __shared__ P red[NT / 32];
    __shared__ unsigned int flag;
    const int64_t nv = C / W;
    const E* __restrict__ Av = reinterpret_cast<const E*>(A);
    const int tid = threadIdx.x;
    const int64_t nblk = R * S;

    for (int64_t blk = blockIdx.x; blk < nblk; blk += gridDim.x) {
        const int64_t row = blk / S;
        const int s = int(blk - row * S);
        const E* __restrict__ Ar = Av + row * nv;
        // the S CTAs of a row interleave in steps of BV vectors (one moving window)
        const int64_t stride = int64_t(S) * BV;
        Acc acc[U];
#pragma unroll
        for (int u = 0; u < U; ++u) Pol::zero(acc[u]);
        P outer = Pol::ident();
        int it = 0;
        int64_t b = int64_t(s) * BV;
        for (; b + tid + int64_t(NT) * (U - 1) < nv; b += stride) {
            E a[U];
#pragma unroll
            for (int u = 0; u < U; ++u) a[u] = ld_stream(Ar + b + tid + int64_t(NT) * u);
#pragma unroll
            for (int u = 0; u < U; ++u) Pol::elem(acc[Pol::kOneSlot ? 0 : u], a[u], b + tid + int64_t(NT) * u);
            if (Pol::kFold && ++it == (Pol::kOneSlot ? FOLD / U : FOLD)) {
                it = 0;
                outer = Pol::comb(outer, b1_slots<OP, U>(acc));
#pragma unroll
                for (int u = 0; u < U; ++u) Pol::zero(acc[u]);
            }
        }
        const int64_t tail_end = min(nv, b + BV);
        for (int64_t v = b + tid; v < tail_end; v += NT) Pol::elem(acc[0], ld_stream(Ar + v), v);
        P val = b1_cta_comb<OP, NT>(Pol::comb(outer, b1_slots<OP, U>(acc)), red);

        if (S == 1) {
            if (tid == 0) Pol::store(y, row, val, R);
        } else {
            if (tid == 0) ws_part[row * S + s] = val;
            if (ticket_is_last(ws_cnt + row, unsigned(S), &flag)) {
                __syncthreads();               // red[] reuse
                P m = Pol::ident();
                for (int k = tid; k < S; k += NT) m = Pol::comb(m, ld_partial_any(ws_part + row * S + k));
                m = b1_cta_comb<OP, NT>(m, red);
                if (tid == 0) Pol::store(y, row, m, R);
            }
        }
        __syncthreads();
    }
}

}  // namespace adaptic
