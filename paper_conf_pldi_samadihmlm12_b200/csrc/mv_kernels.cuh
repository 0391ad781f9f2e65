// mv_kernels.cuh -- contiguous-reduction variants (MV and DOT), sm_100a.
//
//   mv_group_kernel  : MV_SUBWARP (G = 1..16 lanes per row) and MV_WPR (G = 32).
//                      The paper's kernels 4 and 3: one output per lane
//                      group; several rows per warp/CTA is the paper's horizontal
//                      thread integration.
//   mv_cta_kernel    : MV_CPR (S = 1; kernel 2, "each block is responsible for
//                      one row", Fig. 7b) and MV_SPLIT (S > 1; kernel 1,
//                      the two-kernel reduction of P:480 / Fig. 7c with the merge
//                      kernel folded into the same launch by a ticket).
//
// Hot loop (the paper's Fig. 8 global phase): each
// thread keeps RB*U independent 128-bit loads in flight and one 4-wide
// accumulator per load slot; every FOLD iterations the slots are folded into a
// second-level accumulator, so a serial chain is at most FOLD + #folds terms
// (the planner checks the resulting error bound).
#pragma once

#include "common.cuh"
#include "launch.h"

namespace adaptic {

template <class T, bool VEC> struct ElemOf;
template <class T> struct ElemOf<T, true> { using type = vec4_t<T>; static constexpr int W = 4; };
template <class T> struct ElemOf<T, false> { using type = T; static constexpr int W = 1; };

template <class V> __device__ __forceinline__ V zero_of();
template <> __device__ __forceinline__ float zero_of<float>() { return 0.f; }
template <> __device__ __forceinline__ uint32_t zero_of<uint32_t>() { return 0u; }
template <> __device__ __forceinline__ float4 zero_of<float4>() { return make_float4(0.f, 0.f, 0.f, 0.f); }
template <> __device__ __forceinline__ uint4 zero_of<uint4>() { return make_uint4(0u, 0u, 0u, 0u); }

__device__ __forceinline__ void emac(float& acc, float a, float b) { acc = mac(a, b, acc); }
__device__ __forceinline__ void emac(uint32_t& acc, uint32_t a, uint32_t b) { acc = mac(a, b, acc); }
__device__ __forceinline__ void emac(float4& acc, const float4& a, const float4& b) { vmac(acc, a, b); }
__device__ __forceinline__ void emac(uint4& acc, const uint4& a, const uint4& b) { vmac(acc, a, b); }

__device__ __forceinline__ float esum(float a) { return a; }
__device__ __forceinline__ uint32_t esum(uint32_t a) { return a; }
__device__ __forceinline__ float esum(const float4& a) { return vsum(a); }
__device__ __forceinline__ uint32_t esum(const uint4& a) { return vsum(a); }

__device__ __forceinline__ float eadd(float a, float b) { return a + b; }
__device__ __forceinline__ uint32_t eadd(uint32_t a, uint32_t b) { return a + b; }
__device__ __forceinline__ float4 eadd(float4 a, const float4& b) { return vadd(a, b); }
__device__ __forceinline__ uint4 eadd(uint4 a, const uint4& b) { return vadd(a, b); }

// Fixed pairwise tree over N accumulators (N a power of two).
template <int N, class V> __device__ __forceinline__ V tree_sum(V* a) {
#pragma unroll
    for (int w = N / 2; w >= 1; w >>= 1)
#pragma unroll
        for (int i = 0; i < w; ++i) a[i] = eadd(a[i], a[i + w]);
    return a[0];
}

// ------------------------------------------------------------------ x operand modes
// XM_LDG : x read through the read-only path (L1/L2 hits after the first CTA)
// XM_SMEM: x staged ONCE per CTA into shared memory by the TMA bulk-copy engine
//          (the north_star's "TMA/shared-memory staging of x"); every later x
//          read is a conflict-free LDS.  Needs C*4 bytes of dynamic smem.
// XM_ROW : DOT -- the second operand is per row (streamed like A)
constexpr int XM_LDG = 0, XM_SMEM = 1, XM_ROW = 2;

template <int XM, class E> __device__ __forceinline__ E ld_xm(const E* p) {
    if constexpr (XM == XM_SMEM) return *p;
    else return ld_x(p);
}

template <class T, bool VEC, int XM, int NT>
__device__ __forceinline__ const typename ElemOf<T, VEC>::type* stage_x(const T* X, int64_t nv) {
    using E = typename ElemOf<T, VEC>::type;
    if constexpr (XM != XM_SMEM) {
        return reinterpret_cast<const E*>(X);
    } else {
        extern __shared__ __align__(128) unsigned char dyn_smem[];
        __shared__ __align__(8) uint64_t xbar;
        E* xs = reinterpret_cast<E*>(dyn_smem);
        if (VEC) {
            stage_to_smem(xs, X, uint32_t(nv * sizeof(E)), &xbar);     // TMA bulk copy
        } else {
            for (int64_t v = threadIdx.x; v < nv; v += NT) xs[v] = reinterpret_cast<const E*>(X)[v];
            __syncthreads();
        }
        return xs;
    }
}

// ------------------------------------------------------------------ MV_SUBWARP / MV_WPR
// Lane group of G lanes per row.  Warp w owns RB*(32/G) consecutive rows per
// step: row = base + i*(32/G) + g, so the i-th load of a warp covers 32/G
// consecutive rows (fully coalesced when C/4 == G).  Within a row lane li reads
// vectors li, li+G, li+2G, ...  The main loop carries no predicates: rows past
// R read row 0 (valid memory, result discarded) and only the last partial
// stride of a row takes the predicated tail -- so ptxas issues all RB*U
// 128-bit loads of a step before the first FMA.
template <class T, int G, int RB, int U, bool VEC, int XM, int NT>
__global__ void __launch_bounds__(NT)
mv_group_kernel(const T* __restrict__ A, const T* __restrict__ X, T* __restrict__ y,
                int64_t R, int64_t C)
{
    pdl_prologue();
    using E = typename ElemOf<T, VEC>::type;
    constexpr int W = ElemOf<T, VEC>::W;
    constexpr int NG = 32 / G;
    constexpr bool PERROWX = (XM == XM_ROW);
    const int64_t nv = C / W;
    const E* __restrict__ Av = reinterpret_cast<const E*>(A);
    const E* __restrict__ Xv = stage_x<T, VEC, XM, NT>(X, nv);
    const int lane = threadIdx.x & 31;
    const int g = lane / G, li = lane % G;
    const int64_t warp = (int64_t(blockIdx.x) * NT + threadIdx.x) >> 5;
    const int64_t nwarps = (int64_t(gridDim.x) * NT) >> 5;
    const int64_t step = int64_t(RB) * NG;

    for (int64_t base = warp * step; base < R; base += nwarps * step) {
        E acc[RB][U];
#pragma unroll
        for (int i = 0; i < RB; ++i)
#pragma unroll
            for (int u = 0; u < U; ++u) acc[i][u] = zero_of<E>();

        int64_t rowoff[RB];
#pragma unroll
        for (int i = 0; i < RB; ++i) {
            const int64_t row = base + i * NG + g;
            rowoff[i] = (row < R ? row : 0) * nv;
        }

        T outer[RB];
#pragma unroll
        for (int i = 0; i < RB; ++i) outer[i] = T(0);
        int it = 0;
        int64_t j0 = li;
        for (; j0 + int64_t(G) * (U - 1) < nv; j0 += int64_t(G) * U) {
            E a[RB][U];
            E b[PERROWX ? RB : 1][U];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const int64_t v = j0 + int64_t(G) * u;
                if (!PERROWX) b[0][u] = ld_xm<XM>(Xv + v);
#pragma unroll
                for (int i = 0; i < RB; ++i) {
                    a[i][u] = ld_stream(Av + rowoff[i] + v);
                    if (PERROWX) b[PERROWX ? i : 0][u] = ld_stream(Xv + rowoff[i] + v);
                }
            }
#pragma unroll
            for (int i = 0; i < RB; ++i)
#pragma unroll
                for (int u = 0; u < U; ++u) emac(acc[i][u], a[i][u], b[PERROWX ? i : 0][u]);
            if (++it == FOLD) {            // second-level accumulation (chain <= FOLD + folds)
                it = 0;
#pragma unroll
                for (int i = 0; i < RB; ++i) {
                    outer[i] += esum(tree_sum<U>(acc[i]));
#pragma unroll
                    for (int u = 0; u < U; ++u) acc[i][u] = zero_of<E>();
                }
            }
        }
        for (; j0 < nv; j0 += G) {         // tail: fewer than U vectors left for this lane
#pragma unroll
            for (int i = 0; i < RB; ++i) {
                const E a = ld_stream(Av + rowoff[i] + j0);
                const E b = PERROWX ? ld_stream(Xv + rowoff[i] + j0) : ld_xm<XM>(Xv + j0);
                emac(acc[i][0], a, b);
            }
        }

#pragma unroll
        for (int i = 0; i < RB; ++i) {
            T s = outer[i] + esum(tree_sum<U>(acc[i]));
            s = group_sum<G>(s);
            const int64_t row = base + i * NG + g;
            if (li == 0 && row < R) y[row] = s;
        }
    }
}

// ------------------------------------------------------------------ MV_CPR / MV_SPLIT
// One CTA per (group of RB consecutive rows, split).  The rows' vector range is
// cut into S contiguous chunks; thread t reads vectors t, t+NT, ... of its chunk
// for all RB rows at once (RB*U loads in flight, unpredicated main loop +
// predicated tail), so each x vector is fetched once per RB rows -- without
// that, x (C*4 bytes) is re-read from L2 for every row and doubles the
// on-chip traffic of long rows.  RB > 1 is the paper's horizontal thread
// integration applied to the block-per-row kernel.
// S == 1: the CTA writes y for its rows.  S > 1: it writes partials
// ws_part[row*S + s]; the last CTA of the row group (ticket) sums the S partials
// of each row in a fixed order and writes y.
//
// Block combine of RB values: warp butterfly, one smem stage, fixed order.
template <int NT, int RB, class T>
__device__ __forceinline__ void cta_sum_rows(T (&v)[RB], T* red /* RB*(NT/32) */) {
    constexpr int NW = NT / 32;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
#pragma unroll
    for (int i = 0; i < RB; ++i) v[i] = group_sum<32>(v[i]);
    if (lane == 0) {
#pragma unroll
        for (int i = 0; i < RB; ++i) red[i * NW + warp] = v[i];
    }
    __syncthreads();
    if (threadIdx.x < RB) {
        T t = T(0);
#pragma unroll
        for (int w = 0; w < NW; ++w) t += red[threadIdx.x * NW + w];
        v[0] = t;                         // thread i < RB holds row i's total in v[0]
    }
}

template <class T, int NT, int RB, int U, bool VEC, int XM, bool PIPE>
__global__ void __launch_bounds__(NT)
mv_cta_kernel(const T* __restrict__ A, const T* __restrict__ X, T* __restrict__ y,
              int64_t R, int64_t C, int S, int ilv, T* __restrict__ ws_part, unsigned int* __restrict__ ws_cnt)
{
    pdl_prologue();
    using E = typename ElemOf<T, VEC>::type;
    constexpr int W = ElemOf<T, VEC>::W;
    constexpr bool PERROWX = (XM == XM_ROW);
    constexpr int64_t BV = int64_t(NT) * U;       // vectors per CTA step
    __shared__ T red[RB * (NT / 32)];
    __shared__ unsigned int flag;
    const int64_t nv = C / W;
    const int64_t chunk = (nv + S - 1) / S;
    const E* __restrict__ Av = reinterpret_cast<const E*>(A);
    const E* __restrict__ Xv = stage_x<T, VEC, XM, NT>(X, nv);   // XM_SMEM only with S == 1
    const int tid = threadIdx.x;
    const int64_t ngroups = (R + RB - 1) / RB;
    const int64_t nblk = ngroups * S;

    for (int64_t blk = blockIdx.x; blk < nblk; blk += gridDim.x) {
        const int64_t grp = blk / S;
        const int s = int(blk - grp * S);
        const int64_t row0 = grp * RB;
        // split s covers either one contiguous chunk of the row (ilv == 0) or every
        // S-th step of BV vectors (ilv == 1: the S CTAs of a row sweep it together,
        // which keeps the in-flight addresses in one window, like a linear stream)
        const int64_t start = ilv ? int64_t(s) * BV : int64_t(s) * chunk;
        const int64_t stride = ilv ? int64_t(S) * BV : BV;
        const int64_t end = ilv ? nv : min(nv, start + chunk);
        int64_t off[RB];                   // rows past R read row 0 (discarded)
#pragma unroll
        for (int i = 0; i < RB; ++i) off[i] = (row0 + i < R ? row0 + i : 0) * nv;

        E acc[RB][U];
#pragma unroll
        for (int i = 0; i < RB; ++i)
#pragma unroll
            for (int u = 0; u < U; ++u) acc[i][u] = zero_of<E>();
        T outer[RB];
#pragma unroll
        for (int i = 0; i < RB; ++i) outer[i] = T(0);
        int it = 0;
        int64_t base = start;
        // PIPE: register double buffering -- the loads of step k+1 are issued before
        // the FMAs of step k, so RB*U loads stay in flight whatever order ptxas
        // chooses inside a step (measured: it rescues instances where ptxas
        // interleaved loads and FMAs, and costs occupancy elsewhere; the selector
        // table records which one wins per shape).
        E a[RB][U], b[PERROWX ? RB : 1][U];
        auto load_step = [&](int64_t bs, E (&aa)[RB][U], E (&bb)[PERROWX ? RB : 1][U]) {
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const int64_t vv = bs + tid + int64_t(NT) * u;
                if (!PERROWX) bb[0][u] = ld_xm<XM>(Xv + vv);
#pragma unroll
                for (int i = 0; i < RB; ++i) {
                    aa[i][u] = ld_stream(Av + off[i] + vv);
                    if (PERROWX) bb[PERROWX ? i : 0][u] = ld_stream(Xv + off[i] + vv);
                }
            }
        };
        bool have = base + tid + int64_t(NT) * (U - 1) < end;
        if constexpr (!PIPE) {
            // single buffer (1024-thread CTAs have 64 registers/thread: no room for two)
            for (; have; base += stride, have = base + tid + int64_t(NT) * (U - 1) < end) {
                load_step(base, a, b);
#pragma unroll
                for (int i = 0; i < RB; ++i)
#pragma unroll
                    for (int u = 0; u < U; ++u) emac(acc[i][u], a[i][u], b[PERROWX ? i : 0][u]);
                if (++it == FOLD) {
                    it = 0;
#pragma unroll
                    for (int i = 0; i < RB; ++i) {
                        outer[i] += esum(tree_sum<U>(acc[i]));
#pragma unroll
                        for (int u = 0; u < U; ++u) acc[i][u] = zero_of<E>();
                    }
                }
            }
        }
        if (have) load_step(base, a, b);
        while (have) {
            const int64_t nbase = base + stride;
            const bool more = nbase + tid + int64_t(NT) * (U - 1) < end;
            E an[RB][U], bn[PERROWX ? RB : 1][U];
            if (more) load_step(nbase, an, bn);
#pragma unroll
            for (int i = 0; i < RB; ++i)
#pragma unroll
                for (int u = 0; u < U; ++u) emac(acc[i][u], a[i][u], b[PERROWX ? i : 0][u]);
            if (++it == FOLD) {
                it = 0;
#pragma unroll
                for (int i = 0; i < RB; ++i) {
                    outer[i] += esum(tree_sum<U>(acc[i]));
#pragma unroll
                    for (int u = 0; u < U; ++u) acc[i][u] = zero_of<E>();
                }
            }
            base = nbase;
            have = more;
            if (more) {
#pragma unroll
                for (int u = 0; u < U; ++u) {
#pragma unroll
                    for (int i = 0; i < RB; ++i) a[i][u] = an[i][u];
#pragma unroll
                    for (int i = 0; i < (PERROWX ? RB : 1); ++i) b[i][u] = bn[i][u];
                }
            }
        }
        const int64_t tail_end = min(end, base + BV);
        for (int64_t v = base + tid; v < tail_end; v += NT) {   // tail: < U vectors left for this thread
            const E bx = PERROWX ? zero_of<E>() : ld_xm<XM>(Xv + v);
#pragma unroll
            for (int i = 0; i < RB; ++i)
                emac(acc[i][0], ld_stream(Av + off[i] + v), PERROWX ? ld_stream(Xv + off[i] + v) : bx);
        }
        T val[RB];
#pragma unroll
        for (int i = 0; i < RB; ++i) val[i] = outer[i] + esum(tree_sum<U>(acc[i]));
        cta_sum_rows<NT, RB>(val, red);

        if (S == 1) {
            if (tid < RB && row0 + tid < R) y[row0 + tid] = val[0];
        } else {
            if (tid < RB && row0 + tid < R) ws_part[(row0 + tid) * S + s] = val[0];
            if (ticket_is_last(ws_cnt + grp, unsigned(S), &flag)) {
                __syncthreads();  // red[] reuse
                T m[RB];
#pragma unroll
                for (int i = 0; i < RB; ++i) {
                    m[i] = T(0);
                    if (row0 + i < R)
                        for (int k = tid; k < S; k += NT) m[i] += ld_partial(ws_part + (row0 + i) * S + k);
                }
                cta_sum_rows<NT, RB>(m, red);
                if (tid < RB && row0 + tid < R) y[row0 + tid] = m[0];
            }
        }
        __syncthreads();  // red[] / flag reuse in the next grid-stride step
    }
}

}  // namespace adaptic
