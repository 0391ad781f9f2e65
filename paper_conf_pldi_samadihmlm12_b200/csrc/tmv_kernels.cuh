// tmv_kernels.cuh -- strided-reduction variants (TMV on the restructured layout), sm_100a.
//
// B is row-major C x R (B = A^T, the paper's memory-restructured layout, Fig. 3b,
// "each pop access in all threads accesses consecutive elements of one
// row").  y[r] = sum_c B[c*R + r] * x[c].
//
// tmv_kernel<LR, U>: a CTA of NT = 256 threads owns a tile of LR output vectors
// (4*LR outputs when vectorised) and one of S contiguous c-ranges.  Thread
// (lr, lc) = (tid % LR, tid / LR) accumulates outputs of vector lr over
// c = c0 + lc, c0 + lc + LC, ... (LC = NT / LR), U loads in flight.  A warp's
// load therefore covers 32/LR consecutive rows of B x LR*16 bytes: contiguous
// for LR < 32 (the whole output vector for tiny R), 512 B for LR >= 32.
//   TMV_COL     = LR 256 (LC = 1), S = 1: the paper's kernel 5 -- "each thread is
//                 responsible for computing the dot product of a single row"
//                 (P:1248), four rows per thread, on the restructured layout.
//   TMV_SPLITK  = 2-D tiles with S >= 1: the lc-combine is the paper's
//                 shared-memory phase (Fig. 8), the s-combine its merge kernel
//                 (P:480), done by the last CTA of the tile (ticket, fixed order).
//   TMV_REGTILE = one tile holds every output (R <= 4*LR); c split S ways.
#pragma once

#include "common.cuh"
#include "mv_kernels.cuh"

namespace adaptic {

__device__ __forceinline__ void esmac(float& acc, float a, float s) { acc = mac(a, s, acc); }
__device__ __forceinline__ void esmac(uint32_t& acc, uint32_t a, uint32_t s) { acc = mac(a, s, acc); }
__device__ __forceinline__ void esmac(float4& acc, const float4& a, float s) { vmacs(acc, a, s); }
__device__ __forceinline__ void esmac(uint4& acc, const uint4& a, uint32_t s) { vmacs(acc, a, s); }

template <int STRIDE> __device__ __forceinline__ float4 strided_sum_e(float4 v) {
    v.x = strided_sum<STRIDE>(v.x); v.y = strided_sum<STRIDE>(v.y);
    v.z = strided_sum<STRIDE>(v.z); v.w = strided_sum<STRIDE>(v.w); return v;
}
template <int STRIDE> __device__ __forceinline__ uint4 strided_sum_e(uint4 v) {
    v.x = strided_sum<STRIDE>(v.x); v.y = strided_sum<STRIDE>(v.y);
    v.z = strided_sum<STRIDE>(v.z); v.w = strided_sum<STRIDE>(v.w); return v;
}
template <int STRIDE> __device__ __forceinline__ float strided_sum_e(float v) { return strided_sum<STRIDE>(v); }
template <int STRIDE> __device__ __forceinline__ uint32_t strided_sum_e(uint32_t v) { return strided_sum<STRIDE>(v); }

// Combine the LC partials of each lr (fixed tree); result valid for tid < LR.
// red must hold NT elements.  Contains __syncthreads (call uniformly).
template <int NT, int LR, class E>
__device__ __forceinline__ E lc_combine(E v, E* red) {
    constexpr int LC = NT / LR;
    if (LC == 1) return v;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (LR < 32) {
        v = strided_sum_e<(LR < 32 ? LR : 16)>(v);          // lanes with equal lr
        constexpr int NW = NT / 32;
        if (lane < LR) red[warp * LR + lane] = v;
        __syncthreads();
        E t = zero_of<E>();
        if (tid < LR) {
#pragma unroll
            for (int w = 0; w < NW; ++w) t = eadd(t, red[w * LR + tid]);
        }
        return t;
    } else {
        red[tid] = v;                                        // red[lc*LR + lr]
        __syncthreads();
        E t = zero_of<E>();
        if (tid < LR) {
#pragma unroll
            for (int k = 0; k < LC; ++k) t = eadd(t, red[k * LR + tid]);
        }
        return t;
    }
}

// Sum of partials p[k*stride] for k = k0, k0+STEP, ... < S: two independent
// loads in flight per round into two accumulators (kept register-light: the
// kernel's register count -- and so its occupancy -- is set by its largest
// section), then a fixed combine, so the result does not depend on timing.
template <int STEP, class E>
__device__ __forceinline__ E merge_partials(const E* p, int64_t stride, int k0, int S) {
    E m0 = zero_of<E>(), m1 = zero_of<E>();
    int k = k0;
    for (; k + STEP < S; k += 2 * STEP) {
        const E t0 = ld_partial(p + int64_t(k) * stride);
        const E t1 = ld_partial(p + int64_t(k + STEP) * stride);
        m0 = eadd(m0, t0);
        m1 = eadd(m1, t1);
    }
    if (k < S) m0 = eadd(m0, ld_partial(p + int64_t(k) * stride));
    return eadd(m0, m1);
}

template <class T, int LR, int U, bool VEC, int NT>
__global__ void __launch_bounds__(NT, NT <= 256 ? (U <= 2 ? 6 : 4) : 1)
tmv_kernel(const T* __restrict__ B, const T* __restrict__ X, T* __restrict__ y,
           int64_t R, int64_t C, int S, T* __restrict__ ws_part, unsigned int* __restrict__ ws_cnt)
{
    pdl_prologue();
    using E = typename ElemOf<T, VEC>::type;
    constexpr int W = ElemOf<T, VEC>::W;
    constexpr int LC = NT / LR;
    __shared__ E red[LC > 1 ? NT : 1];
    __shared__ unsigned int flag;
    const int64_t rv = R / W;                         // vectors per B row
    const int64_t ntiles = (rv + LR - 1) / LR;
    const int64_t chunk = (C + S - 1) / S;
    const E* __restrict__ Bv = reinterpret_cast<const E*>(B);
    E* __restrict__ yv = reinterpret_cast<E*>(y);
    E* __restrict__ pv = reinterpret_cast<E*>(ws_part);
    const int tid = threadIdx.x;
    const int lr = tid % LR, lc = tid / LR;
    const int64_t nblk = ntiles * S;

    for (int64_t blk = blockIdx.x; blk < nblk; blk += gridDim.x) {
        const int64_t tile = blk % ntiles;
        const int s = int(blk / ntiles);
        const int64_t r4 = tile * LR + lr;
        const bool rok = r4 < rv;
        const int64_t c0 = int64_t(s) * chunk;
        const int64_t c1 = min(C, c0 + chunk);

        E acc[U];
#pragma unroll
        for (int u = 0; u < U; ++u) acc[u] = zero_of<E>();
        E outer = zero_of<E>();
        int it = 0;
        const E* __restrict__ Bc = Bv + (rok ? r4 : 0);      // ragged tile: read column 0, discard
        int64_t c = c0 + lc;
        for (; c + int64_t(LC) * (U - 1) < c1; c += int64_t(LC) * U) {
            E a[U];
            T xs[U];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const int64_t cc = c + int64_t(LC) * u;
                a[u] = ld_stream(Bc + cc * rv);
                xs[u] = ld_x(X + cc);
            }
#pragma unroll
            for (int u = 0; u < U; ++u) esmac(acc[u], a[u], xs[u]);
            if (++it == FOLD) {            // second-level accumulation
                it = 0;
                outer = eadd(outer, tree_sum<U>(acc));
#pragma unroll
                for (int u = 0; u < U; ++u) acc[u] = zero_of<E>();
            }
        }
        for (; c < c1; c += LC)            // tail: fewer than U rows of B left for this thread
            esmac(acc[0], ld_stream(Bc + c * rv), ld_x(X + c));
        E tot = eadd(outer, tree_sum<U>(acc));
        tot = lc_combine<NT, LR>(tot, red);

        if (S == 1) {
            if (tid < LR && rok) yv[r4] = tot;
        } else {
            if (tid < LR && rok) pv[int64_t(s) * rv + r4] = tot;
            if (ticket_is_last(ws_cnt + tile, unsigned(S), &flag)) {
                E m = zero_of<E>();
                if (rok)
                    m = merge_partials<LC>(pv + r4, rv, lc, S);
                __syncthreads();  // red[] reuse
                m = lc_combine<NT, LR>(m, red);
                if (tid < LR && rok) yv[r4] = m;
            }
        }
        __syncthreads();  // red[] / flag reuse
    }
}

}  // namespace adaptic
