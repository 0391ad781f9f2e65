// mmv_kernels.cuh -- multi-vector MV / TMV: Y = A [x_0 .. x_{K-1}] in ONE pass over A, sm_100a.
//
// The paper's horizontal actor integration: "In streaming languages, we
// use a duplicate splitter to allow different actors to work on the same data ...
// instead of launching one kernel for each actor, one kernel is launched to do the
// job of all the actors working on the same data", so off-chip accesses "only
// happen once".  K matrix-vector actors that read the same matrix become one
// kernel: every 128-bit load of A feeds K FMAs (K accumulators per load slot),
// so the bytes per result drop by ~K and the arithmetic intensity rises from
// 0.5 to K/2 flop/byte -- still CUDA-core work for K <= 8 (<= 4 flop/B, about
// 28 TFLOP/s of fp32 at HBM speed, well under the FP32 peak; no tensor cores).
//
// Layouts: X is K x C row-major (vector j at X + j*C), Y is K x R row-major.
//   mmv_group_kernel<K,G,RB,U,VEC>  rows of <= G*U vectors, x held in registers
//                                (MV_SUBWARP / MV_WPR shapes)
//   mmv_cta_kernel<K,NT,U,VEC>   CTA per RB = 8/K rows or S interleaved CTAs per row
//                                group with the same-launch ticket merge (MV_CPR / MV_SPLIT)
//   tmmv_kernel<K,LR,U,VEC>      TMV tiles of LR output vectors x c-lanes, S c-ranges
//                                (TMV_COL / TMV_SPLITK / TMV_REGTILE)
// One accumulator per (vector, row) fed by U loads per step, so the fp32 chain
// folds every FOLD/U steps (the planner's bound uses the same count); the
// short-row kernel's chain is U terms.
#pragma once

#include "mv_kernels.cuh"
#include "tmv_kernels.cuh"

namespace adaptic {

// ------------------------------------------------------------------ MV, short rows: x in registers
// Rows of at most G*U vectors (C <= 4*G*U): lane li of a group always touches the
// same vectors li + G*u of every row, so it loads its K x U x-vectors ONCE into
// registers and then streams RB rows per step with no x traffic at all (re-reading
// x from L1 would cost K times the matrix bytes).
template <int K, int G, int RB, int U, bool VEC, int NT>
__global__ void __launch_bounds__(NT)
mmv_group_kernel(const float* __restrict__ A, const float* __restrict__ X, float* __restrict__ Y,
                 int64_t R, int64_t C)
{
    pdl_prologue();
    using E = typename ElemOf<float, VEC>::type;
    constexpr int W = VEC ? 4 : 1;
    constexpr int NG = 32 / G;
    const int64_t nv = C / W;                          // <= G*U (planner)
    const E* __restrict__ Av = reinterpret_cast<const E*>(A);
    const E* __restrict__ Xv = reinterpret_cast<const E*>(X);
    const int lane = threadIdx.x & 31;
    const int g = lane / G, li = lane % G;
    const int64_t warp = (int64_t(blockIdx.x) * NT + threadIdx.x) >> 5;
    const int64_t nwarps = (int64_t(gridDim.x) * NT) >> 5;
    const int64_t step = int64_t(RB) * NG;

    E xr[K][U];
    bool ok[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
        const int64_t v = li + int64_t(G) * u;
        ok[u] = v < nv;
#pragma unroll
        for (int j = 0; j < K; ++j) xr[j][u] = ok[u] ? ld_x(Xv + j * nv + v) : zero_of<E>();
    }
    for (int64_t base = warp * step; base < R; base += nwarps * step) {
        E a[RB][U];
#pragma unroll
        for (int i = 0; i < RB; ++i) {
            const int64_t row = base + i * NG + g;
            const E* Ar = Av + (row < R ? row : 0) * nv;
#pragma unroll
            for (int u = 0; u < U; ++u) a[i][u] = ok[u] ? ld_stream(Ar + li + int64_t(G) * u) : zero_of<E>();
        }
#pragma unroll
        for (int i = 0; i < RB; ++i) {
            const int64_t row = base + i * NG + g;
#pragma unroll
            for (int j = 0; j < K; ++j) {
                E acc = zero_of<E>();
#pragma unroll
                for (int u = 0; u < U; ++u) emac(acc, a[i][u], xr[j][u]);
                const float sj = group_sum<G>(esum(acc));
                if (li == 0 && row < R) Y[j * R + row] = sj;
            }
        }
    }
}

// ------------------------------------------------------------------ MV, CTA per RB rows (+ splits)
// RB = 8 / K rows per CTA step share every x load (x traffic K/RB times the matrix
// bytes instead of K); S CTAs per row group interleave in steps of NT*U vectors.
// XS: the K x-vectors (K*C*4 bytes, small) are staged once per CTA in shared memory
// (TMA bulk copy on the 128-bit path), so x reads leave L1/L2 alone.
template <int K, int NT, int U, bool VEC, bool XS = false>
__global__ void __launch_bounds__(NT)
mmv_cta_kernel(const float* __restrict__ A, const float* __restrict__ X, float* __restrict__ Y,
               int64_t R, int64_t C, int S, float* __restrict__ ws_part, unsigned int* __restrict__ ws_cnt)
{
    pdl_prologue();
    if constexpr (XS) {
        extern __shared__ __align__(128) unsigned char dyn_smem[];
        __shared__ __align__(8) uint64_t xbar;
        float* xs = reinterpret_cast<float*>(dyn_smem);
        if (VEC) stage_to_smem(xs, X, uint32_t(K * C * 4), &xbar);
        else {
            for (int64_t i = threadIdx.x; i < K * C; i += NT) xs[i] = X[i];
            __syncthreads();
        }
        X = xs;
    }
    using E = typename ElemOf<float, VEC>::type;
    constexpr int W = VEC ? 4 : 1;
    constexpr int RB = (8 / K) > 0 ? 8 / K : 1;
    constexpr int KR = K * RB;
    constexpr int64_t BV = int64_t(NT) * U;
    __shared__ float red[KR * (NT / 32)];
    __shared__ unsigned int flag;
    const int64_t nv = C / W;
    const E* __restrict__ Av = reinterpret_cast<const E*>(A);
    const E* __restrict__ Xv = reinterpret_cast<const E*>(X);
    const int tid = threadIdx.x;
    const int64_t ngroups = (R + RB - 1) / RB;
    const int64_t nblk = ngroups * S;

    for (int64_t blk = blockIdx.x; blk < nblk; blk += gridDim.x) {
        const int64_t grp = blk / S;
        const int s = int(blk - grp * S);
        const int64_t row0 = grp * RB;
        int64_t off[RB];
#pragma unroll
        for (int i = 0; i < RB; ++i) off[i] = (row0 + i < R ? row0 + i : 0) * nv;
        const int64_t stride = int64_t(S) * BV;
        E acc[RB][K];
        float outer[RB][K];
#pragma unroll
        for (int i = 0; i < RB; ++i)
#pragma unroll
            for (int j = 0; j < K; ++j) { acc[i][j] = zero_of<E>(); outer[i][j] = 0.f; }
        int it = 0;
        int64_t b = int64_t(s) * BV;
        for (; b + tid + int64_t(NT) * (U - 1) < nv; b += stride) {
            E a[RB][U];
#pragma unroll
            for (int u = 0; u < U; ++u)
#pragma unroll
                for (int i = 0; i < RB; ++i) a[i][u] = ld_stream(Av + off[i] + b + tid + int64_t(NT) * u);
#pragma unroll
            for (int u = 0; u < U; ++u)
#pragma unroll
                for (int j = 0; j < K; ++j) {
                    const E xv = XS ? Xv[j * nv + b + tid + int64_t(NT) * u] : ld_x(Xv + j * nv + b + tid + int64_t(NT) * u);
#pragma unroll
                    for (int i = 0; i < RB; ++i) emac(acc[i][j], a[i][u], xv);
                }
            if (++it == FOLD / U) {
                it = 0;
#pragma unroll
                for (int i = 0; i < RB; ++i)
#pragma unroll
                    for (int j = 0; j < K; ++j) { outer[i][j] += esum(acc[i][j]); acc[i][j] = zero_of<E>(); }
            }
        }
        const int64_t tail_end = min(nv, b + BV);
        for (int64_t v = b + tid; v < tail_end; v += NT) {
            E a[RB];
#pragma unroll
            for (int i = 0; i < RB; ++i) a[i] = ld_stream(Av + off[i] + v);
#pragma unroll
            for (int j = 0; j < K; ++j) {
                const E xv = XS ? Xv[j * nv + v] : ld_x(Xv + j * nv + v);
#pragma unroll
                for (int i = 0; i < RB; ++i) emac(acc[i][j], a[i], xv);
            }
        }
        float val[KR];                                   // index i*K + j
#pragma unroll
        for (int i = 0; i < RB; ++i)
#pragma unroll
            for (int j = 0; j < K; ++j) val[i * K + j] = outer[i][j] + esum(acc[i][j]);
        cta_sum_rows<NT, KR>(val, red);                  // thread t < KR holds (i, j) = (t / K, t % K)

        const int ti = tid / K, tj = tid % K;
        const bool mine = tid < KR && row0 + ti < R;
        if (S == 1) {
            if (mine) Y[tj * R + row0 + ti] = val[0];
        } else {
            if (mine) ws_part[((row0 + ti) * K + tj) * S + s] = val[0];
            if (ticket_is_last(ws_cnt + grp, unsigned(S), &flag)) {
                __syncthreads();
                float m[KR];
#pragma unroll
                for (int q = 0; q < KR; ++q) {
                    m[q] = 0.f;
                    if (row0 + q / K < R)
                        for (int k = tid; k < S; k += NT) m[q] += ld_partial(ws_part + ((row0 + q / K) * K + q % K) * S + k);
                }
                cta_sum_rows<NT, KR>(m, red);
                if (mine) Y[tj * R + row0 + ti] = m[0];
            }
        }
        __syncthreads();
    }
}

// ------------------------------------------------------------------ MV, medium rows: warp per row, x in smem
// All K x-vectors (K*C*4 bytes <= 48 KB) are staged once per CTA by TMA; each warp then
// streams whole rows (RB per step, U loads per row in flight) and reduces with shuffles:
// no CTA-wide barrier per row (the CTA-per-row kernel's per-row reduction and the
// measured alternative that staged x in column chunks with a per-block ticket dominated rows of a few KB).
template <int K, int RB, int U, int NT>
__global__ void __launch_bounds__(NT, 4)
mmv_warp_kernel(const float* __restrict__ A, const float* __restrict__ X, float* __restrict__ Y,
                int64_t R, int64_t C)
{
    pdl_prologue();
    extern __shared__ __align__(128) unsigned char dyn_smem[];
    __shared__ __align__(8) uint64_t xbar;
    float4* xs = reinterpret_cast<float4*>(dyn_smem);   // [K][nv]
    const int64_t nv = C / 4;
    stage_to_smem(xs, X, uint32_t(K * C * 4), &xbar);
    const float4* __restrict__ Av = reinterpret_cast<const float4*>(A);
    const int lane = threadIdx.x & 31;
    const int64_t warp = (int64_t(blockIdx.x) * NT + threadIdx.x) >> 5;
    const int64_t nwarps = (int64_t(gridDim.x) * NT) >> 5;
    for (int64_t base = warp * RB; base < R; base += nwarps * RB) {
        int64_t off[RB];
#pragma unroll
        for (int i = 0; i < RB; ++i) off[i] = (base + i < R ? base + i : 0) * nv;
        float4 acc[RB][K];
#pragma unroll
        for (int i = 0; i < RB; ++i)
#pragma unroll
            for (int j = 0; j < K; ++j) acc[i][j] = make_float4(0.f, 0.f, 0.f, 0.f);
        float outer[RB][K];
#pragma unroll
        for (int i = 0; i < RB; ++i)
#pragma unroll
            for (int j = 0; j < K; ++j) outer[i][j] = 0.f;
        int it = 0;
        int64_t v = lane;
        for (; v + 32 * (U - 1) < nv; v += 32 * U) {
            float4 a[RB][U];
#pragma unroll
            for (int u = 0; u < U; ++u)
#pragma unroll
                for (int i = 0; i < RB; ++i) a[i][u] = ld_stream(Av + off[i] + v + 32 * u);
#pragma unroll
            for (int u = 0; u < U; ++u)
#pragma unroll
                for (int j = 0; j < K; ++j) {
                    const float4 xv = xs[j * nv + v + 32 * u];
#pragma unroll
                    for (int i = 0; i < RB; ++i) vmac(acc[i][j], a[i][u], xv);
                }
            if (++it == FOLD / U) {
                it = 0;
#pragma unroll
                for (int i = 0; i < RB; ++i)
#pragma unroll
                    for (int j = 0; j < K; ++j) { outer[i][j] += vsum(acc[i][j]); acc[i][j] = make_float4(0.f, 0.f, 0.f, 0.f); }
            }
        }
        for (; v < nv; v += 32) {
#pragma unroll
            for (int i = 0; i < RB; ++i) {
                const float4 a = ld_stream(Av + off[i] + v);
#pragma unroll
                for (int j = 0; j < K; ++j) vmac(acc[i][j], a, xs[j * nv + v]);
            }
        }
#pragma unroll
        for (int i = 0; i < RB; ++i)
#pragma unroll
            for (int j = 0; j < K; ++j) {
                const float t = group_sum<32>(outer[i][j] + vsum(acc[i][j]));
                if (lane == 0 && base + i < R) Y[j * R + base + i] = t;
            }
    }
}

// ------------------------------------------------------------------ TMV tiles
// As tmv_kernel: CTA tile of LR output vectors x LC = NT/LR c-lanes, S c-ranges,
// with K accumulators per thread (one per vector) and the lc-combine per vector.
template <int K, int LR, int U, bool VEC, int NT>
__global__ void __launch_bounds__(NT, 2)
tmmv_kernel(const float* __restrict__ B, const float* __restrict__ X, float* __restrict__ Y,
            int64_t R, int64_t C, int S, float* __restrict__ ws_part, unsigned int* __restrict__ ws_cnt)
{
    pdl_prologue();
    using E = typename ElemOf<float, VEC>::type;
    constexpr int W = VEC ? 4 : 1;
    constexpr int LC = NT / LR;
    __shared__ E red[LC > 1 ? NT : 1];
    __shared__ unsigned int flag;
    const int64_t rv = R / W;
    const int64_t ntiles = (rv + LR - 1) / LR;
    const int64_t chunk = (C + S - 1) / S;
    const E* __restrict__ Bv = reinterpret_cast<const E*>(B);
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
        E acc[K], outer[K];
#pragma unroll
        for (int j = 0; j < K; ++j) { acc[j] = zero_of<E>(); outer[j] = zero_of<E>(); }
        int it = 0;
        const E* __restrict__ Bc = Bv + (rok ? r4 : 0);
        int64_t c = c0 + lc;
        for (; c + int64_t(LC) * (U - 1) < c1; c += int64_t(LC) * U) {
            E a[U];
#pragma unroll
            for (int u = 0; u < U; ++u) a[u] = ld_stream(Bc + (c + int64_t(LC) * u) * rv);
#pragma unroll
            for (int u = 0; u < U; ++u)
#pragma unroll
                for (int j = 0; j < K; ++j) esmac(acc[j], a[u], ld_x(X + j * C + c + int64_t(LC) * u));
            if (++it == FOLD / U) {
                it = 0;
#pragma unroll
                for (int j = 0; j < K; ++j) { outer[j] = eadd(outer[j], acc[j]); acc[j] = zero_of<E>(); }
            }
        }
        for (; c < c1; c += LC) {
            const E a = ld_stream(Bc + c * rv);
#pragma unroll
            for (int j = 0; j < K; ++j) esmac(acc[j], a, ld_x(X + j * C + c));
        }
        E* yv = reinterpret_cast<E*>(Y);
        E* pv = reinterpret_cast<E*>(ws_part);
#pragma unroll
        for (int j = 0; j < K; ++j) {
            E tot = lc_combine<NT, LR>(eadd(outer[j], acc[j]), red);
            if (S == 1) {
                if (tid < LR && rok) yv[j * rv + r4] = tot;
            } else if (tid < LR && rok) {
                pv[(int64_t(s) * K + j) * rv + r4] = tot;
            }
            __syncthreads();                              // red[] reuse by the next vector
        }
        if (S > 1 && ticket_is_last(ws_cnt + tile, unsigned(S), &flag)) {
#pragma unroll
            for (int j = 0; j < K; ++j) {
                E m = zero_of<E>();
                if (rok) m = merge_partials<LC>(pv + int64_t(j) * rv + r4, int64_t(K) * rv, lc, S);
                m = lc_combine<NT, LR>(m, red);
                if (tid < LR && rok) yv[j * rv + r4] = m;
                __syncthreads();
            }
        }
        __syncthreads();
    }
}

}  // namespace adaptic
