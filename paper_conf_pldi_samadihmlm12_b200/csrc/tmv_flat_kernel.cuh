// tmv_flat_kernel.cuh -- TMV with few outputs and R % 4 != 0 (R <= 64), sm_100a.
//
// B (C x R, row-major) is a flat stream of R*C words; output r collects the words
// f with f mod R = r, each times x[f div R].  With R small and not a multiple of 4,
// tiling B by 16-byte output vectors (tmv_kernel / tmv_mis_kernel) wastes lanes and
// loads: a 9-wide row is 36 bytes, so a thread's 16-byte slice straddles rows and
// the funnel path moved 2x the bytes through L2 (3.5-4.3 TB/s measured).  Here the
// flat array itself is streamed: consecutive threads read consecutive aligned
// 128-bit vectors (perfectly coalesced, no duplicated bytes).  Each CTA runs NTa =
// floor(NT/R)*R threads, so the grid-wide stride T = NTa*gridDim is a multiple of R
// and every thread's four words keep FIXED outputs r_j = (4t + j - b0) mod R for
// the whole loop, while their x index advances by 4T/R per step -- no division in
// the loop.  The per-thread partials are combined by output in a fixed order
// (strided sums over the CTA, then over CTAs by the last CTA of the launch -- the
// paper's merge kernel, folded in with a ticket), so a plan is deterministic.
#pragma once

#include "tmv_kernels.cuh"

namespace adaptic {



template <class T, int NT, int U>
__global__ void __launch_bounds__(NT)
tmv_flat_kernel(const T* __restrict__ B, const T* __restrict__ X, T* __restrict__ y,
                int64_t R64, int64_t C, T* __restrict__ ws_part, unsigned int* __restrict__ ws_cnt)
{
    pdl_prologue();
    using E = vec4_t<T>;
    __shared__ T P[4 * NT];
    __shared__ unsigned int flag;
    const int R = int(R64);
    const int NTa = (NT / R) * R;                       // active threads per CTA
    const int tid = threadIdx.x;
    const int b0 = int((reinterpret_cast<uintptr_t>(B) >> 2) & 3u);
    const E* __restrict__ Ba = reinterpret_cast<const E*>(B - b0);
    const int64_t total = R64 * C;                      // words of B
    const int64_t qend = (b0 + total + 3) >> 2;         // aligned vectors covering B
    const int64_t T_ = int64_t(gridDim.x) * NTa;
    const int64_t dc = 4 * T_ / R;                      // x index advance per step (R | T_)

    T acc[4] = {T(0), T(0), T(0), T(0)}, outer[4] = {T(0), T(0), T(0), T(0)};
    if (tid < NTa) {
        const int64_t t = int64_t(blockIdx.x) * NTa + tid;
        // one vector whose words may lie outside B (the first and the last): masked, with
        // the x index by division
        auto edge_vec = [&](int64_t q) {
            const int64_t f0 = 4 * q - b0;
            if (f0 >= 0 && f0 + 3 < total) {
                const E a = ld_stream(Ba + q);
                const T av[4] = {a.x, a.y, a.z, a.w};
#pragma unroll
                for (int j = 0; j < 4; ++j) acc[j] = mac(av[j], ld_x(X + (f0 + j) / R), acc[j]);
            } else {
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    const int64_t f = f0 + j;
                    if (f >= 0 && f < total) acc[j] = mac(ld_stream(B + f), ld_x(X + f / R), acc[j]);
                }
            }
        };
        int64_t q = t;
        // vector 0 may start before B (b0 > 0): peel it, so that the unrolled loop below
        // runs for every thread (thread 0 included) with nonnegative word indices
        if (q == 0) { if (qend > 0) edge_vec(0); q = T_; }
        int64_t c[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) c[j] = (4 * q + j - b0) / R;     // word 4q + j - b0 >= 1
        int it = 0;
        // interior vectors (every word inside B): q in [1, qend - 1)
        for (; q + T_ * (U - 1) < qend - 1; q += T_ * U) {
            E a[U];
            T xv[U][4];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                a[u] = ld_stream(Ba + q + T_ * u);
#pragma unroll
                for (int j = 0; j < 4; ++j) xv[u][j] = ld_x(X + c[j] + dc * u);
            }
#pragma unroll
            for (int u = 0; u < U; ++u) {
                acc[0] = mac(a[u].x, xv[u][0], acc[0]); acc[1] = mac(a[u].y, xv[u][1], acc[1]);
                acc[2] = mac(a[u].z, xv[u][2], acc[2]); acc[3] = mac(a[u].w, xv[u][3], acc[3]);
            }
#pragma unroll
            for (int j = 0; j < 4; ++j) c[j] += dc * U;
            if (++it == FOLD / U) {
                it = 0;
#pragma unroll
                for (int j = 0; j < 4; ++j) { outer[j] += acc[j]; acc[j] = T(0); }
            }
        }
        // the rest, one vector at a time, words outside B masked
        for (; q < qend; q += T_) edge_vec(q);
#pragma unroll
        for (int j = 0; j < 4; ++j) P[4 * tid + j] = outer[j] + acc[j];
    }
    __syncthreads();
    // word position m = 4*tid + j of this CTA belongs to r = (base + m) mod R; as NTa is a
    // multiple of R, m, m + NTa, m + 2 NTa, m + 3 NTa share r: fold them first
    T* Q = P;                                           // reused after the fold below
    T fold = T(0);
    if (tid < NTa) fold = (P[tid] + P[tid + NTa]) + (P[tid + 2 * NTa] + P[tid + 3 * NTa]);
    __syncthreads();
    if (tid < NTa) Q[tid] = fold;
    __syncthreads();
    const int base = int(((int64_t(4) * blockIdx.x * NTa - b0) % R + R) % R);
    if (tid < R) {                                      // output r = tid: positions t' = (r - base) mod R + k R
        T s = T(0);
        for (int tp = ((tid - base) % R + R) % R; tp < NTa; tp += R) s += Q[tp];
        ws_part[int64_t(blockIdx.x) * R + tid] = s;
    }
    if (ticket_is_last(ws_cnt, gridDim.x, &flag)) {
        // (r, k) = (tid % R, tid / R): strided sums over the CTAs, then over k, fixed order
        const int G = int(gridDim.x), NK = NTa / R;
        T s = T(0);
        if (tid < NTa)
            for (int g = tid / R; g < G; g += NK) s += ld_partial(ws_part + int64_t(g) * R + tid % R);
        __syncthreads();
        if (tid < NTa) P[tid] = s;
        __syncthreads();
        if (tid < R) {
            T tot = T(0);
            for (int k = 0; k < NK; ++k) tot += P[tid + k * R];
            y[tid] = tot;
        }
    }
}

}  // namespace adaptic
