// tmv_mis_kernel.cuh -- TMV when B's rows are not 16-byte aligned (R % 4 != 0), sm_100a.
//
// B is C x R row-major; row c starts at element c*R, so with R % 4 != 0 the
// 16-byte alignment of a thread's four outputs 4*r4 .. 4*r4+3 shifts from row to
// row by s_c = (b0 + c*R) mod 4 (b0 = B's own element offset mod 4).  The
// aligned tmv_kernel cannot be used; the scalar one moves 4 bytes per load and
// reached only 2.6-5.2 TB/s (profiles/, perturbed sweep).  Here a thread loads
// the two aligned 128-bit vectors that cover its four elements of row c and
// selects them by s_c (a funnel shift in registers), so the stream stays 128-bit;
// the second vector is the neighbouring thread's first, so HBM traffic is
// unchanged and only L2 sees it twice (L1-allocating loads for the pair were
// measured no faster: profiles/, sweep_tmv_mis2).  Tiling, splits and the merge are those of
// tmv_kernel (TMV_COL / TMV_SPLITK / TMV_REGTILE; the paper's restructured-layout
// kernels).  y and the partials are written per element (y is not
// 16-byte aligned in general), the last vector of a tile row masked to R.
#pragma once

#include "tmv_kernels.cuh"

namespace adaptic {


// Aligned vector q of the aligned view (element e of B is element b0 + e of the view):
// one 128-bit load when all four words lie inside B, else the words inside B one by one
// (zeros elsewhere) -- the first vector of B starts b0 words early and the last may end
// up to 3 words late; those words are never selected, and are not read either.
template <class E, class T> __device__ __forceinline__ E ld_inside(const E* Ba, const T* B, int64_t q, int b0, int64_t total) {
    const int64_t f0 = 4 * q - b0;                    // element of B at lane 0
    if (f0 >= 0 && f0 + 3 < total) return ld_stream(Ba + q);
    E v = zero_of<E>();
    if (f0 >= 0 && f0 < total) v.x = ld_stream(B + f0);
    if (f0 + 1 >= 0 && f0 + 1 < total) v.y = ld_stream(B + f0 + 1);
    if (f0 + 2 >= 0 && f0 + 2 < total) v.z = ld_stream(B + f0 + 2);
    if (f0 + 3 >= 0 && f0 + 3 < total) v.w = ld_stream(B + f0 + 3);
    return v;
}

template <class T, int LR, int U, int NT>
__global__ void __launch_bounds__(NT, U <= 2 ? 4 : U <= 4 ? 3 : 2)
tmv_mis_kernel(const T* __restrict__ B, const T* __restrict__ X, T* __restrict__ y,
               int64_t R, int64_t C, int S, T* __restrict__ ws_part, unsigned int* __restrict__ ws_cnt)
{
    pdl_prologue();
    using E = vec4_t<T>;
    constexpr int LC = NT / LR;
    __shared__ E red[LC > 1 ? NT : 1];
    __shared__ unsigned int flag;
    const int64_t rv = (R + 3) / 4;                   // output vectors (last one partial)
    const int64_t ntiles = (rv + LR - 1) / LR;
    const int64_t chunk = (C + S - 1) / S;
    // aligned view of B: element e of B is element b0 + e of Ba
    const int b0 = int((reinterpret_cast<uintptr_t>(B) >> 2) & 3u);
    const E* __restrict__ Ba = reinterpret_cast<const E*>(B - b0);
    const int64_t qmax = (b0 + R * C - 1) >> 2;       // last aligned vector holding B data
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
        const int64_t col = 4 * (rok ? r4 : 0);       // ragged tile: read column 0, discard

        E acc[U];
#pragma unroll
        for (int u = 0; u < U; ++u) acc[u] = zero_of<E>();
        E outer = zero_of<E>();
        int it = 0;
        int64_t c = c0 + lc;
        for (; c + int64_t(LC) * (U - 1) < c1; c += int64_t(LC) * U) {
            E lo[U], hi[U];
            T xs[U];
            int sh[U];
            // aligned vectors grow with c: when the first load's low vector starts inside B
            // and the last load's high vector ends inside it, every word of every load is
            // inside B and no per-word masking is needed (only the very first / last 16
            // bytes of B take the masked path)
            const int64_t qf = (b0 + c * R + col) >> 2;
            const int64_t ql = (b0 + (c + int64_t(LC) * (U - 1)) * R + col) >> 2;
            if (4 * qf - b0 >= 0 && 4 * (ql + 1) - b0 + 3 < R * C) {
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    const int64_t cc = c + int64_t(LC) * u;
                    const int64_t f = b0 + cc * R + col;
                    const int64_t q = f >> 2;
                    sh[u] = int(f & 3);
                    lo[u] = ld_stream(Ba + q);
                    hi[u] = ld_stream(Ba + q + 1);
                    xs[u] = ld_x(X + cc);
                }
            } else {
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    const int64_t cc = c + int64_t(LC) * u;
                    const int64_t f = b0 + cc * R + col;         // aligned-view element index
                    const int64_t q = f >> 2;
                    sh[u] = int(f & 3);
                    lo[u] = ld_inside(Ba, B, q, b0, R * C);
                    hi[u] = ld_inside(Ba, B, min(q + 1, qmax), b0, R * C);
                    xs[u] = ld_x(X + cc);
                }
            }
#pragma unroll
            for (int u = 0; u < U; ++u) esmac(acc[u], funnel4(lo[u], hi[u], sh[u]), xs[u]);
            if (++it == FOLD) {
                it = 0;
                outer = eadd(outer, tree_sum<U>(acc));
#pragma unroll
                for (int u = 0; u < U; ++u) acc[u] = zero_of<E>();
            }
        }
        for (; c < c1; c += LC) {
            const int64_t f = b0 + c * R + col;
            const int64_t q = f >> 2;
            esmac(acc[0], funnel4(ld_inside(Ba, B, q, b0, R * C), ld_inside(Ba, B, min(q + 1, qmax), b0, R * C),
                                  int(f & 3)), ld_x(X + c));
        }
        E tot = eadd(outer, tree_sum<U>(acc));
        tot = lc_combine<NT, LR>(tot, red);

        auto store4 = [&](T* dst, const E& v) {       // the outputs of vector r4 that exist
            const int64_t r = 4 * r4;
            dst[r] = v.x;
            if (r + 1 < R) dst[r + 1] = v.y;
            if (r + 2 < R) dst[r + 2] = v.z;
            if (r + 3 < R) dst[r + 3] = v.w;
        };
        if (S == 1) {
            if (tid < LR && rok) store4(y, tot);
        } else {
            if (tid < LR && rok) pv[int64_t(s) * rv + r4] = tot;
            if (ticket_is_last(ws_cnt + tile, unsigned(S), &flag)) {
                E m = zero_of<E>();
                if (rok) m = merge_partials<LC>(pv + r4, rv, lc, S);
                __syncthreads();
                m = lc_combine<NT, LR>(m, red);
                if (tid < LR && rok) store4(y, m);
            }
        }
        __syncthreads();
    }
}

}  // namespace adaptic

namespace adaptic {

// Rows off the 16-byte grid WITHOUT the funnel (round 2).  With c-lanes LC a multiple of 4,
// the rows a thread visits (c = c0 + lc + LC k) all have the same word shift
// sh = (b0 + (c0 + lc) R) mod 4, so a thread can stream ONE aligned 128-bit vector per row
// -- the aligned kernel's instruction mix -- and simply remember which outputs its four
// words belong to: thread (lr, lc) of tile t accumulates words 4 lr .. 4 lr + 3 of the
// aligned window that starts at output ob = t WT, i.e. outputs ob - sh + 4 lr + j.  A tile
// owns WT = 4 LR - 4 outputs (the window's 4 LR words cover them at any shift; the extra
// vector per row is re-read by the neighbouring tile: 1 / LR more L2 traffic), and the
// c-lane combine sums, per owned output, each lane's word at its own shift, in lane order.
// Tiling, splits and the ticket merge as tmv_kernel; B's first / last 16 bytes are loaded
// word by word (ld_inside).
template <class T, int LR, int U, int NT>
__global__ void __launch_bounds__(NT, U <= 2 ? 4 : 3)
tmv_shift_kernel(const T* __restrict__ B, const T* __restrict__ X, T* __restrict__ y,
                 int64_t R, int64_t C, int S, T* __restrict__ ws_part, unsigned int* __restrict__ ws_cnt)
{
    pdl_prologue();
    using E = vec4_t<T>;
    constexpr int LC = NT / LR;
    static_assert(LC % 4 == 0, "c-lanes: a multiple of 4 (one word shift per c-lane)");
    constexpr int WT = 4 * LR - 4;                    // outputs owned by a tile
    __shared__ T red[LC * 4 * LR];                    // [lc][4 lr + j]
    __shared__ unsigned int flag;
    const int64_t ntiles = (R + WT - 1) / WT;
    const int64_t Rp = ntiles * WT;                   // partial row length
    const int64_t chunk = (C + S - 1) / S;
    const int b0 = int((reinterpret_cast<uintptr_t>(B) >> 2) & 3u);
    const E* __restrict__ Ba = reinterpret_cast<const E*>(B - b0);
    const int64_t total = R * C;
    const int tid = threadIdx.x;
    const int lr = tid % LR, lc = tid / LR;
    const int64_t nblk = ntiles * S;

    for (int64_t blk = blockIdx.x; blk < nblk; blk += gridDim.x) {
        const int64_t tile = blk % ntiles;
        const int s = int(blk / ntiles);
        const int64_t ob = tile * WT;
        const int64_t c0 = int64_t(s) * chunk;
        const int64_t c1 = min(C, c0 + chunk);
        // NA accumulators (U loads in flight): U = 8 keeps 2, so the 8 loads fit 3 CTAs per SM
        constexpr int NA = U > 4 ? 2 : U;
        E acc[NA];
#pragma unroll
        for (int u = 0; u < NA; ++u) acc[u] = zero_of<E>();
        E outer = zero_of<E>();
        int it = 0;
        int64_t c = c0 + lc;
        for (; c + int64_t(LC) * (U - 1) < c1; c += int64_t(LC) * U) {
            E a[U];
            T xs[U];
            const int64_t qf = ((b0 + c * R + ob) >> 2) + lr;
            const int64_t ql = ((b0 + (c + int64_t(LC) * (U - 1)) * R + ob) >> 2) + lr;
            if (4 * qf - b0 >= 0 && 4 * ql - b0 + 3 < total) {
                // LC % 4 == 0: row c + LC u starts LC R / 4 vectors after row c, exactly
                const E* pa = Ba + qf;
                const int64_t sv = int64_t(LC) * R / 4;
                const T* px = X + c;
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    a[u] = ld_stream(pa + sv * u);
                    xs[u] = ld_x(px + LC * u);
                }
            } else {
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    const int64_t cc = c + int64_t(LC) * u;
                    a[u] = ld_inside(Ba, B, ((b0 + cc * R + ob) >> 2) + lr, b0, total);
                    xs[u] = ld_x(X + cc);
                }
            }
#pragma unroll
            for (int u = 0; u < U; ++u) esmac(acc[u % NA], a[u], xs[u]);
            if (++it == FOLD * NA / U) {                  // <= FOLD products per accumulator
                it = 0;
                outer = eadd(outer, tree_sum<NA>(acc));
#pragma unroll
                for (int u = 0; u < NA; ++u) acc[u] = zero_of<E>();
            }
        }
        for (; c < c1; c += LC)
            esmac(acc[0], ld_inside(Ba, B, ((b0 + c * R + ob) >> 2) + lr, b0, total), ld_x(X + c));
        const E tot = eadd(outer, tree_sum<NA>(acc));
        T* rl = red + lc * 4 * LR + 4 * lr;
        rl[0] = tot.x; rl[1] = tot.y; rl[2] = tot.z; rl[3] = tot.w;
        __syncthreads();
        // owned output rho: lane l's word rho + sh_l, summed in lane order (sh_l = shift of its rows)
        T v = T(0);
        if (tid < WT) {
#pragma unroll 4
            for (int l = 0; l < LC; ++l) {
                const int sh = int((b0 + (c0 + l) * R + ob) & 3);
                v += red[l * 4 * LR + tid + sh];
            }
        }
        const bool rok = tid < WT && ob + tid < R;
        if (S == 1) {
            if (rok) y[ob + tid] = v;
        } else {
            if (tid < WT) ws_part[int64_t(s) * Rp + ob + tid] = v;
            if (ticket_is_last(ws_cnt + tile, unsigned(S), &flag)) {
                T m0 = T(0), m1 = T(0);
                if (rok) {
                    int k = 0;
                    for (; k + 1 < S; k += 2) {
                        m0 += ld_partial(ws_part + int64_t(k) * Rp + ob + tid);
                        m1 += ld_partial(ws_part + int64_t(k + 1) * Rp + ob + tid);
                    }
                    if (k < S) m0 += ld_partial(ws_part + int64_t(k) * Rp + ob + tid);
                    y[ob + tid] = m0 + m1;
                }
            }
        }
        __syncthreads();                              // red / flag reuse
    }
}

}  // namespace adaptic

namespace adaptic {

// Rows off the 16-byte grid with ONE aligned 128-bit load per row and thread and no c-lanes
// (round 2, "sliding window"): thread w of the aligned view streams window w (words 4w..4w+3
// of every row's aligned base); in row c, word j is output 4w + j - s_c (s_c = (b0 + c R)
// mod 4), so over all rows a thread touches outputs 4w - 3 .. 4w + 3 and keeps 7
// accumulators.  s_c has period 4 in c, so rows are taken in groups of 4 whose shift
// pattern (s0, R mod 4) is a template argument: every accumulator index is a compile-time
// constant.  At the end output 4w + k = acc_w[k + 3] + acc_{w+1}[k - 1] (k >= 1): read from
// the next thread through shared memory; the last thread of a tile only supplies that halo
// (tiles of NT - 1 owned windows).  Splits over c, the ticket merge per tile as tmv_kernel.
// tmv_window_warp_kernel (S = 1): the same per thread, but each WARP owns a tile of 31
// windows and takes the halo by shuffle -- no shared memory and no CTA barrier, so warps
// move on to their next tile independently.
template <class T, int S0, int RM, int G8>
__device__ __forceinline__ void win_rows(T (&acc)[7], const vec4_t<T>* __restrict__ Ba, const T* __restrict__ B,
                                         const T* __restrict__ X, int b0, int64_t R, int64_t C, int64_t total,
                                         int64_t w, int64_t c, int64_t c1) {
    using E = vec4_t<T>;
    constexpr int RMN = RM & 3;
    // G8 groups of 4 rows per iteration (4 G8 loads in flight)
    for (; c + 4 * G8 - 1 < c1; c += 4 * G8) {
        E a[4 * G8];
        T xs[4 * G8];
        const int64_t qf = ((b0 + c * R) >> 2) + w;
        const int64_t ql = ((b0 + (c + 4 * G8 - 1) * R) >> 2) + w;
        if (4 * qf - b0 >= 0 && 4 * ql - b0 + 3 < total) {
#pragma unroll
            for (int u = 0; u < 4 * G8; ++u) {
                a[u] = ld_stream(Ba + ((b0 + (c + u) * R) >> 2) + w);
                xs[u] = ld_x(X + c + u);
            }
        } else {
#pragma unroll
            for (int u = 0; u < 4 * G8; ++u) {
                a[u] = ld_inside(Ba, B, ((b0 + (c + u) * R) >> 2) + w, b0, total);
                xs[u] = ld_x(X + c + u);
            }
        }
#pragma unroll
        for (int u = 0; u < 4 * G8; ++u) {
            const int s = (S0 + (u & 3) * RMN) & 3;          // compile-time after unrolling
            // word j -> accumulator j - s + 3
            switch (s) {
                case 0: acc[3] = mac(a[u].x, xs[u], acc[3]); acc[4] = mac(a[u].y, xs[u], acc[4]);
                        acc[5] = mac(a[u].z, xs[u], acc[5]); acc[6] = mac(a[u].w, xs[u], acc[6]); break;
                case 1: acc[2] = mac(a[u].x, xs[u], acc[2]); acc[3] = mac(a[u].y, xs[u], acc[3]);
                        acc[4] = mac(a[u].z, xs[u], acc[4]); acc[5] = mac(a[u].w, xs[u], acc[5]); break;
                case 2: acc[1] = mac(a[u].x, xs[u], acc[1]); acc[2] = mac(a[u].y, xs[u], acc[2]);
                        acc[3] = mac(a[u].z, xs[u], acc[3]); acc[4] = mac(a[u].w, xs[u], acc[4]); break;
                default: acc[0] = mac(a[u].x, xs[u], acc[0]); acc[1] = mac(a[u].y, xs[u], acc[1]);
                         acc[2] = mac(a[u].z, xs[u], acc[2]); acc[3] = mac(a[u].w, xs[u], acc[3]); break;
            }
        }
    }
    for (; c < c1; ++c) {                                   // rows left: runtime shift
        const int64_t f = b0 + c * R;
        const E a = ld_inside(Ba, B, (f >> 2) + w, b0, total);
        const T xv = ld_x(X + c);
        const int s = int(f & 3);
        const T v[4] = {a.x, a.y, a.z, a.w};
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            const int k = j - s + 3;
#pragma unroll
            for (int q = 0; q < 7; ++q)
                if (q == k) acc[q] = mac(v[j], xv, acc[q]);
        }
    }
}

template <class T, int G8, int S0, int RM>
__device__ __forceinline__ void win_dispatch_rm(T (&acc)[7], const vec4_t<T>* Ba, const T* B, const T* X, int b0,
                                                int64_t R, int64_t C, int64_t total, int64_t w, int64_t c, int64_t c1) {
    win_rows<T, S0, RM, G8>(acc, Ba, B, X, b0, R, C, total, w, c, c1);
}

template <class T, int G8>
__device__ __forceinline__ void win_dispatch(T (&acc)[7], const vec4_t<T>* Ba, const T* B, const T* X, int b0,
                                             int64_t R, int64_t C, int64_t total, int64_t w, int64_t c, int64_t c1) {
    const int s0 = int((b0 + c * R) & 3), rm = int(R & 3);
    switch (s0 * 4 + rm) {
#define ADAPTIC_WIN(S, M) case S * 4 + M: win_rows<T, S, M, G8>(acc, Ba, B, X, b0, R, C, total, w, c, c1); break;
        ADAPTIC_WIN(0, 0) ADAPTIC_WIN(0, 1) ADAPTIC_WIN(0, 2) ADAPTIC_WIN(0, 3)
        ADAPTIC_WIN(1, 0) ADAPTIC_WIN(1, 1) ADAPTIC_WIN(1, 2) ADAPTIC_WIN(1, 3)
        ADAPTIC_WIN(2, 0) ADAPTIC_WIN(2, 1) ADAPTIC_WIN(2, 2) ADAPTIC_WIN(2, 3)
        ADAPTIC_WIN(3, 0) ADAPTIC_WIN(3, 1) ADAPTIC_WIN(3, 2) ADAPTIC_WIN(3, 3)
#undef ADAPTIC_WIN
        default: break;
    }
}

template <class T, int G8, int NT>
__global__ void __launch_bounds__(NT, 2)
tmv_window_kernel(const T* __restrict__ B, const T* __restrict__ X, T* __restrict__ y,
                  int64_t R, int64_t C, int S, T* __restrict__ ws_part, unsigned int* __restrict__ ws_cnt)
{
    pdl_prologue();
    using E = vec4_t<T>;
    __shared__ T halo[NT][3];
    __shared__ unsigned int flag;
    const int b0 = int((reinterpret_cast<uintptr_t>(B) >> 2) & 3u);
    const E* __restrict__ Ba = reinterpret_cast<const E*>(B - b0);
    const int64_t total = R * C;
    const int64_t own = (R + 3) / 4;                       // windows that own outputs (4w < R)
    const int64_t ntiles = (own + NT - 2) / (NT - 1);
    const int64_t chunk = (C + S - 1) / S;
    const int tid = threadIdx.x;
    const int64_t nblk = ntiles * S;
    for (int64_t blk = blockIdx.x; blk < nblk; blk += gridDim.x) {
        const int64_t tile = blk % ntiles;
        const int s = int(blk / ntiles);
        const int64_t w = tile * (NT - 1) + tid;             // this thread's window
        const int64_t c0 = min(C, int64_t(s) * chunk), c1 = min(C, c0 + chunk);
        T acc[7];
#pragma unroll
        for (int q = 0; q < 7; ++q) acc[q] = T(0);
        if (4 * w < R + 3) {                                 // windows past the data hold nothing
            // fp32 chains: fold every FOLD rows into a second level
            T outer[7];
#pragma unroll
            for (int q = 0; q < 7; ++q) outer[q] = T(0);
            for (int64_t cb = c0; cb < c1; cb += FOLD) {
                const int64_t ce = min(c1, cb + int64_t(FOLD));
                T a2[7];
#pragma unroll
                for (int q = 0; q < 7; ++q) a2[q] = T(0);
                win_dispatch<T, G8>(a2, Ba, B, X, b0, R, C, total, w, cb, ce);
#pragma unroll
                for (int q = 0; q < 7; ++q) outer[q] += a2[q];
            }
#pragma unroll
            for (int q = 0; q < 7; ++q) acc[q] = outer[q];
        }
        halo[tid][0] = acc[0]; halo[tid][1] = acc[1]; halo[tid][2] = acc[2];
        __syncthreads();
        T out[4];
        out[0] = acc[3];
#pragma unroll
        for (int k = 1; k < 4; ++k) out[k] = acc[3 + k] + (tid + 1 < NT ? halo[tid + 1][k - 1] : T(0));
        const bool owner = tid < NT - 1 && w < own;
        if (S == 1) {
            if (owner)
#pragma unroll
                for (int k = 0; k < 4; ++k)
                    if (4 * w + k < R) y[4 * w + k] = out[k];
        } else {
            if (owner)
#pragma unroll
                for (int k = 0; k < 4; ++k)
                    if (4 * w + k < R) ws_part[int64_t(s) * R + 4 * w + k] = out[k];
            if (ticket_is_last(ws_cnt + tile, unsigned(S), &flag)) {
                if (owner)
#pragma unroll
                    for (int k = 0; k < 4; ++k) {
                        const int64_t o = 4 * w + k;
                        if (o < R) {
                            T m0 = T(0), m1 = T(0);
                            int q = 0;
                            for (; q + 1 < S; q += 2) {
                                m0 += ld_partial(ws_part + int64_t(q) * R + o);
                                m1 += ld_partial(ws_part + int64_t(q + 1) * R + o);
                            }
                            if (q < S) m0 += ld_partial(ws_part + int64_t(q) * R + o);
                            y[o] = m0 + m1;
                        }
                    }
            }
        }
        __syncthreads();
    }
}

template <class T, int G8, int NT, int MINB>
__global__ void __launch_bounds__(NT, MINB)
tmv_window_warp_kernel(const T* __restrict__ B, const T* __restrict__ X, T* __restrict__ y, int64_t R, int64_t C)
{
    pdl_prologue();
    const int b0 = int((reinterpret_cast<uintptr_t>(B) >> 2) & 3u);
    const vec4_t<T>* __restrict__ Ba = reinterpret_cast<const vec4_t<T>*>(B - b0);
    const int64_t total = R * C;
    const int64_t own = (R + 3) / 4;
    const int64_t ntiles = (own + 30) / 31;
    const int lane = threadIdx.x & 31;
    const int64_t nw = int64_t(gridDim.x) * (NT / 32);
    const bool yv = (reinterpret_cast<uintptr_t>(y) & 15) == 0;
    for (int64_t t = int64_t(blockIdx.x) * (NT / 32) + (threadIdx.x >> 5); t < ntiles; t += nw) {
        const int64_t w = t * 31 + lane;
        T acc[7];
#pragma unroll
        for (int q = 0; q < 7; ++q) acc[q] = T(0);
        if (4 * w < R + 3) {
            for (int64_t cb = 0; cb < C; cb += FOLD) {
                const int64_t ce = min(C, cb + int64_t(FOLD));
                T a2[7];
#pragma unroll
                for (int q = 0; q < 7; ++q) a2[q] = T(0);
                win_dispatch<T, G8>(a2, Ba, B, X, b0, R, C, total, w, cb, ce);
#pragma unroll
                for (int q = 0; q < 7; ++q) acc[q] += a2[q];
            }
        }
        T out[4];
        out[0] = acc[3];
#pragma unroll
        for (int k = 1; k < 4; ++k) out[k] = acc[3 + k] + __shfl_down_sync(0xffffffffu, acc[k - 1], 1);
        if (lane < 31 && w < own) {
            if (yv && 4 * w + 3 < R) {
                vec4_t<T> o;
                o.x = out[0]; o.y = out[1]; o.z = out[2]; o.w = out[3];
                *reinterpret_cast<vec4_t<T>*>(y + 4 * w) = o;
            } else {
#pragma unroll
                for (int k = 0; k < 4; ++k)
                    if (4 * w + k < R) y[4 * w + k] = out[k];
            }
        }
    }
}

}  // namespace adaptic
