// mv_mis_kernels.cuh -- MV / DOT on rows that are not 16-byte aligned (C % 4 != 0), sm_100a.
//
// With a row-major R x C matrix and C % 4 != 0, row r starts at element r*C, so
// its 16-byte alignment shifts from row to row and the 128-bit path of
// mv_kernels.cuh cannot be used as is; the first version ran such shapes on the
// scalar (4-byte) loads and lost 15-60 % of bandwidth (3 * 2^k held-out shapes,
// profiles/).  Here every row is split into a scalar HEAD (h = 0..3 elements up
// to the first 16-byte boundary), an aligned BODY of 128-bit vectors and a
// scalar TAIL (0..3 elements): the matrix stream -- the HBM-bound part -- stays
// 128-bit for any C.  x is re-read from L1/L2 (or shared memory) at element
// offset h + 4j, which is misaligned, so it is read as four scalars; DOT's second
// operand has the same layout as A, so when a and b share their address modulo
// 16 (the planner checks) its body is 128-bit too.
//
// Thread shapes are those of the aligned kernels (the paper's K4/K3 lane groups
// and K2/K1 CTA-per-row / split-row reductions): mv_group_mis_kernel
// (MV_SUBWARP / MV_WPR) and mv_cta_mis_kernel (MV_CPR / MV_SPLIT, one row per
// CTA step).
#pragma once

#include "mv_kernels.cuh"

namespace adaptic {

// Elements before the first 16-byte boundary of a row starting at p (0..3).
template <class T> __device__ __forceinline__ int head_elems(const T* p) {
    return int(((16u - (uint32_t(reinterpret_cast<uintptr_t>(p)) & 15u)) & 15u) >> 2);
}

// x for the misaligned kernels: XM_SMEM copies all C elements once per CTA with
// plain loads (C*4 is not a multiple of 16 here, so no bulk copy); otherwise x
// itself (read through the read-only path), or DOT's per-row operand.
template <class T, int XM, int NT>
__device__ __forceinline__ const T* stage_x_scalar(const T* X, int64_t C) {
    if constexpr (XM != XM_SMEM) {
        return X;
    } else {
        extern __shared__ __align__(128) unsigned char dyn_smem[];
        T* xs = reinterpret_cast<T*>(dyn_smem);
        for (int64_t c = threadIdx.x; c < C; c += NT) xs[c] = ld_x(X + c);
        __syncthreads();
        return xs;
    }
}

// four consecutive x values at element offset e (any alignment)
template <int XM, class T> __device__ __forceinline__ vec4_t<T> ld_x4(const T* p) {
    vec4_t<T> v;
    v.x = ld_xm<XM>(p); v.y = ld_xm<XM>(p + 1); v.z = ld_xm<XM>(p + 2); v.w = ld_xm<XM>(p + 3);
    return v;
}

// XM_SHIFT: x arrives as four shifted copies X_h[i] = x[i + h] (h = 0..3, each P =
// round_up(C, 4) elements, 16-byte aligned; written by x_shift_kernel in the same stream
// just before), so the x chunk of a row with head h is ONE aligned 128-bit load,
// X_h[4v .. 4v+3] -- instead of four 32-bit loads at a misaligned offset, which made these
// kernels L1-bound (ncu l1tex 80-87 % of peak on the C+1 shapes).  Copy 0 is x itself.
constexpr int XM_SHIFT = 3;
__host__ __device__ constexpr int64_t xshift_pitch(int64_t C) { return (C + 3) / 4 * 4; }

template <class T>
__global__ void __launch_bounds__(256) x_shift_kernel(const T* __restrict__ X, T* __restrict__ out, int64_t C)
{
    pdl_prologue();
    const int64_t P = xshift_pitch(C);
    for (int64_t i = int64_t(blockIdx.x) * 256 + threadIdx.x; i < 4 * P; i += int64_t(gridDim.x) * 256) {
        const int64_t h = i / P, e = i - h * P + h;
        out[i] = e < C ? X[e] : T(0);
    }
}

// four consecutive x values at element offset h + 4v (the body of a row with head h)
template <int XM, class T> __device__ __forceinline__ vec4_t<T> x_body(const T* Xs, int h, int64_t v, int64_t P) {
    if constexpr (XM == XM_SHIFT) return ld_x(reinterpret_cast<const vec4_t<T>*>(Xs + h * P) + v);
    else return ld_x4<XM>(Xs + h + 4 * v);
}

// ------------------------------------------------------------------ lane groups (MV_SUBWARP / MV_WPR)
template <class T, int G, int RB, int U, int XM, int NT>
__global__ void __launch_bounds__(NT, 2)
mv_group_mis_kernel(const T* __restrict__ A, const T* __restrict__ X, T* __restrict__ y,
                    int64_t R, int64_t C)
{
    pdl_prologue();
    using E = vec4_t<T>;
    constexpr int NG = 32 / G;
    constexpr bool PERROWX = (XM == XM_ROW);
    const T* __restrict__ Xs = stage_x_scalar<T, XM, NT>(X, C);
    const int64_t P = xshift_pitch(C);
    const int lane = threadIdx.x & 31;
    const int g = lane / G, li = lane % G;
    const int64_t warp = (int64_t(blockIdx.x) * NT + threadIdx.x) >> 5;
    const int64_t nwarps = (int64_t(gridDim.x) * NT) >> 5;
    const int64_t step = int64_t(RB) * NG;

    for (int64_t base = warp * step; base < R; base += nwarps * step) {
        const T* rowp[RB];
        const E* av[RB];
        const E* bv[RB];
        int h[RB];
        int64_t nb[RB];
        int64_t nbmin = int64_t(1) << 62;
#pragma unroll
        for (int i = 0; i < RB; ++i) {
            const int64_t row = base + i * NG + g;
            rowp[i] = A + (row < R ? row : 0) * C;          // rows past R read row 0 (discarded)
            h[i] = head_elems(rowp[i]);
            av[i] = reinterpret_cast<const E*>(rowp[i] + h[i]);
            bv[i] = reinterpret_cast<const E*>(Xs + (PERROWX ? (row < R ? row : 0) * C : 0) + h[i]);
            nb[i] = (C - h[i]) >> 2;
            nbmin = min(nbmin, nb[i]);
        }
        E acc[RB][U];
        T outer[RB], edge[RB];
#pragma unroll
        for (int i = 0; i < RB; ++i) {
            outer[i] = T(0); edge[i] = T(0);
#pragma unroll
            for (int u = 0; u < U; ++u) acc[i][u] = zero_of<E>();
        }
        int it = 0;
        int64_t j0 = li;
        for (; j0 + int64_t(G) * (U - 1) < nbmin; j0 += int64_t(G) * U) {
            E a[RB][U], b[RB][U];
#pragma unroll
            for (int u = 0; u < U; ++u)
#pragma unroll
                for (int i = 0; i < RB; ++i) {
                    const int64_t v = j0 + int64_t(G) * u;
                    a[i][u] = ld_stream(av[i] + v);
                    if constexpr (PERROWX) b[i][u] = ld_stream(bv[i] + v);
                    else b[i][u] = x_body<XM>(Xs, h[i], v, P);
                }
#pragma unroll
            for (int i = 0; i < RB; ++i)
#pragma unroll
                for (int u = 0; u < U; ++u) emac(acc[i][u], a[i][u], b[i][u]);
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
#pragma unroll
        for (int i = 0; i < RB; ++i) {
            for (int64_t v = j0; v < nb[i]; v += G) {     // body tail: < U vectors for this lane
                const E b = PERROWX ? ld_stream(bv[i] + v) : x_body<XM>(Xs, h[i], v, P);
                emac(acc[i][0], ld_stream(av[i] + v), b);
            }
            // scalar head [0, h) and tail [h + 4 nb, C): at most 3 + 3 elements per row
            const int64_t t0 = h[i] + 4 * nb[i];
            for (int k = li; k < h[i] + int(C - t0); k += G) {
                const int64_t c = k < h[i] ? k : t0 + (k - h[i]);
                const T xv = PERROWX ? ld_stream(Xs + (rowp[i] - A) + c) : ld_xm<XM>(Xs + c);
                edge[i] = mac(ld_stream(rowp[i] + c), xv, edge[i]);
            }
        }
#pragma unroll
        for (int i = 0; i < RB; ++i) {
            T s = (outer[i] + esum(tree_sum<U>(acc[i]))) + edge[i];
            s = group_sum<G>(s);
            const int64_t row = base + i * NG + g;
            if (li == 0 && row < R) y[row] = s;
        }
    }
}

// ------------------------------------------------------------------ CTA per row (MV_CPR / MV_SPLIT)
// One row per CTA step, S CTAs per row interleaved in steps of NT*U vectors; the
// split s == 0 also takes the scalar head and tail.  Merge as in mv_cta_kernel.
template <class T, int NT, int U, int XM>
__global__ void __launch_bounds__(NT)
mv_cta_mis_kernel(const T* __restrict__ A, const T* __restrict__ X, T* __restrict__ y,
                  int64_t R, int64_t C, int S, int ilv, T* __restrict__ ws_part, unsigned int* __restrict__ ws_cnt)
{
    pdl_prologue();
    using E = vec4_t<T>;
    constexpr bool PERROWX = (XM == XM_ROW);
    constexpr int64_t BV = int64_t(NT) * U;
    __shared__ T red[NT / 32];
    __shared__ unsigned int flag;
    const T* __restrict__ Xs = stage_x_scalar<T, XM, NT>(X, C);
    const int64_t P = xshift_pitch(C);
    const int tid = threadIdx.x;
    const int64_t nblk = R * S;

    for (int64_t blk = blockIdx.x; blk < nblk; blk += gridDim.x) {
        const int64_t row = blk / S;
        const int s = int(blk - row * S);
        const T* rowp = A + row * C;
        const int h = head_elems(rowp);
        const E* av = reinterpret_cast<const E*>(rowp + h);
        const E* bv = reinterpret_cast<const E*>(Xs + (PERROWX ? row * C : 0) + h);
        const int64_t nb = (C - h) >> 2;
        const int64_t chunk = (nb + S - 1) / S;
        const int64_t start = ilv ? int64_t(s) * BV : int64_t(s) * chunk;
        const int64_t stride = ilv ? int64_t(S) * BV : BV;
        const int64_t end = ilv ? nb : min(nb, start + chunk);

        E acc[U];
#pragma unroll
        for (int u = 0; u < U; ++u) acc[u] = zero_of<E>();
        T outer = T(0), edge = T(0);
        int it = 0;
        int64_t b = start;
        for (; b + tid + int64_t(NT) * (U - 1) < end; b += stride) {
            E a[U], x[U];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const int64_t v = b + tid + int64_t(NT) * u;
                a[u] = ld_stream(av + v);
                if constexpr (PERROWX) x[u] = ld_stream(bv + v);
                else x[u] = x_body<XM>(Xs, h, v, P);
            }
#pragma unroll
            for (int u = 0; u < U; ++u) emac(acc[u], a[u], x[u]);
            if (++it == FOLD) {
                it = 0;
                outer += esum(tree_sum<U>(acc));
#pragma unroll
                for (int u = 0; u < U; ++u) acc[u] = zero_of<E>();
            }
        }
        const int64_t tail_end = min(end, b + BV);
        for (int64_t v = b + tid; v < tail_end; v += NT) {
            const E x = PERROWX ? ld_stream(bv + v) : x_body<XM>(Xs, h, v, P);
            emac(acc[0], ld_stream(av + v), x);
        }
        if (s == 0) {                                    // scalar head and tail of the row
            const int64_t t0 = h + 4 * nb;
            if (tid < h + int(C - t0)) {
                const int64_t c = tid < h ? tid : t0 + (tid - h);
                const T xv = PERROWX ? ld_stream(Xs + row * C + c) : ld_xm<XM>(Xs + c);
                edge = mac(ld_stream(rowp + c), xv, edge);
            }
        }
        T val[1] = {(outer + esum(tree_sum<U>(acc))) + edge};
        cta_sum_rows<NT, 1>(val, red);

        if (S == 1) {
            if (tid == 0) y[row] = val[0];
        } else {
            if (tid == 0) ws_part[row * S + s] = val[0];
            if (ticket_is_last(ws_cnt + row, unsigned(S), &flag)) {
                __syncthreads();
                T m[1] = {T(0)};
                for (int k = tid; k < S; k += NT) m[0] += ld_partial(ws_part + row * S + k);
                cta_sum_rows<NT, 1>(m, red);
                if (tid == 0) y[row] = m[0];
            }
        }
        __syncthreads();
    }
}

}  // namespace adaptic

namespace adaptic {

// Misaligned MV rows, RB rows per CTA step that SHARE their x loads (round 2).  A row's
// head h = (a0 + r C) mod 4 depends on r mod 4 only, so rows r, r + 4, r + 8, ... have the
// same head and read the same shifted copy X_h (XM_SHIFT): a group of RB rows of one residue
// class loads each x vector once for RB rows, where the one-row kernel streamed one x
// vector per A vector (L2 -> SM traffic 2x the matrix bytes).  Groups: g -> class g % 4,
// rows class + 4 (g / 4 * RB + i); splits S per group as in mv_cta_mis_kernel (interleaved
// or contiguous), the same-launch ticket merge per group, scalar head / tail per row by
// split 0.  x is the four shifted copies (x_shift_kernel, same stream, just before).
template <class T, int NT, int U, int RB>
__global__ void __launch_bounds__(NT)
mv_cta_mis_rb_kernel(const T* __restrict__ A, const T* __restrict__ Xs, T* __restrict__ y,
                     int64_t R, int64_t C, int S, int ilv, T* __restrict__ ws_part, unsigned int* __restrict__ ws_cnt)
{
    pdl_prologue();
    using E = vec4_t<T>;
    constexpr int64_t BV = int64_t(NT) * U;
    __shared__ T red[RB * (NT / 32)];
    __shared__ unsigned int flag;
    const int64_t P = xshift_pitch(C);
    const int tid = threadIdx.x;
    const int64_t nb4 = (R + 4 * RB - 1) / (4 * RB);         // groups per residue class
    const int64_t nblk = 4 * nb4 * S;

    for (int64_t blk = blockIdx.x; blk < nblk; blk += gridDim.x) {
        const int64_t g = blk / S;
        const int s = int(blk - g * S);
        const int64_t row0 = (g & 3) + 4 * ((g >> 2) * RB);
        if (row0 >= R) continue;                             // uniform over the group's CTAs
        int64_t rows[RB];
        const E* av[RB];
#pragma unroll
        for (int i = 0; i < RB; ++i) rows[i] = row0 + 4 * i;
        const int h = head_elems(A + row0 * C);
#pragma unroll
        for (int i = 0; i < RB; ++i)
            av[i] = reinterpret_cast<const E*>(A + (rows[i] < R ? rows[i] : row0) * C + h);
        const E* xv = reinterpret_cast<const E*>(Xs + h * P);
        const int64_t nb = (C - h) >> 2;
        const int64_t chunk = (nb + S - 1) / S;
        const int64_t start = ilv ? int64_t(s) * BV : int64_t(s) * chunk;
        const int64_t stride = ilv ? int64_t(S) * BV : BV;
        const int64_t end = ilv ? nb : min(nb, start + chunk);

        E acc[RB][U];
#pragma unroll
        for (int i = 0; i < RB; ++i)
#pragma unroll
            for (int u = 0; u < U; ++u) acc[i][u] = zero_of<E>();
        T outer[RB], edge[RB];
#pragma unroll
        for (int i = 0; i < RB; ++i) { outer[i] = T(0); edge[i] = T(0); }
        int it = 0;
        int64_t b = start;
        for (; b + tid + int64_t(NT) * (U - 1) < end; b += stride) {
            E a[RB][U], x[U];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const int64_t v = b + tid + int64_t(NT) * u;
                x[u] = ld_x(xv + v);
#pragma unroll
                for (int i = 0; i < RB; ++i) a[i][u] = ld_stream(av[i] + v);
            }
#pragma unroll
            for (int i = 0; i < RB; ++i)
#pragma unroll
                for (int u = 0; u < U; ++u) emac(acc[i][u], a[i][u], x[u]);
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
        const int64_t tail_end = min(end, b + BV);
        for (int64_t v = b + tid; v < tail_end; v += NT) {
            const E x = ld_x(xv + v);
#pragma unroll
            for (int i = 0; i < RB; ++i) emac(acc[i][0], ld_stream(av[i] + v), x);
        }
        if (s == 0) {                                        // scalar head and tail of every row
            const int64_t t0 = h + 4 * nb;
            if (tid < h + int(C - t0)) {
                const int64_t c = tid < h ? tid : t0 + (tid - h);
                const T xs = ld_x(Xs + c);                   // copy 0 is x itself
#pragma unroll
                for (int i = 0; i < RB; ++i)
                    if (rows[i] < R) edge[i] = mac(ld_stream(A + rows[i] * C + c), xs, edge[i]);
            }
        }
        T val[RB];
#pragma unroll
        for (int i = 0; i < RB; ++i) val[i] = (outer[i] + esum(tree_sum<U>(acc[i]))) + edge[i];
        cta_sum_rows<NT, RB>(val, red);                      // thread i < RB holds row i

        if (S == 1) {
            if (tid < RB && rows[tid] < R) y[rows[tid]] = val[0];
        } else {
            if (tid < RB && rows[tid] < R) ws_part[rows[tid] * S + s] = val[0];
            if (ticket_is_last(ws_cnt + g, unsigned(S), &flag)) {
                __syncthreads();
                T m[RB];
#pragma unroll
                for (int i = 0; i < RB; ++i) {
                    m[i] = T(0);
                    if (rows[i] < R)
                        for (int k = tid; k < S; k += NT) m[i] += ld_partial(ws_part + rows[i] * S + k);
                }
                cta_sum_rows<NT, RB>(m, red);
                if (tid < RB && rows[tid] < R) y[rows[tid]] = m[0];
            }
        }
        __syncthreads();
    }
}

}  // namespace adaptic

namespace adaptic {

// Misaligned MV rows with x read as TWO aligned 128-bit vectors per body vector and a
// COMPILE-TIME funnel (round 2, XSMEM 9): a row with head h needs x[h + 4v .. h + 4v + 3],
// i.e. words h..h+3 of x4[v] ++ x4[v + 1].  h is the same for the whole row, so the row's
// stream loop is instantiated for h = 0..3 and the funnel is register renaming.  Replaces
// four 32-bit x loads per A vector (XM_LDG: L1-bound) without the shifted-copy pre-kernel
// (XM_SHIFT: 4 C words written per call -- on few long rows as long as the matrix pass
// saves).  Needs a 16-byte-aligned x (launch falls back to XM_LDG).
template <int H, class E> __device__ __forceinline__ E funnel_c(const E& lo, const E& hi) {
    if constexpr (H == 0) return lo;
    else if constexpr (H == 1) return E{lo.y, lo.z, lo.w, hi.x};
    else if constexpr (H == 2) return E{lo.z, lo.w, hi.x, hi.y};
    else return E{lo.w, hi.x, hi.y, hi.z};
}

// x4[q] with the words at or beyond C read one by one (the last vector of x may end past it)
template <class T> __device__ __forceinline__ vec4_t<T> ld_x_end(const T* X, int64_t q, int64_t C) {
    using E = vec4_t<T>;
    if (4 * q + 3 < C) return ld_x(reinterpret_cast<const E*>(X) + q);
    E v = zero_of<E>();
    if (4 * q < C) v.x = ld_x(X + 4 * q);
    if (4 * q + 1 < C) v.y = ld_x(X + 4 * q + 1);
    if (4 * q + 2 < C) v.z = ld_x(X + 4 * q + 2);
    return v;
}

// one row's share [start, end) (stride) of body vectors: the fp32 partial of this thread
template <class T, int NT, int U, int H>
__device__ __forceinline__ T mis_fx_stream(const vec4_t<T>* __restrict__ av, const T* __restrict__ X, int64_t C,
                                           int64_t nb, int64_t start, int64_t stride, int64_t end) {
    using E = vec4_t<T>;
    constexpr int64_t BV = int64_t(NT) * U;
    const E* __restrict__ x4 = reinterpret_cast<const E*>(X);
    const int tid = threadIdx.x;
    E acc[U];
#pragma unroll
    for (int u = 0; u < U; ++u) acc[u] = zero_of<E>();
    T outer = T(0);
    int it = 0;
    const int64_t end_main = min(end, nb - 1);                 // x4[v + 1] inside x for v < nb - 1
    int64_t b = start;
    for (; b + tid + int64_t(NT) * (U - 1) < end_main; b += stride) {
        E a[U], lo[U], hi[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t v = b + tid + int64_t(NT) * u;
            a[u] = ld_stream(av + v);
            lo[u] = ld_x(x4 + v);
            if (H != 0) hi[u] = ld_x(x4 + v + 1);
        }
#pragma unroll
        for (int u = 0; u < U; ++u) emac(acc[u], a[u], funnel_c<H>(lo[u], H != 0 ? hi[u] : lo[u]));
        if (++it == FOLD) {
            it = 0;
            outer += esum(tree_sum<U>(acc));
#pragma unroll
            for (int u = 0; u < U; ++u) acc[u] = zero_of<E>();
        }
    }
    const int64_t tail_end = min(end, b + BV);
    for (int64_t v = b + tid; v < tail_end; v += NT) {
        const E lo = ld_x_end(X, v, C);
        const E hi = H != 0 ? ld_x_end(X, v + 1, C) : lo;
        emac(acc[0], ld_stream(av + v), funnel_c<H>(lo, hi));
    }
    return outer + esum(tree_sum<U>(acc));
}

template <class T, int NT, int U>
__global__ void __launch_bounds__(NT)
mv_cta_mis_fx_kernel(const T* __restrict__ A, const T* __restrict__ X, T* __restrict__ y,
                     int64_t R, int64_t C, int S, int ilv, T* __restrict__ ws_part, unsigned int* __restrict__ ws_cnt)
{
    pdl_prologue();
    using E = vec4_t<T>;
    constexpr int64_t BV = int64_t(NT) * U;
    __shared__ T red[NT / 32];
    __shared__ unsigned int flag;
    const int tid = threadIdx.x;
    const int64_t nblk = R * S;
    for (int64_t blk = blockIdx.x; blk < nblk; blk += gridDim.x) {
        const int64_t row = blk / S;
        const int s = int(blk - row * S);
        const T* rowp = A + row * C;
        const int h = head_elems(rowp);
        const E* av = reinterpret_cast<const E*>(rowp + h);
        const int64_t nb = (C - h) >> 2;
        const int64_t chunk = (nb + S - 1) / S;
        const int64_t start = ilv ? int64_t(s) * BV : int64_t(s) * chunk;
        const int64_t stride = ilv ? int64_t(S) * BV : BV;
        const int64_t end = ilv ? nb : min(nb, start + chunk);
        // the body's x starts at word h (its aligned vectors: x4[v], x4[v + 1] shifted by h)
        T part;
        switch (h) {
            case 0: part = mis_fx_stream<T, NT, U, 0>(av, X, C, nb, start, stride, end); break;
            case 1: part = mis_fx_stream<T, NT, U, 1>(av, X + 0, C, nb, start, stride, end); break;
            case 2: part = mis_fx_stream<T, NT, U, 2>(av, X + 0, C, nb, start, stride, end); break;
            default: part = mis_fx_stream<T, NT, U, 3>(av, X + 0, C, nb, start, stride, end); break;
        }
        T edge = T(0);
        if (s == 0) {                                        // scalar head and tail of the row
            const int64_t t0 = h + 4 * nb;
            if (tid < h + int(C - t0)) {
                const int64_t c = tid < h ? tid : t0 + (tid - h);
                edge = mac(ld_stream(rowp + c), ld_x(X + c), edge);
            }
        }
        T val[1] = {part + edge};
        cta_sum_rows<NT, 1>(val, red);
        if (S == 1) {
            if (tid == 0) y[row] = val[0];
        } else {
            if (tid == 0) ws_part[row * S + s] = val[0];
            if (ticket_is_last(ws_cnt + row, unsigned(S), &flag)) {
                __syncthreads();
                T m[1] = {T(0)};
                for (int k = tid; k < S; k += NT) m[0] += ld_partial(ws_part + row * S + k);
                cta_sum_rows<NT, 1>(m, red);
                if (tid == 0) y[row] = m[0];
            }
        }
        __syncthreads();
    }
}

}  // namespace adaptic
