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

// ------------------------------------------------------------------ MV, x tiles in smem (any row length)
// Reduce N = 2^n values across a warp at once (a reduce-scatter butterfly): N - 1 + (5 - n)
// shuffles instead of 5 N.  On return every lane holds the warp total of v[lane >> (5 - n)];
// the addition tree is fixed, so the result is deterministic.
template <int N, class T> __device__ __forceinline__ T warp_multi_sum(T (&v)[N]) {
    static_assert(N >= 1 && N <= 32 && (N & (N - 1)) == 0, "N: power of two <= 32");
    const int lane = threadIdx.x & 31;
    int o = 16;
#pragma unroll
    for (int h = N / 2; h >= 1; h >>= 1, o >>= 1) {
        const bool up = (lane & o) != 0;
#pragma unroll
        for (int i = 0; i < h; ++i) {
            const T send = up ? v[i] : v[i + h];
            const T keep = up ? v[i + h] : v[i];
            v[i] = keep + __shfl_xor_sync(0xffffffffu, send, o);
        }
    }
    T r = v[0];
#pragma unroll
    for (; o >= 1; o >>= 1) r += __shfl_xor_sync(0xffffffffu, r, o);
    return r;
}

// The matrix is cut into column chunks of CW values; the work units are (chunk, row)
// pairs in chunk-major order and CTA b of G owns units [b T / G, (b+1) T / G) (T = nch R),
// so every CTA streams the same number of row segments (no wave tail) and its range is
// a few PIECES (chunk, contiguous rows).  Per piece the K x-chunks (K CW 4 bytes) are
// staged in shared memory by TMA, double-buffered (the next piece's x streams in while
// this one computes); each warp streams RB rows at a time, U 128-bit loads per row in
// flight, every x float4 read from smem feeding RB rows, and reduces the RB K dot
// products with one reduce-scatter butterfly.  A piece with fewer than NW RB rows (few
// long rows) also splits its columns over the idle warps; their sums are combined in
// warp order through shared memory.  One chunk: y is written directly; otherwise
// per-(chunk, row) partials go to the workspace and the CTA that completes a block of MB
// rows (ticket = rows x chunks delivered) sums the chunks in chunk order (G thread groups
// over chunk ranges, second-level accumulator every 32 chunks, groups combined in
// order) -- deterministic, same launch.  x traffic per piece: K CW 4 bytes.
// T = float or uint32_t (int32 modulo 2^32: any order is exact); K > 1 is fp32 only.
template <class T, int K, int RB, int U, int NT>
__global__ void __launch_bounds__(NT, 2)
mmv_tile_kernel(const T* __restrict__ A, const T* __restrict__ X, T* __restrict__ Y,
                int64_t R, int64_t C, int CW, int MB, T* __restrict__ part, unsigned int* __restrict__ cnt)
{
    using V = vec4_t<T>;
    constexpr int N = RB * K;
    constexpr int NW = NT / 32;
    constexpr int LOGN = (N >= 32) ? 5 : (N >= 16) ? 4 : (N >= 8) ? 3 : (N >= 4) ? 2 : (N >= 2) ? 1 : 0;
    static_assert((1 << LOGN) == N, "RB * K must be a power of two");
    pdl_prologue();
    extern __shared__ __align__(128) unsigned char dyn_smem[];
    __shared__ __align__(8) uint64_t xbar[2];
    __shared__ unsigned int s_last[NT];
    __shared__ T s_red[NT];
    __shared__ T s_part[NW][N];
    V* xs0 = reinterpret_cast<V*>(dyn_smem);                   // [2][K][CW / 4]
    const int CWV = CW / 4;
    const int64_t nch = (C + CW - 1) / CW;
    const int64_t TU = nch * R;                                // (chunk, row) units
    const int64_t u_beg = TU * int64_t(blockIdx.x) / gridDim.x;
    const int64_t u_end = TU * (int64_t(blockIdx.x) + 1) / gridDim.x;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int64_t nvr = C / 4;                                  // float4 per matrix row
    const V* __restrict__ Av = reinterpret_cast<const V*>(A);
    auto next_u = [&](int64_t u) {                              // first unit of the following piece
        const int64_t ra = u % R;
        return u + (min(R, ra + (u_end - u)) - ra);
    };
    auto issue = [&](int64_t u, int buf) {                      // thread 0: x chunk of piece u -> buf
        const int64_t c0 = (u / R) * CW;
        const int cw = int(min(int64_t(CW), C - c0));
        mbar_arrive_expect_tx(&xbar[buf], uint32_t(K) * uint32_t(cw) * 4u);
#pragma unroll
        for (int j = 0; j < K; ++j)
            bulk_g2s_keep(xs0 + (buf * K + j) * CWV, X + int64_t(j) * C + c0, uint32_t(cw) * 4u, &xbar[buf]);
    };
    if (threadIdx.x == 0) {
        mbar_init(&xbar[0], 1); mbar_init(&xbar[1], 1);
        fence_mbar_init();
        if (u_beg < u_end) issue(u_beg, 0);
        const int64_t u1 = u_beg < u_end ? next_u(u_beg) : u_end;
        if (u1 < u_end) issue(u1, 1);
    }
    __syncthreads();
    int k = 0;
    for (int64_t u = u_beg; u < u_end; ++k) {
        const int64_t ch = u / R;
        const int64_t ra = u - ch * R;
        const int64_t rb = min(R, ra + (u_end - u));
        const int64_t c0 = ch * CW;
        const int nvv = int(min(int64_t(CW), C - c0)) / 4;
        const int buf = k & 1;
        const V* xs = xs0 + buf * K * CWV;
        mbar_wait(&xbar[buf], uint32_t((k >> 1) & 1));
        const int nrg = int((rb - ra + RB - 1) / RB);           // row groups of this piece
        const int cs = nrg >= NW ? 1 : NW / nrg;                // warps per row group
        const int rg_first = cs == 1 ? warp : warp % nrg;
        const int sub = cs == 1 ? 0 : warp / nrg;
        const int v_lo = int(int64_t(nvv) * sub / cs), v_hi = int(int64_t(nvv) * (sub + 1) / cs);
        for (int rg = rg_first; rg < nrg && sub < cs; rg += (cs == 1 ? NW : nrg)) {
            const int64_t r0 = ra + int64_t(rg) * RB;
            const V* rowp[RB];
#pragma unroll
            for (int i = 0; i < RB; ++i) rowp[i] = Av + (r0 + i < rb ? r0 + i : r0) * nvr + c0 / 4;
            T acc[RB][K];
#pragma unroll
            for (int i = 0; i < RB; ++i)
#pragma unroll
                for (int j = 0; j < K; ++j) acc[i][j] = T(0);
            int v = v_lo + lane;
            for (; v + 32 * (U - 1) < v_hi; v += 32 * U) {
                V a[RB][U];
#pragma unroll
                for (int uu = 0; uu < U; ++uu)
#pragma unroll
                    for (int i = 0; i < RB; ++i) a[i][uu] = ld_stream(rowp[i] + v + 32 * uu);
#pragma unroll
                for (int uu = 0; uu < U; ++uu)
#pragma unroll
                    for (int j = 0; j < K; ++j) {
                        const V xv = xs[j * CWV + v + 32 * uu];
#pragma unroll
                        for (int i = 0; i < RB; ++i) {
                            T t = acc[i][j];
                            t = mac(a[i][uu].x, xv.x, t);
                            t = mac(a[i][uu].y, xv.y, t);
                            t = mac(a[i][uu].z, xv.z, t);
                            acc[i][j] = mac(a[i][uu].w, xv.w, t);
                        }
                    }
            }
            for (; v < v_hi; v += 32) {
                V a[RB];
#pragma unroll
                for (int i = 0; i < RB; ++i) a[i] = ld_stream(rowp[i] + v);
#pragma unroll
                for (int j = 0; j < K; ++j) {
                    const V xv = xs[j * CWV + v];
#pragma unroll
                    for (int i = 0; i < RB; ++i) {
                        T t = acc[i][j];
                        t = mac(a[i].x, xv.x, t);
                        t = mac(a[i].y, xv.y, t);
                        t = mac(a[i].z, xv.z, t);
                        acc[i][j] = mac(a[i].w, xv.w, t);
                    }
                }
            }
            T flat[N];
#pragma unroll
            for (int i = 0; i < RB; ++i)
#pragma unroll
                for (int j = 0; j < K; ++j) flat[i * K + j] = acc[i][j];
            const T tot = warp_multi_sum<N>(flat);
            const int idx = lane >> (5 - LOGN);
            if ((lane & ((1 << (5 - LOGN)) - 1)) == 0) {
                if (cs > 1) {
                    s_part[warp][idx] = tot;
                } else {
                    const int i = idx / K, j = idx - (idx / K) * K;
                    const int64_t row = r0 + i;
                    if (row < rb) {
                        if (nch == 1) Y[int64_t(j) * R + row] = tot;
                        else part[(ch * K + j) * R + row] = tot;
                    }
                }
            }
        }
        if (cs > 1) {                                           // combine the column splits in warp order
            __syncthreads();
            for (int t = threadIdx.x; t < nrg * N; t += NT) {
                const int rg = t / N, idx = t - rg * N;
                T s = T(0);
                for (int q = 0; q < cs; ++q) s += s_part[q * nrg + rg][idx];
                const int i = idx / K, j = idx - (idx / K) * K;
                const int64_t row = ra + int64_t(rg) * RB + i;
                if (row < rb) {
                    if (nch == 1) Y[int64_t(j) * R + row] = s;
                    else part[(ch * K + j) * R + row] = s;
                }
            }
        }
        if (nch > 1) {
            // tickets: rows x chunks delivered per block of MB rows
            __threadfence();
            __syncthreads();
            const int64_t b0 = ra / MB, b1 = (rb - 1) / MB;
            for (int64_t bb = b0; bb <= b1; bb += NT) {
                const int64_t blk = bb + threadIdx.x;
                unsigned int last = 0u;
                if (blk <= b1) {
                    const int64_t lo = blk * MB, hi = min(R, lo + MB);
                    const unsigned int mine = unsigned(min(hi, rb) - max(lo, ra));
                    const unsigned int need = unsigned(hi - lo) * unsigned(nch);
                    const unsigned int old = atomicAdd(cnt + blk, mine);
                    if (old + mine == need) { cnt[blk] = 0u; last = 1u; }
                }
                s_last[threadIdx.x] = last;
                __syncthreads();
                __threadfence();
                const int nb = int(min(int64_t(NT), b1 - bb + 1));
                for (int q = 0; q < nb; ++q) {
                    if (!s_last[q]) continue;
                    const int64_t lo = (bb + q) * MB, hi = min(R, lo + MB);
                    const int rows = int(hi - lo);
                    const int E = K * rows;                     // outputs of the block
                    const int G = E <= NT ? NT / E : 1;         // thread groups over chunk ranges
                    for (int e0 = 0; e0 < E; e0 += NT) {
                        const int e = G > 1 ? int(threadIdx.x) % E : e0 + int(threadIdx.x);
                        const int g = G > 1 ? int(threadIdx.x) / E : 0;
                        T val = T(0);
                        if (g < G && e < E) {
                            const int j = e / rows;
                            const int64_t r = lo + (e - j * rows);
                            const int64_t c_lo = nch * g / G, c_hi = nch * (g + 1) / G;
                            T outer = T(0), inner = T(0);
                            int n32 = 0;
#pragma unroll 8
                            for (int64_t c = c_lo; c < c_hi; ++c) {
                                inner += ld_partial(part + (c * K + j) * R + r);
                                if (++n32 == 32) { outer += inner; inner = T(0); n32 = 0; }
                            }
                            val = outer + inner;
                        }
                        s_red[threadIdx.x] = val;
                        __syncthreads();
                        const int ne = G > 1 ? E : min(E - e0, NT);
                        if (int(threadIdx.x) < ne) {
                            T t = T(0);
                            for (int gg = 0; gg < G; ++gg) t += s_red[gg * E + int(threadIdx.x)];
                            const int ee = e0 + int(threadIdx.x);
                            const int j = ee / rows;
                            Y[int64_t(j) * R + lo + (ee - j * rows)] = t;
                        }
                        __syncthreads();
                    }
                }
                __syncthreads();
            }
        }
        __syncthreads();                                        // every warp is done with xs[buf]
        const int64_t un = u + (rb - ra);
        if (threadIdx.x == 0 && un < u_end) {
            const int64_t u2 = next_u(un);
            if (u2 < u_end) { fence_proxy_async(); issue(u2, buf); }
        }
        u = un;
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

// ------------------------------------------------------------------ TMV tiles, rows in groups of 4 (round 2)
// tmmv_kernel reads x_j[c] as K scalar loads per row (K U loads of x next to U of B per
// iteration: 20 load instructions for 64 FMA at K = U = 4) and keeps U B-vectors in flight in
// registers beside 2K accumulators (ncu: 118-128 registers, 22-25 % occupancy, 0.73-0.76 of
// the copy peak).  Here a c-lane walks GROUPS of 4 consecutive rows, so x_j[4g .. 4g+3] is
// ONE 128-bit load per vector (K loads per 4 rows, 4x fewer), and (PF > 0) every thread
// prefetches its B vectors PF groups ahead into L2 (prefetch.global.L2: no register holds
// the bytes in flight, the later load waits for an L2 hit instead of DRAM).  Needs C % 4 == 0
// and a 16-byte-aligned X (planner); splits cut C at multiples of 4 rows.
__device__ __forceinline__ void prefetch_l2(const void* p) {
    asm volatile("prefetch.global.L2::evict_last [%0];" :: "l"(p));
}

template <int K, int LR, int PF, int NT>
__global__ void __launch_bounds__(NT, 2)
tmmv4_kernel(const float* __restrict__ B, const float* __restrict__ X, float* __restrict__ Y,
             int64_t R, int64_t C, int S, float* __restrict__ ws_part, unsigned int* __restrict__ ws_cnt)
{
    pdl_prologue();
    constexpr int LC = NT / LR;
    __shared__ float4 red[LC > 1 ? NT : 1];
    __shared__ unsigned int flag;
    const int64_t rv = R / 4;
    const int64_t ntiles = (rv + LR - 1) / LR;
    const int64_t ngr = C / 4;                        // groups of 4 rows of B
    const int64_t gchunk = (ngr + S - 1) / S;
    const float4* __restrict__ Bv = reinterpret_cast<const float4*>(B);
    const float4* __restrict__ Xv = reinterpret_cast<const float4*>(X);
    const int tid = threadIdx.x;
    const int lr = tid % LR, lc = tid / LR;
    const int64_t nblk = ntiles * S;

    for (int64_t blk = blockIdx.x; blk < nblk; blk += gridDim.x) {
        const int64_t tile = blk % ntiles;
        const int s = int(blk / ntiles);
        const int64_t r4 = tile * LR + lr;
        const bool rok = r4 < rv;
        const int64_t g0 = int64_t(s) * gchunk;
        const int64_t g1 = min(ngr, g0 + gchunk);
        float4 acc[K], outer[K];
#pragma unroll
        for (int j = 0; j < K; ++j) { acc[j] = make_float4(0.f, 0.f, 0.f, 0.f); outer[j] = acc[j]; }
        int it = 0;
        const float4* __restrict__ Bc = Bv + (rok ? r4 : 0);
        for (int64_t g = g0 + lc; g < g1; g += LC) {
            if (PF > 0 && g + int64_t(PF) * LC < g1) {
#pragma unroll
                for (int u = 0; u < 4; ++u) prefetch_l2(Bc + (4 * (g + int64_t(PF) * LC) + u) * rv);
            }
            float4 b[4];
#pragma unroll
            for (int u = 0; u < 4; ++u) b[u] = ld_stream(Bc + (4 * g + u) * rv);
            float4 xv[K];
#pragma unroll
            for (int j = 0; j < K; ++j) xv[j] = ld_x(Xv + (int64_t(j) * C) / 4 + g);
#pragma unroll
            for (int j = 0; j < K; ++j) {
                vmacs(acc[j], b[0], xv[j].x);
                vmacs(acc[j], b[1], xv[j].y);
                vmacs(acc[j], b[2], xv[j].z);
                vmacs(acc[j], b[3], xv[j].w);
            }
            if (++it == FOLD / 4) {
                it = 0;
#pragma unroll
                for (int j = 0; j < K; ++j) { outer[j] = eadd(outer[j], acc[j]); acc[j] = make_float4(0.f, 0.f, 0.f, 0.f); }
            }
        }
        float4* yv = reinterpret_cast<float4*>(Y);
        float4* pv = reinterpret_cast<float4*>(ws_part);
#pragma unroll
        for (int j = 0; j < K; ++j) {
            float4 tot = lc_combine<NT, LR>(eadd(outer[j], acc[j]), red);
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
                float4 m = make_float4(0.f, 0.f, 0.f, 0.f);
                if (rok) m = merge_partials<LC>(pv + int64_t(j) * rv + r4, int64_t(K) * rv, lc, S);
                m = lc_combine<NT, LR>(m, red);
                if (tid < LR && rok) yv[j * rv + r4] = m;
                __syncthreads();
            }
        }
        __syncthreads();
    }
}

// ------------------------------------------------------------------ TMV tiles, TMA-staged
// Same tiling and split/merge as tmmv_kernel, but the B rows of a (tile, split) block
// arrive in shared memory by TMA bulk copies (one per B row segment of 16 LR bytes,
// issued by the lanes of warp 0) into an ST-deep ring of CR-row stages, so the bytes in
// flight (ST CR LR 16 per CTA) no longer cost registers: with K accumulators per
// thread the register-fed kernel kept only U = 4 float4 in flight per thread and was
// latency-bound (ncu: long-scoreboard stalls, 16 warps/SM, ~4.3 TB/s).  The ring runs
// across the CTA's blocks (stage i + ST is issued as soon as stage i is consumed).
// Threads read b = stage[row][lr] (a warp reads 32 consecutive float4, conflict-free)
// and x_j[c] through L1 (one broadcast per warp when LR >= 32).  When one tile covers
// all outputs (R <= 4 LR) consecutive B rows are contiguous and a stage is ONE bulk copy
// (row pitch R/4 in shared memory): per-row copies of a few hundred bytes ran at 1.9 TB/s.
template <int K, int LR, int NT>
__global__ void __launch_bounds__(NT, 2)
tmmv_tma_kernel(const float* __restrict__ B, const float* __restrict__ X, float* __restrict__ Y,
                int64_t R, int64_t C, int S, float* __restrict__ ws_part, unsigned int* __restrict__ ws_cnt)
{
    pdl_prologue();
    constexpr int LC = NT / LR;
    constexpr int CR = TMMV_TMA_STAGE_V4 / LR;           // B rows per stage
    constexpr int ST = TMMV_TMA_STAGES;
    static_assert(CR % LC == 0 && CR >= LC, "stage rows: a multiple of the c-lanes");
    extern __shared__ __align__(128) unsigned char dyn_smem[];
    float4* ring = reinterpret_cast<float4*>(dyn_smem);  // [ST][CR][LR]
    __shared__ __align__(8) uint64_t full[ST];
    __shared__ float4 red[LC > 1 ? NT : 1];
    __shared__ float4 s_merge[NT];
    __shared__ unsigned int flag;
    const int64_t rv = R / 4;
    const int64_t ntiles = (rv + LR - 1) / LR;
    const int64_t chunk = (C + S - 1) / S;
    const float4* __restrict__ Bv = reinterpret_cast<const float4*>(B);
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int lr = tid % LR, lc = tid / LR;
    const int64_t nblk = ntiles * S;
    const int64_t my_blks = blockIdx.x < nblk ? (nblk - 1 - blockIdx.x) / gridDim.x + 1 : 0;
    auto geom = [&](int64_t m, int64_t& tile, int& s, int64_t& c0, int64_t& c1, int& w) {
        const int64_t blk = blockIdx.x + m * gridDim.x;
        tile = blk % ntiles;
        s = int(blk / ntiles);
        c0 = min(C, int64_t(s) * chunk);
        c1 = min(C, c0 + chunk);
        w = int(min(int64_t(LR), rv - tile * LR));
    };
    // producer (warp 0, uniform state): next (block, stage) to issue
    int64_t pm = 0, pst = 0, issued = 0;
    auto produce = [&]() {
        int64_t tile, c0, c1, nst = 0; int s, w;
        for (; pm < my_blks; ++pm) {                      // skip empty splits
            geom(pm, tile, s, c0, c1, w);
            nst = (c1 - c0 + CR - 1) / CR;
            if (nst > 0) break;
        }
        if (pm >= my_blks) return;
        const int64_t r_lo = c0 + pst * CR;
        const int nr = int(min(int64_t(CR), c1 - r_lo));
        const int slot = int(issued % ST);
        if (lane == 0) mbar_arrive_expect_tx(&full[slot], uint32_t(nr) * uint32_t(w) * 16u);
        __syncwarp();
        fence_proxy_async();
        if (ntiles == 1) {                                // whole rows: the stage is one contiguous block
            if (lane == 0)
                bulk_g2s(ring + size_t(slot) * CR * LR, Bv + r_lo * rv, uint32_t(nr) * uint32_t(w) * 16u, &full[slot]);
        } else {
            for (int q = lane; q < nr; q += 32)
                bulk_g2s(ring + (size_t(slot) * CR + q) * LR, Bv + (r_lo + q) * rv + tile * LR, uint32_t(w) * 16u, &full[slot]);
        }
        ++issued;
        if (++pst == nst) { pst = 0; ++pm; }
    };
    if (tid == 0) {
        for (int i = 0; i < ST; ++i) mbar_init(&full[i], 1);
        fence_mbar_init();
    }
    __syncthreads();
    if (warp == 0)
        while (issued < ST && pm < my_blks) produce();
    int64_t consumed = 0;
    float4* yv = reinterpret_cast<float4*>(Y);
    float4* pv = reinterpret_cast<float4*>(ws_part);
    for (int64_t m = 0; m < my_blks; ++m) {
        int64_t tile, c0, c1; int s, w;
        geom(m, tile, s, c0, c1, w);
        const int64_t nst = (c1 - c0 + CR - 1) / CR;
        const int64_t r4 = tile * LR + lr;
        const bool rok = lr < w;
        float4 acc[K], outer[K];
#pragma unroll
        for (int j = 0; j < K; ++j) { acc[j] = make_float4(0.f, 0.f, 0.f, 0.f); outer[j] = acc[j]; }
        int rows_acc = 0;
        for (int64_t st = 0; st < nst; ++st, ++consumed) {
            const int slot = int(consumed % ST);
            const int64_t r_lo = c0 + st * CR;
            const int nr = int(min(int64_t(CR), c1 - r_lo));
            mbar_wait(&full[slot], uint32_t((consumed / ST) & 1));
            const float4* sb = ring + size_t(slot) * CR * LR;
            const int P = ntiles == 1 ? w : LR;           // smem row pitch (float4)
            if (rok) {
                if (nr == CR) {
#pragma unroll (K <= 4 ? 4 : 2)
                    for (int q = lc; q < CR; q += LC) {
                        const float4 b = sb[q * P + lr];
#pragma unroll
                        for (int j = 0; j < K; ++j) esmac(acc[j], b, ld_x(X + j * C + r_lo + q));
                    }
                } else {
                    for (int q = lc; q < nr; q += LC) {
                        const float4 b = sb[q * P + lr];
#pragma unroll
                        for (int j = 0; j < K; ++j) esmac(acc[j], b, ld_x(X + j * C + r_lo + q));
                    }
                }
            }
            rows_acc += CR / LC;
            if (rows_acc >= FOLD) {                       // bounded fp32 chains (planner: chain_of)
                rows_acc = 0;
#pragma unroll
                for (int j = 0; j < K; ++j) { outer[j] = eadd(outer[j], acc[j]); acc[j] = make_float4(0.f, 0.f, 0.f, 0.f); }
            }
            __syncthreads();                              // every thread is done with the slot
            if (warp == 0 && pm < my_blks) produce();
        }
#pragma unroll
        for (int j = 0; j < K; ++j) {
            const float4 tot = lc_combine<NT, LR>(eadd(outer[j], acc[j]), red);
            if (S == 1) {
                if (tid < LR && rok) yv[j * rv + r4] = tot;
            } else if (tid < LR && rok) {
                pv[(int64_t(s) * K + j) * rv + r4] = tot;
            }
            __syncthreads();                              // red[] reuse by the next vector
        }
        if (S > 1 && ticket_is_last(ws_cnt + tile, unsigned(S), &flag)) {
            // O = K w float4 outputs x S partials: G = NT / O thread groups each sum a contiguous
            // slot range with 4 independent accumulators, then the groups combine in order
            const int O = K * w;
            const int G = O <= NT ? NT / O : 1;
            for (int o0 = 0; o0 < O; o0 += NT) {
                const int o = G > 1 ? tid % O : o0 + tid;
                const int g = G > 1 ? tid / O : 0;
                float4 mm = make_float4(0.f, 0.f, 0.f, 0.f);
                if (g < G && o < O) {
                    const int j = o / w, q = o - (o / w) * w;
                    const float4* base = pv + int64_t(j) * rv + tile * LR + q;
                    const int64_t stride = int64_t(K) * rv;
                    const int64_t s_lo = int64_t(S) * g / G, s_hi = int64_t(S) * (g + 1) / G;
                    float4 m1 = mm, m2 = mm, m3 = mm;
                    int64_t sl = s_lo;
                    for (; sl + 3 < s_hi; sl += 4) {
                        const float4 t0 = ld_partial(base + sl * stride), t1 = ld_partial(base + (sl + 1) * stride);
                        const float4 t2 = ld_partial(base + (sl + 2) * stride), t3 = ld_partial(base + (sl + 3) * stride);
                        mm = eadd(mm, t0); m1 = eadd(m1, t1); m2 = eadd(m2, t2); m3 = eadd(m3, t3);
                    }
                    for (; sl < s_hi; ++sl) mm = eadd(mm, ld_partial(base + sl * stride));
                    mm = eadd(eadd(mm, m1), eadd(m2, m3));
                }
                s_merge[tid] = mm;
                __syncthreads();
                const int no = G > 1 ? O : min(O - o0, NT);
                if (tid < no) {
                    float4 t = make_float4(0.f, 0.f, 0.f, 0.f);
                    for (int gg = 0; gg < G; ++gg) t = eadd(t, s_merge[gg * (G > 1 ? O : 0) + tid]);
                    const int oo = o0 + tid;
                    const int j = oo / w, q = oo - (oo / w) * w;
                    yv[int64_t(j) * rv + tile * LR + q] = t;
                }
                __syncthreads();
            }
        }
        __syncthreads();
    }
}

}  // namespace adaptic
