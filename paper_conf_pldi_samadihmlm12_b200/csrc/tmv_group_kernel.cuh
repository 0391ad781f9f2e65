// tmv_group_kernel.cuh -- TMV with rows off the 16-byte grid (R % 4 != 0, R <= 4096) on
// groups of four rows, sm_100a.  TMV_REGTILE / TMV_SPLITK with [ADAPTIC_P_XSMEM] = 12.
//
// y_r = sum_c B[c][r] x[c] (the TMV actor; B is C x R, row-major).  Four
// consecutive rows of B are 4R words = R whole 128-bit vectors, so on a 16-byte-aligned B
// every group of four rows starts on the 16-byte grid whatever R mod 4 is.  Word 4v + j of
// a group (vector v, component j) is output (4v + j) mod R of the group's row
// (4v + j) div R: the SAME pair for every group.  A thread that owns slot v for the whole
// kernel therefore streams one aligned vector per group into four accumulators with fixed
// outputs, and needs only x[4g + k] and x[4g + k + 1] (k = 4v div R: a vector's four words
// cross at most one row boundary when R >= 4).  No funnel, no shared-memory staging, no
// re-read vector: the instruction mix of the aligned kernels, ~one 128-bit load, two
// broadcast x loads and four FMAs per 16 bytes of B.
//
//   * R < NT: a CTA step covers KG = NT div R consecutive groups (thread t: slot t mod R of
//     group t div R; KG R threads active), S = 1.
//   * R > NT: S slots per thread (v = t, t + NT, ...), one group per step.
// A CTA streams a contiguous range of groups (a contiguous range of B), or ([ORDER] 2) the
// CTAs interleave so that the grid reads one window of consecutive groups per step.  Per CTA the four
// words of every output (k = 0..3) and the KG sub-groups are summed in a fixed order
// through shared memory; the CTA partials are merged in two fixed-order levels by ticket
// (groups of TG_GROUP CTAs, then the group partials: the paper's second merge kernel, P:480,
// folded into the launch).  The last < 4 rows (C mod 4) are added by the final merger.
#pragma once

#include "common.cuh"
#include "launch.h"

namespace adaptic {

constexpr int TG_GROUP = 16;        // CTAs per first-level merge group

template <class T, int S, int U, int MAXNT>
__global__ void __launch_bounds__(MAXNT, 1)
tmv_group_kernel(const T* __restrict__ B, const T* __restrict__ X, T* __restrict__ y,
                 int64_t R64, int64_t C, int ilv, T* __restrict__ ws_part, unsigned int* __restrict__ ws_cnt)
{
    pdl_prologue();
    using E = vec4_t<T>;
    __shared__ T P[4 * MAXNT * S];
    __shared__ unsigned int flag;
    const int R = int(R64);
    const int NT = int(blockDim.x);
    const int tid = int(threadIdx.x);
    const int KG = S == 1 ? max(1, NT / R) : 1;            // groups per CTA step
    const int sub = S == 1 ? tid / R : 0;
    const int64_t NG = C >> 2;                              // whole groups of four rows
    const int64_t G = gridDim.x, b = blockIdx.x;
    const int64_t per = NG / G, rem = NG % G;
    // ilv = 0: this CTA's groups are the contiguous range [g0, g1); ilv = 1: groups
    // (b + n G) KG + sub (a grid-wide window of G KG consecutive groups per step)
    const int64_t g0 = ilv ? b * KG : b * per + min(b, rem);
    const int64_t g1 = ilv ? NG : g0 + per + (b < rem ? 1 : 0);
    const int64_t gs = ilv ? G * KG : int64_t(KG);          // a thread's group stride

    int v[S], kr[S];
    bool ok[S], h1[S], h2[S], h3[S], hx[S];
#pragma unroll
    for (int i = 0; i < S; ++i) {
        v[i] = S == 1 ? tid % R : tid + i * NT;
        ok[i] = S == 1 ? (tid < KG * R) : (v[i] < R);
        kr[i] = ok[i] ? (4 * v[i]) / R : 0;
        const int js = (kr[i] + 1) * R - 4 * v[i];         // words of the vector in row kr (>= 1)
        h1[i] = js <= 1; h2[i] = js <= 2; h3[i] = js <= 3; hx[i] = ok[i] && js < 4;
    }
    T acc[S][4], outer[S][4];
#pragma unroll
    for (int i = 0; i < S; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) { acc[i][j] = T(0); outer[i][j] = T(0); }

    const E* __restrict__ Bv = reinterpret_cast<const E*>(B);
    const int64_t stepv = gs * R;                           // vectors between a thread's groups
    const int64_t stepx = 4 * gs;
    int64_t g = g0 + sub;
    const E* pb = Bv + g * R;
    const T* px = X + 4 * g;
    int it = 0;
    for (; g + gs * (U - 1) < g1; g += gs * U) {
        E a[U][S];
        T xl[U][S], xh[U][S];
#pragma unroll
        for (int u = 0; u < U; ++u)
#pragma unroll
            for (int i = 0; i < S; ++i) {
                if (ok[i]) {
                    a[u][i] = ld_stream(pb + stepv * u + v[i]);
                    xl[u][i] = ld_x(px + stepx * u + kr[i]);
                    xh[u][i] = hx[i] ? ld_x(px + stepx * u + kr[i] + 1) : T(0);
                } else {
                    a[u][i] = vzero<E>(); xl[u][i] = T(0); xh[u][i] = T(0);
                }
            }
#pragma unroll
        for (int u = 0; u < U; ++u)
#pragma unroll
            for (int i = 0; i < S; ++i) {
                acc[i][0] = mac(a[u][i].x, xl[u][i], acc[i][0]);
                acc[i][1] = mac(a[u][i].y, h1[i] ? xh[u][i] : xl[u][i], acc[i][1]);
                acc[i][2] = mac(a[u][i].z, h2[i] ? xh[u][i] : xl[u][i], acc[i][2]);
                acc[i][3] = mac(a[u][i].w, h3[i] ? xh[u][i] : xl[u][i], acc[i][3]);
            }
        pb += stepv * U;
        px += stepx * U;
        if (++it == FOLD / U) {
            it = 0;
#pragma unroll
            for (int i = 0; i < S; ++i)
#pragma unroll
                for (int j = 0; j < 4; ++j) { outer[i][j] += acc[i][j]; acc[i][j] = T(0); }
        }
    }
    for (; g < g1; g += gs) {                               // < U groups left
#pragma unroll
        for (int i = 0; i < S; ++i) {
            if (!ok[i]) continue;
            const E a = ld_stream(pb + v[i]);
            const T xl = ld_x(px + kr[i]);
            const T xh = hx[i] ? ld_x(px + kr[i] + 1) : T(0);
            acc[i][0] = mac(a.x, xl, acc[i][0]);
            acc[i][1] = mac(a.y, h1[i] ? xh : xl, acc[i][1]);
            acc[i][2] = mac(a.z, h2[i] ? xh : xl, acc[i][2]);
            acc[i][3] = mac(a.w, h3[i] ? xh : xl, acc[i][3]);
        }
        pb += stepv;
        px += stepx;
    }

    // word position 4v + j of sub-group `sub` -> P[sub 4R + 4v + j]; output r collects the
    // positions k R + r (k = 0..3) of every sub-group, in (sub, k) order
#pragma unroll
    for (int i = 0; i < S; ++i)
        if (ok[i])
#pragma unroll
            for (int j = 0; j < 4; ++j) P[(sub * R + v[i]) * 4 + j] = outer[i][j] + acc[i][j];
    __syncthreads();
    for (int r = tid; r < R; r += NT) {
        T s = T(0);
        for (int q = 0; q < KG; ++q) {
            const T* pq = P + q * 4 * R + r;
            s += ((pq[0] + pq[R]) + (pq[2 * R] + pq[3 * R]));
        }
        ws_part[b * R + r] = s;
    }

    // n partials of R values at src, summed in order (eight loads in flight) -> dst
    auto merge = [&](const T* src, int n, T* dst, bool tail) {
        for (int r = tid; r < R; r += NT) {
            T s = T(0);
            int q = 0;
            for (; q + 7 < n; q += 8) {
                T p[8];
#pragma unroll
                for (int u = 0; u < 8; ++u) p[u] = ld_partial(src + int64_t(q + u) * R + r);
#pragma unroll
                for (int u = 0; u < 8; ++u) s += p[u];
            }
            for (; q < n; ++q) s += ld_partial(src + int64_t(q) * R + r);
            if (tail)                                        // rows 4 NG .. C - 1
                for (int64_t c = 4 * NG; c < C; ++c) s = mac(ld_stream(B + c * R64 + r), ld_x(X + c), s);
            dst[r] = s;
        }
    };
    const int Gi = int(G);
    const int ngroups = (Gi + TG_GROUP - 1) / TG_GROUP;
    const int grp = int(b) / TG_GROUP;
    const int gsz = min(TG_GROUP, Gi - grp * TG_GROUP);
    T* gpart = ws_part + G * R64;                            // group partials: ngroups x R
    if (ticket_is_last(ws_cnt + 1 + grp, unsigned(gsz), &flag)) {
        merge(ws_part + int64_t(grp) * TG_GROUP * R64, gsz, gpart + int64_t(grp) * R64, false);
        if (ticket_is_last(ws_cnt, unsigned(ngroups), &flag))
            merge(gpart, ngroups, y, true);
    }
}

}  // namespace adaptic
