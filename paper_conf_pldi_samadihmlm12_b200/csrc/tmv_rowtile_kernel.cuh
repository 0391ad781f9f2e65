// tmv_rowtile_kernel.cuh -- TMV with few outputs on TMA-staged tiles of B (sm_100a).
//
// y_r = sum_c B[c, r] x[c] with B (C x R, row-major) short and wide: R <= NT outputs,
// millions of rows c.  When R % 4 != 0 a row of B is not 16-byte aligned, and the
// direct kernels either straddle rows with funnelled 128-bit loads (tmv_mis_kernel:
// every byte through L2 twice) or stream the flat array with per-word x gathers
// (tmv_flat_kernel: 4 scalar x loads per 16 bytes, latency-bound at ~0.55 of peak).
// This kernel is the TMV form of the row-tile kernel (rowtile_kernel.cuh):
//
//  * k consecutive rows of B (k a multiple of 4) are one contiguous run of k*R words;
//    thread 0 bulk-copies its 16-byte-aligned cover and the k matching x values (16-byte
//    aligned since k % 4 == 0) into a STAGES-deep ring, so an SM keeps tens of KB in
//    flight whatever R is.  The matrix's last < 4 words and x's last < 4 values are
//    copied by the threads (nothing is read past either array).
//  * Thread t owns output r = t mod R and row slice s = t div R for the whole kernel
//    (nsl = NT div R slices; R*nsl threads active): it accumulates B[c, r] x[c] over the
//    rows c = s, s + nsl, ... of every tile out of shared memory (consecutive threads,
//    consecutive banks; x[c] is a broadcast), in four interleaved chains folded every
//    FOLD steps (the paper's merged reduction, restructured layout P:354).
//  * The nsl slice partials of a CTA are summed in slice order, the CTA partials are
//    merged by the last CTA of the launch in CTA order (ticket; the paper's second-phase
//    kernel, folded in), so a plan is deterministic.
#pragma once

#include "common.cuh"

namespace adaptic {

constexpr int TRT_MAX_STAGES = 8;
constexpr int TRT_GROUP = 16;       // CTAs per first-level merge group

template <class T, int NT>
__global__ void __launch_bounds__(NT)
tmv_rowtile_kernel(const T* __restrict__ B, const T* __restrict__ X, T* __restrict__ y,
                   int64_t R64, int64_t C, int k, int stages,
                   T* __restrict__ ws_part, unsigned int* __restrict__ ws_cnt)
{
    pdl_prologue();
    extern __shared__ __align__(128) unsigned char smem_raw[];
    __shared__ __align__(8) uint64_t full[TRT_MAX_STAGES];
    __shared__ T P[NT];
    __shared__ unsigned int flag;

    const int R = int(R64);
    const int nsl = NT / R;                             // row slices (R <= NT)
    const int NTa = nsl * R;
    const int tid = threadIdx.x;
    const int r = tid % R, s = tid / R;
    const bool active = tid < NTa;
    const int64_t total = R64 * C;
    const int64_t ntiles = (C + k - 1) / k;
    const int64_t tile_w = ((int64_t(k) * R + 6 + 3) / 4) * 4;   // B words per stage (16-byte multiple)
    const int64_t stage_w = tile_w + k;                           // + x chunk (k % 4 == 0)
    T* ring = reinterpret_cast<T*>(smem_raw);
    const int64_t my_tiles = blockIdx.x < ntiles ? (ntiles - 1 - blockIdx.x) / gridDim.x + 1 : 0;

    if (tid == 0) {
        for (int q = 0; q < stages; ++q) mbar_init(&full[q], 1);
        fence_mbar_init();
    }
    __syncthreads();

    auto issue = [&](int64_t i) {                       // thread 0 only
        const int64_t c0 = (blockIdx.x + i * gridDim.x) * int64_t(k);
        const int64_t nc = min(int64_t(k), C - c0);
        const int64_t w0 = c0 * R64, w1 = (c0 + nc) * R64;
        const int64_t a0 = w0 & ~int64_t(3);
        int64_t a1 = (w1 + 3) & ~int64_t(3);
        if (a1 > total) a1 = w1 & ~int64_t(3);          // last tile: never read past B
        const uint32_t bb = uint32_t((a1 - a0) * int64_t(sizeof(T)));
        const uint32_t xb = uint32_t((nc & ~int64_t(3)) * int64_t(sizeof(T)));
        T* dst = ring + (i % stages) * stage_w;
        uint64_t* bar = &full[i % stages];
        mbar_arrive_expect_tx(bar, bb + xb);
        if (bb) bulk_g2s(dst, B + a0, bb, bar);
        if (xb) bulk_g2s_keep(dst + tile_w, X + c0, xb, bar);
    };
    if (tid == 0) {
        const int64_t pre = min(int64_t(stages), my_tiles);
        for (int64_t i = 0; i < pre; ++i) issue(i);
    }

    T acc[4] = {T(0), T(0), T(0), T(0)};
    T outer = T(0);
    int steps = 0;
    for (int64_t i = 0; i < my_tiles; ++i) {
        const int st = int(i % stages);
        const int64_t c0 = (blockIdx.x + i * gridDim.x) * int64_t(k);
        const int nc = int(min(int64_t(k), C - c0));
        const int64_t w0 = c0 * R64, w1 = w0 + int64_t(nc) * R64;
        T* stg = ring + st * stage_w;
        mbar_wait(&full[st], uint32_t((i / stages) & 1));
        const bool btail = ((w1 + 3) & ~int64_t(3)) > total && (w1 & 3);
        if (btail || (nc & 3)) {                        // last tile only (uniform over the CTA)
            const int64_t a0 = w0 & ~int64_t(3);
            if (btail)
                for (int64_t e = (w1 & ~int64_t(3)) + tid; e < w1; e += NT) stg[e - a0] = B[e];
            for (int c = (nc & ~3) + tid; c < nc; c += NT) stg[tile_w + c] = X[c0 + c];
            __syncthreads();
        }
        if (active) {
            // running 32-bit smem offsets (a stage is < 256 KB): one add per row, no multiplies
            const T* pb = stg + (w0 & 3) + r + s * R;
            const T* px = stg + tile_w + s;
            const int sb = nsl * R;                     // words between a thread's rows
            int c = s;
            for (; c + 3 * nsl < nc; c += 4 * nsl) {
                acc[0] = mac(pb[0], px[0], acc[0]);
                acc[1] = mac(pb[sb], px[nsl], acc[1]);
                acc[2] = mac(pb[2 * sb], px[2 * nsl], acc[2]);
                acc[3] = mac(pb[3 * sb], px[3 * nsl], acc[3]);
                pb += 4 * sb; px += 4 * nsl;
                if (++steps == FOLD) {
                    steps = 0;
                    outer += (acc[0] + acc[1]) + (acc[2] + acc[3]);
                    acc[0] = acc[1] = acc[2] = acc[3] = T(0);
                }
            }
            if (c < nc) acc[0] = mac(pb[0], px[0], acc[0]);                            // < 4 rows left
            if (c + nsl < nc) acc[1] = mac(pb[sb], px[nsl], acc[1]);
            if (c + 2 * nsl < nc) acc[2] = mac(pb[2 * sb], px[2 * nsl], acc[2]);
        }
        __syncthreads();                                // stage st fully read
        if (tid == 0 && i + stages < my_tiles) {
            refill_fence();
            issue(i + stages);
        }
    }

    // slices of this CTA -> one partial per output, in slice order
    P[tid] = active ? outer + ((acc[0] + acc[1]) + (acc[2] + acc[3])) : T(0);
    __syncthreads();
    if (tid < R) {
        T v = T(0);
        for (int q = 0; q < nsl; ++q) v += P[q * R + tid];
        ws_part[int64_t(blockIdx.x) * R + tid] = v;
    }
    // Two-level merge (fixed order at both levels): the last CTA of each group of
    // TRT_GROUP consecutive CTAs sums the group's partials, the last group finisher sums
    // the group partials -- a few dependent L2 round trips instead of G / nsl of them.
    // n partials of R values at src -> P[0 .. R) (thread (r, q) sums rows q, q + nsl, ...
    // eight loads in flight, then the nsl sums per output in q order)
    auto merge = [&](const T* src, int n) {
        T v = T(0);
        if (active) {
            int g = s;
            for (; g + 7 * nsl < n; g += 8 * nsl) {
                T p[8];
#pragma unroll
                for (int u = 0; u < 8; ++u) p[u] = ld_partial(src + int64_t(g + u * nsl) * R + r);
#pragma unroll
                for (int u = 0; u < 8; ++u) v += p[u];
            }
            for (; g < n; g += nsl) v += ld_partial(src + int64_t(g) * R + r);
        }
        __syncthreads();
        P[tid] = v;
        __syncthreads();
        if (tid < R) {
            T tot = T(0);
            for (int q = 0; q < nsl; ++q) tot += P[q * R + tid];
            P[tid] = tot;       // only thread tid reads it back
        }
    };
    const int G = int(gridDim.x);
    const int ngroups = (G + TRT_GROUP - 1) / TRT_GROUP;
    const int grp = int(blockIdx.x) / TRT_GROUP;
    const int gsz = min(TRT_GROUP, G - grp * TRT_GROUP);
    T* gpart = ws_part + int64_t(G) * R;                // group partials: ngroups x R
    if (ticket_is_last(ws_cnt + 1 + grp, unsigned(gsz), &flag)) {
        merge(ws_part + int64_t(grp) * TRT_GROUP * R, gsz);
        if (tid < R) gpart[int64_t(grp) * R + tid] = P[tid];
        if (ticket_is_last(ws_cnt, unsigned(ngroups), &flag)) {
            merge(gpart, ngroups);
            if (tid < R) y[tid] = P[tid];
        }
    }
}

}  // namespace adaptic
