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

template <class T, int NT, int RPT>
__global__ void __launch_bounds__(NT)
tmv_rowtile_kernel(const T* __restrict__ B, const T* __restrict__ X, T* __restrict__ y,
                   int64_t R64, int64_t C, int k, int stages,
                   T* __restrict__ ws_part, unsigned int* __restrict__ ws_cnt)
{
    pdl_prologue();
    extern __shared__ __align__(128) unsigned char smem_raw[];
    __shared__ __align__(8) uint64_t full[TRT_MAX_STAGES];
    constexpr int VT = NT * RPT;                        // virtual threads: tid + j NT, j < RPT
    __shared__ T P[VT];
    __shared__ unsigned int flag;

    const int R = int(R64);
    const int nsl = VT / R;                             // row slices (R <= VT)
    const int NTa = nsl * R;
    const int tid = threadIdx.x;
    int rj[RPT], sj[RPT];
    bool act[RPT];
#pragma unroll
    for (int j = 0; j < RPT; ++j) {
        const int vt = tid + j * NT;
        rj[j] = vt % R; sj[j] = vt / R; act[j] = vt < NTa;
    }
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

    auto issue = [&](int64_t i, int slot) {             // thread 0 only; tile i -> ring stage slot
        const int64_t c0 = (blockIdx.x + i * gridDim.x) * int64_t(k);
        const int64_t nc = min(int64_t(k), C - c0);
        const int64_t w0 = c0 * R64, w1 = (c0 + nc) * R64;
        const int64_t a0 = w0 & ~int64_t(3);
        int64_t a1 = (w1 + 3) & ~int64_t(3);
        if (a1 > total) a1 = w1 & ~int64_t(3);          // last tile: never read past B
        const uint32_t bb = uint32_t((a1 - a0) * int64_t(sizeof(T)));
        const uint32_t xb = uint32_t((nc & ~int64_t(3)) * int64_t(sizeof(T)));
        T* dst = ring + slot * stage_w;
        uint64_t* bar = &full[slot];
        mbar_arrive_expect_tx(bar, bb + xb);
        if (bb) bulk_g2s(dst, B + a0, bb, bar);
        if (xb) bulk_g2s_keep(dst + tile_w, X + c0, xb, bar);
    };
    if (tid == 0) {
        const int64_t pre = min(int64_t(stages), my_tiles);
        for (int64_t i = 0; i < pre; ++i) issue(i, int(i));
    }

    T acc[RPT][4], outer[RPT];
#pragma unroll
    for (int j = 0; j < RPT; ++j) { acc[j][0] = acc[j][1] = acc[j][2] = acc[j][3] = T(0); outer[j] = T(0); }
    int steps[RPT];
#pragma unroll
    for (int j = 0; j < RPT; ++j) steps[j] = 0;
    int st = 0;
    uint32_t ph = 0;
    for (int64_t i = 0; i < my_tiles; ++i, ring_advance(st, ph, stages)) {
        const int64_t c0 = (blockIdx.x + i * gridDim.x) * int64_t(k);
        const int nc = int(min(int64_t(k), C - c0));
        const int64_t w0 = c0 * R64, w1 = w0 + int64_t(nc) * R64;
        T* stg = ring + st * stage_w;
        mbar_wait(&full[st], ph);
        const bool btail = ((w1 + 3) & ~int64_t(3)) > total && (w1 & 3);
        if (btail || (nc & 3)) {                        // last tile only (uniform over the CTA)
            const int64_t a0 = w0 & ~int64_t(3);
            if (btail)
                for (int64_t e = (w1 & ~int64_t(3)) + tid; e < w1; e += NT) stg[e - a0] = B[e];
            for (int c = (nc & ~3) + tid; c < nc; c += NT) stg[tile_w + c] = X[c0 + c];
            __syncthreads();
        }
#pragma unroll
        for (int j = 0; j < RPT; ++j) {
            if (!act[j]) continue;
            // running 32-bit smem offsets (a stage is < 256 KB): one add per row, no multiplies
            const T* pb = stg + (w0 & 3) + rj[j] + sj[j] * R;
            const T* px = stg + tile_w + sj[j];
            const int sb = nsl * R;                     // words between a thread's rows
            T* a = acc[j];
            int c = sj[j];
            for (; c + 3 * nsl < nc; c += 4 * nsl) {
                a[0] = mac(pb[0], px[0], a[0]);
                a[1] = mac(pb[sb], px[nsl], a[1]);
                a[2] = mac(pb[2 * sb], px[2 * nsl], a[2]);
                a[3] = mac(pb[3 * sb], px[3 * nsl], a[3]);
                pb += 4 * sb; px += 4 * nsl;
                if (++steps[j] == FOLD) {
                    steps[j] = 0;
                    outer[j] += (a[0] + a[1]) + (a[2] + a[3]);
                    a[0] = a[1] = a[2] = a[3] = T(0);
                }
            }
            if (c < nc) a[0] = mac(pb[0], px[0], a[0]);                                // < 4 rows left
            if (c + nsl < nc) a[1] = mac(pb[sb], px[nsl], a[1]);
            if (c + 2 * nsl < nc) a[2] = mac(pb[2 * sb], px[2 * nsl], a[2]);
        }
        __syncthreads();                                // stage st fully read
        if (tid == 0 && i + stages < my_tiles) {
            refill_fence();
            issue(i + stages, st);
        }
    }

    // slices of this CTA -> one partial per output, in slice order
#pragma unroll
    for (int j = 0; j < RPT; ++j)
        P[tid + j * NT] = act[j] ? outer[j] + ((acc[j][0] + acc[j][1]) + (acc[j][2] + acc[j][3])) : T(0);
    __syncthreads();
    for (int rr = tid; rr < R; rr += NT) {
        T v = T(0);
        for (int q = 0; q < nsl; ++q) v += P[q * R + rr];
        ws_part[int64_t(blockIdx.x) * R + rr] = v;
    }
    // Two-level merge (fixed order at both levels): the last CTA of each group of
    // TRT_GROUP consecutive CTAs sums the group's partials, the last group finisher sums
    // the group partials -- a few dependent L2 round trips instead of G / nsl of them.
    // n partials of R values at src -> P[0 .. R) (thread (r, q) sums rows q, q + nsl, ...
    // eight loads in flight, then the nsl sums per output in q order)
    auto merge = [&](const T* src, int n) {
        T v[RPT];
#pragma unroll
        for (int j = 0; j < RPT; ++j) {
            v[j] = T(0);
            if (!act[j]) continue;
            int g = sj[j];
            for (; g + 7 * nsl < n; g += 8 * nsl) {
                T p[8];
#pragma unroll
                for (int u = 0; u < 8; ++u) p[u] = ld_partial(src + int64_t(g + u * nsl) * R + rj[j]);
#pragma unroll
                for (int u = 0; u < 8; ++u) v[j] += p[u];
            }
            for (; g < n; g += nsl) v[j] += ld_partial(src + int64_t(g) * R + rj[j]);
        }
        __syncthreads();
#pragma unroll
        for (int j = 0; j < RPT; ++j) P[tid + j * NT] = v[j];
        __syncthreads();
        T tot[RPT];
#pragma unroll
        for (int j = 0; j < RPT; ++j) {
            tot[j] = T(0);
            const int rr = tid + j * NT;
            if (rr < R)
                for (int q = 0; q < nsl; ++q) tot[j] += P[q * R + rr];
        }
        __syncthreads();
#pragma unroll
        for (int j = 0; j < RPT; ++j)
            if (tid + j * NT < R) P[tid + j * NT] = tot[j];   // output rr's total at P[rr]
        __syncthreads();
    };
    const int G = int(gridDim.x);
    const int ngroups = (G + TRT_GROUP - 1) / TRT_GROUP;
    const int grp = int(blockIdx.x) / TRT_GROUP;
    const int gsz = min(TRT_GROUP, G - grp * TRT_GROUP);
    T* gpart = ws_part + int64_t(G) * R;                // group partials: ngroups x R
    if (ticket_is_last(ws_cnt + 1 + grp, unsigned(gsz), &flag)) {
        merge(ws_part + int64_t(grp) * TRT_GROUP * R, gsz);
        for (int rr = tid; rr < R; rr += NT) gpart[int64_t(grp) * R + rr] = P[rr];
        if (ticket_is_last(ws_cnt, unsigned(ngroups), &flag)) {
            merge(gpart, ngroups);
            for (int rr = tid; rr < R; rr += NT) y[rr] = P[rr];
        }
    }
}

}  // namespace adaptic
