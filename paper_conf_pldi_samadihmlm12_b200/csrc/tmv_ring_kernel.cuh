// tmv_ring_kernel.cuh -- TMV (y = B^T [x_0 .. x_{K-1}], B row-major C x R) with B and x
// staged by TMA in an mbarrier ring (round 2), sm_100a.
//
// The paper's restructured layout: every output is a column of B, so a CTA
// owns a TILE of TW consecutive outputs and streams rows of B through it.  The register-
// fed TMV kernels hold K accumulators per output next to the loads in flight (multi-vector:
// 118-128 registers, 22-25 % occupancy, 0.73-0.76 of the copy peak), and rows off the
// 16-byte grid (R % 4 != 0) needed two overlapping 128-bit loads and a funnel shift per
// float4 (0.72-0.83).  Here a producer warp moves B AND the x chunks of the stage's rows by
// cp.async.bulk and the consumers only compute, for ANY alignment and any R:
//
//   * work: the flat (tile, row) positions are cut evenly over one CTA per SM (stream-K);
//     a tile covering all outputs (TW >= R) streams stages of CR WHOLE rows of B -- one
//     contiguous bulk copy -- otherwise a stage is CR row segments of TW words (one copy
//     each); plus, per vector, the stage's x chunk (one copy);
//   * every copy moves the 16-byte-aligned COVER of its words, clamped to the operand's
//     16-byte interior; data lands at a word shift in [0, 3]; the at most 3 + 3 words of B
//     (and of each x) outside the interior are read from global memory in the one or two
//     stages that contain them (the "edge" stages);
//   * flat mode (one tile, R <= 256): thread t < L = (256 / R) R owns output t % R and rows
//     t / R + (256 / R) k of every stage -- a warp reads consecutive words of the stage at
//     any R; the 256 / R row lanes of an output are summed in order at the segment end;
//   * tile mode: lane l of a warp owns tile words l + 32 m (m < OPT) of its column group
//     (consecutive words at any shift: conflict-free), the 8 warps are TW / (32 OPT) column
//     groups x LC row lanes, summed in order at the segment end;
//   * a segment (tile change or end of the CTA's range) covered by one CTA writes y,
//     otherwise partials + a ticket per tile: the last CTA sums the slots in CTA order
//     (deterministic); fp32 chains fold every FOLD rows (planner bound).
// T = float or uint32_t (int32 modulo 2^32, K = 1).  Consumers synchronise with a named
// barrier; the producer warp leaves early.
#pragma once

#include "mmv_ring_kernel.cuh"

namespace adaptic {

constexpr int TRING_COPY_MAX = 32768;      // bytes per bulk copy (a contiguous stage is cut)

// Stage layout (words): B part -- CR whole rows + the cover's slack (one tile), or CR row
// segments at pitch TW + 8 -- then K x chunks at pitch CR + 8; multiples of 32 words.
__host__ __device__ inline int64_t tring_a_words(int64_t R, int TW, int CR) {
    const int64_t w = (TW >= R) ? int64_t(CR) * R + 8 : int64_t(CR) * (TW + 8);
    return (w + 31) / 32 * 32;
}
__host__ __device__ inline int tring_x_pitch(int CR) { return (CR + 8 + 31) / 32 * 32; }
__host__ __device__ inline int64_t tring_stage_words(int64_t R, int TW, int CR, int K) {
    return tring_a_words(R, TW, CR) + int64_t(K) * tring_x_pitch(CR);
}

template <class T, int K, int OPT>
__global__ void __launch_bounds__(MRING_NT + 32, 1)
tmv_ring_kernel(const T* __restrict__ B, const T* __restrict__ X, T* __restrict__ Y, int64_t R, int64_t C,
                int TW, int CR, int stages, int stage_words, int maxs, T* __restrict__ part,
                unsigned int* __restrict__ cnt, int dbg)
{
    constexpr int NT = MRING_NT, NW = NT / 32, WW = 32 * OPT;
    pdl_prologue();
    extern __shared__ __align__(128) unsigned char dyn_smem[];
    __shared__ __align__(8) uint64_t full[MRING_MAX_STAGES], empty[MRING_MAX_STAGES];
    __shared__ unsigned int s_flag;
    __shared__ vec4_t<T> s_m[MRING_NT];
    T* ring = reinterpret_cast<T*>(dyn_smem);
    T* red = ring + int64_t(stages) * stage_words;             // segment sums of the row lanes
    const int64_t ntiles = (R + TW - 1) / TW;
    const bool contig = ntiles == 1;
    const bool flat = contig && R <= NT;
    const int pitch = contig ? int(R) : TW + 8;
    const int xoff = int(tring_a_words(R, TW, CR)), XP = tring_x_pitch(CR);
    const int WPT = flat ? 1 : TW / WW, LC = NW / WPT;
    const int RS = flat ? NT / int(R) : 1, L = flat ? RS * int(R) : NT;
    const int64_t Tw = ntiles * C;
    const int64_t G = gridDim.x, b = blockIdx.x;
    const int64_t f0 = Tw * b / G, f1 = Tw * (b + 1) / G;
    // operand interiors: [lo16, hi16) is 16-byte aligned; the words outside come from global
    const uintptr_t bb = reinterpret_cast<uintptr_t>(B), xb = reinterpret_cast<uintptr_t>(X);
    const uintptr_t be = bb + uintptr_t(R) * uintptr_t(C) * 4u;
    const uintptr_t b16lo = (bb + 15) & ~uintptr_t(15), b16hi = be & ~uintptr_t(15);
    const int64_t Bn = R * C;
    const int64_t head = int64_t(b16lo - bb) / 4, tailw = int64_t(be - b16hi) / 4;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0) {
        for (int i = 0; i < stages; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], NW); }
        fence_mbar_init();
    }
    __syncthreads();
    auto cover = [](uintptr_t lo, uintptr_t hi, uintptr_t ilo, uintptr_t ihi, uintptr_t& a0, uintptr_t& a1) {
        a0 = max(lo & ~uintptr_t(15), ilo);
        a1 = min((hi + 15u) & ~uintptr_t(15), ihi);
    };
    auto x_interior = [&](int j, uintptr_t& lo16, uintptr_t& hi16) {
        const uintptr_t x0 = xb + uintptr_t(j) * uintptr_t(C) * 4u;
        lo16 = (x0 + 15) & ~uintptr_t(15);
        hi16 = (x0 + uintptr_t(C) * 4u) & ~uintptr_t(15);
    };

    if (warp == NW) {                                          // ---- producer warp
        // every lane owns at most one copy per stage (a row segment, a piece of a contiguous
        // stage, or the x chunk of vector lane - (32 - K)); the stage's byte count is a warp sum
        const bool xl = lane >= 32 - K;
        const int xj = xl ? lane - (32 - K) : 0;
        uintptr_t xlo16 = 0, xhi16 = 0, xbase = 0;
        if (xl) {
            x_interior(xj, xlo16, xhi16);
            xbase = xb + uintptr_t(xj) * uintptr_t(C) * 4u;
        }
        int st = 0;
        uint32_t ph = 0;
        int64_t i = 0, f = f0, t = f0 / C, c = f0 - (f0 / C) * C;
        while (f < f1) {
            const int len = int(min(min(int64_t(CR), C - c), f1 - f));
            unsigned char* sb = reinterpret_cast<unsigned char*>(ring + int64_t(st) * stage_words);
            uintptr_t a0 = 0, a1 = 0, dst = 0;
            if (xl) {
                const uintptr_t x0 = xbase + uintptr_t(c) * 4u;
                cover(x0, x0 + uintptr_t(len) * 4u, xlo16, xhi16, a0, a1);
                dst = uintptr_t(sb) + (uintptr_t(xoff) + uintptr_t(xj) * uintptr_t(XP)) * 4u;
            } else if (contig) {
                uintptr_t c0, c1;
                cover(bb + uintptr_t(c * R) * 4u, bb + uintptr_t((c + len) * R) * 4u, b16lo, b16hi, c0, c1);
                const uintptr_t off = uintptr_t(lane) * TRING_COPY_MAX;
                if (c0 + off < c1) {
                    a0 = c0 + off;
                    a1 = min(c1, a0 + TRING_COPY_MAX);
                    dst = uintptr_t(sb) + off;
                }
            } else if (lane < len) {
                const uintptr_t g = bb + uintptr_t((c + lane) * R + t * TW) * 4u;
                cover(g, g + uintptr_t(min(int64_t(TW), R - t * TW)) * 4u, b16lo, b16hi, a0, a1);
                dst = uintptr_t(sb) + uintptr_t(lane) * uintptr_t(pitch) * 4u;
            }
            uint32_t n = a1 > a0 ? uint32_t(a1 - a0) : 0u;
            if (dbg & 2) n = 0;
            const uint32_t tx = __reduce_add_sync(0xffffffffu, n);
            if (i >= stages) mbar_wait(&empty[st], ph ^ 1u);
            if (lane == 0) mbar_arrive_expect_tx(&full[st], tx);
            __syncwarp();
            if (n) {
                if (xl) bulk_g2s_keep(reinterpret_cast<void*>(dst), reinterpret_cast<const void*>(a0), n, &full[st]);
                else bulk_g2s(reinterpret_cast<void*>(dst), reinterpret_cast<const void*>(a0), n, &full[st]);
            }
            ++i;
            ring_advance(st, ph, stages);
            f += len;
            c += len;
            if (c == C) { c = 0; ++t; }
        }
        return;
    }

    // ---- consumer warps.  flat: output t % R, row lane t / R (t < L); tile: c-lane lc,
    // column group wc, words colbase + 32 m
    const int lc = flat ? 0 : warp / WPT, wc = flat ? 0 : warp - (warp / WPT) * WPT;
    const int colbase = wc * WW + lane;
    const int fr = flat ? tid % int(R) : 0, fq = flat ? tid / int(R) : 0;
    T acc[OPT][K], outer[OPT][K];
#pragma unroll
    for (int m = 0; m < OPT; ++m)
#pragma unroll
        for (int j = 0; j < K; ++j) { acc[m][j] = T(0); outer[m][j] = T(0); }
    int rows_acc = 0, st = 0;
    uint32_t ph = 0;
    // word phases (address / 4 mod 4): a non-edge copy starts at the aligned-down address, so
    // the word shift of any row / x chunk in the stage is a 2-bit function of these
    const int bph = int((bb >> 2) & 3u), Rm4 = int(R & 3);
    int xph[K];
    int64_t xhmax = 0, xtmax = 0;                              // x words outside the 16-byte interiors
#pragma unroll
    for (int j = 0; j < K; ++j) {
        xph[j] = int(((xb >> 2) + uintptr_t(j) * uintptr_t(C & 3)) & 3u);
        uintptr_t lo16, hi16;
        x_interior(j, lo16, hi16);
        const uintptr_t x0 = xb + uintptr_t(j) * uintptr_t(C) * 4u;
        xhmax = max(xhmax, int64_t(lo16 - x0) / 4);
        xtmax = max(xtmax, int64_t(x0 + uintptr_t(C) * 4u - hi16) / 4);
    }
    int64_t f = f0, t = f0 / C, c = f0 - (f0 / C) * C;
    while (f < f1) {
        const int len = int(min(min(int64_t(CR), C - c), f1 - f));
        const int tw = int(min(int64_t(TW), R - t * TW));
        // edge stage: B's first / last unaligned words, or an x chunk at either end of x
        const bool edge = (t == 0 && c == 0 && head > 0) || (t == ntiles - 1 && c + len == C && tailw > 0) ||
                          c < xhmax || c + len > C - xtmax;
        const int cm4 = int(c & 3);
        mbar_wait(&full[st], ph);
        const T* sb = ring + int64_t(st) * stage_words;
        if (dbg & 1) {
        } else if (!edge) {
            int xo[K];                                         // smem index of x_j[c]
#pragma unroll
            for (int j = 0; j < K; ++j) xo[j] = xoff + j * XP + ((xph[j] + cm4) & 3);
            if (flat) {
                if (tid < L) {
                    const T* pa = sb + ((bph + cm4 * Rm4) & 3) + fq * int(R) + fr;
                    int q = fq;
#pragma unroll 4
                    for (; q < len; q += RS, pa += L) {
                        const T v = *pa;
#pragma unroll
                        for (int j = 0; j < K; ++j) acc[0][j] = mac(v, sb[xo[j] + q], acc[0][j]);
                    }
                }
                rows_acc += (len + RS - 1) / RS;
            } else {
                const int s0 = (bph + cm4 * Rm4) & 3;
                for (int q = lc; q < len; q += LC) {
                    const int base = contig ? s0 + q * int(R) : q * pitch + ((bph + (cm4 + q) * Rm4) & 3);
                    T xq[K];
#pragma unroll
                    for (int j = 0; j < K; ++j) xq[j] = sb[xo[j] + q];
                    const T* pr = sb + base + colbase;
                    if (tw == TW) {
#pragma unroll
                        for (int m = 0; m < OPT; ++m) {
                            const T v = pr[32 * m];
#pragma unroll
                            for (int j = 0; j < K; ++j) acc[m][j] = mac(v, xq[j], acc[m][j]);
                        }
                    } else {
#pragma unroll
                        for (int m = 0; m < OPT; ++m) {
                            if (colbase + 32 * m < tw) {
                                const T v = pr[32 * m];
#pragma unroll
                                for (int j = 0; j < K; ++j) acc[m][j] = mac(v, xq[j], acc[m][j]);
                            }
                        }
                    }
                }
                rows_acc += (len + LC - 1) / LC;
            }
        } else {
            // generic (slow) path: covers recomputed, out-of-interior words from global memory
            int xs[K];
#pragma unroll
            for (int j = 0; j < K; ++j) {
                uintptr_t lo16, hi16, a0, a1;
                x_interior(j, lo16, hi16);
                const uintptr_t x0 = xb + uintptr_t(int64_t(j) * C + c) * 4u;
                cover(x0, x0 + uintptr_t(len) * 4u, lo16, hi16, a0, a1);
                xs[j] = int((int64_t(x0) - int64_t(a0)) / 4);
            }
            auto xval = [&](int j, int q) -> T {
                const int64_t cc = c + q;
                const uintptr_t xa = xb + uintptr_t(int64_t(j) * C + cc) * 4u;
                uintptr_t lo16, hi16;
                x_interior(j, lo16, hi16);
                if (xa < lo16 || xa >= hi16) return X[int64_t(j) * C + cc];
                return sb[xoff + j * XP + xs[j] + q];
            };
            int64_t s0 = 0;
            if (contig) {
                uintptr_t a0, a1;
                cover(bb + uintptr_t(c * R) * 4u, bb + uintptr_t((c + len) * R) * 4u, b16lo, b16hi, a0, a1);
                s0 = (int64_t(bb + uintptr_t(c * R) * 4u) - int64_t(a0)) / 4;
            }
            if (flat) {
                if (tid < L)
                    for (int q = fq; q < len; q += RS) {
                        const int64_t g = (c + q) * R + fr;
                        const T v = (g < head || g >= Bn - tailw) ? B[g] : sb[s0 + int64_t(q) * R + fr];
#pragma unroll
                        for (int j = 0; j < K; ++j) acc[0][j] = mac(v, xval(j, q), acc[0][j]);
                    }
                rows_acc += (len + RS - 1) / RS;
            } else {
                for (int q = lc; q < len; q += LC) {
                    const int64_t g0 = (c + q) * R + t * TW;   // word of (row c + q, tile start)
                    int64_t eb;
                    if (contig) {
                        eb = s0 + int64_t(q) * R;
                    } else {
                        uintptr_t a0, a1;
                        const uintptr_t g = bb + uintptr_t(g0) * 4u;
                        cover(g, g + uintptr_t(tw) * 4u, b16lo, b16hi, a0, a1);
                        eb = int64_t(q) * pitch + (int64_t(g) - int64_t(a0)) / 4;
                    }
                    T xq[K];
#pragma unroll
                    for (int j = 0; j < K; ++j) xq[j] = xval(j, q);
#pragma unroll
                    for (int m = 0; m < OPT; ++m) {
                        const int w = colbase + 32 * m;
                        if (w < tw) {
                            const int64_t g = g0 + w;
                            const T v = (g < head || g >= Bn - tailw) ? B[g] : sb[eb + w];
#pragma unroll
                            for (int j = 0; j < K; ++j) acc[m][j] = mac(v, xq[j], acc[m][j]);
                        }
                    }
                }
                rows_acc += (len + LC - 1) / LC;
            }
        }
        __syncwarp();
        if (lane == 0) mbar_arrive(&empty[st]);
        ring_advance(st, ph, stages);
        if (rows_acc >= FOLD) {
            rows_acc = 0;
#pragma unroll
            for (int m = 0; m < OPT; ++m)
#pragma unroll
                for (int j = 0; j < K; ++j) { outer[m][j] += acc[m][j]; acc[m][j] = T(0); }
        }
        if (c + len == C || f + len == f1) {                   // end of this CTA's segment of tile t
            T v[OPT][K];
#pragma unroll
            for (int m = 0; m < OPT; ++m)
#pragma unroll
                for (int j = 0; j < K; ++j) {
                    v[m][j] = outer[m][j] + acc[m][j];
                    acc[m][j] = T(0);
                    outer[m][j] = T(0);
                }
            rows_acc = 0;
            const int64_t b_lo = mring_cta_of(t * C, Tw, G), b_hi = mring_cta_of(t * C + C - 1, Tw, G);
            const unsigned int count = unsigned(b_hi - b_lo + 1);
            T* pp = part + (t * maxs + (b - b_lo)) * int64_t(K) * TW;
            if (flat) {                                        // row lanes -> red[fq][j][r], summed in order
                if (tid < L)
#pragma unroll
                    for (int j = 0; j < K; ++j) red[(int64_t(fq) * K + j) * R + fr] = v[0][j];
                consumer_sync();
                for (int e = tid; e < K * int(R); e += NT) {
                    const int j = e / int(R), r = e - (e / int(R)) * int(R);
                    T sum = T(0);
                    for (int l = 0; l < RS; ++l) sum += red[(int64_t(l) * K + j) * R + r];
                    if (count == 1) Y[int64_t(j) * R + r] = sum;
                    else pp[int64_t(j) * TW + r] = sum;
                }
            } else {
                if (LC > 1) {                                  // c-lanes 1.. -> smem, lane 0 sums in order
                    if (lc > 0)
#pragma unroll
                        for (int m = 0; m < OPT; ++m)
#pragma unroll
                            for (int j = 0; j < K; ++j)
                                red[(int64_t(lc - 1) * K + j) * TW + colbase + 32 * m] = v[m][j];
                    consumer_sync();
                    if (lc == 0)
                        for (int l = 1; l < LC; ++l)
#pragma unroll
                            for (int m = 0; m < OPT; ++m)
#pragma unroll
                                for (int j = 0; j < K; ++j)
                                    v[m][j] += red[(int64_t(l - 1) * K + j) * TW + colbase + 32 * m];
                }
                if (lc == 0)
#pragma unroll
                    for (int m = 0; m < OPT; ++m) {
                        const int w = colbase + 32 * m;
                        if (w < tw)
#pragma unroll
                            for (int j = 0; j < K; ++j) {
                                if (count == 1) Y[int64_t(j) * R + t * TW + w] = v[m][j];
                                else pp[int64_t(j) * TW + w] = v[m][j];
                            }
                    }
            }
            if (count > 1 && !(dbg & 8)) {
                __threadfence();
                consumer_sync();
                if (tid == 0) {
                    const unsigned int old = atomicAdd(cnt + t, 1u);
                    const bool last = old + 1u == count;
                    if (last) cnt[t] = 0u;                     // re-arm for the next run
                    s_flag = last ? 1u : 0u;
                }
                consumer_sync();
                if (s_flag) {
                    __threadfence();
                    // thread groups over slot ranges (NG groups, 4 independent chains each), the
                    // groups combined in order; 16-byte partial loads when the tile allows
                    const T* p0 = part + t * maxs * int64_t(K) * TW;
                    const bool v4 = (TW & 3) == 0 && (tw & 3) == 0;
                    const int W4 = v4 ? 4 : 1;
                    const int n = K * tw / W4;                 // outputs (of W4 words) of the tile
                    const int NG = n >= NT ? 1 : NT / n;
                    for (int e0 = 0; e0 < n; e0 += NT / NG) {
                        const int e = e0 + tid % (NT / NG), g = tid / (NT / NG);
                        vec4_t<T> m = {T(0), T(0), T(0), T(0)};
                        if (e < n && g < NG) {
                            const int j = e / (tw / W4), w = (e - j * (tw / W4)) * W4;
                            const unsigned int s_lo = count * unsigned(g) / NG, s_hi = count * unsigned(g + 1) / NG;
                            vec4_t<T> a[4];
#pragma unroll
                            for (int u = 0; u < 4; ++u) a[u] = m;
                            unsigned int sl = s_lo;
                            if (v4) {
                                const vec4_t<T>* q = reinterpret_cast<const vec4_t<T>*>(p0 + int64_t(j) * TW + w);
                                const int64_t stride = int64_t(K) * TW / 4;
                                for (; sl + 3 < s_hi; sl += 4)
#pragma unroll
                                    for (int u = 0; u < 4; ++u) a[u] = vadd(a[u], ld_partial(q + (sl + u) * stride));
                                for (; sl < s_hi; ++sl) a[0] = vadd(a[0], ld_partial(q + sl * stride));
                            } else {
                                const T* q = p0 + int64_t(j) * TW + w;
                                const int64_t stride = int64_t(K) * TW;
                                for (; sl + 3 < s_hi; sl += 4)
#pragma unroll
                                    for (int u = 0; u < 4; ++u) a[u].x += ld_partial(q + (sl + u) * stride);
                                for (; sl < s_hi; ++sl) a[0].x += ld_partial(q + sl * stride);
                            }
                            m = vadd(vadd(a[0], a[1]), vadd(a[2], a[3]));
                        }
                        s_m[tid] = m;
                        consumer_sync();
                        if (g == 0 && e < n) {
                            vec4_t<T> r4 = s_m[tid];
                            for (int gg = 1; gg < NG; ++gg) r4 = vadd(r4, s_m[gg * (NT / NG) + tid % (NT / NG)]);
                            const int j = e / (tw / W4), w = (e - j * (tw / W4)) * W4;
                            T* yo = Y + int64_t(j) * R + t * TW + w;
                            yo[0] = r4.x;
                            if (v4) { yo[1] = r4.y; yo[2] = r4.z; yo[3] = r4.w; }
                        }
                        consumer_sync();
                    }
                }
            }
            consumer_sync();                                   // red / s_flag reuse
        }
        f += len;
        c += len;
        if (c == C) { c = 0; ++t; }
    }
}

}  // namespace adaptic
