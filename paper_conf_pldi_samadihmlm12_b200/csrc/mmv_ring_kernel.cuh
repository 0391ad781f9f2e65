// mmv_ring_kernel.cuh -- multi-vector MV with the MATRIX staged by TMA (round 2), sm_100a.
//
// Y = A [x_0 .. x_{K-1}] for long rows (C % 4 == 0, C >= 2048), one pass over A -- the
// paper's horizontal actor integration.  The register-fed kernels of
// mmv_kernels.cuh kept the bytes in flight in registers, next to K accumulators per row,
// and ran out of both: ncu on 64 x 1M at K = 4 showed 127 registers, 25 % occupancy,
// DRAM 1.02x algorithmic -- latency-bound at 0.52 of the copy peak.  Here a producer
// warp streams A through an mbarrier ring in shared memory (cp.async.bulk: the TMA engine,
// no registers per byte in flight) and eight consumer warps only compute:
//
//   * work: rows in groups of RT = 8; the flat range of (group, float4 column) positions,
//     group-major, is cut evenly over the persistent CTAs (stream-K: every CTA streams the
//     same bytes, no wave tail); a CTA's range is a few SEGMENTS (group, column range);
//   * stage: the RT row segments of CH = 256 float4 (8 x 4 KB = 32 KB, RT bulk copies) and,
//     unless x is resident in shared memory (K C 4 <= 64 KB, loaded once), the K matching
//     x chunks (K bulk copies);
//   * consumer thread t owns float4 column t of every stage: K x float4 and RT A float4
//     from shared memory (conflict-free), RT K accumulators, 4 FMA each -- every x load
//     feeds RT rows, every A load K vectors;
//   * a segment's RT K dot products: one reduce-scatter butterfly per warp
//     (warp_multi_sum), the eight warps summed in order through shared memory; a group
//     covered by one CTA writes Y, otherwise its CTAs write partials and the last one (a
//     ticket per group) sums them in CTA order -- deterministic, same launch;
//   * fp32 chains: 4 terms per position, folded every FOLDP positions (planner: chain
//     4 FOLDP + positions / FOLDP + tree depth <= the 1e-4 bound).
// T = float or uint32_t (int32 modulo 2^32); K in {1, 2, 4, 8}.  Consumers synchronise
// with a named barrier (the producer warp leaves early).
#pragma once

#include "common.cuh"
#include "mmv_kernels.cuh"

namespace adaptic {

constexpr int MRING_RT = 8;            // rows per group
constexpr int MRING_CH = 256;          // float4 per row per stage (one per consumer thread)
constexpr int MRING_NT = 256;          // consumer threads (+ one producer warp)
constexpr int MRING_FOLDP = 128;       // positions per thread between folds of the fp32 chains
constexpr int MRING_MAX_STAGES = 8;
constexpr int64_t MRING_XRES_BYTES = 64 * 1024;   // x resident in smem up to K C 4 bytes

__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" :: "r"(smem_u32(bar)) : "memory");
}
// 128-bit shared-memory load that ptxas keeps in program order with the other ones (the
// consumer issues every load of a position before its FMAs; see the stage loop)
__device__ __forceinline__ float4 lds128(const float4* p) {
    float4 v;
    asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];"
                 : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(smem_u32(p)));
    return v;
}
__device__ __forceinline__ uint4 lds128(const uint4* p) {
    uint4 v;
    asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(smem_u32(p)));
    return v;
}
__device__ __forceinline__ void consumer_sync() {            // the MRING_NT consumer threads
    asm volatile("bar.sync 1, %0;" :: "n"(MRING_NT) : "memory");
}

// CTA b of G owns flat positions [Tw b / G, Tw (b+1) / G); the first / last CTA whose range
// touches position p (ranges are non-empty: G <= Tw).
__device__ __forceinline__ int64_t mring_cta_of(int64_t p, int64_t Tw, int64_t G) {
    int64_t b = (p * G) / Tw;                                  // p * G < 2^63 (planner)
    while (b + 1 < G && Tw * (b + 1) / G <= p) ++b;
    while (b > 0 && Tw * b / G > p) --b;
    return b;
}

template <class T, int K>
__global__ void __launch_bounds__(MRING_NT + 32, 1)
mmv_ring_kernel(const T* __restrict__ A, const T* __restrict__ X, T* __restrict__ Y, int64_t R, int64_t C,
                int stages, int xres_dbg, int maxs, T* __restrict__ part, unsigned int* __restrict__ cnt)
{
    const int xres = xres_dbg & 1;
    const bool dbg_nocompute = (xres_dbg & 2) != 0;     // experiments: consumers only wait/release
    using V = vec4_t<T>;
    constexpr int RT = MRING_RT, CH = MRING_CH, NT = MRING_NT, NW = NT / 32;
    constexpr int N = RT * K;                                  // outputs per group
    constexpr int NH = N > 32 ? 32 : N;                        // per butterfly
    constexpr int LOGH = (NH >= 32) ? 5 : (NH >= 16) ? 4 : 3;
    static_assert((1 << LOGH) == NH, "RT K: 8, 16, 32 or 64");
    pdl_prologue();
    extern __shared__ __align__(128) unsigned char dyn_smem[];
    __shared__ __align__(8) uint64_t full[MRING_MAX_STAGES], empty[MRING_MAX_STAGES];
    __shared__ __align__(8) uint64_t xbar;
    __shared__ T s_red[NW][N];
    __shared__ T s_m[NT];
    __shared__ unsigned int s_flag;
    const int64_t nv = C / 4;
    const int64_t ngroups = (R + RT - 1) / RT;
    const int64_t Tw = ngroups * nv;
    const int64_t G = gridDim.x, b = blockIdx.x;
    const int64_t f0 = Tw * b / G, f1 = Tw * (b + 1) / G;
    const V* __restrict__ Av = reinterpret_cast<const V*>(A);
    const V* __restrict__ Xv = reinterpret_cast<const V*>(X);
    V* xs = reinterpret_cast<V*>(dyn_smem);                    // [K][nv] when x is resident
    V* ring = xs + (xres ? int64_t(K) * nv : 0);
    const int sv4 = (RT + (xres ? 0 : K)) * CH;                // float4 per stage
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0) {
        for (int i = 0; i < stages; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], NW); }
        mbar_init(&xbar, 1);
        fence_mbar_init();
        if (xres) {
            const uint32_t bytes = uint32_t(K) * uint32_t(C) * uint32_t(sizeof(T));
            mbar_arrive_expect_tx(&xbar, bytes);
            for (uint32_t off = 0; off < bytes; off += 32768u)
                bulk_g2s_keep(reinterpret_cast<char*>(xs) + off, reinterpret_cast<const char*>(X) + off,
                              bytes - off < 32768u ? bytes - off : 32768u, &xbar);
        }
    }
    __syncthreads();

    if (warp == NW) {                                          // ---- producer warp
        int st = 0;
        uint32_t ph = 0;
        int64_t i = 0, f = f0, g = f0 / nv, col = f0 - (f0 / nv) * nv;
        while (f < f1) {
            const int len = int(min(min(int64_t(CH), nv - col), f1 - f));
            const int rows = int(min(int64_t(RT), R - g * RT));
            if (i >= stages) mbar_wait(&empty[st], ph ^ 1u);
            if (lane == 0)
                mbar_arrive_expect_tx(&full[st], uint32_t(rows + (xres ? 0 : K)) * uint32_t(len) * 16u);
            __syncwarp();
            V* sA = ring + int64_t(st) * sv4;
            if (lane < rows)
                bulk_g2s(sA + lane * CH, Av + (g * RT + lane) * nv + col, uint32_t(len) * 16u, &full[st]);
            else if (!xres && lane >= RT && lane < RT + K)
                bulk_g2s_keep(sA + lane * CH, Xv + (lane - RT) * nv + col, uint32_t(len) * 16u, &full[st]);
            ++i;
            ring_advance(st, ph, stages);
            f += len;
            col += len;
            if (col == nv) { col = 0; ++g; }
        }
        return;
    }

    // ---- consumer warps
    if (xres) mbar_wait(&xbar, 0);
    T acc[RT][K], outer[RT][K];
#pragma unroll
    for (int r = 0; r < RT; ++r)
#pragma unroll
        for (int j = 0; j < K; ++j) { acc[r][j] = T(0); outer[r][j] = T(0); }
    int npos = 0, st = 0;
    uint32_t ph = 0;
    int64_t f = f0, g = f0 / nv, col = f0 - (f0 / nv) * nv;
    while (f < f1) {
        const int len = int(min(min(int64_t(CH), nv - col), f1 - f));
        mbar_wait(&full[st], ph);
        const V* sA = ring + int64_t(st) * sv4;
        if (tid < len && !dbg_nocompute) {
            // every shared-memory load of the position first (RA rows at a time), then the
            // FMAs: a row-by-row load -> 4K FMA order made each LDS wait for the previous
            // row's FMAs to release its registers (ncu: FFMA stalls on short scoreboard)
            constexpr int RA = K >= 8 ? RT / 2 : RT;
            V xv[K];
#pragma unroll
            for (int j = 0; j < K; ++j) xv[j] = lds128(xres ? xs + j * nv + col + tid : sA + (RT + j) * CH + tid);
#pragma unroll
            for (int r0 = 0; r0 < RT; r0 += RA) {
                V a[RA];
#pragma unroll
                for (int r = 0; r < RA; ++r) a[r] = lds128(sA + (r0 + r) * CH + tid);
#pragma unroll
                for (int r = 0; r < RA; ++r)
#pragma unroll
                    for (int j = 0; j < K; ++j) {
                        T t = acc[r0 + r][j];
                        t = mac(a[r].x, xv[j].x, t);
                        t = mac(a[r].y, xv[j].y, t);
                        t = mac(a[r].z, xv[j].z, t);
                        acc[r0 + r][j] = mac(a[r].w, xv[j].w, t);
                    }
            }
        }
        __syncwarp();
        if (lane == 0) mbar_arrive(&empty[st]);
        ring_advance(st, ph, stages);
        if (++npos == MRING_FOLDP) {
            npos = 0;
#pragma unroll
            for (int r = 0; r < RT; ++r)
#pragma unroll
                for (int j = 0; j < K; ++j) { outer[r][j] += acc[r][j]; acc[r][j] = T(0); }
        }
        if (col + len == nv || f + len == f1) {                // end of this CTA's segment of group g
            T flat[N];
#pragma unroll
            for (int r = 0; r < RT; ++r)
#pragma unroll
                for (int j = 0; j < K; ++j) {
                    flat[r * K + j] = outer[r][j] + acc[r][j];
                    acc[r][j] = T(0);
                    outer[r][j] = T(0);
                }
            npos = 0;
#pragma unroll
            for (int c = 0; c < N / NH; ++c) {
                T sub[NH];
#pragma unroll
                for (int q = 0; q < NH; ++q) sub[q] = flat[c * NH + q];
                const T tot = warp_multi_sum<NH>(sub);
                if ((lane & ((1 << (5 - LOGH)) - 1)) == 0) s_red[warp][c * NH + (lane >> (5 - LOGH))] = tot;
            }
            consumer_sync();
            T val = T(0);
            if (tid < N)
#pragma unroll
                for (int w = 0; w < NW; ++w) val += s_red[w][tid];
            const int r = tid / K, j = tid - (tid / K) * K;
            const int64_t row = g * RT + r;
            const int64_t b_lo = mring_cta_of(g * nv, Tw, G), b_hi = mring_cta_of(g * nv + nv - 1, Tw, G);
            const unsigned int count = unsigned(b_hi - b_lo + 1);
            if (count == 1) {
                if (tid < N && row < R) Y[int64_t(j) * R + row] = val;
            } else {
                if (tid < N) part[(g * maxs + (b - b_lo)) * N + tid] = val;
                __threadfence();
                consumer_sync();
                if (tid == 0) {
                    const unsigned int old = atomicAdd(cnt + g, 1u);
                    const bool last = old + 1u == count;
                    if (last) cnt[g] = 0u;                     // re-arm for the next run
                    s_flag = last ? 1u : 0u;
                }
                consumer_sync();
                if (s_flag) {
                    __threadfence();
                    constexpr int NG = NT / N;                 // thread groups over slot ranges
                    const int o = tid % N, sg = tid / N;
                    const unsigned int s_lo = count * unsigned(sg) / NG, s_hi = count * unsigned(sg + 1) / NG;
                    T m = T(0);
                    for (unsigned int s = s_lo; s < s_hi; ++s) m += ld_partial(part + (g * maxs + s) * N + o);
                    s_m[tid] = m;
                    consumer_sync();
                    if (tid < N) {
                        T t = T(0);
#pragma unroll
                        for (int q = 0; q < NG; ++q) t += s_m[q * N + tid];
                        if (row < R) Y[int64_t(j) * R + row] = t;
                    }
                }
            }
            consumer_sync();                                   // s_red / s_m / s_flag reuse
        }
        f += len;
        col += len;
        if (col == nv) { col = 0; ++g; }
    }
}

}  // namespace adaptic
