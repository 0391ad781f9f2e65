// rowtile_kernel.cuh -- MV / DOT lane groups on TMA-staged row tiles (sm_100a).
//
// The paper's K4/K3 thread shapes ("several threads ... the dot product of
// one row", rows merged adaptively into one block) for rows of C <= 32*G elements
// whose start is NOT 16-byte aligned (C % 4 != 0) -- the held-out 3*2^k shapes where
// the direct kernels (mv_mis_kernels.cuh: 128-bit body + scalar head/tail) run at
// 0.4-0.7 of the copy peak because a short row leaves each lane one or two loads in
// flight.  Here the load side and the reduction side are decoupled:
//
//  * k consecutive rows are one contiguous run of k*C words.  Thread 0 copies the
//    16-byte-aligned cover of that run ([floor4(r0*C), ceil4((r0+k)*C)) words) with
//    one cp.async.bulk into a STAGES-deep ring guarded by mbarriers, so every SM
//    keeps STAGES-1 whole tiles (tens of KB) in flight no matter how short the rows.
//    Only the last tile of the matrix may end inside a 16-byte word group; its < 4
//    remaining words are copied by the threads (no read past the matrix).
//  * G lanes reduce one row out of shared memory: lane li reads words li + G*m
//    (consecutive lanes, consecutive banks), x[li + G*m] lives in registers for the
//    whole kernel (it is the same for every row), and the G partials are combined
//    with a log2(G)-step butterfly (group_sum).  DOT (PERROWX) stages its second
//    operand tile beside the first; both bases are 16-byte aligned, so the two tiles
//    share the head offset.
//
// Accumulation order per row is fixed (lane partials over m in two interleaved
// chains, then the butterfly), so a plan is deterministic (P7 invariants).
#pragma once

#include "common.cuh"

namespace adaptic {

constexpr int RT_MAX_STAGES = 8;
constexpr int RT_MAXM = 32;          // x values per lane: C <= 32*G

template <class T, int NT, int G, bool PERROWX>
__global__ void __launch_bounds__(NT)
mv_rowtile_kernel(const T* __restrict__ A, const T* __restrict__ X, T* __restrict__ y,
                  int64_t R, int64_t C, int k, int stages)
{
    pdl_prologue();
    extern __shared__ __align__(128) unsigned char smem_raw[];
    __shared__ __align__(8) uint64_t full[RT_MAX_STAGES];

    const int tid = threadIdx.x;
    const int li = tid % G;
    constexpr int NGR = NT / G;
    const int Ci = int(C);
    const int64_t total = R * C;
    const int64_t ntiles = (R + k - 1) / k;
    // words per operand tile: k*C plus up to 3 head and 3 tail words, rounded to 16 bytes
    const int64_t tile_w = ((int64_t(k) * C + 6 + 3) / 4) * 4;
    T* ring = reinterpret_cast<T*>(smem_raw);
    const int64_t stage_w = tile_w * (PERROWX ? 2 : 1);
    const int64_t my_tiles = blockIdx.x < ntiles ? (ntiles - 1 - blockIdx.x) / gridDim.x + 1 : 0;

    if (tid == 0) {
        for (int s = 0; s < stages; ++s) mbar_init(&full[s], 1);
        fence_mbar_init();
    }
    __syncthreads();

    // local tile i -> ring stage `slot` (thread 0 only)
    auto issue = [&](int64_t i, int slot) {
        const int64_t r0 = (blockIdx.x + i * gridDim.x) * int64_t(k);
        const int64_t w0 = r0 * C, w1 = min(R, r0 + k) * C;
        const int64_t a0 = w0 & ~int64_t(3);
        int64_t a1 = (w1 + 3) & ~int64_t(3);
        if (a1 > total) a1 = w1 & ~int64_t(3);          // last tile: never read past the matrix
        const uint32_t bytes = uint32_t((a1 - a0) * int64_t(sizeof(T)));
        T* dst = ring + slot * stage_w;
        uint64_t* bar = &full[slot];
        mbar_arrive_expect_tx(bar, PERROWX ? 2 * bytes : bytes);
        if (bytes) {
            bulk_g2s(dst, A + a0, bytes, bar);
            if (PERROWX) bulk_g2s(dst + tile_w, X + a0, bytes, bar);
        }
    };

    if (tid == 0) {
        const int64_t pre = min(int64_t(stages), my_tiles);
        for (int64_t i = 0; i < pre; ++i) issue(i, int(i));
    }

    // x slice of this lane, kept in registers across all rows (MV only)
    T xr[RT_MAXM];
    if constexpr (!PERROWX) {
#pragma unroll
        for (int m = 0; m < RT_MAXM; ++m) {
            const int c = li + G * m;
            xr[m] = c < Ci ? ld_x(X + c) : T(0);
        }
    }

    int st = 0;
    uint32_t ph = 0;
    for (int64_t i = 0; i < my_tiles; ++i, ring_advance(st, ph, stages)) {
        const int64_t r0 = (blockIdx.x + i * gridDim.x) * int64_t(k);
        const int nrows = int(min(int64_t(k), R - r0));
        const int64_t w0 = r0 * C;
        const int head = int(w0 & 3);
        T* stg = ring + st * stage_w;
        mbar_wait(&full[st], ph);
        const int64_t w1 = w0 + int64_t(nrows) * C;
        if (((w1 + 3) & ~int64_t(3)) > total && (w1 & 3)) {  // the matrix's last < 4 words
            const int64_t a0 = w0 & ~int64_t(3);
            for (int64_t e = (w1 & ~int64_t(3)) + tid; e < w1; e += NT) {
                stg[e - a0] = A[e];
                if (PERROWX) stg[tile_w + e - a0] = X[e];
            }
            __syncthreads();
        }
        const T* base = stg + head;
        // whole warps step together (the butterfly needs all 32 lanes): groups whose
        // row is past the tile contribute nothing and write nothing
        for (int rb = (tid >> 5) * (32 / G); rb < nrows; rb += NGR) {
            const int row = rb + (tid & 31) / G;
            const bool live = row < nrows;
            const T* ar = base + int64_t(live ? row : 0) * Ci;
            T acc0 = T(0), acc1 = T(0);
#pragma unroll
            for (int m = 0; m < RT_MAXM; m += 2) {
                if (G * m >= Ci) break;                 // uniform: C is the same for every lane
                const int c0 = li + G * m, c1 = c0 + G;
                if (live && c0 < Ci) acc0 = mac(ar[c0], PERROWX ? ar[tile_w + c0] : xr[m], acc0);
                if (live && c1 < Ci) acc1 = mac(ar[c1], PERROWX ? ar[tile_w + c1] : xr[m + 1], acc1);
            }
            const T s = group_sum<G>(acc0 + acc1);
            if (live && li == 0) y[r0 + row] = s;
        }
        __syncthreads();                                // every thread is done with stage st
        if (tid == 0 && i + stages < my_tiles) {
            refill_fence();                        // generic-proxy reads before the async refill
            issue(i + stages, st);
        }
    }
}

// ---------------------------------------------------------------------------------------
// Long rows off the 16-byte grid (round 2, MV_CPR with [ADAPTIC_P_XSMEM] = 11): C up to ~18K
// elements, C % 4 != 0 -- 65536 x 1025 ran 0.72-0.74 of the copy peak on the direct
// misaligned-row kernels (a warp per row has 8 vectors per lane: two round trips and a
// butterfly per 4 KB row).  Loading is the row-tile ring above (k <= RTC_KMAX whole rows per
// bulk copy); the reduction uses the WHOLE CTA on all k rows of a tile at once: thread t takes
// columns t + NT*m (m < MX) of every row (k <= KR, a template bound so that absent rows
// cost no predicated instructions) with x[t + NT*m] in registers for the whole kernel,
// so each element costs one conflict-free 32-bit shared load and one FMA.  The k row sums
// leave each warp through a transposing butterfly (offset 16 exchanges 4 of the 8 row
// partials, 8 exchanges 2, 4 exchanges 1, then 2 and 1 finish: 9 shuffles for 8 rows instead
// of 40), and one barrier per tile (per-warp partials double-buffered by tile parity, so the
// same barrier frees the stage for its refill).  Fixed order throughout (P7).
constexpr int RTC_KMAX = 8;

template <class T, int NT, int MX, int KR>
__global__ void __launch_bounds__(NT)
mv_rowtile_cta_kernel(const T* __restrict__ A, const T* __restrict__ X, T* __restrict__ y,
                      int64_t R, int64_t C, int k, int stages)
{
    pdl_prologue();
    extern __shared__ __align__(128) unsigned char smem_raw[];
    __shared__ __align__(8) uint64_t full[RT_MAX_STAGES];
    __shared__ T red[2][NT / 32][RTC_KMAX];
    constexpr int NW = NT / 32;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int Ci = int(C);
    const int64_t total = R * C;
    const int64_t ntiles = (R + k - 1) / k;
    const int64_t tile_w = ((int64_t(k) * C + 6 + 3) / 4) * 4;
    T* ring = reinterpret_cast<T*>(smem_raw);
    const int64_t my_tiles = blockIdx.x < ntiles ? (ntiles - 1 - blockIdx.x) / gridDim.x + 1 : 0;

    if (tid == 0) {
        for (int s = 0; s < stages; ++s) mbar_init(&full[s], 1);
        fence_mbar_init();
    }
    __syncthreads();
    auto issue = [&](int64_t i, int slot) {
        const int64_t r0 = (blockIdx.x + i * gridDim.x) * int64_t(k);
        const int64_t w0 = r0 * C, w1 = min(R, r0 + k) * C;
        const int64_t a0 = w0 & ~int64_t(3);
        int64_t a1 = (w1 + 3) & ~int64_t(3);
        if (a1 > total) a1 = w1 & ~int64_t(3);
        const uint32_t bytes = uint32_t((a1 - a0) * int64_t(sizeof(T)));
        mbar_arrive_expect_tx(&full[slot], bytes);
        if (bytes) bulk_g2s(ring + slot * tile_w, A + a0, bytes, &full[slot]);
    };
    if (tid == 0) {
        const int64_t pre = min(int64_t(stages), my_tiles);
        for (int64_t i = 0; i < pre; ++i) issue(i, int(i));
    }
    T xr[MX];
#pragma unroll
    for (int m = 0; m < MX; ++m) xr[m] = tid + NT * m < Ci ? ld_x(X + tid + NT * m) : T(0);

    int st = 0;
    uint32_t ph = 0;
    for (int64_t i = 0; i < my_tiles; ++i, ring_advance(st, ph, stages)) {
        const int64_t r0 = (blockIdx.x + i * gridDim.x) * int64_t(k);
        const int nrows = int(min(int64_t(k), R - r0));
        const int64_t w0 = r0 * C;
        T* stg = ring + st * tile_w;
        mbar_wait(&full[st], ph);
        const int64_t w1 = w0 + int64_t(nrows) * C;
        if (((w1 + 3) & ~int64_t(3)) > total && (w1 & 3)) {   // the matrix's last < 4 words
            const int64_t a0 = w0 & ~int64_t(3);
            for (int64_t e = (w1 & ~int64_t(3)) + tid; e < w1; e += NT) stg[e - a0] = A[e];
            __syncthreads();
        }
        const T* base = stg + (w0 & 3) + tid;
        T v[RTC_KMAX];
#pragma unroll
        for (int r = 0; r < RTC_KMAX; ++r) v[r] = T(0);
#pragma unroll
        for (int m = 0; m < MX; ++m) {
            if (tid + NT * m < Ci) {
#pragma unroll
                for (int r = 0; r < KR; ++r)          // KR >= k rows: no issue slots for absent rows
                    if (r < nrows) v[r] = mac(base[r * Ci + NT * m], xr[m], v[r]);
            }
        }
        // transposing butterfly: lane bit 4 keeps rows 4b4..4b4+3, bit 3 two of those, bit 2 one
        {
            const bool b4 = lane & 16, b3 = lane & 8, b2 = lane & 4;
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                const T send = b4 ? v[j] : v[j + 4];
                const T keep = b4 ? v[j + 4] : v[j];
                v[j] = keep + __shfl_xor_sync(0xffffffffu, send, 16);
            }
#pragma unroll
            for (int j = 0; j < 2; ++j) {
                const T send = b3 ? v[j] : v[j + 2];
                const T keep = b3 ? v[j + 2] : v[j];
                v[j] = keep + __shfl_xor_sync(0xffffffffu, send, 8);
            }
            {
                const T send = b2 ? v[0] : v[1];
                const T keep = b2 ? v[1] : v[0];
                v[0] = keep + __shfl_xor_sync(0xffffffffu, send, 4);
            }
            v[0] += __shfl_xor_sync(0xffffffffu, v[0], 2);
            v[0] += __shfl_xor_sync(0xffffffffu, v[0], 1);
        }
        const int par = int(i & 1);
        if ((lane & 3) == 0) red[par][warp][lane >> 2] = v[0];    // row (b4 b3 b2) = lane / 4
        __syncthreads();                       // partials written; stage st fully read
        if (tid == 0 && i + stages < my_tiles) {
            refill_fence();
            issue(i + stages, st);
        }
        if (tid < nrows) {
            T s0 = T(0), s1 = T(0);
#pragma unroll
            for (int w = 0; w + 1 < NW; w += 2) { s0 += red[par][w][tid]; s1 += red[par][w + 1][tid]; }
            if (NW & 1) s0 += red[par][NW - 1][tid];
            y[r0 + tid] = s0 + s1;
        }
    }
}

// Rows too long for x in registers (C > 36 NT; MV_CPR / MV_SPLIT with [ADAPTIC_P_XSMEM] = 13):
// the staged whole-CTA reduction above on COLUMN CHUNKS.  Chunk j = columns
// [j W, min(C, (j + 1) W)), W <= NT MX.  Units (chunk j, block of k rows), chunk-major, are
// split into one contiguous range per CTA, so a CTA keeps one chunk of x in registers
// (x[j W + t + NT m]) for most of its units and reloads it when its range crosses into the next
// chunk: x is read from L2 about once per CTA instead of once per row.  A tile is the k row
// segments of one unit, each bulk-copied by its own 16-byte-aligned cover into its slot of the
// stage (row r's segment starts (r C + j W) mod 4 words into its slot: any C, any row
// alignment).  One PRODUCER warp issues the copies (full / empty mbarrier ring) and NT
// consumer threads only reduce, synchronising on a named barrier: with the issuing thread
// inside the consumer loop every tile paid a fixed ~0.7 us (the copy issue waits for TMA queue
// space while the other warps wait at the tile barrier) -- 0.55 of peak at 32 KB tiles.  The k
// row partials leave through the transposing butterfly; unit (j, r) writes part[j R + r], and
// the last CTA of the launch (ticket: the paper's merge kernel) sums each row's chunk
// partials with L lanes per row (each strided over j in order) and an L-lane butterfly.
// Unit, chunk and ring positions advance incrementally (no 64-bit division per tile).  Fixed
// order throughout (P7).
__device__ __forceinline__ void mbar_arrive1(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" :: "r"(smem_u32(bar)) : "memory");
}
template <int NT> __device__ __forceinline__ void consumers_sync() {     // barrier 1: NT threads
    asm volatile("bar.sync 1, %0;" :: "n"(NT) : "memory");
}

template <class T, int NT, int MX, int KR>
__global__ void __launch_bounds__(NT + 32, 1)
mv_chunk_cta_kernel(const T* __restrict__ A, const T* __restrict__ X, T* __restrict__ y,
                    int64_t R, int64_t C, int k, int stages, int W, T* __restrict__ part,
                    unsigned int* __restrict__ cnt)
{
    pdl_prologue();
    extern __shared__ __align__(128) unsigned char smem_raw[];
    __shared__ __align__(8) uint64_t full[RT_MAX_STAGES], empty[RT_MAX_STAGES];
    __shared__ T red[2][NT / 32][RTC_KMAX];
    __shared__ unsigned int flag;
    constexpr int NW = NT / 32;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int64_t total = R * C;
    const int64_t nch = (C + W - 1) / W;
    const int64_t nrb = (R + k - 1) / k;
    const int64_t units = nch * nrb;
    const int64_t G = gridDim.x, b = blockIdx.x;
    const int64_t per = units / G, rem = units % G;
    const int64_t u0 = b * per + (b < rem ? b : rem);
    const int64_t my = per + (b < rem ? 1 : 0);
    const int slot_w = ((W + 6 + 3) / 4) * 4;
    const int64_t stage_w = int64_t(slot_w) * k;
    T* ring = reinterpret_cast<T*>(smem_raw);
    const int64_t j0 = u0 / nrb, rb0 = u0 - j0 * nrb;        // one division per CTA

    if (tid == 0) {
        for (int s = 0; s < stages; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 1); }
        fence_mbar_init();
    }
    __syncthreads();
    // cover [a0, a1) of the segment [w0, w0 + wj): 16-byte aligned, never past the matrix
    auto cover = [&](int64_t w0, int wj, int64_t& a0, int64_t& a1) {
        const int64_t w1 = w0 + wj;
        a0 = w0 & ~int64_t(3);
        a1 = (w1 + 3) & ~int64_t(3);
        if (a1 > total) a1 = w1 & ~int64_t(3);
    };

    if (warp == NW) {                                        // ---- producer warp (lane 0)
        if (lane == 0) {
            int64_t pj = j0, prb = rb0;
            int st = 0;
            uint32_t ph = 0;
            for (int64_t i = 0; i < my; ++i, ring_advance(st, ph, stages)) {
                if (i >= stages) mbar_wait(&empty[st], ph ^ 1u);
                const int64_t r0 = prb * k;
                const int nr = int(min(int64_t(k), R - r0));
                const int64_t c0 = pj * W;
                const int wj = int(min(int64_t(W), C - c0));
                uint32_t bytes = 0;
                for (int r = 0; r < nr; ++r) {
                    int64_t a0, a1;
                    cover((r0 + r) * C + c0, wj, a0, a1);
                    bytes += uint32_t((a1 - a0) * int64_t(sizeof(T)));
                }
                mbar_arrive_expect_tx(&full[st], bytes);
                for (int r = 0; r < nr; ++r) {
                    int64_t a0, a1;
                    cover((r0 + r) * C + c0, wj, a0, a1);
                    if (a1 > a0)
                        bulk_g2s(ring + st * stage_w + int64_t(r) * slot_w, A + a0,
                                 uint32_t((a1 - a0) * int64_t(sizeof(T))), &full[st]);
                }
                if (++prb == nrb) { prb = 0; ++pj; }
            }
        }
    } else {                                                 // ---- NT consumer threads
        T xr[MX];
        int64_t cj = -1, j = j0, rb = rb0;
        int st = 0;
        uint32_t ph = 0;
        for (int64_t i = 0; i < my; ++i, ring_advance(st, ph, stages)) {
            const int64_t c0 = j * W;
            const int wj = int(min(int64_t(W), C - c0));
            if (j != cj) {                                   // this CTA's range entered chunk j
#pragma unroll
                for (int m = 0; m < MX; ++m) xr[m] = tid + NT * m < wj ? ld_x(X + c0 + tid + NT * m) : T(0);
                cj = j;
            }
            const int64_t r0 = rb * k;
            const int nrows = int(min(int64_t(k), R - r0));
            T* stg = ring + st * stage_w;
            mbar_wait(&full[st], ph);
            {                                                // the matrix's last < 4 words
                const int64_t w0 = (r0 + nrows - 1) * C + c0, w1 = w0 + wj;
                if (((w1 + 3) & ~int64_t(3)) > total && (w1 & 3)) {
                    const int64_t a0 = w0 & ~int64_t(3);
                    for (int64_t e = (w1 & ~int64_t(3)) + tid; e < w1; e += NT)
                        stg[int64_t(nrows - 1) * slot_w + (e - a0)] = A[e];
                    consumers_sync<NT>();
                }
            }
            T v[RTC_KMAX];
#pragma unroll
            for (int r = 0; r < RTC_KMAX; ++r) v[r] = T(0);
#pragma unroll
            for (int r = 0; r < KR; ++r) {
                if (r < nrows) {
                    const T* base = stg + r * slot_w + int(((r0 + r) * C + c0) & 3) + tid;
#pragma unroll
                    for (int m = 0; m < MX; ++m)
                        if (tid + NT * m < wj) v[r] = mac(base[NT * m], xr[m], v[r]);
                }
            }
            {                                                // transposing butterfly (as above)
                const bool b4 = lane & 16, b3 = lane & 8, b2 = lane & 4;
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const T send = b4 ? v[q] : v[q + 4];
                    const T keep = b4 ? v[q + 4] : v[q];
                    v[q] = keep + __shfl_xor_sync(0xffffffffu, send, 16);
                }
#pragma unroll
                for (int q = 0; q < 2; ++q) {
                    const T send = b3 ? v[q] : v[q + 2];
                    const T keep = b3 ? v[q + 2] : v[q];
                    v[q] = keep + __shfl_xor_sync(0xffffffffu, send, 8);
                }
                {
                    const T send = b2 ? v[0] : v[1];
                    const T keep = b2 ? v[1] : v[0];
                    v[0] = keep + __shfl_xor_sync(0xffffffffu, send, 4);
                }
                v[0] += __shfl_xor_sync(0xffffffffu, v[0], 2);
                v[0] += __shfl_xor_sync(0xffffffffu, v[0], 1);
            }
            const int par = int(i & 1);
            if ((lane & 3) == 0) red[par][warp][lane >> 2] = v[0];
            consumers_sync<NT>();                            // partials written; stage st fully read
            if (tid == 0) mbar_arrive1(&empty[st]);
            if (tid < nrows) {
                T s0 = T(0), s1 = T(0);
#pragma unroll
                for (int w = 0; w + 1 < NW; w += 2) { s0 += red[par][w][tid]; s1 += red[par][w + 1][tid]; }
                if (NW & 1) s0 += red[par][NW - 1][tid];
                if (nch == 1) y[r0 + tid] = s0 + s1;
                else part[j * R + r0 + tid] = s0 + s1;
            }
            if (++rb == nrb) { rb = 0; ++j; }
        }
    }
    if (nch == 1) return;
    if (ticket_is_last(cnt, unsigned(G), &flag) && warp < NW) {
        int L = 1;                                           // lanes per row
        while (L < 32 && int64_t(2 * L) * R <= NT) L *= 2;
        const int rpp = NT / L;
        const int l = tid % L;
        for (int64_t rbase = 0; rbase < R; rbase += rpp) {
            const int64_t r = rbase + tid / L;
            T s = T(0);
            if (r < R) {
                int64_t q = l;
                for (; q + 7 * L < nch; q += 8 * L) {
                    T pv[8];
#pragma unroll
                    for (int u = 0; u < 8; ++u) pv[u] = ld_partial(part + (q + u * L) * R + r);
#pragma unroll
                    for (int u = 0; u < 8; ++u) s += pv[u];
                }
                for (; q < nch; q += L) s += ld_partial(part + q * R + r);
            }
            for (int o = L / 2; o >= 1; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
            if (l == 0 && r < R) y[r] = s;
        }
    }
}

}  // namespace adaptic
