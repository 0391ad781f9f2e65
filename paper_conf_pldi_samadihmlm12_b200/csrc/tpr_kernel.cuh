// tpr_kernel.cuh -- MV_TPR: thread per row with TMA bulk staging (sm_100a).
//
// The paper's kernel 5 gives each thread "the dot product of a single
// row".  On the MV layout a thread's row is contiguous, so a warp's direct loads
// would not coalesce (Fig. 3a).  The paper's fix is to restructure the
// data on the CPU; its rejected alternative is a coalesced cooperative
// copy into shared memory, rejected for shared-memory size and address
// arithmetic on Fermi.  Neither objection holds on B200 (228 KB smem/SM; the
// TMA engine does the addressing), so this variant stages tiles of NT
// consecutive rows -- a contiguous NT*C*4-byte block -- with cp.async.bulk into a
// STAGES-deep ring guarded by mbarriers, and each thread then reduces its own
// row out of shared memory.  The rotation k' = (k + t) mod (C/4) makes the
// 128-bit shared loads of 8 consecutive threads hit distinct banks.
// SCAL (C % 4 != 0): a tile is still a contiguous NT*C*4-byte block whose size is a
// multiple of 16 (NT*4 = 512 or 1024), so the bulk copies stay 16-byte granular;
// only the last, partial tile copies its < 16-byte remainder with plain loads, and
// x (C*4 bytes) is staged by the threads.  Rows are read as 32-bit words; thread t
// starts at word t*C + rot*t with rot = (C odd ? 0 : 1), so the C+rot words between
// neighbouring threads are odd and the 32 lanes hit 32 distinct banks.
#pragma once

#include "common.cuh"

namespace adaptic {

constexpr int TPR_MAX_STAGES = 8;

// Dynamic smem layout: [x: C elems][stage 0: NT*C (+ NT*C for DOT's b)] ... ; 16B aligned.
template <class T, int NT, bool PERROWX, bool SCAL = false>
__global__ void __launch_bounds__(NT)
mv_tpr_kernel(const T* __restrict__ A, const T* __restrict__ X, T* __restrict__ y,
              int64_t R, int64_t C, int stages)
{
    pdl_prologue();
    using V = vec4_t<T>;
    extern __shared__ __align__(128) unsigned char smem_raw[];
    __shared__ __align__(8) uint64_t full[TPR_MAX_STAGES];
    __shared__ __align__(8) uint64_t xbar;

    const int tid = threadIdx.x;
    const int c4 = int(C / 4);                               // vectors per row (C % 4 == 0)
    const int64_t ntiles = (R + NT - 1) / NT;
    const size_t tile_elems = size_t(NT) * C;
    T* xs = reinterpret_cast<T*>(smem_raw);
    T* ring = xs + (PERROWX ? 0 : ((C + 31) / 32) * 32);      // keep 128B alignment
    const size_t stage_elems = tile_elems * (PERROWX ? 2 : 1);

    // tiles of this CTA: blockIdx.x, blockIdx.x + gridDim.x, ...
    const int64_t my_tiles = blockIdx.x < ntiles ? (ntiles - 1 - blockIdx.x) / gridDim.x + 1 : 0;

    if (tid == 0) {
        for (int s = 0; s < stages; ++s) mbar_init(&full[s], 1);
        mbar_init(&xbar, 1);
        fence_mbar_init();
    }
    __syncthreads();

    auto issue = [&](int64_t i, int slot) {  // local tile i -> ring stage slot (thread 0 only)
        const int64_t tile = blockIdx.x + i * gridDim.x;
        const int64_t r0 = tile * NT;
        const int64_t nrows = min(int64_t(NT), R - r0);
        const uint32_t bytes = uint32_t(nrows * C * sizeof(T)) & (SCAL ? ~15u : ~0u);
        T* dst = ring + size_t(slot) * stage_elems;
        uint64_t* bar = &full[slot];
        mbar_arrive_expect_tx(bar, PERROWX ? 2 * bytes : bytes);
        if (bytes) {
            bulk_g2s(dst, A + r0 * C, bytes, bar);
            if (PERROWX) bulk_g2s(dst + tile_elems, X + r0 * C, bytes, bar);
        }
    };

    if (tid == 0) {
        if (!PERROWX && !SCAL) {
            mbar_arrive_expect_tx(&xbar, uint32_t(C * sizeof(T)));
            bulk_g2s_keep(xs, X, uint32_t(C * sizeof(T)), &xbar);
        }
        const int64_t pre = min(int64_t(stages), my_tiles);
        for (int64_t i = 0; i < pre; ++i) issue(i, int(i));
    }
    if (!PERROWX && !SCAL) mbar_wait(&xbar, 0);
    if (!PERROWX && SCAL) {
        for (int64_t c = tid; c < C; c += NT) xs[c] = ld_x(X + c);
        __syncthreads();
    }

    const V* xv = reinterpret_cast<const V*>(xs);
    int st = 0;
    uint32_t ph = 0;
    for (int64_t i = 0; i < my_tiles; ++i, ring_advance(st, ph, stages)) {
        mbar_wait(&full[st], ph);
        const int64_t r0 = (blockIdx.x + i * gridDim.x) * int64_t(NT);
        if constexpr (SCAL) {
            T* stg = ring + size_t(st) * stage_elems;
            const int64_t nel = min(int64_t(NT), R - r0) * C;
            const int64_t bulk = int64_t((uint64_t(nel) * sizeof(T)) & ~uint64_t(15)) / int64_t(sizeof(T));
            if (bulk < nel) {                 // last partial tile: < 16-byte remainder
                for (int64_t e = bulk + tid; e < nel; e += NT) {
                    stg[e] = A[r0 * C + e];
                    if (PERROWX) stg[tile_elems + e] = X[r0 * C + e];
                }
                __syncthreads();
            }
            const T* ar = stg + size_t(tid) * C;
            const T* br = PERROWX ? stg + tile_elems + size_t(tid) * C : xs;
            if (r0 + tid < R) {
                const int Ci = int(C);
                T acc0 = T(0), acc1 = T(0);
                int k = (Ci & 1) ? 0 : tid % Ci;
                int n = 0;
                for (; n + 1 < Ci; n += 2) {
                    const int k1 = (k + 1 == Ci) ? 0 : k + 1;
                    acc0 = mac(ar[k], br[k], acc0);
                    acc1 = mac(ar[k1], br[k1], acc1);
                    k = (k1 + 1 == Ci) ? 0 : k1 + 1;
                }
                if (n < Ci) acc0 = mac(ar[k], br[k], acc0);
                y[r0 + tid] = acc0 + acc1;
            }
            __syncthreads();
            if (tid == 0 && i + stages < my_tiles) {
                refill_fence();
                issue(i + stages, st);
            }
            continue;
        }
        const V* av = reinterpret_cast<const V*>(ring + size_t(st) * stage_elems) + size_t(tid) * c4;
        const V* bv = PERROWX ? reinterpret_cast<const V*>(ring + size_t(st) * stage_elems + tile_elems) + size_t(tid) * c4
                              : xv;
        if (r0 + tid < R) {
            V acc0 = zero_of<V>(), acc1 = zero_of<V>();
            int k = tid % c4;
            int n = 0;
            for (; n + 1 < c4; n += 2) {
                const int k1 = (k + 1 == c4) ? 0 : k + 1;
                vmac(acc0, av[k], bv[k]);
                vmac(acc1, av[k1], bv[k1]);
                k = (k1 + 1 == c4) ? 0 : k1 + 1;
            }
            if (n < c4) vmac(acc0, av[k], bv[k]);
            y[r0 + tid] = vsum(vadd(acc0, acc1));
        }
        __syncthreads();                      // every thread is done with stage st
        if (tid == 0 && i + stages < my_tiles) {
            refill_fence();              // generic-proxy reads before async-proxy refill
            issue(i + stages, st);
        }
    }
}

}  // namespace adaptic
