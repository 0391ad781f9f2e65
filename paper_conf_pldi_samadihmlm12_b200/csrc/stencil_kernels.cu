// stencil_kernels.cu -- five-point stencil with input-adaptive super tiles (SURVEY 8(f)
// rank 4, second item), sm_100a.
//
// The paper's neighbouring-access optimization (Sec. 4.1.2): a point and
// its four neighbours are read for every output, so reading them straight from
// global memory touches the input five times; instead each block brings a tile plus
// its halo into shared memory, and to shrink the halo overhead several tiles are
// merged into a SUPER TILE whose size and shape follow the input: "for small input
// sizes it is beneficial to use smaller super tiles in order to have more blocks.
// Large super tiles are advantageous for large input sizes", chosen by the reuse
// metric sum(element accesses) / halo size.  v = c u + n (T + B + L + R)
// inside, v = u on the edge (reading R19); x holds {c, n} on the device.
//
//   st_direct_kernel  no shared memory: 4 outputs per thread, neighbours from L1/L2
//                     (a grid-stride sweep keeps the rows above and below L2-resident)
//   st_tile_kernel    super tiles of TH x TW outputs; the (TH+2) x (TW+8) input block
//                     (16-byte-aligned halo of 4 columns; 1 used) arrives by TMA bulk
//                     copies, one per row, double-buffered: the next super tile of the
//                     CTA streams in while the current one is computed.
#include "common.cuh"
#include "launch.h"

namespace adaptic {

__device__ __forceinline__ float st_point(float c, float n, float ce, float t, float b, float l, float r) {
    return fmaf(c, ce, n * ((t + b) + (l + r)));
}

// --------------------------------------------------------------------------- direct
// q / nvr by multiply-high (Granlund-Montgomery, 33-bit magic 2^32 + m): exact for every
// 32-bit q; a 64-bit division per element cost ~60 integer instructions (half the issue
// slots of the kernel, SASS count) -- grids below 2^32 vectors take this path.
struct FastDiv32 {
    uint32_t d, m, l;
    __device__ explicit FastDiv32(uint32_t dd) : d(dd) {
        l = dd > 1 ? 32u - uint32_t(__clz(dd - 1u)) : 0u;
        m = uint32_t((((uint64_t(1) << l) - dd) << 32) / dd + 1u);
    }
    __device__ __forceinline__ uint32_t div(uint32_t q) const {
        return uint32_t((uint64_t(__umulhi(q, m)) + q) >> l);
    }
};

template <bool VEC, int NT>
__global__ void __launch_bounds__(NT)
st_direct_kernel(const float* __restrict__ u, const float* __restrict__ coef, float* __restrict__ v,
                 int64_t H, int64_t W)
{
    pdl_prologue();
    const float c = __ldg(coef), n = __ldg(coef + 1);
    const int64_t nvr = VEC ? W / 4 : W;              // vectors per row
    const int64_t total = H * nvr;
    const bool small = total <= int64_t(0xffffffffu) - int64_t(gridDim.x) * NT;
    const FastDiv32 fd(uint32_t(small ? nvr : 1));
    for (int64_t q = int64_t(blockIdx.x) * NT + threadIdx.x; q < total; q += int64_t(gridDim.x) * NT) {
        int64_t i, k;
        if (small) { i = fd.div(uint32_t(q)); k = q - i * nvr; }
        else { i = q / nvr; k = q - i * nvr; }
        const int64_t at = i * W + (VEC ? 4 * k : k);
        if constexpr (VEC) {
            const float4 ce = *reinterpret_cast<const float4*>(u + at);
            float4 o = ce;
            if (i > 0 && i < H - 1) {
                const float4 t = __ldg(reinterpret_cast<const float4*>(u + at - W));
                const float4 b = __ldg(reinterpret_cast<const float4*>(u + at + W));
                const float l = k > 0 ? __ldg(u + at - 1) : 0.f;
                const float r = k < nvr - 1 ? __ldg(u + at + 4) : 0.f;
                if (k > 0) o.x = st_point(c, n, ce.x, t.x, b.x, l, ce.y);
                o.y = st_point(c, n, ce.y, t.y, b.y, ce.x, ce.z);
                o.z = st_point(c, n, ce.z, t.z, b.z, ce.y, ce.w);
                if (k < nvr - 1) o.w = st_point(c, n, ce.w, t.w, b.w, ce.z, r);
            }
            *reinterpret_cast<float4*>(v + at) = o;
        } else {
            const float ce = u[at];
            float o = ce;
            if (i > 0 && i < H - 1 && k > 0 && k < W - 1)
                o = st_point(c, n, ce, __ldg(u + at - W), __ldg(u + at + W), __ldg(u + at - 1), __ldg(u + at + 1));
            v[at] = o;
        }
    }
}

// Row-major sweep, two float4 outputs per thread per step (q and q + stride): all six
// float4 and four scalar loads are issued before the first FMA, v is stored evict-first
// (keeps u's neighbour rows in L2 longer).  Planner ORDER 4.
template <int NT>
__global__ void __launch_bounds__(NT)
st_direct2_kernel(const float* __restrict__ u, const float* __restrict__ coef, float* __restrict__ v,
                  int64_t H, int64_t W)
{
    pdl_prologue();
    const float c = __ldg(coef), n = __ldg(coef + 1);
    const int64_t nvr = W / 4;
    const int64_t total = H * nvr;
    const int64_t stride = int64_t(gridDim.x) * NT;
    const bool small = total + stride <= int64_t(0xffffffffu);
    const FastDiv32 fd(uint32_t(small ? nvr : 1));
    const float4* __restrict__ u4 = reinterpret_cast<const float4*>(u);
    float4* __restrict__ v4 = reinterpret_cast<float4*>(v);
    for (int64_t q0 = int64_t(blockIdx.x) * NT + threadIdx.x; q0 < total; q0 += 2 * stride) {
        int64_t qq[2], i[2], k[2];
        bool ok[2], in[2];
        float4 ce[2], t[2], b[2];
        float l[2], r[2];
#pragma unroll
        for (int e = 0; e < 2; ++e) {
            qq[e] = q0 + e * stride;
            ok[e] = qq[e] < total;
            const int64_t q = ok[e] ? qq[e] : q0;
            i[e] = small ? int64_t(fd.div(uint32_t(q))) : q / nvr;
            k[e] = q - i[e] * nvr;
            in[e] = i[e] > 0 && i[e] < H - 1;
            ce[e] = __ldg(u4 + q);
            t[e] = in[e] ? __ldg(u4 + q - nvr) : ce[e];
            b[e] = in[e] ? __ldg(u4 + q + nvr) : ce[e];
            l[e] = (in[e] && k[e] > 0) ? __ldg(u + 4 * q - 1) : 0.f;
            r[e] = (in[e] && k[e] < nvr - 1) ? __ldg(u + 4 * q + 4) : 0.f;
        }
#pragma unroll
        for (int e = 0; e < 2; ++e) {
            if (!ok[e]) continue;
            float4 o = ce[e];
            if (in[e]) {
                if (k[e] > 0) o.x = st_point(c, n, ce[e].x, t[e].x, b[e].x, l[e], ce[e].y);
                o.y = st_point(c, n, ce[e].y, t[e].y, b[e].y, ce[e].x, ce[e].z);
                o.z = st_point(c, n, ce[e].z, t[e].z, b[e].z, ce[e].y, ce[e].w);
                if (k[e] < nvr - 1) o.w = st_point(c, n, ce[e].w, t[e].w, b[e].w, ce[e].z, r[e]);
            }
            __stcs(v4 + qq[e], o);
        }
    }
}

// --------------------------------------------------------------------------- L2 strips
// The B200 form of the paper's super tile: the grid is cut into vertical strips of SV
// = NT V float4 columns and the work items (strip, row) are taken strip-major, so the
// CTAs in flight at any time cover a band of consecutive rows of ONE strip and a row's
// top and bottom neighbours are read by concurrently running CTAs -- the reuse is
// captured by L2 (126 MB) instead of a shared-memory halo.  Without strips a long row
// (8 x 8M: 32 MB per row) is evicted before the next row needs it (measured 3.9 TB/s
// row-major vs 6.2 with strips; equal for rows up to ~2 MB).  Each thread issues its V centre/top/bottom float4 loads and its
// 2 V edge scalars before the first FMA; v is stored evict-first.
template <int NT, int V>
__global__ void __launch_bounds__(NT)
st_strip_kernel(const float* __restrict__ u, const float* __restrict__ coef, float* __restrict__ v,
                int64_t H, int64_t W)
{
    pdl_prologue();
    constexpr int SV = NT * V;
    const float c = __ldg(coef), n = __ldg(coef + 1);
    const int64_t nvr = W / 4;
    const int64_t nstrips = (nvr + SV - 1) / SV;
    const int64_t items = nstrips * H;
    const float4* __restrict__ u4 = reinterpret_cast<const float4*>(u);
    float4* __restrict__ v4 = reinterpret_cast<float4*>(v);
    for (int64_t it = blockIdx.x; it < items; it += gridDim.x) {
        const int64_t s = it / H, i = it - s * H;
        const bool inner = i > 0 && i < H - 1;
        const int64_t row = i * nvr;
        float4 ce[V], t[V], b[V];
        float l[V], r[V];
#pragma unroll
        for (int q = 0; q < V; ++q) {
            const int64_t k = s * SV + q * NT + threadIdx.x;
            const int64_t kk = k < nvr ? k : nvr - 1;             // stay in bounds; result discarded
            ce[q] = __ldg(u4 + row + kk);
            if (inner) {
                t[q] = __ldg(u4 + row - nvr + kk);
                b[q] = __ldg(u4 + row + nvr + kk);
                l[q] = kk > 0 ? __ldg(u + 4 * (row + kk) - 1) : 0.f;
                r[q] = kk < nvr - 1 ? __ldg(u + 4 * (row + kk) + 4) : 0.f;
            }
        }
#pragma unroll
        for (int q = 0; q < V; ++q) {
            const int64_t k = s * SV + q * NT + threadIdx.x;
            if (k >= nvr) continue;
            float4 o = ce[q];
            if (inner) {
                if (k > 0) o.x = st_point(c, n, ce[q].x, t[q].x, b[q].x, l[q], ce[q].y);
                o.y = st_point(c, n, ce[q].y, t[q].y, b[q].y, ce[q].x, ce[q].z);
                o.z = st_point(c, n, ce[q].z, t[q].z, b[q].z, ce[q].y, ce[q].w);
                if (k < nvr - 1) o.w = st_point(c, n, ce[q].w, t[q].w, b[q].w, ce[q].z, r[q]);
            }
            __stcs(v4 + row + k, o);
        }
    }
}

// --------------------------------------------------------------------------- column sweep
// Register sliding window: a CTA owns NT float4 columns x TH rows and each thread walks
// down its column keeping rows i-1, i, i+1 in registers, so every input float4 is loaded
// ONCE (plus 2 halo rows per tile) instead of three times through L1/L2; the left/right
// neighbours come from the adjacent lanes by shuffles (scalar loads only at the warp
// edges).  The next D rows are loaded together (D float4 in flight per thread).  Tiles
// are taken column-strip-major so vertically adjacent tiles -- which share halo rows --
// run at the same time.
template <int NT, int D>
__global__ void __launch_bounds__(NT)
st_column_kernel(const float* __restrict__ u, const float* __restrict__ coef, float* __restrict__ v,
                 int64_t H, int64_t W, int TH)
{
    pdl_prologue();
    const float c = __ldg(coef), n = __ldg(coef + 1);
    const int64_t nvr = W / 4;
    const int64_t tiles_c = (nvr + NT - 1) / NT, tiles_r = (H + TH - 1) / TH;
    const int64_t ntiles = tiles_c * tiles_r;
    const float4* __restrict__ u4 = reinterpret_cast<const float4*>(u);
    float4* __restrict__ v4 = reinterpret_cast<float4*>(v);
    const int lane = threadIdx.x & 31;
    const float4 z = make_float4(0.f, 0.f, 0.f, 0.f);
    for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
        const int64_t tc = t / tiles_r, tr = t - tc * tiles_r;
        const int64_t k = tc * NT + threadIdx.x;
        const bool ok = k < nvr;
        const int64_t kk = ok ? k : nvr - 1;                    // in bounds; results discarded
        const int64_t r0 = tr * TH, r1 = min(H, r0 + TH);
        const bool lo_edge = (k == 0), hi_edge = (k == nvr - 1);
        // lane 0 / lane 31 (and the last column) take their outer neighbour from memory
        const bool need_l = (lane == 0) && k > 0 && ok;          // (idle lanes read nothing: kk is clamped)
        const bool need_r = (lane == 31 || threadIdx.x == NT - 1) && k < nvr - 1;
        float4 up = r0 > 0 ? __ldg(u4 + (r0 - 1) * nvr + kk) : z;
        float4 q[D + 1];
#pragma unroll
        for (int d = 0; d <= D; ++d) q[d] = (r0 + d < H) ? __ldg(u4 + (r0 + d) * nvr + kk) : z;
        for (int64_t i = r0; i < r1; i += D) {
#pragma unroll
            for (int d = 0; d < D; ++d) {
                const int64_t row = i + d;
                if (row >= r1) break;
                const float4 ce = q[d], dn = q[d + 1];
                float l = __shfl_up_sync(0xffffffffu, ce.w, 1);
                float r = __shfl_down_sync(0xffffffffu, ce.x, 1);
                if (need_l) l = __ldg(u + 4 * (row * nvr + kk) - 1);
                if (need_r) r = __ldg(u + 4 * (row * nvr + kk) + 4);
                float4 o = ce;
                if (row > 0 && row < H - 1) {
                    if (!lo_edge) o.x = st_point(c, n, ce.x, up.x, dn.x, l, ce.y);
                    o.y = st_point(c, n, ce.y, up.y, dn.y, ce.x, ce.z);
                    o.z = st_point(c, n, ce.z, up.z, dn.z, ce.y, ce.w);
                    if (!hi_edge) o.w = st_point(c, n, ce.w, up.w, dn.w, ce.z, r);
                }
                if (ok) __stcs(v4 + row * nvr + k, o);
                up = ce;
            }
            q[0] = q[D];
#pragma unroll
            for (int d = 1; d <= D; ++d)                        // rows up to r1 (the last row's dn)
                q[d] = (i + D + d < H && i + D + d <= r1) ? __ldg(u4 + (i + D + d) * nvr + kk) : z;
        }
    }
}

// --------------------------------------------------------------------------- super tiles
// Shared buffer b holds input rows row0-1 .. row0+TH (clamped to the grid) and columns
// col0-4 .. col0+TW+3 (clamped), at smem column (global column - col0 + 4).
template <int TH, int TW, int NT>
__global__ void __launch_bounds__(NT)
st_tile_kernel(const float* __restrict__ u, const float* __restrict__ coef, float* __restrict__ v,
               int64_t H, int64_t W)
{
    pdl_prologue();
    constexpr int SW = TW + 8;                        // smem row pitch (floats), 16-byte multiple
    constexpr int SH = TH + 2;
    extern __shared__ __align__(128) unsigned char dyn_smem[];
    float* buf = reinterpret_cast<float*>(dyn_smem);  // [2][SH][SW]
    __shared__ __align__(8) uint64_t bar[2];
    const float c = __ldg(coef), n = __ldg(coef + 1);
    const int64_t tiles_c = (W + TW - 1) / TW, tiles_r = (H + TH - 1) / TH;
    const int64_t ntiles = tiles_r * tiles_c;
    const int tid = threadIdx.x;
    const int64_t my = blockIdx.x < ntiles ? (ntiles - 1 - blockIdx.x) / gridDim.x + 1 : 0;

    auto issue = [&](int64_t li) {                    // thread 0: local tile li -> buffer li & 1
        const int64_t tile = blockIdx.x + li * gridDim.x;
        const int64_t tr = tile / tiles_c, tc = tile - tr * tiles_c;
        const int64_t row0 = tr * TH, col0 = tc * TW;
        const int64_t r_lo = max(row0 - 1, int64_t(0)), r_hi = min(row0 + TH + 1, H);
        const int64_t c_lo = max(col0 - 4, int64_t(0)), c_hi = min(col0 + TW + 4, W);
        const uint32_t bytes = uint32_t(c_hi - c_lo) * 4u;
        float* dst = buf + (li & 1) * (SH * SW);
        mbar_arrive_expect_tx(&bar[li & 1], bytes * uint32_t(r_hi - r_lo));
        for (int64_t r = r_lo; r < r_hi; ++r)
            bulk_g2s(dst + (r - row0 + 1) * SW + (c_lo - col0 + 4), u + r * W + c_lo, bytes, &bar[li & 1]);
    };
    if (tid == 0) {
        mbar_init(&bar[0], 1); mbar_init(&bar[1], 1);
        fence_mbar_init();
        if (my > 0) issue(0);
        if (my > 1) issue(1);
    }
    __syncthreads();
    constexpr int TWV = TW / 4;
    for (int64_t li = 0; li < my; ++li) {
        const int64_t tile = blockIdx.x + li * gridDim.x;
        const int64_t tr = tile / tiles_c, tc = tile - tr * tiles_c;
        const int64_t row0 = tr * TH, col0 = tc * TW;
        mbar_wait(&bar[li & 1], uint32_t((li >> 1) & 1));
        const float* s = buf + (li & 1) * (SH * SW);
        for (int e = tid; e < TH * TWV; e += NT) {
            const int rr = e / TWV, kv = e - rr * TWV;
            const int64_t i = row0 + rr, j = col0 + 4 * kv;
            if (i >= H || j >= W) continue;
            const float* sc = s + (rr + 1) * SW + 4 + 4 * kv;
            const float4 ce = *reinterpret_cast<const float4*>(sc);
            float4 o = ce;
            if (i > 0 && i < H - 1) {
                const float4 t = *reinterpret_cast<const float4*>(sc - SW);
                const float4 b = *reinterpret_cast<const float4*>(sc + SW);
                if (j > 0) o.x = st_point(c, n, ce.x, t.x, b.x, sc[-1], ce.y);
                o.y = st_point(c, n, ce.y, t.y, b.y, ce.x, ce.z);
                o.z = st_point(c, n, ce.z, t.z, b.z, ce.y, ce.w);
                if (j + 4 < W) o.w = st_point(c, n, ce.w, t.w, b.w, ce.z, sc[4]);
            }
            *reinterpret_cast<float4*>(v + i * W + j) = o;
        }
        __syncthreads();                              // buffer li & 1 is free again
        if (tid == 0 && li + 2 < my) {
            fence_proxy_async();
            issue(li + 2);
        }
    }
}

// --------------------------------------------------------------------------- instances
void* st_direct_fn(bool vec) {
    return vec ? reinterpret_cast<void*>(&st_direct_kernel<true, 256>)
               : reinterpret_cast<void*>(&st_direct_kernel<false, 256>);
}

void* st_strip_fn() { return reinterpret_cast<void*>(&st_strip_kernel<256, 4>); }
void* st_direct2_fn() { return reinterpret_cast<void*>(&st_direct2_kernel<256>); }
void* st_column_fn() { return reinterpret_cast<void*>(&st_column_kernel<256, 4>); }

template <int TH>
static void* st_tile_w(int TW) {
    switch (TW) {
        case 128: return reinterpret_cast<void*>(&st_tile_kernel<TH, 128, 256>);
        case 256: return reinterpret_cast<void*>(&st_tile_kernel<TH, 256, 256>);
        case 512: return reinterpret_cast<void*>(&st_tile_kernel<TH, 512, 256>);
        default: return nullptr;
    }
}

void* st_tile_fn(int TH, int TW) {
    switch (TH) {
        case 4: return st_tile_w<4>(TW);
        case 8: return st_tile_w<8>(TW);
        case 16: return st_tile_w<16>(TW);
        case 32: return st_tile_w<32>(TW);
        default: return nullptr;
    }
}

}  // namespace adaptic
