// Scratch experiments: what load structure reaches HBM peak for a 256 MiB MV / TMV.
#include <cstdio>
#include <cstdint>
#include <vector>
#include <algorithm>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("err %s line %d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

__device__ __forceinline__ float4 lds256(const float4* p) {
    float4 v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::256B.v4.f32 {%0,%1,%2,%3}, [%4];"
        : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
    return v;
}
__device__ __forceinline__ float4 ldcs(const float4* p) { return __ldcs(p); }
__device__ __forceinline__ void fma4(float4& acc, const float4& a, const float4& b) {
    acc.x = fmaf(a.x, b.x, acc.x); acc.y = fmaf(a.y, b.y, acc.y); acc.z = fmaf(a.z, b.z, acc.z); acc.w = fmaf(a.w, b.w, acc.w);
}

__global__ void init(float* p, int64_t n) {
    for (int64_t i = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; i < n; i += int64_t(gridDim.x) * blockDim.x)
        p[i] = float((i * 2654435761u) % 1000) * 1e-3f - 0.5f;
}

// pure read ceiling: each thread sums float4s grid-stride, U loads in flight
template <int U>
__global__ void __launch_bounds__(256) readsum(const float4* __restrict__ A, int64_t n4, float* out) {
    float4 acc = make_float4(0, 0, 0, 0);
    int64_t stride = int64_t(gridDim.x) * 256;
    int64_t i = blockIdx.x * 256 + threadIdx.x;
    for (; i + stride * (U - 1) < n4; i += stride * U) {
        float4 a[U];
#pragma unroll
        for (int u = 0; u < U; ++u) a[u] = lds256(A + i + stride * u);
#pragma unroll
        for (int u = 0; u < U; ++u) { acc.x += a[u].x; acc.y += a[u].y; acc.z += a[u].z; acc.w += a[u].w; }
    }
    if (acc.x == 12345.f) out[0] = acc.y + acc.z + acc.w;
}

// WPR, x via __ldg (baseline)
template <int U, int XMODE>   // XMODE 0: __ldg, 1: smem (staged once per CTA)
__global__ void __launch_bounds__(256) wpr(const float4* __restrict__ A, const float4* __restrict__ X, float* y, int64_t R, int64_t nv) {
    extern __shared__ float4 xs[];
    if (XMODE == 1) {
        for (int64_t v = threadIdx.x; v < nv; v += 256) xs[v] = X[v];
        __syncthreads();
    }
    const int lane = threadIdx.x & 31;
    int64_t warp = (int64_t(blockIdx.x) * 256 + threadIdx.x) >> 5;
    int64_t nw = (int64_t(gridDim.x) * 256) >> 5;
    for (int64_t row = warp; row < R; row += nw) {
        const float4* Ar = A + row * nv;
        float4 acc[U];
#pragma unroll
        for (int u = 0; u < U; ++u) acc[u] = make_float4(0, 0, 0, 0);
        for (int64_t j = lane; j + 32 * (U - 1) < nv; j += 32 * U) {
            float4 a[U];
#pragma unroll
            for (int u = 0; u < U; ++u) a[u] = lds256(Ar + j + 32 * u);
#pragma unroll
            for (int u = 0; u < U; ++u) fma4(acc[u], a[u], XMODE == 1 ? xs[j + 32 * u] : __ldg(X + j + 32 * u));
        }
        float s = 0;
#pragma unroll
        for (int u = 0; u < U; ++u) s += (acc[u].x + acc[u].y) + (acc[u].z + acc[u].w);
        for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(~0u, s, o);
        if (lane == 0) y[row] = s;
    }
}

// TMV col: thread per float4 of outputs, C small, all C rows loaded at once (x in regs via __ldg of scalars)
template <int CC>
__global__ void __launch_bounds__(256) tmvcol(const float4* __restrict__ B, const float* __restrict__ X, float4* y, int64_t rv) {
    float xr[CC];
#pragma unroll
    for (int c = 0; c < CC; ++c) xr[c] = __ldg(X + c);
    for (int64_t r = blockIdx.x * 256 + threadIdx.x; r < rv; r += int64_t(gridDim.x) * 256) {
        float4 a[CC];
#pragma unroll
        for (int c = 0; c < CC; ++c) a[c] = lds256(B + c * rv + r);
        float4 acc = make_float4(0, 0, 0, 0);
#pragma unroll
        for (int c = 0; c < CC; ++c) { acc.x = fmaf(a[c].x, xr[c], acc.x); acc.y = fmaf(a[c].y, xr[c], acc.y); acc.z = fmaf(a[c].z, xr[c], acc.z); acc.w = fmaf(a[c].w, xr[c], acc.w); }
        y[r] = acc;
    }
}

// TMV col with two output vectors per thread per iteration (more MLP)
template <int CC, int RPT>
__global__ void __launch_bounds__(256) tmvcol2(const float4* __restrict__ B, const float* __restrict__ X, float4* y, int64_t rv) {
    float xr[CC];
#pragma unroll
    for (int c = 0; c < CC; ++c) xr[c] = __ldg(X + c);
    int64_t stride = int64_t(gridDim.x) * 256;
    for (int64_t r = blockIdx.x * 256 + threadIdx.x; r < rv; r += stride * RPT) {
        float4 a[RPT][CC];
#pragma unroll
        for (int k = 0; k < RPT; ++k)
#pragma unroll
            for (int c = 0; c < CC; ++c) a[k][c] = (r + k * stride < rv) ? lds256(B + c * rv + r + k * stride) : make_float4(0,0,0,0);
#pragma unroll
        for (int k = 0; k < RPT; ++k) {
            float4 acc = make_float4(0, 0, 0, 0);
#pragma unroll
            for (int c = 0; c < CC; ++c) { acc.x = fmaf(a[k][c].x, xr[c], acc.x); acc.y = fmaf(a[k][c].y, xr[c], acc.y); acc.z = fmaf(a[k][c].z, xr[c], acc.z); acc.w = fmaf(a[k][c].w, xr[c], acc.w); }
            if (r + k * stride < rv) y[r + k * stride] = acc;
        }
    }
}

template <class F>
float timeit(F f, int reps = 20) {
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    for (int i = 0; i < 3; ++i) f();
    cudaDeviceSynchronize();
    std::vector<float> ts;
    for (int i = 0; i < reps; ++i) {
        cudaEventRecord(a); f(); cudaEventRecord(b); cudaEventSynchronize(b);
        float ms; cudaEventElapsedTime(&ms, a, b); ts.push_back(ms);
    }
    std::sort(ts.begin(), ts.end());
    return ts[reps / 2];
}
#include <algorithm>

int main() {
    const int64_t N = int64_t(1) << 26;   // 256 MiB fp32
    float *A, *X, *Y;
    CK(cudaMalloc(&A, N * 4)); CK(cudaMalloc(&X, 8 << 20)); CK(cudaMalloc(&Y, 64 << 20));
    init<<<1184, 256>>>(A, N); init<<<148, 256>>>(X, 2 << 20);
    CK(cudaDeviceSynchronize());
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    auto gb = [&](double bytes, float ms) { return bytes / (ms * 1e-3) / 1e9; };
    for (int occ : {4, 8, 16}) {
        float ms = timeit([&] { readsum<8><<<sms * occ, 256>>>((const float4*)A, N / 4, Y); });
        printf("readsum U=8 occ=%d: %.1f us %.0f GB/s\n", occ, ms * 1e3, gb(N * 4.0, ms));
        ms = timeit([&] { readsum<4><<<sms * occ, 256>>>((const float4*)A, N / 4, Y); });
        printf("readsum U=4 occ=%d: %.1f us %.0f GB/s\n", occ, ms * 1e3, gb(N * 4.0, ms));
    }
    const int64_t R = 8192, C = 8192;
    for (int occ : {2, 4, 8}) {
        float ms = timeit([&] { wpr<8, 0><<<sms * occ, 256>>>((const float4*)A, (const float4*)X, Y, R, C / 4); });
        printf("wpr U=8 ldg occ=%d: %.1f us %.0f GB/s\n", occ, ms * 1e3, gb(N * 4.0, ms));
        cudaFuncSetAttribute(wpr<8, 1>, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 << 10);
        cudaFuncSetAttribute(wpr<4, 1>, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 << 10);
        ms = timeit([&] { wpr<8, 1><<<sms * occ, 256, C * 4>>>((const float4*)A, (const float4*)X, Y, R, C / 4); });
        printf("wpr U=8 smem occ=%d: %.1f us %.0f GB/s\n", occ, ms * 1e3, gb(N * 4.0, ms));
        ms = timeit([&] { wpr<4, 1><<<sms * occ, 256, C * 4>>>((const float4*)A, (const float4*)X, Y, R, C / 4); });
        printf("wpr U=4 smem occ=%d: %.1f us %.0f GB/s\n", occ, ms * 1e3, gb(N * 4.0, ms));
    }
    {
        const int64_t Rt = int64_t(1) << 23;  // 8M outputs, C = 8
        for (int occ : {2, 4, 8}) {
            float ms = timeit([&] { tmvcol<8><<<sms * occ, 256>>>((const float4*)A, X, (float4*)Y, Rt / 4); });
            printf("tmvcol C=8 occ=%d: %.1f us %.0f GB/s\n", occ, ms * 1e3, gb(N * 4.0 + Rt * 4, ms));
            ms = timeit([&] { tmvcol2<8, 2><<<sms * occ, 256>>>((const float4*)A, X, (float4*)Y, Rt / 4); });
            printf("tmvcol2 C=8 R2 occ=%d: %.1f us %.0f GB/s\n", occ, ms * 1e3, gb(N * 4.0 + Rt * 4, ms));
        }
        const int64_t R2 = int64_t(1) << 19;  // 512K outputs, C = 128: 16 row-batches of 8
        float ms = timeit([&] { for (int k = 0; k < 1; ++k) tmvcol<8><<<sms * 4, 256>>>((const float4*)A, X, (float4*)Y, R2 / 4); });
        printf("(ref) tmvcol C=8 on R=512K: %.1f us\n", ms * 1e3);
    }
    return 0;
}
