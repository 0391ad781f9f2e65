// Does the access order matter?  256 MiB read: linear grid-stride vs per-CTA contiguous chunks.
#include <cstdio>
#include <cstdint>
#include <vector>
#include <algorithm>
#include <cuda_runtime.h>

__device__ __forceinline__ float4 lds(const float4* p) {
    float4 v;
    asm("ld.global.nc.L1::no_allocate.L2::256B.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
    return v;
}
template <int U, int NT>
__global__ void __launch_bounds__(NT) linear(const float4* __restrict__ A, int64_t n4, float* out) {
    float4 acc = make_float4(0, 0, 0, 0);
    int64_t stride = int64_t(gridDim.x) * NT;
    int64_t i = blockIdx.x * NT + threadIdx.x;
    for (; i + stride * (U - 1) < n4; i += stride * U) {
        float4 a[U];
#pragma unroll
        for (int u = 0; u < U; ++u) a[u] = lds(A + i + stride * u);
#pragma unroll
        for (int u = 0; u < U; ++u) { acc.x += a[u].x; acc.y += a[u].y; acc.z += a[u].z; acc.w += a[u].w; }
    }
    if (acc.x == 12345.f) out[0] = acc.y;
}
// each work unit = contiguous chunk of `chunk4` float4; CTAs grid-stride over units
template <int U, int NT>
__global__ void __launch_bounds__(NT) chunked(const float4* __restrict__ A, int64_t n4, int64_t chunk4, float* out) {
    float4 acc = make_float4(0, 0, 0, 0);
    const int64_t nunits = n4 / chunk4;
    for (int64_t unit = blockIdx.x; unit < nunits; unit += gridDim.x) {
        const float4* Au = A + unit * chunk4;
        int64_t i = threadIdx.x;
        for (; i + NT * (U - 1) < chunk4; i += NT * U) {
            float4 a[U];
#pragma unroll
            for (int u = 0; u < U; ++u) a[u] = lds(Au + i + NT * u);
#pragma unroll
            for (int u = 0; u < U; ++u) { acc.x += a[u].x; acc.y += a[u].y; acc.z += a[u].z; acc.w += a[u].w; }
        }
    }
    if (acc.x == 12345.f) out[0] = acc.y;
}

template <class F> float timeit(F f, int reps = 20) {
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    for (int i = 0; i < 3; ++i) f();
    cudaDeviceSynchronize();
    std::vector<float> ts;
    for (int i = 0; i < reps; ++i) { cudaEventRecord(a); f(); cudaEventRecord(b); cudaEventSynchronize(b); float ms; cudaEventElapsedTime(&ms, a, b); ts.push_back(ms); }
    std::sort(ts.begin(), ts.end());
    return ts[reps / 2];
}
// back-to-back: 10 launches between two events -> per-launch time without launch gaps
template <class F> float timeit_b2b(F f, int n = 10) {
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    for (int i = 0; i < 3; ++i) f();
    cudaDeviceSynchronize();
    cudaEventRecord(a); for (int i = 0; i < n; ++i) f(); cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b); return ms / n;
}

int main() {
    const int64_t N = int64_t(1) << 26;
    float *A, *Y;
    cudaMalloc(&A, N * 4); cudaMalloc(&Y, 1024);
    cudaMemset(A, 0, N * 4);
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    auto gb = [&](float ms) { return N * 4.0 / (ms * 1e-3) / 1e9; };
    for (int occ : {4, 8}) {
        printf("linear U8 NT256 occ%d: single %.0f  b2b %.0f GB/s\n", occ,
               gb(timeit([&] { linear<8, 256><<<sms * occ, 256>>>((const float4*)A, N / 4, Y); })),
               gb(timeit_b2b([&] { linear<8, 256><<<sms * occ, 256>>>((const float4*)A, N / 4, Y); })));
        printf("linear U4 NT256 occ%d: single %.0f  b2b %.0f GB/s\n", occ,
               gb(timeit([&] { linear<4, 256><<<sms * occ, 256>>>((const float4*)A, N / 4, Y); })),
               gb(timeit_b2b([&] { linear<4, 256><<<sms * occ, 256>>>((const float4*)A, N / 4, Y); })));
    }
    for (int64_t chunk_kb : {16, 64, 256, 1024}) {
        int64_t c4 = chunk_kb * 1024 / 16;
        for (int occ : {4, 8}) {
            printf("chunked %4lld KB U4 NT256 occ%d: single %.0f  b2b %.0f GB/s\n", (long long)chunk_kb, occ,
                   gb(timeit([&] { chunked<4, 256><<<sms * occ, 256>>>((const float4*)A, N / 4, c4, Y); })),
                   gb(timeit_b2b([&] { chunked<4, 256><<<sms * occ, 256>>>((const float4*)A, N / 4, c4, Y); })));
        }
    }
    return 0;
}
