// synth_gen.cu -- device-side copy of the shared input generator (synth/__init__.py).
//
// Not part of the product path and holds none of the method's arithmetic: it
// only maps (seed, logical index) to an input value, so full-size inputs
// (16-64 GiB) can be generated in HBM.  Written independently of the numpy
// version; tests/test_gpu_parity.py checks the two agree element by element.
//
//   h = splitmix64(seed ^ (i * 0x9E3779B97F4A7C15)),  i = r*C + c (logical index)
//   kinds: 0 uniform, 1 positive, 2 ones, 3 smallint, 4 smallint4, 5 identity,
//          6 perm, 7 diag, 8 rowscale, 9 diagdom   (see synth/__init__.py for the formulas)
#include <cstdint>
#include <type_traits>
#include <cuda_runtime.h>

namespace {

__device__ __forceinline__ uint64_t splitmix64(uint64_t z) {
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

__device__ __forceinline__ float f32_of(uint64_t h, int kind) {
    switch (kind) {
        case 1: return float(int64_t((h >> 40) & 0xFFFFFFull)) * 5.9604644775390625e-08f;         // 2^-24
        case 3: return float(int64_t((h >> 40) % 3ull) - 1);
        case 4: return float(int64_t((h >> 40) % 9ull) - 4);
        default: return float(int64_t((h >> 40) & 0xFFFFFFull) - 8388608) * 1.1920928955078125e-07f;  // 2^-23
    }
}
__device__ __forceinline__ int32_t i32_of(uint64_t h, int kind) {
    switch (kind) {
        case 1: return int32_t((h >> 56) & 0x7Full);
        case 3: return int32_t((h >> 40) % 3ull) - 1;
        case 4: return int32_t((h >> 40) % 9ull) - 4;
        default: return int32_t((h >> 56) & 0xFFull) - 128;
    }
}

// One element of the logical matrix a(r, c).
template <class T> __device__ __forceinline__ T elem(uint64_t seed, int kind, int64_t R, int64_t C, int64_t r, int64_t c);

template <> __device__ __forceinline__ float elem<float>(uint64_t seed, int kind, int64_t R, int64_t C, int64_t r, int64_t c) {
    if (kind == 2) return 1.f;
    if (kind == 5) return r == c ? 1.f : 0.f;
    if (kind == 6) return c == R - 1 - r ? 1.f : 0.f;
    const uint64_t i = uint64_t(r) * uint64_t(C) + uint64_t(c);
    float v = f32_of(splitmix64(seed ^ (i * 0x9E3779B97F4A7C15ull)), kind);
    if (kind == 7) return r == c ? v : 0.f;
    if (kind == 8) return v * ldexpf(1.f, int(r % 41) - 20);
    if (kind == 9) return r == c ? float(C) : v;
    return v;
}
template <> __device__ __forceinline__ int32_t elem<int32_t>(uint64_t seed, int kind, int64_t R, int64_t C, int64_t r, int64_t c) {
    if (kind == 2) return 1;
    if (kind == 5) return r == c ? 1 : 0;
    if (kind == 6) return c == R - 1 - r ? 1 : 0;
    const uint64_t i = uint64_t(r) * uint64_t(C) + uint64_t(c);
    int32_t v = i32_of(splitmix64(seed ^ (i * 0x9E3779B97F4A7C15ull)), kind);
    if (kind == 7) return r == c ? v : 0;
    if (kind == 9) return r == c ? int32_t(C) : v;
    return v;
}

template <class T>
__global__ void fill_matrix(T* out, int layout, int kind, uint64_t seed, int64_t R, int64_t C,
                            int64_t r0, int64_t r1, int64_t c0, int64_t c1) {
    const int64_t nr = r1 - r0, nc = c1 - c0, n = nr * nc;
    for (int64_t k = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; k < n; k += int64_t(gridDim.x) * blockDim.x) {
        int64_t r, c;
        if (layout == 0) { r = r0 + k / nc; c = c0 + k % nc; }      // out[r - r0][c - c0]
        else { c = c0 + k / nr; r = r0 + k % nr; }                  // out[c - c0][r - r0]
        out[k] = elem<T>(seed, kind, R, C, r, c);
    }
}

template <class T>
__global__ void fill_vector(T* out, int kind, uint64_t seed, int64_t start, int64_t n) {
    for (int64_t k = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; k < n; k += int64_t(gridDim.x) * blockDim.x) {
        const uint64_t i = uint64_t(start + k);
        if (kind == 2) { out[k] = T(1); continue; }
        const uint64_t h = splitmix64(seed ^ (i * 0x9E3779B97F4A7C15ull));
        if constexpr (std::is_same<T, float>::value) out[k] = f32_of(h, kind);
        else out[k] = i32_of(h, kind);
    }
}

}  // namespace

extern "C" {

// dtype 0 = fp32, 1 = int32; layout 0 = MV (row-major R x C block), 1 = TMV (C x R block).
int synth_fill_matrix(void* out, int dtype, int layout, int kind, uint64_t seed, int64_t R, int64_t C,
                      int64_t r0, int64_t r1, int64_t c0, int64_t c1, void* stream) {
    const int64_t n = (r1 - r0) * (c1 - c0);
    if (n <= 0) return 0;
    const int grid = int(n / 256 + 1 < 148 * 16 ? n / 256 + 1 : 148 * 16);
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    if (dtype == 0) fill_matrix<float><<<grid, 256, 0, s>>>(static_cast<float*>(out), layout, kind, seed, R, C, r0, r1, c0, c1);
    else fill_matrix<int32_t><<<grid, 256, 0, s>>>(static_cast<int32_t*>(out), layout, kind, seed, R, C, r0, r1, c0, c1);
    return int(cudaGetLastError());
}

int synth_fill_vector(void* out, int dtype, int kind, uint64_t seed, int64_t start, int64_t n, void* stream) {
    if (n <= 0) return 0;
    const int grid = int(n / 256 + 1 < 148 * 16 ? n / 256 + 1 : 148 * 16);
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    if (dtype == 0) fill_vector<float><<<grid, 256, 0, s>>>(static_cast<float*>(out), kind, seed, start, n);
    else fill_vector<int32_t><<<grid, 256, 0, s>>>(static_cast<int32_t*>(out), kind, seed, start, n);
    return int(cudaGetLastError());
}

}  // extern "C"
