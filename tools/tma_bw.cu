// TMA 1-D bulk copy streaming throughput vs copy size / ring depth (1 CTA per SM).
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
__device__ __forceinline__ uint32_t su(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__global__ void __launch_bounds__(288, 1) k(const char* src, size_t per_cta, int csize, int stages, int stage_bytes, unsigned long long* sink, int rows, size_t rowpitch, int hint, int ncons) {
    extern __shared__ __align__(128) char sm[];
    __shared__ __align__(8) uint64_t full[16], empty[16];
    int tid = threadIdx.x;
    if (tid == 0) { for (int i = 0; i < stages; ++i) { asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(su(&full[i]))); asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(su(&empty[i])), "r"(ncons)); } asm volatile("fence.mbarrier_init.release.cluster;"); }
    __syncthreads();
    const char* base = src + (size_t)blockIdx.x * (rows == 1 ? per_cta : rows * rowpitch);
    size_t nst = per_cta / stage_bytes;
    if (tid >= 32 * ncons) {   // producer warp
        if (tid >= 32 * ncons + 32) return;
        int lane = tid & 31; int st = 0; uint32_t ph = 0;
        int ncopy = stage_bytes / csize;
        for (size_t i = 0; i < nst; ++i) {
            if (i >= (size_t)stages) { uint32_t p = ph ^ 1; asm volatile("{.reg .pred q; W: mbarrier.try_wait.parity.shared::cta.b64 q, [%0], %1; @!q bra W;}" :: "r"(su(&empty[st])), "r"(p)); }
            if (lane == 0) asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(su(&full[st])), "r"(stage_bytes));
            __syncwarp();
            for (int c = lane; c < ncopy; c += 32) {
                int r = c % rows; size_t off = (i * (stage_bytes / rows)) + (size_t)(c / rows) * csize;
                const char* g = base + r * rowpitch + off;
                if (hint) asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" :: "r"(su(sm + st * stage_bytes + c * csize)), "l"(g), "r"(csize), "r"(su(&full[st])), "l"(0x12F0000000000000ull) : "memory");
                else asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" :: "r"(su(sm + st * stage_bytes + c * csize)), "l"(g), "r"(csize), "r"(su(&full[st])) : "memory");
            }
            if (++st == stages) { st = 0; ph ^= 1; }
        }
    } else {
        int st = 0; uint32_t ph = 0; unsigned long long acc = 0;
        for (size_t i = 0; i < nst; ++i) {
            asm volatile("{.reg .pred q; W: mbarrier.try_wait.parity.shared::cta.b64 q, [%0], %1; @!q bra W;}" :: "r"(su(&full[st])), "r"(ph));
            acc += ((volatile int*)(sm + st * stage_bytes))[tid];
            __syncwarp();
            if ((tid & 31) == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" :: "r"(su(&empty[st])));
            if (++st == stages) { st = 0; ph ^= 1; }
        }
        if (acc == 12345) sink[0] = acc;
    }
}
int main() {
    size_t total = (size_t)1 << 32;  // 4 GiB
    char* src; cudaMalloc(&src, total); cudaMemset(src, 1, total);
    unsigned long long* sink; cudaMalloc(&sink, 8);
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 220 * 1024);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    for (int hint = 0; hint < 2; ++hint)
    for (int ncons : {1, 8})
    for (int stages : {3, 4, 6}) {
        int rows = 8; size_t pitch = 1 << 20; int csize = 4096, stage = 32768;
        size_t stream = (size_t(1) << 20) * rows;
        int nth = 32 * ncons + 32;
        k<<<sms, nth, stages * stage>>>(src, stream, csize, stages, stage, sink, rows, pitch, hint, ncons);
        cudaEventRecord(e0);
        for (int r = 0; r < 5; ++r) k<<<sms, nth, stages * stage>>>(src, stream, csize, stages, stage, sink, rows, pitch, hint, ncons);
        cudaEventRecord(e1); cudaEventSynchronize(e1);
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        printf("hint %d consumers %d stages %d : %.0f GB/s (%s)\n", hint, ncons, stages, 5.0 * stream * sms / (ms / 1e3) / 1e9, cudaGetErrorString(cudaGetLastError()));
    }
}
