// bicgstab.cu -- BiCGSTAB on the adaptive MV, sm_100a.
//
// The paper's second case study (Sec. 5.2.2): BiCGSTAB has "11 linear
// steps"; written with CUBLAS each step is "several sub-steps" (Sgemv, Sdot,
// Sscal, Saxpy), which "leads to more memory accesses and kernel launch overhead",
// whereas "Adaptic merges all these sub-steps together and launches a single
// kernel for one step" (vertical integration, Sec. 4.3.1).  Here one iteration is
// five launches on one stream, no host round trip:
//   bicg_step1  steps 1-3   rho = (r^, r); beta; p = r + beta (p - omega v)
//   MV          step 4      v = A p            (adaptic_plan's selected kernel)
//   bicg_step2  steps 5-7   alpha = rho / (r^, v); s = r - alpha v; ||s||; early stop
//   MV          step 8      t = A s
//   bicg_step3  steps 9-11  omega = (t, s) / (t, t); x += alpha p + omega s;
//                           r = s - omega t; ||r||; stop test
// Every scalar lives in a device state block; the step kernels read it, so beta,
// alpha, omega never travel to the host.  After convergence (or breakdown) the step
// kernels return at once and x stays frozen; the MVs still run (their inputs are
// frozen too), so a batch of iterations can be enqueued blindly and checked every
// few iterations.  The step kernels are single 1024-thread CTAs: their vectors are
// n <= 64K floats (<= 1.5 MB for the six of them, L2-resident), so one SM streams
// them in a few microseconds while the two n x n MVs move 2*4n^2 bytes of HBM.
// fp32 throughout (the paper's Sgemv/Sdot); dots reduce per thread then by a
// fixed warp/CTA tree, so a run is deterministic.
#include "adaptic.h"
#include "common.cuh"

#include <algorithm>
#include <climits>
#include <cmath>
#include <cstring>
#include <new>

namespace adaptic {

struct BicgState {
    float rho_prev, rho, alpha, omega, bnorm, relres;
    int iters, done, breakdown, pad;
};

constexpr int BICG_NT = 1024;

// Block-wide sums of NV values per thread (fixed tree); result valid in every thread.
template <int NV>
__device__ __forceinline__ void block_sums(float (&v)[NV], float* red /* NV * 32 */) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
#pragma unroll
    for (int k = 0; k < NV; ++k) v[k] = group_sum<32>(v[k]);
    if (lane == 0) {
#pragma unroll
        for (int k = 0; k < NV; ++k) red[k * 32 + warp] = v[k];
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < NV; ++k) v[k] = group_sum<32>(red[k * 32 + lane]);   // 32 warps
    __syncthreads();
}

__global__ void __launch_bounds__(BICG_NT)
bicg_init(const float* __restrict__ b, float* __restrict__ x, float* __restrict__ r, float* __restrict__ rhat,
          float* __restrict__ p, float* __restrict__ v, BicgState* st, int64_t n)
{
    pdl_prologue();
    __shared__ float red[32];
    float acc[1] = {0.f};
    for (int64_t i = threadIdx.x; i < n; i += BICG_NT) {
        const float bi = b[i];
        x[i] = 0.f; r[i] = bi; rhat[i] = bi; p[i] = 0.f; v[i] = 0.f;
        acc[0] = fmaf(bi, bi, acc[0]);
    }
    block_sums<1>(acc, red);
    if (threadIdx.x == 0) {
        st->rho_prev = 1.f; st->rho = 1.f; st->alpha = 1.f; st->omega = 1.f;
        st->bnorm = sqrtf(acc[0]); st->relres = 1.f;
        st->iters = 0; st->done = acc[0] == 0.f ? 1 : 0; st->breakdown = 0; st->pad = 0;
    }
}

// steps 1-3
__global__ void __launch_bounds__(BICG_NT)
bicg_step1(const float* __restrict__ r, const float* __restrict__ rhat, float* __restrict__ p,
           const float* __restrict__ v, BicgState* st, int64_t n)
{
    pdl_prologue();
    __shared__ float red[32];
    if (st->done) return;
    float acc[1] = {0.f};
    for (int64_t i = threadIdx.x; i < n; i += BICG_NT) acc[0] = fmaf(rhat[i], r[i], acc[0]);
    block_sums<1>(acc, red);
    const float rho = acc[0];
    if (rho == 0.f) {                                   // breakdown: (r^, r) = 0
        if (threadIdx.x == 0) { st->done = 1; st->breakdown = 1; }
        return;
    }
    const float beta = (rho / st->rho_prev) * (st->alpha / st->omega);
    const float omega = st->omega;
    for (int64_t i = threadIdx.x; i < n; i += BICG_NT) p[i] = fmaf(beta, fmaf(-omega, v[i], p[i]), r[i]);
    if (threadIdx.x == 0) st->rho = rho;
}

// steps 5-7
__global__ void __launch_bounds__(BICG_NT)
bicg_step2(const float* __restrict__ r, const float* __restrict__ rhat, const float* __restrict__ p,
           const float* __restrict__ v, float* __restrict__ s, float* __restrict__ x, BicgState* st,
           int64_t n, float tol)
{
    pdl_prologue();
    __shared__ float red[32];
    if (st->done) return;
    float acc[1] = {0.f};
    for (int64_t i = threadIdx.x; i < n; i += BICG_NT) acc[0] = fmaf(rhat[i], v[i], acc[0]);
    block_sums<1>(acc, red);
    if (acc[0] == 0.f) {
        if (threadIdx.x == 0) { st->done = 1; st->breakdown = 1; }
        return;
    }
    const float alpha = st->rho / acc[0];
    float ss[1] = {0.f};
    for (int64_t i = threadIdx.x; i < n; i += BICG_NT) {
        const float si = fmaf(-alpha, v[i], r[i]);
        s[i] = si;
        ss[0] = fmaf(si, si, ss[0]);
    }
    block_sums<1>(ss, red);
    const float relres = sqrtf(ss[0]) / st->bnorm;
    const bool stop = relres < tol;
    if (stop)                                           // step 7: x = x + alpha p, done
        for (int64_t i = threadIdx.x; i < n; i += BICG_NT) x[i] = fmaf(alpha, p[i], x[i]);
    __syncthreads();
    if (threadIdx.x == 0) {
        st->alpha = alpha;
        if (stop) { st->relres = relres; st->iters += 1; st->done = 1; }
    }
}

// steps 9-11
__global__ void __launch_bounds__(BICG_NT)
bicg_step3(float* __restrict__ x, float* __restrict__ r, const float* __restrict__ p,
           const float* __restrict__ s, const float* __restrict__ t, BicgState* st, int64_t n, float tol)
{
    pdl_prologue();
    __shared__ float red[64];
    if (st->done) return;
    float acc[2] = {0.f, 0.f};                          // (t, s), (t, t)
    for (int64_t i = threadIdx.x; i < n; i += BICG_NT) {
        const float ti = t[i];
        acc[0] = fmaf(ti, s[i], acc[0]);
        acc[1] = fmaf(ti, ti, acc[1]);
    }
    block_sums<2>(acc, red);
    const float omega = acc[1] != 0.f ? acc[0] / acc[1] : 0.f;
    const float alpha = st->alpha;
    float rr[1] = {0.f};
    for (int64_t i = threadIdx.x; i < n; i += BICG_NT) {
        const float si = s[i];
        x[i] = fmaf(omega, si, fmaf(alpha, p[i], x[i]));
        const float ri = fmaf(-omega, t[i], si);
        r[i] = ri;
        rr[0] = fmaf(ri, ri, rr[0]);
    }
    block_sums<1>(rr, red);
    if (threadIdx.x == 0) {
        const float relres = sqrtf(rr[0]) / st->bnorm;
        st->omega = omega;
        st->rho_prev = st->rho;
        st->relres = relres;
        st->iters += 1;
        if (relres < tol) st->done = 1;
        if (omega == 0.f && !(relres < tol)) { st->done = 1; st->breakdown = 1; }
    }
}

}  // namespace adaptic

using namespace adaptic;

struct adaptic_bicgstab_s {
    int64_t n;
    adaptic_plan_t mv;          // v = A p and t = A s (the selector's plan for n x n)
    size_t mv_ws, vec_off, state_off, total;
    char* ws;
    size_t ws_cap;
};

namespace {

size_t align256(size_t v) { return (v + 255) / 256 * 256; }

adaptic_status launch1(void* fn, void** args, cudaStream_t stream) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(1);
    cfg.blockDim = dim3(BICG_NT);
    cfg.stream = stream;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    const cudaError_t e = cudaLaunchKernelExC(&cfg, fn, args);
    if (e != cudaSuccess) { (void)cudaGetLastError(); return ADAPTIC_ERR_CUDA; }
    return ADAPTIC_OK;
}

struct Vecs { float *r, *rhat, *p, *v, *s, *t; BicgState* st; };

Vecs vecs_of(adaptic_bicgstab_s* S) {
    float* base = reinterpret_cast<float*>(S->ws + S->vec_off);
    const size_t stride = align256(size_t(S->n) * 4) / 4;
    Vecs V;
    V.r = base; V.rhat = base + stride; V.p = base + 2 * stride; V.v = base + 3 * stride;
    V.s = base + 4 * stride; V.t = base + 5 * stride;
    V.st = reinterpret_cast<BicgState*>(S->ws + S->state_off);
    return V;
}

}  // namespace

extern "C" {

adaptic_status adaptic_bicgstab_create(int64_t n, adaptic_bicgstab_t* out) {
    if (!out) return ADAPTIC_ERR_INVALID_ARG;
    *out = nullptr;
    if (n < 1 || n > ADAPTIC_BICGSTAB_MAX_N) return n < 1 ? ADAPTIC_ERR_INVALID_ARG : ADAPTIC_ERR_UNSUPPORTED;
    adaptic_bicgstab_s* S = new (std::nothrow) adaptic_bicgstab_s();
    if (!S) return ADAPTIC_ERR_INVALID_ARG;
    S->n = n;
    adaptic_status st = adaptic_plan(ADAPTIC_OP_MV, n, n, ADAPTIC_F32, &S->mv);
    if (st != ADAPTIC_OK) { delete S; return st; }
    S->mv_ws = align256(adaptic_plan_workspace_bytes(S->mv));
    S->vec_off = S->mv_ws;
    S->state_off = S->vec_off + 6 * align256(size_t(n) * 4);
    S->total = S->state_off + align256(sizeof(BicgState));
    S->ws = nullptr; S->ws_cap = 0;
    *out = S;
    return ADAPTIC_OK;
}

size_t adaptic_bicgstab_workspace_bytes(adaptic_bicgstab_t S) { return S ? S->total : 0; }

adaptic_status adaptic_bicgstab_set_workspace(adaptic_bicgstab_t S, void* dev_ptr, size_t bytes) {
    if (!S || !dev_ptr) return ADAPTIC_ERR_INVALID_ARG;
    if ((reinterpret_cast<uintptr_t>(dev_ptr) & 255u) != 0) return ADAPTIC_ERR_MISALIGNED;
    if (bytes < S->total) return ADAPTIC_ERR_NO_WORKSPACE;
    const size_t mvb = adaptic_plan_workspace_bytes(S->mv);
    adaptic_status st = mvb ? adaptic_plan_set_workspace(S->mv, dev_ptr, mvb) : ADAPTIC_OK;
    if (st != ADAPTIC_OK) return st;
    S->ws = static_cast<char*>(dev_ptr);
    S->ws_cap = bytes;
    return ADAPTIC_OK;
}

adaptic_status adaptic_bicgstab_start(adaptic_bicgstab_t S, const void* b, void* x, void* stream) {
    if (!S || !b || !x) return ADAPTIC_ERR_INVALID_ARG;
    if (!S->ws) return ADAPTIC_ERR_NO_WORKSPACE;
    Vecs V = vecs_of(S);
    const float* bp = static_cast<const float*>(b);
    float* xp = static_cast<float*>(x);
    int64_t n = S->n;
    void* args[] = {&bp, &xp, &V.r, &V.rhat, &V.p, &V.v, &V.st, &n};
    return launch1(reinterpret_cast<void*>(&bicg_init), args, static_cast<cudaStream_t>(stream));
}

adaptic_status adaptic_bicgstab_iterate(adaptic_bicgstab_t S, const void* A, void* x, int32_t iters, float tol,
                                        void* stream_) {
    if (!S || !A || !x || iters < 0 || !(tol >= 0.f)) return ADAPTIC_ERR_INVALID_ARG;
    if (!S->ws) return ADAPTIC_ERR_NO_WORKSPACE;
    cudaStream_t stream = static_cast<cudaStream_t>(stream_);
    Vecs V = vecs_of(S);
    float* xp = static_cast<float*>(x);
    int64_t n = S->n;
    for (int it = 0; it < iters; ++it) {
        void* a1[] = {&V.r, &V.rhat, &V.p, &V.v, &V.st, &n};
        adaptic_status st = launch1(reinterpret_cast<void*>(&bicg_step1), a1, stream);
        if (st == ADAPTIC_OK) st = adaptic_run(S->mv, A, V.p, V.v, stream_);
        void* a2[] = {&V.r, &V.rhat, &V.p, &V.v, &V.s, &xp, &V.st, &n, &tol};
        if (st == ADAPTIC_OK) st = launch1(reinterpret_cast<void*>(&bicg_step2), a2, stream);
        if (st == ADAPTIC_OK) st = adaptic_run(S->mv, A, V.s, V.t, stream_);
        void* a3[] = {&xp, &V.r, &V.p, &V.s, &V.t, &V.st, &n, &tol};
        if (st == ADAPTIC_OK) st = launch1(reinterpret_cast<void*>(&bicg_step3), a3, stream);
        if (st != ADAPTIC_OK) return st;
    }
    return ADAPTIC_OK;
}

adaptic_status adaptic_bicgstab_state(adaptic_bicgstab_t S, int32_t* iters, float* relres, int32_t* done,
                                      void* stream) {
    if (!S) return ADAPTIC_ERR_INVALID_ARG;
    if (!S->ws) return ADAPTIC_ERR_NO_WORKSPACE;
    BicgState h;
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    cudaError_t e = cudaMemcpyAsync(&h, S->ws + S->state_off, sizeof(h), cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) { (void)cudaGetLastError(); return ADAPTIC_ERR_CUDA; }
    if (iters) *iters = h.iters;
    if (relres) *relres = h.relres;
    if (done) *done = h.done ? (h.breakdown ? 2 : 1) : 0;
    return ADAPTIC_OK;
}

adaptic_status adaptic_bicgstab_solve(adaptic_bicgstab_t S, const void* A, const void* b, void* x, int32_t max_iters,
                                      float tol, int32_t check_every, int32_t* iters_out, float* relres_out,
                                      void* stream) {
    if (!S || max_iters < 0) return ADAPTIC_ERR_INVALID_ARG;
    if (check_every < 1) check_every = 8;
    adaptic_status st = adaptic_bicgstab_start(S, b, x, stream);
    int32_t it = 0, done = 0;
    float rel = 1.f;
    for (int32_t k = 0; st == ADAPTIC_OK && k < max_iters && !done; k += check_every) {
        st = adaptic_bicgstab_iterate(S, A, x, std::min(check_every, max_iters - k), tol, stream);
        if (st == ADAPTIC_OK) st = adaptic_bicgstab_state(S, &it, &rel, &done, stream);
    }
    if (st == ADAPTIC_OK && max_iters == 0) st = adaptic_bicgstab_state(S, &it, &rel, &done, stream);
    if (iters_out) *iters_out = it;
    if (relres_out) *relres_out = rel;
    return st;
}

void adaptic_bicgstab_destroy(adaptic_bicgstab_t S) {
    if (!S) return;
    adaptic_plan_destroy(S->mv);
    delete S;
}

}  // extern "C"
