/*
 * oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, single-threaded CPU statement of what the Adaptic hot path
 * computes.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library.  The product path
 * (paper_conf_pldi_samadihmlm12_b200/) never links, imports or calls it, and this
 * file shares no code, header or constant with the CUDA sources.
 *
 * What it follows (P:N = line N of the paper text, PAPER.md):
 *   - P:476 (Sec. 4.2.1 Stream Reduction): the reduction kernel "receives
 *     N_arrays different arrays with N_elements elements each as input, and
 *     produces one element per array as output".  Here N_arrays = R (rows, the
 *     number of outputs) and N_elements = C (cols, the reduction length).
 *   - P:472: the tree method needs only that the operation is "associative and
 *     commutative"; Fig. 8 starts from Result = 0 and folds each
 *     input with one operator, read as "+" (the glyph is lost in extraction,
 *     DESIGN.md reading R3).  Any summation order therefore yields a correct
 *     result, so the oracle is the plain definition, summed in increasing c.
 *   - P:1248 (Sec. 5.2.1 TMV): each kernel computes "the dot product of one row
 *     with the input vector".
 *   - P:614 (Sec. 5.1): Scalar Product "computes scalar products of pairs of
 *     vectors".
 *   - P:350-354 + Fig. 3 (Sec. 4.1.1 Memory Restructuring): thread t's k-th pop
 *     moves from word P*t + k to word T*k + t; this fixes the TMV layout as the
 *     transpose of the MV layout (reading R2).
 *
 * Arithmetic (readings R4, R5):
 *   - fp32 inputs are widened exactly to double; each product a*x of two fp32
 *     values is exact in double (24+24 <= 53 significand bits); the only
 *     rounding is the double-precision running sum.  S_r = sum |a*x| is returned
 *     beside y_r for the tolerance |y_gpu - y_r| <= 1e-4 * S_r.
 *   - int32 inputs are reduced modulo 2^32: products and sums in uint32_t, which
 *     wraps by definition in C; the result is reinterpreted as int32.
 *
 * Build: gcc -O2 -ffp-contract=off -fPIC -shared (no -ffast-math, no OpenMP).
 */
#include <stdint.h>
#include <stddef.h>
#include <math.h>

/* ---- MV: y_r = sum_{c=0}^{C-1} A[r*C + c] * x[c], A row-major R x C ----------- */
int oracle_mv_f64(const float* A, const float* x, int64_t R, int64_t C,
                  double* y, double* S)
{
    if (R < 0 || C < 0) return 1;
    for (int64_t r = 0; r < R; ++r) {
        double acc = 0.0, mag = 0.0;
        for (int64_t c = 0; c < C; ++c) {
            double p = (double)A[r * C + c] * (double)x[c];
            acc += p;
            mag += fabs(p);
        }
        y[r] = acc;
        if (S) S[r] = mag;
    }
    return 0;
}

/* ---- TMV: y_r = sum_c B[c*R + r] * x[c], B row-major C x R (B = A^T) ----------
 * Same per-row order c = 0, 1, 2, ... as oracle_mv_f64; the loop is c-outer so
 * that B is read in storage order.  Accumulators live in y and S. */
int oracle_tmv_f64(const float* B, const float* x, int64_t R, int64_t C,
                   double* y, double* S)
{
    if (R < 0 || C < 0) return 1;
    for (int64_t r = 0; r < R; ++r) { y[r] = 0.0; if (S) S[r] = 0.0; }
    for (int64_t c = 0; c < C; ++c) {
        double xc = (double)x[c];
        for (int64_t r = 0; r < R; ++r) {
            double p = (double)B[c * R + r] * xc;
            y[r] += p;
            if (S) S[r] += fabs(p);
        }
    }
    return 0;
}

/* ---- DOT: y_n = sum_e a[n*L + e] * b[n*L + e], N pairs of length L ------------- */
int oracle_dot_f64(const float* a, const float* b, int64_t N, int64_t L,
                   double* y, double* S)
{
    if (N < 0 || L < 0) return 1;
    for (int64_t n = 0; n < N; ++n) {
        double acc = 0.0, mag = 0.0;
        for (int64_t e = 0; e < L; ++e) {
            double p = (double)a[n * L + e] * (double)b[n * L + e];
            acc += p;
            mag += fabs(p);
        }
        y[n] = acc;
        if (S) S[n] = mag;
    }
    return 0;
}

/* ---- int32, modulo 2^32 --------------------------------------------------------- */
int oracle_mv_u32(const int32_t* A, const int32_t* x, int64_t R, int64_t C, int32_t* y)
{
    if (R < 0 || C < 0) return 1;
    for (int64_t r = 0; r < R; ++r) {
        uint32_t acc = 0u;
        for (int64_t c = 0; c < C; ++c)
            acc += (uint32_t)A[r * C + c] * (uint32_t)x[c];
        y[r] = (int32_t)acc;
    }
    return 0;
}

int oracle_tmv_u32(const int32_t* B, const int32_t* x, int64_t R, int64_t C, int32_t* y)
{
    if (R < 0 || C < 0) return 1;
    for (int64_t r = 0; r < R; ++r) {
        uint32_t acc = 0u;
        for (int64_t c = 0; c < C; ++c)
            acc += (uint32_t)B[c * R + r] * (uint32_t)x[c];
        y[r] = (int32_t)acc;
    }
    return 0;
}

int oracle_dot_u32(const int32_t* a, const int32_t* b, int64_t N, int64_t L, int32_t* y)
{
    if (N < 0 || L < 0) return 1;
    for (int64_t n = 0; n < N; ++n) {
        uint32_t acc = 0u;
        for (int64_t e = 0; e < L; ++e)
            acc += (uint32_t)a[n * L + e] * (uint32_t)b[n * L + e];
        y[n] = (int32_t)acc;
    }
    return 0;
}

/* ---- selected outputs only (for full-size configs, computed one by one) --------
 * layout 0 = MV (A row-major R x C), 1 = TMV (B row-major C x R).  rows[] lists the
 * outputs to compute; y/S receive them in the same order. */
int oracle_rows_f64(int layout, const float* M, const float* x, int64_t R, int64_t C,
                    const int64_t* rows, int64_t nrows, double* y, double* S)
{
    if (R < 0 || C < 0 || nrows < 0) return 1;
    for (int64_t i = 0; i < nrows; ++i) {
        int64_t r = rows[i];
        if (r < 0 || r >= R) return 2;
        double acc = 0.0, mag = 0.0;
        for (int64_t c = 0; c < C; ++c) {
            float a = layout == 0 ? M[r * C + c] : M[c * R + r];
            double p = (double)a * (double)x[c];
            acc += p;
            mag += fabs(p);
        }
        y[i] = acc;
        if (S) S[i] = mag;
    }
    return 0;
}

int oracle_rows_u32(int layout, const int32_t* M, const int32_t* x, int64_t R, int64_t C,
                    const int64_t* rows, int64_t nrows, int32_t* y)
{
    if (R < 0 || C < 0 || nrows < 0) return 1;
    for (int64_t i = 0; i < nrows; ++i) {
        int64_t r = rows[i];
        if (r < 0 || r >= R) return 2;
        uint32_t acc = 0u;
        for (int64_t c = 0; c < C; ++c) {
            int32_t a = layout == 0 ? M[r * C + c] : M[c * R + r];
            acc += (uint32_t)a * (uint32_t)x[c];
        }
        y[i] = (int32_t)acc;
    }
    return 0;
}

/* ---- Memory restructuring, Fig. 3 / P:350-354 ---------------------------------
 * T threads each pop P consecutive words: before restructuring thread t's k-th
 * pop reads word P*t + k; afterwards it reads word T*k + t.  out[T*k + t] =
 * in[P*t + k].  With T = R and P = C this maps the MV buffer to the TMV buffer. */
int oracle_restructure_f32(const float* in, int64_t T, int64_t P, float* out)
{
    if (T < 0 || P < 0) return 1;
    for (int64_t t = 0; t < T; ++t)
        for (int64_t k = 0; k < P; ++k)
            out[T * k + t] = in[P * t + k];
    return 0;
}

/* ---- BLAS-1 reductions ------------------------------------
 * The paper's Fig. 9 input-portability benchmarks include the CUBLAS routines
 * Isamax/Isamin, Snrm2 and Sasum, sped up by "actor segmentation and actor
 * integration" (Sec. 5.1) -- the same one-output-per-array stream
 * reduction as above with a different operator.  Definitions (BLAS):
 *   asum : y_n = sum_e |a[n,e]|
 *   nrm2 : y_n = sqrt(sum_e a[n,e]^2)        (squares of fp32 are exact in double)
 *   iamax: smallest 1-based e with |a[n,e]| = max_k |a[n,k]|   (0 when L == 0)
 *   iamin: smallest 1-based e with |a[n,e]| = min_k |a[n,k]|   (0 when L == 0)
 * N vectors of length L, row-major (rows = N outputs, cols = L). */
int oracle_asum_f64(const float* a, int64_t N, int64_t L, double* y)
{
    if (N < 0 || L < 0) return 1;
    for (int64_t n = 0; n < N; ++n) {
        double acc = 0.0;
        for (int64_t e = 0; e < L; ++e) acc += fabs((double)a[n * L + e]);
        y[n] = acc;
    }
    return 0;
}

int oracle_nrm2_f64(const float* a, int64_t N, int64_t L, double* y, double* ssq)
{
    if (N < 0 || L < 0) return 1;
    for (int64_t n = 0; n < N; ++n) {
        double acc = 0.0;
        for (int64_t e = 0; e < L; ++e) {
            double v = (double)a[n * L + e];
            acc += v * v;
        }
        if (ssq) ssq[n] = acc;
        y[n] = sqrt(acc);
    }
    return 0;
}

/* which = +1: iamax, -1: iamin.  |a| of an fp32 value is exact in fp32, so the
 * comparison (and so the index) is exact; ties keep the first index. */
int oracle_iamaxmin(const float* a, int64_t N, int64_t L, int which, int64_t* idx)
{
    if (N < 0 || L < 0 || (which != 1 && which != -1)) return 1;
    for (int64_t n = 0; n < N; ++n) {
        int64_t best = 0;
        float bv = 0.0f;
        for (int64_t e = 0; e < L; ++e) {
            float v = fabsf(a[n * L + e]);
            if (e == 0 || (which == 1 ? v > bv : v < bv)) { bv = v; best = e + 1; }
        }
        idx[n] = best;
    }
    return 0;
}

/* ---- five-point stencil (second item) -----------------------
 * The paper's neighbouring-access actor (Sec. 4.1.2, Fig. 4a): every
 * point reads its top, bottom, left and right neighbours and itself and pushes
 * func(Top, Bottom, Right, Left, Center); points on the edge are skipped ("if (not on
 * edge)").  func is not printed; reading R19: the weighted Jacobi form
 *   v[i][j] = c * u[i][j] + n * (u[i-1][j] + u[i+1][j] + u[i][j-1] + u[i][j+1])
 * for 1 <= i < H-1, 1 <= j < W-1, and v = u on the edge.  u, v are H x W row-major
 * fp32; the oracle evaluates in double (products of fp32 values are exact) and
 * returns S = |c u| + |n| (|T| + |B| + |L| + |R|) per point for the tolerance. */
int oracle_stencil5_f64(const float* u, int64_t H, int64_t W, double c, double n, double* v, double* S)
{
    if (H < 0 || W < 0) return 1;
    for (int64_t i = 0; i < H; ++i) {
        for (int64_t j = 0; j < W; ++j) {
            const int64_t k = i * W + j;
            if (i == 0 || j == 0 || i == H - 1 || j == W - 1) {
                v[k] = (double)u[k];
                if (S) S[k] = fabs((double)u[k]);
                continue;
            }
            const double t = u[k - W], b = u[k + W], l = u[k - 1], r = u[k + 1], ce = u[k];
            v[k] = c * ce + n * (t + b + l + r);
            if (S) S[k] = fabs(c * ce) + fabs(n) * (fabs(t) + fabs(b) + fabs(l) + fabs(r));
        }
    }
    return 0;
}
