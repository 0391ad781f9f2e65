/*
 * adaptic.h -- C ABI of the B200-native input-adaptive reduction library.
 *
 * What it computes (P:N = line N of the paper text, PAPER.md, Samadi et al.,
 * "Adaptive Input-aware Compilation for Graphics Engines", PLDI'12):
 *
 *   The hot path is the paper's stream-reduction actor (Sec. 4.2.1): a kernel
 *   that "receives N_arrays different arrays with N_elements elements each as
 *   input, and produces one element per array as output", evaluated by
 *   a tree over an associative and commutative operator -- here
 *   multiply-accumulate.  Three operations use it:
 *
 *     ADAPTIC_OP_MV   y[r] = sum_c A[r*C + c] * x[c]     A row-major R x C
 *                     (each output is "the dot product of one row with the
 *                     input vector"; reductions are contiguous)
 *     ADAPTIC_OP_TMV  y[r] = sum_c B[c*R + r] * x[c]     B row-major C x R, B = A^T
 *                     (the paper's memory-restructured layout, Fig. 3 /
 *                     thread t's k-th pop reads word T*k + t; outputs
 *                     are contiguous, reductions are strided).  TMV(B) == MV(B^T).
 *     ADAPTIC_OP_DOT  y[n] = sum_e a[n*L + e] * b[n*L + e]  (Scalar Product,
 *                     "scalar products of pairs of vectors"; Sdot is
 *                     N = 1).  rows = N, cols = L, x := b (N x L).
 *
 *   For every op, `rows` (R) is the number of outputs and `cols` (C) is the
 *   reduction length (reading R1).
 *
 *   BLAS-1 reductions on the same engine: the paper's Fig. 9
 *   input-portability benchmarks include the CUBLAS routines Sasum, Snrm2 and
 *   Isamax/Isamin (Sec. 5.1) -- the same one-output-per-array reduction
 *    with another associative/commutative operator.  For N
 *   vectors of length L (a row-major N x L; rows = N, cols = L; x unused):
 *     ADAPTIC_OP_ASUM   y[n] = sum_e |a[n*L + e]|                  (float y)
 *     ADAPTIC_OP_NRM2   y[n] = sqrt(sum_e a[n*L + e]^2)            (float y)
 *     ADAPTIC_OP_IAMAX  y[n] = smallest 1-based e with |a[n*L+e-1]| maximal
 *     ADAPTIC_OP_IAMIN  y[n] = smallest 1-based e with |a[n*L+e-1]| minimal
 *                       (int32 y; 0 when L == 0; BLAS NaN rule: a NaN never
 *                       replaces the running extreme, so only a leading NaN
 *                       yields 1.  L must be <= 2^31 - 1, else UNSUPPORTED.)
 *   Arithmetic: ASUM accumulates in fp32 like MV (same 1e-4 * sum|a| bound);
 *   NRM2 accumulates the exact fp64 squares in fp64 (no overflow / underflow for
 *   any finite fp32 input) and rounds sqrt once to fp32; IAMAX/IAMIN compare
 *   |a| exactly, so the index is exact.  dtype must be ADAPTIC_F32
 *   (else UNSUPPORTED).  Variants: MV_SUBWARP, MV_WPR, MV_CPR, MV_SPLIT
 *   (MV_TPR and the TMV family -> UNSUPPORTED).  Workspace (MV_SPLIT): 8-byte
 *   partials per (row, split) plus one counter per row.
 *   ADAPTIC_OP_B1ALL is the paper's horizontal actor integration ("a
 *   program that needs maximum and summation of all elements in an array ...
 *   Adaptic launches one kernel to compute both"): the four reductions above from
 *   one read of a, written as four N-vectors back to back in y (16*N bytes: asum,
 *   nrm2 as float, then iamax, iamin as int32); same arithmetic and results as the
 *   four separate ops; workspace partials are 32 bytes.
 *
 * The input-adaptive part (Fig. 2): adaptic_plan() is the paper's
 * "runtime kernel management" -- on the CPU, from the actual input dimensions,
 * it selects one of several hand-written kernels and fixes its launch
 * parameters (blocks, threads, shared memory).  The selection comes from
 * a threshold table fitted on B200 sweeps (not from the paper, whose break-even
 * points were for a Tesla C2050).  The variants map to the paper's five TMV
 * kernels:
 *
 *     MV_TPR      K5  thread per row; rows staged in shared memory by the TMA
 *                     bulk-copy engine (the paper's shared-memory alternative to
 *                     restructuring)
 *     MV_SUBWARP  K4  g lanes per row (g = 1..16), shuffle reduction
 *     MV_WPR      K3  warp per row, several rows per CTA (horizontal thread
 *                     integration)
 *     MV_CPR      K2  CTA per row, single-kernel reduction (Fig. 7b)
 *     MV_SPLIT    K1  several CTAs per row + merge (two-phase reduction, P:480,
 *                     Fig. 7c); the merge is done in the same kernel by the last
 *                     CTA to finish a row (atomic ticket), in fixed order
 *     TMV_COL     K5 on the restructured layout: thread per 4 outputs, loop over c
 *     TMV_SPLITK  2-D tiles of outputs x c-ranges, CTA combine + ticket merge
 *     TMV_REGTILE TMV_SPLITK whose tile holds every output (R <= 1024)
 *   DOT uses the MV variants with a per-row second operand.
 *
 * Arithmetic (readings R4, R5):
 *   ADAPTIC_F32: fp32 inputs, fp32 accumulation, round-to-nearest-even, FMA
 *     contraction allowed, no FTZ / fast-math.  Summation order is a tree
 *     whose serial chain per accumulator is <= 1024 terms, so every output is
 *     within 1e-4 * sum_c |a(r,c) x_c| of the exact value.  Different variants
 *     may return different roundings; a given plan is deterministic (it does not
 *     depend on CTA arrival order).
 *   ADAPTIC_I32: int32 inputs; products and sums modulo 2^32 (two's
 *     complement wrap).  Bit-exact for every variant.
 *   alpha = 1, beta = 0: y is fully overwritten; A and x are never written.
 *
 * Conventions:
 *   - Sizes are int64_t.  rows < 0 or cols < 0, or rows*cols*4 overflowing
 *     size_t -> ADAPTIC_ERR_INVALID_ARG.  rows == 0: success, nothing launched.
 *     cols == 0: y is zero-filled (one memset on the stream).
 *   - Pointers passed to adaptic_run are DEVICE pointers owned by the caller
 *     (PyTorch allocates them); they must stay valid until the stream work
 *     completes.  The library never allocates device memory.
 *   - Pointers must be element (4-byte) aligned, else ADAPTIC_ERR_MISALIGNED.
 *     16-byte aligned A/x/y with a multiple-of-4 contiguous extent use 128-bit
 *     loads; anything else runs the same variant's scalar-load instance
 *     (correct, slower).
 *   - y must not overlap A or x (byte ranges), else ADAPTIC_ERR_ALIAS.
 *   - Variants that merge across CTAs (MV_SPLIT, TMV_SPLITK, TMV_REGTILE with
 *     splits > 1) need a workspace of adaptic_plan_workspace_bytes() bytes,
 *     device memory, ZERO-FILLED when attached with adaptic_plan_set_workspace;
 *     every run leaves it zero-filled again.  Running such a plan without one
 *     returns ADAPTIC_ERR_NO_WORKSPACE.  One plan with a workspace must not run
 *     on two streams concurrently.
 *   - adaptic_run only enqueues work on `stream` (cudaStream_t; NULL = legacy
 *     default stream) and returns; launch errors are reported as
 *     ADAPTIC_ERR_CUDA with the cudaError_t available from
 *     adaptic_last_cuda_error() (thread-local).  Sticky CUDA errors are not
 *     cleared.  No entry point aborts.
 *   - Plans are immutable after creation except for the attached workspace;
 *     adaptic_plan / adaptic_plan_forced are thread-safe.  A plan is computed
 *     for the SM count of the device current at plan time (148 on B200; 148
 *     is assumed if no device is present, so planning works on a CPU host).
 */
#ifndef ADAPTIC_H_
#define ADAPTIC_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define ADAPTIC_ABI_VERSION 6

typedef enum {
    ADAPTIC_OK = 0,
    ADAPTIC_ERR_INVALID_ARG = 1,   /* bad op/dtype/variant/size, NULL plan or pointer  */
    ADAPTIC_ERR_UNSUPPORTED = 2,   /* forced variant cannot run this op / shape        */
    ADAPTIC_ERR_MISALIGNED = 3,    /* a pointer is not 4-byte aligned                  */
    ADAPTIC_ERR_ALIAS = 4,         /* y overlaps A or x                                */
    ADAPTIC_ERR_NO_WORKSPACE = 5,  /* plan needs a workspace and has none / too small  */
    ADAPTIC_ERR_CUDA = 6           /* a CUDA runtime call failed; see last_cuda_error  */
} adaptic_status;

typedef enum {
    ADAPTIC_OP_MV = 0,    /* y[R] = A x,    A row-major R x C                       */
    ADAPTIC_OP_TMV = 1,   /* y[R] = B^T x,  B row-major C x R                       */
    ADAPTIC_OP_DOT = 2,   /* y[N] = <a_n, b_n>, a and b row-major N x L; x := b     */
    /* BLAS-1 reductions of N vectors a_n of length L (a row-major N x L, rows = N,
     * cols = L; x is unused and may be NULL).  fp32 only (ADAPTIC_F32).        */
    ADAPTIC_OP_ASUM = 3,  /* float y[N] = sum_e |a_n[e]|                            */
    ADAPTIC_OP_NRM2 = 4,  /* float y[N] = sqrt(sum_e a_n[e]^2)                      */
    ADAPTIC_OP_IAMAX = 5, /* int32 y[N] = smallest 1-based e maximising |a_n[e]|    */
    ADAPTIC_OP_IAMIN = 6, /* int32 y[N] = smallest 1-based e minimising |a_n[e]|    */
    ADAPTIC_OP_B1ALL = 7, /* all four in ONE pass over a (horizontal actor integration,
                           * P:600): y = [asum N floats | nrm2 N floats | iamax N int32 |
                           * iamin N int32], 16*N bytes                               */
    /* Five-point stencil (the paper's neighbouring-access actor, Sec. 4.1.2, Fig. 4a):
     * A = u (rows = H, cols = W, fp32 row-major), x = {c, n} (2 device floats),
     * y = v (H x W): v = c u + n (T + B + L + R) inside, v = u on the edge.        */
    ADAPTIC_OP_STENCIL5 = 8
} adaptic_op;

typedef enum {
    ADAPTIC_F32 = 0,      /* fp32 in / fp32 accumulate                              */
    ADAPTIC_I32 = 1       /* int32, arithmetic modulo 2^32                          */
} adaptic_dtype;

typedef enum {
    ADAPTIC_V_AUTO = 0,
    ADAPTIC_V_MV_TPR = 1,
    ADAPTIC_V_MV_SUBWARP = 2,
    ADAPTIC_V_MV_WPR = 3,
    ADAPTIC_V_MV_CPR = 4,
    ADAPTIC_V_MV_SPLIT = 5,
    ADAPTIC_V_TMV_COL = 6,
    ADAPTIC_V_TMV_SPLITK = 7,
    ADAPTIC_V_TMV_REGTILE = 8,
    ADAPTIC_V_ST_DIRECT = 9,   /* stencil: no shared memory, neighbours from L1/L2          */
    ADAPTIC_V_ST_TILE = 10,    /* stencil: TMA-staged super tiles, double-buffered */
    ADAPTIC_V_COUNT = 11
} adaptic_variant;

/* Optional parameters for adaptic_plan_forced: an array of ADAPTIC_NPARAMS
 * int32 values (ADAPTIC_NPARAMS of them); a value <= 0 means "choose automatically".
 *   [ADAPTIC_P_LANES]  MV_SUBWARP: lanes per row g in {1,2,4,8,16};
 *                      MV_CPR / MV_SPLIT: threads per CTA in {256, 1024};
 *                      TMV_*: float4 lanes along the outputs per CTA tile,
 *                      a power of two in [1, 256].
 *   [ADAPTIC_P_SPLITS] MV_SPLIT / TMV_SPLITK / TMV_REGTILE: CTAs per
 *                      reduction (split count S >= 1).
 *   [ADAPTIC_P_CTAS_PER_SM] target resident CTAs per SM used to size grids.
 *   [ADAPTIC_P_UNROLL] independent 128-bit loads per thread per step {1,2,4,8}
 *                      (MV_TPR: pipeline stages 2..8).
 *   [ADAPTIC_P_XSMEM]  MV_SUBWARP / MV_WPR / MV_CPR: 1 = read x through the
 *                      read-only cache path, 2 = stage x in shared memory once per
 *                      CTA with a TMA bulk copy (needs cols*4 <= 200 KB).
 *                      MV_CPR / MV_SPLIT, fp32, cols % 4 == 0: 3 = the x-tile
 *                      stream-K kernel (column chunks of [ADAPTIC_P_LANES] values,
 *                      x chunks TMA-staged and double-buffered, (chunk, row) units
 *                      split evenly over the CTAs, chunk partials merged in order
 *                      per block of [ADAPTIC_P_ROWS] rows); 4-byte-aligned pointers
 *                      then run the CTA-per-row kernel.  Multi-vector TMV: 3 = B
 *                      rows staged by TMA, 1 = register-fed tiles.
 *                      MV_SUBWARP / MV_WPR (MV and DOT, fp32 / int32, cols <= 32 *
 *                      lanes): 4 = row tiles -- [ADAPTIC_P_ROWS] consecutive rows
 *                      (0: ~24 KB; -n: ~n KB) bulk-copied (TMA) as one 16-byte-
 *                      aligned block into a ring of [ADAPTIC_P_UNROLL] stages, each
 *                      row reduced by [ADAPTIC_P_LANES] lanes with x held in
 *                      registers ([ADAPTIC_P_BLOCK] 256 or 512 threads).  A, and
 *                      DOT's b, must be 16-byte aligned for it; other pointers run
 *                      the variant's direct kernel.  TMV_REGTILE (rows <= 4096):
 *                      4 = tiles of [ADAPTIC_P_ROWS] rows of B (a multiple of 4;
 *                      0 / -n as above) and their x values staged by TMA, thread
 *                      (r, slice) accumulating output r over its rows of every
 *                      tile, [ADAPTIC_P_BLOCK] 256 / 512 / 1024 threads with 1, 2
 *                      or 4 outputs each (rows <= 4 x threads, 4 needs >= 512);
 *                      16-byte-aligned B and x, else the direct kernel.  A tile
 *                      height is capped so that two ring stages fit.
 *                      MV (not DOT) with cols % 4 != 0, MV_SUBWARP / MV_WPR /
 *                      MV_CPR / MV_SPLIT: 5 = x copied first (same stream, same
 *                      call) into four shifted 16-byte-aligned copies in the
 *                      workspace, so every row reads x with 128-bit loads.
 *                      Further forced modes (round 2; the fitted table may select
 *                      them, DESIGN.md section 4 describes each):
 *                      7 = TMV_SPLITK / TMV_COL rows off the 16-byte grid at a constant
 *                      word shift per c-lane; 9 = MV_CPR / MV_SPLIT misaligned rows with
 *                      x read as two aligned 128-bit loads and a funnel (16-byte-aligned
 *                      x, else the direct kernel); 10 = TMV sliding-window kernel (rows
 *                      off the grid, one aligned load per row and thread); 11 = MV_CPR
 *                      long rows (cols <= 36 x threads) on staged row tiles reduced by
 *                      the whole CTA; 12 = TMV_REGTILE / TMV_SPLITK rows off the grid on
 *                      groups of four rows (4 <= rows <= 2560, [ADAPTIC_P_ROWS] slots per
 *                      thread, [ADAPTIC_P_ORDER] 2 = interleaved CTA ranges); 13 = MV_CPR /
 *                      MV_SPLIT rows of any length and alignment on staged COLUMN CHUNKS
 *                      ([ADAPTIC_P_LANES] x values per thread in {8, 16, 36},
 *                      [ADAPTIC_P_BLOCK] 256 | 512 consumer threads plus one producer
 *                      warp, [ADAPTIC_P_ROWS] row segments per tile <= 4).  Modes 11-13
 *                      need a 16-byte-aligned matrix base; other pointers run the
 *                      variant's direct kernel (same results, slower).
 *   [ADAPTIC_P_BLOCK]  TMV_*: threads per CTA, 256 or 1024 (unroll <= 4 at 1024).
 *   [ADAPTIC_P_ROWS]   MV_CPR / MV_SPLIT: rows per CTA step sharing each x load,
 *                      (rows, unroll) in {(1,2),(1,4),(1,8),(2,2),(2,4),(4,2)}.
 *   [ADAPTIC_P_ORDER]  MV_SPLIT: 1 = each split reads one contiguous chunk of
 *                      the row, 2 = the splits interleave in steps of
 *                      threads*unroll vectors (default when splits > 1).
 *   [ADAPTIC_P_PIPE]   MV_CPR / MV_SPLIT with 256 threads: 1 = single-buffered
 *                      loads (default), 2 = register double-buffered main loop.
 *   ST_DIRECT: [ADAPTIC_P_ORDER] 1 = row-major grid-stride sweep, 2 = L2 strips
 *                      (default for rows >= 2 MB), 3 = register sliding window down
 *                      float4 columns, [ADAPTIC_P_ROWS] rows per tile (default 64).
 *   ST_TILE: [ADAPTIC_P_ROWS] super-tile height TH in {4, 8, 16, 32}, [ADAPTIC_P_LANES]
 *                      width TW in {128, 256, 512} (default: the paper's reuse metric
 *                      sum(accesses)/halo, among tilings with enough blocks). */
#define ADAPTIC_P_LANES 0
#define ADAPTIC_P_SPLITS 1
#define ADAPTIC_P_CTAS_PER_SM 2
#define ADAPTIC_P_UNROLL 3
#define ADAPTIC_P_XSMEM 4
#define ADAPTIC_P_BLOCK 5
#define ADAPTIC_P_ROWS 6
#define ADAPTIC_P_ORDER 7
#define ADAPTIC_P_PIPE 8
#define ADAPTIC_NPARAMS 9

typedef struct adaptic_plan_s* adaptic_plan_t;   /* opaque; owned by the caller */

/* Selector (host only, O(1), no device work): picks the variant and its launch
 * parameters for (op, rows, cols, dtype) from the fitted threshold table (P:230-236:
 * the runtime kernel management unit picks the kernel and its launch shape from the
 * actual input).  The table's nearest-cell answer is memoised per (op, dtype, load
 * class, floor(log2 R), floor(log2 C)) cell and the derived plan per (op, dtype, R, C,
 * device), so a repeated shape costs one hash lookup and a struct copy
 * (tools/plan_latency.c measures it).  Thread-safe.  *out receives a new plan (free
 * with adaptic_plan_destroy). */
adaptic_status adaptic_plan(adaptic_op op, int64_t rows, int64_t cols, adaptic_dtype dtype,
                            adaptic_plan_t* out);

/* Same, with the variant fixed by the caller (fixed-variant sweeps and tests).
 * params: NULL or ADAPTIC_NPARAMS values as above.  Returns
 * ADAPTIC_ERR_UNSUPPORTED if the variant does not implement `op`. */
adaptic_status adaptic_plan_forced(adaptic_op op, int64_t rows, int64_t cols,
                                   adaptic_dtype dtype, adaptic_variant variant,
                                   const int32_t* params, adaptic_plan_t* out);

/* Multi-vector form: Y = A [x_0 ... x_{K-1}] (op = ADAPTIC_OP_MV) or
 * Y = B^T [x_0 ... x_{K-1}] (op = ADAPTIC_OP_TMV) with K = nvec vectors sharing ONE
 * pass over the matrix -- the paper's horizontal actor integration (actors
 * "working on the same data" run as one kernel, so "off-chip memory accesses and
 * synchronizations only happen once").  nvec in {1, 2, 4, 8} (1 = adaptic_plan /
 * adaptic_plan_forced; other counts -> UNSUPPORTED: split them into these sizes);
 * fp32 only.  adaptic_run then takes x = X, a K x C row-major array (vector j at
 * X + j*C), and y = Y, a K x R row-major array (Y + j*R = A x_j); results equal K
 * separate calls up to rounding (same 1e-4 bound; one accumulator per vector folded
 * every FOLD/U steps).  Variants: MV_SUBWARP / MV_WPR (rows of at most G*U loads,
 * x held in registers), MV_CPR / MV_SPLIT (8/K rows per CTA share each x load),
 * TMV_COL / TMV_SPLITK / TMV_REGTILE; variant = ADAPTIC_V_AUTO selects (params
 * ignored).  A 128-bit-shape plan run on pointers that are 4-byte but not 16-byte
 * aligned runs a fallback planned with it (MV_CPR / MV_SPLIT or register-fed TMV_SPLITK
 * on 4-byte loads: correct, slower; its workspace is included in
 * adaptic_plan_workspace_bytes); only pointers that are not 4-byte aligned return
 * ADAPTIC_ERR_MISALIGNED. */
adaptic_status adaptic_plan_multi(adaptic_op op, int64_t rows, int64_t cols, int32_t nvec,
                                  adaptic_dtype dtype, adaptic_variant variant,
                                  const int32_t* params, adaptic_plan_t* out);

/* What the plan will run. */
adaptic_variant adaptic_plan_variant(adaptic_plan_t plan);

/* Plan details as a NUL-terminated JSON object (variant, grid, block, lanes,
 * splits, unroll, chain, workspace bytes ...).  Writes at most `cap` bytes;
 * returns the full length needed (excluding the NUL), or -1 on a NULL plan. */
int adaptic_plan_describe(adaptic_plan_t plan, char* buf, size_t cap);

/* Device workspace the plan needs (0 for single-phase variants). */
size_t adaptic_plan_workspace_bytes(adaptic_plan_t plan);

/* Attach a caller-owned, zero-filled device buffer of >= workspace_bytes bytes
 * (NULL with bytes = 0 detaches).  ADAPTIC_ERR_NO_WORKSPACE if too small. */
adaptic_status adaptic_plan_set_workspace(adaptic_plan_t plan, void* dev_ptr, size_t bytes);

/* Enqueue y = op(A, x) on `stream` (a cudaStream_t passed as void*).
 * A, x, y: device pointers (see conventions above).  Asynchronous. */
adaptic_status adaptic_run(adaptic_plan_t plan, const void* A, const void* x, void* y,
                           void* stream);

/* Batched form: n independent problems (plans[i] on A[i], x[i] -> y[i], device
 * pointers as for adaptic_run) issued round-robin on up to `streams` (1..8) CUDA
 * streams forked from `stream` and joined back to it: when the call returns, all work
 * is enqueued and `stream` is ordered after every problem.  Independent reductions on
 * one stream serialise each kernel's ramp-up and tail; on concurrent streams the next
 * problem's loads overlap the previous one's drain (measured: +13.6 % on the 42-problem
 * 256 MiB sweep at streams = 2, profiles/r1_bench2_streams2.json).  Problems must not
 * write what another problem of the batch reads.  Repeated entries of a plan with a
 * workspace are kept on one stream (a workspace serialises its runs).  All problems are
 * validated before any is issued (all-or-nothing; statuses as adaptic_run).  The side
 * streams and events are the library's, per host thread and device, created on first use. */
adaptic_status adaptic_run_batch(int32_t n, const adaptic_plan_t* plans, const void* const* A,
                                 const void* const* x, void* const* y, int32_t streams, void* stream);

/* End-to-end form with HOST buffers: enqueue on `stream` the host->device copy
 * of A and x into the caller's device buffers dA, dx (sizes as for
 * adaptic_run), the kernel into dy, and the device->host copy of dy into y_host,
 * in that order on the one stream (x, then A as ONE copy, then the kernel: the
 * transfer is PCIe-bound, ~55 GB/s against the kernel's ~7 TB/s, so a row-block
 * pipeline would hide at most ~1 % of the call; callers overlap problems instead by
 * issuing them on several streams).  Host buffers should be page-locked for the
 * copies to be asynchronous.  Sizes are the plan's (R, C, nvec): the caller guarantees
 * A_host/dA hold R*C elements, x_host/dx C*nvec (DOT: R*C), y_host/dy R*nvec (B1ALL:
 * 4*R; STENCIL5: R*C) -- the Python binding checks them.  Returns after enqueueing;
 * the caller synchronises the stream before reading y_host. */
adaptic_status adaptic_run_host(adaptic_plan_t plan, const void* A_host, const void* x_host,
                                void* y_host, void* dA, void* dx, void* dy, void* stream);

void adaptic_plan_destroy(adaptic_plan_t plan);

/* ---------------------------------------------------------------------------------
 * BiCGSTAB on the adaptive MV (the paper's Sec. 5.2.2 case study,
 * P:1252-1304).  Solves A x = b for a dense, row-major n x n fp32 A (nonsymmetric),
 * x0 = 0, shadow residual r^ = b, the textbook unpreconditioned iteration (DESIGN.md
 * lists its 11 steps).  The paper's point is vertical integration: the sub-steps that
 * CUBLAS needs separate Sdot/Sscal/Saxpy calls for are merged into one kernel per step
 * ("Adaptic merges all these sub-steps together and launches a single kernel for one
 * step").  One iteration = 5 launches on `stream` (3 fused step kernels + 2 MVs
 * from adaptic_plan(MV, n, n)); every scalar stays on the device.
 *
 * Ownership: the solver object is the library's (free with adaptic_bicgstab_destroy);
 * it needs a caller-owned device workspace of adaptic_bicgstab_workspace_bytes() bytes,
 * 256-byte aligned and ZERO-FILLED when attached (it holds the MV plan's workspace,
 * six n-vectors and the scalar state).  A, b, x are caller-owned device pointers,
 * 16-byte aligned for the 128-bit MV path (else the scalar kernels run).
 *   create   : 1 <= n <= ADAPTIC_BICGSTAB_MAX_N, else INVALID_ARG / UNSUPPORTED.
 *   start    : enqueue x = 0, r = r^ = b, p = v = 0 and the state (||b||, ...).
 *   iterate  : enqueue `iters` iterations; after convergence (||r|| / ||b|| < tol, or
 *              ||s|| / ||b|| < tol at step 7) or a breakdown ((r^, r) = 0, (r^, v) = 0,
 *              omega = 0) the step kernels leave x untouched, so batches can be
 *              enqueued without host checks.
 *   state    : synchronises `stream` and reads back iterations done, the recurrence
 *              residual ||r|| / ||b||, and done (0 running, 1 converged, 2 breakdown).
 *   solve    : start + iterate in batches of check_every (<= 0: 8) + state, until done
 *              or max_iters; blocking.  Outputs may be NULL. */
#define ADAPTIC_BICGSTAB_MAX_N 65536
typedef struct adaptic_bicgstab_s* adaptic_bicgstab_t;
adaptic_status adaptic_bicgstab_create(int64_t n, adaptic_bicgstab_t* out);
size_t adaptic_bicgstab_workspace_bytes(adaptic_bicgstab_t solver);
adaptic_status adaptic_bicgstab_set_workspace(adaptic_bicgstab_t solver, void* dev_ptr, size_t bytes);
adaptic_status adaptic_bicgstab_start(adaptic_bicgstab_t solver, const void* b, void* x, void* stream);
adaptic_status adaptic_bicgstab_iterate(adaptic_bicgstab_t solver, const void* A, void* x, int32_t iters,
                                        float tol, void* stream);
adaptic_status adaptic_bicgstab_state(adaptic_bicgstab_t solver, int32_t* iters, float* relres,
                                      int32_t* done, void* stream);
adaptic_status adaptic_bicgstab_solve(adaptic_bicgstab_t solver, const void* A, const void* b, void* x,
                                      int32_t max_iters, float tol, int32_t check_every,
                                      int32_t* iters_out, float* relres_out, void* stream);
void adaptic_bicgstab_destroy(adaptic_bicgstab_t solver);

const char* adaptic_status_string(adaptic_status status);
const char* adaptic_variant_name(adaptic_variant variant);

/* cudaError_t of the last failing CUDA call made by this thread (0 if none). */
int adaptic_last_cuda_error(void);

/* ADAPTIC_ABI_VERSION of the loaded library. */
int adaptic_abi_version(void);

#ifdef __cplusplus
}
#endif

#endif /* ADAPTIC_H_ */
