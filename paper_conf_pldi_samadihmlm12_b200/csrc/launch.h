// launch.h -- internal interface between the planner (adaptic.cu) and the
// kernel translation units.  Not part of the public ABI (include/adaptic.h).
#pragma once

#include <cstddef>
#include <cstdint>
#include <cuda_runtime.h>

namespace adaptic {

// Iterations of a thread's load loop accumulated before folding into a
// second-level accumulator: keeps every serial chain short even for forced
// off-regime variants.
constexpr int FOLD = 512;

enum Dtype { DT_F32 = 0, DT_I32 = 1 };

constexpr int GROUP_NT = 256;   // threads per CTA, mv_group_kernel
constexpr int TMV_NT = 256;     // default threads per CTA, tmv_kernel (256 or 1024)

// Kernel instance lookup: a __global__ function pointer for cudaLaunchKernel /
// cudaOccupancyMaxActiveBlocksPerMultiprocessor, or nullptr when the instance
// is not compiled.  Kernel signatures:
//   group: (const T* A, const T* X, T* y, int64_t R, int64_t C)
//   cta  : (const T* A, const T* X, T* y, int64_t R, int64_t C, int S, int ilv, T* part, unsigned* cnt)
//          (RB rows per CTA step; (RB, U) in {(1,2),(1,4),(1,8),(2,2),(2,4),(4,2)})
//   tmv  : (const T* B, const T* X, T* y, int64_t R, int64_t C, int S, T* part, unsigned* cnt)
//   tpr  : (const T* A, const T* X, T* y, int64_t R, int64_t C, int stages)   [dynamic smem]
// x operand modes of the MV-family kernels (mv_kernels.cuh): 0 read-only path,
// 1 staged in shared memory by TMA (dynamic smem = C*4 bytes), 2 per-row (DOT)
void* group_fn_f32(int G, int U, bool vec, int xmode);
void* group_fn_i32(int G, int U, bool vec, int xmode);
void* tmv_fn_f32(int LR, int U, bool vec, int NT);
void* tmv_fn_i32(int LR, int U, bool vec, int NT);
void* cta_fn(int dtype, int NT, int RB, int U, bool vec, int xmode, bool pipe);
void* tpr_fn(int dtype, int NT, bool perrowx, bool scal = false);   // scal: C % 4 != 0 rows

// Misaligned-row MV/DOT (mv_mis_kernels.cuh; C % 4 != 0, 128-bit body + scalar head/tail):
//   group: (const T* A, const T* X, T* y, int64_t R, int64_t C), RB = max(1, 4/U)
//   cta  : (const T* A, const T* X, T* y, int64_t R, int64_t C, int S, int ilv, T* part, unsigned* cnt)
void* mis_group_fn_f32(int G, int U, int xmode);
void* mis_group_fn_i32(int G, int U, int xmode);
void* mis_cta_fn_f32(int NT, int U, int xmode);
void* mis_cta_fn_i32(int NT, int U, int xmode);
// x_shift_kernel (xmode 3 = XM_SHIFT): (const T* X, T* out, int64_t C), 256 threads; out holds
// four copies of pitch round_up(C, 4), copy h = x shifted left by h elements
void* mis_shift_fn_f32();
void* mis_shift_fn_i32();
// shifted-x CTA kernel, RB rows of one residue class (r mod 4) per step sharing x: the
// mis_cta arguments; NT = 256, U in {2, 4}, RB in {2, 4} (MV_CPR / MV_SPLIT, XSMEM 5, ROWS RB)
void* mis_cta_rb_fn_f32(int NT, int U, int RB);
void* mis_cta_rb_fn_i32(int NT, int U, int RB);
// x as two aligned 128-bit loads + a compile-time funnel per row head (mv_cta_mis_fx_kernel):
// the mis_cta arguments; NT = 256, U in {2, 4, 8}; needs a 16-byte-aligned x (XSMEM 9)
void* mis_cta_fx_fn_f32(int NT, int U);
void* mis_cta_fx_fn_i32(int NT, int U);
constexpr int XM_FX_MODE = 9;
constexpr int XM_SHIFT_MODE = 3;
// Misaligned-row TMV (tmv_mis_kernel.cuh; R % 4 != 0, two aligned loads + funnel shift), NT = 256:
//   (const T* B, const T* X, T* y, int64_t R, int64_t C, int S, T* part, unsigned* cnt)
void* tmv_mis_fn_f32(int LR, int U);
void* tmv_mis_fn_i32(int LR, int U);
// Flat-stream TMV for few outputs (tmv_flat_kernel.cuh; R <= 256, R % 4 != 0), NT = 256
// (R <= 64) or 1024 (R > 64):
//   (const T* B, const T* X, T* y, int64_t R, int64_t C, T* part, unsigned* cnt)
constexpr int TMV_FLAT_MAX_R = 256;
constexpr int TMV_FLAT_NT_SMALL_R = 64;     // R above this: 1024-thread CTAs
void* tmv_flat_fn(int dtype, int U, int NT);

// Lane groups on TMA-staged row tiles (rowtile_kernel.cuh; MV_SUBWARP / MV_WPR with
// [ADAPTIC_P_XSMEM] = 4), C <= 32*G, 16-byte-aligned A (and DOT's b), NT in {256, 512}:
//   (const T* A, const T* X, T* y, int64_t R, int64_t C, int k, int stages)   [dynamic smem]
constexpr int RT_MAX_C_PER_LANE = 32;
constexpr int RTC_KMAX_H = 8;                // rows per long-row staged tile (rowtile_kernel.cuh RTC_KMAX)
constexpr int RT_MAX_STAGES_H = 8;          // == RT_MAX_STAGES, TRT_MAX_STAGES (mbarriers per CTA; static_assert in k_rowtile.cu)
void* rowtile_fn(int dtype, int NT, int G, bool px);
size_t rowtile_tile_words(int64_t k, int64_t C);
// TMV with R <= NT outputs on staged tiles of B (tmv_rowtile_kernel.cuh; TMV_REGTILE with
// [ADAPTIC_P_XSMEM] = 4), 16-byte-aligned B and x, k % 4 == 0, NT in {256, 512, 1024}:
//   (const T* B, const T* X, T* y, int64_t R, int64_t C, int k, int stages, T* part, unsigned* cnt)
void* tmv_rowtile_fn(int dtype, int NT, int rpt);   // rpt: power of two >= R / NT, in {1, 2, 4}

// Multi-vector MV / TMV (mmv_kernels.cuh), fp32, K in {2, 4, 8}; X is K x C, Y is K x R:
//   group: (const float* A, const float* X, float* Y, int64_t R, int64_t C), rows of <= G*U vectors
//   cta  : (A, X, Y, R, C, int S, float* part, unsigned* cnt), RB = 8/K rows per CTA, NT = 256
//   tmmv : (B, X, Y, R, C, int S, float* part, unsigned* cnt), NT = 256, U in {2, 4}
constexpr int MMV_GROUP_RB = 2;
void* mmv_group_fn(int K, int G, int U, bool vec);
void* mmv_cta_fn(int K, int U, bool vec, bool xs);   // xs: K*C*4 bytes of x staged in smem
void* tmmv_fn(int K, int LR, int U, bool vec);
//   tmmv4: tmmv arguments; rows in groups of 4 (x_j as one float4 per group), L2 prefetch PF
//          groups ahead; C % 4 == 0, 16-byte-aligned B, X, Y; NT = 256 (XSMEM 8, UNROLL = PF)
void* tmmv4_fn(int K, int LR, int PF);
//   warp : (A, X, Y, R, C), warp per row, all K x-vectors in smem (K * C * 4 <= MMV_WARP_SMEM)
void* mmv_warp_fn(int K);
//   tile : (A, X, Y, R, C, int CW, int MB, float* part, unsigned* cnt), x chunks of CW values
//          staged in smem per piece of a stream-K range of (chunk, row) units, NT = 256
void* mmv_tile_fn(int dt, int K);
//   tmma : tmmv arguments; B rows staged by TMA in TMMV_TMA_STAGES stages of
//          TMMV_TMA_STAGE_V4 float4 (CR = STAGE_V4 / LR rows of LR float4), NT = 256, LR in {16..256}
void* tmmv_tma_fn(int K, int LR);
//   ring : (A, X, Y, R, C, int stages, int xres, int maxs, T* part, unsigned* cnt): the MATRIX
//          staged by TMA in an mbarrier ring (producer warp + 8 consumer warps, NT = 288),
//          groups of 8 rows x 256-float4 stages, stream-K over (group, column) positions;
//          K in {1, 2, 4, 8} (fp32), K = 1 also int32 (mmv_ring_kernel.cuh)
void* mmv_ring_fn(int dt, int K);
constexpr int MRING_BLOCK = 288;
//   tring: (B, X, Y, R, C, int TW, int CR, int stages, int stage_words, int maxs, T* part,
//          unsigned* cnt): TMV with B staged by TMA (tiles of TW outputs, CR rows per stage,
//          16-byte covers of any alignment), NT = 288; fp32 K in {1,2,4,8}, int32 K = 1;
//          opt = words per lane per row (tmv_ring_kernel.cuh)
void* tmv_ring_fn(int dt, int K, int opt);
//   tshift: tmv arguments (B, X, y, R, C, S, part, cnt); rows off the 16-byte grid, one aligned
//           128-bit load per row and thread at a constant word shift per c-lane; tiles of
//           4 LR - 4 outputs, LR in {16, 32, 64}, U in {2, 4, 8}, NT = 256 (tmv_mis_kernel.cuh)
void* tmv_shift_fn(int dt, int LR, int U);
//   twin: tmv arguments; rows off the 16-byte grid, one aligned load per row per thread, 7
//         accumulators and a compile-time shift pattern per 4 rows (tmv_window_kernel), tiles of
//         NT - 1 owned windows, G8 in {1, 2} groups of 4 rows in flight, NT = 256 (XSMEM 10)
void* tmv_window_fn(int dt, int G8);
void* rowtile_cta_fn(int dtype, int NT, int MX, int k);   // MX in {4, 8, 16, 36}: C <= NT * MX; k <= 8 rows
//   chunk: (A, X, y, R, C, int k, int stages, int W, T* part, unsigned* cnt): the long-row staged
//          CTA reduction on column chunks of W <= NT * MX (MX in {8, 16, 36}), k <= 4 row
//          segments per tile, chunk partials merged by the last CTA (XSMEM 13)
void* chunk_cta_fn(int dtype, int NT, int MX, int k);
void* tmv_window_warp_fn(int dt, int G8, int minb);
//   tgroup: (B, X, y, R, C, int ilv, T* part, unsigned* cnt): rows off the 16-byte grid on groups of four
//           rows (4R words = R aligned vectors), S slots per thread with fixed outputs, U groups
//           in flight, two-level ticket merge; 16-byte-aligned B, any x (tmv_group_kernel.cuh,
//           XSMEM 12); (S, U) in {(1,4), (1,8), (2,4), (3,2), (4,2)}, blockDim <= tmv_group_maxnt
void* tmv_group_fn(int dt, int S, int U);
int tmv_group_maxnt(int S, int U);
constexpr int TG_GROUP_H = 16;                      // == TG_GROUP (static_assert in k_tgroup.cu)
int64_t tring_stage_words_h(int64_t R, int TW, int CR, int K);
constexpr int64_t MRING_SMEM_BUDGET = 220 * 1024;
constexpr int TMMV_TMA_STAGE_V4 = 2048;              // 32 KB per stage
constexpr int TMMV_TMA_STAGES = 3;
constexpr int64_t MMV_TILE_XBYTES = 32 * 1024;       // x bytes per piece (all K vectors)
constexpr int64_t MMV_TILE_ONE_CHUNK = 48 * 1024;    // up to this K C 4: one chunk, no merge

// Five-point stencil (stencil_kernels.cu), 256 threads:
//   direct: (const float* u, const float* coef, float* v, int64_t H, int64_t W)
//   tile  : same arguments, dynamic smem 2 * (TH + 2) * (TW + 8) * 4 bytes
void* st_direct_fn(bool vec);
//   strip : same arguments; (strip of ST_STRIP_SV float4 columns, row) items, strip-major
void* st_strip_fn();
//   column: (u, coef, v, H, W, int TH): NT = 256 float4 columns x TH rows per tile, register
//           sliding window down each column (D = 4 rows loaded ahead)
void* st_column_fn();
//   direct2: direct arguments; row-major, two float4 outputs per thread per step (ORDER 4)
void* st_direct2_fn();
constexpr int ST_STRIP_SV = 256 * 4;
constexpr int64_t ST_STRIP_MIN_ROW = 131072;       // float4 per row from which strips are used
void* st_tile_fn(int TH, int TW);
constexpr int MMV_WARP_SMEM = 40 * 1024;

// BLAS-1 reductions (blas1_kernels.cuh), fp32 input, one translation unit per operator:
//   b1 group: (const float* A, void* y, int64_t R, int64_t C); rbu 0 = (RB 4, U 2), 1 = (RB 1, U 8)
//   b1 cta  : (const float* A, void* y, int64_t R, int64_t C, int S, P* part, unsigned* cnt)
constexpr int B1_CTA_NT = 256;
void* b1_group_fn_asum(int G, int rbu, bool vec);
void* b1_group_fn_nrm2(int G, int rbu, bool vec);
void* b1_group_fn_iamax(int G, int rbu, bool vec);
void* b1_group_fn_iamin(int G, int rbu, bool vec);
void* b1_cta_fn_asum(bool vec);
void* b1_cta_fn_nrm2(bool vec);
void* b1_cta_fn_iamax(bool vec);
void* b1_cta_fn_iamin(bool vec);
void* b1_group_fn_all(int G, int rbu, bool vec);
void* b1_cta_fn_all(bool vec);

}  // namespace adaptic
