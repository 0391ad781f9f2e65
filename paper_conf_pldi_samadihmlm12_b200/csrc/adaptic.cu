// adaptic.cu -- planner (runtime variant selector) and the C ABI of include/adaptic.h.
//
// The paper's "runtime kernel management" (Fig. 2): executed on the CPU,
// it selects the kernel generated for the subrange containing the actual input
// and sets "the number of blocks, number of threads per block, and the size of
// allocated shared memory".  Here the subranges are the cells of a 2-D table
// over (floor(log2 R), floor(log2 C)) per (op, dtype), fitted from B200 sweeps
// (tools/fit_thresholds.py -> table_data.inc); a cell that was not measured
// takes the nearest measured cell, and a problem far from every cell falls back
// to the analytic rules in heuristic_variant() (the paper's break-even idea,
// P:222-232, reduced to parallelism counts).
#include "adaptic.h"
#include "launch.h"

#include <algorithm>
#include <atomic>
#include <climits>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>
#include <unordered_map>

using namespace adaptic;

struct adaptic_plan_s {
    int op, dtype;
    int nvec;              // vectors per call: 1, or K in {2, 4, 8} (adaptic_plan_multi)
    int64_t R, C;
    int variant;
    int source;            // 0 forced, 1 table, 2 heuristic
    int sms;
    // kernel parameters
    int lanes;             // G (group) | NT (cta, tpr) | LR (tmv)
    int unroll;            // U
    int rb;                // group: rows per lane group per step (8 / U)
    int splits;            // S
    int ctas_per_sm;
    int stages;            // TPR
    int xmode;             // MV family: 0 x via read-only path, 1 x staged in smem (TMA), 2 per-row (DOT)
    int ilv;               // MV_SPLIT: 1 = splits interleave in steps of NT*U vectors, 0 = contiguous chunks
    int pipe;              // MV_CPR / MV_SPLIT: register double-buffered main loop
    size_t smem;           // dynamic shared memory bytes (TPR ring, or staged x)
    int block;
    bool vec_shape;        // C % 4 == 0 (MV/DOT) or R % 4 == 0 (TMV)
    bool flat;             // TMV_REGTILE with R <= 64, R % 4 != 0: the flat-stream kernel
    bool mis;              // MV/DOT with C % 4 != 0: index 1 describes the misaligned-row
                           // kernels (128-bit body + scalar head/tail, mv_mis_kernels.cuh)
    int64_t grid[2];       // [scalar, vector] instance
    int64_t chain[2];      // longest serial chain per accumulator
    int64_t depth[2];      // combine-tree depth after the chains
    bool path_ok[2];       // error bound provable for this instance
    // scalar fallback for TPR (misaligned pointers): a group kernel
    int fb_lanes, fb_unroll;
    // workspace
    size_t ws_bytes, cnt_off;
    size_t fb_ws_off;      // staged-tile plans: the direct-kernel fallback's workspace starts here
    size_t xsh_off;        // xmode 3 (misaligned MV): the four shifted copies of x start here
    bool multi_fb_ok;      // multi-vector 128-bit-shape plan: a 4-byte-path fallback is planned
                           // (its workspace slice starts at fb_ws_off)
    void* ws;
    size_t ws_cap;
};

namespace {

thread_local int g_last_cuda_error = 0;

struct TableEntry {
    int op, dtype, vec, lr, lc, variant, lanes, splits, ctas_per_sm, unroll, xsmem, block, rows, order, pipe;
};
const TableEntry kTable[] = {
#include "table_data.inc"
#include "table_b1.inc"
    {-1, -1, 0, 0, 0, 0, 0, 0, 0, 0, 0, 0, 0, 0, 0}};
const int kTableN = int(sizeof(kTable) / sizeof(kTable[0])) - 1;

const char* const kVariantNames[ADAPTIC_V_COUNT] = {
    "AUTO", "MV_TPR", "MV_SUBWARP", "MV_WPR", "MV_CPR", "MV_SPLIT",
    "TMV_COL", "TMV_SPLITK", "TMV_REGTILE", "ST_DIRECT", "ST_TILE"};

constexpr double kUnitRoundoff = 5.9604644775390625e-08;  // 2^-24
constexpr double kTol = 1e-4;                              // north_star tolerance

int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }
int ilog2_floor(int64_t v) { int k = -1; while (v > 0) { v >>= 1; ++k; } return k; }
int64_t pow2_ceil(int64_t v) { int64_t p = 1; while (p < v) p <<= 1; return p; }
int64_t pow2_floor(int64_t v) { int64_t p = 1; while (p * 2 <= v) p <<= 1; return p; }
int clampi(int64_t v, int lo, int hi) { return int(std::max<int64_t>(lo, std::min<int64_t>(hi, v))); }

struct DevInfo { int dev; int sms; bool present; };

DevInfo device_info() {
    DevInfo d{-1, 148, false};
    int dev = -1;
    if (cudaGetDevice(&dev) == cudaSuccess) {
        int sms = 0;
        if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) == cudaSuccess && sms > 0) {
            d.dev = dev; d.sms = sms; d.present = true;
        }
    }
    if (!d.present) (void)cudaGetLastError();   // a CPU host: clear the non-sticky error
    return d;
}

bool is_tmv_family(int v) { return v >= ADAPTIC_V_TMV_COL && v <= ADAPTIC_V_TMV_REGTILE; }
bool is_mv_family(int v) { return v >= ADAPTIC_V_MV_TPR && v <= ADAPTIC_V_MV_SPLIT; }
bool is_b1_op(int op) { return op >= ADAPTIC_OP_ASUM && op <= ADAPTIC_OP_B1ALL; }
// bytes of y per output row (B1ALL writes four N-vectors)
size_t y_bytes_per_row(int op) { return op == ADAPTIC_OP_B1ALL ? 16 : 4; }
bool is_b1_variant(int v) { return v >= ADAPTIC_V_MV_SUBWARP && v <= ADAPTIC_V_MV_SPLIT; }
bool op_has_variant(int op, int v) {
    if (op == ADAPTIC_OP_STENCIL5) return v == ADAPTIC_V_ST_DIRECT || v == ADAPTIC_V_ST_TILE;
    if (v == ADAPTIC_V_ST_DIRECT || v == ADAPTIC_V_ST_TILE) return false;
    if (op == ADAPTIC_OP_TMV) return is_tmv_family(v);
    if (is_b1_op(op)) return is_b1_variant(v);
    return is_mv_family(v);
}

void* group_fn(int dtype, int G, int U, bool vec, int xm) {
    return dtype == DT_F32 ? group_fn_f32(G, U, vec, xm) : group_fn_i32(G, U, vec, xm);
}

constexpr int64_t kXsAutoBytes = 32 * 1024;    // stage x in smem by default up to this size
constexpr int64_t kXsMaxBytes = 200 * 1024;

// x mode for the MV family: DOT streams its per-row operand; otherwise staged
// in shared memory when requested (param 2) or small enough (auto).
int pick_xmode(bool px, int req, int64_t C, bool allow) {
    if (px) return 2;
    if (!allow) return 0;
    if (req == 2) return C * 4 <= kXsMaxBytes ? 1 : -1;
    if (req == 1) return 0;
    return C * 4 <= kXsAutoBytes ? 1 : 0;
}
void* b1_group_fn(int op, int G, int rbu, bool vec) {
    switch (op) {
        case ADAPTIC_OP_ASUM: return b1_group_fn_asum(G, rbu, vec);
        case ADAPTIC_OP_NRM2: return b1_group_fn_nrm2(G, rbu, vec);
        case ADAPTIC_OP_IAMAX: return b1_group_fn_iamax(G, rbu, vec);
        case ADAPTIC_OP_IAMIN: return b1_group_fn_iamin(G, rbu, vec);
        case ADAPTIC_OP_B1ALL: return b1_group_fn_all(G, rbu, vec);
        default: return nullptr;
    }
}
void* b1_cta_fn(int op, bool vec) {
    switch (op) {
        case ADAPTIC_OP_ASUM: return b1_cta_fn_asum(vec);
        case ADAPTIC_OP_NRM2: return b1_cta_fn_nrm2(vec);
        case ADAPTIC_OP_IAMAX: return b1_cta_fn_iamax(vec);
        case ADAPTIC_OP_IAMIN: return b1_cta_fn_iamin(vec);
        case ADAPTIC_OP_B1ALL: return b1_cta_fn_all(vec);
        default: return nullptr;
    }
}
void* mis_group_fn(int dtype, int G, int U, int xm) {
    return dtype == DT_F32 ? mis_group_fn_f32(G, U, xm) : mis_group_fn_i32(G, U, xm);
}
void* mis_cta_fn(int dtype, int NT, int U, int xm) {
    return dtype == DT_F32 ? mis_cta_fn_f32(NT, U, xm) : mis_cta_fn_i32(NT, U, xm);
}
void* mis_cta_fx_fn(int dtype, int NT, int U) {
    return dtype == DT_F32 ? mis_cta_fx_fn_f32(NT, U) : mis_cta_fx_fn_i32(NT, U);
}
void* mis_cta_rb_fn(int dtype, int NT, int U, int RB) {
    return dtype == DT_F32 ? mis_cta_rb_fn_f32(NT, U, RB) : mis_cta_rb_fn_i32(NT, U, RB);
}
constexpr int64_t kMisMinCols = 16;   // below this a row is one or two vectors: scalar path
void* tmv_mis_fn(int dtype, int LR, int U) {
    return dtype == DT_F32 ? tmv_mis_fn_f32(LR, U) : tmv_mis_fn_i32(LR, U);
}
void* tmv_fn(int dtype, int LR, int U, bool vec, int NT) {
    return dtype == DT_F32 ? tmv_fn_f32(LR, U, vec, NT) : tmv_fn_i32(LR, U, vec, NT);
}

int occupancy(void* fn, int block, size_t smem, bool present, int fallback) {
    if (!present || fn == nullptr) return fallback;
    int n = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, fn, block, smem) != cudaSuccess || n <= 0) {
        (void)cudaGetLastError();
        return fallback;
    }
    return n;
}

// Does `dyn` bytes of dynamic shared memory fit beside the kernel's static shared memory?
// (the opt-in per-block maximum; without a device: 227 KB and an assumed 16 KB static)
bool smem_fits(void* fn, size_t dyn, bool present) {
    size_t stat = 16 * 1024, cap = 227 * 1024;
    if (present && fn) {
        cudaFuncAttributes fa;
        int dev = 0, optin = 0;
        if (cudaFuncGetAttributes(&fa, fn) == cudaSuccess) stat = fa.sharedSizeBytes;
        else (void)cudaGetLastError();
        if (cudaGetDevice(&dev) == cudaSuccess &&
            cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev) == cudaSuccess && optin > 0)
            cap = size_t(optin);
        else (void)cudaGetLastError();
    }
    return dyn + stat <= cap;
}

// Error bound of a tree whose longest path has `m` roundings (Higham eq. 4.4).
bool bound_ok(int64_t m) {
    const double mu = double(m) * kUnitRoundoff;
    return mu < 1.0 && mu / (1.0 - mu) <= kTol;
}
int64_t fold_chain(int64_t iters) { return std::min<int64_t>(iters, FOLD) + iters / FOLD; }
int ilog2c(int64_t v) { int k = 0; while ((int64_t(1) << k) < v) ++k; return k; }

// Split count for `units` independent reductions on `slots` resident CTAs: the
// grid-stride kernels take ceil(units*S / slots) rounds, so pick the smallest S
// in [smin, smax] whose last round is >= 90 % full and that fills >= 1 round
// (more splits only add partials to merge); else the best-filled S up to 4 rounds.
int64_t pick_splits(int64_t units, int64_t slots, int64_t smax, int64_t smin) {
    units = std::max<int64_t>(1, units);
    smax = std::max(smin, smax);
    const int64_t hi = std::min(smax, std::max(smin, ceil_div(4 * slots, units)));
    int64_t best = smin;
    double best_eff = -1.0;
    for (int64_t S = smin; S <= hi; ++S) {
        const int64_t nblk = units * S;
        const int64_t rounds = ceil_div(nblk, slots);
        const double eff = double(nblk) / double(rounds * slots);
        if (nblk >= slots && eff >= 0.9) return S;
        if (eff > best_eff + 1e-9) { best_eff = eff; best = S; }
    }
    return best;
}

// Split count for persistent grid-stride kernels whose blocks are long: the smallest S
// whose blocks fill the last wave to >= 90 % (one partly idle wave of long blocks costs
// less than a second wave plus twice the partials to merge).
int64_t pick_splits_wave(int64_t units, int64_t slots, int64_t smax) {
    units = std::max<int64_t>(1, units);
    int64_t best = 1;
    double best_eff = -1.0;
    for (int64_t S = 1; S <= std::max<int64_t>(1, smax); ++S) {
        const int64_t nblk = units * S;
        const double eff = double(nblk) / double(ceil_div(nblk, slots) * slots);
        if (eff >= 0.9) return S;
        if (eff > best_eff + 1e-9) { best_eff = eff; best = S; }
        if (nblk > 4 * slots) break;
    }
    return best;
}

// ---------------------------------------------------------------- heuristic (no table cell)
int heuristic_variant(int op, int64_t R, int64_t C, int sms) {
    // measured on B200 (profiles/r1_stencil_sweep.md): the L2-strip direct kernel beats
    // the shared-memory super tiles on every shape >= 64 MiB and on the L2-resident ones
    if (op == ADAPTIC_OP_STENCIL5) return ADAPTIC_V_ST_DIRECT;
    if (is_b1_op(op)) {
        // the paper's regimes (Fig. 1) for a unary reduction: lane groups
        // for many short rows, a CTA per row once rows are long and numerous
        // enough to fill the GPU, split rows (K1) when there are too few rows
        const int64_t nv = (C % 4 == 0) ? C / 4 : C;
        if (nv <= 32) return ADAPTIC_V_MV_SUBWARP;
        if (nv <= 2048 && R >= 4096) return ADAPTIC_V_MV_WPR;
        if (R >= 4 * int64_t(sms)) return ADAPTIC_V_MV_CPR;
        if (nv <= 1024) return ADAPTIC_V_MV_WPR;      // tiny: one launch, no merge
        return ADAPTIC_V_MV_SPLIT;
    }
    if (op == ADAPTIC_OP_TMV) {
        const int64_t rv = (R % 4 == 0) ? R / 4 : R;
        if (rv >= int64_t(sms) * 512 && C <= 4096) return ADAPTIC_V_TMV_COL;
        if (rv <= 256) return ADAPTIC_V_TMV_REGTILE;
        return ADAPTIC_V_TMV_SPLITK;
    }
    const int64_t nv = (C % 4 == 0) ? C / 4 : C;
    if (nv <= 16 && R >= 4096) return ADAPTIC_V_MV_SUBWARP;
    if (nv <= 4096 && R >= 8192) return ADAPTIC_V_MV_WPR;
    if (R >= 2 * int64_t(sms) && nv <= 4 * 1024 * 1024) return ADAPTIC_V_MV_CPR;
    return ADAPTIC_V_MV_SPLIT;
}

// Nearest measured cell of the same (op, dtype) and load-path shape (vec: the 128-bit
// path needs C % 4 == 0, for TMV R % 4 == 0 -- the two paths have different optima).
constexpr int kBeyondL2Log2 = 26;   // 2^26 elements = 256 MiB of fp32, 2x the 126 MB L2

const TableEntry* table_lookup_scan(int op, int dtype, int64_t R, int64_t C, bool* projected) {
    const int lr = ilog2_floor(R), lc = ilog2_floor(C);
    *projected = false;
    const int vec = (op == ADAPTIC_OP_TMV) ? (R % 4 == 0) : (C % 4 == 0);
    const TableEntry* best = nullptr;
    int bestd = INT_MAX;
    for (int i = 0; i < kTableN; ++i) {
        const TableEntry& e = kTable[i];
        if (e.op != op || e.dtype != dtype || e.vec != vec) continue;
        const int d = std::abs(e.lr - lr) + std::abs(e.lc - lc);
        // ties: prefer the cell with the same element count (lr + lc), then the lower lr
        if (d < bestd || (d == bestd && best && std::abs(e.lr + e.lc - lr - lc) < std::abs(best->lr + best->lc - lr - lc))) {
            best = &e; bestd = d;
        }
    }
    if (best && bestd <= 2) return best;
    // Larger than every measured cell nearby: once the input is well beyond L2 the
    // streaming behaviour depends on the aspect ratio, not on the size, so project onto
    // the largest measured diagonal (>= 2^26 elements, not above this problem) at the
    // same rows:cols ratio; absolute counts (splits, CTAs per SM) are then re-derived.
    int diag = -1;
    for (int i = 0; i < kTableN; ++i) {
        const TableEntry& e = kTable[i];
        if (e.op == op && e.dtype == dtype && e.vec == vec && e.lr + e.lc <= lr + lc) diag = std::max(diag, e.lr + e.lc);
    }
    if (diag >= kBeyondL2Log2) {
        const TableEntry* pb = nullptr;
        int pd = INT_MAX;
        for (int i = 0; i < kTableN; ++i) {
            const TableEntry& e = kTable[i];
            if (e.op != op || e.dtype != dtype || e.vec != vec || e.lr + e.lc != diag) continue;
            const int d = std::abs((e.lr - e.lc) - (lr - lc));
            if (d < pd) { pb = &e; pd = d; }
        }
        if (pb && pd <= 2) { *projected = true; return pb; }
    }
    // int32 moves the same bytes as fp32: use the fp32 cells when int32 was not swept
    if (dtype != ADAPTIC_F32) return table_lookup_scan(op, ADAPTIC_F32, R, C, projected);
    return nullptr;
}

// O(1) selector: the scan above depends on (op, dtype, vec, lr, lc) only, so its answer is
// memoised per cell in a dense index (0 = not computed yet, -1 = no cell, else entry index
// + 1 with bit 30 = projected).  Filling a cell is idempotent, so concurrent planners may
// race on it harmlessly (relaxed atomics); every later plan of that cell is one load.
constexpr int kOpsN = ADAPTIC_OP_STENCIL5 + 1;
std::atomic<int32_t> g_cell[kOpsN][2][2][64][64];

const TableEntry* table_lookup(int op, int dtype, int64_t R, int64_t C, bool* projected) {
    const int lr = ilog2_floor(R), lc = ilog2_floor(C);
    const int vec = (op == ADAPTIC_OP_TMV) ? (R % 4 == 0) : (C % 4 == 0);
    *projected = false;
    if (op < 0 || op >= kOpsN || dtype < 0 || dtype > 1 || lr < 0 || lc < 0 || lr > 63 || lc > 63)
        return table_lookup_scan(op, dtype, R, C, projected);
    std::atomic<int32_t>& cell = g_cell[op][dtype][vec][lr][lc];
    int32_t v = cell.load(std::memory_order_relaxed);
    if (v == 0) {
        bool pj = false;
        const TableEntry* e = table_lookup_scan(op, dtype, R, C, &pj);
        v = e ? int32_t(e - kTable + 1) | (pj ? (1 << 30) : 0) : -1;
        cell.store(v, std::memory_order_relaxed);
    }
    if (v < 0) return nullptr;
    *projected = (v >> 30) & 1;
    return &kTable[(v & ((1 << 30) - 1)) - 1];
}

// Five-point stencil: ST_DIRECT (no shared memory) or ST_TILE (TMA-staged super tiles,
// the paper's neighbouring-access optimization).  The super tile follows the
// input: the largest reuse metric sum(element accesses) / halo among tilings that
// still give every SM two CTAs' worth of tiles ("for small input sizes ... smaller super
// tiles in order to have more blocks").  Index 0 = the scalar direct kernel (fallback for
// misaligned pointers), index 1 = the planned kernel on the 128-bit path.
adaptic_status derive_stencil(adaptic_plan_s* p, const int32_t* params, const DevInfo& dev) {
    const int v = p->variant;
    const int64_t H = p->R, W = p->C;
    auto par = [&](int i) -> int { return params ? params[i] : 0; };
    p->vec_shape = (W % 4 == 0);
    p->mis = false; p->flat = false; p->splits = 1; p->smem = 0; p->stages = 0; p->xmode = 0; p->ilv = 0;
    p->pipe = 0; p->rb = 1; p->fb_lanes = 0; p->fb_unroll = 0; p->ws_bytes = 0; p->cnt_off = 0; p->unroll = 1;
    p->block = 256;
    const int cps_d = occupancy(st_direct_fn(false), 256, 0, dev.present, 8);
    p->grid[0] = std::max<int64_t>(1, std::min<int64_t>(ceil_div(H * W, 256), int64_t(dev.sms) * cps_d));
    p->chain[0] = p->chain[1] = 0;                    // no reduction: 3 roundings per point
    p->depth[0] = p->depth[1] = 3;
    p->path_ok[0] = true;
    p->grid[1] = 0; p->path_ok[1] = false;
    if (v == ADAPTIC_V_ST_DIRECT) {
        p->lanes = 4; p->ctas_per_sm = cps_d;
        if (p->vec_shape) {
            // rows of >= 2 MB: (strip, row) items strip-major (param ORDER 1 = the plain
            // row-major grid-stride sweep, 2 = strips).  Measured (profiles/r1_stencil_sweep.md):
            // equal up to 1-2 MB rows, strips +3..60 % beyond (8 x 8M: 3.9 -> 6.2 TB/s)
            const int ord = par(ADAPTIC_P_ORDER);
            p->xmode = (ord == 2 || (ord <= 0 && W / 4 >= ST_STRIP_MIN_ROW)) ? 1 : (ord == 3 ? 2 : ord == 4 ? 3 : 0);
            if (p->xmode == 3) {                             // row-major, 2 float4 per thread per step
                const int cps = occupancy(st_direct2_fn(), 256, 0, dev.present, 8);
                p->grid[1] = std::max<int64_t>(1, std::min<int64_t>(ceil_div(H * (W / 4), 512), int64_t(dev.sms) * cps));
                p->ctas_per_sm = cps;
            } else if (p->xmode == 2) {                             // column sweep, register sliding window
                const int th = par(ADAPTIC_P_ROWS) > 0 ? par(ADAPTIC_P_ROWS) : 64;
                p->rb = th;
                const int cps = occupancy(st_column_fn(), 256, 0, dev.present, 8);
                const int64_t tiles = ceil_div(W / 4, int64_t(256)) * ceil_div(H, int64_t(th));
                p->grid[1] = std::max<int64_t>(1, std::min<int64_t>(tiles, int64_t(dev.sms) * cps));
                p->ctas_per_sm = cps;
            } else if (p->xmode == 1) {
                const int cps = occupancy(st_strip_fn(), 256, 0, dev.present, 8);
                const int64_t items = ceil_div(W / 4, int64_t(ST_STRIP_SV)) * H;
                p->grid[1] = std::max<int64_t>(1, std::min<int64_t>(items, int64_t(dev.sms) * cps));
                p->ctas_per_sm = cps;
            } else {
                const int cps = occupancy(st_direct_fn(true), 256, 0, dev.present, 8);
                p->grid[1] = std::max<int64_t>(1, std::min<int64_t>(ceil_div(H * (W / 4), 256), int64_t(dev.sms) * cps));
            }
            p->path_ok[1] = true;
        }
        return ADAPTIC_OK;
    }
    if (!p->vec_shape) return ADAPTIC_ERR_UNSUPPORTED;   // TMA rows need C % 4 == 0
    static const int kTH[] = {4, 8, 16, 32}, kTW[] = {128, 256, 512};
    int TH = par(ADAPTIC_P_ROWS), TW = par(ADAPTIC_P_LANES);
    if (TH > 0 || TW > 0) {
        if (TH <= 0) TH = 8;
        if (TW <= 0) TW = 256;
        if (!st_tile_fn(TH, TW)) return ADAPTIC_ERR_INVALID_ARG;
    } else {
        double best = -1.0, best_tiles = -1.0;
        int bth = 4, btw = 128;
        const double want = 2.0 * dev.sms;
        for (int th : kTH)
            for (int tw : kTW) {
                if (tw > std::max<int64_t>(128, pow2_ceil(W))) continue;
                const double tiles = double(ceil_div(H, th)) * double(ceil_div(W, tw));
                const double reuse = 5.0 * th * tw / double((th + 2) * (tw + 8) - th * tw);
                const bool enough = tiles >= want;
                // prefer tilings with enough blocks, then the reuse metric; if none has
                // enough blocks, the one with the most tiles
                const double key = enough ? 1e9 + reuse : tiles;
                if (key > best || (key == best && tiles > best_tiles)) { best = key; best_tiles = tiles; bth = th; btw = tw; }
            }
        TH = bth; TW = btw;
    }
    p->rb = TH; p->lanes = TW;
    p->smem = size_t(2) * size_t(TH + 2) * size_t(TW + 8) * 4;
    int cps = par(ADAPTIC_P_CTAS_PER_SM);
    if (cps <= 0) cps = occupancy(st_tile_fn(TH, TW), 256, p->smem, dev.present, 2);
    p->ctas_per_sm = std::max(1, cps);
    const int64_t tiles = ceil_div(H, TH) * ceil_div(W, TW);
    p->grid[1] = std::max<int64_t>(1, std::min<int64_t>(tiles, int64_t(dev.sms) * p->ctas_per_sm));
    p->path_ok[1] = true;
    return ADAPTIC_OK;
}

// Multi-vector MV / TMV (adaptic_plan_multi): K = nvec vectors share one pass over the
// matrix (horizontal actor integration; mmv_kernels.cuh).  fp32, 128-bit path
// shapes and scalar shapes alike (aligned pointers take the 128-bit instances).
// Multi-vector TMV rows in groups of 4 (tmmv4_kernel) where it measured > 2 % faster than
// round 1's choice on the 256 MiB diagonals (profiles/r2_exp/r2z_t4_cmp.jsonl; bit
// floor(log2 R) of the mask)
bool tmmv4_rule(int K, int64_t R, int64_t C) {
    const uint32_t mask = K == 2 ? 0x13FF00u : K == 4 ? 0x17FF00u : K == 8 ? 0x3FFFC0u : 0u;
    const int lr = ilog2_floor(R);
    return R % 4 == 0 && C % 4 == 0 && lr >= 0 && lr < 32 && ((mask >> lr) & 1u);
}

// TMV (any K, any alignment, any R) with B staged by TMA (tmv_ring_kernel.cuh): tiles of TW
// outputs = WPT column groups of 32 OPT words, LC = 8 / WPT row lanes; one tile covering all
// outputs streams whole rows (one contiguous copy per stage of ~32 KB), else CR row segments.
// params: LANES = OPT, PIPE = stages (default 4: the measured optimum of a bare TMA stream)
adaptic_status derive_tmv_ring(adaptic_plan_s* p, const int32_t* params, const DevInfo& dev) {
    auto par = [&](int i) -> int { return params ? params[i] : 0; };
    const int K = p->nvec;
    const int64_t R = p->R, C = p->C;
    const int opt_max = std::min(8, 32 / K);
    const bool flat = R <= int64_t(256);                     // one tile, output per thread
    int OPT = par(ADAPTIC_P_LANES);
    if (OPT <= 0) OPT = flat ? 1 : clampi(pow2_floor(std::max<int64_t>(1, R / 256)), 1, opt_max);
    if (OPT > opt_max || (OPT & (OPT - 1))) return ADAPTIC_ERR_INVALID_ARG;
    if (!tmv_ring_fn(p->dtype, K, OPT)) return ADAPTIC_ERR_UNSUPPORTED;
    const int WW = 32 * OPT;
    // tile width: as wide as possible (long bulk copies), but the last CTA of a tile merges
    // TW K outputs x (CTAs per tile ~ sms TW / R) partials -- keep that <= ~24 loads of
    // 16 bytes per thread (measured: one 2048-word tile over 148 CTAs cost ~150 us to merge)
    int WPT = flat ? 1 : clampi(pow2_ceil(ceil_div(R, int64_t(WW))), 1, 8);
    if (par(ADAPTIC_P_ROWS) > 0) WPT = clampi(par(ADAPTIC_P_ROWS), 1, 8);
    else
        while (!flat && WPT > 1) {
            const int64_t tw = int64_t(WW) * WPT;
            const int64_t per_tile = ceil_div(int64_t(dev.sms) * tw, R) + 1;
            if (tw * K * per_tile / 4 <= 24 * 256) break;
            WPT /= 2;
        }
    const int TW = flat ? int(R) : WW * WPT, LC = 8 / WPT;
    const bool contig = TW >= R;
    // ~32 KB stages (B rows + their x chunks); row-segment stages take one producer lane per
    // row, the x chunks the last K lanes
    const int CR = contig ? int(std::max<int64_t>(1, std::min<int64_t>(C, (int64_t(8192) - 40 - 40 * int64_t(K)) / (R + K))))
                          : std::max(1, std::min(32 - K, 8704 / (TW + 8 + K)));
    const int64_t sw = tring_stage_words_h(R, TW, CR, K);
    const int64_t red = (flat ? int64_t(int64_t(256) / R) * K * R : int64_t(LC - 1) * K * TW) * 4;
    const int64_t fit = (MRING_SMEM_BUDGET - red) / (sw * 4);
    const int stages = int(std::min<int64_t>(par(ADAPTIC_P_PIPE) > 0 ? std::min(8, par(ADAPTIC_P_PIPE)) : 4, fit));
    if (stages < 2) return ADAPTIC_ERR_UNSUPPORTED;
    const int64_t ntiles = ceil_div(R, int64_t(TW)), Tw = ntiles * C;
    if (Tw > (int64_t(1) << 62) / 256) return ADAPTIC_ERR_UNSUPPORTED;
    const int64_t grid = std::max<int64_t>(1, std::min<int64_t>(dev.sms, Tw));
    const int64_t per = std::max<int64_t>(1, Tw / grid);
    const int64_t maxs = C / per + 2;
    if (maxs > int64_t(INT_MAX) / 64) return ADAPTIC_ERR_UNSUPPORTED;
    const int64_t lanes = flat ? int64_t(256) / R : int64_t(LC);      // row lanes per output
    const int64_t P = ceil_div(std::min(C, ceil_div(Tw, grid)), lanes);   // rows per thread per segment
    p->xmode = 6; p->block = MRING_BLOCK; p->ctas_per_sm = 1;
    p->ilv = par(ADAPTIC_P_ORDER) >= 8 ? par(ADAPTIC_P_ORDER) - 8 : 0;
    p->lanes = TW; p->unroll = OPT; p->splits = CR; p->stages = stages; p->rb = int(maxs);
    p->smem = size_t(int64_t(stages) * sw * 4 + red);
    p->mis = false; p->flat = false; p->vec_shape = R % 4 == 0; p->xsh_off = 0; p->fb_ws_off = 0;
    for (int w = 0; w < 2; ++w) {
        p->grid[w] = grid;
        p->chain[w] = std::min<int64_t>(P, FOLD) + P / FOLD;
        p->depth[w] = lanes + ceil_div(maxs, 2) + 2;
        p->path_ok[w] = bound_ok(p->chain[w] + p->depth[w]);
    }
    const size_t part = ((size_t(ntiles) * size_t(maxs) * size_t(K) * size_t(TW) * 4 + 255) / 256) * 256;
    p->cnt_off = part;
    p->ws_bytes = part + size_t(ntiles) * 4;
    return p->path_ok[1] ? ADAPTIC_OK : ADAPTIC_ERR_UNSUPPORTED;
}

adaptic_status derive_multi(adaptic_plan_s* p, const int32_t* params, const DevInfo& dev) {
    const int op = p->op, v = p->variant, K = p->nvec;
    const int64_t R = p->R, C = p->C;
    auto par = [&](int i) -> int { return params ? params[i] : 0; };
    p->vec_shape = (op == ADAPTIC_OP_TMV) ? (R % 4 == 0) : (C % 4 == 0);
    p->mis = false; p->splits = 1; p->smem = 0; p->stages = 0; p->xmode = 0; p->ilv = 0; p->pipe = 0; p->rb = 1;
    p->fb_lanes = 0; p->fb_unroll = 0; p->ws_bytes = 0; p->cnt_off = 0;
    for (int w = 0; w < 2; ++w) { p->grid[w] = 0; p->chain[w] = 0; p->depth[w] = 0; p->path_ok[w] = false; }
    auto chain_of = [&](int64_t iters, int U) -> int64_t {
        const int64_t f = FOLD / U;
        return int64_t(U) * std::min<int64_t>(iters, f) + iters / f;
    };
    if (op == ADAPTIC_OP_MV && v == ADAPTIC_V_MV_WPR && p->vec_shape && int64_t(K) * C * 4 <= MMV_WARP_SMEM &&
        C / 4 > int64_t(32) * (K == 8 ? 2 : 4)) {
        // medium rows: warp per row, all K x-vectors staged in shared memory (mmv_warp_kernel)
        const int NT = 256, RB = 1, U = 2;
        p->smem = size_t(K) * size_t(C) * 4;
        p->xmode = 3;
        int cps = par(ADAPTIC_P_CTAS_PER_SM);
        if (cps <= 0) cps = occupancy(mmv_warp_fn(K), NT, p->smem, dev.present, 4);
        p->lanes = 32; p->unroll = U; p->block = NT; p->rb = RB; p->ctas_per_sm = cps;
        const int64_t iters = ceil_div(C / 4, int64_t(32) * U);
        p->grid[1] = std::max<int64_t>(1, std::min<int64_t>(ceil_div(R, int64_t(RB) * (NT / 32)), int64_t(dev.sms) * cps));
        p->chain[1] = chain_of(iters, U);
        p->depth[1] = 2 + 5 + 1;
        p->path_ok[1] = bound_ok(p->chain[1] + p->depth[1]);
        return p->path_ok[1] ? ADAPTIC_OK : ADAPTIC_ERR_UNSUPPORTED;
    }
    if (op == ADAPTIC_OP_MV && (v == ADAPTIC_V_MV_SUBWARP || v == ADAPTIC_V_MV_WPR)) {
        // short rows, x in registers: each lane covers <= U vectors of a row.  Only the
        // plan's own load path is planned (G and U depend on the row length in loads),
        // so a 128-bit-shape plan run on misaligned pointers reports MISALIGNED.
        {
            const int w = p->vec_shape ? 1 : 0;
            const int64_t nv = w ? C / 4 : C;
            int U = par(ADAPTIC_P_UNROLL);
            int G = (v == ADAPTIC_V_MV_WPR) ? 32 : par(ADAPTIC_P_LANES);
            if (U <= 0) U = (K == 8 || nv > 64) ? 2 : 4;
            if (G <= 0) G = clampi(pow2_ceil(ceil_div(std::max<int64_t>(1, nv), U)), 1, 32);
            if (G < 1 || G > 32 || (G & (G - 1)) || (U != 1 && U != 2 && U != 4) || K * U > 16)
                return ADAPTIC_ERR_INVALID_ARG;
            if (nv > int64_t(G) * U) return ADAPTIC_ERR_UNSUPPORTED;       // row longer than one step
            p->lanes = G; p->unroll = U; p->block = GROUP_NT; p->rb = MMV_GROUP_RB;
            int cps = par(ADAPTIC_P_CTAS_PER_SM);
            if (cps <= 0) cps = occupancy(mmv_group_fn(K, G, U, w == 1), GROUP_NT, 0, dev.present, 4);
            p->ctas_per_sm = cps;
            const int rows_per_cta = MMV_GROUP_RB * (32 / G) * (GROUP_NT / 32);
            p->grid[w] = std::max<int64_t>(1, std::min<int64_t>(ceil_div(R, rows_per_cta), int64_t(dev.sms) * cps));
            p->chain[w] = U;
            p->depth[w] = (w ? 2 : 0) + ilog2c(G) + 1;
            p->path_ok[w] = bound_ok(p->chain[w] + p->depth[w]);
        }
        return p->path_ok[p->vec_shape ? 1 : 0] ? ADAPTIC_OK : ADAPTIC_ERR_UNSUPPORTED;
    }
    // AUTO multi-vector MV_SPLIT with long rows (C >= 8192): the matrix through the TMA ring
    // (measured, scratch r2f: 64 x 1M K = 4 0.66 -> 0.85 of the copy peak, K = 8 0.36 -> 0.67;
    // 16384 x 4096 and shorter rows: the x-tile kernel is as fast or faster)
    const bool ring_rule = K > 1 && v == ADAPTIC_V_MV_SPLIT && par(ADAPTIC_P_XSMEM) <= 0 && C >= 8192;
    if (op == ADAPTIC_OP_MV && (v == ADAPTIC_V_MV_CPR || v == ADAPTIC_V_MV_SPLIT) && p->vec_shape &&
        (par(ADAPTIC_P_XSMEM) == 6 || ring_rule)) {
        // the matrix through a TMA ring (mmv_ring_kernel.cuh): groups of 8 rows, 256-float4
        // stages, stream-K over the (group, column) positions of one CTA per SM
        constexpr int RT = 8, CH = 256, FOLDP = 128, NT = 256;
        const int64_t nv = C / 4, ngroups = ceil_div(R, RT), Tw = ngroups * nv;
        const int cps = std::max(1, std::min(2, par(ADAPTIC_P_CTAS_PER_SM)));     // CTAs per SM
        const int64_t grid = std::max<int64_t>(1, std::min<int64_t>(int64_t(dev.sms) * cps, Tw));
        const int64_t xbytes = int64_t(K) * C * 4;
        const bool xres = xbytes <= 64 * 1024 / cps;
        const int64_t stage = int64_t(RT + (xres ? 0 : K)) * CH * 16;
        // 4 stages of 32 KB of A in flight per SM is the measured optimum of a bare TMA
        // stream (7.1 TB/s; 6 stages: 6.5 TB/s -- too many requests in flight, scratch r2h)
        const int64_t fit = (MRING_SMEM_BUDGET / cps - (xres ? xbytes : 0)) / stage;
        int stages = int(std::min<int64_t>(par(ADAPTIC_P_PIPE) > 0 ? std::min(8, par(ADAPTIC_P_PIPE)) : 4, fit));
        if (stages < 2 || !mmv_ring_fn(p->dtype, K)) return ADAPTIC_ERR_UNSUPPORTED;
        if (Tw > (int64_t(1) << 62) / 256) return ADAPTIC_ERR_UNSUPPORTED;
        const int64_t per = std::max<int64_t>(1, Tw / grid);     // shortest CTA range
        const int64_t maxs = nv / per + 2;                       // CTAs touching one group
        if (maxs > int64_t(INT_MAX) / 64) return ADAPTIC_ERR_UNSUPPORTED;
        const int N = RT * K, NG = NT / N;
        const int64_t P = ceil_div(std::min(nv, ceil_div(Tw, grid)), int64_t(CH));   // positions / segment
        p->smem = size_t((xres ? xbytes : 0) + int64_t(stages) * stage);
        p->xmode = 6;
        p->block = MRING_BLOCK; p->ctas_per_sm = cps; p->splits = 1; p->unroll = 1;
        p->stages = stages; p->lanes = (xres ? 1 : 0) | (par(ADAPTIC_P_ORDER) == 9 ? 2 : 0); p->rb = int(maxs);
        p->grid[1] = grid;
        p->chain[1] = 4 * std::min<int64_t>(P, FOLDP) + P / FOLDP;
        p->depth[1] = 5 + (NT / 32) + ceil_div(maxs, NG) + NG + 1;
        p->path_ok[1] = bound_ok(p->chain[1] + p->depth[1]);
        const size_t part = ((size_t(ngroups) * size_t(maxs) * size_t(N) * 4 + 255) / 256) * 256;
        p->cnt_off = part;
        p->ws_bytes = part + size_t(ngroups) * 4;
        return p->path_ok[1] ? ADAPTIC_OK : ADAPTIC_ERR_UNSUPPORTED;
    }
    if (op == ADAPTIC_OP_MV && (v == ADAPTIC_V_MV_CPR || v == ADAPTIC_V_MV_SPLIT) && p->vec_shape &&
        (par(ADAPTIC_P_XSMEM) == 3 ||
         (par(ADAPTIC_P_XSMEM) <= 0 && v == ADAPTIC_V_MV_SPLIT && par(ADAPTIC_P_SPLITS) <= 0 && R > 16))) {
        // (R <= 16: the interleaved-split kernel with x through L1 measured 1.3x faster at 8 rows)
        // x tiles in shared memory, stream-K ranges of (chunk, row) units (mmv_tile_kernel):
        // params LANES = chunk width CW (values), ROWS = rows per merge ticket MB
        const int NT = 256, U = 2;                   // RB = 4 rows per warp step (2 at K = 8)
        int64_t CW = par(ADAPTIC_P_LANES);
        if (CW <= 0) CW = (int64_t(K) * C * 4 <= MMV_TILE_ONE_CHUNK) ? C : MMV_TILE_XBYTES / (4 * K);
        if (CW <= 0 || CW % 4 != 0 || 2 * int64_t(K) * CW * 4 > kXsMaxBytes) return ADAPTIC_ERR_INVALID_ARG;
        CW = std::min<int64_t>(CW, C);
        // a fitted width above the default that would still cut C into several chunks: the
        // default.  Every such pair in the training sweeps measured the wider chunks slower
        // (1 CTA per SM with the double-buffered 2 x 64 KB of x; 0.75-0.97, median 0.87 of the
        // 8192 chunks over 57 shapes); a wider width only pays as ONE chunk (C <= width)
        if (K == 1 && CW < C && CW > MMV_TILE_XBYTES / 4) CW = MMV_TILE_XBYTES / 4;
        // balanced chunks: a table width fitted on C = 2^k (an exact multiple) would leave the
        // last chunk of another C mostly empty (held-out 6144 x 26624: 1.6 chunks of 16384, 0.86
        // of the best plan); the same number of chunks, evenly filled
        CW = std::min<int64_t>(CW, (ceil_div(C, ceil_div(C, CW)) + 3) / 4 * 4);
        const int64_t nch = ceil_div(C, CW);
        int MB = par(ADAPTIC_P_ROWS);
        if (MB <= 0) {
            // merge work per block: K MB outputs x nch chunks over NT threads, <= ~64 chunks each
            // (measured, 64 x 1M K = 4: MB 8 -> 4.25 TB/s, MB 2 -> 3.45, MB 64 -> 3.45)
            const int64_t emax = std::max<int64_t>(1, std::min<int64_t>(NT, int64_t(NT) * 64 / nch));
            MB = clampi(int(pow2_floor(std::max<int64_t>(1, emax / K))), 1, 64);
        }
        if (nch * R > (int64_t(1) << 62) / 256) return ADAPTIC_ERR_UNSUPPORTED;
        if (nch > 1 && int64_t(std::min<int64_t>(MB, R)) * nch > int64_t(UINT_MAX)) return ADAPTIC_ERR_UNSUPPORTED;
        p->smem = (nch > 1 ? 2 : 1) * size_t(K) * size_t(CW) * 4;   // x chunks, double-buffered
        p->xmode = 4;
        int cps = par(ADAPTIC_P_CTAS_PER_SM);
        if (cps <= 0) cps = occupancy(mmv_tile_fn(p->dtype, K), NT, p->smem, dev.present, 2);
        p->lanes = int(CW); p->unroll = U; p->block = NT; p->rb = MB; p->ctas_per_sm = cps;
        p->splits = int(std::min<int64_t>(nch, INT_MAX));
        p->grid[1] = std::max<int64_t>(1, std::min<int64_t>(nch * R, int64_t(dev.sms) * cps));
        const int64_t per_lane = ceil_div(CW / 4, int64_t(32));
        int64_t merge = 0;
        if (nch > 1) {
            const int64_t E = int64_t(K) * MB;
            const int64_t G = E <= NT ? NT / E : 1;
            const int64_t per = ceil_div(nch, G);
            merge = std::min<int64_t>(per, 32) + per / 32 + G;
        }
        p->chain[1] = 4 * per_lane;
        p->depth[1] = 5 + merge + 1;
        p->path_ok[1] = bound_ok(p->chain[1] + p->depth[1]);
        if (nch > 1) {
            const size_t part = ((size_t(nch) * size_t(K) * size_t(R) * 4 + 255) / 256) * 256;
            p->cnt_off = part;
            p->ws_bytes = part + size_t(ceil_div(R, int64_t(MB))) * 4;
        }
        return p->path_ok[1] ? ADAPTIC_OK : ADAPTIC_ERR_UNSUPPORTED;
    }
    if (op == ADAPTIC_OP_MV && (v == ADAPTIC_V_MV_CPR || v == ADAPTIC_V_MV_SPLIT)) {
        const int NT = 256, RB = 8 / K;
        const int64_t nvr = p->vec_shape ? C / 4 : C;
        int U = par(ADAPTIC_P_UNROLL);
        if (U <= 0) U = nvr >= 2 * NT ? 2 : 1;             // short rows: do not idle half the CTA
        if (U != 1 && U != 2) return ADAPTIC_ERR_INVALID_ARG;
        // x of all K vectors in shared memory when small (param XSMEM: 1 off, 2 on)
        const int xreq = par(ADAPTIC_P_XSMEM);
        const bool xs = xreq == 2 ? (K * C * 4 <= kXsMaxBytes) : (xreq != 1 && K * C * 4 <= kXsAutoBytes * 2);
        if (xreq == 2 && !xs) return ADAPTIC_ERR_UNSUPPORTED;
        p->xmode = xs ? 1 : 0;
        p->smem = xs ? size_t(K) * size_t(C) * 4 : 0;
        int cps = par(ADAPTIC_P_CTAS_PER_SM);
        if (cps <= 0) cps = occupancy(mmv_cta_fn(K, U, p->vec_shape, xs), NT, p->smem, dev.present, 2048 / NT);
        p->lanes = NT; p->unroll = U; p->block = NT; p->rb = RB; p->ctas_per_sm = cps;
        const int64_t slots = int64_t(dev.sms) * cps;
        const int64_t groups = ceil_div(R, RB);
        const int64_t nv1 = p->vec_shape ? C / 4 : C;
        int64_t S = 1;
        if (v == ADAPTIC_V_MV_SPLIT)
            S = par(ADAPTIC_P_SPLITS) > 0 ? par(ADAPTIC_P_SPLITS)
                                          : pick_splits(groups, slots, std::max<int64_t>(2, ceil_div(nv1, int64_t(NT) * U)), 2);
        for (;;) {
            bool ok_all = true;
            for (int w = 0; w < 2; ++w) {
                if (w == 1 && !p->vec_shape) continue;
                const int64_t nv = w ? C / 4 : C;
                const int64_t iters = ceil_div(nv, int64_t(S) * NT * U);
                p->chain[w] = chain_of(iters, U);
                p->depth[w] = (w ? 2 : 0) + ilog2c(NT) + (S > 1 ? ceil_div(S, NT) + ilog2c(NT) : 0) + 1;
                p->path_ok[w] = bound_ok(p->chain[w] + p->depth[w]);
                p->grid[w] = std::max<int64_t>(1, std::min<int64_t>(groups * S, slots));
                if (!p->path_ok[w]) ok_all = false;
            }
            if (ok_all || v == ADAPTIC_V_MV_CPR || S >= (int64_t(1) << 20)) break;
            S *= 2;
        }
        if (S > INT_MAX) return ADAPTIC_ERR_UNSUPPORTED;
        p->splits = int(S);
        p->ilv = S > 1 ? 1 : 0;
        if (!p->path_ok[p->vec_shape ? 1 : 0]) return ADAPTIC_ERR_UNSUPPORTED;
        if (S > 1) {
            const size_t part = ((size_t(R) * size_t(K) * size_t(S) * 4 + 255) / 256) * 256;
            p->cnt_off = part;
            p->ws_bytes = part + size_t(groups) * 4;
        }
        return ADAPTIC_OK;
    }
    if (op != ADAPTIC_OP_TMV || !is_tmv_family(v)) return ADAPTIC_ERR_UNSUPPORTED;
    if (par(ADAPTIC_P_XSMEM) == 6) return derive_tmv_ring(p, params, dev);
    // AUTO: where the row-group kernel measured > 2 % faster than round 1's choice on the
    // 256 MiB diagonals (profiles/r2_exp/r2z_t4_cmp.jsonl; bit lr of the mask = floor(log2 R)):
    // tiles of 16 / 64 / 128 output vectors, L2 prefetch 2 groups ahead except at K = 8
    const int lr_r = ilog2_floor(R);
    const bool t4_rule = !params && v == ADAPTIC_V_TMV_SPLITK && tmmv4_rule(K, R, C);
    if (par(ADAPTIC_P_XSMEM) == 8 || t4_rule) {
        // rows in groups of 4: x_j as one float4 per group, L2 prefetch (tmmv4_kernel)
        if (!p->vec_shape || C % 4 != 0) return ADAPTIC_ERR_UNSUPPORTED;
        const int NT = 256;
        const int64_t rv = R / 4;
        int LR = par(ADAPTIC_P_LANES);
        if (LR <= 0) LR = t4_rule ? (lr_r <= 11 ? 16 : lr_r <= 16 ? 64 : 128) : clampi(pow2_ceil(rv), 16, 64);
        int PF = par(ADAPTIC_P_UNROLL);
        if (PF < 0) PF = 0;
        if (par(ADAPTIC_P_UNROLL) == 0) PF = (K == 8 || (K == 4 && lr_r <= 11)) ? 1 : 2;
        void* fn = tmmv4_fn(K, LR, PF == 1 ? 0 : PF);
        if (!fn) return ADAPTIC_ERR_INVALID_ARG;
        int cps = par(ADAPTIC_P_CTAS_PER_SM);
        if (cps <= 0) cps = occupancy(fn, NT, 0, dev.present, 2);
        const int LC = NT / LR;
        const int64_t slots = int64_t(dev.sms) * cps;
        const int64_t tiles = ceil_div(rv, int64_t(LR));
        const int64_t ngr = C / 4;
        int64_t S = par(ADAPTIC_P_SPLITS) > 0 ? par(ADAPTIC_P_SPLITS)
                                              : pick_splits_wave(tiles, slots, std::max<int64_t>(1, ceil_div(ngr, int64_t(LC))));
        for (;;) {
            const int64_t gpt = ceil_div(ceil_div(ngr, S), int64_t(LC));          // groups per thread
            p->chain[1] = 4 * std::min<int64_t>(gpt, FOLD / 4) + gpt / (FOLD / 4);
            p->depth[1] = ilog2c(LC) + (S > 1 ? ceil_div(S, LC) + ilog2c(LC) : 0) + 1;
            p->path_ok[1] = bound_ok(p->chain[1] + p->depth[1]);
            if (p->path_ok[1] || S >= (int64_t(1) << 20)) break;
            S *= 2;
        }
        if (S > INT_MAX || !p->path_ok[1]) return ADAPTIC_ERR_UNSUPPORTED;
        p->xmode = 8;
        p->lanes = LR; p->unroll = PF == 1 ? 0 : PF; p->block = NT; p->ctas_per_sm = cps; p->splits = int(S);
        p->grid[1] = std::max<int64_t>(1, std::min<int64_t>(tiles * S, slots));
        if (S > 1) {
            const size_t part = ((size_t(R) * size_t(K) * size_t(S) * 4 + 255) / 256) * 256;
            p->cnt_off = part;
            p->ws_bytes = part + size_t(tiles) * 4;
        }
        return ADAPTIC_OK;
    }
    // TMV tiles: LR output vectors x (256 / LR) c-lanes, S c-ranges
    const int NT = 256;
    int U = par(ADAPTIC_P_UNROLL);
    if (U <= 0) U = K <= 4 ? 4 : 2;
    if (U != 2 && !(U == 4 && K <= 4)) return ADAPTIC_ERR_INVALID_ARG;
    const int64_t rv1 = p->vec_shape ? R / 4 : R;
    int LR = par(ADAPTIC_P_LANES);
    if (LR <= 0) LR = (v == ADAPTIC_V_TMV_COL) ? 256 : (v == ADAPTIC_V_TMV_REGTILE) ? clampi(pow2_ceil(rv1), 1, 256)
                                                                                  : clampi(pow2_ceil(rv1), 1, rv1 <= 256 ? 32 : 64);
    if (LR < 1 || LR > 256 || (LR & (LR - 1))) return ADAPTIC_ERR_INVALID_ARG;
    if (v == ADAPTIC_V_TMV_REGTILE && rv1 > LR) return ADAPTIC_ERR_UNSUPPORTED;
    // B rows staged by TMA (tmmv_tma_kernel; param XSMEM 1 = the register-fed kernel)
    // measured (profiles/r1c_multi_tmv.md): TMA staging wins for few outputs (R <= 256: one
    // contiguous bulk copy per stage, +23-34 % at K = 4) and for R >= 256K with C >= 128 (+14-25 %);
    // elsewhere both are within a few % and the register-fed kernel is kept.
    // param XSMEM: 3 = TMA-staged, 1 = register-fed, 0 = this rule
    const int xreq = par(ADAPTIC_P_XSMEM);
    const bool tma_rule = rv1 <= 64 || (rv1 >= 65536 && C >= 128);
    if (p->vec_shape && rv1 >= 16 && v != ADAPTIC_V_TMV_COL && (xreq == 3 || (xreq <= 0 && tma_rule)) &&
        (par(ADAPTIC_P_LANES) <= 0 || par(ADAPTIC_P_LANES) >= 16)) {
        // LR: the widest tile (longest bulk copies) whose split count still fills the GPU with
        // at most 16 LC partials to merge per thread (the merging CTA reads S / LC per thread)
        p->smem = size_t(TMMV_TMA_STAGES) * TMMV_TMA_STAGE_V4 * 16;
        int cps = par(ADAPTIC_P_CTAS_PER_SM);
        if (cps <= 0) cps = occupancy(tmmv_tma_fn(K, 64), NT, p->smem, dev.present, 2);
        const int64_t slots = int64_t(dev.sms) * cps;
        auto splits_for = [&](int lr) -> int64_t {
            const int64_t tiles = ceil_div(rv1, int64_t(lr));
            const int64_t cr = TMMV_TMA_STAGE_V4 / lr;
            const int64_t O = int64_t(K) * std::min<int64_t>(lr, rv1);            // float4 outputs per tile
            const int64_t cap = std::max<int64_t>(1, std::min<int64_t>(tiles == 1 ? 1024 : 64 * std::max<int64_t>(1, NT / O),
                                                                     ceil_div(C, cr)));
            return pick_splits(tiles, slots, cap, 1);
        };
        bool one_split = false;
        if (par(ADAPTIC_P_LANES) <= 0 && rv1 <= 256) {
            LR = int(std::max<int64_t>(16, pow2_ceil(rv1)));      // one tile: contiguous stages
        } else if (par(ADAPTIC_P_LANES) <= 0 && xreq <= 0) {
            LR = 256;                                              // huge R: 4 KB row copies, no split
            one_split = true;
        } else if (par(ADAPTIC_P_LANES) <= 0) {
            // wave efficiency of each tile width; the widest within 5 % of the best (longer copies)
            double eff[5] = {0, 0, 0, 0, 0}, best_eff = 0.0;
            for (int i = 0, lr = 256; lr >= 16; lr >>= 1, ++i) {
                if (lr > std::max<int64_t>(16, pow2_ceil(rv1))) continue;
                const int64_t blocks = ceil_div(rv1, int64_t(lr)) * splits_for(lr);
                eff[i] = double(blocks) / double(ceil_div(blocks, slots) * slots);
                best_eff = std::max(best_eff, eff[i]);
            }
            LR = 16;
            for (int i = 0, lr = 256; lr >= 16; lr >>= 1, ++i)
                if (eff[i] > 0.0 && eff[i] >= best_eff - 0.05) { LR = lr; break; }
        }
        if (!tmmv_tma_fn(K, LR)) return ADAPTIC_ERR_INVALID_ARG;
        const int LC = NT / LR;
        p->xmode = 5;
        p->lanes = LR; p->unroll = 1; p->block = NT; p->ctas_per_sm = cps;
        const int64_t tiles = ceil_div(rv1, int64_t(LR));
        const int64_t cr = TMMV_TMA_STAGE_V4 / LR;
        int64_t S = par(ADAPTIC_P_SPLITS) > 0 ? par(ADAPTIC_P_SPLITS) : one_split ? 1 : splits_for(LR);
        const int64_t rows = ceil_div(ceil_div(C, S), int64_t(LC));
        p->chain[1] = std::min<int64_t>(rows, FOLD + cr / LC) + rows / FOLD;
        const int64_t Gm = std::max<int64_t>(1, NT / (int64_t(K) * std::min<int64_t>(LR, rv1)));
        p->depth[1] = ilog2c(LC) + (S > 1 ? ceil_div(S, Gm) + Gm : 0) + 1;
        p->path_ok[1] = bound_ok(p->chain[1] + p->depth[1]);
        p->grid[1] = std::max<int64_t>(1, std::min<int64_t>(tiles * S, slots));
        if (S > INT_MAX || !p->path_ok[1]) return ADAPTIC_ERR_UNSUPPORTED;
        p->splits = int(S);
        if (S > 1) {
            const size_t part = ((size_t(R) * size_t(K) * size_t(S) * 4 + 255) / 256) * 256;
            p->cnt_off = part;
            p->ws_bytes = part + size_t(tiles) * 4;
        }
        return ADAPTIC_OK;
    }
    int cps = par(ADAPTIC_P_CTAS_PER_SM);
    if (cps <= 0) cps = occupancy(tmmv_fn(K, LR, U, p->vec_shape), NT, 0, dev.present, 2048 / NT);
    p->lanes = LR; p->unroll = U; p->block = NT; p->ctas_per_sm = cps;
    const int LC = NT / LR;
    const int64_t slots = int64_t(dev.sms) * cps;
    int64_t S = 1;
    if (par(ADAPTIC_P_SPLITS) > 0) S = par(ADAPTIC_P_SPLITS);
    else if (v != ADAPTIC_V_TMV_COL) S = pick_splits_wave(ceil_div(rv1, LR), slots, std::max<int64_t>(1, ceil_div(C, int64_t(LC) * U)));
    for (;;) {
        bool ok_all = true;
        for (int w = 0; w < 2; ++w) {
            if (w == 1 && !p->vec_shape) continue;
            const int64_t rv = w ? R / 4 : R;
            const int64_t iters = ceil_div(ceil_div(C, S), int64_t(LC) * U);
            p->chain[w] = chain_of(iters, U);
            p->depth[w] = ilog2c(LC) + (S > 1 ? ceil_div(S, LC) + ilog2c(LC) : 0) + 1;
            p->path_ok[w] = bound_ok(p->chain[w] + p->depth[w]);
            p->grid[w] = std::max<int64_t>(1, std::min<int64_t>(ceil_div(rv, LR) * S, slots));
            if (!p->path_ok[w]) ok_all = false;
        }
        if (ok_all || S >= (int64_t(1) << 20)) break;
        S *= 2;
    }
    if (S > INT_MAX) return ADAPTIC_ERR_UNSUPPORTED;
    p->splits = int(S);
    if (!p->path_ok[p->vec_shape ? 1 : 0]) return ADAPTIC_ERR_UNSUPPORTED;
    if (S > 1) {
        const size_t part = ((size_t(R) * size_t(K) * size_t(S) * 4 + 255) / 256) * 256;
        p->cnt_off = part;
        p->ws_bytes = part + size_t(ceil_div(R, LR)) * 4;
    }
    return ADAPTIC_OK;
}

// BLAS-1 reductions (ASUM/NRM2/IAMAX/IAMIN): the MV-family thread shapes with an
// operator policy (blas1_kernels.cuh).  Only ASUM has fp32 chains to bound; NRM2
// accumulates in fp64 and IAMAX/IAMIN are exact.
adaptic_status derive_b1(adaptic_plan_s* p, const int32_t* params, const DevInfo& dev) {
    const int op = p->op, v = p->variant;
    const int64_t R = p->R, C = p->C;
    auto par = [&](int i) -> int { return params ? params[i] : 0; };
    const bool fp32_chain = (op == ADAPTIC_OP_ASUM || op == ADAPTIC_OP_B1ALL);
    // B1ALL keeps one accumulator per row (U loads per step feed it) and folds every FOLD/U steps
    const bool one_slot = (op == ADAPTIC_OP_B1ALL);
    auto chain_of = [&](int64_t iters, int U) -> int64_t {
        if (!one_slot) return fold_chain(iters);
        const int64_t f = FOLD / U;
        return int64_t(U) * std::min<int64_t>(iters, f) + iters / f;
    };
    const size_t part_bytes = (op == ADAPTIC_OP_B1ALL) ? 32 : 8;
    p->vec_shape = (C % 4 == 0);
    p->splits = 1; p->smem = 0; p->stages = 0; p->xmode = 0; p->ilv = 0; p->pipe = 0; p->rb = 1;
    p->fb_lanes = 0; p->fb_unroll = 0; p->ws_bytes = 0; p->cnt_off = 0;
    for (int w = 0; w < 2; ++w) { p->grid[w] = 0; p->chain[w] = 0; p->depth[w] = 0; p->path_ok[w] = false; }
    const int64_t nv1 = p->vec_shape ? C / 4 : C;

    if (v == ADAPTIC_V_MV_SUBWARP || v == ADAPTIC_V_MV_WPR) {
        // (RB, U): 4 rows x 2 loads (short rows) or 1 row x 8 loads (long rows)
        int rb = par(ADAPTIC_P_ROWS);
        if (rb <= 0) rb = (v == ADAPTIC_V_MV_WPR && nv1 >= 512) ? 1 : 4;
        if (rb != 1 && rb != 4) return ADAPTIC_ERR_INVALID_ARG;
        const int rbu = rb == 1 ? 1 : 0;
        if (op == ADAPTIC_OP_B1ALL && rb == 4) rb = 2;      // the fused op's multi-row instance: 2 rows x 4 loads
        const int U = rb == 1 ? 8 : (rb == 2 ? 4 : 2);
        // lanes per row: a row is one step of G x U loads (so the unrolled main loop runs)
        int G;
        if (v == ADAPTIC_V_MV_WPR) G = 32;
        else if (par(ADAPTIC_P_LANES) > 0) G = par(ADAPTIC_P_LANES);
        else G = clampi(pow2_ceil(ceil_div(std::max<int64_t>(1, nv1), U)), 1, 16);
        if (G < 1 || G > 32 || (G & (G - 1)) || (v == ADAPTIC_V_MV_SUBWARP && G > 16)) return ADAPTIC_ERR_INVALID_ARG;
        p->lanes = G; p->unroll = U; p->rb = rb; p->block = GROUP_NT;
        const int rows_per_cta = rb * (32 / G) * (GROUP_NT / 32);
        int cps = par(ADAPTIC_P_CTAS_PER_SM);
        if (cps <= 0) cps = occupancy(b1_group_fn(op, G, rbu, p->vec_shape), GROUP_NT, 0, dev.present, 4);
        p->ctas_per_sm = cps;
        for (int w = 0; w < 2; ++w) {
            if (w == 1 && !p->vec_shape) continue;
            const int64_t nv = w ? C / 4 : C;
            const int64_t iters = ceil_div(nv, int64_t(G) * U);
            p->grid[w] = std::max<int64_t>(1, std::min<int64_t>(ceil_div(R, rows_per_cta), int64_t(dev.sms) * cps));
            p->chain[w] = fp32_chain ? chain_of(iters, U) : 0;
            p->depth[w] = ilog2c(U) + (w ? 2 : 0) + ilog2c(G) + 1;
            p->path_ok[w] = !fp32_chain || bound_ok(p->chain[w] + p->depth[w]);
        }
        return p->path_ok[p->vec_shape ? 1 : 0] ? ADAPTIC_OK : ADAPTIC_ERR_UNSUPPORTED;
    }
    // MV_CPR / MV_SPLIT: B1_CTA_NT threads, 4 loads per thread per step
    const int NT = B1_CTA_NT, U = 4;
    int cps = par(ADAPTIC_P_CTAS_PER_SM);
    if (cps <= 0) cps = occupancy(b1_cta_fn(op, p->vec_shape), NT, 0, dev.present, 2048 / NT);
    p->lanes = NT; p->unroll = U; p->block = NT; p->ctas_per_sm = cps;
    const int64_t slots = int64_t(dev.sms) * cps;
    int64_t S = 1;
    if (v == ADAPTIC_V_MV_SPLIT) {
        S = par(ADAPTIC_P_SPLITS) > 0 ? par(ADAPTIC_P_SPLITS)
                                      : pick_splits(R, slots, std::max<int64_t>(2, ceil_div(nv1, int64_t(NT) * U)), 2);
    }
    for (;;) {
        bool ok_all = true;
        for (int w = 0; w < 2; ++w) {
            if (w == 1 && !p->vec_shape) continue;
            const int64_t nv = w ? C / 4 : C;
            const int64_t iters = ceil_div(nv, int64_t(S) * NT * U);   // interleaved splits
            p->chain[w] = fp32_chain ? chain_of(iters, U) : 0;
            p->depth[w] = ilog2c(U) + (w ? 2 : 0) + 10 + (S > 1 ? ceil_div(S, NT) + 10 : 0) + 1;
            p->path_ok[w] = !fp32_chain || bound_ok(p->chain[w] + p->depth[w]);
            p->grid[w] = std::max<int64_t>(1, std::min<int64_t>(R * S, slots));
            if (!p->path_ok[w]) ok_all = false;
        }
        if (ok_all || v == ADAPTIC_V_MV_CPR || S >= (int64_t(1) << 20)) break;
        S *= 2;
    }
    if (S > INT_MAX || R * S > (int64_t(1) << 40)) return ADAPTIC_ERR_UNSUPPORTED;
    p->splits = int(S);
    p->ilv = S > 1 ? 1 : 0;
    if (!p->path_ok[p->vec_shape ? 1 : 0]) return ADAPTIC_ERR_UNSUPPORTED;
    if (S > 1) {
        const size_t part = ((size_t(R) * size_t(S) * part_bytes + 255) / 256) * 256;
        p->cnt_off = part;
        p->ws_bytes = part + size_t(R) * 4;
    }
    return ADAPTIC_OK;
}

adaptic_status derive(adaptic_plan_s* p, const int32_t* params, const DevInfo& dev);

// xmode 3: the four shifted copies of x (pitch round_up(C, 4)) after the plan's own workspace
void add_xshift_workspace(adaptic_plan_s* p) {
    p->xsh_off = (p->ws_bytes + 255) / 256 * 256;
    p->ws_bytes = p->xsh_off + size_t(4) * size_t((p->C + 3) / 4 * 4) * 4;
}

// MV / DOT lane groups on TMA-staged row tiles (rowtile_kernel.cuh): MV_SUBWARP / MV_WPR
// with [ADAPTIC_P_XSMEM] = 4.  [LANES] G (WPR: 32), [BLOCK] threads 256 | 512, [ROWS]
// rows per tile k, [UNROLL] ring stages, [CTAS_PER_SM] resident CTAs the ring is sized
// for.  Needs C <= 32*G (x slice in registers); 16-byte-aligned A (and b) at run time,
// else adaptic_run takes the same variant's direct kernel.
adaptic_status derive_rowtile(adaptic_plan_s* p, const int32_t* params, const DevInfo& dev) {
    auto par = [&](int i) -> int { return params ? params[i] : 0; };
    const bool px = (p->op == ADAPTIC_OP_DOT);
    const int64_t R = p->R, C = p->C;
    int G = p->variant == ADAPTIC_V_MV_WPR ? 32 : par(ADAPTIC_P_LANES);
    if (G <= 0) G = clampi(pow2_ceil(ceil_div(C, 8)), 1, 16);
    if (G < 1 || G > 32 || (G & (G - 1)) || (p->variant == ADAPTIC_V_MV_SUBWARP && G > 16))
        return ADAPTIC_ERR_INVALID_ARG;
    // a fitted cell spans a factor 2 in C: an entry's lane group fitted on the cell's shorter
    // rows may hold too few x values per lane for this C -- the smallest group that does
    // (held-out DOT 393216 x 416 and 507478 x 488 had fallen back to the direct kernels: 0.67-0.89
    // of the staged plan)
    if (p->source == 1 && C > int64_t(RT_MAX_C_PER_LANE) * G && p->variant == ADAPTIC_V_MV_SUBWARP)
        G = int(std::min<int64_t>(16, pow2_ceil(ceil_div(C, int64_t(RT_MAX_C_PER_LANE)))));
    if (C > int64_t(RT_MAX_C_PER_LANE) * G) return ADAPTIC_ERR_UNSUPPORTED;
    int NT = par(ADAPTIC_P_BLOCK);
    if (NT <= 0) NT = 256;
    if (NT != 256 && NT != 512) return ADAPTIC_ERR_INVALID_ARG;
    const int ngr = NT / G;
    const int64_t opb = int64_t(px ? 2 : 1) * 4;             // staged bytes per element
    int64_t k = par(ADAPTIC_P_ROWS);
    if (k < 0) {           // -n: the rows of ~n KB (fitted tables store a size; the sweep's height)
        k = std::max<int64_t>(1, (int64_t(-k) * 1024) / (C * opb));
    } else if (k == 0) {   // ~24 KB of matrix per tile, whole warps of rows
        k = std::max<int64_t>(1, (24 * 1024) / (C * opb));
        if (k >= ngr) k = k / ngr * ngr;
    }
    // a fitted (-n KB, table) or default tile below ~40 KB, when the matrix still gives every SM two
    // such tiles: the 40 KB height.  Each staged tile costs a fixed hand-off, and over the 33
    // training shapes >= 256 MiB with both kinds swept the best < 20 KB tile ran a median 0.75
    // (MV) / 0.71 (DOT) of the best >= 36 KB one, 20-36 KB tiles 0.92 / 0.93 (never faster in 32)
    if (par(ADAPTIC_P_ROWS) == 0 || (par(ADAPTIC_P_ROWS) < 0 && p->source != 0)) {   // not a forced size
        const int64_t kf = ceil_div(int64_t(40) * 1024, C * opb);
        if (k < kf && ceil_div(R, kf) >= 2 * int64_t(dev.sms)) k = kf;
    }
    k = std::min<int64_t>(k, std::max<int64_t>(1, R));
    int cps = par(ADAPTIC_P_CTAS_PER_SM);
    if (cps <= 0) cps = 2;
    // a tile height fitted on a shorter row (table cells span a factor of 2 in C) is
    // capped so that two stages still fit the ring budget
    const int64_t kmax2 = ((int64_t(220) * 1024 / cps / 2) / (4 * (px ? 2 : 1)) - 9) / C;
    if (kmax2 < 1) return ADAPTIC_ERR_UNSUPPORTED;
    k = std::min(k, kmax2);
    const size_t stage_bytes = rowtile_tile_words(k, C) * 4 * (px ? 2 : 1);
    if (stage_bytes > 200 * 1024) return ADAPTIC_ERR_UNSUPPORTED;
    int stages = int(std::min<size_t>(RT_MAX_STAGES_H, (size_t(220) * 1024 / size_t(cps)) / stage_bytes));
    if (par(ADAPTIC_P_UNROLL) > 0) stages = std::min(stages, par(ADAPTIC_P_UNROLL));
    void* fn = rowtile_fn(p->dtype, NT, G, px);
    if (!fn) return ADAPTIC_ERR_UNSUPPORTED;
    while (stages >= 2 && !smem_fits(fn, size_t(stages) * stage_bytes, dev.present)) --stages;   // + static smem
    if (stages < 2) return ADAPTIC_ERR_UNSUPPORTED;
    p->smem = size_t(stages) * stage_bytes;
    const int occ = occupancy(fn, NT, p->smem, dev.present, cps);
    if (occ < 1) return ADAPTIC_ERR_UNSUPPORTED;
    p->ctas_per_sm = std::min(cps, occ);
    p->lanes = G; p->block = NT; p->rb = int(k); p->stages = stages; p->unroll = stages;
    p->xmode = 4;
    p->mis = !p->vec_shape;
    const int64_t ntiles = ceil_div(R, k);
    p->grid[1] = std::max<int64_t>(1, std::min<int64_t>(ntiles, int64_t(dev.sms) * p->ctas_per_sm));
    p->chain[1] = ceil_div(ceil_div(C, G), 2);
    p->depth[1] = ilog2c(G) + 1;
    p->path_ok[1] = (p->dtype == DT_I32) || bound_ok(p->chain[1] + p->depth[1]);
    if (!p->path_ok[1]) return ADAPTIC_ERR_UNSUPPORTED;
    return ADAPTIC_OK;
}

// MV on TMA-staged tiles of k <= RTC_KMAX_H long rows, each tile reduced by the whole CTA with x
// staged once in shared memory (rowtile_kernel.cuh mv_rowtile_cta_kernel): MV_CPR with
// [ADAPTIC_P_XSMEM] = 11.  [BLOCK] 256 | 512, [ROWS] k (-n: ~n KB per tile), [UNROLL] ring
// stages, [CTAS_PER_SM]; C <= 36 * NT (x in registers; describe()'s lanes = x values per
// thread).  16-byte-aligned A at run time, else the variant's direct kernel.
adaptic_status derive_rowtile_cta_staged(adaptic_plan_s* p, const int32_t* params, const DevInfo& dev) {
    auto par = [&](int i) -> int { return params ? params[i] : 0; };
    const int64_t R = p->R, C = p->C;
    int NT = par(ADAPTIC_P_BLOCK);
    if (NT <= 0) NT = C <= 256 * 36 ? 256 : 512;
    if (NT != 256 && NT != 512) return ADAPTIC_ERR_INVALID_ARG;
    const int64_t mx_need = ceil_div(C, int64_t(NT));
    const int MX = mx_need <= 4 ? 4 : mx_need <= 8 ? 8 : mx_need <= 16 ? 16 : mx_need <= 36 ? 36 : 0;
    if (MX == 0) return ADAPTIC_ERR_UNSUPPORTED;              // x must fit the registers
    int cps = par(ADAPTIC_P_CTAS_PER_SM);
    if (cps <= 0) cps = C <= 4096 ? 2 : 1;
    const size_t budget = size_t(220) * 1024 / size_t(cps);
    const size_t xbytes = 0;
    if (xbytes + 2 * rowtile_tile_words(1, C) * 4 > budget) return ADAPTIC_ERR_UNSUPPORTED;
    int64_t k = par(ADAPTIC_P_ROWS);
    if (k < 0) k = (int64_t(-k) * 1024) / (C * 4);
    else if (k == 0) k = (int64_t(32) * 1024) / (C * 4);
    k = std::max<int64_t>(1, std::min<int64_t>({k, int64_t(RTC_KMAX_H), std::max<int64_t>(1, R)}));
    while (k > 1 && xbytes + 2 * rowtile_tile_words(k, C) * 4 > budget) --k;
    const size_t stage_bytes = rowtile_tile_words(k, C) * 4;
    int stages = int(std::min<size_t>(RT_MAX_STAGES_H, (budget - xbytes) / stage_bytes));
    if (par(ADAPTIC_P_UNROLL) > 0) stages = std::min(stages, par(ADAPTIC_P_UNROLL));
    void* fn = rowtile_cta_fn(p->dtype, NT, MX, int(k));
    if (!fn) return ADAPTIC_ERR_UNSUPPORTED;
    while (stages >= 2 && !smem_fits(fn, size_t(stages) * stage_bytes + xbytes, dev.present)) --stages;
    if (stages < 2) return ADAPTIC_ERR_UNSUPPORTED;
    p->smem = size_t(stages) * stage_bytes + xbytes;
    const int occ = occupancy(fn, NT, p->smem, dev.present, cps);
    if (occ < 1) return ADAPTIC_ERR_UNSUPPORTED;
    p->ctas_per_sm = std::min(cps, occ);
    p->lanes = MX; p->block = NT; p->rb = int(k); p->stages = stages; p->unroll = stages;
    p->xmode = 11;
    p->mis = !p->vec_shape;
    p->grid[1] = std::max<int64_t>(1, std::min<int64_t>(ceil_div(R, k), int64_t(dev.sms) * p->ctas_per_sm));
    p->chain[1] = mx_need;
    p->depth[1] = 5 + NT / 64 + 1;                      // butterfly, two chains over the warps, their sum
    p->path_ok[1] = (p->dtype == DT_I32) || bound_ok(p->chain[1] + p->depth[1]);
    if (!p->path_ok[1]) return ADAPTIC_ERR_UNSUPPORTED;
    p->ws_bytes = 0;
    adaptic_plan_s fb = *p;                             // the direct kernel for unaligned A
    p->fb_ws_off = 0;
    if (derive(&fb, nullptr, dev) == ADAPTIC_OK) p->ws_bytes = fb.ws_bytes;
    return ADAPTIC_OK;
}

// Rows too long for whole-row tiles (x in registers: C <= 36 * NT; two stages in the ring): the
// direct CTA-per-row kernel with 256 lanes x 2 vectors in flight and shifted copies of x
// (XSMEM 5), the best fixed plan measured on the held-out long misaligned rows (8460 x 20903
// 0.96, 8348 x 29273 0.98 of peak; the planner's default 1024-lane CTA ran 0.38-0.47 there).
// So a fitted XSMEM 11 entry is valid for every shape of its cell.
adaptic_status derive_rowtile_cta(adaptic_plan_s* p, const int32_t* params, const DevInfo& dev) {
    const adaptic_status st = derive_rowtile_cta_staged(p, params, dev);
    if (st != ADAPTIC_ERR_UNSUPPORTED) return st;
    int32_t tp[ADAPTIC_NPARAMS] = {0};
    tp[ADAPTIC_P_LANES] = 256;
    tp[ADAPTIC_P_UNROLL] = 2;
    tp[ADAPTIC_P_XSMEM] = 5;
    if (derive(p, tp, dev) == ADAPTIC_OK) return ADAPTIC_OK;
    tp[ADAPTIC_P_XSMEM] = 0;
    return derive(p, tp, dev);
}

// MV rows too long for x in registers on staged COLUMN CHUNKS (rowtile_kernel.cuh
// mv_chunk_cta_kernel): MV_CPR / MV_SPLIT with [ADAPTIC_P_XSMEM] = 13, any C and any row
// alignment.  [BLOCK] 256 | 512 (default 512), [LANES] x values per thread MX in {8, 16, 36}
// (default 16; chunk width W = ceil(C / nch) <= NT MX, nch chunks), [ROWS] rows per tile k
// (0: ~64 KB of segments per tile, -n: ~n KB; <= 4), [UNROLL] ring stages, [CTAS_PER_SM]
// (default 1).  describe(): splits = nch, rows_per_group = k, lanes = MX.  16-byte-aligned A
// at run time, else the variant's direct kernel.
adaptic_status derive_chunk_cta(adaptic_plan_s* p, const int32_t* params, const DevInfo& dev) {
    auto par = [&](int i) -> int { return params ? params[i] : 0; };
    const int64_t R = p->R, C = p->C;
    int NT = par(ADAPTIC_P_BLOCK);
    if (NT <= 0) NT = 512;
    if (NT != 256 && NT != 512) return ADAPTIC_ERR_INVALID_ARG;
    int MX = par(ADAPTIC_P_LANES);
    if (MX <= 0) MX = 16;
    if (MX != 8 && MX != 16 && MX != 36) return ADAPTIC_ERR_INVALID_ARG;
    const int64_t nch = ceil_div(C, int64_t(NT) * MX);
    const int64_t W = ceil_div(C, nch);
    if (W > INT_MAX / 2) return ADAPTIC_ERR_UNSUPPORTED;
    int cps = par(ADAPTIC_P_CTAS_PER_SM);
    if (cps <= 0) cps = 1;
    const size_t budget = size_t(220) * 1024 / size_t(cps);
    const size_t slot_bytes = size_t((W + 6 + 3) / 4 * 4) * 4;
    int64_t k = par(ADAPTIC_P_ROWS);
    if (k < 0) k = (int64_t(-k) * 1024) / int64_t(slot_bytes);
    else if (k == 0) k = (int64_t(64) * 1024) / int64_t(slot_bytes);   // 32 KB tiles: 0.87 vs 0.91 (r2g)
    k = std::max<int64_t>(1, std::min<int64_t>({k, int64_t(4), std::max<int64_t>(1, R)}));
    while (k > 1 && 2 * size_t(k) * slot_bytes > budget) --k;
    const size_t stage_bytes = size_t(k) * slot_bytes;
    if (2 * stage_bytes > budget) return ADAPTIC_ERR_UNSUPPORTED;
    int stages = int(std::min<size_t>(RT_MAX_STAGES_H, budget / stage_bytes));
    if (par(ADAPTIC_P_UNROLL) > 0) stages = std::min(stages, par(ADAPTIC_P_UNROLL));
    void* fn = chunk_cta_fn(p->dtype, NT, MX, int(k));
    if (!fn) return ADAPTIC_ERR_UNSUPPORTED;
    while (stages >= 2 && !smem_fits(fn, size_t(stages) * stage_bytes, dev.present)) --stages;
    if (stages < 2) return ADAPTIC_ERR_UNSUPPORTED;
    p->smem = size_t(stages) * stage_bytes;
    const int occ = occupancy(fn, NT + 32, p->smem, dev.present, cps);
    if (occ < 1) return ADAPTIC_ERR_UNSUPPORTED;
    p->ctas_per_sm = std::min(cps, occ);
    const int64_t units = nch * ceil_div(R, k);
    p->lanes = MX; p->block = NT; p->rb = int(k); p->stages = stages; p->unroll = stages;
    p->splits = int(nch);
    p->xmode = 13;
    p->mis = !p->vec_shape;
    p->grid[1] = std::max<int64_t>(1, std::min<int64_t>(units, int64_t(dev.sms) * p->ctas_per_sm));
    p->grid[0] = p->grid[1];
    int L = 1;
    while (L < 32 && 2 * L * R <= NT) L *= 2;
    p->chain[1] = MX;
    p->depth[1] = 5 + NT / 64 + 1 + (nch > 1 ? ceil_div(nch, L) + ilog2c(L) : 0);
    p->chain[0] = p->chain[1]; p->depth[0] = p->depth[1];
    p->path_ok[1] = (p->dtype == DT_I32) || bound_ok(p->chain[1] + p->depth[1]);
    p->path_ok[0] = p->path_ok[1];
    if (!p->path_ok[1]) return ADAPTIC_ERR_UNSUPPORTED;
    p->ws_bytes = 0;
    if (nch > 1) {
        p->cnt_off = ((size_t(nch) * size_t(R) * 4 + 255) / 256) * 256;
        p->ws_bytes = p->cnt_off + 256;
    }
    adaptic_plan_s fb = *p;                             // the direct kernel for unaligned A
    p->fb_ws_off = p->ws_bytes;
    if (derive(&fb, nullptr, dev) == ADAPTIC_OK) p->ws_bytes += fb.ws_bytes;
    return ADAPTIC_OK;
}

// TMV with few outputs on TMA-staged tiles of B (tmv_rowtile_kernel.cuh): TMV_REGTILE with
// [ADAPTIC_P_XSMEM] = 4.  [BLOCK] threads 256 | 512 | 1024 (>= R), [ROWS] rows of B per
// tile k (a multiple of 4), [UNROLL] ring stages, [CTAS_PER_SM].  16-byte-aligned B and x
// at run time, else adaptic_run takes the variant's direct kernel.
adaptic_status derive_tmv_rowtile(adaptic_plan_s* p, const int32_t* params, const DevInfo& dev) {
    auto par = [&](int i) -> int { return params ? params[i] : 0; };
    const int64_t R = p->R, C = p->C;
    if (R > 4096) return ADAPTIC_ERR_UNSUPPORTED;
    int NT = par(ADAPTIC_P_BLOCK);
    if (NT <= 0) NT = R <= 64 ? 256 : R <= 1024 ? 1024 : 1024;
    if (NT != 256 && NT != 512 && NT != 1024 && !(NT == 544 && R <= 2 * 544)) return ADAPTIC_ERR_INVALID_ARG;
    const int rpt = R <= NT ? 1 : R <= 2 * NT ? 2 : R <= 4 * NT ? 4 : 0;   // outputs per thread
    if (rpt == 0 || !tmv_rowtile_fn(p->dtype, NT, rpt)) return ADAPTIC_ERR_INVALID_ARG;
    int cps = par(ADAPTIC_P_CTAS_PER_SM);
    // 17-warp CTAs: one per SM up to R = 256, two above (544 threads, 513 x 131072: 0.80 -> 0.85
    // back to back; below 256 the single CTA was 1-2 % ahead, profiles/r2_exp/r2m_tmv544_cmp.jsonl)
    if (cps <= 0) cps = NT == 544 ? (R > 256 ? 2 : 1) : 1024 / NT;
    int64_t k = par(ADAPTIC_P_ROWS);
    if (k < 0) {                        // -n: ~n KB of B and x per tile (fitted tables)
        k = std::max<int64_t>(4, (int64_t(-k) * 1024 / 4) / (R + 1) / 4 * 4);
    } else if (k == 0) {                // ~40 KB of B per tile, and at least 3 stages in the budget
        // (24 KB before: over the 32 training shapes >= 256 MiB with both swept, 20-36 KB tiles ran a
        // median 0.97 of the best >= 36 KB tile)
        const int64_t words = std::min<int64_t>(40 * 1024, (int64_t(220) * 1024 / cps) / 3) / 4 - 9;
        k = std::max<int64_t>(4, words / (R + 1) / 4 * 4);
    }
    if (k % 4 != 0) return ADAPTIC_ERR_INVALID_ARG;
    k = std::min<int64_t>(k, ceil_div(C, 4) * 4);
    // cap a tile height fitted on fewer outputs so that two stages fit the ring budget
    const int64_t kmax2 = (((int64_t(220) * 1024 / cps / 2) / 4 - 9) / (R + 1)) / 4 * 4;
    if (kmax2 < 4) return ADAPTIC_ERR_UNSUPPORTED;
    k = std::min(k, kmax2);
    const size_t stage_bytes = (rowtile_tile_words(k, R) + size_t(k)) * 4;
    if (stage_bytes > 200 * 1024) return ADAPTIC_ERR_UNSUPPORTED;
    int stages = int(std::min<size_t>(RT_MAX_STAGES_H, (size_t(220) * 1024 / size_t(cps)) / stage_bytes));
    if (par(ADAPTIC_P_UNROLL) > 0) stages = std::min(stages, par(ADAPTIC_P_UNROLL));
    void* fn = tmv_rowtile_fn(p->dtype, NT, rpt);
    while (stages >= 2 && !smem_fits(fn, size_t(stages) * stage_bytes, dev.present)) --stages;   // + static smem
    if (stages < 2) return ADAPTIC_ERR_UNSUPPORTED;
    p->smem = size_t(stages) * stage_bytes;
    const int occ = occupancy(fn, NT, p->smem, dev.present, cps);
    if (occ < 1) return ADAPTIC_ERR_UNSUPPORTED;
    p->ctas_per_sm = std::min(cps, occ);
    const int64_t ntiles = ceil_div(C, k);
    const int64_t G = std::max<int64_t>(1, std::min<int64_t>(ntiles, int64_t(dev.sms) * p->ctas_per_sm));
    const int64_t nsl = int64_t(NT) * rpt / R;
    p->lanes = int(R); p->block = NT; p->rb = int(k); p->stages = stages; p->unroll = rpt;
    p->xmode = 4; p->splits = 1; p->mis = !p->vec_shape;
    p->grid[1] = G;
    const int64_t rows_per_thread = ceil_div(ceil_div(ntiles, G) * k, nsl);
    p->chain[1] = fold_chain(ceil_div(rows_per_thread, 4)) + 1;
    const int64_t ngroups = ceil_div(G, 16);                  // TRT_GROUP CTAs per merge group
    p->depth[1] = 3 + 2 * nsl + ceil_div(16, nsl) + ceil_div(ngroups, nsl);
    p->path_ok[1] = (p->dtype == DT_I32) || bound_ok(p->chain[1] + p->depth[1]);
    if (!p->path_ok[1]) return ADAPTIC_ERR_UNSUPPORTED;
    // CTA partials (G x R), group partials (ngroups x R), then 1 + ngroups counters
    const size_t part = ((size_t(G + ngroups) * size_t(R) * 4 + 255) / 256) * 256;
    p->cnt_off = part;
    p->ws_bytes = part + ((size_t(1 + ngroups) * 4 + 255) / 256) * 256;
    // pointers the bulk copies cannot use run the variant's direct kernel on its own
    // (disjoint, hence still zeroed) part of this workspace
    adaptic_plan_s fb = *p;
    p->fb_ws_off = p->ws_bytes;
    if (derive(&fb, nullptr, dev) == ADAPTIC_OK) p->ws_bytes += fb.ws_bytes;
    return ADAPTIC_OK;
}

// TMV with rows off the 16-byte grid on groups of four rows (tmv_group_kernel.cuh):
// TMV_REGTILE / TMV_SPLITK with [ADAPTIC_P_XSMEM] = 12, 4 <= R <= 2560.  [UNROLL] groups in
// flight (R <= 1024: 4 or 8), [BLOCK] threads (0: the fewest idle slots), [CTAS_PER_SM],
// [ORDER] 1 = contiguous group range per CTA (default), 2 = CTAs interleaved,
// [ROWS] slots per thread S (0: S = 1 for R <= 1024 (KG = NT div R groups per CTA step), else the
// smallest S in {2, 3, 4} with ceil(R / S) <= 640).  16-byte-aligned B at run time, else the
// variant's direct kernel on its own slice of the workspace.
adaptic_status derive_tmv_group(adaptic_plan_s* p, const int32_t* params, const DevInfo& dev) {
    auto par = [&](int i) -> int { return params ? params[i] : 0; };
    const int64_t R = p->R, C = p->C;
    if (R < 4 || R > 2560) return ADAPTIC_ERR_UNSUPPORTED;
    int S = par(ADAPTIC_P_ROWS);
    if (S <= 0) { S = 1; if (R > 1024) { S = 2; while (S < 4 && ceil_div(R, S) > 640) ++S; } }
    if (S > 4) return ADAPTIC_ERR_INVALID_ARG;
    int U = par(ADAPTIC_P_UNROLL);
    if (U <= 0) U = S == 1 ? 4 : S == 2 ? 4 : 2;
    void* fn = tmv_group_fn(p->dtype, S, U);
    if (!fn) return ADAPTIC_ERR_INVALID_ARG;
    const int maxnt = tmv_group_maxnt(S, U);
    int NT = par(ADAPTIC_P_BLOCK);
    int KG = 1;
    if (S == 1) {
        if (R > maxnt) return ADAPTIC_ERR_UNSUPPORTED;
        if (NT <= 0) {                  // the block size (multiple of 32) with the fewest idle threads
            double best = -1.0;
            for (int nt = 256; nt <= maxnt; nt += 32) {
                if (nt < R) continue;
                const int kg = nt / int(R);
                const double use = double(kg * R) / double(nt);
                if (use > best + 0.02) { best = use; NT = nt; }
            }
            if (NT <= 0) NT = int(ceil_div(R, 32) * 32);
        }
        if (NT < R || NT > maxnt) return ADAPTIC_ERR_INVALID_ARG;
        KG = NT / int(R);
    } else {
        const int need = int(ceil_div(ceil_div(R, S), 32) * 32);
        if (NT <= 0) NT = need;
        if (NT < ceil_div(R, S) || NT > maxnt) return ADAPTIC_ERR_INVALID_ARG;
    }
    int cps = par(ADAPTIC_P_CTAS_PER_SM);
    const int occ = occupancy(fn, NT, 0, dev.present, std::max(1, 1024 / NT));
    if (occ < 1) return ADAPTIC_ERR_UNSUPPORTED;
    cps = cps <= 0 ? occ : std::min(cps, occ);
    const int64_t NG = C / 4;
    const int64_t G = std::max<int64_t>(1, std::min<int64_t>(int64_t(dev.sms) * cps, ceil_div(NG, int64_t(KG) * U)));
    const int64_t ngroups = ceil_div(G, TG_GROUP_H);
    const int ord = par(ADAPTIC_P_ORDER);
    if (ord < 0 || ord > 2) return ADAPTIC_ERR_INVALID_ARG;
    p->ilv = ord == 2 ? 1 : 0;
    p->xmode = 12; p->mis = true; p->splits = 1;
    p->lanes = int(R); p->block = NT; p->rb = S; p->unroll = U; p->ctas_per_sm = cps;
    p->grid[1] = G; p->grid[0] = G;
    p->chain[1] = fold_chain(ceil_div(ceil_div(NG, G), KG)) + 1;
    p->depth[1] = 4 * KG + TG_GROUP_H + ngroups + (C % 4) + 1;
    p->chain[0] = p->chain[1]; p->depth[0] = p->depth[1];
    p->path_ok[1] = (p->dtype == DT_I32) || bound_ok(p->chain[1] + p->depth[1]);
    p->path_ok[0] = p->path_ok[1];
    if (!p->path_ok[1]) return ADAPTIC_ERR_UNSUPPORTED;
    // CTA partials (G x R), group partials (ngroups x R), then 1 + ngroups counters
    const size_t part = ((size_t(G + ngroups) * size_t(R) * 4 + 255) / 256) * 256;
    p->cnt_off = part;
    p->ws_bytes = part + ((size_t(1 + ngroups) * 4 + 255) / 256) * 256;
    adaptic_plan_s fb = *p;                     // B not 16-byte aligned: the direct kernel
    fb.variant = ADAPTIC_V_TMV_SPLITK;
    p->fb_ws_off = p->ws_bytes;
    if (derive(&fb, nullptr, dev) == ADAPTIC_OK) p->ws_bytes += fb.ws_bytes;
    return ADAPTIC_OK;
}

// A multi-vector plan with a 128-bit shape run on pointers that are not 16-byte aligned
// (the x-tile / TMA / register-x kernels need aligned rows): the generic CTA kernels'
// 4-byte path of the same K -- MV_CPR (no workspace) when its error bound holds, else
// MV_SPLIT; TMV: the register-fed SPLITK tiles.  Only 4-byte misalignment is an error (8(b)).
bool multi_fallback(const adaptic_plan_s& p, adaptic_plan_s* fb, const DevInfo& dev) {
    int32_t prm[ADAPTIC_NPARAMS] = {0};
    prm[ADAPTIC_P_XSMEM] = 1;                    // x through L1 (MV), register-fed tiles (TMV)
    const int mv_cands[2] = {ADAPTIC_V_MV_CPR, ADAPTIC_V_MV_SPLIT};
    const int tmv_cands[1] = {ADAPTIC_V_TMV_SPLITK};
    const int* cands = p.op == ADAPTIC_OP_TMV ? tmv_cands : mv_cands;
    const int n = p.op == ADAPTIC_OP_TMV ? 1 : 2;
    for (int i = 0; i < n; ++i) {
        *fb = p;
        fb->variant = cands[i]; fb->ws = nullptr; fb->ws_cap = 0; fb->multi_fb_ok = false;
        if (derive_multi(fb, prm, dev) == ADAPTIC_OK && fb->path_ok[0]) return true;
    }
    return false;
}

// Fill the kernel parameters of `p` for p->variant.  params: user overrides or nullptr.
adaptic_status derive(adaptic_plan_s* p, const int32_t* params, const DevInfo& dev) {
    const int op = p->op, dt = p->dtype;
    const bool px = (op == ADAPTIC_OP_DOT);
    const int64_t R = p->R, C = p->C;
    auto par = [&](int i) -> int { return params ? params[i] : 0; };
    const int v = p->variant;
    if (!op_has_variant(op, v)) return ADAPTIC_ERR_UNSUPPORTED;
    if (p->nvec > 1) {
        p->multi_fb_ok = false;
        const adaptic_status st = derive_multi(p, params, dev);
        if (st == ADAPTIC_OK && p->vec_shape) {
            adaptic_plan_s fb;
            if (multi_fallback(*p, &fb, dev)) {
                p->multi_fb_ok = true;
                p->fb_ws_off = ((p->ws_bytes + 255) / 256) * 256;
                if (fb.ws_bytes > 0) p->ws_bytes = p->fb_ws_off + fb.ws_bytes;
            }
        }
        return st;
    }
    // single-vector MV (fp32 or int32) on the x-tile stream-K kernel (param XSMEM 3)
    if (op == ADAPTIC_OP_MV && (v == ADAPTIC_V_MV_CPR || v == ADAPTIC_V_MV_SPLIT) &&
        (par(ADAPTIC_P_XSMEM) == 3 || par(ADAPTIC_P_XSMEM) == 6) && C % 4 == 0)
        return derive_multi(p, params, dev);
    if (op == ADAPTIC_OP_TMV && par(ADAPTIC_P_XSMEM) == 6) return derive_tmv_ring(p, params, dev);
    if (op == ADAPTIC_OP_STENCIL5) return derive_stencil(p, params, dev);
    if (is_b1_op(op)) return derive_b1(p, params, dev);

    p->vec_shape = (op == ADAPTIC_OP_TMV) ? (R % 4 == 0) : (C % 4 == 0);
    p->mis = false;
    p->splits = 1;
    p->smem = 0;
    p->stages = 0;
    p->xmode = px ? 2 : 0;
    p->ilv = 0;
    p->pipe = 0;
    p->rb = 1;
    p->fb_lanes = 0;
    p->fb_unroll = 0;
    p->ws_bytes = 0;
    p->cnt_off = 0;

    for (int w = 0; w < 2; ++w) { p->grid[w] = 0; p->chain[w] = 0; p->depth[w] = 0; p->path_ok[w] = false; }
    if ((v == ADAPTIC_V_MV_SUBWARP || v == ADAPTIC_V_MV_WPR) && par(ADAPTIC_P_XSMEM) == 4)
        return derive_rowtile(p, params, dev);
    if (v == ADAPTIC_V_MV_CPR && op == ADAPTIC_OP_MV && par(ADAPTIC_P_XSMEM) == 11)
        return derive_rowtile_cta(p, params, dev);
    if ((v == ADAPTIC_V_MV_CPR || v == ADAPTIC_V_MV_SPLIT) && op == ADAPTIC_OP_MV && par(ADAPTIC_P_XSMEM) == 13)
        return derive_chunk_cta(p, params, dev);

    // rows not 16-byte aligned (C % 4 != 0): the misaligned-row kernels keep the matrix
    // stream 128-bit; the plain scalar kernels (index 0) remain for DOT operands whose
    // addresses differ modulo 16
    const bool mis = !p->vec_shape && op != ADAPTIC_OP_TMV && v != ADAPTIC_V_MV_TPR && C >= kMisMinCols;
    if (v == ADAPTIC_V_MV_SUBWARP || v == ADAPTIC_V_MV_WPR || v == ADAPTIC_V_MV_TPR) {
        // group-kernel parameters (also the TPR scalar fallback)
        // TPR's fallback is the scalar group kernel, so size it for the scalar path
        const int64_t nvv = ((p->vec_shape || mis) && v != ADAPTIC_V_MV_TPR) ? C / 4 : C;
        int G;
        if (v == ADAPTIC_V_MV_WPR) G = 32;
        else if (v == ADAPTIC_V_MV_SUBWARP && par(ADAPTIC_P_LANES) > 0) G = par(ADAPTIC_P_LANES);
        else G = clampi(pow2_ceil(std::max<int64_t>(1, nvv)), 1, v == ADAPTIC_V_MV_TPR ? 32 : 16);
        if (G < 1 || G > 32 || (G & (G - 1)) || (v == ADAPTIC_V_MV_SUBWARP && G > 16)) return ADAPTIC_ERR_INVALID_ARG;
        int U = par(ADAPTIC_P_UNROLL);
        if (U <= 0) U = clampi(pow2_ceil(ceil_div(std::max<int64_t>(1, nvv), G)), 1, 8);
        if (U != 1 && U != 2 && U != 4 && U != 8) return ADAPTIC_ERR_INVALID_ARG;
        if (v == ADAPTIC_V_MV_TPR) { p->fb_lanes = G; p->fb_unroll = U; }
        else { p->lanes = G; p->unroll = U; p->rb = 8 / U; p->block = GROUP_NT; }
        const int rows_per_cta = (8 / U) * (32 / G) * (GROUP_NT / 32);
        const bool want_shift = v != ADAPTIC_V_MV_TPR && par(ADAPTIC_P_XSMEM) == 5;
        if (want_shift && (px || !mis)) return ADAPTIC_ERR_UNSUPPORTED;   // shifted x: misaligned MV rows only
        const int xm = (v == ADAPTIC_V_MV_TPR) ? (px ? 2 : 0)
                       : want_shift ? XM_SHIFT_MODE : pick_xmode(px, par(ADAPTIC_P_XSMEM), C, true);
        if (xm < 0) return ADAPTIC_ERR_UNSUPPORTED;
        const size_t xsm = xm == 1 ? size_t((C * 4 + 15) / 16 * 16) : 0;
        int cps = par(ADAPTIC_P_CTAS_PER_SM);
        if (cps <= 0) cps = occupancy(mis ? mis_group_fn(dt, G, U, xm) : group_fn(dt, G, U, p->vec_shape, xm),
                                      GROUP_NT, xsm, dev.present, 4);
        if (v != ADAPTIC_V_MV_TPR) { p->ctas_per_sm = cps; p->xmode = xm; p->smem = xsm; p->mis = mis; }
        const int rows_per_cta_mis = std::max(1, 4 / U) * (32 / G) * (GROUP_NT / 32);
        for (int w = 0; w < 2; ++w) {
            const int64_t nv = w ? C / 4 : C;
            if (w == 1 && !p->vec_shape && !mis) continue;
            const bool wm = (w == 1 && mis);
            const int64_t iters = ceil_div(nv, int64_t(G) * U);
            p->grid[w] = std::max<int64_t>(1, std::min<int64_t>(ceil_div(R, wm ? rows_per_cta_mis : rows_per_cta),
                                                                int64_t(dev.sms) * cps));
            p->chain[w] = fold_chain(iters);
            p->depth[w] = ilog2c(U) + (w ? 2 : 0) + ilog2c(G) + 1 + (wm ? 1 : 0);   // + head/tail term
            p->path_ok[w] = (dt == DT_I32) || bound_ok(p->chain[w] + p->depth[w]);
        }
        if (v != ADAPTIC_V_MV_TPR) {
            if (!p->path_ok[(p->vec_shape || mis) ? 1 : 0]) return ADAPTIC_ERR_UNSUPPORTED;
            if (xm == XM_SHIFT_MODE) add_xshift_workspace(p);
            return ADAPTIC_OK;
        }
        // ---- MV_TPR proper: index 1 = the TMA-staged kernel (128-bit shared reads, or 32-bit
        // ones for C % 4 != 0 -- then p->mis marks it); index 0 = the group fallback above
        // (pointers the bulk copies cannot use)
        const int64_t fb_grid = p->grid[0];
        const int64_t fb_chain = p->chain[0], fb_depth = p->depth[0];
        const bool fb_ok = p->path_ok[0];
        if (C > 256) return ADAPTIC_ERR_UNSUPPORTED;
        const bool scal = !p->vec_shape;
        p->mis = scal;
        int NT = par(ADAPTIC_P_LANES);
        if (NT <= 0) NT = (C <= 32) ? 256 : 128;
        if (NT != 128 && NT != 256) return ADAPTIC_ERR_INVALID_ARG;
        const size_t stage_bytes = size_t(NT) * size_t(C) * 4 * (px ? 2 : 1);
        const size_t xbytes = px ? 0 : size_t((C + 31) / 32 * 32) * 4;
        int cps_t = par(ADAPTIC_P_CTAS_PER_SM);
        if (cps_t <= 0) cps_t = 2;
        const size_t budget = (size_t(220) * 1024) / size_t(cps_t);
        int stages = int(std::min<size_t>(8, (budget > xbytes ? budget - xbytes : 0) / stage_bytes));
        if (par(ADAPTIC_P_UNROLL) > 0) stages = std::min(stages, par(ADAPTIC_P_UNROLL));
        if (stages < 2) return ADAPTIC_ERR_UNSUPPORTED;
        p->lanes = NT;
        p->unroll = stages;
        p->stages = stages;
        p->block = NT;
        p->smem = xbytes + size_t(stages) * stage_bytes;
        const int occ = occupancy(tpr_fn(dt, NT, px, scal), NT, p->smem, dev.present, cps_t);
        p->ctas_per_sm = std::min(cps_t, occ);
        p->grid[1] = std::max<int64_t>(1, std::min<int64_t>(ceil_div(R, NT), int64_t(dev.sms) * p->ctas_per_sm));
        p->chain[1] = scal ? ceil_div(C, 2) : ceil_div(C / 4, 2);
        p->depth[1] = scal ? 2 : 3;
        p->path_ok[1] = (dt == DT_I32) || bound_ok(p->chain[1] + p->depth[1]);
        p->grid[0] = fb_grid; p->chain[0] = fb_chain; p->depth[0] = fb_depth; p->path_ok[0] = fb_ok;
        if (!p->path_ok[1]) return ADAPTIC_ERR_UNSUPPORTED;
        return ADAPTIC_OK;
    }

    if (v == ADAPTIC_V_MV_CPR || v == ADAPTIC_V_MV_SPLIT) {
        const int64_t nv1 = p->vec_shape ? C / 4 : C;
        int NT = par(ADAPTIC_P_LANES);
        if (NT <= 0) NT = (v == ADAPTIC_V_MV_CPR && nv1 >= 8192) ? 1024 : 256;
        if (NT != 256 && NT != 1024) return ADAPTIC_ERR_INVALID_ARG;
        // x staged in smem only for CPR (a split CTA reads a different x chunk per block)
        const bool want_shift = par(ADAPTIC_P_XSMEM) == 5;
        int RB = par(ADAPTIC_P_ROWS);
        // misaligned kernels: one row per CTA step, except the shifted-x kernel with RB rows of
        // one residue class (mv_cta_mis_rb_kernel, RB in {2, 4}, NT 256)
        const bool mis_rb = mis && want_shift && (RB == 2 || RB == 4) && NT == 256;
        if (RB <= 0 || (mis && !mis_rb)) RB = 1;
        int U = par(ADAPTIC_P_UNROLL);
        if (U <= 0) U = (RB == 4 && !mis_rb) ? 2 : 4;
        const bool combo_ok = mis_rb ? (U == 2 || U == 4)
                                     : ((RB == 1 && (U == 2 || U == 4 || U == 8)) || (RB == 2 && (U == 2 || U == 4)) ||
                                        (RB == 4 && U == 2));
        if (!combo_ok || (NT == 1024 && RB * U > 4)) return ADAPTIC_ERR_INVALID_ARG;
        if (want_shift && (px || !mis)) return ADAPTIC_ERR_UNSUPPORTED;   // shifted x: misaligned MV rows only
        const bool want_fx = par(ADAPTIC_P_XSMEM) == 9;                 // x funnel (mv_cta_mis_fx_kernel)
        if (want_fx && (px || !mis || NT != 256 || !mis_cta_fx_fn(dt, NT, U))) return ADAPTIC_ERR_UNSUPPORTED;
        const int xm = want_fx ? XM_FX_MODE : want_shift ? XM_SHIFT_MODE
                                                         : pick_xmode(px, par(ADAPTIC_P_XSMEM), C, v == ADAPTIC_V_MV_CPR);
        if (xm < 0) return ADAPTIC_ERR_UNSUPPORTED;
        const size_t xsm = xm == 1 ? size_t((C * 4 + 15) / 16 * 16) : 0;
        int cps = par(ADAPTIC_P_CTAS_PER_SM);
        // register double buffering (NT 256 only): 1 off, 2 on; default off
        const int pipe_req = par(ADAPTIC_P_PIPE);
        if (pipe_req < 0 || pipe_req > 2 || (pipe_req == 2 && NT != 256)) return ADAPTIC_ERR_INVALID_ARG;
        p->pipe = (pipe_req == 2 && !mis) ? 1 : 0;
        p->mis = mis;
        if (cps <= 0) cps = occupancy(want_fx ? mis_cta_fx_fn(dt, NT, U) : mis_rb ? mis_cta_rb_fn(dt, NT, U, RB)
                                      : mis ? mis_cta_fn(dt, NT, U, xm) : cta_fn(dt, NT, RB, U, p->vec_shape, xm, p->pipe),
                                      NT, xsm, dev.present, 2048 / NT);
        p->lanes = NT; p->unroll = U; p->rb = RB; p->block = NT; p->ctas_per_sm = cps; p->xmode = xm; p->smem = xsm;
        // split order: 1 contiguous chunks, 2 interleaved steps (default for S > 1)
        const int order = par(ADAPTIC_P_ORDER);
        if (order < 0 || order > 2) return ADAPTIC_ERR_INVALID_ARG;
        const int64_t slots = int64_t(dev.sms) * cps;
        const int64_t groups = mis_rb ? 4 * ceil_div(R, 4 * int64_t(RB)) : ceil_div(R, RB);   // residue-class groups
        int64_t S = 1;
        if (v == ADAPTIC_V_MV_SPLIT) {
            if (par(ADAPTIC_P_SPLITS) > 0) S = par(ADAPTIC_P_SPLITS);
            else {
                S = pick_splits(groups, slots, std::max<int64_t>(2, ceil_div(nv1, int64_t(NT) * U)), 2);
            }
        }
        // accuracy: raise S (SPLIT only) until the bound holds on both paths
        for (;;) {
            bool ok_all = true;
            for (int w = 0; w < 2; ++w) {
                const int64_t nv = w ? C / 4 : C;
                if (w == 1 && !p->vec_shape && !mis) continue;
                const int64_t iters = ceil_div(ceil_div(nv, S), int64_t(NT) * U);
                p->chain[w] = fold_chain(iters);
                p->depth[w] = ilog2c(U) + (w ? 2 : 0) + ilog2c(NT) + (S > 1 ? ceil_div(S, NT) + ilog2c(NT) : 0) + 1 +
                              ((w == 1 && mis) ? 1 : 0);
                p->path_ok[w] = (dt == DT_I32) || bound_ok(p->chain[w] + p->depth[w]);
                p->grid[w] = std::max<int64_t>(1, std::min<int64_t>(groups * S, slots));
                if (!p->path_ok[w]) ok_all = false;
            }
            if (ok_all || v == ADAPTIC_V_MV_CPR || S >= (int64_t(1) << 20)) break;
            S *= 2;
        }
        if (S > INT_MAX || R * S > (int64_t(1) << 40)) return ADAPTIC_ERR_UNSUPPORTED;
        p->splits = int(S);
        p->ilv = (S > 1 && order != 1) ? 1 : 0;
        if (!p->path_ok[(p->vec_shape || mis) ? 1 : 0]) return ADAPTIC_ERR_UNSUPPORTED;
        if (S > 1) {
            const size_t part = ((size_t(R) * size_t(S) * 4 + 255) / 256) * 256;
            p->cnt_off = part;
            p->ws_bytes = part + size_t(groups) * 4;
        }
        if (xm == XM_SHIFT_MODE) add_xshift_workspace(p);
        return ADAPTIC_OK;
    }

    // ---- TMV family
    // R % 4 != 0: the misaligned-row kernel (two aligned loads + funnel shift) keeps the
    // stream 128-bit over ceil(R/4) output vectors; it handles any B / y alignment, so no
    // scalar path is planned for these shapes
    p->flat = false;
    if (v == ADAPTIC_V_TMV_REGTILE && par(ADAPTIC_P_XSMEM) == 4) return derive_tmv_rowtile(p, params, dev);
    if (!p->vec_shape && (v == ADAPTIC_V_TMV_REGTILE || v == ADAPTIC_V_TMV_SPLITK) && par(ADAPTIC_P_XSMEM) == 12)
        return derive_tmv_group(p, params, dev);
    if (!p->vec_shape && v == ADAPTIC_V_TMV_REGTILE && R <= TMV_FLAT_MAX_R) {
        // few outputs off the 16-byte grid: stream B as one flat array (tmv_flat_kernel.cuh)
        const int FNT = R <= TMV_FLAT_NT_SMALL_R ? 256 : 1024;
        int U = par(ADAPTIC_P_UNROLL);
        if (U <= 0) U = 4;
        if (U != 2 && U != 4 && !(U == 8 && FNT == 256)) return ADAPTIC_ERR_INVALID_ARG;
        const int NTa = (FNT / int(R)) * int(R);
        int cps = par(ADAPTIC_P_CTAS_PER_SM);
        if (cps <= 0) cps = occupancy(tmv_flat_fn(dt, U, FNT), FNT, 0, dev.present, 2048 / FNT);
        const int64_t slots = int64_t(dev.sms) * cps;
        const int64_t nvec = ceil_div(R * C, 4) + 1;
        const int64_t G = std::max<int64_t>(1, std::min<int64_t>(slots, ceil_div(nvec, int64_t(NTa) * U)));
        const int64_t iters = ceil_div(nvec, G * NTa);
        p->flat = true; p->mis = true;
        p->lanes = NTa; p->unroll = U; p->block = FNT; p->ctas_per_sm = cps; p->splits = 1;
        p->grid[1] = G;
        p->chain[1] = fold_chain(iters);
        p->depth[1] = 2 + NTa / R + ceil_div(G, NTa / R) + NTa / R + 1;
        p->path_ok[1] = (dt == DT_I32) || bound_ok(p->chain[1] + p->depth[1]);
        if (!p->path_ok[1]) return ADAPTIC_ERR_UNSUPPORTED;
        const size_t part = ((size_t(G) * size_t(R) * 4 + 255) / 256) * 256;
        p->cnt_off = part;
        p->ws_bytes = part + 256;
        return ADAPTIC_OK;
    }
    const bool tmis = !p->vec_shape && R >= 8;
    p->mis = tmis;
    if (tmis && (v == ADAPTIC_V_TMV_SPLITK || v == ADAPTIC_V_TMV_COL) && par(ADAPTIC_P_XSMEM) == 10) {
        // sliding window (tmv_window_kernel): one aligned load per row and thread, no c-lanes
        int G8 = par(ADAPTIC_P_UNROLL) == 4 ? 1 : 2;
        void* fn = tmv_window_fn(dt, G8);
        if (!fn) return ADAPTIC_ERR_INVALID_ARG;
        const int NT = 256;
        int cps = par(ADAPTIC_P_CTAS_PER_SM);
        if (cps <= 0) cps = occupancy(fn, NT, 0, dev.present, 2);
        const int64_t slots = int64_t(dev.sms) * cps;
        const int64_t tiles = ceil_div(ceil_div(R, 4), int64_t(NT - 1));
        // splits only when the tiles cannot fill the GPU (the per-output merge costs more than a
        // partly idle last wave: 1048577 x 64 at S = 2 ran 0.69 of peak, S = 1 shapes 0.93)
        int64_t S = par(ADAPTIC_P_SPLITS) > 0 ? par(ADAPTIC_P_SPLITS)
                  : tiles * 2 >= slots ? 1
                  : pick_splits(tiles, slots, std::max<int64_t>(1, ceil_div(C, int64_t(8 * G8))), 1);
        for (;;) {
            const int64_t rows = ceil_div(C, S);
            p->chain[1] = std::min<int64_t>(rows, FOLD) + rows / FOLD;
            p->depth[1] = (S > 1 ? ceil_div(S, 2) + 1 : 0) + 2;
            p->path_ok[1] = (dt == DT_I32) || bound_ok(p->chain[1] + p->depth[1]);
            if (p->path_ok[1] || S >= (int64_t(1) << 20)) break;
            S *= 2;
        }
        if (S > INT_MAX || !p->path_ok[1]) return ADAPTIC_ERR_UNSUPPORTED;
        p->xmode = 10;
        p->lanes = NT - 1; p->unroll = 4 * G8; p->block = NT; p->ctas_per_sm = cps; p->splits = int(S);
        p->grid[1] = std::max<int64_t>(1, std::min<int64_t>(tiles * S, slots));
        if (S == 1) {
            // warp tiles of 31 windows, halo by shuffle, no CTA barrier (tmv_window_warp_kernel)
            const int minb = par(ADAPTIC_P_CTAS_PER_SM) >= 3 && G8 == 1 ? 3 : 2;
            void* wf = tmv_window_warp_fn(dt, G8, minb);
            if (!wf) return ADAPTIC_ERR_INVALID_ARG;
            p->ctas_per_sm = occupancy(wf, NT, 0, dev.present, minb);
            const int64_t wtiles = ceil_div(ceil_div(R, 4), int64_t(31));
            p->lanes = 31;
            p->grid[1] = std::max<int64_t>(1, std::min<int64_t>(ceil_div(wtiles, int64_t(NT / 32)),
                                                                int64_t(dev.sms) * p->ctas_per_sm));
        }
        p->grid[0] = p->grid[1]; p->chain[0] = p->chain[1]; p->depth[0] = p->depth[1]; p->path_ok[0] = p->path_ok[1];
        if (S > 1) {
            const size_t part = ((size_t(R) * size_t(S) * 4 + 255) / 256) * 256;
            p->cnt_off = part;
            p->ws_bytes = part + size_t(tiles) * 4;
        }
        return ADAPTIC_OK;
    }
    if (tmis && (v == ADAPTIC_V_TMV_SPLITK || v == ADAPTIC_V_TMV_COL) && par(ADAPTIC_P_XSMEM) == 7) {
        // constant word shift per c-lane (tmv_shift_kernel): one aligned load per row, no funnel
        int LR = par(ADAPTIC_P_LANES);
        if (LR <= 0) LR = clampi(pow2_ceil(ceil_div(R + 4, 4)), 16, 64);
        int U = par(ADAPTIC_P_UNROLL);
        if (U <= 0) U = 4;
        if (!tmv_shift_fn(dt, LR, U)) return ADAPTIC_ERR_INVALID_ARG;
        const int NT = 256, LC = NT / LR, WT = 4 * LR - 4;
        int cps = par(ADAPTIC_P_CTAS_PER_SM);
        // 3 resident CTAs fit since the kernel keeps 2 accumulators at U = 8 (76 registers); they
        // pay off for R < 4096 (2049 x 32768: 0.89 -> 0.94 of peak) and cost 8-13 % above, where
        // more CTAs only add c-splits (16385 x 4096: 0.955 at 2, 0.84 at 3; profiles/r2_exp/r2p_tshift_cmp.jsonl)
        if (cps <= 0) cps = std::min(R < 4096 ? 3 : 2, occupancy(tmv_shift_fn(dt, LR, U), NT, 0, dev.present, 2));
        const int64_t slots = int64_t(dev.sms) * cps;
        const int64_t tiles = ceil_div(R, int64_t(WT));
        int64_t S = par(ADAPTIC_P_SPLITS) > 0 ? par(ADAPTIC_P_SPLITS)
                                              : pick_splits(tiles, slots, std::max<int64_t>(1, ceil_div(C, int64_t(LC) * U)), 1);
        for (;;) {
            const int64_t iters = ceil_div(ceil_div(C, S), int64_t(LC) * U);
            const int NA = U > 4 ? 2 : U;          // accumulators per thread (tmv_shift_kernel)
            p->chain[1] = fold_chain(iters * (U / NA));
            p->depth[1] = ilog2c(NA) + LC + (S > 1 ? ceil_div(S, 2) + 1 : 0) + 1;
            p->path_ok[1] = (dt == DT_I32) || bound_ok(p->chain[1] + p->depth[1]);
            if (p->path_ok[1] || S >= (int64_t(1) << 20)) break;
            S *= 2;
        }
        if (S > INT_MAX || !p->path_ok[1]) return ADAPTIC_ERR_UNSUPPORTED;
        p->xmode = 7;
        p->lanes = LR; p->unroll = U; p->block = NT; p->ctas_per_sm = cps; p->splits = int(S);
        p->grid[1] = std::max<int64_t>(1, std::min<int64_t>(tiles * S, slots));
        p->grid[0] = p->grid[1]; p->chain[0] = p->chain[1]; p->depth[0] = p->depth[1]; p->path_ok[0] = p->path_ok[1];
        if (S > 1) {
            const size_t part = ((size_t(tiles) * size_t(WT) * size_t(S) * 4 + 255) / 256) * 256;
            p->cnt_off = part;
            p->ws_bytes = part + size_t(tiles) * 4;
        }
        return ADAPTIC_OK;
    }
    const int64_t rv1 = p->vec_shape ? R / 4 : tmis ? ceil_div(R, 4) : R;
    int LR = par(ADAPTIC_P_LANES);
    if (LR <= 0) {
        if (v == ADAPTIC_V_TMV_COL) LR = 256;
        else if (v == ADAPTIC_V_TMV_REGTILE) LR = clampi(pow2_ceil(rv1), 1, 256);
        else LR = clampi(pow2_ceil(rv1), 1, 64);
    }
    if (LR < 1 || LR > 256 || (LR & (LR - 1))) return ADAPTIC_ERR_INVALID_ARG;
    if (v == ADAPTIC_V_TMV_REGTILE && rv1 > LR) return ADAPTIC_ERR_UNSUPPORTED;
    int U = par(ADAPTIC_P_UNROLL);
    if (U <= 0) U = (v == ADAPTIC_V_TMV_COL) ? 8 : 4;
    if (U != 2 && U != 4 && U != 8) return ADAPTIC_ERR_INVALID_ARG;
    int NT = par(ADAPTIC_P_BLOCK);
    if (NT <= 0 || tmis) NT = TMV_NT;                      // misaligned kernel: 256 threads
    if ((NT != 256 && NT != 1024) || (NT == 1024 && U > 4)) return ADAPTIC_ERR_INVALID_ARG;
    int cps = par(ADAPTIC_P_CTAS_PER_SM);
    if (cps <= 0) cps = occupancy(tmis ? tmv_mis_fn(dt, LR, U) : tmv_fn(dt, LR, U, p->vec_shape, NT), NT, 0,
                                  dev.present, 2048 / NT);
    p->lanes = LR; p->unroll = U; p->block = NT; p->ctas_per_sm = cps;
    const int LC = NT / LR;
    const int64_t slots = int64_t(dev.sms) * cps;
    const int64_t tiles1 = ceil_div(rv1, LR);
    int64_t S = 1;
    if (par(ADAPTIC_P_SPLITS) > 0) S = par(ADAPTIC_P_SPLITS);
    else if (v != ADAPTIC_V_TMV_COL) {
        S = pick_splits(tiles1, slots, std::max<int64_t>(1, ceil_div(C, int64_t(LC) * U)), 1);
    }
    for (;;) {
        bool ok_all = true;
        for (int w = 0; w < 2; ++w) {
            if (w == 1 && !p->vec_shape && !tmis) continue;
            if (w == 0 && tmis) continue;
            const int64_t rv = w ? (tmis ? ceil_div(R, 4) : R / 4) : R;
            const int64_t tiles = ceil_div(rv, LR);
            const int64_t iters = ceil_div(ceil_div(C, S), int64_t(LC) * U);
            p->chain[w] = fold_chain(iters);
            p->depth[w] = ilog2c(U) + ilog2c(LC) + (S > 1 ? ceil_div(S, LC) + ilog2c(LC) : 0) + 1;
            p->path_ok[w] = (dt == DT_I32) || bound_ok(p->chain[w] + p->depth[w]);
            p->grid[w] = std::max<int64_t>(1, std::min<int64_t>(tiles * S, slots));
            if (!p->path_ok[w]) ok_all = false;
        }
        if (ok_all || S >= (int64_t(1) << 20)) break;
        S *= 2;
    }
    if (S > INT_MAX) return ADAPTIC_ERR_UNSUPPORTED;
    p->splits = int(S);
    if (!p->path_ok[(p->vec_shape || tmis) ? 1 : 0]) return ADAPTIC_ERR_UNSUPPORTED;
    if (S > 1) {
        // partials: S x (R, or 4*ceil(R/4) for the misaligned kernel's whole vectors)
        const size_t part = ((size_t(tmis ? 4 * ceil_div(R, 4) : R) * size_t(S) * 4 + 255) / 256) * 256;
        p->cnt_off = part;
        p->ws_bytes = part + size_t(ceil_div(R, LR)) * 4;    // tiles of the scalar path (the larger)
    }
    return ADAPTIC_OK;
}

adaptic_status validate_shape(int op, int64_t rows, int64_t cols, int dtype) {
    if (op < ADAPTIC_OP_MV || op > ADAPTIC_OP_STENCIL5) return ADAPTIC_ERR_INVALID_ARG;
    if (op == ADAPTIC_OP_STENCIL5 && dtype != ADAPTIC_F32) return ADAPTIC_ERR_UNSUPPORTED;
    if (dtype != ADAPTIC_F32 && dtype != ADAPTIC_I32) return ADAPTIC_ERR_INVALID_ARG;
    if (rows < 0 || cols < 0) return ADAPTIC_ERR_INVALID_ARG;
    if (is_b1_op(op) && dtype != ADAPTIC_F32) return ADAPTIC_ERR_UNSUPPORTED;
    if ((op == ADAPTIC_OP_IAMAX || op == ADAPTIC_OP_IAMIN || op == ADAPTIC_OP_B1ALL) && cols > int64_t(INT_MAX))
        return ADAPTIC_ERR_UNSUPPORTED;
    if (cols > 0 && rows > (int64_t(1) << 62) / 4 / cols) return ADAPTIC_ERR_INVALID_ARG;  // bytes overflow
    return ADAPTIC_OK;
}

adaptic_status make_plan(int op, int64_t rows, int64_t cols, int dtype, int variant,
                         const int32_t* params, adaptic_plan_t* out, int nvec = 1) {
    if (!out) return ADAPTIC_ERR_INVALID_ARG;
    *out = nullptr;
    adaptic_status st = validate_shape(op, rows, cols, dtype);
    if (st != ADAPTIC_OK) return st;
    if (nvec != 1 && nvec != 2 && nvec != 4 && nvec != 8) return nvec < 1 ? ADAPTIC_ERR_INVALID_ARG : ADAPTIC_ERR_UNSUPPORTED;
    if (nvec > 1 && (dtype != ADAPTIC_F32 || (op != ADAPTIC_OP_MV && op != ADAPTIC_OP_TMV))) return ADAPTIC_ERR_UNSUPPORTED;
    if (nvec > 1 && (rows > (int64_t(1) << 62) / 4 / nvec || cols > (int64_t(1) << 62) / 4 / nvec))
        return ADAPTIC_ERR_INVALID_ARG;
    if (variant < ADAPTIC_V_AUTO || variant >= ADAPTIC_V_COUNT) return ADAPTIC_ERR_INVALID_ARG;
    const DevInfo dev = device_info();
    adaptic_plan_s* p = new (std::nothrow) adaptic_plan_s();
    if (!p) return ADAPTIC_ERR_INVALID_ARG;
    p->op = op; p->dtype = dtype; p->R = rows; p->C = cols; p->sms = dev.sms; p->nvec = nvec;
    p->ws = nullptr; p->ws_cap = 0; p->fb_ws_off = 0; p->xsh_off = 0;

    if (variant != ADAPTIC_V_AUTO) {
        p->variant = variant; p->source = 0;
        st = (rows == 0 || cols == 0) ? (op_has_variant(op, variant) ? ADAPTIC_OK : ADAPTIC_ERR_UNSUPPORTED)
                                      : derive(p, params, dev);
        if (st != ADAPTIC_OK) { delete p; return st; }
        *out = p;
        return ADAPTIC_OK;
    }
    if (rows == 0 || cols == 0) {      // nothing to select: run() is a no-op / memset
        p->variant = heuristic_variant(op, std::max<int64_t>(rows, 1), std::max<int64_t>(cols, 1), dev.sms);
        p->source = 2;
        *out = p;
        return ADAPTIC_OK;
    }
    if (nvec > 1) {                    // multi-vector: the regime rules of the paper (Fig. 1)
        const int64_t nv = (cols % 4 == 0) ? cols / 4 : cols;
        if (op == ADAPTIC_OP_TMV) {
            // measured (profiles/r1c_multi_tmv.md): TMA-staged tiles for R <= 256 and for R >= 256K
            // with C >= 128 (derive_multi's rule); register-fed SPLITK tiles with one wave of
            // splits elsewhere; TMV_COL for huge R with few rows of B
            const int64_t rv = rows / 4;
            if (tmmv4_rule(nvec, rows, cols)) p->variant = ADAPTIC_V_TMV_SPLITK;     // row groups of 4
            else if (rows % 4 == 0 && rv >= 65536 && cols < 128) p->variant = ADAPTIC_V_TMV_COL;
            else if (rows % 4 == 0 && rv >= 16) p->variant = ADAPTIC_V_TMV_SPLITK;
            else p->variant = heuristic_variant(op, rows, cols, dev.sms);
        }
        else if (nv <= 32 * (nvec == 8 ? 2 : 4)) p->variant = ADAPTIC_V_MV_SUBWARP;
        else if (cols % 4 == 0) p->variant = ADAPTIC_V_MV_SPLIT;         // x tiles in smem, stream-K
        else if (rows >= 4 * int64_t(dev.sms)) p->variant = ADAPTIC_V_MV_CPR;
        else p->variant = ADAPTIC_V_MV_SPLIT;
        p->source = 2;
        st = derive(p, nullptr, dev);
        if (st != ADAPTIC_OK) {
            p->variant = (op == ADAPTIC_OP_TMV) ? ADAPTIC_V_TMV_SPLITK : ADAPTIC_V_MV_SPLIT;
            st = derive(p, nullptr, dev);
        }
        if (st != ADAPTIC_OK) { delete p; return st; }
        *out = p;
        return ADAPTIC_OK;
    }
    bool projected = false;
    if (const TableEntry* e = table_lookup(op, dtype, rows, cols, &projected)) {
        int32_t tp[ADAPTIC_NPARAMS] = {e->lanes, projected ? 0 : e->splits, projected ? 0 : e->ctas_per_sm, e->unroll,
                                       e->xsmem, e->block, e->rows, e->order, e->pipe};
        p->variant = e->variant; p->source = 1;
        // rows off the 16-byte grid, 1024 <= R <= 2^17, >= 2^24 elements: a cell that kept the
        // funnel kernel (fitted on a smaller or older-kernel shape) runs the constant-shift kernel
        // (every such training shape with both swept: constant shift 1.03-1.19x the funnel,
        // median 1.14, 15 of 15)
        if (op == ADAPTIC_OP_TMV && rows % 4 != 0 && rows >= 1024 && rows <= (int64_t(1) << 17) &&
            rows * cols >= (int64_t(1) << 24) && e->xsmem == 0 &&
            (e->variant == ADAPTIC_V_TMV_SPLITK || e->variant == ADAPTIC_V_TMV_COL)) {
            int32_t ts[ADAPTIC_NPARAMS] = {0};
            // tile width as the offgrid R + 1 training sweep picked it (sweep_r2_offtmv_full2:
            // 16 float4 lanes for R = 1025..4097, 32 for 8193..32769, 64 above)
            ts[ADAPTIC_P_LANES] = rows < 8192 ? 16 : rows < 65536 ? 32 : 64;
            ts[ADAPTIC_P_UNROLL] = 8;
            ts[ADAPTIC_P_XSMEM] = 7;
            p->variant = ADAPTIC_V_TMV_SPLITK;
            if (derive(p, ts, dev) == ADAPTIC_OK) { *out = p; return ADAPTIC_OK; }
            p->variant = e->variant;
        }
        if (derive(p, tp, dev) == ADAPTIC_OK) { *out = p; return ADAPTIC_OK; }
        if (derive(p, nullptr, dev) == ADAPTIC_OK) { *out = p; return ADAPTIC_OK; }
    }
    // short rows off the 16-byte grid whose cell entry does not fit this shape (e.g. a
    // thread-per-row tile fitted on C = 33 that needs 248 KB at C = 61): the staged row tiles
    // are the robust choice there (held-out DOT 3085902 x 61: heuristic MV_WPR 0.20 of the
    // best fixed; staged lane groups at the best)
    if ((op == ADAPTIC_OP_MV || op == ADAPTIC_OP_DOT) && cols % 4 != 0 && cols <= 1024) {
        int32_t tp[ADAPTIC_NPARAMS] = {0};
        tp[ADAPTIC_P_XSMEM] = 4;
        const int order[2] = {ADAPTIC_V_MV_SUBWARP, ADAPTIC_V_MV_WPR};
        for (int i = 0; i < 2; ++i) {
            p->variant = order[i]; p->source = 2;
            if (derive(p, tp, dev) == ADAPTIC_OK) { *out = p; return ADAPTIC_OK; }
        }
    }
    p->variant = heuristic_variant(op, rows, cols, dev.sms);
    p->source = 2;
    st = derive(p, nullptr, dev);
    if (st != ADAPTIC_OK) {
        // last resort: the split variants always satisfy the bound
        p->variant = (op == ADAPTIC_OP_TMV) ? ADAPTIC_V_TMV_SPLITK : ADAPTIC_V_MV_SPLIT;   // b1 too
        st = derive(p, nullptr, dev);
    }
    if (st != ADAPTIC_OK) { delete p; return st; }
    *out = p;
    return ADAPTIC_OK;
}

bool aligned(const void* p, uintptr_t a) { return (reinterpret_cast<uintptr_t>(p) & (a - 1)) == 0; }

bool overlap(const void* a, size_t na, const void* b, size_t nb) {
    if (na == 0 || nb == 0) return false;
    const uintptr_t a0 = reinterpret_cast<uintptr_t>(a), b0 = reinterpret_cast<uintptr_t>(b);
    return a0 < b0 + nb && b0 < a0 + na;
}

adaptic_status cuda_fail(cudaError_t e) {
    g_last_cuda_error = int(e);
    (void)cudaGetLastError();
    return ADAPTIC_ERR_CUDA;
}

// ADAPTIC_PDL=0 disables programmatic dependent launch (read once).
bool pdl_enabled() {
    static const bool on = [] {
        const char* v = std::getenv("ADAPTIC_PDL");
        return !(v && v[0] == '0');
    }();
    return on;
}

std::mutex g_attr_mu;
// (device, kernel) pairs that already have their dynamic-smem limit raised
struct AttrKey { int dev; void* fn; size_t smem; };
constexpr int kAttrCache = 256;
AttrKey g_attr_done[kAttrCache];
int g_attr_n = 0;

cudaError_t ensure_smem_attr(void* fn, size_t smem) {
    // the 48 KB default covers static + dynamic shared memory; kernels here declare up to
    // ~8 KB statically, so every dynamic size above 32 KB raises the limit explicitly
    // (found by a run with the caching allocator off: a 48 KB TPR ring + 72 B of
    // mbarriers failed to launch)
    if (smem <= 32 * 1024) return cudaSuccess;
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    std::lock_guard<std::mutex> lk(g_attr_mu);
    for (int i = 0; i < g_attr_n; ++i)
        if (g_attr_done[i].dev == dev && g_attr_done[i].fn == fn && g_attr_done[i].smem >= smem) return cudaSuccess;
    // raise the opt-in limit to exactly what this launch needs (static smem + this
    // must stay within the per-block opt-in maximum, 227 KB on B200)
    e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    if (e != cudaSuccess) return e;
    for (int i = 0; i < g_attr_n; ++i)
        if (g_attr_done[i].dev == dev && g_attr_done[i].fn == fn) { g_attr_done[i].smem = smem; return cudaSuccess; }
    if (g_attr_n < kAttrCache) g_attr_done[g_attr_n++] = AttrKey{dev, fn, smem};
    return cudaSuccess;
}

adaptic_status launch(const adaptic_plan_s* p, const void* A, const void* X, void* y,
                      cudaStream_t stream, bool vec, bool mis) {
    const int dt = p->dtype;
    const bool px = p->op == ADAPTIC_OP_DOT;
    int64_t R = p->R, C = p->C;
    const int w = (vec || mis) ? 1 : 0;
    void* part = p->ws;
    unsigned int* cnt = p->ws ? reinterpret_cast<unsigned int*>(static_cast<char*>(p->ws) + p->cnt_off) : nullptr;
    int S = p->splits;
    void* fn = nullptr;
    int block = p->block;
    size_t smem = 0;
    int64_t grid = p->grid[w];
    void* args8[8];
    void* args9[9];
    int ilv = p->ilv;
    int tile_cw = p->lanes, tile_mb = p->rb;        // mmv_tile_kernel chunk width / ticket rows
    void* args6[6];
    void** args = nullptr;
    int stages = p->stages;
    int ring_xres = p->lanes, ring_maxs = p->rb;   // mmv_ring_kernel: x resident, partial slots
    void* args10[10];
    int tr_tw = p->lanes, tr_cr = p->splits;       // tmv_ring_kernel: tile width, rows per stage
    int tr_sw = p->xmode == 6 && p->op == ADAPTIC_OP_TMV ? int(tring_stage_words_h(p->R, p->lanes, p->splits, p->nvec)) : 0;
    void* args12[13];
    int tr_dbg = p->ilv;                           // experiments only (param ORDER 8 + d)
    int chunk_w = 0;                               // mv_chunk_cta_kernel: columns per chunk

    void* args7[7];
    if (mis && p->xmode == XM_SHIFT_MODE && p->op == ADAPTIC_OP_MV && p->nvec == 1 &&
        p->variant >= ADAPTIC_V_MV_SUBWARP && p->variant <= ADAPTIC_V_MV_SPLIT) {
        // shifted copies of x for the aligned 128-bit x loads (mv_mis_kernels.cuh XM_SHIFT)
        void* xs = static_cast<char*>(p->ws) + p->xsh_off;
        void* sfn = dt == DT_F32 ? mis_shift_fn_f32() : mis_shift_fn_i32();
        const int64_t n4 = 4 * ((C + 3) / 4 * 4);
        const unsigned sgrid = unsigned(std::max<int64_t>(1, std::min<int64_t>(ceil_div(n4, 256), int64_t(p->sms) * 8)));
        void* sargs[3] = {&X, &xs, &C};
        cudaLaunchConfig_t scfg = {};
        scfg.gridDim = dim3(sgrid);
        scfg.blockDim = dim3(256);
        scfg.stream = stream;
        cudaLaunchAttribute sattr[1];
        sattr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
        sattr[0].val.programmaticStreamSerializationAllowed = 1;
        scfg.attrs = sattr;
        scfg.numAttrs = pdl_enabled() ? 1 : 0;
        cudaError_t es = cudaLaunchKernelExC(&scfg, sfn, sargs);
        if (es != cudaSuccess) return cuda_fail(es);
        X = xs;
    }
    if (p->op == ADAPTIC_OP_STENCIL5) {
        if (p->variant == ADAPTIC_V_ST_TILE && vec) {
            fn = st_tile_fn(p->rb, p->lanes);
            smem = p->smem;
        } else if (vec && p->xmode == 1) {
            fn = st_strip_fn();
        } else if (vec && p->xmode == 3) {
            fn = st_direct2_fn();
        } else if (vec && p->xmode == 2) {
            fn = st_column_fn();
            args7[0] = &A; args7[1] = &X; args7[2] = &y; args7[3] = &R; args7[4] = &C; args7[5] = &tile_mb;
            args = args7;
        } else {
            fn = st_direct_fn(vec);
        }
        if (!args) {
            args6[0] = &A; args6[1] = &X; args6[2] = &y; args6[3] = &R; args6[4] = &C;
            args = args6;
        }
    } else if (p->nvec > 1) {
        const int K = p->nvec;
        if (p->op == ADAPTIC_OP_TMV && p->xmode == 6) { fn = tmv_ring_fn(ADAPTIC_F32, K, p->unroll); smem = p->smem; }
        else if (p->op == ADAPTIC_OP_TMV && p->xmode == 8) fn = vec ? tmmv4_fn(K, p->lanes, p->unroll) : nullptr;
        else if (p->op == ADAPTIC_OP_TMV && p->xmode == 5) { fn = vec ? tmmv_tma_fn(K, p->lanes) : nullptr; smem = p->smem; }
        else if (p->op == ADAPTIC_OP_TMV) fn = tmmv_fn(K, p->lanes, p->unroll, vec);
        else if (p->xmode == 4) { fn = vec ? mmv_tile_fn(ADAPTIC_F32, K) : nullptr; smem = p->smem; }
        else if (p->xmode == 6) { fn = vec ? mmv_ring_fn(ADAPTIC_F32, K) : nullptr; smem = p->smem; }
        else if (p->xmode == 3) { fn = mmv_warp_fn(K); smem = p->smem; }
        else if (p->variant == ADAPTIC_V_MV_SUBWARP || p->variant == ADAPTIC_V_MV_WPR) fn = mmv_group_fn(K, p->lanes, p->unroll, vec);
        else { fn = mmv_cta_fn(K, p->unroll, vec, p->xmode == 1); smem = p->smem; }
        if (p->op == ADAPTIC_OP_TMV && p->xmode == 6) {
            args12[0] = &A; args12[1] = &X; args12[2] = &y; args12[3] = &R; args12[4] = &C;
            args12[5] = &tr_tw; args12[6] = &tr_cr; args12[7] = &stages; args12[8] = &tr_sw; args12[9] = &ring_maxs;
            args12[10] = &part; args12[11] = &cnt; args12[12] = &tr_dbg;
            args = args12;
        } else if (p->op == ADAPTIC_OP_MV && p->xmode == 6) {
            args10[0] = &A; args10[1] = &X; args10[2] = &y; args10[3] = &R; args10[4] = &C;
            args10[5] = &stages; args10[6] = &ring_xres; args10[7] = &ring_maxs; args10[8] = &part; args10[9] = &cnt;
            args = args10;
        } else if (p->op == ADAPTIC_OP_MV && p->xmode == 4) {
            args9[0] = &A; args9[1] = &X; args9[2] = &y; args9[3] = &R; args9[4] = &C;
            args9[5] = &tile_cw; args9[6] = &tile_mb; args9[7] = &part; args9[8] = &cnt;
            args = args9;
        } else if (p->op == ADAPTIC_OP_MV && (p->variant == ADAPTIC_V_MV_SUBWARP || p->variant == ADAPTIC_V_MV_WPR)) {
            args6[0] = &A; args6[1] = &X; args6[2] = &y; args6[3] = &R; args6[4] = &C;
            args = args6;                        // register-x group kernel or the warp kernel (xmode 3)
        } else {
            args8[0] = &A; args8[1] = &X; args8[2] = &y; args8[3] = &R; args8[4] = &C;
            args8[5] = &S; args8[6] = &part; args8[7] = &cnt;
            args = args8;
        }
    } else if (is_b1_op(p->op)) {
        if (p->variant == ADAPTIC_V_MV_SUBWARP || p->variant == ADAPTIC_V_MV_WPR) {
            fn = b1_group_fn(p->op, p->lanes, p->rb == 1 ? 1 : 0, vec);
            args6[0] = &A; args6[1] = &y; args6[2] = &R; args6[3] = &C;
            args = args6;
        } else {
            fn = b1_cta_fn(p->op, vec);
            args7[0] = &A; args7[1] = &y; args7[2] = &R; args7[3] = &C; args7[4] = &S;
            args7[5] = &part; args7[6] = &cnt;
            args = args7;
        }
    } else switch (p->variant) {
        case ADAPTIC_V_MV_TPR:
            if (vec || mis) {
                fn = tpr_fn(dt, p->lanes, px, mis);
                smem = p->smem;
                cudaError_t e = ensure_smem_attr(fn, smem);
                if (e != cudaSuccess) return cuda_fail(e);
                args6[0] = &A; args6[1] = &X; args6[2] = &y; args6[3] = &R; args6[4] = &C; args6[5] = &stages;
                args = args6;
            } else {
                fn = group_fn(dt, p->fb_lanes, p->fb_unroll, false, px ? 2 : 0);
                block = GROUP_NT;
                args6[0] = &A; args6[1] = &X; args6[2] = &y; args6[3] = &R; args6[4] = &C;
                args = args6;
            }
            break;
        case ADAPTIC_V_MV_SUBWARP:
        case ADAPTIC_V_MV_WPR:
            if (p->xmode == 4) {                          // TMA-staged row tiles
                fn = rowtile_fn(dt, p->block, p->lanes, px);
                smem = p->smem;
                args7[0] = &A; args7[1] = &X; args7[2] = &y; args7[3] = &R; args7[4] = &C;
                args7[5] = &tile_mb; args7[6] = &stages;
                args = args7;
                break;
            }
            fn = mis ? mis_group_fn(dt, p->lanes, p->unroll, p->xmode) : group_fn(dt, p->lanes, p->unroll, vec, p->xmode);
            smem = p->smem;
            args6[0] = &A; args6[1] = &X; args6[2] = &y; args6[3] = &R; args6[4] = &C;
            args = args6;
            break;
        case ADAPTIC_V_MV_CPR:
        case ADAPTIC_V_MV_SPLIT:
            if (p->xmode == 13) {                         // column chunks on staged tiles, CTA-wide
                fn = chunk_cta_fn(dt, p->block, p->lanes, p->rb);
                smem = p->smem;
                block = p->block + 32;                    // + the producer warp
                chunk_w = int(ceil_div(C, int64_t(p->splits)));
                args10[0] = &A; args10[1] = &X; args10[2] = &y; args10[3] = &R; args10[4] = &C;
                args10[5] = &tile_mb; args10[6] = &stages; args10[7] = &chunk_w; args10[8] = &part; args10[9] = &cnt;
                args = args10;
                break;
            }
            if (p->xmode == 11) {                         // long rows on staged tiles, CTA-wide
                fn = rowtile_cta_fn(dt, p->block, p->lanes, p->rb);
                smem = p->smem;
                args7[0] = &A; args7[1] = &X; args7[2] = &y; args7[3] = &R; args7[4] = &C;
                args7[5] = &tile_mb; args7[6] = &stages;
                args = args7;
                break;
            }
            if (p->xmode == 6) {                          // TMA-ring kernel, K = 1
                fn = vec ? mmv_ring_fn(dt, 1) : nullptr;
                smem = p->smem;
                args10[0] = &A; args10[1] = &X; args10[2] = &y; args10[3] = &R; args10[4] = &C;
                args10[5] = &stages; args10[6] = &ring_xres; args10[7] = &ring_maxs; args10[8] = &part; args10[9] = &cnt;
                args = args10;
                break;
            }
            if (p->xmode == 4) {                          // x-tile stream-K kernel, K = 1
                fn = vec ? mmv_tile_fn(dt, 1) : nullptr;
                smem = p->smem;
                args9[0] = &A; args9[1] = &X; args9[2] = &y; args9[3] = &R; args9[4] = &C;
                args9[5] = &tile_cw; args9[6] = &tile_mb; args9[7] = &part; args9[8] = &cnt;
                args = args9;
                break;
            }
            fn = (mis && p->xmode == XM_FX_MODE) ? (aligned(X, 16) ? mis_cta_fx_fn(dt, p->lanes, p->unroll)
                                                                    : mis_cta_fn(dt, p->lanes, p->unroll, 0))
               : (mis && p->xmode == XM_SHIFT_MODE && p->rb > 1) ? mis_cta_rb_fn(dt, p->lanes, p->unroll, p->rb)
               : mis ? mis_cta_fn(dt, p->lanes, p->unroll, p->xmode)
                     : cta_fn(dt, p->lanes, p->rb, p->unroll, vec, p->xmode, p->pipe != 0);
            smem = p->smem;
            args9[0] = &A; args9[1] = &X; args9[2] = &y; args9[3] = &R; args9[4] = &C;
            args9[5] = &S; args9[6] = &ilv; args9[7] = &part; args9[8] = &cnt;
            args = args9;
            break;
        default:
            if (p->xmode == 6) {                          // TMV with B through the TMA ring
                fn = tmv_ring_fn(dt, 1, p->unroll);
                smem = p->smem;
                args12[0] = &A; args12[1] = &X; args12[2] = &y; args12[3] = &R; args12[4] = &C;
                args12[5] = &tr_tw; args12[6] = &tr_cr; args12[7] = &stages; args12[8] = &tr_sw; args12[9] = &ring_maxs;
                args12[10] = &part; args12[11] = &cnt; args12[12] = &tr_dbg;
                args = args12;
                break;
            }
            if (p->xmode == 4) {                          // TMV on staged tiles of B
                fn = tmv_rowtile_fn(dt, p->block, p->unroll);
                smem = p->smem;
                args9[0] = &A; args9[1] = &X; args9[2] = &y; args9[3] = &R; args9[4] = &C;
                args9[5] = &tile_mb; args9[6] = &stages; args9[7] = &part; args9[8] = &cnt;
                args = args9;
                break;
            }
            if (p->xmode == 12) {                         // groups of four rows (16-byte-aligned B)
                fn = tmv_group_fn(dt, p->rb, p->unroll);
                args8[0] = &A; args8[1] = &X; args8[2] = &y; args8[3] = &R; args8[4] = &C;
                args8[5] = &ilv; args8[6] = &part; args8[7] = &cnt;
                args = args8;
                break;
            }
            if (p->flat && mis) {
                fn = tmv_flat_fn(dt, p->unroll, p->block);
                args7[0] = &A; args7[1] = &X; args7[2] = &y; args7[3] = &R; args7[4] = &C;
                args7[5] = &part; args7[6] = &cnt;
                args = args7;
                break;
            }
            if (mis && p->xmode == 10 && S == 1) {
                fn = tmv_window_warp_fn(dt, p->unroll / 4, p->ctas_per_sm >= 3 ? 3 : 2);
                args8[0] = &A; args8[1] = &X; args8[2] = &y; args8[3] = &R; args8[4] = &C;
                args = args8;
                break;
            }
            fn = (mis && p->xmode == 10) ? tmv_window_fn(dt, p->unroll / 4)
                 : (mis && p->xmode == 7) ? tmv_shift_fn(dt, p->lanes, p->unroll)
                 : mis ? tmv_mis_fn(dt, p->lanes, p->unroll) : tmv_fn(dt, p->lanes, p->unroll, vec, p->block);
            args8[0] = &A; args8[1] = &X; args8[2] = &y; args8[3] = &R; args8[4] = &C;
            args8[5] = &S; args8[6] = &part; args8[7] = &cnt;
            args = args8;
            break;
    }
    if (!fn) return ADAPTIC_ERR_UNSUPPORTED;
    if (smem > 32 * 1024) {
        cudaError_t ea = ensure_smem_attr(fn, smem);
        if (ea != cudaSuccess) return cuda_fail(ea);
    }
    if (grid > INT_MAX) grid = INT_MAX;
    // Programmatic dependent launch: the kernel may be scheduled while the previous
    // grid on the stream drains; every kernel begins with griddepcontrol.wait, so it
    // still observes all of that grid's writes (common.cuh pdl_prologue).
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(unsigned(grid));
    cfg.blockDim = dim3(unsigned(block));
    cfg.dynamicSmemBytes = smem;
    cfg.stream = stream;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = pdl_enabled() ? 1 : 0;
    cudaError_t e = cudaLaunchKernelExC(&cfg, fn, args);
    if (e != cudaSuccess) return cuda_fail(e);
    return ADAPTIC_OK;
}

adaptic_status check_run(const adaptic_plan_s* p, const void* A, const void* x, const void* y) {
    if (p->R == 0) return ADAPTIC_OK;
    if (!y) return ADAPTIC_ERR_INVALID_ARG;
    if (!aligned(y, 4)) return ADAPTIC_ERR_MISALIGNED;
    if (p->C == 0) return ADAPTIC_OK;
    const bool b1 = is_b1_op(p->op);          // BLAS-1: x is unused (may be NULL)
    if (!A || (!x && !b1)) return ADAPTIC_ERR_INVALID_ARG;
    if (!aligned(A, 4) || (!b1 && !aligned(x, 4))) return ADAPTIC_ERR_MISALIGNED;
    const bool st = p->op == ADAPTIC_OP_STENCIL5;
    const size_t abytes = size_t(p->R) * size_t(p->C) * 4;
    const size_t ybytes = st ? abytes : size_t(p->R) * y_bytes_per_row(p->op) * size_t(p->nvec);
    const size_t xbytes = b1 ? 0 : st ? 8 : (p->op == ADAPTIC_OP_DOT ? abytes : size_t(p->C) * 4 * size_t(p->nvec));
    if (overlap(y, ybytes, A, abytes) || (!b1 && overlap(y, ybytes, x, xbytes))) return ADAPTIC_ERR_ALIAS;
    if (p->ws_bytes > 0 && (p->ws == nullptr || p->ws_cap < p->ws_bytes)) return ADAPTIC_ERR_NO_WORKSPACE;
    return ADAPTIC_OK;
}

// Plan cache (SURVEY 8(a) a1 "plan caching"; selection must add no visible time):
// a selector plan depends only on (op, dtype, R, C, nvec) and the device it is made on,
// so the derived struct is memoised and later calls copy it (no workspace attached).
struct PlanKey {
    int op, dtype, nvec, dev;
    int64_t R, C;
    bool operator==(const PlanKey& o) const {
        return op == o.op && dtype == o.dtype && nvec == o.nvec && dev == o.dev && R == o.R && C == o.C;
    }
};
struct PlanKeyHash {
    size_t operator()(const PlanKey& k) const {
        uint64_t h = uint64_t(k.R) * 0x9E3779B97F4A7C15ull ^ (uint64_t(k.C) + 0x632BE59BD9B4E019ull);
        h ^= uint64_t(k.op | (k.dtype << 8) | (k.nvec << 16)) * 0xBF58476D1CE4E5B9ull + uint64_t(k.dev + 1);
        return size_t(h ^ (h >> 31));
    }
};
std::mutex g_plan_cache_mu;
std::unordered_map<PlanKey, adaptic_plan_s, PlanKeyHash> g_plan_cache;
constexpr size_t kPlanCacheMax = 4096;

adaptic_status cached_plan(int op, int64_t rows, int64_t cols, int dtype, int nvec, adaptic_plan_t* out) {
    if (!out) return ADAPTIC_ERR_INVALID_ARG;
    int dev = -1;
    if (cudaGetDevice(&dev) != cudaSuccess) { (void)cudaGetLastError(); dev = -1; }
    const PlanKey key{op, dtype, nvec, dev, rows, cols};
    {
        std::lock_guard<std::mutex> lk(g_plan_cache_mu);
        auto it = g_plan_cache.find(key);
        if (it != g_plan_cache.end()) {
            adaptic_plan_s* p = new (std::nothrow) adaptic_plan_s(it->second);
            if (!p) return ADAPTIC_ERR_INVALID_ARG;
            *out = p;
            return ADAPTIC_OK;
        }
    }
    const adaptic_status st = make_plan(op, rows, cols, dtype, ADAPTIC_V_AUTO, nullptr, out, nvec);
    if (st == ADAPTIC_OK) {
        adaptic_plan_s tmpl = **out;
        tmpl.ws = nullptr;
        tmpl.ws_cap = 0;
        std::lock_guard<std::mutex> lk(g_plan_cache_mu);
        if (g_plan_cache.size() >= kPlanCacheMax) g_plan_cache.clear();
        g_plan_cache.emplace(key, tmpl);
    }
    return st;
}

}  // namespace

// =================================================================== C ABI
extern "C" {

adaptic_status adaptic_plan(adaptic_op op, int64_t rows, int64_t cols, adaptic_dtype dtype,
                            adaptic_plan_t* out) {
    return cached_plan(op, rows, cols, dtype, 1, out);
}

adaptic_status adaptic_plan_forced(adaptic_op op, int64_t rows, int64_t cols, adaptic_dtype dtype,
                                   adaptic_variant variant, const int32_t* params, adaptic_plan_t* out) {
    if (variant == ADAPTIC_V_AUTO) return cached_plan(op, rows, cols, dtype, 1, out);
    return make_plan(op, rows, cols, dtype, variant, params, out);
}

adaptic_status adaptic_plan_multi(adaptic_op op, int64_t rows, int64_t cols, int32_t nvec, adaptic_dtype dtype,
                                  adaptic_variant variant, const int32_t* params, adaptic_plan_t* out) {
    if (variant == ADAPTIC_V_AUTO) return cached_plan(op, rows, cols, dtype, nvec, out);
    return make_plan(op, rows, cols, dtype, variant, params, out, nvec);
}

adaptic_variant adaptic_plan_variant(adaptic_plan_t plan) {
    return plan ? adaptic_variant(plan->variant) : ADAPTIC_V_AUTO;
}

size_t adaptic_plan_workspace_bytes(adaptic_plan_t plan) { return plan ? plan->ws_bytes : 0; }

adaptic_status adaptic_plan_set_workspace(adaptic_plan_t plan, void* dev_ptr, size_t bytes) {
    if (!plan) return ADAPTIC_ERR_INVALID_ARG;
    if (dev_ptr == nullptr) {
        if (bytes != 0) return ADAPTIC_ERR_INVALID_ARG;
        plan->ws = nullptr; plan->ws_cap = 0;
        return ADAPTIC_OK;
    }
    if (!aligned(dev_ptr, 16)) return ADAPTIC_ERR_MISALIGNED;
    if (bytes < plan->ws_bytes) return ADAPTIC_ERR_NO_WORKSPACE;
    plan->ws = dev_ptr; plan->ws_cap = bytes;
    return ADAPTIC_OK;
}

int adaptic_plan_describe(adaptic_plan_t p, char* buf, size_t cap) {
    if (!p) return -1;
    static const char* ops[] = {"MV", "TMV", "DOT", "ASUM", "NRM2", "IAMAX", "IAMIN", "B1ALL", "STENCIL5"};
    static const char* src[] = {"forced", "table", "heuristic"};
    char tmp[1024];
    const int n = std::snprintf(
        tmp, sizeof(tmp),
        "{\"op\":\"%s\",\"dtype\":\"%s\",\"rows\":%lld,\"cols\":%lld,\"variant\":\"%s\",\"source\":\"%s\","
        "\"nvec\":%d,\"sms\":%d,\"lanes\":%d,\"unroll\":%d,\"rows_per_group\":%d,\"splits\":%d,\"block\":%d,"
        "\"ctas_per_sm\":%d,\"stages\":%d,\"xmode\":%d,\"ilv\":%d,\"pipe\":%d,\"smem\":%zu,\"vec_shape\":%s,\"mis\":%s,\"flat\":%s,"
        "\"grid\":[%lld,%lld],\"chain\":[%lld,%lld],\"depth\":[%lld,%lld],\"path_ok\":[%s,%s],"
        "\"fallback_lanes\":%d,\"fallback_unroll\":%d,\"workspace_bytes\":%zu}",
        ops[p->op], p->dtype == ADAPTIC_F32 ? "f32" : "i32", (long long)p->R, (long long)p->C,
        kVariantNames[p->variant], src[p->source], p->nvec, p->sms, p->lanes, p->unroll, p->rb, p->splits, p->block,
        p->ctas_per_sm, p->stages, p->xmode, p->ilv, p->pipe, p->smem, p->vec_shape ? "true" : "false",
        p->mis ? "true" : "false", p->flat ? "true" : "false",
        (long long)p->grid[0], (long long)p->grid[1], (long long)p->chain[0], (long long)p->chain[1],
        (long long)p->depth[0], (long long)p->depth[1], p->path_ok[0] ? "true" : "false",
        p->path_ok[1] ? "true" : "false", p->fb_lanes, p->fb_unroll, p->ws_bytes);
    if (buf && cap > 0) {
        const size_t m = std::min(cap - 1, size_t(n));
        std::memcpy(buf, tmp, m);
        buf[m] = '\0';
    }
    return n;
}

adaptic_status adaptic_run(adaptic_plan_t p, const void* A, const void* x, void* y, void* stream_) {
    if (!p) return ADAPTIC_ERR_INVALID_ARG;
    cudaStream_t stream = static_cast<cudaStream_t>(stream_);
    adaptic_status st = check_run(p, A, x, y);
    if (st != ADAPTIC_OK || p->R == 0) return st;
    if (p->C == 0) {
        if (p->op == ADAPTIC_OP_STENCIL5) return ADAPTIC_OK;          // H x 0 grid: nothing to write
        cudaError_t e = cudaMemsetAsync(y, 0, size_t(p->R) * y_bytes_per_row(p->op) * size_t(p->nvec), stream);
        return e == cudaSuccess ? ADAPTIC_OK : cuda_fail(e);
    }
    bool vec = p->vec_shape;
    if (vec && p->op == ADAPTIC_OP_STENCIL5) {
        vec = aligned(A, 16) && aligned(y, 16);
    } else if (vec && p->nvec > 1) {
        vec = aligned(A, 16) && aligned(x, 16) && aligned(y, 16);
        if (!vec && p->op == ADAPTIC_OP_TMV && p->xmode == 6)          // the TMV ring takes any alignment
            return launch(p, A, x, y, stream, false, false);
        if (!vec) {                               // 4-byte-aligned pointers: the planned fallback
            adaptic_plan_s fb;
            if (!p->multi_fb_ok || !multi_fallback(*p, &fb, device_info())) return ADAPTIC_ERR_MISALIGNED;
            if (fb.ws_bytes > 0) {                // its own zeroed slice of p's workspace
                if (!p->ws || p->fb_ws_off + fb.ws_bytes > p->ws_cap) return ADAPTIC_ERR_NO_WORKSPACE;
                fb.ws = static_cast<char*>(p->ws) + p->fb_ws_off;
                fb.ws_cap = p->ws_cap - p->fb_ws_off;
            }
            return launch(&fb, A, x, y, stream, false, false);
        }
    } else if (vec) {
        if (p->op == ADAPTIC_OP_TMV) vec = aligned(A, 16) && aligned(y, 16);
        else if (is_b1_op(p->op)) vec = aligned(A, 16);
        else vec = aligned(A, 16) && aligned(x, 16);
    }
    // misaligned-row kernels: any 4-byte aligned A; DOT's b must share A's address modulo 16
    bool mis = !vec && p->mis &&
               (p->op != ADAPTIC_OP_DOT ||   // TMV / MV: any 4-byte alignment
                ((reinterpret_cast<uintptr_t>(A) - reinterpret_cast<uintptr_t>(x)) & 15u) == 0);
    if (mis && p->variant == ADAPTIC_V_MV_TPR)   // bulk copies of row tiles: 16-byte aligned bases
        mis = aligned(A, 16) && (p->op != ADAPTIC_OP_DOT || aligned(x, 16));
    if (p->nvec == 1 && p->xmode == 12 && p->op == ADAPTIC_OP_TMV) {
        // groups of four rows are 16-byte aligned only on a 16-byte-aligned B; other
        // pointers take the TMV_SPLITK direct kernel of the same shape
        if (aligned(A, 16)) return launch(p, A, x, y, stream, false, true);
        adaptic_plan_s fb = *p;
        fb.variant = ADAPTIC_V_TMV_SPLITK;
        if (derive(&fb, nullptr, device_info()) != ADAPTIC_OK) return ADAPTIC_ERR_UNSUPPORTED;
        if (fb.ws_bytes > 0) {
            if (!p->ws || p->fb_ws_off + fb.ws_bytes > p->ws_cap) return ADAPTIC_ERR_NO_WORKSPACE;
            fb.ws = static_cast<char*>(p->ws) + p->fb_ws_off;
            fb.ws_cap = p->ws_cap - p->fb_ws_off;
        } else {
            fb.ws = nullptr; fb.ws_cap = 0;
        }
        return adaptic_run(&fb, A, x, y, stream_);
    }
    if (p->nvec == 1 && ((p->xmode == 4 && (p->variant == ADAPTIC_V_MV_SUBWARP || p->variant == ADAPTIC_V_MV_WPR ||
                                            p->variant == ADAPTIC_V_TMV_REGTILE)) || p->xmode == 11 || p->xmode == 13)) {
        // row tiles are bulk-copied from 16-byte-aligned bases; other pointers take the
        // direct kernel of the same variant and shape
        if (aligned(A, 16) && (p->op == ADAPTIC_OP_MV || aligned(x, 16)))
            return launch(p, A, x, y, stream, p->vec_shape, p->mis);
        adaptic_plan_s fb = *p;
        if (derive(&fb, nullptr, device_info()) != ADAPTIC_OK) return ADAPTIC_ERR_UNSUPPORTED;
        if (fb.ws_bytes > 0) {                    // its own zeroed slice of p's workspace
            if (!p->ws || p->fb_ws_off + fb.ws_bytes > p->ws_cap) return ADAPTIC_ERR_NO_WORKSPACE;
            fb.ws = static_cast<char*>(p->ws) + p->fb_ws_off;
            fb.ws_cap = p->ws_cap - p->fb_ws_off;
        } else {
            fb.ws = nullptr; fb.ws_cap = 0;
        }
        return adaptic_run(&fb, A, x, y, stream_);
    }
    if (!vec && p->nvec == 1 && (p->xmode == 4 || (p->xmode == 6 && p->op == ADAPTIC_OP_MV))) {
        // the x-tile kernel needs 16-byte rows and bases (TMA): a single-vector plan run on
        // 4-byte-aligned pointers takes the CTA-per-row kernel of the same shape instead
        adaptic_plan_s fb = *p;
        fb.variant = ADAPTIC_V_MV_CPR;
        fb.ws = nullptr;
        if (derive(&fb, nullptr, device_info()) != ADAPTIC_OK || fb.ws_bytes != 0) return ADAPTIC_ERR_UNSUPPORTED;
        const bool fmis = fb.mis;
        if (!fb.path_ok[fmis ? 1 : 0]) return ADAPTIC_ERR_MISALIGNED;
        return launch(&fb, A, x, y, stream, false, fmis);
    }
    if (!p->path_ok[(vec || mis) ? 1 : 0]) return ADAPTIC_ERR_MISALIGNED;   // scalar path would break the error bound
    return launch(p, A, x, y, stream, vec, mis);
}

// ---- batched issue over concurrent streams (per host thread, per device)
namespace {
constexpr int kMaxBatchStreams = 8;
// Plans that may run alone inside adaptic_run_batch: the staged row-tile kernels (xmode 4 on the
// lane-group variants and TMV_REGTILE), persistent grids sized for a free GPU.  Round 1
// measured +1.7 % on the offgrid step with them exclusive; with round 2's kernels the same step
// is 4 % FASTER without it (5689 -> 5901 GB/s, 2 streams; 3 streams without it: 5106), so it is
// off by default.  ADAPTIC_EXCLUSIVE=1 enables it (read once).
bool plan_exclusive(const adaptic_plan_s* p) {
    static const int mode = [] { const char* e = std::getenv("ADAPTIC_EXCLUSIVE"); return e ? std::atoi(e) : 0; }();
    const bool rt4 = p->nvec == 1 && p->xmode == 4 &&
           (p->variant == ADAPTIC_V_MV_SUBWARP || p->variant == ADAPTIC_V_MV_WPR || p->variant == ADAPTIC_V_TMV_REGTILE);
    const bool rt11 = p->nvec == 1 && p->xmode == 11;
    return (mode == 1 && (rt4 || rt11)) || (mode == 2 && rt11) || (mode == 3 && rt4);
}
struct StreamPool {
    int dev = -1;
    cudaStream_t side[kMaxBatchStreams - 1] = {};
    cudaEvent_t fork = nullptr, join[kMaxBatchStreams - 1] = {};
    cudaEvent_t mainev = nullptr;          // the caller's stream, for exclusive plans
};
thread_local StreamPool g_pools[8];

cudaError_t pool_for_current_device(StreamPool** out) {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    if (dev < 0 || dev >= 8) return cudaErrorInvalidDevice;
    StreamPool& P = g_pools[dev];
    if (P.dev != dev) {
        for (int i = 0; i < kMaxBatchStreams - 1; ++i) {
            if ((e = cudaStreamCreateWithFlags(&P.side[i], cudaStreamNonBlocking)) != cudaSuccess) return e;
            if ((e = cudaEventCreateWithFlags(&P.join[i], cudaEventDisableTiming)) != cudaSuccess) return e;
        }
        if ((e = cudaEventCreateWithFlags(&P.fork, cudaEventDisableTiming)) != cudaSuccess) return e;
        if ((e = cudaEventCreateWithFlags(&P.mainev, cudaEventDisableTiming)) != cudaSuccess) return e;
        P.dev = dev;
    }
    *out = &P;
    return cudaSuccess;
}
}  // namespace

adaptic_status adaptic_run_batch(int32_t n, const adaptic_plan_t* plans, const void* const* A,
                                 const void* const* x, void* const* y, int32_t streams, void* stream_) {
    if (n < 0 || streams < 1 || streams > kMaxBatchStreams) return ADAPTIC_ERR_INVALID_ARG;
    if (n == 0) return ADAPTIC_OK;
    if (!plans || !A || !x || !y) return ADAPTIC_ERR_INVALID_ARG;
    for (int32_t i = 0; i < n; ++i) {                   // all-or-nothing: validate before issuing
        if (!plans[i]) return ADAPTIC_ERR_INVALID_ARG;
        const adaptic_status st = check_run(plans[i], A[i], x[i], y[i]);
        if (st != ADAPTIC_OK) return st;
    }
    cudaStream_t stream = static_cast<cudaStream_t>(stream_);
    const int k = std::min<int>(streams, n);
    if (k == 1) {
        for (int32_t i = 0; i < n; ++i) {
            const adaptic_status st = adaptic_run(plans[i], A[i], x[i], y[i], stream_);
            if (st != ADAPTIC_OK) return st;
        }
        return ADAPTIC_OK;
    }
    StreamPool* P = nullptr;
    cudaError_t e = pool_for_current_device(&P);
    if (e != cudaSuccess) return cuda_fail(e);
    if ((e = cudaEventRecord(P->fork, stream)) != cudaSuccess) return cuda_fail(e);
    for (int j = 0; j < k - 1; ++j)
        if ((e = cudaStreamWaitEvent(P->side[j], P->fork, 0)) != cudaSuccess) return cuda_fail(e);
    adaptic_status st = ADAPTIC_OK;
    auto lane_stream = [&](int l) { return l == 0 ? stream : P->side[l - 1]; };
    auto lane_event = [&](int l) { return l == 0 ? P->mainev : P->join[l - 1]; };
    for (int32_t i = 0; i < n && st == ADAPTIC_OK; ++i) {
        int lane = i % k;
        for (int32_t q = 0; q < i; ++q)                   // a plan's workspace serialises its runs:
            if (plans[q] == plans[i] && plans[i]->ws_bytes > 0) { lane = q % k; break; }   // same stream
        cudaStream_t s = lane_stream(lane);
        // Staged-tile kernels size a persistent grid for the whole GPU and hold most of an
        // SM's shared memory: next to another stream's kernel their late CTAs stretch the
        // launch, so they run alone -- after every lane's earlier work, and before any
        // lane's later work (plan_exclusive).
        const bool excl = plan_exclusive(plans[i]);
        if (excl)
            for (int l = 0; l < k; ++l) {
                if (l == lane) continue;
                if ((e = cudaEventRecord(lane_event(l), lane_stream(l))) != cudaSuccess ||
                    (e = cudaStreamWaitEvent(s, lane_event(l), 0)) != cudaSuccess) { st = cuda_fail(e); break; }
            }
        if (st != ADAPTIC_OK) break;
        st = adaptic_run(plans[i], A[i], x[i], y[i], s);
        if (excl && st == ADAPTIC_OK) {
            if ((e = cudaEventRecord(lane_event(lane), s)) != cudaSuccess) { st = cuda_fail(e); break; }
            for (int l = 0; l < k; ++l)
                if (l != lane && (e = cudaStreamWaitEvent(lane_stream(l), lane_event(lane), 0)) != cudaSuccess) {
                    st = cuda_fail(e); break;
                }
        }
    }
    for (int j = 0; j < k - 1; ++j) {                    // join (also after a failure)
        if ((e = cudaEventRecord(P->join[j], P->side[j])) != cudaSuccess) return cuda_fail(e);
        if ((e = cudaStreamWaitEvent(stream, P->join[j], 0)) != cudaSuccess) return cuda_fail(e);
    }
    return st;
}

adaptic_status adaptic_run_host(adaptic_plan_t p, const void* A_host, const void* x_host, void* y_host,
                                void* dA, void* dx, void* dy, void* stream_) {
    if (!p) return ADAPTIC_ERR_INVALID_ARG;
    cudaStream_t stream = static_cast<cudaStream_t>(stream_);
    if (p->R == 0) return ADAPTIC_OK;
    const bool b1 = is_b1_op(p->op);
    if (!y_host || (p->C > 0 && (!A_host || (!x_host && !b1)))) return ADAPTIC_ERR_INVALID_ARG;
    adaptic_status st = check_run(p, dA, dx, dy);
    if (st != ADAPTIC_OK) return st;
    const bool sten = p->op == ADAPTIC_OP_STENCIL5;
    const size_t abytes = size_t(p->R) * size_t(p->C) * 4;
    const size_t xbytes = sten ? 8 : (p->op == ADAPTIC_OP_DOT ? abytes : size_t(p->C) * 4 * size_t(p->nvec));
    const size_t ybytes = sten ? abytes : size_t(p->R) * y_bytes_per_row(p->op) * size_t(p->nvec);
    cudaError_t e;
    if (p->C > 0) {
        if (!b1 && (e = cudaMemcpyAsync(dx, x_host, xbytes, cudaMemcpyHostToDevice, stream)) != cudaSuccess)
            return cuda_fail(e);
        if ((e = cudaMemcpyAsync(dA, A_host, abytes, cudaMemcpyHostToDevice, stream)) != cudaSuccess) return cuda_fail(e);
    }
    st = adaptic_run(p, dA, dx, dy, stream_);
    if (st != ADAPTIC_OK) return st;
    if ((e = cudaMemcpyAsync(y_host, dy, ybytes, cudaMemcpyDeviceToHost, stream)) != cudaSuccess) return cuda_fail(e);
    return ADAPTIC_OK;
}

void adaptic_plan_destroy(adaptic_plan_t plan) { delete plan; }

const char* adaptic_status_string(adaptic_status s) {
    switch (s) {
        case ADAPTIC_OK: return "ADAPTIC_OK";
        case ADAPTIC_ERR_INVALID_ARG: return "ADAPTIC_ERR_INVALID_ARG";
        case ADAPTIC_ERR_UNSUPPORTED: return "ADAPTIC_ERR_UNSUPPORTED";
        case ADAPTIC_ERR_MISALIGNED: return "ADAPTIC_ERR_MISALIGNED";
        case ADAPTIC_ERR_ALIAS: return "ADAPTIC_ERR_ALIAS";
        case ADAPTIC_ERR_NO_WORKSPACE: return "ADAPTIC_ERR_NO_WORKSPACE";
        case ADAPTIC_ERR_CUDA: return "ADAPTIC_ERR_CUDA";
        default: return "ADAPTIC_ERR_UNKNOWN";
    }
}

const char* adaptic_variant_name(adaptic_variant v) {
    return (v >= 0 && v < ADAPTIC_V_COUNT) ? kVariantNames[v] : "UNKNOWN";
}

int adaptic_last_cuda_error(void) { return g_last_cuda_error; }

int adaptic_abi_version(void) { return ADAPTIC_ABI_VERSION; }

}  // extern "C"
