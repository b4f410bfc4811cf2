// ifl_internal.h -- launch entry points between the C ABI (ifl_api.cpp) and
// the kernel translation units.  Not installed; not part of the ABI.
#pragma once
#include <cuda_runtime.h>
#include <stddef.h>
#include <stdint.h>

#include "../../include/ifl.h"

namespace ifl {

// Arguments of one segred/segscan call after validation and version choice.
struct SegArgs {
    const void* in;
    void* out;
    int64_t n, m;
    int dt, op, f;
    uint32_t ne_bits;  // neutral element d as raw 32-bit pattern
    void* ws;
    size_t ws_bytes;
    cudaStream_t stream;
    const void* seed = nullptr;  // segscan: per-row d (device [n]) or NULL = ne_bits for every row
    bool rev = false;            // segscan: reversed scan (row read from its last element)
    int gshift = 0;              // V_MIDDLE group size x 2^gshift (the tuned group-size dimension, R19)
};

// Flat engine tile geometry (flat.cu).  ws layout: 256-byte header then one
// 64-bit status word per tile.
constexpr int kFlatThreads = 256;
constexpr int kFlatItems = 20;
constexpr int64_t kFlatTile = (int64_t)kFlatThreads * kFlatItems;
size_t flat_ws_bytes(int64_t total_elems);

// Version kernels: return the launch error (cudaSuccess on success).
cudaError_t launch_segred_top(const SegArgs& a);
cudaError_t launch_segred_mid(const SegArgs& a);
cudaError_t launch_segscan_top(const SegArgs& a);
cudaError_t launch_segscan_mid(const SegArgs& a);
cudaError_t launch_flat(const SegArgs& a, bool scan);
cudaError_t launch_segred_rows512(const SegArgs& a);  // V_MIDDLE segred, m >= 8192 (flat.cu)
// V_CLUSTER (flat.cu): a thread-block cluster per segment, DSMEM combine
cudaError_t launch_segred_cluster(const SegArgs& a);
cudaError_t launch_segscan_cluster(const SegArgs& a);  // cudaErrorNotSupported when a row does not fit
int64_t cluster_size_scan(int64_t n, int64_t m);       // 0: a row does not fit 16 pieces
constexpr int64_t kClusterBmax = 8192;                 // Par_cl = n * min(m, 8192) (reading R18)
cudaError_t launch_fill(void* out, int64_t count, uint32_t bits, cudaStream_t s);

// Group size (threads per segment) used by the V_MIDDLE kernels.
int mid_group_size(int64_t m);
int midscan_group_size(int64_t m);

// Column (axis-0) segred / segscan, G4 (colred.cu).  version 0/1/2 = TOP /
// MIDDLE / FLAT; FLAT needs col_ws_bytes of workspace (per-chunk partials).
struct ColGeom {
    int64_t nv, mv;  // the (possibly virtual, narrow mode) [nv][mv] view the kernels walk
    int64_t ntiles, P, rows_per_chunk;
};
ColGeom col_geom(int64_t n, int64_t m, int version, bool vec4, int narrow_width);
size_t col_ws_bytes(int64_t n, int64_t m, int version);
cudaError_t launch_col(const SegArgs& a, bool scan, int version);
constexpr int64_t kColGroup = 8;  // threads per column in V_MIDDLE (reading R3's group size)

// Nested reduce [n][m][k] (seg2.cu): out[i] = d_o (+)_j (d_i (x)_q f(x[i][j][q])).
struct Seg2Args {
    const void* in;
    void* out;
    int64_t n, m, k;
    int dt, op_o, op_i, f;
    uint32_t ne_o, ne_i;
    cudaStream_t stream;
};
cudaError_t launch_seg2(const Seg2Args& a, int version);  // V_TOP / V_MIDDLE (V_FLAT: two segreds, ifl_api.cpp)

// Tuple-valued per-row argmin / argmax (arg.cu).
struct ArgArgs {
    const void* in;
    void* val;
    int* idx;
    int64_t n, m;
    int dt, which;  // which: 0 argmin, 1 argmax
    void* ws;
    size_t ws_bytes;
    cudaStream_t stream;
};
size_t arg_ws_bytes(int64_t n, int64_t m, int version);
cudaError_t launch_arg(const ArgArgs& a, int version);

// Irregular segments (irr.cu): segment i = in[off[i] .. off[i+1]-1].
struct IrrArgs {
    const void* in;
    void* out;
    const int64_t* off;  // device [n + 1]
    int64_t n, total;
    int dt, op, f;
    uint32_t ne_bits;
    void* ws;
    size_t ws_bytes;
    cudaStream_t stream;
};
int64_t irr_tiles(int64_t n, int64_t total);
size_t irr_ws_bytes(int64_t n, int64_t total, int version);
cudaError_t launch_irr(const IrrArgs& a, bool scan, int version);
cudaError_t launch_irr_inspect(const int64_t* off, int64_t n, void* res16, cudaStream_t s);

// redomap2 (redomap2.cu) and tridag (tridag.cu)
struct MmArgs {
    const void* A;
    const void* B;
    float* C;
    int64_t n, m, p;
    int in_dt, b_kmajor;
    void* ws;
    size_t ws_bytes;
    cudaStream_t stream;
};
// redomap2 workspace: [V_FLAT arrival counters: kMmCntBytes][yss^T][split-K partials]
constexpr size_t kMmCntBytes = 16384;
size_t redomap2_ws_bytes(int64_t n, int64_t m, int64_t p, int version);
cudaError_t launch_redomap2(int version, const MmArgs& a);
bool redomap2_tc_ok(const MmArgs& a);
// row-level leaves of the matmul tree (mm_row.cu); Bt is [p][m]
constexpr int64_t kMmRowMaxM = 8192;  // V_ROW_MIDDLE keeps a row of A in shared memory
bool mm_row_mid_fits(int64_t m);
cudaError_t launch_mm_row(int version, const void* A, const void* Bt, float* C, int64_t n, int64_t m, int64_t p,
                          int in_dt, cudaStream_t s);

struct TriArgs {
    const float *a, *b, *c, *y;
    float* x;
    int64_t S, L, coef_rows;
    void* ws;
    size_t ws_bytes;
    cudaStream_t stream;
};
size_t tridag_ws_bytes(int64_t coef_rows, int64_t L, int version);
bool tridag_mid_fits(int64_t L);
cudaError_t launch_tridag(int version, const TriArgs& a);       // coef + solve
cudaError_t launch_tridag_coef(int version, const TriArgs& a);  // (+) scan of the coefficient rows -> ws
cudaError_t launch_tridag_solve(int version, const TriArgs& a); // (x) and (.) scans per system (ws from _coef)

// Whole LocVolCalib-shaped program (lvc.cu): V_OUTER keeps every system in
// registers across all numT steps.  fits: both lengths <= kLvcMaxL.
constexpr int64_t kLvcMaxL = 512;
struct LvcSite {
    float* xs;       // [S][L] in place
    int64_t S, L, R; // systems, length, coefficient rows
    const float *invb, *alpha, *delta;  // [R][L] each, from launch_tridag_coef
};
cudaError_t launch_lvc_outer(const LvcSite& x, const LvcSite& y, int64_t numT, cudaStream_t s);
// ifl_lvc with the outermost branch optionally disabled (the tuner's alternative)
int lvc_run(float* xsss, float* ysss, const float* ax, const float* bx, const float* cx, const float* ay,
            const float* by, const float* cy, int64_t numS, int64_t numT, int64_t numX, int64_t numY, int version,
            void* ws, size_t ws_bytes, void* stream, ifl_choice* choice, bool allow_outer);

}  // namespace ifl
