// tune.cpp -- the offline threshold tuner.
//
// The paper tunes one LogIntegerParameter per threshold with OpenTuner,
// summing runtimes over user datasets, and memoises repeated paths
// through the branching tree; it suggests using the tree to avoid
// redundant settings altogether.  That is what this does, exactly:
//   1. measure: run every forced version on every training shape, R reps,
//      CUDA events on the caller's stream, median -> cost_table[s][v];
//   2. search: the only thresholds that matter are those between adjacent
//      training Par values (anything in between gives the same path), so
//      enumerate t_top over {min Par_top, geometric midpoints, +inf} and
//      t_intra likewise, map each pair to its path (one version per shape),
//      evaluate each DISTINCT path once (memoised), keep the cheapest.
#include <cuda_runtime.h>
#include <string.h>

#include <algorithm>
#include <cmath>
#include <limits>
#include <map>
#include <vector>

#include "../../include/ifl.h"
#include "ifl_internal.h"

namespace {

// Minimax cost (cost = 1): paths whose worst slowdown is within 1 % of the
// best achievable one are a measurement tie (per-shape medians of a few reps
// move that much from box to box), and among them the smallest sum of
// runtimes wins -- so a near-equal worst shape no longer decides the versions
// of all the other shapes.  Two passes (optimum first, then the tie set), so
// ties cannot chain.  cost = 0 (the paper's sum): exact minimum.
constexpr double kTieTol = 0.01;

struct PathCost {
    double primary, sum;
    size_t order;  // first enumeration position (deterministic tie-break)
};

template <typename Map>
typename Map::const_iterator pick_path(const Map& memo, int cost) {
    double best = std::numeric_limits<double>::infinity();
    for (auto& kv : memo) best = std::min(best, kv.second.first.primary);
    const double lim = cost == 1 ? best * (1.0 + kTieTol) : best;
    auto pick = memo.end();
    for (auto it = memo.begin(); it != memo.end(); ++it) {
        const PathCost& c = it->second.first;
        if (c.primary > lim) continue;
        if (pick == memo.end() || c.sum < pick->second.first.sum ||
            (c.sum == pick->second.first.sum && c.order < pick->second.first.order))
            pick = it;
    }
    return pick;
}

std::vector<int64_t> candidates(std::vector<int64_t> v) {
    std::sort(v.begin(), v.end());
    v.erase(std::unique(v.begin(), v.end()), v.end());
    std::vector<int64_t> c;
    if (v.empty()) return {INT64_MAX};
    c.push_back(v.front());  // every shape passes the guard
    for (size_t i = 0; i + 1 < v.size(); ++i) {
        // geometric midpoint, strictly above v[i] and at most v[i+1] (reading q)
        double g = std::ceil(std::sqrt((double)v[i] * (double)v[i + 1]));
        int64_t t = (int64_t)g;
        if (t <= v[i]) t = v[i] + 1;
        if (t > v[i + 1]) t = v[i + 1];
        c.push_back(t);
    }
    c.push_back(INT64_MAX);  // no shape passes the guard
    return c;
}

}  // namespace

extern "C" int ifl_tune_search(const int64_t* par_top, const int64_t* par_mid, const double* cost_table, int nshapes,
                               int cost, int64_t* t_top, int64_t* t_intra, int* n_paths) {
    if (nshapes <= 0 || !par_top || !par_mid || !cost_table || (cost != 0 && cost != 1)) return IFL_EINVAL;
    std::vector<int64_t> pt(par_top, par_top + nshapes), pm(par_mid, par_mid + nshapes);
    const std::vector<int64_t> ct = candidates(pt), ci = candidates(pm);
    std::vector<double> best(nshapes, std::numeric_limits<double>::infinity());
    for (int s = 0; s < nshapes; ++s)
        for (int v = 0; v < 3; ++v) best[s] = std::min(best[s], cost_table[s * 3 + v]);

    // path -> (cost, thresholds of its first enumeration)
    std::map<std::vector<int>, std::pair<PathCost, std::pair<int64_t, int64_t>>> memo;
    for (int64_t a : ct) {
        for (int64_t b : ci) {
            std::vector<int> path(nshapes);
            for (int s = 0; s < nshapes; ++s)
                path[s] = pt[s] >= a ? IFL_V_TOP : (pm[s] >= b ? IFL_V_MIDDLE : IFL_V_FLAT);
            if (memo.count(path)) continue;
            double sum = 0, worst = 0;
            for (int s = 0; s < nshapes; ++s) {
                const double c = cost_table[s * 3 + path[s]];
                sum += c;
                worst = std::max(worst, c / best[s]);
            }
            memo.emplace(path, std::make_pair(PathCost{cost == 0 ? sum : worst, sum, memo.size()},
                                              std::make_pair(a, b)));
        }
    }
    auto it = pick_path(memo, cost);
    const double bp = it == memo.end() ? std::numeric_limits<double>::infinity() : it->second.first.primary;
    const int64_t btop = it == memo.end() ? ct.back() : it->second.second.first;
    const int64_t bintra = it == memo.end() ? ci.back() : it->second.second.second;
    if (t_top) *t_top = btop;
    if (t_intra) *t_intra = bintra;
    if (n_paths) *n_paths = (int)memo.size();
    return std::isfinite(bp) ? IFL_OK : IFL_ENOTFIT;
}

// Generalised search for a CHAIN of G guards -- the branching trees of Fig 5
// (P:374): leaf k < G is taken when par[s][k] >= t_k and every earlier guard
// failed, leaf G otherwise.  Every combination of candidate thresholds (the
// geometric midpoints between adjacent training Par values, per guard) maps to
// a path (one leaf per shape); each DISTINCT path is costed once (P:374-378
// memoisation), and once every shape is placed, the later guards are not
// enumerated at all.  Cost as in ifl_tune_search; ties broken by the sum.
namespace {
struct ChainSearch {
    const int64_t* par;
    const double* cost;
    int ns, G, kind;
    std::vector<std::vector<int64_t>> cand;
    std::vector<double> best;
    std::map<std::vector<int>, std::pair<PathCost, std::vector<int64_t>>> memo;  // path -> (cost, thresholds)
    std::vector<int> path;
    std::vector<int64_t> cur;

    void eval() {
        if (memo.count(path)) return;
        double sum = 0, worst = 0;
        for (int s = 0; s < ns; ++s) {
            const double c = cost[s * (G + 1) + path[s]];
            sum += c;
            worst = std::max(worst, c / best[s]);
        }
        memo.emplace(path, std::make_pair(PathCost{kind == 0 ? sum : worst, sum, memo.size()}, cur));
    }
    void rec(int k, int left) {
        if (k == G || left == 0) {
            for (int j = k; j < G; ++j) cur[j] = INT64_MAX;  // later guards are irrelevant
            std::vector<int> rest;
            for (int s = 0; s < ns; ++s)
                if (path[s] < 0) {
                    path[s] = G;  // the else-leaf
                    rest.push_back(s);
                }
            eval();
            for (int s : rest) path[s] = -1;
            return;
        }
        for (int64_t t : cand[k]) {
            cur[k] = t;
            std::vector<int> took;
            for (int s = 0; s < ns; ++s)
                if (path[s] < 0 && par[s * G + k] >= t) {
                    path[s] = k;
                    took.push_back(s);
                }
            rec(k + 1, left - (int)took.size());
            for (int s : took) path[s] = -1;
        }
    }
};
}  // namespace

extern "C" int ifl_tune_search_chain(const int64_t* par, const double* cost_table, int nshapes, int G, int cost,
                                     int64_t* thresholds, int* n_paths) {
    if (nshapes <= 0 || G <= 0 || G > 8 || !par || !cost_table || (cost != 0 && cost != 1)) return IFL_EINVAL;
    ChainSearch cs;
    cs.par = par;
    cs.cost = cost_table;
    cs.ns = nshapes;
    cs.G = G;
    cs.kind = cost;
    cs.cand.resize(G);
    for (int k = 0; k < G; ++k) {
        std::vector<int64_t> v(nshapes);
        for (int s = 0; s < nshapes; ++s) v[s] = par[s * G + k];
        cs.cand[k] = candidates(v);
    }
    cs.best.assign(nshapes, std::numeric_limits<double>::infinity());
    for (int s = 0; s < nshapes; ++s)
        for (int v = 0; v <= G; ++v) cs.best[s] = std::min(cs.best[s], cost_table[s * (G + 1) + v]);
    cs.path.assign(nshapes, -1);
    cs.cur.assign(G, INT64_MAX);
    cs.rec(0, nshapes);
    auto it = pick_path(cs.memo, cost);
    if (thresholds)
        for (int k = 0; k < G; ++k) thresholds[k] = it == cs.memo.end() ? INT64_MAX : it->second.second[k];
    if (n_paths) *n_paths = (int)cs.memo.size();
    return (it != cs.memo.end() && std::isfinite(it->second.first.primary)) ? IFL_OK : IFL_ENOTFIT;
}

namespace {

enum Kind { K_SEGRED, K_SEGSCAN, K_MM_F32, K_MM_BF16, K_TRIDAG, K_LVC, K_COLRED, K_COLSCAN, K_TREE_F32, K_TREE_BF16,
            K_SEGRED_CL, K_SEGSCAN_CL, K_SEGRED_MIDG, K_SEGSCAN_MIDG, K_BAD };

Kind kind_of(const char* site) {
    if (!site) return K_BAD;
    if (!strcmp(site, "segred.b4")) return K_SEGRED;
    if (!strcmp(site, "segscan.b4")) return K_SEGSCAN;
    if (!strcmp(site, "redomap2.f32")) return K_MM_F32;
    if (!strcmp(site, "redomap2.bf16")) return K_MM_BF16;
    if (!strcmp(site, "tridag")) return K_TRIDAG;
    if (!strcmp(site, "lvc")) return K_LVC;
    if (!strcmp(site, "colred.b4")) return K_COLRED;
    if (!strcmp(site, "colscan.b4")) return K_COLSCAN;
    if (!strcmp(site, "redomap2.f32.tree")) return K_TREE_F32;
    if (!strcmp(site, "redomap2.bf16.tree")) return K_TREE_BF16;
    if (!strcmp(site, "segred.b4.tree")) return K_SEGRED_CL;
    if (!strcmp(site, "segscan.b4.tree")) return K_SEGSCAN_CL;
    if (!strcmp(site, "segred.b4.midg")) return K_SEGRED_MIDG;
    if (!strcmp(site, "segscan.b4.midg")) return K_SEGSCAN_MIDG;
    return K_BAD;
}

// the 4-leaf segred / segscan chain (TOP, MIDDLE, CLUSTER, FLAT; reading R18)
// runs the plain site's calls with one more forced version
Kind mm_of(Kind k) {
    return k == K_TREE_F32 ? K_MM_F32 : k == K_TREE_BF16 ? K_MM_BF16 : (k == K_SEGRED_CL || k == K_SEGRED_MIDG) ? K_SEGRED
         : (k == K_SEGSCAN_CL || k == K_SEGSCAN_MIDG) ? K_SEGSCAN : k;
}
bool is_midg(Kind k) { return k == K_SEGRED_MIDG || k == K_SEGSCAN_MIDG; }
bool is_tree(Kind k) { return k == K_TREE_F32 || k == K_TREE_BF16; }
bool is_cl(Kind k) { return k == K_SEGRED_CL || k == K_SEGSCAN_CL; }

int arity(Kind k) {
    return (k == K_SEGRED || k == K_SEGSCAN || k == K_COLRED || k == K_COLSCAN || k == K_SEGRED_CL || k == K_SEGSCAN_CL ||
            k == K_SEGRED_MIDG || k == K_SEGSCAN_MIDG)
               ? 2
           : k == K_LVC ? 4
                        : 3;
}

size_t align256(size_t b) { return (b + 255) & ~(size_t)255; }
int64_t ceil_div_i64(int64_t a, int64_t b) { return (a + b - 1) / b; }

size_t ws_bytes_of(Kind k, const int64_t* s) {
    k = mm_of(k);
    switch (k) {
    case K_SEGRED: return ifl_workspace_bytes("segred", s[0], s[1], 0, IFL_F32, -1);
    case K_SEGSCAN: return ifl_workspace_bytes("segscan", s[0], s[1], 0, IFL_F32, -1);
    case K_MM_F32: return ifl_workspace_bytes("redomap2", s[0], s[1], s[2], IFL_F32, -1);
    case K_MM_BF16: return ifl_workspace_bytes("redomap2", s[0], s[1], s[2], IFL_BF16, -1);
    case K_TRIDAG: return ifl_workspace_bytes("tridag", s[0], s[1], s[2], IFL_F32, -1);
    case K_LVC: return ifl_workspace_bytes("lvc", s[2], s[3], 0, IFL_F32, -1);
    case K_COLRED: return ifl_workspace_bytes("colred", s[0], s[1], 0, IFL_F32, -1);
    case K_COLSCAN: return ifl_workspace_bytes("colscan", s[0], s[1], 0, IFL_F32, -1);
    default: return 0;
    }
}

// Scratch layout per shape: [in/A/...][out][ws], each 256-byte aligned.
size_t base_shape_bytes(Kind k, const int64_t* s) {
    k = mm_of(k);
    switch (k) {
    case K_SEGRED: {
        const int64_t n = s[0], m = s[1];
        return align256(n * m * 4) + align256(n * 4) + align256(ifl_workspace_bytes("segred", n, m, 0, IFL_F32, -1));
    }
    case K_SEGSCAN: {
        const int64_t n = s[0], m = s[1];
        return 2 * align256(n * m * 4) + align256(ifl_workspace_bytes("segscan", n, m, 0, IFL_F32, -1));
    }
    case K_MM_F32:
    case K_MM_BF16: {
        const int64_t n = s[0], m = s[1], p = s[2], e = k == K_MM_F32 ? 4 : 2;
        return align256(n * m * e) + align256(m * p * e) + align256(n * p * 4) +
               align256(ifl_workspace_bytes("redomap2", n, m, p, k == K_MM_F32 ? IFL_F32 : IFL_BF16, -1));
    }
    case K_TRIDAG: {
        const int64_t S = s[0], L = s[1], R = s[2];
        return 3 * align256(R * L * 4) + 2 * align256(S * L * 4) +
               align256(ifl_workspace_bytes("tridag", S, L, R, IFL_F32, -1));
    }
    case K_COLRED: {
        const int64_t n = s[0], m = s[1];
        return align256(n * m * 4) + align256(m * 4) + align256(ws_bytes_of(k, s));
    }
    case K_COLSCAN: {
        const int64_t n = s[0], m = s[1];
        return 2 * align256(n * m * 4) + align256(ws_bytes_of(k, s));
    }
    case K_LVC: {  // (numS, numT, numX, numY): xsss, ysss, 6 coefficient arrays, ws
        const int64_t E = s[0] * s[2] * s[3], RL = s[2] * s[3];
        return 2 * align256(E * 4) + 6 * align256(RL * 4) + align256(ws_bytes_of(k, s));
    }
    default: return 0;
    }
}

size_t shape_bytes(Kind k, const int64_t* s) { return base_shape_bytes(k, s); }

int run_forced(Kind k, const int64_t* s, int version, char* scratch, cudaStream_t st) {
    k = mm_of(k);
    switch (k) {
    case K_SEGRED: {
        const int64_t n = s[0], m = s[1];
        char* out = scratch + align256(n * m * 4);
        char* ws = out + align256(n * 4);
        char* in = scratch;
        return ifl_segred(in, out, n, m, IFL_F32, IFL_SUM, IFL_F_ID, nullptr, version, ws,
                          ifl_workspace_bytes("segred", n, m, 0, IFL_F32, -1), st, nullptr);
    }
    case K_SEGSCAN: {
        const int64_t n = s[0], m = s[1];
        char* out = scratch + align256(n * m * 4);
        char* ws = out + align256(n * m * 4);
        char* in = scratch;
        return ifl_segscan(in, out, n, m, IFL_F32, IFL_SUM, IFL_F_ID, nullptr, 0, version, ws,
                           ifl_workspace_bytes("segscan", n, m, 0, IFL_F32, -1), st, nullptr);
    }
    case K_MM_F32:
    case K_MM_BF16: {
        const int64_t n = s[0], m = s[1], p = s[2], e = k == K_MM_F32 ? 4 : 2;
        const int dt = k == K_MM_F32 ? IFL_F32 : IFL_BF16;
        char* A = scratch;
        char* B = A + align256(n * m * e);
        char* C = B + align256(m * p * e);
        char* ws = C + align256(n * p * 4);
        return ifl_redomap2(A, B, (float*)C, n, m, p, dt, 1, version, ws,
                            ifl_workspace_bytes("redomap2", n, m, p, dt, -1), st, nullptr);
    }
    case K_TRIDAG: {
        const int64_t S = s[0], L = s[1], R = s[2];
        char* a = scratch;
        char* b = a + align256(R * L * 4);
        char* c = b + align256(R * L * 4);
        char* y = c + align256(R * L * 4);
        char* x = y + align256(S * L * 4);
        char* ws = x + align256(S * L * 4);
        return ifl_tridag((float*)a, (float*)b, (float*)c, (float*)y, (float*)x, S, L, R, version, ws,
                          ifl_workspace_bytes("tridag", S, L, R, IFL_F32, -1), st, nullptr);
    }
    case K_COLRED:
    case K_COLSCAN: {
        const int64_t n = s[0], m = s[1];
        const bool scan = k == K_COLSCAN;
        char* out = scratch + align256(n * m * 4);
        char* in = scratch;
        char* ws = out + align256((scan ? n * m : m) * 4);
        return (scan ? ifl_colscan : ifl_colred)(in, out, n, m, IFL_F32, IFL_SUM, IFL_F_ID, nullptr, version, ws,
                                                 ws_bytes_of(k, s), st, nullptr);
    }
    case K_LVC: {
        // table slot 0 (TOP) = the outermost version V_OUTER, slot 2 (FLAT) =
        // its else-branch (per-step, per-site G3); slot 1 is unavailable
        if (version == IFL_V_MIDDLE) return IFL_ENOTFIT;
        const int64_t E = s[0] * s[2] * s[3], RL = s[2] * s[3];
        float* xs = (float*)scratch;
        float* ys = (float*)(scratch + align256(E * 4));
        char* co = scratch + 2 * align256(E * 4);
        const float* cf[6];
        for (int q = 0; q < 6; ++q) cf[q] = (const float*)(co + q * align256(RL * 4));
        char* ws = co + 6 * align256(RL * 4);
        return ifl::lvc_run(xs, ys, cf[0], cf[1], cf[2], cf[3], cf[4], cf[5], s[0], s[1], s[2], s[3],
                            version == IFL_V_TOP ? IFL_V_OUTER : IFL_AUTO, ws, ws_bytes_of(k, s), st, nullptr, false);
    }
    default: return IFL_EINVAL;
    }
}

// An L2-flush region (> 2x the 126 MB L2) follows the largest shape's layout:
// it is overwritten before every timed repetition, so small training shapes
// are timed from HBM as the test shapes will be (tuning sets differ from test
// sets, and the B200 L2 would otherwise hold a 2^22-element input).
constexpr size_t kFlushBytes = (size_t)256 << 20;

// Evict the L2 by overwriting the flush region (untimed).  (Tried on B200:
// evicting by READING it instead -- clean lines, no write-back in the timed
// call -- made the tuned segscan thresholds unstable between runs.)
void flush_l2(char* flush, cudaStream_t st, int q = 0) { cudaMemsetAsync(flush, q & 0xff, kFlushBytes, st); }

size_t max_shape_bytes(Kind k, const int64_t* shapes, int nshapes) {
    size_t mx = 0;
    for (int i = 0; i < nshapes; ++i) mx = std::max(mx, shape_bytes(k, shapes + i * arity(k)));
    return align256(mx);
}

// Column sites: a forced TOP / MIDDLE on a narrow array runs a handful of
// threads down millions of rows (seconds per run).  Such a version cannot win
// (do not spend the budget on settings that cannot), so it is not run:
// TOP needs >= 4096 column threads, MIDDLE >= 64 column-tile CTAs.
bool hopeless(Kind k, const int64_t* s, int v) {
    if (k != K_COLRED && k != K_COLSCAN) return false;
    const int64_t m = s[1];
    if (v == IFL_V_TOP) return (m % 4 == 0 ? m / 4 : m) < 4096;
    if (v == IFL_V_MIDDLE) return ceil_div_i64(m, (m >= 128 && m % 4 == 0) ? 128 : 32) < 64;
    return false;
}

// Capture one forced call into an executable graph (nullptr when it cannot be
// captured: no capture stream, or a version that synchronises or reads back).
cudaGraphExec_t capture_call(Kind k, const int64_t* s, int v, char* scratch, cudaStream_t cs) {
    if (!cs || cudaStreamBeginCapture(cs, cudaStreamCaptureModeThreadLocal) != cudaSuccess) {
        (void)cudaGetLastError();
        return nullptr;
    }
    const int r = run_forced(k, s, v, scratch, cs);
    cudaGraph_t g = nullptr;
    const cudaError_t ce = cudaStreamEndCapture(cs, &g);
    cudaGraphExec_t ge = nullptr;
    if (r != IFL_OK || ce != cudaSuccess || !g || cudaGraphInstantiate(&ge, g, 0) != cudaSuccess) ge = nullptr;
    if (g) cudaGraphDestroy(g);
    (void)cudaGetLastError();
    return ge;
}

}  // namespace

extern "C" size_t ifl_tune_scratch_bytes(const char* site, const int64_t* shapes, int nshapes) {
    const Kind k = kind_of(site);
    if (k == K_BAD || !shapes || nshapes <= 0) return 0;
    return max_shape_bytes(k, shapes, nshapes) + kFlushBytes;
}

extern "C" int ifl_tune(const char* site, const int64_t* shapes, int nshapes, int reps, int cost, void* scratch,
                        size_t scratch_bytes, void* stream, int64_t* t_top, int64_t* t_intra, double* cost_table) {
    const Kind k = kind_of(site);
    if (k == K_BAD || !shapes || nshapes <= 0 || reps <= 0 || !scratch) return IFL_EINVAL;
    if (scratch_bytes < ifl_tune_scratch_bytes(site, shapes, nshapes)) return IFL_EWORKSPACE;
    const int ar = arity(k);
    cudaStream_t st = (cudaStream_t)stream;
    char* flush = (char*)scratch + max_shape_bytes(k, shapes, nshapes);
    if (cudaMemsetAsync(flush, 0, kFlushBytes, st) != cudaSuccess) return IFL_ECUDA;  // valid floats, once
    // the matmul tree sites time five leaves (ROW_TOP, ROW_MIDDLE, TOP, MIDDLE,
    // FLAT) and search a chain of four guards; every other site three versions
    const bool tree = is_tree(k), cl = is_cl(k), midg = is_midg(k);
    // ".midg" sites: the V_MIDDLE group size is the tuned dimension -- slots
    // 0..4 are group-size exponents -2..+2 of the MIDDLE version (reading R19)
    const int NV = tree ? 5 : cl ? 4 : midg ? 5 : 3;
    const char* gsite = k == K_SEGSCAN_MIDG ? "segscan.b4.midg" : "segred.b4.midg";
    static const int kTreeVersion[5] = {IFL_V_ROW_TOP, IFL_V_ROW_MIDDLE, IFL_V_TOP, IFL_V_MIDDLE, IFL_V_FLAT};
    static const int kClVersion[4] = {IFL_V_TOP, IFL_V_MIDDLE, IFL_V_CLUSTER, IFL_V_FLAT};
    std::vector<double> table(nshapes * NV, std::numeric_limits<double>::infinity());
    std::vector<int64_t> ptop(nshapes), pmid(nshapes), pchain(tree ? nshapes * 4 : cl ? nshapes * 3 : 0);
    cudaEvent_t e0, e1;
    if (cudaEventCreate(&e0) != cudaSuccess || cudaEventCreate(&e1) != cudaSuccess) return IFL_ECUDA;
    cudaStream_t cs = nullptr;  // capture stream (the caller's may be the uncapturable legacy stream)
    if (cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking) != cudaSuccess) {
        (void)cudaGetLastError();
        cs = nullptr;
    }
    int rc = IFL_OK;
    for (int i = 0; i < nshapes && rc == IFL_OK; ++i) {
        const int64_t* s = shapes + i * ar;
        ifl_choice c;
        const char* psite = tree ? (k == K_TREE_F32 ? "redomap2.f32" : "redomap2.bf16")
                          : cl ? (k == K_SEGRED_CL ? "segred.b4" : "segscan.b4")
                               : site;
        ifl_select(psite, s[0], s[1], ar == 3 && k != K_TRIDAG ? s[2] : 0, &c);
        if (k == K_LVC) c.par_mid = 0;  // one guard: Par = numS
        ptop[i] = c.par_top;
        pmid[i] = c.par_mid;
        if (tree) {  // Par of the four guards: n, n*min(p,8)*32, n*p, n*p*min(m,1024)
            pchain[i * 4 + 0] = s[0];
            pchain[i * 4 + 1] = s[0] * std::min<int64_t>(s[2], 8) * 32;
            pchain[i * 4 + 2] = c.par_top;
            pchain[i * 4 + 3] = c.par_mid;
        }
        if (cl) {  // Par of the three guards: n, n*min(m,1024), n*min(m,8192) (par mode 0: n*m)
            pchain[i * 3 + 0] = c.par_top;
            pchain[i * 3 + 1] = c.par_mid;
            pchain[i * 3 + 2] = ifl_get_par_mode() == 1 ? s[0] * std::min<int64_t>(s[1], ifl::kClusterBmax) : s[0] * s[1];
        }
        // zero this shape's workspace (the tail of its scratch layout); the
        // input region keeps the caller's data
        const size_t tot = base_shape_bytes(k, s), wsb = ws_bytes_of(k, s);
        if (wsb && cudaMemsetAsync((char*)scratch + (tot - align256(wsb)), 0, align256(wsb), st) != cudaSuccess) {
            rc = IFL_ECUDA;
            break;
        }
        // versions in the order flat, middle, top; a version whose warm-up run
        // is > 50x slower than the best timed so far is recorded from that one
        // run (avoid spending the budget on settings that cannot win)
        double best_ms = std::numeric_limits<double>::infinity();
        for (int vv = 0; vv < NV; ++vv) {
            const int slot = NV - 1 - vv;                     // table column
            const int v = tree ? kTreeVersion[slot] : cl ? kClVersion[slot] : midg ? (int)IFL_V_MIDDLE : slot;
            if (midg) ifl_set_thresholds(gsite, 8 + (slot - 2), 0);  // this slot's group size
            if (hopeless(k, s, v)) continue;  // stays +inf: unavailable to the search
            flush_l2(flush, st);
            cudaEventRecord(e0, st);
            int r = run_forced(k, s, v, (char*)scratch, st);  // warm-up; also feasibility (ENOTFIT)
            cudaEventRecord(e1, st);
            if (r == IFL_ENOTFIT || r == IFL_EUNSUPPORTED) continue;
            if (r != IFL_OK) {
                rc = r;
                break;
            }
            // a second, warm eager run (the first pays lazy module loading) is
            // what the 50x test compares
            flush_l2(flush, st);
            cudaEventRecord(e0, st);
            run_forced(k, s, v, (char*)scratch, st);
            cudaEventRecord(e1, st);
            cudaEventSynchronize(e1);
            float warm = 0;
            cudaEventElapsedTime(&warm, e0, e1);
            if (warm > 50.0 * best_ms) {
                table[i * NV + slot] = warm;
                continue;
            }
            // each rep: L2 evicted, then one call.  (Measured on B200: timing 4
            // back-to-back calls alternating two input copies instead moved the
            // tuned thresholds away from the 2^26 test sweep's best -- 5.37 vs
            // 5.60 TB/s -- so it is one call per rep.)
            // The call is replayed as a CUDA graph when it can be captured, so a
            // multi-kernel version is not charged eager launch gaps the graph-
            // replayed program does not pay (B200: FLAT segred's two kernels
            // vs MIDDLE's one at n = 8 flipped the R3 guard); otherwise eager.
            cudaGraphExec_t ge = capture_call(k, s, v, (char*)scratch, cs);
            std::vector<float> ms(reps);
            for (int q = 0; q < reps; ++q) {
                flush_l2(flush, st, q);  // evict the L2 (untimed)
                cudaEventRecord(e0, st);
                if (ge)
                    cudaGraphLaunch(ge, st);
                else
                    run_forced(k, s, v, (char*)scratch, st);
                cudaEventRecord(e1, st);
                cudaEventSynchronize(e1);
                cudaEventElapsedTime(&ms[q], e0, e1);
            }
            if (ge) cudaGraphExecDestroy(ge);
            std::sort(ms.begin(), ms.end());
            table[i * NV + slot] = ms[reps / 2];
            best_ms = std::min(best_ms, (double)ms[reps / 2]);
        }
    }
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    if (cs) cudaStreamDestroy(cs);
    if (rc != IFL_OK) return rc;
    if (cost_table) std::copy(table.begin(), table.end(), cost_table);
    if (tree) {
        int64_t th[4];
        int np;
        rc = ifl_tune_search_chain(pchain.data(), table.data(), nshapes, 4, cost, th, &np);
        if (rc != IFL_OK) return rc;
        if (t_top) *t_top = th[2];
        if (t_intra) *t_intra = th[3];
        const bool bf = k == K_TREE_BF16;
        rc = ifl_set_thresholds(bf ? "redomap2.bf16.row" : "redomap2.f32.row", th[0], th[1]);
        if (rc != IFL_OK) return rc;
        return ifl_set_thresholds(bf ? "redomap2.bf16" : "redomap2.f32", th[2], th[3]);
    }
    if (midg) {  // one exponent for the site: the paper's sum of runtimes, or the minimax with the 1 % tie rule
        std::vector<double> best(nshapes, std::numeric_limits<double>::infinity());
        for (int i = 0; i < nshapes; ++i)
            for (int q = 0; q < NV; ++q) best[i] = std::min(best[i], table[i * NV + q]);
        std::vector<double> prim(NV), sum(NV, 0.0);
        for (int q = 0; q < NV; ++q) {
            double worst = 0;
            for (int i = 0; i < nshapes; ++i) {
                sum[q] += table[i * NV + q];
                worst = std::max(worst, table[i * NV + q] / best[i]);
            }
            prim[q] = cost == 0 ? sum[q] : worst;
        }
        const double opt = *std::min_element(prim.begin(), prim.end());
        int pick = 2;  // the untuned group size unless another one is better
        for (int q = 0; q < NV; ++q) {
            const bool tie = cost == 1 ? prim[q] <= opt * (1.0 + kTieTol) : prim[q] == opt;
            const bool pick_tie = cost == 1 ? prim[pick] <= opt * (1.0 + kTieTol) : prim[pick] == opt;
            if (tie && (!pick_tie || sum[q] < sum[pick])) pick = q;
        }
        if (!std::isfinite(prim[pick])) return IFL_ENOTFIT;
        if (t_top) *t_top = 8 + (pick - 2);
        if (t_intra) *t_intra = 0;
        return ifl_set_thresholds(gsite, 8 + (pick - 2), 0);
    }
    if (cl) {
        int64_t th[3];
        int np;
        rc = ifl_tune_search_chain(pchain.data(), table.data(), nshapes, 3, cost, th, &np);
        if (rc != IFL_OK) return rc;
        if (t_top) *t_top = th[0];
        if (t_intra) *t_intra = th[1];
        const bool sc = k == K_SEGSCAN_CL;
        rc = ifl_set_thresholds(sc ? "segscan.b4.cl" : "segred.b4.cl", th[2], th[2]);
        if (rc != IFL_OK) return rc;
        return ifl_set_thresholds(sc ? "segscan.b4" : "segred.b4", th[0], th[1]);
    }
    int64_t a, b;
    int np;
    rc = ifl_tune_search(ptop.data(), pmid.data(), table.data(), nshapes, cost, &a, &b, &np);
    if (rc != IFL_OK) return rc;
    if (t_top) *t_top = a;
    if (t_intra) *t_intra = b;
    return ifl_set_thresholds(site, a, b);
}
