// ifl_api.cpp -- the C ABI of include/ifl.h: argument validation, the G3
// version selector, the per-site threshold table (P:201,
// default 2^15 per P:370), workspace sizing and error reporting.
#include <cuda_runtime.h>
#include <stdarg.h>
#include <stdio.h>
#include <string.h>

#include <algorithm>
#include <cmath>
#include <map>
#include <mutex>
#include <string>

#include "../../include/ifl.h"
#include "ifl_internal.h"

namespace {

thread_local std::string g_err;

int fail(int code, const char* fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    g_err = buf;
    return code;
}

int cuda_status(cudaError_t e, const char* what) {
    if (e == cudaSuccess) return IFL_OK;
    if (e == cudaErrorNotSupported) return fail(IFL_EUNSUPPORTED, "%s: not supported", what);
    return fail(IFL_ECUDA, "%s: %s (%s)", what, cudaGetErrorName(e), cudaGetErrorString(e));
}

constexpr int64_t kDefaultThreshold = 1 << 15;
constexpr int64_t kBmax = 1024;                  // largest CTA of a V_MIDDLE kernel (reading R3)

const char* const kSites[] = {"segred.b4", "segscan.b4", "redomap2.f32", "redomap2.bf16", "tridag", "lvc",
                              "colred.b4", "colscan.b4", "segred.irr", "segscan.irr", "segarg.b4",
                              "redomap2.f32.row", "redomap2.bf16.row", "segred2.b4", "segred.b4.cl",
                              "segscan.b4.cl", "segred.b4.midg", "segscan.b4.midg"};
// ".midg" sites hold V_MIDDLE's group-size exponent, biased: t_top = 8 + shift
// (group size x 2^shift, shift in [-3, 3]; reading R19)
constexpr int64_t kMidgBias = 8;

struct Table {
    std::mutex mu;
    std::map<std::string, std::pair<int64_t, int64_t>> thr;
    int par_mode = 1;
    Table() { reset(); }
    void reset() {
        thr.clear();
        for (const char* s : kSites)  // the matmul row level and the cluster level are off until tuned (R17, R18)
            thr[s] = strstr(s, ".midg")                        ? std::make_pair(kMidgBias, (int64_t)0)
                     : (strstr(s, ".row") || strstr(s, ".cl")) ? std::make_pair(INT64_MAX, INT64_MAX)
                                                               : std::make_pair(kDefaultThreshold, kDefaultThreshold);
        par_mode = 1;
    }
};
Table& table() {
    static Table t;
    return t;
}

bool known_site(const char* s) {
    if (!s) return false;
    for (const char* k : kSites)
        if (strcmp(s, k) == 0) return true;
    return false;
}

int64_t sat_mul(int64_t a, int64_t b) {
    if (a <= 0 || b <= 0) return 0;
    if (a > INT64_MAX / b) return INT64_MAX;
    return a * b;
}

bool mul_overflows(int64_t a, int64_t b) { return a > 0 && b > 0 && a > INT64_MAX / b; }

// Par(Sigma') and Par(e_middle) of rule G3 for a site and shape.
void par_values(const char* site, int64_t n, int64_t m, int64_t p, int mode, int64_t* ptop, int64_t* pmid) {
    int64_t outer = n;
    if (strncmp(site, "redomap2", 8) == 0) outer = sat_mul(n, p);
    if (strncmp(site, "col", 3) == 0) {  // G4: the segments are the m columns, each of n rows
        *ptop = m;
        *pmid = mode == 1 ? sat_mul(m, std::min(n, ifl::kColGroup)) : sat_mul(m, n);
        return;
    }
    *ptop = outer;
    *pmid = mode == 1 ? sat_mul(outer, std::min(m, kBmax)) : sat_mul(outer, m);
}

int select_version(const char* site, int64_t n, int64_t m, int64_t p, bool mid_fits, ifl_choice* c) {
    Table& T = table();
    int64_t tt, ti;
    int mode;
    {
        std::lock_guard<std::mutex> g(T.mu);
        auto it = T.thr.find(site);
        tt = it->second.first;
        ti = it->second.second;
        mode = T.par_mode;
    }
    int64_t ptop, pmid;
    par_values(site, n, m, p, mode, &ptop, &pmid);
    int v;
    if (ptop >= tt) v = IFL_V_TOP;  // G3 guard 1 (reading R1: >=)
    else if (pmid >= ti && mid_fits) v = IFL_V_MIDDLE;  // guard 2 + fit clause (R4)
    else v = IFL_V_FLAT;
    if (c) {
        c->version = v;
        c->par_top = ptop;
        c->par_mid = pmid;
        c->t_top = tt;
        c->t_intra = ti;
    }
    return v;
}

// The cluster level of the segred / segscan guard chain (reading R18):
// after TOP and MIDDLE fail, Par_cl = n * min(m, 8192) (R3's utilized
// parallelism: a cluster of up to 16 x 512 threads per segment) >= t_cl picks
// V_CLUSTER when it fits, else V_FLAT.
void cluster_guard(bool scan, int64_t n, int64_t m, ifl_choice* c) {
    if (c->version != IFL_V_FLAT) return;
    int64_t tcl, unused;
    int mode;
    {
        Table& T = table();
        std::lock_guard<std::mutex> g(T.mu);
        auto it = T.thr.find(scan ? "segscan.b4.cl" : "segred.b4.cl");
        tcl = it->second.first;
        unused = it->second.second;
        mode = T.par_mode;
    }
    (void)unused;
    const int64_t pcl = mode == 1 ? sat_mul(n, std::min(m, ifl::kClusterBmax)) : sat_mul(n, m);
    const bool fits = !scan || ifl::cluster_size_scan(n, m) != 0;
    if (pcl >= tcl && fits) c->version = IFL_V_CLUSTER;
}

// Irregular segments: G3 with the inspector's imbalance measure.
// Par_top = total / max_len (longest-segment equivalents: what a thread per
// segment really runs in parallel), or n when max_len is unknown (0);
// Par_mid = n * min(mean length, 32) (a warp per segment, reading R3).
void irr_par(int64_t n, int64_t total, int64_t max_len, int64_t* ptop, int64_t* pmid) {
    *ptop = max_len > 0 ? std::min(n, total / max_len) : n;
    const int64_t mean = n > 0 ? (total + n - 1) / n : 0;
    *pmid = sat_mul(n, std::min<int64_t>(mean, 32));
}

// The matmul branching tree (5 leaves): the row-level guards
// of G3 on the outer map, then the existing G3 over the two-map context.
void mm_tree_select(int in_dt, int64_t n, int64_t m, int64_t p, ifl_choice* c) {
    const char* site = in_dt == IFL_BF16 ? "redomap2.bf16" : "redomap2.f32";
    const char* rsite = in_dt == IFL_BF16 ? "redomap2.bf16.row" : "redomap2.f32.row";
    select_version(site, n, m, p, true, c);
    int64_t trt, tri;
    ifl_get_thresholds(rsite, &trt, &tri);
    if (n >= trt) c->version = IFL_V_ROW_TOP;
    else if (sat_mul(n, std::min<int64_t>(p, 8) * 32) >= tri && ifl::mm_row_mid_fits(m)) c->version = IFL_V_ROW_MIDDLE;
}

uint32_t canonical_bits(int dt, int op) {
    if (dt == IFL_I32) {
        switch (op) {
        case IFL_SUM: return 0u;
        case IFL_PROD: return 1u;
        case IFL_MIN: return 0x7fffffffu;
        case IFL_MAX: return 0x80000000u;
        case IFL_AND: return 0xffffffffu;
        default: return 0u;
        }
    }
    switch (op) {
    case IFL_SUM: return 0x00000000u;  // 0.0f
    case IFL_PROD: return 0x3f800000u; // 1.0f
    case IFL_MIN: return 0x7f800000u;  // +inf
    case IFL_MAX: return 0xff800000u;  // -inf
    default: return 0u;
    }
}

bool overlap(const void* a, size_t an, const void* b, size_t bn) {
    const char* x = (const char*)a;
    const char* y = (const char*)b;
    return x < y + bn && y < x + an;
}

int validate_seg(bool scan, const void* in, void* out, int64_t n, int64_t m, int dt, int op, int f, int version,
                 const char* what, bool cluster_ok = false) {
    if (n < 0 || m < 0) return fail(IFL_EINVAL, "%s: negative size n=%lld m=%lld", what, (long long)n, (long long)m);
    if (mul_overflows(n, m) || mul_overflows(n * m, 4))
        return fail(IFL_EINVAL, "%s: n*m overflows int64", what);
    if (dt != IFL_I32 && dt != IFL_F32) return fail(IFL_EUNSUPPORTED, "%s: dtype %d unsupported", what, dt);
    if (op < IFL_SUM || op > IFL_XOR) return fail(IFL_EINVAL, "%s: bad op %d", what, op);
    if (dt == IFL_F32 && op > IFL_MAX) return fail(IFL_EUNSUPPORTED, "%s: bitwise op on f32", what);
    if (f < IFL_F_ID || f > IFL_F_ABS) return fail(IFL_EINVAL, "%s: bad map %d", what, f);
    if ((version < IFL_AUTO || version > IFL_V_FLAT) && !(cluster_ok && version == IFL_V_CLUSTER))
        return fail(IFL_EINVAL, "%s: bad version %d", what, version);
    if (n > 0 && m > 0 && in == nullptr) return fail(IFL_EINVAL, "%s: in is NULL", what);
    if ((scan ? n * m : n) > 0 && out == nullptr) return fail(IFL_EINVAL, "%s: out is NULL", what);
    if (((uintptr_t)in % 4) || ((uintptr_t)out % 4)) return fail(IFL_EINVAL, "%s: pointers not element-aligned", what);
    return IFL_OK;
}

}  // namespace

extern "C" {

const char* ifl_last_error(void) { return g_err.c_str(); }

const char* ifl_build_info(void) {
    return "ifl " __DATE__ " sm_100a; versions: top/middle/flat(/outer); segred segscan colred colscan redomap2 tridag "
           "lvc tune";
}

int ifl_select(const char* site, int64_t n, int64_t m, int64_t p, ifl_choice* choice) {
    if (!known_site(site)) return fail(IFL_EINVAL, "ifl_select: unknown site '%s'", site ? site : "(null)");
    if (n < 0 || m < 0 || p < 0) return fail(IFL_EINVAL, "ifl_select: negative size");
    bool fits = true;
    if (strcmp(site, "lvc") == 0) {  // outermost guard of Fig 6c: numS >= t0 (and V_OUTER fits)
        int64_t t0, tu;
        ifl_get_thresholds("lvc", &t0, &tu);
        ifl_choice c{(n >= t0 && m <= ifl::kLvcMaxL && p <= ifl::kLvcMaxL) ? IFL_V_OUTER : IFL_AUTO,
                     n, sat_mul(n, sat_mul(m, p)), t0, tu};
        if (choice) *choice = c;
        return IFL_OK;
    }
    if (strstr(site, ".irr")) {  // (n, total, max_len)
        int64_t tt, ti;
        ifl_get_thresholds(site, &tt, &ti);
        ifl_choice c{IFL_V_FLAT, 0, 0, tt, ti};
        irr_par(n, m, p, &c.par_top, &c.par_mid);
        if (c.par_top >= tt) c.version = IFL_V_TOP;
        else if (c.par_mid >= ti) c.version = IFL_V_MIDDLE;
        if (choice) *choice = c;
        return IFL_OK;
    }
    if (strcmp(site, "redomap2.f32") == 0 || strcmp(site, "redomap2.bf16") == 0) {
        // the version ifl_redomap2 runs: the 5-leaf tree (row-level guards first, R17)
        ifl_choice c;
        mm_tree_select(strcmp(site, "redomap2.bf16") == 0 ? IFL_BF16 : IFL_F32, n, m, p, &c);
        if (choice) *choice = c;
        return IFL_OK;
    }
    if (strcmp(site, "tridag") == 0) fits = ifl::tridag_mid_fits(m);
    if (strcmp(site, "segred.b4") == 0 || strcmp(site, "segscan.b4") == 0) {  // the 4-leaf chain (R18)
        ifl_choice c;
        select_version(site, n, m, p, true, &c);
        cluster_guard(strncmp(site, "segscan", 7) == 0, n, m, &c);
        if (choice) *choice = c;
        return IFL_OK;
    }
    return select_version(site, n, m, p, fits, choice) >= 0 ? IFL_OK : IFL_EINVAL;
}

int ifl_set_thresholds(const char* site, int64_t t_top, int64_t t_intra) {
    if (!known_site(site)) return fail(IFL_EINVAL, "unknown site '%s'", site ? site : "(null)");
    if (t_top < 0 || t_intra < 0) return fail(IFL_EINVAL, "negative threshold");
    Table& T = table();
    std::lock_guard<std::mutex> g(T.mu);
    T.thr[site] = {t_top, t_intra};
    return IFL_OK;
}

int ifl_get_thresholds(const char* site, int64_t* t_top, int64_t* t_intra) {
    if (!known_site(site)) return fail(IFL_EINVAL, "unknown site '%s'", site ? site : "(null)");
    Table& T = table();
    std::lock_guard<std::mutex> g(T.mu);
    auto& v = T.thr[site];
    if (t_top) *t_top = v.first;
    if (t_intra) *t_intra = v.second;
    return IFL_OK;
}

int ifl_reset_thresholds(void) {
    Table& T = table();
    std::lock_guard<std::mutex> g(T.mu);
    T.reset();
    return IFL_OK;
}

int ifl_set_par_mode(int mode) {
    if (mode != 0 && mode != 1) return fail(IFL_EINVAL, "par mode must be 0 or 1");
    Table& T = table();
    std::lock_guard<std::mutex> g(T.mu);
    T.par_mode = mode;
    return IFL_OK;
}

int ifl_get_par_mode(void) {
    Table& T = table();
    std::lock_guard<std::mutex> g(T.mu);
    return T.par_mode;
}

int ifl_save_thresholds(const char* path) {
    if (!path) return fail(IFL_EINVAL, "NULL path");
    FILE* fp = fopen(path, "w");
    if (!fp) return fail(IFL_EINVAL, "cannot open %s", path);
    Table& T = table();
    {
        std::lock_guard<std::mutex> g(T.mu);
        fprintf(fp, "# ifl thresholds: site t_top t_intra (par_mode %d)\n", T.par_mode);
        for (auto& kv : T.thr)
            fprintf(fp, "%s %lld %lld\n", kv.first.c_str(), (long long)kv.second.first, (long long)kv.second.second);
    }
    fclose(fp);
    return IFL_OK;
}

int ifl_load_thresholds(const char* path) {
    if (!path) return fail(IFL_EINVAL, "NULL path");
    FILE* fp = fopen(path, "r");
    if (!fp) return fail(IFL_EINVAL, "cannot open %s", path);
    char line[256];
    int rc = IFL_OK;
    while (fgets(line, sizeof line, fp)) {
        if (line[0] == '#' || line[0] == '\n') continue;
        char site[64];
        long long a, b;
        if (sscanf(line, "%63s %lld %lld", site, &a, &b) != 3) {
            rc = fail(IFL_EINVAL, "malformed line in %s: %s", path, line);
            break;
        }
        if ((rc = ifl_set_thresholds(site, a, b)) != IFL_OK) break;
    }
    fclose(fp);
    return rc;
}

size_t ifl_workspace_bytes(const char* entry, int64_t n, int64_t m, int64_t p, int dt, int version) {
    (void)dt;
    if (!entry || n < 0 || m < 0 || p < 0 || mul_overflows(n, m)) return 0;
    if (strcmp(entry, "segred") == 0 || strcmp(entry, "segscan") == 0) {
        if (version == IFL_V_FLAT || version == IFL_AUTO) return n * m > 0 ? ifl::flat_ws_bytes(n * m) : 0;
        return 0;
    }
    if (strcmp(entry, "redomap2") == 0) return ifl::redomap2_ws_bytes(n, m, p, version);
    if (strcmp(entry, "colred") == 0 || strcmp(entry, "colscan") == 0) return ifl::col_ws_bytes(n, m, version);
    if (strcmp(entry, "segarg") == 0) return ifl::arg_ws_bytes(n, m, version);
    if (strcmp(entry, "segred2") == 0) {  // (n, m, k): V_FLAT's inner results + the larger flat workspace
        if (version != IFL_V_FLAT && version != IFL_AUTO) return 0;
        if (mul_overflows(n, m) || mul_overflows(n * m, p)) return 0;
        return (((size_t)(n * m) * 4 + 255) & ~(size_t)255) +
               std::max(n * m * p > 0 ? ifl::flat_ws_bytes(n * m * p) : 0, n * m > 0 ? ifl::flat_ws_bytes(n * m) : 0);
    }
    if (strcmp(entry, "segred_irr") == 0 || strcmp(entry, "segscan_irr") == 0) return ifl::irr_ws_bytes(n, m, version);
    if (strcmp(entry, "tridag") == 0) return ifl::tridag_ws_bytes(p > 0 ? p : n, m, version);
    if (strcmp(entry, "lvc") == 0)  // (numX, numY): the coefficient scans of both sites
        return ifl::tridag_ws_bytes(n, m, version) + ifl::tridag_ws_bytes(m, n, version);
    return 0;
}

int ifl_workspace_init(void* ws, size_t ws_bytes, void* stream) {
    if (ws_bytes == 0) return IFL_OK;
    if (!ws) return fail(IFL_EINVAL, "workspace is NULL");
    return cuda_status(cudaMemsetAsync(ws, 0, ws_bytes, (cudaStream_t)stream), "ifl_workspace_init");
}

static int run_seg(bool scan, const void* in, void* out, int64_t n, int64_t m, int dt, int op, int f,
                   const void* ne, int version, void* ws, size_t ws_bytes, void* stream, ifl_choice* choice,
                   const void* seed = nullptr, bool rev = false) {
    const char* what = seed ? "ifl_segscan_seeded" : scan ? "ifl_segscan" : "ifl_segred";
    int rc = validate_seg(scan, in, out, n, m, dt, op, f, version, what, true);
    if (rc) return rc;
    const size_t ob = (size_t)(scan ? n * m : n) * 4, ib = (size_t)(n * m) * 4;
    if (scan) {
        if (in != out && overlap(in, ib, out, ob)) return fail(IFL_EINVAL, "%s: in/out partially overlap", what);
    } else if (overlap(in, ib, out, ob)) {
        return fail(IFL_EINVAL, "%s: out overlaps in", what);
    }
    if (seed && (overlap(seed, (size_t)n * 4, out, ob) || overlap(seed, (size_t)n * 4, in, ib)))
        return fail(IFL_EINVAL, "%s: seed overlaps in/out", what);
    uint32_t bits = canonical_bits(dt, op);
    if (ne) memcpy(&bits, ne, 4);
    const char* site = scan ? "segscan.b4" : "segred.b4";
    ifl_choice c;
    const int v = select_version(site, n, m, 0, true, &c);
    cluster_guard(scan, n, m, &c);
    if (version != IFL_AUTO) c.version = version;
    if (choice) *choice = c;
    if (c.version == IFL_V_CLUSTER && scan && n * m > 0 && ifl::cluster_size_scan(n, m) == 0)
        return fail(IFL_ENOTFIT, "%s: V_CLUSTER keeps a row in 16 shared-memory pieces (m <= 655360)", what);
    if (n == 0) return IFL_OK;
    if (m == 0) {  // reduce of an empty list is d; scan of it is empty
        if (scan) return IFL_OK;
        return cuda_status(ifl::launch_fill(out, n, bits, (cudaStream_t)stream), what);
    }
    (void)v;
    ifl::SegArgs a{in, out, n, m, dt, op, f, bits, ws, ws_bytes, (cudaStream_t)stream, seed, rev};
    {
        int64_t g, unused;
        ifl_get_thresholds(scan ? "segscan.b4.midg" : "segred.b4.midg", &g, &unused);
        a.gshift = (int)std::max<int64_t>(-3, std::min<int64_t>(3, g - kMidgBias));
    }
    cudaError_t e;
    switch (c.version) {
    case IFL_V_TOP: e = scan ? ifl::launch_segscan_top(a) : ifl::launch_segred_top(a); break;
    case IFL_V_MIDDLE: e = scan ? ifl::launch_segscan_mid(a) : ifl::launch_segred_mid(a); break;
    case IFL_V_CLUSTER: e = scan ? ifl::launch_segscan_cluster(a) : ifl::launch_segred_cluster(a); break;
    default: {
        const size_t need = ifl::flat_ws_bytes(n * m);
        if (!ws || ws_bytes < need)
            return fail(IFL_EWORKSPACE, "%s: V_FLAT needs %zu workspace bytes, got %zu", what, need, ws_bytes);
        e = ifl::launch_flat(a, scan);
    }
    }
    return cuda_status(e, what);
}

// Column (axis-0) reduce / scan (G4).  out: [m] (reduce) or [n][m] (scan).
static int run_col(bool scan, const void* in, void* out, int64_t n, int64_t m, int dt, int op, int f, const void* ne,
                   int version, void* ws, size_t ws_bytes, void* stream, ifl_choice* choice) {
    const char* what = scan ? "ifl_colscan" : "ifl_colred";
    // validate_seg checks the [n][m] input; the output of a column reduce has m elements
    int rc = validate_seg(true, in, scan ? out : (n * m > 0 ? out : const_cast<void*>(in)), n, m, dt, op, f, version, what);
    if (rc) return rc;
    if (!scan && m > 0 && !out) return fail(IFL_EINVAL, "%s: out is NULL", what);
    const size_t ob = (size_t)(scan ? n * m : m) * 4, ib = (size_t)(n * m) * 4;
    if (scan ? (in != out && overlap(in, ib, out, ob)) : overlap(in, ib, out, ob))
        return fail(IFL_EINVAL, "%s: in/out overlap", what);
    uint32_t bits = canonical_bits(dt, op);
    if (ne) memcpy(&bits, ne, 4);
    ifl_choice c;
    select_version(scan ? "colscan.b4" : "colred.b4", n, m, 0, true, &c);
    if (version != IFL_AUTO) c.version = version;
    if (choice) *choice = c;
    if (m == 0) return IFL_OK;
    if (n == 0) return scan ? IFL_OK : cuda_status(ifl::launch_fill(out, m, bits, (cudaStream_t)stream), what);
    if (c.version == IFL_V_FLAT) {
        const size_t need = ifl::col_ws_bytes(n, m, IFL_V_FLAT);
        if (!ws || ws_bytes < need)
            return fail(IFL_EWORKSPACE, "%s: V_FLAT needs %zu workspace bytes, got %zu", what, need, ws_bytes);
    }
    ifl::SegArgs a{in, out, n, m, dt, op, f, bits, ws, ws_bytes, (cudaStream_t)stream, nullptr};
    return cuda_status(ifl::launch_col(a, scan, c.version), what);
}

static int run_irr(bool scan, const void* in, void* out, const int64_t* off, int64_t n, int64_t total,
                   int64_t max_len, int dt, int op, int f, const void* ne, int version, void* ws, size_t ws_bytes,
                   void* stream, ifl_choice* choice) {
    const char* what = scan ? "ifl_segscan_irr" : "ifl_segred_irr";
    if (n < 0 || total < 0 || max_len < 0) return fail(IFL_EINVAL, "%s: negative size", what);
    if (mul_overflows(total, 4)) return fail(IFL_EINVAL, "%s: size overflow", what);
    int rc = validate_seg(true, in, out, 1, total, dt, op, f, version, what);  // element checks on [total]
    if (rc && !(total == 0 && rc == IFL_EINVAL)) return rc;
    if (n > 0 && !off) return fail(IFL_EINVAL, "%s: offsets is NULL", what);
    if (!scan && n > 0 && !out) return fail(IFL_EINVAL, "%s: out is NULL", what);
    if (version < IFL_AUTO || version > IFL_V_FLAT) return fail(IFL_EINVAL, "%s: bad version", what);
    const size_t ob = (size_t)(scan ? total : n) * 4, ib = (size_t)total * 4;
    if (scan ? (in != out && overlap(in, ib, out, ob)) : overlap(in, ib, out, ob))
        return fail(IFL_EINVAL, "%s: in/out overlap", what);
    uint32_t bits = canonical_bits(dt, op);
    if (ne) memcpy(&bits, ne, 4);
    const char* site = scan ? "segscan.irr" : "segred.irr";
    int64_t tt, ti;
    ifl_get_thresholds(site, &tt, &ti);
    ifl_choice c{IFL_V_FLAT, 0, 0, tt, ti};
    irr_par(n, total, max_len, &c.par_top, &c.par_mid);
    if (c.par_top >= tt) c.version = IFL_V_TOP;
    else if (c.par_mid >= ti) c.version = IFL_V_MIDDLE;
    if (version != IFL_AUTO) c.version = version;
    if (choice) *choice = c;
    if (n == 0) return IFL_OK;
    if (total == 0) return scan ? IFL_OK : cuda_status(ifl::launch_fill(out, n, bits, (cudaStream_t)stream), what);
    if (c.version == IFL_V_FLAT) {
        const size_t need = ifl::irr_ws_bytes(n, total, IFL_V_FLAT);
        if (!ws || ws_bytes < need)
            return fail(IFL_EWORKSPACE, "%s: V_FLAT needs %zu workspace bytes, got %zu", what, need, ws_bytes);
    }
    ifl::IrrArgs a{in, out, off, n, total, dt, op, f, bits, ws, ws_bytes, (cudaStream_t)stream};
    return cuda_status(ifl::launch_irr(a, scan, c.version), what);
}

int ifl_segred_irr(const void* in, void* out, const int64_t* offsets, int64_t n, int64_t total, int64_t max_len,
                   int dt, int op, int f, const void* ne, int version, void* ws, size_t ws_bytes, void* stream,
                   ifl_choice* choice) {
    return run_irr(false, in, out, offsets, n, total, max_len, dt, op, f, ne, version, ws, ws_bytes, stream, choice);
}

int ifl_segscan_irr(const void* in, void* out, const int64_t* offsets, int64_t n, int64_t total, int64_t max_len,
                    int dt, int op, int f, const void* ne, int version, void* ws, size_t ws_bytes, void* stream,
                    ifl_choice* choice) {
    return run_irr(true, in, out, offsets, n, total, max_len, dt, op, f, ne, version, ws, ws_bytes, stream, choice);
}

int ifl_irr_inspect(const int64_t* offsets, int64_t n, int64_t total, void* ws16, void* stream, int64_t* max_len) {
    if (n < 0 || total < 0 || (n > 0 && (!offsets || !ws16))) return fail(IFL_EINVAL, "ifl_irr_inspect: bad argument");
    if (max_len) *max_len = 0;
    if (n == 0) return total == 0 ? IFL_OK : fail(IFL_EINVAL, "ifl_irr_inspect: no segments but total > 0");
    cudaStream_t st = (cudaStream_t)stream;
    cudaError_t e = ifl::launch_irr_inspect(offsets, n, ws16, st);
    unsigned long long res[2] = {0, 0};
    int64_t last = 0;
    if (e == cudaSuccess) e = cudaMemcpyAsync(res, ws16, 16, cudaMemcpyDeviceToHost, st);
    if (e == cudaSuccess) e = cudaMemcpyAsync(&last, offsets + n, 8, cudaMemcpyDeviceToHost, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) return cuda_status(e, "ifl_irr_inspect");
    if (res[1] || last != total)
        return fail(IFL_EINVAL, "ifl_irr_inspect: offsets are not a segment descriptor (off[0] = 0, nondecreasing, "
                                "off[n] = total = %lld; got off[n] = %lld)", (long long)total, (long long)last);
    if (max_len) *max_len = (int64_t)res[0];
    return IFL_OK;
}

int ifl_segred2(const void* in, void* out, int64_t n, int64_t m, int64_t k, int dt, int op_o, int op_i, int f,
                const void* ne_o, const void* ne_i, int version, void* ws, size_t ws_bytes, void* stream,
                ifl_choice* choice) {
    const char* what = "ifl_segred2";
    if (n < 0 || m < 0 || k < 0) return fail(IFL_EINVAL, "%s: negative size", what);
    if (mul_overflows(n, m) || mul_overflows(n * m, k) || mul_overflows(n * m * k, 4))
        return fail(IFL_EINVAL, "%s: size overflow", what);
    int rc = validate_seg(false, in, out, n, m * k, dt, op_i, f, version, what);
    if (rc) return rc;
    rc = validate_seg(false, in, out, n, m * k, dt, op_o, IFL_F_ID, version, what);
    if (rc) return rc;
    if (overlap(in, (size_t)(n * m * k) * 4, out, (size_t)n * 4)) return fail(IFL_EINVAL, "%s: out overlaps in", what);
    uint32_t bo = canonical_bits(dt, op_o), bi = canonical_bits(dt, op_i);
    if (ne_o) memcpy(&bo, ne_o, 4);
    if (ne_i) memcpy(&bi, ne_i, 4);
    ifl_choice c;
    select_version("segred2.b4", n, m, 0, true, &c);  // Par_top = n, Par_mid = n*min(m, 1024) (R3)
    if (version != IFL_AUTO) c.version = version;
    if (choice) *choice = c;
    if (n == 0) return IFL_OK;
    cudaStream_t st = (cudaStream_t)stream;
    if (m == 0) return cuda_status(ifl::launch_fill(out, n, bo, st), what);
    if (c.version == IFL_V_FLAT) {
        // G9 flattened: segred^1 over the [n*m][k] inner segments, then over [n][m]
        const size_t tb = ((size_t)(n * m) * 4 + 255) & ~(size_t)255;
        const size_t need = ifl_workspace_bytes("segred2", n, m, k, dt, IFL_V_FLAT);
        if (!ws || ws_bytes < need)
            return fail(IFL_EWORKSPACE, "%s: V_FLAT needs %zu workspace bytes, got %zu", what, need, ws_bytes);
        void* tmp = ws;
        void* fws = (char*)ws + tb;
        rc = ifl_segred(in, tmp, n * m, k, dt, op_i, f, &bi, IFL_AUTO, fws, ws_bytes - tb, stream, nullptr);
        if (rc) return rc;
        return ifl_segred(tmp, out, n, m, dt, op_o, IFL_F_ID, &bo, IFL_AUTO, fws, ws_bytes - tb, stream, nullptr);
    }
    ifl::Seg2Args a{in, out, n, m, k, dt, op_o, op_i, f, bo, bi, st};
    return cuda_status(ifl::launch_seg2(a, c.version), what);
}

int ifl_segarg(const void* in, void* val, int32_t* idx, int64_t n, int64_t m, int dt, int which, int version,
               void* ws, size_t ws_bytes, void* stream, ifl_choice* choice) {
    const char* what = "ifl_segarg";
    int rc = validate_seg(false, in, val, n, m, dt, IFL_MIN, IFL_F_ID, version, what);
    if (rc) return rc;
    if (which != 0 && which != 1) return fail(IFL_EINVAL, "%s: which must be 0 (argmin) or 1 (argmax)", what);
    if (n > 0 && !idx) return fail(IFL_EINVAL, "%s: idx is NULL", what);
    if (m > 0x7fffffffLL) return fail(IFL_EINVAL, "%s: rows longer than 2^31 - 1 (int32 indices)", what);
    if (overlap(in, (size_t)(n * m) * 4, val, (size_t)n * 4) || overlap(in, (size_t)(n * m) * 4, idx, (size_t)n * 4) ||
        overlap(val, (size_t)n * 4, idx, (size_t)n * 4))
        return fail(IFL_EINVAL, "%s: overlapping arrays", what);
    ifl_choice c;
    select_version("segarg.b4", n, m, 0, true, &c);
    if (version != IFL_AUTO) c.version = version;
    if (choice) *choice = c;
    if (n == 0) return IFL_OK;
    if (m == 0) {  // (d, -1) per row
        const uint32_t dbits = canonical_bits(dt, which ? IFL_MAX : IFL_MIN);
        cudaError_t e = ifl::launch_fill(val, n, dbits, (cudaStream_t)stream);
        if (e == cudaSuccess) e = ifl::launch_fill(idx, n, 0xffffffffu, (cudaStream_t)stream);
        return cuda_status(e, what);
    }
    if (c.version == IFL_V_FLAT) {
        const size_t need = ifl::arg_ws_bytes(n, m, IFL_V_FLAT);
        if (!ws || ws_bytes < need)
            return fail(IFL_EWORKSPACE, "%s: V_FLAT needs %zu workspace bytes, got %zu", what, need, ws_bytes);
    }
    ifl::ArgArgs a{in, val, idx, n, m, dt, which, ws, ws_bytes, (cudaStream_t)stream};
    return cuda_status(ifl::launch_arg(a, c.version), what);
}

int ifl_colred(const void* in, void* out, int64_t n, int64_t m, int dt, int op, int f, const void* ne, int version,
               void* ws, size_t ws_bytes, void* stream, ifl_choice* choice) {
    return run_col(false, in, out, n, m, dt, op, f, ne, version, ws, ws_bytes, stream, choice);
}

int ifl_colscan(const void* in, void* out, int64_t n, int64_t m, int dt, int op, int f, const void* ne, int version,
                void* ws, size_t ws_bytes, void* stream, ifl_choice* choice) {
    return run_col(true, in, out, n, m, dt, op, f, ne, version, ws, ws_bytes, stream, choice);
}

int ifl_segred(const void* in, void* out, int64_t n, int64_t m, int dt, int op, int f, const void* ne, int version,
               void* ws, size_t ws_bytes, void* stream, ifl_choice* choice) {
    return run_seg(false, in, out, n, m, dt, op, f, ne, version, ws, ws_bytes, stream, choice);
}

int ifl_segscan(const void* in, void* out, int64_t n, int64_t m, int dt, int op, int f, const void* ne, int reverse,
                int version, void* ws, size_t ws_bytes, void* stream, ifl_choice* choice) {
    if (reverse != 0 && reverse != 1) return fail(IFL_EINVAL, "ifl_segscan: reverse must be 0 or 1");
    return run_seg(true, in, out, n, m, dt, op, f, ne, version, ws, ws_bytes, stream, choice, nullptr, reverse == 1);
}

int ifl_segscan_seeded(const void* in, void* out, int64_t n, int64_t m, int dt, int op, int f, const void* seed,
                       int version, void* ws, size_t ws_bytes, void* stream, ifl_choice* choice) {
    if (n > 0 && m > 0 && !seed) return fail(IFL_EINVAL, "ifl_segscan_seeded: seed is NULL");
    return run_seg(true, in, out, n, m, dt, op, f, nullptr, version, ws, ws_bytes, stream, choice, seed);
}

int ifl_redomap2(const void* A, const void* B, float* C, int64_t n, int64_t m, int64_t p, int in_dt, int b_kmajor,
                 int version, void* ws, size_t ws_bytes, void* stream, ifl_choice* choice) {
    if (n < 0 || m < 0 || p < 0) return fail(IFL_EINVAL, "ifl_redomap2: negative size");
    if (mul_overflows(n, m) || mul_overflows(m, p) || mul_overflows(n, p) || mul_overflows(sat_mul(n, p), m))
        return fail(IFL_EINVAL, "ifl_redomap2: size overflow");
    if (in_dt != IFL_F32 && in_dt != IFL_BF16) return fail(IFL_EUNSUPPORTED, "ifl_redomap2: dtype %d", in_dt);
    if (version < IFL_AUTO || version > IFL_V_ROW_MIDDLE || version == IFL_V_OUTER)
        return fail(IFL_EINVAL, "ifl_redomap2: bad version");
    if (n * p > 0 && !C) return fail(IFL_EINVAL, "ifl_redomap2: C is NULL");
    if (n * m > 0 && !A) return fail(IFL_EINVAL, "ifl_redomap2: A is NULL");
    if (m * p > 0 && !B) return fail(IFL_EINVAL, "ifl_redomap2: B is NULL");
    const char* site = in_dt == IFL_BF16 ? "redomap2.bf16" : "redomap2.f32";
    ifl_choice c;
    mm_tree_select(in_dt, n, m, p, &c);
    if (version != IFL_AUTO) c.version = version;
    if (choice) *choice = c;
    (void)site;
    if (c.version == IFL_V_ROW_MIDDLE && !ifl::mm_row_mid_fits(m))
        return fail(IFL_ENOTFIT, "ifl_redomap2: V_ROW_MIDDLE keeps a row of A in shared memory (m <= %lld)",
                    (long long)ifl::kMmRowMaxM);
    if (n * p == 0) return IFL_OK;
    ifl::MmArgs a{A, B, C, n, m, p, in_dt, b_kmajor ? 1 : 0, ws, ws_bytes, (cudaStream_t)stream};
    // actual need: B transposition (b_kmajor = 0) + split-K partials (V_FLAT)
    const size_t esz = in_dt == IFL_BF16 ? 2 : 4;
    size_t need = ifl::redomap2_ws_bytes(n, m, p, c.version) - (((size_t)m * p * 4 + 255) & ~(size_t)255);
    if (!b_kmajor) need += ((size_t)m * p * esz + 255) & ~(size_t)255;
    if (c.version != IFL_V_FLAT && need == ifl::kMmCntBytes) need = 0;  // the counters serve V_FLAT only
    if (need && (!ws || ws_bytes < need))
        return fail(IFL_EWORKSPACE, "ifl_redomap2: needs %zu workspace bytes, got %zu", need, ws_bytes);
    return cuda_status(ifl::launch_redomap2(c.version, a), "ifl_redomap2");
}

int ifl_tridag(const float* a, const float* b, const float* c, const float* y, float* x, int64_t S, int64_t L,
               int64_t coef_rows, int version, void* ws, size_t ws_bytes, void* stream, ifl_choice* choice) {
    if (S < 0 || L < 0 || coef_rows <= 0) return fail(IFL_EINVAL, "ifl_tridag: bad sizes");
    if (mul_overflows(S, L) || mul_overflows(coef_rows, L)) return fail(IFL_EINVAL, "ifl_tridag: size overflow");
    if (version < IFL_AUTO || version > IFL_V_FLAT) return fail(IFL_EINVAL, "ifl_tridag: bad version");
    if (S * L > 0 && (!a || !b || !c || !y || !x)) return fail(IFL_EINVAL, "ifl_tridag: NULL pointer");
    const bool fits = ifl::tridag_mid_fits(L);
    ifl_choice ch;
    select_version("tridag", S, L, 0, fits, &ch);
    if (version != IFL_AUTO) ch.version = version;
    if (choice) *choice = ch;
    if (ch.version == IFL_V_MIDDLE && !fits)
        return fail(IFL_ENOTFIT, "ifl_tridag: V_MIDDLE does not fit L=%lld in shared memory", (long long)L);
    if (S * L == 0) return IFL_OK;
    const size_t need = ifl::tridag_ws_bytes(coef_rows, L, ch.version);
    if (need && (!ws || ws_bytes < need))
        return fail(IFL_EWORKSPACE, "ifl_tridag: needs %zu workspace bytes, got %zu", need, ws_bytes);
    ifl::TriArgs t{a, b, c, y, x, S, L, coef_rows, ws, ws_bytes, (cudaStream_t)stream};
    return cuda_status(ifl::launch_tridag(ch.version, t), "ifl_tridag");
}

int ifl_lvc(float* xsss, float* ysss, const float* ax, const float* bx, const float* cx, const float* ay,
            const float* by, const float* cy, int64_t numS, int64_t numT, int64_t numX, int64_t numY, int version,
            void* ws, size_t ws_bytes, void* stream, ifl_choice* choice) {
    return ifl::lvc_run(xsss, ysss, ax, bx, cx, ay, by, cy, numS, numT, numX, numY, version, ws, ws_bytes, stream,
                        choice, true);
}

}  // extern "C"

// allow_outer = false: the else-branch of the outermost guard (per-step,
// per-site G3) even when numS >= t0 -- what the tuner times as the alternative.
int ifl::lvc_run(float* xsss, float* ysss, const float* ax, const float* bx, const float* cx, const float* ay,
                 const float* by, const float* cy, int64_t numS, int64_t numT, int64_t numX, int64_t numY,
                 int version, void* ws, size_t ws_bytes, void* stream, ifl_choice* choice, bool allow_outer) {
    if (numS < 0 || numT < 0 || numX < 0 || numY < 0) return fail(IFL_EINVAL, "ifl_lvc: negative size");
    if (mul_overflows(numX, numY) || mul_overflows(numS, numX * numY) || mul_overflows(numS * numX * numY, 4))
        return fail(IFL_EINVAL, "ifl_lvc: size overflow");
    if (version < IFL_AUTO || version > IFL_V_OUTER) return fail(IFL_EINVAL, "ifl_lvc: bad version %d", version);
    const int64_t E = numS * numX * numY;
    if (E > 0 && (!xsss || !ysss || !ax || !bx || !cx || !ay || !by || !cy))
        return fail(IFL_EINVAL, "ifl_lvc: NULL pointer");
    if (E > 0 && overlap(xsss, (size_t)E * 4, ysss, (size_t)E * 4)) return fail(IFL_EINVAL, "ifl_lvc: xsss overlaps ysss");
    const bool outer_fits = numX <= ifl::kLvcMaxL && numY <= ifl::kLvcMaxL;
    // outermost guard of Fig 6c: if numS >= t0 then V_OUTER (reading R1: >=)
    int64_t t0, t_unused;
    ifl_get_thresholds("lvc", &t0, &t_unused);
    ifl_choice ch{IFL_AUTO, numS, numS * numX * numY, t0, t_unused};
    if (allow_outer && numS >= t0 && outer_fits) ch.version = IFL_V_OUTER;
    if (version != IFL_AUTO) ch.version = version;
    if (choice) *choice = ch;
    if (ch.version == IFL_V_OUTER && !outer_fits)
        return fail(IFL_ENOTFIT, "ifl_lvc: V_OUTER keeps systems in registers; needs numX, numY <= %lld",
                    (long long)ifl::kLvcMaxL);
    if (ch.version == IFL_V_MIDDLE && !(ifl::tridag_mid_fits(numX) && ifl::tridag_mid_fits(numY)))
        return fail(IFL_ENOTFIT, "ifl_lvc: V_MIDDLE does not fit");
    if (E == 0 || numT == 0) return IFL_OK;
    const size_t need = ifl_workspace_bytes("lvc", numX, numY, 0, IFL_F32, IFL_AUTO);
    if (!ws || ws_bytes < need) return fail(IFL_EWORKSPACE, "ifl_lvc: needs %zu workspace bytes, got %zu", need, ws_bytes);
    cudaStream_t st = (cudaStream_t)stream;
    float* wx = (float*)ws;
    float* wy = wx + 3 * numX * numY;
    // site x: numS*numX systems of length numY, coefficient rows [numX][numY]; site y mirrored
    ifl::TriArgs tx{ax, bx, cx, xsss, xsss, numS * numX, numY, numX, wx, (size_t)numX * numY * 12, st};
    ifl::TriArgs ty{ay, by, cy, ysss, ysss, numS * numY, numX, numY, wy, (size_t)numX * numY * 12, st};
    int vx = ch.version, vy = ch.version;
    if (ch.version == IFL_AUTO) {  // recurse: G3 of the per-site tridag (Fig 6c versions 1-3)
        vx = select_version("tridag", tx.S, tx.L, 0, ifl::tridag_mid_fits(tx.L), nullptr);
        vy = select_version("tridag", ty.S, ty.L, 0, ifl::tridag_mid_fits(ty.L), nullptr);
    }
    // the (+) scan of the coefficients is loop-invariant: once per site
    cudaError_t e = ifl::launch_tridag_coef(vx == IFL_V_TOP ? 0 : 1, tx);
    if (e == cudaSuccess) e = ifl::launch_tridag_coef(vy == IFL_V_TOP ? 0 : 1, ty);
    if (e != cudaSuccess) return cuda_status(e, "ifl_lvc");
    if (ch.version == IFL_V_OUTER) {
        const int64_t RLx = numX * numY;
        ifl::LvcSite sx{xsss, tx.S, tx.L, tx.coef_rows, wx, wx + RLx, wx + 2 * RLx};
        ifl::LvcSite sy{ysss, ty.S, ty.L, ty.coef_rows, wy, wy + RLx, wy + 2 * RLx};
        return cuda_status(ifl::launch_lvc_outer(sx, sy, numT, st), "ifl_lvc");
    }
    for (int64_t t = 0; t < numT; ++t) {  // one step: both sites, in place
        e = ifl::launch_tridag_solve(vx, tx);
        if (e == cudaSuccess) e = ifl::launch_tridag_solve(vy, ty);
        if (e != cudaSuccess) return cuda_status(e, "ifl_lvc");
    }
    return IFL_OK;
}


