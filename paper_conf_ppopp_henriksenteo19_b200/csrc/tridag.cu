// tridag.cu -- batched tridiagonal solves as three scans (LocVolCalib,
// P:400-420; Fig 6b "tridag as = scan (+) . scan (x) . scan (.)"), in the three
// versions Fig 6c shows:
//   V_TOP    segmap^1 <xs> (tridag xs): one thread per system, the scans run
//            sequentially (they are then just the Thomas recurrences);
//   V_MIDDLE segmap^1 <xs> (segscan^0 ...): a thread group per system, all
//            three scans in registers / shared memory (needs the system to
//            fit: the A-fit clause of P:358);
//   V_FLAT   three segscan^1 over the flattened S*L array in global memory:
//            y' is written out by the forward scan and read back by the
//            backward one ("at least two global accesses per element for each
//            scan").
// The paper does not give the operators; reading R8:
//   (+)  2x2 matrix products, M_j = [[b_j, -a_j c_{j-1}], [1, 0]]; with
//        P_j = M_j...M_0 the eliminated diagonal is beta_j = P_j[0][0] /
//        P_j[1][0]; every product is renormalised (scale-invariant ratio);
//   (x)  affine maps y'_j = alpha_j y'_{j-1} + y_j, alpha_j = -a_j / beta_{j-1};
//   (.)  reversed affine maps x_j = delta_j x_{j+1} + y'_j / beta_j,
//        delta_j = -c_j / beta_j.
// Coefficients are [R][L], shared by every system s with s % R == r (R9), so
// the (+) scan runs once per coefficient row into the workspace (invbeta,
// alpha, delta), and the per-system work is the two affine scans.  alpha_0 = 0
// and delta_{L-1} = 0, so the affine scans reset at system boundaries on their
// own: the flattened scans need no segment flags.
#include <algorithm>

#include "common.cuh"
#include "ifl_internal.h"

namespace ifl {

// ------------------------------------------------------------ operators

struct Aff {  // x -> a*x + g
    float a, g;
};
// compose: newer o older
__device__ __forceinline__ Aff aff_after(Aff newer, Aff older) {
    return {newer.a * older.a, fmaf(newer.a, older.g, newer.g)};
}

struct Mat2 {
    float m00, m01, m10, m11;
};
__device__ __forceinline__ Mat2 mat_mul(Mat2 y, Mat2 x) {  // y * x (newer on the left)
    Mat2 r{fmaf(y.m00, x.m00, y.m01 * x.m10), fmaf(y.m00, x.m01, y.m01 * x.m11),
           fmaf(y.m10, x.m00, y.m11 * x.m10), fmaf(y.m10, x.m01, y.m11 * x.m11)};
    const float s = fabsf(r.m00) + fabsf(r.m01) + fabsf(r.m10) + fabsf(r.m11);
    const float inv = s > 0.f ? 1.0f / s : 1.0f;
    return {r.m00 * inv, r.m01 * inv, r.m10 * inv, r.m11 * inv};
}
__device__ __forceinline__ Mat2 mat_id() { return {1.f, 0.f, 0.f, 1.f}; }

// ------------------------------------------------- scan (+): coefficients

// V_TOP: one thread per coefficient row, sequential (the Thomas recurrence).
__global__ void tridag_coef_seq(const float* __restrict__ a, const float* __restrict__ b, const float* __restrict__ c,
                                float* __restrict__ invb, float* __restrict__ alpha, float* __restrict__ delta,
                                int64_t R, int64_t L) {
    for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < R; r += (int64_t)gridDim.x * blockDim.x) {
        const float* ar = a + r * L;
        const float* br = b + r * L;
        const float* cr = c + r * L;
        float beta = br[0];
        alpha[r * L] = 0.f;
        for (int64_t j = 0; j < L; ++j) {
            if (j > 0) {
                const float al = -ar[j] / beta;
                alpha[r * L + j] = al;
                beta = fmaf(al, cr[j - 1], br[j]);  // b_j - a_j c_{j-1} / beta_{j-1}
            }
            invb[r * L + j] = 1.0f / beta;
            delta[r * L + j] = j + 1 < L ? -cr[j] / beta : 0.f;
        }
    }
}

// V_MIDDLE / V_FLAT: a CTA per coefficient row, the normalised 2x2 matrix
// scan of the paper's first scan, in shared memory.  256 threads, each a
// contiguous run of ceil(L/256) rows.
__global__ void __launch_bounds__(256) tridag_coef_mat2(const float* __restrict__ a, const float* __restrict__ b,
                                                        const float* __restrict__ c, float* __restrict__ invb,
                                                        float* __restrict__ alpha, float* __restrict__ delta,
                                                        int64_t L) {
    __shared__ Mat2 wsum[8];
    __shared__ float sbeta_prev[257];
    const int64_t r = blockIdx.x;
    const float* ar = a + r * L;
    const float* br = b + r * L;
    const float* cr = c + r * L;
    const int t = threadIdx.x, lane = t & 31, w = t >> 5;
    const int64_t per = ceil_div(L, 256);
    const int64_t j0 = t * per, j1 = std::min(L, j0 + per);
    auto Mj = [&](int64_t j) -> Mat2 {
        return j == 0 ? Mat2{br[0], 0.f, 1.f, 0.f} : Mat2{br[j], -ar[j] * cr[j - 1], 1.f, 0.f};
    };
    // thread aggregate (product of its run, newer on the left)
    Mat2 agg = mat_id();
    for (int64_t j = j0; j < j1; ++j) agg = mat_mul(Mj(j), agg);
    // inclusive warp scan, then across warps
    Mat2 inc = agg;
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
        Mat2 o{__shfl_up_sync(0xffffffffu, inc.m00, off), __shfl_up_sync(0xffffffffu, inc.m01, off),
               __shfl_up_sync(0xffffffffu, inc.m10, off), __shfl_up_sync(0xffffffffu, inc.m11, off)};
        if (lane >= off) inc = mat_mul(inc, o);
    }
    if (lane == 31) wsum[w] = inc;
    Mat2 ex{__shfl_up_sync(0xffffffffu, inc.m00, 1), __shfl_up_sync(0xffffffffu, inc.m01, 1),
            __shfl_up_sync(0xffffffffu, inc.m10, 1), __shfl_up_sync(0xffffffffu, inc.m11, 1)};
    if (lane == 0) ex = mat_id();
    __syncthreads();
    Mat2 pre = mat_id();
    for (int k = 0; k < w; ++k) pre = mat_mul(wsum[k], pre);
    ex = mat_mul(ex, pre);
    // walk the run: P_j = M_j ... M_0, beta_j = P_j[0][0] / P_j[1][0]
    Mat2 P = ex;
    float beta_last = 0.f;
    for (int64_t j = j0; j < j1; ++j) {
        P = mat_mul(Mj(j), P);
        const float beta = P.m00 / P.m10;
        invb[r * L + j] = 1.0f / beta;
        delta[r * L + j] = j + 1 < L ? -cr[j] / beta : 0.f;
        beta_last = beta;
    }
    sbeta_prev[t + 1] = beta_last;  // beta at the end of this thread's run
    __syncthreads();
    // alpha_j = -a_j / beta_{j-1}: the first item of a run needs the previous run's beta
    for (int64_t j = j0; j < j1; ++j) {
        float bprev;
        if (j == 0) {
            alpha[r * L] = 0.f;
            continue;
        }
        if (j == j0) {
            int q = t;  // nearest preceding non-empty run
            while (q > 0 && (int64_t)(q - 1) * per >= L) --q;
            bprev = sbeta_prev[q];
        } else {
            bprev = 1.0f / invb[r * L + j - 1];
        }
        alpha[r * L + j] = -ar[j] / bprev;
    }
}

// ---------------------------------------------------------------- V_TOP

// One thread per system; the forward scan stores y' into x, the backward
// scan overwrites it with x.  Coefficient arrays are tiny and L2-resident.
__global__ void __launch_bounds__(256) tridag_top_kernel(const float* __restrict__ y, float* __restrict__ x,
                                                         const float* __restrict__ invb, const float* __restrict__ alpha,
                                                         const float* __restrict__ delta, int64_t S, int64_t L,
                                                         int64_t R) {
    for (int64_t s = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; s < S; s += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = s % R;
        const float* ys = y + s * L;
        float* xs = x + s * L;
        const float* al = alpha + r * L;
        const float* ib = invb + r * L;
        const float* de = delta + r * L;
        float v = 0.f;
        for (int64_t j = 0; j < L; ++j) {  // (x): y'_j = alpha_j y'_{j-1} + y_j
            v = fmaf(__ldg(al + j), v, __ldg(ys + j));
            xs[j] = v;
        }
        float u = 0.f;
        for (int64_t j = L - 1; j >= 0; --j) {  // (.): x_j = delta_j x_{j+1} + y'_j / beta_j
            u = fmaf(__ldg(de + j), u, xs[j] * __ldg(ib + j));
            xs[j] = u;
        }
    }
}

// ------------------------------------------------------------- V_MIDDLE

constexpr int kTriItems = 8;

// Group-wide exclusive scan of affine maps (older lanes first).  G threads
// per group; G <= 32 uses shuffles only, larger groups go through shared
// memory (warp totals).  REV scans from the last lane backwards.
template <bool REV, int G>
__device__ __forceinline__ Aff group_exscan(Aff v, Aff* wtot, Aff& total) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    constexpr int width = G < 32 ? G : 32;
    const int gl = threadIdx.x % width;
    Aff inc = v;
#pragma unroll
    for (int off = 1; off < width; off <<= 1) {
        const float oa = REV ? __shfl_down_sync(0xffffffffu, inc.a, off, width) : __shfl_up_sync(0xffffffffu, inc.a, off, width);
        const float og = REV ? __shfl_down_sync(0xffffffffu, inc.g, off, width) : __shfl_up_sync(0xffffffffu, inc.g, off, width);
        const bool ok = REV ? (gl + off < width) : (gl >= off);
        if (ok) inc = aff_after(inc, Aff{oa, og});
    }
    Aff ex;
    ex.a = REV ? __shfl_down_sync(0xffffffffu, inc.a, 1, width) : __shfl_up_sync(0xffffffffu, inc.a, 1, width);
    ex.g = REV ? __shfl_down_sync(0xffffffffu, inc.g, 1, width) : __shfl_up_sync(0xffffffffu, inc.g, 1, width);
    const bool first = REV ? (gl == width - 1) : (gl == 0);
    if (first) ex = Aff{1.f, 0.f};
    if constexpr (G <= 32) {
        const int src = REV ? 0 : width - 1;
        total = Aff{__shfl_sync(0xffffffffu, inc.a, src, width), __shfl_sync(0xffffffffu, inc.g, src, width)};
        return ex;
    }
    constexpr int wpg = G >> 5;
    const int w0 = (threadIdx.x / G) * wpg;
    if (REV ? lane == 0 : lane == 31) wtot[w] = inc;
    __syncthreads();
    Aff before{1.f, 0.f};
    total = Aff{1.f, 0.f};
#pragma unroll
    for (int k = 0; k < wpg; ++k) {
        const int kk = REV ? (wpg - 1 - k) : k;  // oldest first
        const Aff t = wtot[w0 + kk];
        if (REV ? (w0 + kk > w) : (w0 + kk < w)) before = aff_after(t, before);
        total = aff_after(t, total);
    }
    __syncthreads();
    return aff_after(ex, before);
}

int tridag_group(int64_t L) {
    int64_t g = 1;
    while (g < 256 && g * kTriItems < L) g <<= 1;
    return (int)std::max<int64_t>(g, 1);
}

// A group of G threads (IT items each) solves `spg` systems that share one
// coefficient row r (s = r + R*q, R9): the row's alpha / invbeta / delta are
// loaded once into registers, and the next system's y is prefetched while
// the current one is scanned.  Consecutive groups take consecutive r, so a
// warp-wide load still covers adjacent systems.
template <int IT, int G>
__global__ void __launch_bounds__(256) tridag_mid_kernel(const float* __restrict__ y, float* __restrict__ x,
                                                         const float* __restrict__ invb, const float* __restrict__ alpha,
                                                         const float* __restrict__ delta, int64_t S, int64_t L,
                                                         int64_t R, int spg) {
    __shared__ Aff wtot[8];
    const int g = threadIdx.x % G;
    const int64_t gid = (int64_t)blockIdx.x * (blockDim.x / G) + threadIdx.x / G;
    const int64_t qc = gid / R, r = gid - qc * R, q0 = qc * spg;
    // systems of this group: s = r + R*(q0 + i), i < nq
    const int nq = r + R * q0 < S ? (int)std::min<int64_t>(spg, (S - 1 - r) / R + 1 - q0) : 0;
    const bool live = nq > 0;  // (a dead group still joins the group scans)
    const int64_t j0 = (int64_t)g * IT;
    float yv[IT], yn[IT], al[IT], ib[IT], de[IT];
    const bool vec = (L % 4 == 0) && (j0 + IT <= L) && (((uintptr_t)y & 15) == 0) && (((uintptr_t)x & 15) == 0) &&
                     (((uintptr_t)(alpha + r * L) & 15) == 0);
    if (vec && live) {
#pragma unroll
        for (int k = 0; k < IT; k += 4) {
            const float4 a4 = __ldg(reinterpret_cast<const float4*>(alpha + r * L + j0 + k));
            const float4 i4 = __ldg(reinterpret_cast<const float4*>(invb + r * L + j0 + k));
            const float4 d4 = __ldg(reinterpret_cast<const float4*>(delta + r * L + j0 + k));
            al[k] = a4.x; al[k + 1] = a4.y; al[k + 2] = a4.z; al[k + 3] = a4.w;
            ib[k] = i4.x; ib[k + 1] = i4.y; ib[k + 2] = i4.z; ib[k + 3] = i4.w;
            de[k] = d4.x; de[k + 1] = d4.y; de[k + 2] = d4.z; de[k + 3] = d4.w;
        }
    } else {
#pragma unroll
        for (int k = 0; k < IT; ++k) {
            const bool ok = live && j0 + k < L;
            al[k] = ok ? __ldg(alpha + r * L + j0 + k) : 1.f;
            ib[k] = ok ? __ldg(invb + r * L + j0 + k) : 0.f;
            de[k] = ok ? __ldg(delta + r * L + j0 + k) : 1.f;
        }
    }
    const int64_t stride = R * L;
    const float* yp = y + (live ? (r + R * q0) * L : 0) + j0;
    float* xp = x + (live ? (r + R * q0) * L : 0) + j0;
    auto load_y = [&](int i, float (&dst)[IT]) {
        const bool ok = i < nq;
        const float* ys = yp + (ok ? i * stride : 0);
        if (vec && ok) {
#pragma unroll
            for (int k = 0; k < IT; k += 4) {
                const float4 y4 = ldg_stream4<float>(ys + k);
                dst[k] = y4.x; dst[k + 1] = y4.y; dst[k + 2] = y4.z; dst[k + 3] = y4.w;
            }
        } else {
#pragma unroll
            for (int k = 0; k < IT; ++k) dst[k] = (ok && j0 + k < L) ? __ldg(ys + k) : 0.f;
        }
    };
    load_y(0, yv);
    // every group runs the same trip count so that group scans over shared
    // memory (G > 32) stay block-uniform
    for (int i = 0; i < spg; ++i) {
        if (spg > 1) load_y(i + 1, yn);  // prefetch the next system of this row
        // (x) forward: thread composite of its items, group exclusive prefix, apply
        Aff f{1.f, 0.f};
#pragma unroll
        for (int k = 0; k < IT; ++k) f = aff_after(Aff{al[k], yv[k]}, f);
        Aff tot;
        const Aff pf = group_exscan<false, G>(f, wtot, tot);
        float v = pf.g;  // y' before this thread's first item (the prefix applied to 0)
#pragma unroll
        for (int k = 0; k < IT; ++k) {
            v = fmaf(al[k], v, yv[k]);
            yv[k] = v * ib[k];  // epsilon_j = y'_j / beta_j
        }
        // (.) backward
        Aff bk{1.f, 0.f};
#pragma unroll
        for (int k = IT - 1; k >= 0; --k) bk = aff_after(Aff{de[k], yv[k]}, bk);
        const Aff pb = group_exscan<true, G>(bk, wtot, tot);
        float u = pb.g;
#pragma unroll
        for (int k = IT - 1; k >= 0; --k) {
            u = fmaf(de[k], u, yv[k]);
            yv[k] = u;
        }
        if (i < nq) {
            float* xs = xp + i * stride;
            if (vec) {
#pragma unroll
                for (int k = 0; k < IT; k += 4)
                    __stcs(reinterpret_cast<float4*>(xs + k), make_float4(yv[k], yv[k + 1], yv[k + 2], yv[k + 3]));
            } else {
#pragma unroll
                for (int k = 0; k < IT; ++k)
                    if (j0 + k < L) xs[k] = yv[k];
            }
        }
#pragma unroll
        for (int k = 0; k < IT; ++k) yv[k] = yn[k];
    }
}

bool tridag_mid_fits(int64_t L) { return L >= 1 && L <= 256 * 16; }

// --------------------------------------------------------------- V_FLAT

// One affine scan over the flattened S*L array.  A CTA takes a tile of whole
// systems (tile = L * floor(4096 / L), or one system when L > 4096), 256
// threads each a contiguous run; the CTA scans the thread composites (no
// segment flags: alpha_0 = 0 / delta_{L-1} = 0 reset the maps).
// FWD: y'_j = alpha_j y'_{j-1} + y_j   (reads y, writes y' into x)
// BWD: x_j = delta_j x_{j+1} + y'_j / beta_j   (reads and writes x)
template <bool FWD>
__global__ void __launch_bounds__(256) tridag_flat_kernel(const float* __restrict__ y, float* __restrict__ x,
                                                          const float* __restrict__ invb,
                                                          const float* __restrict__ alpha,
                                                          const float* __restrict__ delta, int64_t S, int64_t L,
                                                          int64_t R, int64_t sys_per_tile) {
    __shared__ Aff wtot[8];
    const int64_t s0 = (int64_t)blockIdx.x * sys_per_tile;
    const int64_t nsys = std::min(sys_per_tile, S - s0);
    const int64_t base = s0 * L, cnt = nsys * L;
    const int64_t per = ceil_div(cnt, 256);
    const int64_t e0 = threadIdx.x * per, e1 = std::min(cnt, e0 + per);
    // walk (system, position) incrementally: one division per thread, not per element
    auto walk = [&](auto&& body) {
        if (e0 >= e1) return;
        if (FWD) {
            int64_t s = s0 + e0 / L, j = e0 % L, r = s % R;
            for (int64_t e = e0; e < e1; ++e) {
                body(base + e, r * L + j);
                if (++j == L) {
                    j = 0;
                    if (++r == R) r = 0;
                }
            }
        } else {
            int64_t s = s0 + (e1 - 1) / L, j = (e1 - 1) % L, r = s % R;
            for (int64_t e = e1 - 1; e >= e0; --e) {
                body(base + e, r * L + j);
                if (j-- == 0) {
                    j = L - 1;
                    r = (r == 0) ? R - 1 : r - 1;
                }
            }
        }
    };
    auto coef = [&](int64_t gi, int64_t ci, float& mm, float& add) {
        if (FWD) {
            mm = __ldg(alpha + ci);
            add = __ldg(y + gi);
        } else {
            mm = __ldg(delta + ci);
            add = x[gi] * __ldg(invb + ci);
        }
    };
    Aff f{1.f, 0.f};
    walk([&](int64_t gi, int64_t ci) {
        float mm, ad;
        coef(gi, ci, mm, ad);
        f = aff_after(Aff{mm, ad}, f);
    });
    Aff tot;
    const Aff pf = group_exscan<!FWD, 256>(f, wtot, tot);
    float v = pf.g;
    walk([&](int64_t gi, int64_t ci) {
        float mm, ad;
        coef(gi, ci, mm, ad);
        v = fmaf(mm, v, ad);
        x[gi] = v;
    });
}

// Fast path of the flattened scans when L is a multiple of 16 dividing the
// 4096-element tile: every thread's 16 consecutive elements lie in one
// system, so y / x and the coefficient runs move as 128-bit words.
template <bool FWD>
__global__ void __launch_bounds__(256) tridag_flat16_kernel(const float* __restrict__ y, float* __restrict__ x,
                                                            const float* __restrict__ invb,
                                                            const float* __restrict__ alpha,
                                                            const float* __restrict__ delta, int64_t S, int64_t L,
                                                            int64_t R) {
    __shared__ Aff wtot[8];
    constexpr int IT = 16;
    const int64_t e0 = (int64_t)blockIdx.x * 4096 + threadIdx.x * IT;  // global flat index of the run
    const bool live = e0 < S * L;
    const int64_t s = live ? e0 / L : 0, j0 = live ? e0 - s * L : 0, r = s % R;
    float mm[IT], ad[IT];
    if (live) {
#pragma unroll
        for (int q = 0; q < IT; q += 4) {
            const float4 c4 = __ldg(reinterpret_cast<const float4*>((FWD ? alpha : delta) + r * L + j0 + q));
            mm[q] = c4.x; mm[q + 1] = c4.y; mm[q + 2] = c4.z; mm[q + 3] = c4.w;
            if (FWD) {
                const float4 y4 = __ldg(reinterpret_cast<const float4*>(y + e0 + q));
                ad[q] = y4.x; ad[q + 1] = y4.y; ad[q + 2] = y4.z; ad[q + 3] = y4.w;
            } else {
                const float4 x4 = *reinterpret_cast<const float4*>(x + e0 + q);
                const float4 i4 = __ldg(reinterpret_cast<const float4*>(invb + r * L + j0 + q));
                ad[q] = x4.x * i4.x; ad[q + 1] = x4.y * i4.y; ad[q + 2] = x4.z * i4.z; ad[q + 3] = x4.w * i4.w;
            }
        }
    } else {
#pragma unroll
        for (int q = 0; q < IT; ++q) {
            mm[q] = 1.f;
            ad[q] = 0.f;
        }
    }
    Aff f{1.f, 0.f};
    if (FWD) {
#pragma unroll
        for (int q = 0; q < IT; ++q) f = aff_after(Aff{mm[q], ad[q]}, f);
    } else {
#pragma unroll
        for (int q = IT - 1; q >= 0; --q) f = aff_after(Aff{mm[q], ad[q]}, f);
    }
    Aff tot;
    const Aff pf = group_exscan<!FWD, 256>(f, wtot, tot);
    float v = pf.g;
    if (FWD) {
#pragma unroll
        for (int q = 0; q < IT; ++q) ad[q] = v = fmaf(mm[q], v, ad[q]);
    } else {
#pragma unroll
        for (int q = IT - 1; q >= 0; --q) ad[q] = v = fmaf(mm[q], v, ad[q]);
    }
    if (live) {
#pragma unroll
        for (int q = 0; q < IT; q += 4)
            *reinterpret_cast<float4*>(x + e0 + q) = make_float4(ad[q], ad[q + 1], ad[q + 2], ad[q + 3]);
    }
}

// ------------------------------------------------------------------ launch

// invbeta, alpha, delta: one float each per coefficient element ([R][L])
size_t tridag_ws_bytes(int64_t R, int64_t L, int version) {
    (void)version;
    return (size_t)R * L * 3 * sizeof(float);
}

// The (+) scan of every coefficient row into the workspace (invbeta, alpha,
// delta): sequential per row for V_TOP, the CTA-wide 2x2 matrix scan otherwise.
cudaError_t launch_tridag_coef(int version, const TriArgs& t) {
    const int64_t R = t.coef_rows, L = t.L;
    float* invb = (float*)t.ws;
    float* alpha = invb + R * L;
    float* delta = alpha + R * L;
    if (version == 0) {
        const int g = (int)std::min<int64_t>(ceil_div(R, 128), 148 * 8);
        tridag_coef_seq<<<g, 128, 0, t.stream>>>(t.a, t.b, t.c, invb, alpha, delta, R, L);
    } else {
        tridag_coef_mat2<<<(unsigned)R, 256, 0, t.stream>>>(t.a, t.b, t.c, invb, alpha, delta, L);
    }
    return cudaGetLastError();
}

cudaError_t launch_tridag(int version, const TriArgs& t) {
    cudaError_t e = launch_tridag_coef(version, t);
    if (e != cudaSuccess) return e;
    return launch_tridag_solve(version, t);
}

// The per-system (x) / (.) scans, given the coefficient scans in the workspace.
cudaError_t launch_tridag_solve(int version, const TriArgs& t) {
    const int64_t R = t.coef_rows, L = t.L, S = t.S;
    float* invb = (float*)t.ws;
    float* alpha = invb + R * L;
    float* delta = alpha + R * L;
    cudaError_t e;
    if (version == 0) {
        const int g = (int)std::min<int64_t>(ceil_div(S, 256), 148 * 16);
        tridag_top_kernel<<<g, 256, 0, t.stream>>>(t.y, t.x, invb, alpha, delta, S, L, R);
        return cudaGetLastError();
    }
    if (version == 1) {
        const int G = tridag_group(L);
        const int B = std::max(G, 32) > 256 ? G : 256;
        // systems per group: as many as keep ~8 CTAs' worth of groups on
        // every SM (one coefficient load then serves them all)
        const int64_t Rr = std::min(R, S), Q = ceil_div(S, Rr);
        const int64_t want_groups = (int64_t)148 * 8 * (B / G);
        const int spg = (int)std::max<int64_t>(1, std::min<int64_t>({(int64_t)8, Q, (Rr * Q) / want_groups}));
        const int64_t groups = Rr * ceil_div(Q, spg);
        const int64_t grid = ceil_div(groups, B / G);
        const int64_t it = ceil_div(L, G);
        auto go = [&](auto kern) {
            kern<<<(unsigned)grid, B, 0, t.stream>>>(t.y, t.x, invb, alpha, delta, S, L, Rr, spg);
        };
        switch (G) {
            case 1: go(it <= 4 ? tridag_mid_kernel<4, 1> : tridag_mid_kernel<8, 1>); break;
            case 2: go(it <= 4 ? tridag_mid_kernel<4, 2> : tridag_mid_kernel<8, 2>); break;
            case 4: go(it <= 4 ? tridag_mid_kernel<4, 4> : tridag_mid_kernel<8, 4>); break;
            case 8: go(it <= 4 ? tridag_mid_kernel<4, 8> : tridag_mid_kernel<8, 8>); break;
            case 16: go(it <= 4 ? tridag_mid_kernel<4, 16> : tridag_mid_kernel<8, 16>); break;
            case 32: go(it <= 4 ? tridag_mid_kernel<4, 32> : tridag_mid_kernel<8, 32>); break;
            case 64: go(it <= 4 ? tridag_mid_kernel<4, 64> : tridag_mid_kernel<8, 64>); break;
            case 128: go(it <= 4 ? tridag_mid_kernel<4, 128> : tridag_mid_kernel<8, 128>); break;
            default:
                go(it <= 4 ? tridag_mid_kernel<4, 256> : it <= 8 ? tridag_mid_kernel<8, 256> : tridag_mid_kernel<16, 256>);
        }
        return cudaGetLastError();
    }
    const bool aligned = ((uintptr_t)t.y % 16 == 0) && ((uintptr_t)t.x % 16 == 0) && ((uintptr_t)t.ws % 16 == 0);
    if (aligned && L % 16 == 0 && 4096 % L == 0) {
        const int64_t grid16 = ceil_div(S * L, 4096);
        tridag_flat16_kernel<true><<<(unsigned)grid16, 256, 0, t.stream>>>(t.y, t.x, invb, alpha, delta, S, L, R);
        if ((e = cudaGetLastError()) != cudaSuccess) return e;
        tridag_flat16_kernel<false><<<(unsigned)grid16, 256, 0, t.stream>>>(t.y, t.x, invb, alpha, delta, S, L, R);
        return cudaGetLastError();
    }
    const int64_t spt = std::max<int64_t>(1, 4096 / L);
    const int64_t grid = ceil_div(S, spt);
    tridag_flat_kernel<true><<<(unsigned)grid, 256, 0, t.stream>>>(t.y, t.x, invb, alpha, delta, S, L, R, spt);
    if ((e = cudaGetLastError()) != cudaSuccess) return e;
    tridag_flat_kernel<false><<<(unsigned)grid, 256, 0, t.stream>>>(t.y, t.x, invb, alpha, delta, S, L, R, spt);
    return cudaGetLastError();
}

}  // namespace ifl
