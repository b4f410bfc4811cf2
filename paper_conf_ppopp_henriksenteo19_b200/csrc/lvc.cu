// lvc.cu -- V_OUTER of the whole LocVolCalib-shaped program (Fig 6a, P:400;
// the `if numS > t0 then ...` branch of Fig 6c).
//
//   map (\xss yss -> loop (xss, yss) for t < numT do (map tridag xss, map tridag yss))
//
// The two sites never read each other's array, so the loop distributes over
// them, and every system's numT solves depend only on that system: the loop
// moves inside the per-system map (map-loop interchange, the reverse of G7,
// P:404).  V_OUTER therefore runs ONE kernel for the whole program: a group
// of G lanes owns one system for all numT steps, holding its IT*G values and
// its coefficient row's (alpha, 1/beta, delta) in registers, so HBM sees one
// read and one write per element for the whole run instead of one per step.
// Each step is tridag's (x) forward and (.) backward affine scans (the (+)
// scan of the coefficients is loop-invariant and done once by
// launch_tridag_coef).  Both sites run in the same launch: blocks [0, gx)
// take the x-site, the rest the y-site.
#include <stdlib.h>

#include <algorithm>

#include "common.cuh"
#include "ifl_internal.h"

namespace ifl {

namespace {

constexpr int kLvcThreads = 256;
#ifndef IFL_LVC_CHAINS
#define IFL_LVC_CHAINS 2  // independent scan chains per lane (2 = the half chains of round 1)
#endif

template <int IT>
__global__ void __launch_bounds__(kLvcThreads) lvc_outer_kernel(LvcSite sx, LvcSite sy, int gx, int Gx, int Gy,
                                                                int64_t numT) {
    const bool isx = (int)blockIdx.x < gx;
    const LvcSite& st = isx ? sx : sy;
    const int G = isx ? Gx : Gy;
    const int64_t blk = isx ? blockIdx.x : blockIdx.x - gx;
    const int gl = threadIdx.x & (G - 1);
    const int64_t s = blk * (kLvcThreads / G) + threadIdx.x / G;
    const int64_t L = st.L;
    const bool live = s < st.S;  // dead groups still take part in the shuffles
    const int64_t j0 = (int64_t)gl * IT;
    const int64_t r = live ? s % st.R : 0;
    float* xs = st.xs + (live ? s * L : 0);
    const float* al_r = st.alpha + r * L;
    const float* ib_r = st.invb + r * L;
    const float* de_r = st.delta + r * L;
    float yv[IT], al[IT], ib[IT], de[IT];
    const bool vec = live && (L % 4 == 0) && (j0 + IT <= L) && (((uintptr_t)st.xs & 15) == 0) &&
                     (((uintptr_t)st.alpha & 15) == 0) && (((uintptr_t)st.invb & 15) == 0) &&
                     (((uintptr_t)st.delta & 15) == 0);
    if (vec) {
#pragma unroll
        for (int k = 0; k < IT; k += 4) {
            const float4 a4 = __ldg(reinterpret_cast<const float4*>(al_r + j0 + k));
            const float4 i4 = __ldg(reinterpret_cast<const float4*>(ib_r + j0 + k));
            const float4 d4 = __ldg(reinterpret_cast<const float4*>(de_r + j0 + k));
            const float4 y4 = *reinterpret_cast<const float4*>(xs + j0 + k);
            al[k] = a4.x; al[k + 1] = a4.y; al[k + 2] = a4.z; al[k + 3] = a4.w;
            ib[k] = i4.x; ib[k + 1] = i4.y; ib[k + 2] = i4.z; ib[k + 3] = i4.w;
            de[k] = d4.x; de[k + 1] = d4.y; de[k + 2] = d4.z; de[k + 3] = d4.w;
            yv[k] = y4.x; yv[k + 1] = y4.y; yv[k + 2] = y4.z; yv[k + 3] = y4.w;
        }
    } else {
#pragma unroll
        for (int k = 0; k < IT; ++k) {  // dead items are identity maps: (1, 0) forward and backward
            const bool ok = live && j0 + k < L;
            al[k] = ok ? __ldg(al_r + j0 + k) : 1.f;
            ib[k] = ok ? __ldg(ib_r + j0 + k) : 0.f;
            de[k] = ok ? __ldg(de_r + j0 + k) : 1.f;
            yv[k] = ok ? xs[j0 + k] : 0.f;
        }
    }
    // Loop-invariant parts of both affine scans, computed once: an affine
    // map's slope depends only on the coefficients, so every product of
    // slopes (within the lane, and at each shuffle round of the group scan)
    // is the same in all numT steps; each step only carries the offsets g.
    //   forward  y'_j = alpha_j y'_{j-1} + y_j: lane-local scan from 0, then
    //            y'_k = loc_k + P_k * p  with P_k = alpha_{j0} ... alpha_{j0+k}
    //            and p the group-exclusive prefix (the value entering the lane);
    //   backward x_j = delta_j x_{j+1} + eps_j, mirrored with suffix products.
    // The lane's items are scanned as NC independent chains of C = IT / NC
    // items (NC-fold instruction-level parallelism), joined with their slope
    // products:
    //   Q[k] = alpha_{chain start} ... alpha_{j0+k},  QE[c] = Q at chain c's end
    //   E[k] = delta_{j0+k} ... delta_{chain end},    EE[c] = E at chain c's start
    constexpr int NC = IFL_LVC_CHAINS, C = IT / NC;
    static_assert(IT % NC == 0 && C >= 1, "chains");
    float Q[IT], E[IT], QE[NC], EE[NC];
#pragma unroll
    for (int c = 0; c < NC; ++c) {
        float pr = 1.f;
#pragma unroll
        for (int k = c * C; k < (c + 1) * C; ++k) Q[k] = pr = pr * al[k];
        QE[c] = pr;
        pr = 1.f;
#pragma unroll
        for (int k = (c + 1) * C - 1; k >= c * C; --k) E[k] = pr = pr * de[k];
        EE[c] = pr;
    }
    float raf[5], rab[5];  // slope of the running inclusive map before each shuffle round
    {
        float af = 1.f, ab = 1.f;
#pragma unroll
        for (int c = 0; c < NC; ++c) {
            af *= QE[c];
            ab *= EE[c];
        }
#pragma unroll
        for (int r = 0; r < 5; ++r) {
            const int off = 1 << r;
            raf[r] = af;
            rab[r] = ab;
            if (off < G) {
                const float of = __shfl_up_sync(0xffffffffu, af, off, G);
                const float ob = __shfl_down_sync(0xffffffffu, ab, off, G);
                if (gl >= off) af *= of;
                if (gl + off < G) ab *= ob;
            }
        }
    }
    for (int64_t t = 0; t < numT; ++t) {
        // (x) forward: chains from 0, then the lane total e = QE[c] e + g_c
        float gc[NC];
#pragma unroll
        for (int c = 0; c < NC; ++c) gc[c] = 0.f;
#pragma unroll
        for (int k = 0; k < C; ++k)
#pragma unroll
            for (int c = 0; c < NC; ++c) yv[c * C + k] = gc[c] = fmaf(al[c * C + k], gc[c], yv[c * C + k]);
        float g = gc[0];
#pragma unroll
        for (int c = 1; c < NC; ++c) g = fmaf(QE[c], g, gc[c]);
#pragma unroll
        for (int r = 0; r < 5; ++r) {
            const int off = 1 << r;
            if (off < G) {
                const float o = __shfl_up_sync(0xffffffffu, g, off, G);
                if (gl >= off) g = fmaf(raf[r], o, g);
            }
        }
        float p = __shfl_up_sync(0xffffffffu, g, 1, G);
        if (gl == 0) p = 0.f;
        float vin[NC];  // y' entering each chain
        vin[0] = p;
#pragma unroll
        for (int c = 1; c < NC; ++c) vin[c] = fmaf(QE[c - 1], vin[c - 1], gc[c - 1]);
#pragma unroll
        for (int k = 0; k < C; ++k)
#pragma unroll
            for (int c = 0; c < NC; ++c)
                yv[c * C + k] = fmaf(Q[c * C + k], vin[c], yv[c * C + k]) * ib[c * C + k];  // eps_j = y'_j / beta_j
        // (.) backward: chains from 0 at their right ends, lane total from the right
        float hc[NC];
#pragma unroll
        for (int c = 0; c < NC; ++c) hc[c] = 0.f;
#pragma unroll
        for (int k = C - 1; k >= 0; --k)
#pragma unroll
            for (int c = 0; c < NC; ++c) yv[c * C + k] = hc[c] = fmaf(de[c * C + k], hc[c], yv[c * C + k]);
        float h = hc[NC - 1];
#pragma unroll
        for (int c = NC - 2; c >= 0; --c) h = fmaf(EE[c], h, hc[c]);
#pragma unroll
        for (int r = 0; r < 5; ++r) {
            const int off = 1 << r;
            if (off < G) {
                const float o = __shfl_down_sync(0xffffffffu, h, off, G);
                if (gl + off < G) h = fmaf(rab[r], o, h);
            }
        }
        float u = __shfl_down_sync(0xffffffffu, h, 1, G);
        if (gl == G - 1) u = 0.f;
        float win[NC];  // x entering each chain from the right
        win[NC - 1] = u;
#pragma unroll
        for (int c = NC - 2; c >= 0; --c) win[c] = fmaf(EE[c + 1], win[c + 1], hc[c + 1]);
#pragma unroll
        for (int k = 0; k < C; ++k)
#pragma unroll
            for (int c = 0; c < NC; ++c) yv[c * C + k] = fmaf(E[c * C + k], win[c], yv[c * C + k]);
    }
    if (vec) {
#pragma unroll
        for (int k = 0; k < IT; k += 4)
            *reinterpret_cast<float4*>(xs + j0 + k) = make_float4(yv[k], yv[k + 1], yv[k + 2], yv[k + 3]);
    } else if (live) {
#pragma unroll
        for (int k = 0; k < IT; ++k)
            if (j0 + k < L) xs[j0 + k] = yv[k];
    }
}

int pow2_at_least(int64_t v) {
    int g = 1;
    while (g < v) g <<= 1;
    return g;
}

}  // namespace

cudaError_t launch_lvc_outer(const LvcSite& x, const LvcSite& y, int64_t numT, cudaStream_t s) {
    // Items per lane.  16 halves the shuffle rounds per element but doubles the
    // registers (2 CTAs/SM); 8 doubles the lanes, which wins when the problem
    // is too small to fill the GPU (B200, LocVolCalib datasets: small 98 vs
    // 105 us at 8 / 16, medium 84 vs 70, large 1100 vs 902).  L > 256 needs 16.
    // -DIFL_LVC_IT=8|16 forces one (experiment builds only).
    const int64_t Lmax = std::max(x.L, y.L);
#ifdef IFL_LVC_IT
    constexpr int it_env = IFL_LVC_IT;
#else
    constexpr int it_env = 0;
#endif
    const int64_t lanes8 = x.S * pow2_at_least(std::max<int64_t>(1, ceil_div(x.L, 8))) +
                           y.S * pow2_at_least(std::max<int64_t>(1, ceil_div(y.L, 8)));
    int IT = (Lmax > 256 || lanes8 >= (int64_t)148 * 1024) ? 16 : 8;
    if (it_env == 16 || (it_env == 8 && Lmax <= 256)) IT = it_env;
    const int Gx = pow2_at_least(std::max<int64_t>(1, ceil_div(x.L, IT)));
    const int Gy = pow2_at_least(std::max<int64_t>(1, ceil_div(y.L, IT)));
    if (Gx > 32 || Gy > 32) return cudaErrorInvalidValue;
    const int64_t gx = x.S * x.L > 0 ? ceil_div(x.S, (int64_t)(kLvcThreads / Gx)) : 0;
    const int64_t gy = y.S * y.L > 0 ? ceil_div(y.S, (int64_t)(kLvcThreads / Gy)) : 0;
    if (gx + gy == 0) return cudaSuccess;
    if (gx + gy > 0x7fffffffLL) return cudaErrorInvalidValue;
    if (IT == 8)
        lvc_outer_kernel<8><<<(unsigned)(gx + gy), kLvcThreads, 0, s>>>(x, y, (int)gx, Gx, Gy, numT);
    else
        lvc_outer_kernel<16><<<(unsigned)(gx + gy), kLvcThreads, 0, s>>>(x, y, (int)gx, Gx, Gy, numT);
    return cudaGetLastError();
}

}  // namespace ifl
