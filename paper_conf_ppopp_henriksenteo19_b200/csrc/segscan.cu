// segscan.cu -- the V_TOP and V_MIDDLE versions of segscan (Fig 6c
// versions 1 and 2) for an [n][m] row-major array.
//
//   V_TOP    segmap^1 <xs in xss> (scanomap (+) f d xs): one thread per row,
//            [256][32] column tiles staged through padded shared memory
//            (coalesced 128-bit loads and stores), each thread scans its row
//            sequentially in place with a running carry.
//   V_MIDDLE segmap^1 <xs in xss> (segscan^0 <x in xs> (+) d (f x)): a group
//            of G threads per row; per round each thread scans 8 consecutive
//            elements in registers, the group scans the thread totals with
//            warp shuffles (+ shared memory when G > 32) and carries the
//            round total to the next round.
#include <string.h>

#include <algorithm>

#include "common.cuh"
#include "dispatch.cuh"
#include "ifl_internal.h"

#ifndef IFL_MIDSCAN_GMAX
#define IFL_MIDSCAN_GMAX 256  // largest V_MIDDLE scan group (threads per segment; longer rows take
                              // several pipelined rounds -- 512 / 1024 measured slower)
#endif
#ifndef IFL_ROW_L1
#define IFL_ROW_L1 0  // row kernels: L1-allocating loads (a row's 16-byte words share sectors)
#endif
#ifndef IFL_TOP_ROW
#define IFL_TOP_ROW 1  // m in {8,16,32}: thread-per-row register kernel (0: smem-staged warp tiles)
#endif

namespace ifl {

constexpr int kTopThreads = 256;
constexpr int kTopKT = 32;
constexpr int kTopElems = kTopThreads * kTopKT;
constexpr int kTopWords = kTopElems + kTopElems / 32;

__device__ __forceinline__ int spadq(int q) { return q + (q >> 5); }
__host__ __device__ __forceinline__ int stop_rpt(int64_t m) { return m <= kTopKT ? (int)(kTopKT / m) : 1; }

// Copy between a global window and the padded smem tile (see segred.cu).
// LOAD: global -> smem; STORE: smem -> global.
template <bool LOAD, typename T>
__device__ __forceinline__ void top_xfer(T* tile, const T* in, T* out, int64_t r0,
                                         int rows, int64_t m, int64_t k0, int kt, bool whole, bool vec,
                                         bool rev = false) {
    // rev (reverse scans): logical column c of a row is physical column m-1-c
    // (vec is false then: the scalar paths below do the mirroring)
    auto ph = [&](int64_t g) -> int64_t {
        if (!rev) return g;
        const int64_t r = g / m;
        return r * m + (m - 1 - (g - r * m));
    };
    const int t = threadIdx.x;
    using V = typename Vec4<T>::type;
    if (whole) {
        const int cnt = rows * (int)m;
        int p0 = 0;
        if (vec) {
            const int nv = cnt >> 2;
            for (int v = t; v < nv; v += kTopThreads) {
                if (LOAD) {
                    T e[4];
                    unpack4<T>(ld_coh4(in + r0 * m + 4 * v), e);
#pragma unroll
                    for (int u = 0; u < 4; ++u) tile[spadq(4 * v + u)] = e[u];
                } else {
                    V q;
                    q.x = tile[spadq(4 * v)];
                    q.y = tile[spadq(4 * v + 1)];
                    q.z = tile[spadq(4 * v + 2)];
                    q.w = tile[spadq(4 * v + 3)];
                    *reinterpret_cast<V*>(out + r0 * m + 4 * v) = q;
                }
            }
            p0 = nv << 2;
        }
        for (int p = p0 + t; p < cnt; p += kTopThreads) {
            if (LOAD) tile[spadq(p)] = ld_coh1(in + ph(r0 * m + p));
            else out[ph(r0 * m + p)] = tile[spadq(p)];
        }
    } else if (vec && kt == kTopKT) {
        for (int v = t; v < rows * 8; v += kTopThreads) {
            const int row = v >> 3, c4 = v & 7;
            const int64_t gi = (r0 + row) * m + k0 + 4 * c4;
            const int q0 = row * kTopKT + 4 * c4;
            if (LOAD) {
                T e[4];
                unpack4<T>(ld_coh4(in + gi), e);
#pragma unroll
                for (int u = 0; u < 4; ++u) tile[spadq(q0 + u)] = e[u];
            } else {
                V q;
                q.x = tile[spadq(q0)];
                q.y = tile[spadq(q0 + 1)];
                q.z = tile[spadq(q0 + 2)];
                q.w = tile[spadq(q0 + 3)];
                *reinterpret_cast<V*>(out + gi) = q;
            }
        }
    } else {
        for (int p = t; p < rows * kTopKT; p += kTopThreads) {
            const int row = p >> 5, col = p & 31;
            if (col < kt) {
                const int64_t gi = (r0 + row) * m + k0 + col;
                if (LOAD) tile[spadq(p)] = ld_coh1(in + ph(gi));
                else out[ph(gi)] = tile[spadq(p)];
            }
        }
    }
}

template <typename T, int OP, int F>
__global__ void __launch_bounds__(kTopThreads) segscan_top_kernel(const T* in, T* out, int64_t n, int64_t m, T d,
                                                                  bool vec, const T* __restrict__ seed,
                                                                  bool rev = false) {
    __shared__ T tile[kTopWords];
    const int t = threadIdx.x;
    const int rpt = stop_rpt(m);
    const int64_t rows_blk = (int64_t)kTopThreads * rpt;
    const int64_t nblk = ceil_div(n, rows_blk);
    for (int64_t b = blockIdx.x; b < nblk; b += gridDim.x) {
        const int64_t r0 = b * rows_blk;
        const int rows = (int)min(rows_blk, n - r0);
        if (m <= kTopKT) {
            top_xfer<true>(tile, in, out, r0, rows, m, 0, (int)m, true, vec, rev);
            __syncthreads();
            const int mm = (int)m;
            for (int j = 0; j < rpt; ++j) {
                const int r = t + j * kTopThreads;
                if (r < rows) {
                    Acc<OP, T> a(seed ? seed[r0 + r] : d);  // d (+) f(x0) (+) ...: d applied once, at the row start
                    for (int k = 0; k < mm; ++k) {
                        a.add(apply_map<F>(tile[spadq(r * mm + k)]));
                        tile[spadq(r * mm + k)] = a.get();
                    }
                }
            }
            __syncthreads();
            top_xfer<false>(tile, in, out, r0, rows, m, 0, (int)m, true, vec, rev);
            __syncthreads();
        } else {
            Acc<OP, T> a((seed && t < rows) ? seed[r0 + t] : d);
            for (int64_t k0 = 0; k0 < m; k0 += kTopKT) {
                const int kt = (int)min((int64_t)kTopKT, m - k0);
                top_xfer<true>(tile, in, out, r0, rows, m, k0, kt, false, vec, rev);
                __syncthreads();
                if (t < rows) {
                    if (kt == kTopKT) {
#pragma unroll
                        for (int k = 0; k < kTopKT; ++k) {
                            a.add(apply_map<F>(tile[spadq(t * kTopKT + k)]));
                            tile[spadq(t * kTopKT + k)] = a.get();
                        }
                    } else {
                        for (int k = 0; k < kt; ++k) {
                            a.add(apply_map<F>(tile[spadq(t * kTopKT + k)]));
                            tile[spadq(t * kTopKT + k)] = a.get();
                        }
                    }
                }
                __syncthreads();
                top_xfer<false>(tile, in, out, r0, rows, m, k0, kt, false, vec, rev);
                __syncthreads();
            }
        }
    }
}

// V_TOP for m in {1, 2, 4} with 16-byte-aligned in/out: each 128-bit word
// holds 4/m whole rows, scanned in registers and stored back as one word.
template <typename T, int OP, int F, int M>
__global__ void __launch_bounds__(256) segscan_top_small_kernel(const T* in, T* out, int64_t n, T d,
                                                                const T* __restrict__ seed) {
    using V = typename Vec4<T>::type;
    const int64_t N = n * M, nv = N >> 2;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v0 < nv; v0 += 4 * stride) {
        V q[4];
#pragma unroll
        for (int u = 0; u < 4; ++u)
            if (v0 + u * stride < nv) q[u] = ld_coh4(in + 4 * (v0 + u * stride));
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            const int64_t v = v0 + u * stride;
            if (v >= nv) break;
            T e[4];
            unpack4<T>(q[u], e);
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                const T x = apply_map<F>(e[k]);
                e[k] = (k % M == 0) ? combine<OP>(seed ? seed[(4 * v + k) / M] : d, x)
                                    : combine<OP>(e[k - 1 < 0 ? 0 : k - 1], x);
            }
            V r;
            r.x = e[0]; r.y = e[1]; r.z = e[2]; r.w = e[3];
            *reinterpret_cast<V*>(out + 4 * v) = r;
        }
    }
    const int64_t r0 = (nv * 4) / M;
    for (int64_t r = r0 + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < n; r += stride) {
        T a = seed ? seed[r] : d;
        for (int k = 0; k < M; ++k) {
            a = combine<OP>(a, apply_map<F>(in[r * M + k]));
            out[r * M + k] = a;
        }
    }
}

// V_TOP for m in {8, 16, 32}, 16-byte-aligned: each warp takes 32 consecutive
// rows (a contiguous 32*m-element block), loads and stores it with fully
// coalesced 128-bit accesses through a padded per-warp tile, and every lane
// walks its own row sequentially (conflict-free: one pad word per 32).
template <typename T, int OP, int F, int M, bool SCAN>
__global__ void __launch_bounds__(256) top_warp_kernel(const T* in, T* out, int64_t n, T d, const T* __restrict__ seed) {
    using V = typename Vec4<T>::type;
    constexpr int W4 = M / 4;
    __shared__ T sm[8][32 * M + M];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    T* s = sm[warp];
    const int64_t nw = (int64_t)gridDim.x * 8;
    for (int64_t wc = (int64_t)blockIdx.x * 8 + warp; wc * 32 < n; wc += nw) {
        const int64_t r0 = wc * 32;
        const int rows = (int)min((int64_t)32, n - r0);
        const T* src = in + r0 * M;
#pragma unroll
        for (int u = 0; u < W4; ++u) {
            const int q4 = lane + 32 * u;
            if (q4 < rows * W4) {
                T e[4];
                unpack4<T>(ld_coh4(src + 4 * q4), e);
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    const int q = 4 * q4 + k;
                    s[q + (q >> 5)] = e[k];
                }
            }
        }
        __syncwarp();
        if (lane < rows) {  // rows of <= 32 elements: plain chains (no compensation needed)
            if constexpr (SCAN) {
                T a = seed ? seed[r0 + lane] : d;
#pragma unroll
                for (int k = 0; k < M; ++k) {
                    const int q = lane * M + k;
                    a = combine<OP>(a, apply_map<F>(s[q + (q >> 5)]));
                    s[q + (q >> 5)] = a;
                }
            } else {
                T a0 = d, a1 = identity<OP, T>();
#pragma unroll
                for (int k = 0; k < M; k += 2) {
                    const int q = lane * M + k;
                    a0 = combine<OP>(a0, apply_map<F>(s[q + (q >> 5)]));
                    a1 = combine<OP>(a1, apply_map<F>(s[q + 1 + ((q + 1) >> 5)]));
                }
                out[r0 + lane] = combine<OP>(a0, a1);
            }
        }
        if (SCAN) {
            __syncwarp();
            T* dst = out + r0 * M;
#pragma unroll
            for (int u = 0; u < W4; ++u) {
                const int q4 = lane + 32 * u;
                if (q4 < rows * W4) {
                    V v;
                    int q = 4 * q4;
                    v.x = s[q + (q >> 5)];
                    ++q;
                    v.y = s[q + (q >> 5)];
                    ++q;
                    v.z = s[q + (q >> 5)];
                    ++q;
                    v.w = s[q + (q >> 5)];
                    *reinterpret_cast<V*>(dst + 4 * q4) = v;
                }
            }
        }
        __syncwarp();
    }
}

// V_TOP for m in {8, 16, 32}, 16-byte-aligned: one thread per row, its m/4
// 128-bit words loaded straight into registers, scanned, stored back.
template <typename T, int OP, int F, int M>
__global__ void __launch_bounds__(256) segscan_top_row_kernel(const T* in, T* out,
                                                              int64_t n, T d, const T* __restrict__ seed) {
    using V = typename Vec4<T>::type;
    const int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (r >= n) return;
    const T* p = in + r * M;
    V q[M / 4];
#pragma unroll
    for (int u = 0; u < M / 4; ++u) q[u] = ld_coh4(p + 4 * u);
    T a = seed ? seed[r] : d;
    T* o = out + r * M;
#pragma unroll
    for (int u = 0; u < M / 4; ++u) {
        T e[4];
        unpack4<T>(q[u], e);
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            a = combine<OP>(a, apply_map<F>(e[k]));
            e[k] = a;
        }
        V w;
        w.x = e[0]; w.y = e[1]; w.z = e[2]; w.w = e[3];
        *reinterpret_cast<V*>(o + 4 * u) = w;
    }
}

static int stop_grid(int64_t nblk) {
    static int sms = 0;
    if (!sms) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        if (sms <= 0) sms = 148;
    }
    return (int)min(nblk, (int64_t)sms * 6);
}

cudaError_t launch_segscan_top(const SegArgs& a) {
    return dispatch_all(a.dt, a.op, a.f, [&](auto tt, auto opc, auto fc) -> cudaError_t {
        using T = decltype(tt);
        constexpr int OP = decltype(opc)::value, F = decltype(fc)::value;
        const T* seed = (const T*)a.seed;
        // reverse scans take the generic kernel's scalar (mirroring) paths
        const bool vec = !a.rev && ((uintptr_t)a.in % 16 == 0) && ((uintptr_t)a.out % 16 == 0) &&
                         (a.m <= kTopKT || a.m % 4 == 0);
        if (vec && (a.m == 1 || a.m == 2 || a.m == 4)) {
            const int64_t nv = ceil_div(a.n * a.m, 4);
            const int grid = stop_grid(ceil_div(nv, 256 * 4)) * 2;
            const T d = bits_to<T>(a.ne_bits);
            if (a.m == 1)
                segscan_top_small_kernel<T, OP, F, 1><<<grid, 256, 0, a.stream>>>((const T*)a.in, (T*)a.out, a.n, d, seed);
            else if (a.m == 2)
                segscan_top_small_kernel<T, OP, F, 2><<<grid, 256, 0, a.stream>>>((const T*)a.in, (T*)a.out, a.n, d, seed);
            else
                segscan_top_small_kernel<T, OP, F, 4><<<grid, 256, 0, a.stream>>>((const T*)a.in, (T*)a.out, a.n, d, seed);
            return cudaGetLastError();
        }
        if (vec && a.m == 64) {
            top_tile_kernel<T, OP, F, 64, true><<<(unsigned)ceil_div(a.n, 32 * top_tile_warps(64)),
                                                  32 * top_tile_warps(64), 0, a.stream>>>(
                (const T*)a.in, (T*)a.out, a.n, bits_to<T>(a.ne_bits), seed);
            return cudaGetLastError();
        }
        if (IFL_TOP_ROW && vec && (a.m == 8 || a.m == 16 || a.m == 32)) {
            const unsigned grid = (unsigned)ceil_div(a.n, 256);
            const T d = bits_to<T>(a.ne_bits);
            if (a.m == 8)
                segscan_top_row_kernel<T, OP, F, 8><<<grid, 256, 0, a.stream>>>((const T*)a.in, (T*)a.out, a.n, d, seed);
            else if (a.m == 16)
                top_tile_kernel<T, OP, F, 16, true><<<grid, 256, 0, a.stream>>>((const T*)a.in, (T*)a.out, a.n, d, seed);
            else
                top_tile_kernel<T, OP, F, 32, true><<<grid, 256, 0, a.stream>>>((const T*)a.in, (T*)a.out, a.n, d, seed);
            return cudaGetLastError();
        }
        if (vec && (a.m == 8 || a.m == 16 || a.m == 32)) {
            const int grid = stop_grid(ceil_div(a.n, 256));
            const T d = bits_to<T>(a.ne_bits);
            if (a.m == 8)
                top_warp_kernel<T, OP, F, 8, true><<<grid, 256, 0, a.stream>>>((const T*)a.in, (T*)a.out, a.n, d, seed);
            else if (a.m == 16)
                top_warp_kernel<T, OP, F, 16, true><<<grid, 256, 0, a.stream>>>((const T*)a.in, (T*)a.out, a.n, d, seed);
            else
                top_warp_kernel<T, OP, F, 32, true><<<grid, 256, 0, a.stream>>>((const T*)a.in, (T*)a.out, a.n, d, seed);
            return cudaGetLastError();
        }
        const int64_t nblk = ceil_div(a.n, (int64_t)kTopThreads * stop_rpt(a.m));
        segscan_top_kernel<T, OP, F><<<stop_grid(nblk), kTopThreads, 0, a.stream>>>(
            (const T*)a.in, (T*)a.out, a.n, a.m, bits_to<T>(a.ne_bits), vec, seed, a.rev);
        return cudaGetLastError();
    });
}

// --------------------------------------------------------------- V_MIDDLE

constexpr int kMidItems = 8;  // consecutive elements per thread per round

int midscan_group_size(int64_t m) {
    int64_t g = 1;  // rows of <= 8 (16) elements: one thread already holds a whole row
    while (g < IFL_MIDSCAN_GMAX && g * kMidItems < m) g <<= 1;
    return (int)g;
}

template <typename T, int OP, int F>
__global__ void __launch_bounds__(1024) segscan_mid_kernel(const T* in, T* out, int64_t n, int64_t m, T d, int G,
                                                           bool vec, const T* __restrict__ seed, bool rev = false) {
    __shared__ T wtot[2][32];
    using V = typename Vec4<T>::type;
    const int g = threadIdx.x % G;
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int64_t i = (int64_t)blockIdx.x * (blockDim.x / G) + threadIdx.x / G;
    const bool live = i < n;
    const T* row = in + (live ? i * m : 0);
    T* orow = out + (live ? i * m : 0);
    T carry = (seed && live) ? seed[i] : d;  // rows of one round (m <= G * 8): no long carry chain
    int par = 0;
    for (int64_t base = 0; base < m; base += (int64_t)G * kMidItems, par ^= 1) {
        const int64_t k0 = base + (int64_t)g * kMidItems;
        T v[kMidItems];
#pragma unroll
        for (int h = 0; h < kMidItems / 4; ++h) {  // two 128-bit halves, each vectorised when whole
            const int64_t kh = k0 + 4 * h;
            if (live && vec && kh + 4 <= m) {
                T e[4];
                unpack4<T>(ld_coh4(row + kh), e);
#pragma unroll
                for (int u = 0; u < 4; ++u) v[4 * h + u] = apply_map<F>(e[u]);
            } else {
#pragma unroll
                for (int u = 0; u < 4; ++u)
                    v[4 * h + u] = (live && kh + u < m) ? apply_map<F>(ld_coh1(row + (rev ? m - 1 - (kh + u) : kh + u))) : identity<OP, T>();
            }
        }
#pragma unroll
        for (int u = 1; u < kMidItems; ++u) v[u] = combine<OP>(v[u - 1], v[u]);
        // inclusive scan of thread totals across the group
        T s = v[kMidItems - 1];
        const int width = G < 32 ? G : 32;
        const int gl = threadIdx.x % width;  // lane within the (sub)warp group
        for (int off = 1; off < width; off <<= 1) {
            T o = __shfl_up_sync(0xffffffffu, s, off, width);
            if (gl >= off) s = combine<OP>(o, s);
        }
        T ex = __shfl_up_sync(0xffffffffu, s, 1, width);
        if (gl == 0) ex = identity<OP, T>();
        T total;
        if (G <= 32) {
            total = __shfl_sync(0xffffffffu, s, width - 1, width);
        } else {
            if (lane == 31) wtot[par][w] = s;
            __syncthreads();
            const int wpg = G >> 5, w0 = (threadIdx.x / G) * wpg;
            T before = identity<OP, T>();
            total = identity<OP, T>();
            for (int k = 0; k < wpg; ++k) {
                if (w0 + k < w) before = combine<OP>(before, wtot[par][w0 + k]);
                total = combine<OP>(total, wtot[par][w0 + k]);
            }
            ex = combine<OP>(before, ex);
        }
        const T pre = combine<OP>(carry, ex);
#pragma unroll
        for (int u = 0; u < kMidItems; ++u) v[u] = combine<OP>(pre, v[u]);
        if (live) {
#pragma unroll
            for (int h = 0; h < kMidItems / 4; ++h) {
                const int64_t kh = k0 + 4 * h;
                if (vec && kh + 4 <= m) {
                    V q;
                    q.x = v[4 * h]; q.y = v[4 * h + 1]; q.z = v[4 * h + 2]; q.w = v[4 * h + 3];
                    *reinterpret_cast<V*>(orow + kh) = q;
                } else {
#pragma unroll
                    for (int u = 0; u < 4; ++u)
                        if (kh + u < m) orow[rev ? m - 1 - (kh + u) : kh + u] = v[4 * h + u];
                }
            }
        }
        carry = combine<OP>(carry, total);
    }
}

#ifndef IFL_MULTI_MINB
#define IFL_MULTI_MINB 6
#endif
// V_MIDDLE for rows of several rounds: the next round's items are loaded before
// this round is scanned (register double buffer), so every round's loads overlap
// the previous round's group scan and barriers.
template <typename T, int OP, int F>
__global__ void __launch_bounds__(IFL_MIDSCAN_GMAX, IFL_MULTI_MINB)
    segscan_mid_multi_kernel(const T* in, T* out, int64_t n, int64_t m, T d, int G, bool vec,
                             const T* __restrict__ seed, bool rev = false) {
    __shared__ T wtot[2][32];
    using V = typename Vec4<T>::type;
    const int g = threadIdx.x % G;
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int64_t i = (int64_t)blockIdx.x * (blockDim.x / G) + threadIdx.x / G;
    const bool live = i < n;
    const T* row = in + (live ? i * m : 0);
    T* orow = out + (live ? i * m : 0);
    // running carry across rounds: Kahan-compensated for f32 sums (a row of
    // 4 x 10^8 elements adds 10^5 round totals into it; plain f32 drifts past
    // the 1e-5 * sum|f(x)| bound)
    Acc<OP, T> carry((seed && live) ? seed[i] : d);
    int par = 0;
    const int64_t step = (int64_t)G * kMidItems;
    // raw items of one round (two 128-bit halves, each vectorised when whole; f applied at use,
    // so the next round's loads stay in flight while this round is scanned)
    auto load_round = [&](int64_t base, T (&r)[kMidItems]) {
        const int64_t k0 = base + (int64_t)g * kMidItems;
#pragma unroll
        for (int h = 0; h < kMidItems / 4; ++h) {
            const int64_t kh = k0 + 4 * h;
            if (live && vec && kh + 4 <= m) {
                T e[4];
                unpack4<T>(ld_coh4(row + kh), e);
#pragma unroll
                for (int u = 0; u < 4; ++u) r[4 * h + u] = e[u];
            } else {
#pragma unroll
                for (int u = 0; u < 4; ++u) r[4 * h + u] = (live && kh + u < m) ? ld_coh1(row + (rev ? m - 1 - (kh + u) : kh + u)) : T();
            }
        }
    };
    T nxt[kMidItems];
    load_round(0, nxt);
    for (int64_t base = 0; base < m; base += step, par ^= 1) {
        const int64_t k0 = base + (int64_t)g * kMidItems;
        T v[kMidItems];
#pragma unroll
        for (int u = 0; u < kMidItems; ++u) v[u] = nxt[u];
        if (base + step < m) load_round(base + step, nxt);  // prefetch the next round
#pragma unroll
        for (int u = 0; u < kMidItems; ++u)
            v[u] = (live && k0 + u < m) ? apply_map<F>(v[u]) : identity<OP, T>();
#pragma unroll
        for (int u = 1; u < kMidItems; ++u) v[u] = combine<OP>(v[u - 1], v[u]);
        // inclusive scan of thread totals across the group
        T s = v[kMidItems - 1];
        const int width = G < 32 ? G : 32;
        const int gl = threadIdx.x % width;  // lane within the (sub)warp group
        for (int off = 1; off < width; off <<= 1) {
            T o = __shfl_up_sync(0xffffffffu, s, off, width);
            if (gl >= off) s = combine<OP>(o, s);
        }
        T ex = __shfl_up_sync(0xffffffffu, s, 1, width);
        if (gl == 0) ex = identity<OP, T>();
        T total;
        if (G <= 32) {
            total = __shfl_sync(0xffffffffu, s, width - 1, width);
        } else {
            if (lane == 31) wtot[par][w] = s;
            __syncthreads();
            const int wpg = G >> 5, w0 = (threadIdx.x / G) * wpg;
            T before = identity<OP, T>();
            total = identity<OP, T>();
            for (int k = 0; k < wpg; ++k) {
                if (w0 + k < w) before = combine<OP>(before, wtot[par][w0 + k]);
                total = combine<OP>(total, wtot[par][w0 + k]);
            }
            ex = combine<OP>(before, ex);
        }
        const T pre = combine<OP>(carry.get(), ex);
#pragma unroll
        for (int u = 0; u < kMidItems; ++u) v[u] = combine<OP>(pre, v[u]);
        if (live) {
#pragma unroll
            for (int h = 0; h < kMidItems / 4; ++h) {
                const int64_t kh = k0 + 4 * h;
                if (vec && kh + 4 <= m) {
                    V q;
                    q.x = v[4 * h]; q.y = v[4 * h + 1]; q.z = v[4 * h + 2]; q.w = v[4 * h + 3];
                    *reinterpret_cast<V*>(orow + kh) = q;
                } else {
#pragma unroll
                    for (int u = 0; u < 4; ++u)
                        if (kh + u < m) orow[rev ? m - 1 - (kh + u) : kh + u] = v[4 * h + u];
                }
            }
        }
        carry.add(total);
    }
}

cudaError_t launch_segscan_mid(const SegArgs& a) {
    return dispatch_all(a.dt, a.op, a.f, [&](auto tt, auto opc, auto fc) -> cudaError_t {
        using T = decltype(tt);
        constexpr int OP = decltype(opc)::value, F = decltype(fc)::value;
        const int G0 = midscan_group_size(a.m);
        const int G = std::max(1, std::min(IFL_MIDSCAN_GMAX, a.gshift >= 0 ? G0 << a.gshift : G0 >> -a.gshift));
        const int B = G > 256 ? G : 256;
        const bool vec = !a.rev && ((uintptr_t)a.in % 16 == 0) && ((uintptr_t)a.out % 16 == 0) && (a.m % 4 == 0);
        const int64_t grid = ceil_div(a.n, B / G);
        if (a.m > (int64_t)G * kMidItems)  // several rounds per row: pipelined loads
            segscan_mid_multi_kernel<T, OP, F><<<(unsigned)grid, B, 0, a.stream>>>(
                (const T*)a.in, (T*)a.out, a.n, a.m, bits_to<T>(a.ne_bits), G, vec, (const T*)a.seed, a.rev);
        else
            segscan_mid_kernel<T, OP, F><<<(unsigned)grid, B, 0, a.stream>>>(
                (const T*)a.in, (T*)a.out, a.n, a.m, bits_to<T>(a.ne_bits), G, vec, (const T*)a.seed, a.rev);
        return cudaGetLastError();
    });
}

}  // namespace ifl
