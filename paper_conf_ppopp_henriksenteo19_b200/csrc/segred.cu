// segred.cu -- the V_TOP and V_MIDDLE versions of segred (rule G3's e_top and
// e_middle) for an [n][m] row-major array.
//
//   V_TOP    segmap^1 <xs in xss> (redomap (+) f d xs)
//            one thread per segment; the CTA's 256 rows are staged through
//            shared memory in [256][32] column tiles with coalesced 128-bit
//            loads, then each thread walks its own row sequentially
//            (bank-conflict-free: one pad word per 32).
//   V_MIDDLE segmap^1 <xs in xss> (segred^0 <x in xs> (+) d (f x))
//            one thread group of G threads per segment (G = m/16 rounded to a
//            power of two in [2, 1024]); 128-bit loads with per-row scalar
//            head/tail for any alignment, then a warp-shuffle / shared-memory
//            tree -- the level-0 reduction of P:346-358.
#include <string.h>

#include <algorithm>

#include "common.cuh"
#include "dispatch.cuh"
#include "ifl_internal.h"

#ifndef IFL_MID_GMAX
#define IFL_MID_GMAX 512  // largest V_MIDDLE group (threads per segment; 1024 measured slower)
#endif
#ifndef IFL_ROW_L1
#define IFL_ROW_L1 0  // row kernels: L1-allocating loads (a row's 16-byte words share sectors)
#endif
#ifndef IFL_TOP_ROW
#define IFL_TOP_ROW 1  // m in {8,16,32}: thread-per-row register kernel (0: smem-staged warp tiles)
#endif

namespace ifl {

// ------------------------------------------------------------------ V_TOP

constexpr int kTopThreads = 256;  // threads per CTA
constexpr int kTopKT = 32;        // columns per smem tile (128 B of f32 per row)
constexpr int kTopElems = kTopThreads * kTopKT;          // 8192 staged elements
constexpr int kTopWords = kTopElems + kTopElems / 32;    // + one pad word per 32

__device__ __forceinline__ int padq(int q) { return q + (q >> 5); }

// Rows per thread in whole-row mode (m <= 32): rpt rows of m elements each,
// so a CTA stages 256*rpt*m <= 8192 contiguous elements.
__host__ __device__ __forceinline__ int top_rpt(int64_t m) { return m <= kTopKT ? (int)(kTopKT / m) : 1; }

// Stage the CTA's tile into shared memory.  Whole-row mode: the region
// [r0*m, (r0+rows)*m) is contiguous and copied linearly.  Column-tile mode:
// columns [k0, k0+kt) of `rows` rows.  Padded index padq(q), q = row*KT + col
// (KT = m in whole-row mode, 32 otherwise): walking a row is conflict-free.
template <typename T>
__device__ __forceinline__ void top_load_tile(T* tile, const T* __restrict__ in, int64_t r0, int rows,
                                              int64_t m, int64_t k0, int kt, bool whole, bool vec) {
    const int t = threadIdx.x;
    using V = typename Vec4<T>::type;
    if (whole) {
        const int cnt = rows * (int)m;
        const T* src = in + r0 * m;
        int p0 = 0;
        if (vec) {
            const int nv = cnt >> 2;
            for (int v = t; v < nv; v += kTopThreads) {
                T e[4];
                unpack4<T>(ldg_stream4(src + 4 * v), e);
#pragma unroll
                for (int u = 0; u < 4; ++u) tile[padq(4 * v + u)] = e[u];
            }
            p0 = nv << 2;
        }
        for (int p = p0 + t; p < cnt; p += kTopThreads) tile[padq(p)] = ldg1(src + p);
    } else if (vec && kt == kTopKT) {
        // rows x 8 float4 per tile; a warp covers 4 rows x 128 B per load.
        for (int v = t; v < rows * 8; v += kTopThreads) {
            const int row = v >> 3, c4 = v & 7;
            T e[4];
            unpack4<T>(ldg_stream4(in + (r0 + row) * m + k0 + 4 * c4), e);
#pragma unroll
            for (int u = 0; u < 4; ++u) tile[padq(row * kTopKT + 4 * c4 + u)] = e[u];
        }
    } else {
        for (int p = t; p < rows * kTopKT; p += kTopThreads) {
            const int row = p >> 5, col = p & 31;
            if (col < kt) tile[padq(p)] = ldg1(in + (r0 + row) * m + k0 + col);
        }
    }
}

template <typename T, int OP, int F, bool COLS>
__global__ void __launch_bounds__(kTopThreads) segred_top_kernel(const T* __restrict__ in, T* __restrict__ out,
                                                                 int64_t n, int64_t m, T d, bool vec) {
    __shared__ T tile[kTopWords];
    const int t = threadIdx.x;
    const int rpt = top_rpt(m);
    const int64_t rows_blk = (int64_t)kTopThreads * rpt;
    const int64_t nblk = ceil_div(n, rows_blk);
    for (int64_t b = blockIdx.x; b < nblk; b += gridDim.x) {
        const int64_t r0 = b * rows_blk;
        const int rows = (int)min(rows_blk, n - r0);
        if constexpr (!COLS) {
            top_load_tile(tile, in, r0, rows, m, 0, (int)m, true, vec);
            __syncthreads();
            const int mm = (int)m;
            for (int j = 0; j < rpt; ++j) {
                const int r = t + j * kTopThreads;
                if (r < rows) {
                    Acc<OP, T> a(d);
                    for (int k = 0; k < mm; ++k) a.add(apply_map<F>(tile[padq(r * mm + k)]));
                    out[r0 + r] = a.get();
                }
            }
            __syncthreads();
        } else {
            Acc<OP, T> a0(d), a1(identity<OP, T>()), a2(identity<OP, T>()), a3(identity<OP, T>());
            using V = typename Vec4<T>::type;
            const int64_t nfull = vec ? (m / kTopKT) : 0;  // full 32-column tiles on the vector path
            // software pipeline over the full column tiles: the next tile's eight
            // 128-bit loads per thread are in flight while this tile is summed
            V pre[8];
            auto issue = [&](int64_t k0) {
#pragma unroll
                for (int j = 0; j < 8; ++j) {
                    const int v = t + j * kTopThreads, row = v >> 3, c4 = v & 7;
                    if (row < rows) pre[j] = ldg_stream4(in + (r0 + row) * m + k0 + 4 * c4);
                }
            };
            if (nfull > 0) issue(0);
            for (int64_t ti = 0; ti * kTopKT < m; ++ti) {
                const int64_t k0 = ti * kTopKT;
                const int kt = (int)min((int64_t)kTopKT, m - k0);
                if (ti < nfull) {
#pragma unroll
                    for (int j = 0; j < 8; ++j) {
                        const int v = t + j * kTopThreads, row = v >> 3, c4 = v & 7;
                        if (row < rows) {
                            T e[4];
                            unpack4<T>(pre[j], e);
#pragma unroll
                            for (int u = 0; u < 4; ++u) tile[padq(row * kTopKT + 4 * c4 + u)] = e[u];
                        }
                    }
                    if (ti + 1 < nfull) issue(k0 + kTopKT);
                } else {
                    top_load_tile(tile, in, r0, rows, m, k0, kt, false, false);
                }
                __syncthreads();
                if (t < rows) {
                    if (kt == kTopKT) {
#pragma unroll
                        for (int k = 0; k < kTopKT; k += 4) {
                            a0.add(apply_map<F>(tile[padq(t * kTopKT + k)]));
                            a1.add(apply_map<F>(tile[padq(t * kTopKT + k + 1)]));
                            a2.add(apply_map<F>(tile[padq(t * kTopKT + k + 2)]));
                            a3.add(apply_map<F>(tile[padq(t * kTopKT + k + 3)]));
                        }
                    } else {
                        for (int k = 0; k < kt; ++k) a0.add(apply_map<F>(tile[padq(t * kTopKT + k)]));
                    }
                }
                __syncthreads();
            }
            if (t < rows) {
                a0.add(a1.get());
                a2.add(a3.get());
                a0.add(a2.get());
                out[r0 + t] = a0.get();
            }
        }
    }
}

// V_TOP for m in {1, 2, 4} with 16-byte-aligned input: every 128-bit load
// holds 4/m whole rows, so each thread reduces its rows straight from
// registers -- fully coalesced warp-striped loads, no shared memory.
template <typename T, int OP, int F, int M>
__global__ void __launch_bounds__(256) segred_top_small_kernel(const T* __restrict__ in, T* __restrict__ out,
                                                               int64_t n, T d) {
    using V = typename Vec4<T>::type;
    const int64_t N = n * M, nv = N >> 2;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v0 < nv; v0 += 4 * stride) {
        V q[4];
#pragma unroll
        for (int u = 0; u < 4; ++u)
            if (v0 + u * stride < nv) q[u] = ldg_stream4(in + 4 * (v0 + u * stride));
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            const int64_t v = v0 + u * stride;
            if (v >= nv) break;
            T e[4];
            unpack4<T>(q[u], e);
            if constexpr (M == 1) {
                V r;
                r.x = combine<OP>(d, apply_map<F>(e[0]));
                r.y = combine<OP>(d, apply_map<F>(e[1]));
                r.z = combine<OP>(d, apply_map<F>(e[2]));
                r.w = combine<OP>(d, apply_map<F>(e[3]));
                *reinterpret_cast<V*>(out + 4 * v) = r;
            } else if constexpr (M == 2) {
                out[2 * v] = combine<OP>(combine<OP>(d, apply_map<F>(e[0])), apply_map<F>(e[1]));
                out[2 * v + 1] = combine<OP>(combine<OP>(d, apply_map<F>(e[2])), apply_map<F>(e[3]));
            } else {
                T a = combine<OP>(d, apply_map<F>(e[0]));
                a = combine<OP>(a, apply_map<F>(e[1]));
                a = combine<OP>(a, apply_map<F>(e[2]));
                out[v] = combine<OP>(a, apply_map<F>(e[3]));
            }
        }
    }
    // rows not covered by whole 128-bit words (N % 4 != 0)
    const int64_t r0 = (nv * 4) / M;
    for (int64_t r = r0 + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < n; r += stride) {
        T a = d;
        for (int k = 0; k < M; ++k) a = combine<OP>(a, apply_map<F>(in[r * M + k]));
        out[r] = a;
    }
}

// V_TOP for m in {8, 16, 32}, 16-byte-aligned: each warp takes 32 consecutive
// rows (a contiguous 32*m-element block), loads and stores it with fully
// coalesced 128-bit accesses through a padded per-warp tile, and every lane
// walks its own row sequentially (conflict-free: one pad word per 32).
template <typename T, int OP, int F, int M, bool SCAN>
__global__ void __launch_bounds__(256) top_warp_kernel(const T* in, T* out, int64_t n, T d) {
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
                unpack4<T>(ldg_stream4(src + 4 * q4), e);
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
                T a = d;
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
// 128-bit words loaded straight into registers (all in flight at once); a
// warp's 32 rows are one contiguous block, so every word of it is used.
template <typename T, int OP, int F, int M>
__global__ void __launch_bounds__(256) segred_top_row_kernel(const T* __restrict__ in, T* __restrict__ out, int64_t n,
                                                             T d) {
    using V = typename Vec4<T>::type;
    const int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (r >= n) return;
    const T* p = in + r * M;
    V q[M / 4];
#pragma unroll
    for (int u = 0; u < M / 4; ++u) q[u] = IFL_ROW_L1 ? __ldg(reinterpret_cast<const V*>(p + 4 * u)) : ldg_stream4(p + 4 * u);
    T a[4] = {d, identity<OP, T>(), identity<OP, T>(), identity<OP, T>()};
#pragma unroll
    for (int u = 0; u < M / 4; ++u) {
        T e[4];
        unpack4<T>(q[u], e);
#pragma unroll
        for (int k = 0; k < 4; ++k) a[k] = combine<OP>(a[k], apply_map<F>(e[k]));
    }
    out[r] = combine<OP>(combine<OP>(a[0], a[1]), combine<OP>(a[2], a[3]));
}

static int top_grid(int64_t nblk) {
    static int sms = 0;
    if (!sms) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        if (sms <= 0) sms = 148;
    }
    return (int)min(nblk, (int64_t)sms * 6);
}

cudaError_t launch_segred_top(const SegArgs& a) {
    return dispatch_all(a.dt, a.op, a.f, [&](auto tt, auto opc, auto fc) -> cudaError_t {
        using T = decltype(tt);
        constexpr int OP = decltype(opc)::value, F = decltype(fc)::value;
        const bool vec = ((uintptr_t)a.in % 16 == 0) && (a.m <= kTopKT || a.m % 4 == 0);
        if (vec && (a.m == 1 || a.m == 2 || a.m == 4) && ((uintptr_t)a.out % 16 == 0)) {
            const int64_t nv = ceil_div(a.n * a.m, 4);
            const int grid = top_grid(ceil_div(nv, 256 * 4)) * 2;
            const T d = bits_to<T>(a.ne_bits);
            if (a.m == 1)
                segred_top_small_kernel<T, OP, F, 1><<<grid, 256, 0, a.stream>>>((const T*)a.in, (T*)a.out, a.n, d);
            else if (a.m == 2)
                segred_top_small_kernel<T, OP, F, 2><<<grid, 256, 0, a.stream>>>((const T*)a.in, (T*)a.out, a.n, d);
            else
                segred_top_small_kernel<T, OP, F, 4><<<grid, 256, 0, a.stream>>>((const T*)a.in, (T*)a.out, a.n, d);
            return cudaGetLastError();
        }
        if (vec && a.m == 64) {
            top_tile_kernel<T, OP, F, 64, false><<<(unsigned)ceil_div(a.n, 32 * top_tile_warps(64)),
                                                   32 * top_tile_warps(64), 0, a.stream>>>(
                (const T*)a.in, (T*)a.out, a.n, bits_to<T>(a.ne_bits), nullptr);
            return cudaGetLastError();
        }
        if (IFL_TOP_ROW && vec && (a.m == 8 || a.m == 16 || a.m == 32)) {
            const unsigned grid = (unsigned)ceil_div(a.n, 256);
            const T d = bits_to<T>(a.ne_bits);
            if (a.m == 8)
                segred_top_row_kernel<T, OP, F, 8><<<grid, 256, 0, a.stream>>>((const T*)a.in, (T*)a.out, a.n, d);
            else if (a.m == 16)
                segred_top_row_kernel<T, OP, F, 16><<<grid, 256, 0, a.stream>>>((const T*)a.in, (T*)a.out, a.n, d);
            else
                top_tile_kernel<T, OP, F, 32, false><<<(unsigned)ceil_div(a.n, 256), 256, 0, a.stream>>>(
                    (const T*)a.in, (T*)a.out, a.n, d, nullptr);
            return cudaGetLastError();
        }
        if (vec && (a.m == 8 || a.m == 16 || a.m == 32)) {
            const int grid = top_grid(ceil_div(a.n, 256));
            const T d = bits_to<T>(a.ne_bits);
            if (a.m == 8)
                top_warp_kernel<T, OP, F, 8, false><<<grid, 256, 0, a.stream>>>((const T*)a.in, (T*)a.out, a.n, d);
            else if (a.m == 16)
                top_warp_kernel<T, OP, F, 16, false><<<grid, 256, 0, a.stream>>>((const T*)a.in, (T*)a.out, a.n, d);
            else
                top_warp_kernel<T, OP, F, 32, false><<<grid, 256, 0, a.stream>>>((const T*)a.in, (T*)a.out, a.n, d);
            return cudaGetLastError();
        }
        const int64_t nblk = ceil_div(a.n, (int64_t)kTopThreads * top_rpt(a.m));
        if (a.m <= kTopKT)
            segred_top_kernel<T, OP, F, false><<<top_grid(nblk), kTopThreads, 0, a.stream>>>(
                (const T*)a.in, (T*)a.out, a.n, a.m, bits_to<T>(a.ne_bits), vec);
        else
            segred_top_kernel<T, OP, F, true><<<top_grid(nblk), kTopThreads, 0, a.stream>>>(
                (const T*)a.in, (T*)a.out, a.n, a.m, bits_to<T>(a.ne_bits), vec);
        return cudaGetLastError();
    });
}

// --------------------------------------------------------------- V_MIDDLE

int mid_group_size(int64_t m) {
    int64_t g = 1;  // rows of <= 8 (16) elements: one thread already holds a whole row
    while (g < IFL_MID_GMAX && g * 16 < m) g <<= 1;
    return (int)g;
}

// Reduce `acc` over the G threads of a group.  G <= 32: shuffles inside the
// warp; G > 32: warp shuffles, then the group's warp totals via shared memory.
template <int OP, typename T>
__device__ __forceinline__ T group_reduce(T acc, int G, T* red) {
    if (G <= 32) {
        for (int off = G >> 1; off > 0; off >>= 1) acc = combine<OP>(acc, __shfl_xor_sync(0xffffffffu, acc, off));
        return acc;
    }
    acc = warp_reduce<OP>(acc);
    const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (lane == 0) red[w] = acc;
    __syncthreads();
    const int wpg = G >> 5, w0 = (threadIdx.x / G) * wpg;
    T r = identity<OP, T>();
    for (int k = 0; k < wpg; ++k) r = combine<OP>(r, red[w0 + k]);
    return r;
}

template <typename T, int OP, int F>
__global__ void __launch_bounds__(1024) segred_mid_kernel(const T* __restrict__ in, T* __restrict__ out,
                                                          int64_t n, int64_t m, T d, int G) {
    __shared__ T red[32];
    using V = typename Vec4<T>::type;
    const int g = threadIdx.x % G;
    const int64_t i = (int64_t)blockIdx.x * (blockDim.x / G) + threadIdx.x / G;
    T acc = identity<OP, T>();
    if (i < n) {
        const T* row = in + i * m;
        int64_t h = (int64_t)(((16u - ((uint32_t)(uintptr_t)row & 15u)) & 15u) / sizeof(T));
        if (h > m) h = m;
        const int64_t nvec = (m - h) >> 2;
        for (int64_t k = g; k < h; k += G) acc = combine<OP>(acc, apply_map<F>(ldg1(row + k)));
        const T* body = row + h;
        T a4[4] = {identity<OP, T>(), identity<OP, T>(), identity<OP, T>(), identity<OP, T>()};
        int64_t v = g;
        for (; v + 3 * (int64_t)G < nvec; v += 4 * (int64_t)G) {
            V q[4];
#pragma unroll
            for (int u = 0; u < 4; ++u) q[u] = ldg_stream4(body + 4 * (v + u * (int64_t)G));
#pragma unroll
            for (int u = 0; u < 4; ++u) {
                T e[4];
                unpack4<T>(q[u], e);
#pragma unroll
                for (int c = 0; c < 4; ++c) a4[c] = combine<OP>(a4[c], apply_map<F>(e[c]));
            }
        }
        for (; v < nvec; v += G) {
            T e[4];
            unpack4<T>(ldg_stream4(body + 4 * v), e);
#pragma unroll
            for (int c = 0; c < 4; ++c) a4[c] = combine<OP>(a4[c], apply_map<F>(e[c]));
        }
        const int64_t t0 = h + 4 * nvec;
        for (int64_t k = t0 + g; k < m; k += G) acc = combine<OP>(acc, apply_map<F>(ldg1(row + k)));
        acc = combine<OP>(acc, combine<OP>(combine<OP>(a4[0], a4[1]), combine<OP>(a4[2], a4[3])));
    }
    acc = group_reduce<OP>(acc, G, red);
    if (g == 0 && i < n) out[i] = combine<OP>(d, acc);
}

// Aligned rows (m % 4 == 0, 16-byte aligned base) of at most 16*G elements:
// every thread owns <= 4 128-bit vectors of its row, all issued before the
// first combine, with 32-bit index arithmetic and no scalar head/tail loops.
// B200, n*m = 2^26 f32, m = 32..4096: 39-41 us (6.6-6.9 TB/s) against
// 45-48 us for the generic kernel below.  Taking two or four slabs of rows
// per CTA (8/16 loads in flight) measured slower (44-55 us).
template <typename T, int OP, int F>
__global__ void __launch_bounds__(512) segred_mid_vec_kernel(const T* __restrict__ in, T* __restrict__ out,
                                                             int64_t n, int m, T d, int G) {
    __shared__ T red[32];
    using V = typename Vec4<T>::type;
    const int g = threadIdx.x % G;
    const int64_t i = (int64_t)blockIdx.x * (blockDim.x / G) + threadIdx.x / G;
    const int nvec = m >> 2;
    const T* row = in + i * m;
    V q[4];
#pragma unroll
    for (int u = 0; u < 4; ++u)
        if (i < n && g + u * G < nvec) q[u] = ldg_stream4(row + 4 * (g + u * G));
    T acc = identity<OP, T>();
#pragma unroll
    for (int u = 0; u < 4; ++u)
        if (i < n && g + u * G < nvec) {
            T e[4];
            unpack4<T>(q[u], e);
            acc = combine<OP>(acc, combine<OP>(combine<OP>(apply_map<F>(e[0]), apply_map<F>(e[1])),
                                               combine<OP>(apply_map<F>(e[2]), apply_map<F>(e[3]))));
        }
    acc = group_reduce<OP>(acc, G, red);
    if (g == 0 && i < n) out[i] = combine<OP>(d, acc);
}

cudaError_t launch_segred_mid(const SegArgs& a) {
    if (a.m >= 8192) return launch_segred_rows512(a);  // one 512-thread group per row (flat.cu)
    const int G0 = mid_group_size(a.m);
    const int G = std::max(1, std::min(IFL_MID_GMAX, a.gshift >= 0 ? G0 << a.gshift : G0 >> -a.gshift));
    const int B = G > 256 ? G : 256;
    const int64_t grid = ceil_div(a.n, B / G);
    if (a.m > 0 && a.m % 4 == 0 && ((uintptr_t)a.in & 15u) == 0 && a.m <= 16 * (int64_t)G)
        return dispatch_all(a.dt, a.op, a.f, [&](auto tt, auto opc, auto fc) -> cudaError_t {
            using T = decltype(tt);
            constexpr int OP = decltype(opc)::value, F = decltype(fc)::value;
            segred_mid_vec_kernel<T, OP, F><<<(unsigned)grid, B, 0, a.stream>>>(
                (const T*)a.in, (T*)a.out, a.n, (int)a.m, bits_to<T>(a.ne_bits), G);
            return cudaGetLastError();
        });
    return dispatch_all(a.dt, a.op, a.f, [&](auto tt, auto opc, auto fc) -> cudaError_t {
        using T = decltype(tt);
        constexpr int OP = decltype(opc)::value, F = decltype(fc)::value;
        segred_mid_kernel<T, OP, F><<<(unsigned)grid, B, 0, a.stream>>>((const T*)a.in, (T*)a.out, a.n, a.m,
                                                                        bits_to<T>(a.ne_bits), G);
        return cudaGetLastError();
    });
}

// ------------------------------------------------------------ m == 0 fill

__global__ void fill_kernel(uint32_t* out, int64_t count, uint32_t bits) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += (int64_t)gridDim.x * blockDim.x)
        out[i] = bits;
}

cudaError_t launch_fill(void* out, int64_t count, uint32_t bits, cudaStream_t s) {
    if (count <= 0) return cudaSuccess;
    const int64_t grid = min(ceil_div(count, 256), (int64_t)148 * 16);
    fill_kernel<<<(unsigned)grid, 256, 0, s>>>((uint32_t*)out, count, bits);
    return cudaGetLastError();
}

}  // namespace ifl
