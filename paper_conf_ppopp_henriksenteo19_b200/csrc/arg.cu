// arg.cu -- tuple-valued reduction per row: argmin / argmax, the (value,
// index) pair of the first minimum / maximum (P:81-83 tuple SOACs; the
// argmin of NN-shaped workloads).  The operator
//   (v1,i1) (+) (v2,i2) = better(v2, v1) || (v2 == v1 && i2 < i1) ? (v2,i2) : (v1,i1)
// is associative AND commutative (ties resolved by the index), so every
// version returns the unique first occurrence whatever its reduction order.
// Versions as for segred (G3): V_TOP thread per row; V_MIDDLE a
// group per row (warp for short rows, 512-thread CTA for long ones); V_FLAT
// uniform row pieces across CTAs + a per-row combine of the piece pairs.
#include <algorithm>

#include "common.cuh"
#include "ifl_internal.h"

namespace ifl {

namespace {

template <typename T, bool MAX>
__device__ __forceinline__ void arg_take(T& bv, int& bi, T v, int i) {
    const bool better = MAX ? (v > bv) : (v < bv);
    if (better || (v == bv && (unsigned)i < (unsigned)bi)) {  // bi = -1 (none) compares as the largest index
        bv = v;
        bi = i;
    }
}

template <typename T, bool MAX>
__device__ __forceinline__ T arg_d() {
    if constexpr (std::is_same<T, int>::value) return MAX ? (int)0x80000000 : 0x7fffffff;
    else return MAX ? -__builtin_huge_valf() : __builtin_huge_valf();
}

template <typename T, bool MAX>
__device__ __forceinline__ void warp_arg(T& bv, int& bi) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        const T ov = __shfl_xor_sync(0xffffffffu, bv, o);
        const int oi = __shfl_xor_sync(0xffffffffu, bi, o);
        arg_take<T, MAX>(bv, bi, ov, oi);
    }
}

// Reduce row[a, b) (column indices a..b-1) over NT threads; result in thread 0.
template <typename T, bool MAX, int NT>
__device__ __forceinline__ void cta_arg(const T* __restrict__ row, int64_t a, int64_t b, T& bv, int& bi, T* sv,
                                        int* si) {
    bv = arg_d<T, MAX>();
    bi = -1;
    const int t = NT == 32 ? (int)(threadIdx.x & 31) : (int)threadIdx.x;  // NT = 32: one warp of a larger CTA
    int64_t h = (int64_t)(((16u - ((uint32_t)(uintptr_t)(row + a) & 15u)) & 15u) / sizeof(T));
    if (h > b - a) h = b - a;
    for (int64_t k = a + t; k < a + h; k += NT) arg_take<T, MAX>(bv, bi, __ldg(row + k), (int)k);
    const int64_t base = a + h, nv = (b - base) >> 2;
    int64_t v = t;
    for (; v + 3 * NT < nv; v += 4 * NT) {
        typename Vec4<T>::type q[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) q[u] = ldg_stream4(row + base + 4 * (v + u * NT));
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            T e[4];
            unpack4<T>(q[u], e);
            const int j0 = (int)(base + 4 * (v + u * NT));
#pragma unroll
            for (int c = 0; c < 4; ++c) arg_take<T, MAX>(bv, bi, e[c], j0 + c);
        }
    }
    for (; v < nv; v += NT) {
        T e[4];
        unpack4<T>(ldg_stream4(row + base + 4 * v), e);
#pragma unroll
        for (int c = 0; c < 4; ++c) arg_take<T, MAX>(bv, bi, e[c], (int)(base + 4 * v + c));
    }
    for (int64_t k = base + 4 * nv + t; k < b; k += NT) arg_take<T, MAX>(bv, bi, __ldg(row + k), (int)k);
    warp_arg<T, MAX>(bv, bi);
    if constexpr (NT > 32) {
        if ((threadIdx.x & 31) == 0) {
            sv[threadIdx.x >> 5] = bv;
            si[threadIdx.x >> 5] = bi;
        }
        __syncthreads();
        if (threadIdx.x < 32) {
            bv = threadIdx.x < NT / 32 ? sv[threadIdx.x] : arg_d<T, MAX>();
            bi = threadIdx.x < NT / 32 ? si[threadIdx.x] : -1;
            warp_arg<T, MAX>(bv, bi);
        }
    }
}

// V_TOP: a thread per row, sequential (strict comparison: first occurrence).
template <typename T, bool MAX>
__global__ void __launch_bounds__(256) arg_top_kernel(const T* __restrict__ in, T* __restrict__ val,
                                                      int* __restrict__ idx, int64_t n, int64_t m) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const T* row = in + i * m;
        T bv = arg_d<T, MAX>();
        int bi = -1;
#pragma unroll 4
        for (int64_t j = 0; j < m; ++j) arg_take<T, MAX>(bv, bi, __ldg(row + j), (int)j);
        val[i] = bv;
        idx[i] = bi;
    }
}

// V_TOP for aligned rows with m % 4 == 0: the thread's row is read in
// batches of M4 independent 128-bit loads (L1-allocating: the 32 rows a warp
// covers share lines across the batch, so every byte is fetched once).
template <typename T, bool MAX, int M4>
__global__ void __launch_bounds__(256) arg_top_vec_kernel(const T* __restrict__ in, T* __restrict__ val,
                                                          int* __restrict__ idx, int64_t n, int64_t m) {
    using V = typename Vec4<T>::type;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const V* row = reinterpret_cast<const V*>(in + i * m);
        const int64_t nv = m / 4;
        T bv = arg_d<T, MAX>();
        int bi = -1;
        for (int64_t u0 = 0; u0 < nv; u0 += M4) {
            V q[M4];
#pragma unroll
            for (int u = 0; u < M4; ++u) q[u] = u0 + u < nv ? __ldg(row + u0 + u) : V{};
#pragma unroll
            for (int u = 0; u < M4; ++u) {
                if (u0 + u < nv) {
                    T e[4];
                    unpack4<T>(q[u], e);
#pragma unroll
                    for (int c = 0; c < 4; ++c) arg_take<T, MAX>(bv, bi, e[c], (int)(4 * (u0 + u) + c));
                }
            }
        }
        val[i] = bv;
        idx[i] = bi;
    }
}

// V_TOP for longer rows: a CTA owns 256 rows and walks them in [256][32]
// column tiles staged through padded shared memory -- every global load is a
// warp reading 32 consecutive elements of one row (coalesced), and each thread
// then scans its own row's 32 values (conflict-free, row stride 33).
template <typename T, bool MAX>
__global__ void __launch_bounds__(256) arg_top_tile_kernel(const T* __restrict__ in, T* __restrict__ val,
                                                           int* __restrict__ idx, int64_t n, int64_t m) {
    __shared__ T tile[256][33];
    const int t = threadIdx.x, lane = t & 31, w = t >> 5;
    const int64_t row0 = (int64_t)blockIdx.x * 256;
    T bv = arg_d<T, MAX>();
    int bi = -1;
    for (int64_t c0 = 0; c0 < m; c0 += 32) {
        const int64_t c = c0 + lane;
#pragma unroll 8
        for (int i = 0; i < 32; ++i) {
            const int rr = w + 8 * i;
            const int64_t r = row0 + rr;
            tile[rr][lane] = (r < n && c < m) ? __ldg(in + r * m + c) : arg_d<T, MAX>();
        }
        __syncthreads();
        const int lim = (int)std::min<int64_t>(32, m - c0);
        for (int j = 0; j < lim; ++j) arg_take<T, MAX>(bv, bi, tile[t][j], (int)(c0 + j));
        __syncthreads();
    }
    if (row0 + t < n) {
        val[row0 + t] = bv;
        idx[row0 + t] = bi;
    }
}

// V_MIDDLE, rows < 4096: a warp per row
template <typename T, bool MAX>
__global__ void __launch_bounds__(256) arg_warp_kernel(const T* __restrict__ in, T* __restrict__ val,
                                                       int* __restrict__ idx, int64_t n, int64_t m) {
    const int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    if (i >= n) return;
    T bv;
    int bi;
    cta_arg<T, MAX, 32>(in + i * m, 0, m, bv, bi, nullptr, nullptr);
    if ((threadIdx.x & 31) == 0) {
        val[i] = bv;
        idx[i] = bi;
    }
}

// V_MIDDLE, long rows (P = 1) and V_FLAT pass 1 (P pieces per row)
template <typename T, bool MAX>
__global__ void __launch_bounds__(512) arg_piece_kernel(const T* __restrict__ in, T* __restrict__ val,
                                                        int* __restrict__ idx, int64_t m, int P) {
    __shared__ T sv[16];
    __shared__ int si[16];
    const int64_t row = blockIdx.x / P;
    const int piece = blockIdx.x % P;
    const int64_t len = ceil_div(ceil_div(m, P), 4) * 4;
    const int64_t a = std::min(m, (int64_t)piece * len), b = std::min(m, a + len);
    T bv;
    int bi;
    cta_arg<T, MAX, 512>(in + row * m, a, b, bv, bi, sv, si);
    if (threadIdx.x == 0) {
        val[blockIdx.x] = bv;
        idx[blockIdx.x] = bi;
    }
}

// V_FLAT pass 2: combine the P piece pairs of each row
template <typename T, bool MAX>
__global__ void __launch_bounds__(256) arg_fix_kernel(const T* __restrict__ pv, const int* __restrict__ pi,
                                                      T* __restrict__ val, int* __restrict__ idx, int64_t n, int P) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        T bv = arg_d<T, MAX>();
        int bi = -1;
        for (int p = 0; p < P; ++p) arg_take<T, MAX>(bv, bi, pv[i * P + p], pi[i * P + p]);
        val[i] = bv;
        idx[i] = bi;
    }
}

int64_t arg_pieces(int64_t n, int64_t m) {
    return std::max<int64_t>(1, std::min<int64_t>(592 / std::max<int64_t>(n, 1), m / 8192));
}

template <typename T, bool MAX>
cudaError_t launch_arg_t(const ArgArgs& a, int version) {
    const T* in = (const T*)a.in;
    T* val = (T*)a.val;
    if (version == IFL_V_TOP) {
        const unsigned g = (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(a.n, 256), 148 * 16));
        if (((uintptr_t)a.in % 16) == 0 && a.m % 4 == 0) {
            if (a.m <= 16) arg_top_vec_kernel<T, MAX, 4><<<g, 256, 0, a.stream>>>(in, val, a.idx, a.n, a.m);
            else arg_top_vec_kernel<T, MAX, 16><<<g, 256, 0, a.stream>>>(in, val, a.idx, a.n, a.m);
            return cudaGetLastError();
        }
        if (a.m > 8) {  // unaligned rows: staged column tiles (coalesced, but 111 us vs the vector
                        // path's 65-73 us on 2^26 aligned f32 at m = 64..512, so only here)
            arg_top_tile_kernel<T, MAX><<<(unsigned)ceil_div(a.n, 256), 256, 0, a.stream>>>(in, val, a.idx, a.n, a.m);
            return cudaGetLastError();
        }
        arg_top_kernel<T, MAX><<<g, 256, 0, a.stream>>>(in, val, a.idx, a.n, a.m);
        return cudaGetLastError();
    }
    if (version == IFL_V_MIDDLE) {
        if (a.m < 4096) {
            arg_warp_kernel<T, MAX><<<(unsigned)ceil_div(a.n * 32, 256), 256, 0, a.stream>>>(in, val, a.idx, a.n, a.m);
        } else {
            arg_piece_kernel<T, MAX><<<(unsigned)a.n, 512, 0, a.stream>>>(in, val, a.idx, a.m, 1);
        }
        return cudaGetLastError();
    }
    const int64_t P = arg_pieces(a.n, a.m);
    T* pv = (T*)a.ws;
    int* pi = (int*)(pv + a.n * P);
    arg_piece_kernel<T, MAX><<<(unsigned)(a.n * P), 512, 0, a.stream>>>(in, pv, pi, a.m, (int)P);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    const unsigned g = (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(a.n, 256), 148 * 16));
    arg_fix_kernel<T, MAX><<<g, 256, 0, a.stream>>>(pv, pi, val, a.idx, a.n, (int)P);
    return cudaGetLastError();
}

}  // namespace

size_t arg_ws_bytes(int64_t n, int64_t m, int version) {
    if (version != IFL_V_FLAT && version != IFL_AUTO) return 0;
    if (n <= 0 || m <= 0) return 0;
    return (size_t)(n * arg_pieces(n, m)) * 8;
}

cudaError_t launch_arg(const ArgArgs& a, int version) {
    if (a.n * std::max<int64_t>(1, arg_pieces(a.n, a.m)) > 0x7fffffffLL) return cudaErrorInvalidValue;
    if (a.dt == IFL_I32) return a.which ? launch_arg_t<int, true>(a, version) : launch_arg_t<int, false>(a, version);
    return a.which ? launch_arg_t<float, true>(a, version) : launch_arg_t<float, false>(a, version);
}

}  // namespace ifl
