// seg2.cu -- a reduce whose map function itself reduces (rule G9's e_rec,
// P:311-332, the Heston-like map / redomap / reduce nest):
//   out[i] = d_o (+) g_i0 (+) ... (+) g_i(m-1),   g_ij = d_i (x) f(x[i][j][0]) (x) ... (x) f(x[i][j][k-1])
// over an [n][m][k] array.  G3 at the outer map and G9's recursion into the
// map function give three versions here:
//   V_TOP     a thread per i, both inner levels sequential;
//   V_MIDDLE  a CTA per i: the j-level over its warps / threads, the k-level
//             inside a warp (k >= 32) or sequential in a thread (short k);
//   V_FLAT    (ifl_api.cpp) both levels flattened: segred^1 over the [n*m][k]
//             inner segments into a workspace, then segred^1 over [n][m] --
//             each through the library's own G3 selection.
#include <algorithm>

#include "common.cuh"
#include "dispatch.cuh"
#include "ifl_internal.h"

namespace ifl {

namespace {

template <typename T, int OPO, int OPI, int F>
__global__ void __launch_bounds__(256) seg2_top_kernel(const T* __restrict__ in, T* __restrict__ out, int64_t n,
                                                       int64_t m, int64_t k, T d_o, T d_i) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        Acc<OPO, T> acc(d_o);
        const T* row = in + i * m * k;
        for (int64_t j = 0; j < m; ++j) {
            Acc<OPI, T> g(d_i);
#pragma unroll 4
            for (int64_t q = 0; q < k; ++q) g.add(apply_map<F>(__ldg(row + j * k + q)));
            acc.add(g.get());
        }
        out[i] = acc.get();
    }
}

constexpr int kSeg2Threads = 256;

template <typename T, int OPO, int OPI, int F, bool WARP_INNER>
__global__ void __launch_bounds__(kSeg2Threads) seg2_mid_kernel(const T* __restrict__ in, T* __restrict__ out,
                                                                int64_t n, int64_t m, int64_t k, T d_o, T d_i) {
    __shared__ T red[kSeg2Threads / 32];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    for (int64_t i = blockIdx.x; i < n; i += gridDim.x) {
        const T* row = in + i * m * k;
        T acc = identity<OPO, T>();
        if constexpr (WARP_INNER) {  // a warp per inner segment j, k over the lanes
            for (int64_t j = w; j < m; j += kSeg2Threads / 32) {
                T g = identity<OPI, T>();
                for (int64_t q = lane; q < k; q += 32) g = combine<OPI>(g, apply_map<F>(__ldg(row + j * k + q)));
                g = warp_reduce<OPI>(g);
                acc = combine<OPO>(acc, combine<OPI>(d_i, g));  // lanes agree after the butterfly
            }
            if (lane != 0) acc = identity<OPO, T>();
        } else {  // a thread per inner segment j, k sequential
            for (int64_t j = threadIdx.x; j < m; j += kSeg2Threads) {
                T g = d_i;
                for (int64_t q = 0; q < k; ++q) g = combine<OPI>(g, apply_map<F>(__ldg(row + j * k + q)));
                acc = combine<OPO>(acc, g);
            }
        }
        acc = warp_reduce<OPO>(acc);
        if (lane == 0) red[w] = acc;
        __syncthreads();
        if (threadIdx.x == 0) {
            T r = d_o;
            for (int q = 0; q < kSeg2Threads / 32; ++q) r = combine<OPO>(r, red[q]);
            out[i] = r;
        }
        __syncthreads();
    }
}

template <typename T, int OPO, int OPI, int F>
cudaError_t launch_seg2_t(const Seg2Args& a, int version) {
    const T d_o = bits_to<T>(a.ne_o), d_i = bits_to<T>(a.ne_i);
    if (version == IFL_V_TOP) {
        const unsigned g = (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(a.n, 256), 148 * 16));
        seg2_top_kernel<T, OPO, OPI, F><<<g, 256, 0, a.stream>>>((const T*)a.in, (T*)a.out, a.n, a.m, a.k, d_o, d_i);
        return cudaGetLastError();
    }
    const unsigned g = (unsigned)std::max<int64_t>(1, std::min<int64_t>(a.n, (int64_t)148 * 8));
    if (a.k >= 32)
        seg2_mid_kernel<T, OPO, OPI, F, true><<<g, kSeg2Threads, 0, a.stream>>>((const T*)a.in, (T*)a.out, a.n, a.m,
                                                                                 a.k, d_o, d_i);
    else
        seg2_mid_kernel<T, OPO, OPI, F, false><<<g, kSeg2Threads, 0, a.stream>>>((const T*)a.in, (T*)a.out, a.n, a.m,
                                                                                  a.k, d_o, d_i);
    return cudaGetLastError();
}

// (outer op) x (inner op) x map x dtype: the inner op and the map come from
// the usual dispatch, the outer op from a second switch
template <typename T, int OPI, int F>
cudaError_t dispatch_outer(const Seg2Args& a, int version) {
    switch (a.op_o) {
    case OP_SUM: return launch_seg2_t<T, OP_SUM, OPI, F>(a, version);
    case OP_PROD: return launch_seg2_t<T, OP_PROD, OPI, F>(a, version);
    case OP_MIN: return launch_seg2_t<T, OP_MIN, OPI, F>(a, version);
    case OP_MAX: return launch_seg2_t<T, OP_MAX, OPI, F>(a, version);
    default: break;
    }
    if constexpr (std::is_same<T, int>::value) {
        switch (a.op_o) {
        case OP_AND: return launch_seg2_t<T, OP_AND, OPI, F>(a, version);
        case OP_OR: return launch_seg2_t<T, OP_OR, OPI, F>(a, version);
        case OP_XOR: return launch_seg2_t<T, OP_XOR, OPI, F>(a, version);
        default: break;
        }
    }
    return cudaErrorInvalidValue;
}

}  // namespace

cudaError_t launch_seg2(const Seg2Args& a, int version) {
    return dispatch_all(a.dt, a.op_i, a.f, [&](auto tt, auto opc, auto fc) -> cudaError_t {
        using T = decltype(tt);
        constexpr int OPI = decltype(opc)::value, F = decltype(fc)::value;
        return dispatch_outer<T, OPI, F>(a, version);
    });
}

}  // namespace ifl
