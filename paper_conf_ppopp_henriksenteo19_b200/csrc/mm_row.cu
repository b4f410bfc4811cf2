// mm_row.cu -- the row-level leaves of matrix multiplication's branching tree
// (SURVEY 8(f) NEXT-2).  Rule G3 applied to the OUTER map of
//   map (\xs -> map (\ys -> redomap (+) (*) 0 xs ys) (transpose yss)) xss
// (Par = n rows) gives, before the recursion into the two-map context that
// the three existing redomap2 versions cover:
//   IFL_V_ROW_TOP     segmap^1 <xs> (map (\ys -> redomap ...) yss'): a thread
//                     per row of C, the inner map and redomap sequential;
//   IFL_V_ROW_MIDDLE  segmap^1 <xs> (segmap^0 <ys> (redomap ...)): a CTA per
//                     row of C -- the row of A staged once in shared memory
//                     (fit clause: m <= 8192), a warp per output j of
//                     the row, k across the lanes.
// Both read B as yss^T [p][m] (the k-major layout the library keeps; a
// row-major B is transposed first, as for the other versions).
#include <cuda_bf16.h>

#include <algorithm>

#include "common.cuh"
#include "ifl_internal.h"

namespace ifl {

namespace {

__device__ __forceinline__ float ld_f(const float* p) { return __ldg(p); }
__device__ __forceinline__ float ld_f(const __nv_bfloat16* p) { return __bfloat162float(p[0]); }

template <typename Tin>
__global__ void __launch_bounds__(256) mm_row_top_kernel(const Tin* __restrict__ A, const Tin* __restrict__ Bt,
                                                         float* __restrict__ C, int64_t n, int64_t m, int64_t p) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const Tin* a = A + i * m;
        for (int64_t j = 0; j < p; ++j) {  // every thread of a warp reads the same row of B: a broadcast
            const Tin* b = Bt + j * m;
            float acc0 = 0.f, acc1 = 0.f;
            int64_t k = 0;
            for (; k + 1 < m; k += 2) {
                acc0 = fmaf(ld_f(a + k), ld_f(b + k), acc0);
                acc1 = fmaf(ld_f(a + k + 1), ld_f(b + k + 1), acc1);
            }
            if (k < m) acc0 = fmaf(ld_f(a + k), ld_f(b + k), acc0);
            C[i * p + j] = acc0 + acc1;
        }
    }
}

constexpr int kRowMidThreads = 256;

template <typename Tin>
__global__ void __launch_bounds__(kRowMidThreads) mm_row_mid_kernel(const Tin* __restrict__ A,
                                                                     const Tin* __restrict__ Bt, float* __restrict__ C,
                                                                     int64_t n, int64_t m, int64_t p) {
    extern __shared__ float s_a[];  // the row of A, as f32
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    for (int64_t i = blockIdx.x; i < n; i += gridDim.x) {
        __syncthreads();  // the previous row's readers are done
        for (int64_t k = threadIdx.x; k < m; k += kRowMidThreads) s_a[k] = ld_f(A + i * m + k);
        __syncthreads();
        for (int64_t j = w; j < p; j += kRowMidThreads / 32) {
            const Tin* b = Bt + j * m;
            float acc = 0.f;
            for (int64_t k = lane; k < m; k += 32) acc = fmaf(s_a[k], ld_f(b + k), acc);
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
            if (lane == 0) C[i * p + j] = acc;
        }
    }
}

template <typename Tin>
cudaError_t run_row(int version, const Tin* A, const Tin* Bt, float* C, int64_t n, int64_t m, int64_t p,
                    cudaStream_t s) {
    if (version == IFL_V_ROW_TOP) {
        const unsigned g = (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, 256), 148 * 16));
        mm_row_top_kernel<Tin><<<g, 256, 0, s>>>(A, Bt, C, n, m, p);
        return cudaGetLastError();
    }
    const size_t smem = (size_t)std::max<int64_t>(m, 1) * sizeof(float);
    auto k = mm_row_mid_kernel<Tin>;
    if (smem > 48 * 1024) cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    const unsigned g = (unsigned)std::max<int64_t>(1, std::min<int64_t>(n, (int64_t)148 * 8));
    k<<<g, kRowMidThreads, smem, s>>>(A, Bt, C, n, m, p);
    return cudaGetLastError();
}

}  // namespace

bool mm_row_mid_fits(int64_t m) { return m <= kMmRowMaxM; }

cudaError_t launch_mm_row(int version, const void* A, const void* Bt, float* C, int64_t n, int64_t m, int64_t p,
                          int in_dt, cudaStream_t s) {
    if (in_dt == IFL_F32) return run_row<float>(version, (const float*)A, (const float*)Bt, C, n, m, p, s);
    return run_row<__nv_bfloat16>(version, (const __nv_bfloat16*)A, (const __nv_bfloat16*)Bt, C, n, m, p, s);
}

}  // namespace ifl
