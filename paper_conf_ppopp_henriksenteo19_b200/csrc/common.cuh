// common.cuh -- element types, operators (+), maps f and sm_100a PTX helpers
// shared by the segred / segscan / redomap2 / tridag kernels.
//
// Operators follow P:79 (reduce/scan with an associative (+) and a neutral
// element 0_(+)); maps follow P:85 (redomap/scanomap = reduce/scan . map).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#include <math_constants.h>

#include <type_traits>

namespace ifl {

enum OpCode { OP_SUM = 0, OP_PROD = 1, OP_MIN = 2, OP_MAX = 3, OP_AND = 4, OP_OR = 5, OP_XOR = 6 };
enum MapCode { F_ID = 0, F_SQ = 1, F_ABS = 2 };

// ---------------------------------------------------------------- operators

template <int OP, typename T>
__host__ __device__ __forceinline__ T identity() {
    if constexpr (std::is_same<T, int>::value) {
        if constexpr (OP == OP_SUM) return 0;
        if constexpr (OP == OP_PROD) return 1;
        if constexpr (OP == OP_MIN) return 0x7fffffff;
        if constexpr (OP == OP_MAX) return (int)0x80000000;
        if constexpr (OP == OP_AND) return -1;
        if constexpr (OP == OP_OR) return 0;
        if constexpr (OP == OP_XOR) return 0;
    } else {
        if constexpr (OP == OP_SUM) return 0.0f;
        if constexpr (OP == OP_PROD) return 1.0f;
        if constexpr (OP == OP_MIN) return __builtin_huge_valf();
        if constexpr (OP == OP_MAX) return -__builtin_huge_valf();
    }
    return T();
}

// a (+) b.  int32 sum/prod wrap modulo 2^32 (computed unsigned).
template <int OP, typename T>
__device__ __forceinline__ T combine(T a, T b) {
    if constexpr (std::is_same<T, int>::value) {
        if constexpr (OP == OP_SUM) return (int)((unsigned)a + (unsigned)b);
        if constexpr (OP == OP_PROD) return (int)((unsigned)a * (unsigned)b);
        if constexpr (OP == OP_MIN) return min(a, b);
        if constexpr (OP == OP_MAX) return max(a, b);
        if constexpr (OP == OP_AND) return a & b;
        if constexpr (OP == OP_OR) return a | b;
        if constexpr (OP == OP_XOR) return a ^ b;
    } else {
        if constexpr (OP == OP_SUM) return a + b;
        if constexpr (OP == OP_PROD) return a * b;
        if constexpr (OP == OP_MIN) return fminf(a, b);
        if constexpr (OP == OP_MAX) return fmaxf(a, b);
    }
    return a;
}

// f(x).  f32 SQ uses __fmul_rn so it is never contracted into an FMA: the
// square is rounded to f32 exactly as the f32 -> f32 map of P:85 says.
template <int F, typename T>
__device__ __forceinline__ T apply_map(T x) {
    if constexpr (F == F_ID) return x;
    if constexpr (std::is_same<T, int>::value) {
        if constexpr (F == F_SQ) return (int)((unsigned)x * (unsigned)x);
        if constexpr (F == F_ABS) return x < 0 ? (int)(0u - (unsigned)x) : x;
    } else {
        if constexpr (F == F_SQ) return __fmul_rn(x, x);
        if constexpr (F == F_ABS) return fabsf(x);
    }
    return x;
}

template <typename T>
__device__ __forceinline__ uint32_t to_bits(T v) {
    if constexpr (std::is_same<T, int>::value) return (uint32_t)v;
    else return __float_as_uint(v);
}
template <typename T>
__device__ __forceinline__ T from_bits(uint32_t u) {
    if constexpr (std::is_same<T, int>::value) return (int)u;
    else return __uint_as_float(u);
}

// Vector of 4 elements (16 bytes) for 128-bit loads.
template <typename T> struct Vec4;
template <> struct Vec4<int> { using type = int4; };
template <> struct Vec4<float> { using type = float4; };

template <typename T>
__device__ __forceinline__ void unpack4(const typename Vec4<T>::type& v, T (&o)[4]) {
    o[0] = v.x; o[1] = v.y; o[2] = v.z; o[3] = v.w;
}

// Streaming 128-bit global load (read once: do not keep in L1).
template <typename T>
__device__ __forceinline__ typename Vec4<T>::type ldg_stream4(const T* p) {
    typename Vec4<T>::type r;
    if constexpr (std::is_same<T, int>::value) {
        asm volatile("ld.global.nc.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];"
                     : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
    } else {
        asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
                     : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "l"(p));
    }
    return r;
}

template <typename T>
__device__ __forceinline__ T ldg1(const T* p) { return __ldg(p); }

// Coherent (weak, non-.nc) loads for kernels whose input may alias their output
// (in-place scans, ifl.h): ld.global.nc requires memory that the kernel does not
// write, so the scan kernels read through these instead.
template <typename T>
__device__ __forceinline__ typename Vec4<T>::type ld_coh4(const T* p) {
    typename Vec4<T>::type r;
    if constexpr (std::is_same<T, int>::value) {
        asm volatile("ld.global.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];"
                     : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p) : "memory");
    } else {
        asm volatile("ld.global.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
                     : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "l"(p) : "memory");
    }
    return r;
}
template <typename T>
__device__ __forceinline__ T ld_coh1(const T* p) { return *p; }

// Running (+)-accumulator.  For f32 sums it is Kahan-compensated, so a long
// sequential chain (a thread-per-segment walk over m ~ 2^26 elements) stays
// within the 1e-5 relative parity bound; every other (+) is exact or
// associative already.
template <int OP, typename T>
struct Acc {
    T s;
    __device__ __forceinline__ Acc() {}
    __device__ __forceinline__ explicit Acc(T init) : s(init) {}
    __device__ __forceinline__ void add(T x) { s = combine<OP>(s, x); }
    __device__ __forceinline__ T get() const { return s; }
};
template <>
struct Acc<OP_SUM, float> {
    float s, c;
    __device__ __forceinline__ Acc() {}
    __device__ __forceinline__ explicit Acc(float init) : s(init), c(0.0f) {}
    __device__ __forceinline__ void add(float x) {
        const float y = __fsub_rn(x, c);
        const float t = __fadd_rn(s, y);
        c = __fsub_rn(__fsub_rn(t, s), y);
        if (!isfinite(c)) c = 0.0f;  // an infinite term: the sum is +-inf (or NaN), no compensation
        s = t;
    }
    __device__ __forceinline__ float get() const { return s; }
};

// ------------------------------------------------------- warp primitives

template <int OP, typename T>
__device__ __forceinline__ T warp_reduce(T v, int width = 32) {
    for (int off = width >> 1; off > 0; off >>= 1) v = combine<OP>(v, __shfl_xor_sync(0xffffffffu, v, off));
    return v;
}

// ------------------------------------------------------------ sm_100a PTX
// mbarrier + bulk async copy (TMA engine, cp.async.bulk) helpers.

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}

__device__ __forceinline__ void fence_mbar_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}

__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.release.cta.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
                 "r"(bytes)
                 : "memory");
}

__device__ __forceinline__ bool mbar_try_wait(uint64_t* bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.acquire.cta.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
    return ok != 0;
}

__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    while (!mbar_try_wait(bar, parity)) {
    }
}

// 1-D bulk copy global -> shared (TMA engine), completion on an mbarrier.
// dst/src 16-byte aligned, bytes a multiple of 16.
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
            smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar))
        : "memory");
}

// L2 cache policies for bulk copies (createpolicy): keep-in-L2 / stream-through.
__device__ __forceinline__ uint64_t policy_evict_last() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ void bulk_g2s_hint(void* dst, const void* src, uint32_t bytes, uint64_t* bar,
                                              uint64_t policy) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
            smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(policy)
        : "memory");
}
__device__ __forceinline__ void bulk_s2g_hint(void* dst, const void* src, uint32_t bytes, uint64_t policy) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group.L2::cache_hint [%0], [%1], %2, %3;" ::"l"(dst),
                 "r"(smem_u32(src)), "r"(bytes), "l"(policy)
                 : "memory");
}

// 1-D bulk copy shared -> global (TMA engine), bulk-group completion.
__device__ __forceinline__ void bulk_s2g(void* dst, const void* src, uint32_t bytes) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(smem_u32(src)),
                 "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_read0() {
    asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
}
__device__ __forceinline__ void bulk_wait_read1() {
    asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
}
template <int N>
__device__ __forceinline__ void bulk_wait_read_n() {
    asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ void bulk_wait0() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

// Make generic-proxy shared-memory writes visible to the async (TMA) proxy.
__device__ __forceinline__ void fence_proxy_async_smem() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

// ------------------------------------------------------- global atomics

__device__ __forceinline__ uint64_t ld_acquire_u64(const uint64_t* p) {
    uint64_t v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_u64(uint64_t* p, uint64_t v) {
    asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed_u64(uint64_t* p, uint64_t v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t ld_relaxed_u64(const uint64_t* p) {
    uint64_t v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ uint32_t ld_relaxed_u32(const uint32_t* p) {
    uint32_t v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

__host__ __device__ constexpr int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

// ------------------------------------------------ V_TOP warp-tile kernel
// V_TOP (thread per segment) for m = M in {16, 32, 64}, 16-byte-aligned in/out:
// each warp owns 32 consecutive rows (one contiguous 32*M-element block).  The
// block is loaded with coalesced 128-bit loads (all in flight at once), staged
// in shared memory with a row stride of M+4 words (16-byte aligned; the
// 128-bit stores and the lanes' row walks are bank-conflict-free), and each
// lane then walks its own row sequentially -- the inner level of P:233's e_top.
// For SCAN the results go back through the same tile and leave with coalesced
// 128-bit stores.  Non-persistent: one warp-tile per warp, top_tile_warps(M)
// warps per CTA (the tile is 32 * (M + 4) words per warp).
__host__ __device__ constexpr int top_tile_warps(int M) { return M <= 32 ? 8 : 4; }
template <typename T, int OP, int F, int M, bool SCAN>
__global__ void __launch_bounds__(32 * top_tile_warps(M)) top_tile_kernel(const T* in, T* out,
                                                                          int64_t n, T d, const T* __restrict__ seed) {
    using V = typename Vec4<T>::type;
    constexpr int S = M + 4, W4 = M / 4, WPC = top_tile_warps(M);  // row stride (words), words per row
    __shared__ __align__(16) T sm[WPC][32 * S];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    T* s = sm[warp];
    const int64_t r0 = ((int64_t)blockIdx.x * WPC + warp) * 32;
    if (r0 >= n) return;
    const int rows = (int)min((int64_t)32, n - r0);
    const T* src = in + r0 * M;
    V q[W4];
#pragma unroll
    for (int u = 0; u < W4; ++u) {
        const int q4 = lane + 32 * u;  // 16-byte word of the block
        if (q4 < rows * W4) q[u] = SCAN ? ld_coh4(src + 4 * q4) : ldg_stream4(src + 4 * q4);  // scans may be in place
    }
#pragma unroll
    for (int u = 0; u < W4; ++u) {
        const int q4 = lane + 32 * u;
        if (q4 < rows * W4) *reinterpret_cast<V*>(&s[(q4 / W4) * S + 4 * (q4 % W4)]) = q[u];
    }
    __syncwarp();
    if (lane < rows) {
        T* row = s + lane * S;
        if constexpr (SCAN) {
            T a = seed ? seed[r0 + lane] : d;
#pragma unroll
            for (int j = 0; j < W4; ++j) {
                V v = *reinterpret_cast<const V*>(row + 4 * j);
                a = combine<OP>(a, apply_map<F>(v.x));
                v.x = a;
                a = combine<OP>(a, apply_map<F>(v.y));
                v.y = a;
                a = combine<OP>(a, apply_map<F>(v.z));
                v.z = a;
                a = combine<OP>(a, apply_map<F>(v.w));
                v.w = a;
                *reinterpret_cast<V*>(row + 4 * j) = v;
            }
        } else {
            T a[4] = {d, identity<OP, T>(), identity<OP, T>(), identity<OP, T>()};
#pragma unroll
            for (int j = 0; j < W4; ++j) {
                const V v = *reinterpret_cast<const V*>(row + 4 * j);
                a[0] = combine<OP>(a[0], apply_map<F>(v.x));
                a[1] = combine<OP>(a[1], apply_map<F>(v.y));
                a[2] = combine<OP>(a[2], apply_map<F>(v.z));
                a[3] = combine<OP>(a[3], apply_map<F>(v.w));
            }
            out[r0 + lane] = combine<OP>(combine<OP>(a[0], a[1]), combine<OP>(a[2], a[3]));
        }
    }
    if constexpr (SCAN) {
        __syncwarp();
        T* dst = out + r0 * M;
#pragma unroll
        for (int u = 0; u < W4; ++u) {
            const int q4 = lane + 32 * u;
            if (q4 < rows * W4) *reinterpret_cast<V*>(dst + 4 * q4) = *reinterpret_cast<const V*>(&s[(q4 / W4) * S + 4 * (q4 % W4)]);
        }
    }
}

}  // namespace ifl
