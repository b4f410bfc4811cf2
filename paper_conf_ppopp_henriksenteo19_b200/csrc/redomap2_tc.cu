// redomap2_tc.cu -- V_TOP of redomap2 for bf16 inputs on the 5th-generation
// tensor cores: segmap^1 <i><j> (redomap (+) (*) 0 xs ys) with block tiling
// (paper versions 2/3), where the "register tiling" of the paper
// becomes a TMEM accumulator tile.
//
// One CTA computes a 128 x 256 fp32 tile of C = A * Bt^T (A [n][m], Bt [p][m],
// both K-major bf16 -- exactly the layout P:122 maps over):
//   warp 0 (one lane)  TMA producer: cp.async.bulk.tensor 2-D loads of the
//                      128x64 A and 256x64 Bt k-tiles (128-byte swizzle) into a
//                      4-stage shared-memory ring, completion on mbarriers;
//   warp 1 (one lane)  MMA issuer: tcgen05.mma.cta_group::1.kind::f16,
//                      M=128 N=256 K=16, accumulating in TMEM (256 columns);
//                      tcgen05.commit frees ring stages and signals the end;
//   warps 0-3          epilogue: tcgen05.ld 32x32b -> registers -> C (fp32).
// No CUTLASS: descriptors and PTX are written out here.
#include <cuda.h>
#include <cuda_bf16.h>

#include <algorithm>
#include <mutex>

#include "common.cuh"
#include "ifl_internal.h"

namespace ifl {

constexpr int TC_BM = 128, TC_BN = 256, TC_BK = 64, TC_STAGES = 4;
constexpr int TC_A_BYTES = TC_BM * TC_BK * 2;  // 16 KB
constexpr int TC_B_BYTES = TC_BN * TC_BK * 2;  // 32 KB
constexpr int TC_STAGE_BYTES = TC_A_BYTES + TC_B_BYTES;
constexpr int TC_SMEM = TC_STAGES * TC_STAGE_BYTES + 1024;  // + alignment slack
constexpr int TC_TMEM_COLS = 256;

// ---------------------------------------------------------------- PTX wrappers

__device__ __forceinline__ void tma_load_2d(void* dst, const CUtensorMap* map, int c0, int c1, uint64_t* bar) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(
            smem_u32(dst)),
        "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(smem_u32(bar))
        : "memory");
}

// UMMA shared-memory descriptor (sm_100): K-major operand, 128-byte swizzle,
// 8-row core-matrix groups 1024 bytes apart.
__device__ __forceinline__ uint64_t umma_desc_sw128(uint32_t saddr) {
    uint64_t d = 0;
    d |= (uint64_t)((saddr & 0x3FFFFu) >> 4);  // start address
    d |= (uint64_t)1 << 16;                    // leading byte offset (unused for swizzled K-major)
    d |= (uint64_t)(1024 >> 4) << 32;          // stride byte offset: 8 rows x 128 B
    d |= (uint64_t)1 << 46;                    // descriptor version (sm_100)
    d |= (uint64_t)2 << 61;                    // layout: SWIZZLE_128B
    return d;
}

// UMMA shared-memory descriptor for an MN-major operand (B given as yss
// [m][p]: n contiguous), 128-byte swizzle: atoms of 64 n x 8 k (8 rows of
// 128 B), 8-k-row groups SBO = 1024 B apart, 64-wide n blocks LBO apart (the
// TMA boxes of one stage, 64 k-rows x 128 B = 8 KB each).
__device__ __forceinline__ uint64_t umma_desc_mn_sw128(uint32_t saddr, uint32_t lbo) {
    uint64_t d = 0;
    d |= (uint64_t)((saddr & 0x3FFFFu) >> 4);  // start address
    d |= (uint64_t)((lbo >> 4) & 0x3FFFu) << 16;  // leading byte offset: between n blocks
    d |= (uint64_t)(1024 >> 4) << 32;          // stride byte offset: between 8-row k groups
    d |= (uint64_t)1 << 46;                    // descriptor version (sm_100)
    d |= (uint64_t)2 << 61;                    // layout: SWIZZLE_128B
    return d;
}

// instruction descriptor, kind::f16: D f32, A/B bf16, both K-major, M x N
__host__ __device__ constexpr uint32_t umma_idesc_bf16(int M, int N) {
    return (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}

__device__ __forceinline__ void umma_bf16(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                          uint32_t accumulate) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
        "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate)
        : "memory");
}

__device__ __forceinline__ void umma_commit(uint64_t* bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(bar))
                 : "memory");
}

__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

__device__ __forceinline__ void tmem_ld_32x32b_x32(uint32_t taddr, uint32_t (&r)[32]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
        "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
          "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
          "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
        : "r"(taddr));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}

// ------------------------------------------------------------------ kernel

// Persistent, warp-specialised: 6 warps.
//   warp 0 (lane 0)  TMA producer over every (tile, k-tile) of the CTA's items
//   warp 1           TMEM allocation (512 columns = two 256-column fp32
//                    accumulators); lane 0 issues the MMAs
//   warps 2-5        epilogue; warp w reads TMEM lanes 32*(w % 4) .. +31
// Item = (k-split z, output tile); items are strided by gridDim.x.  The MMA
// warp accumulates item i into accumulator i & 1 while the epilogue drains
// item i-1 from the other one (tmem_full / tmem_empty mbarriers).
// Epilogue: with TST (C 16-byte aligned, p % 4 == 0) each warp writes its
// 32 x 32 fp32 chunk into a 128-byte-swizzled, double-buffered staging tile
// and one lane stores it with a 3-D TMA bulk-tensor store ({col,row,split});
// otherwise a padded smem transpose feeds coalesced row stores.
constexpr int TC_THREADS = 192;
#ifndef IFL_TC_GROUP
#define IFL_TC_GROUP 16
#endif
constexpr int TC_EPI_BYTES = 4 * 2 * 32 * 32 * 4;  // 4 warps x 2 buffers x 4 KB (>= 4 x 32 x 33 x 4)
constexpr int TC_SMEM_P = TC_STAGES * TC_STAGE_BYTES + TC_EPI_BYTES + 1024;

__device__ __forceinline__ void tma_store_3d(const CUtensorMap* map, const void* src, int c0, int c1, int c2) {
    asm volatile("cp.async.bulk.tensor.3d.global.shared::cta.bulk_group [%0, {%2, %3, %4}], [%1];" ::"l"(
                     reinterpret_cast<uint64_t>(map)),
                 "r"(smem_u32(src)), "r"(c0), "r"(c1), "r"(c2)
                 : "memory");
}

// BMN: B is yss [m][p] (MN-major, read in place: four 64-column TMA boxes per
// stage, MN-major descriptors, the b_major bit of the instruction descriptor).
template <bool TST, bool BMN>
__global__ void __launch_bounds__(TC_THREADS, 1)
    mm_top_tc_kernel(const __grid_constant__ CUtensorMap mapA, const __grid_constant__ CUtensorMap mapB,
                     const __grid_constant__ CUtensorMap mapC, float* C, float* part, int64_t n, int64_t m,
                     int64_t p, int kps, int splits, int group) {
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~(uintptr_t)1023);
    float* stage_base = reinterpret_cast<float*>(smem + TC_STAGES * TC_STAGE_BYTES);
    __shared__ alignas(8) uint64_t full[TC_STAGES], empty[TC_STAGES], tfull[2], tempty[2];
    __shared__ uint32_t tmem_base;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int ntx = (int)ceil_div(p, TC_BN), nty = (int)ceil_div(n, TC_BM);
    const int ntiles = ntx * nty;
    const int items = ntiles * splits;
    const int nk_all = (int)ceil_div(m, TC_BK);
    // Grouped tile order: bands of TC_GROUP row tiles, walked column by column
    // inside a band, so the ~148 tiles in flight share a few A row bands and
    // B column tiles through L2 (plain row order re-streams all of B once per
    // wave: 4.3x the algorithmic DRAM bytes at 8192^3).
    auto decode = [&](int it, int& z, int& m0, int& n0, int& kt0, int& nk) {
        z = it / ntiles;
        const int rem = it - z * ntiles;
        const int gsz = group * ntx;
        const int g = rem / gsz, r = rem - g * gsz;
        const int rows = min(group, nty - g * group);
        m0 = (g * group + r % rows) * TC_BM;
        n0 = (r / rows) * TC_BN;
        kt0 = z * kps;
        nk = min(kps, nk_all - kt0);
    };

    if (threadIdx.x == 0) {
        for (int s = 0; s < TC_STAGES; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], 1);
        }
        for (int a = 0; a < 2; ++a) {
            mbar_init(&tfull[a], 1);
            mbar_init(&tempty[a], 4);
        }
        fence_mbar_init();
        asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&mapA)) : "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&mapB)) : "memory");
        if (TST) asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&mapC)) : "memory");
    }
    if (warp == 1) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tmem_base)),
                     "n"(2 * TC_TMEM_COLS)
                     : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = tmem_base;

    if (warp == 0) {
        if (lane == 0) {  // ---- TMA producer
            int gk = 0;
            for (int it = blockIdx.x; it < items; it += gridDim.x) {
                int z, m0, n0, kt0, nk;
                decode(it, z, m0, n0, kt0, nk);
                for (int kt = 0; kt < nk; ++kt, ++gk) {
                    const int s = gk % TC_STAGES;
                    mbar_wait(&empty[s], ((gk / TC_STAGES) & 1) ^ 1);
                    uint8_t* sa = smem + s * TC_STAGE_BYTES;
                    mbar_arrive_expect_tx(&full[s], TC_STAGE_BYTES);
                    tma_load_2d(sa, &mapA, (kt0 + kt) * TC_BK, m0, &full[s]);
                    if constexpr (BMN) {
#pragma unroll
                        for (int q = 0; q < TC_BN / 64; ++q)
                            tma_load_2d(sa + TC_A_BYTES + q * (TC_BK * 128), &mapB, n0 + 64 * q, (kt0 + kt) * TC_BK,
                                        &full[s]);
                    } else {
                        tma_load_2d(sa + TC_A_BYTES, &mapB, (kt0 + kt) * TC_BK, n0, &full[s]);
                    }
                }
            }
        }
    } else if (warp == 1) {
        if (lane == 0) {  // ---- MMA issuer
            constexpr uint32_t idesc = umma_idesc_bf16(TC_BM, TC_BN) | (BMN ? (1u << 16) : 0u);
            int gk = 0, li = 0;
            for (int it = blockIdx.x; it < items; it += gridDim.x, ++li) {
                int z, m0, n0, kt0, nk;
                decode(it, z, m0, n0, kt0, nk);
                const int acc = li & 1;
                mbar_wait(&tempty[acc], ((li >> 1) & 1) ^ 1);  // epilogue has drained this accumulator
                tc_fence_after();
                const uint32_t d = tmem + (uint32_t)(acc * TC_TMEM_COLS);
                for (int kt = 0; kt < nk; ++kt, ++gk) {
                    const int s = gk % TC_STAGES;
                    mbar_wait(&full[s], (gk / TC_STAGES) & 1);
                    tc_fence_after();
                    const uint32_t sa = smem_u32(smem + s * TC_STAGE_BYTES);
                    const uint32_t sb = sa + TC_A_BYTES;
#pragma unroll
                    for (int kk = 0; kk < TC_BK / 16; ++kk) {
                        // K = 16 per MMA: 32 bytes along a K-major row, 16 rows (2 KB) of an MN-major box
                        const uint64_t bd = BMN ? umma_desc_mn_sw128(sb + kk * 2048, TC_BK * 128)
                                                : umma_desc_sw128(sb + kk * 32);
                        umma_bf16(d, umma_desc_sw128(sa + kk * 32), bd, idesc, (kt | kk) != 0 ? 1u : 0u);
                    }
                    umma_commit(&empty[s]);
                }
                umma_commit(&tfull[acc]);
            }
        }
    } else {
        // ---- epilogue warps 2..5: TMEM -> registers -> padded smem -> coalesced rows
        const int quad = warp & 3;  // TMEM lane quadrant this warp may access
        float* stage = stage_base + (warp - 2) * (2 * 32 * 32);
        int li = 0, nst = 0;
        for (int it = blockIdx.x; it < items; it += gridDim.x, ++li) {
            int z, m0, n0, kt0, nk;
            decode(it, z, m0, n0, kt0, nk);
            float* out = splits == 1 ? C : part + (int64_t)z * n * p;
            const int acc = li & 1;
            mbar_wait(&tfull[acc], (li >> 1) & 1);
            __syncwarp();
            tc_fence_after();
#pragma unroll 1
            for (int c = 0; c < TC_BN; c += 32) {
                uint32_t r[32];
                tmem_ld_32x32b_x32(tmem + ((uint32_t)(quad * 32) << 16) + (uint32_t)(acc * TC_TMEM_COLS + c), r);
                if (c + 32 == TC_BN) {  // accumulator drained: let the MMA warp reuse it
                    tc_fence_before();
                    __syncwarp();
                    if (lane == 0) mbar_arrive_expect_tx(&tempty[acc], 0);
                }
                if constexpr (TST) {
                    if (n0 + c >= p) continue;
                    float* buf = stage + (nst & 1) * (32 * 32);
                    if (lane == 0) bulk_wait_read1();  // the store that last read buf has finished
                    __syncwarp();
                    float4* row = reinterpret_cast<float4*>(buf + lane * 32);
#pragma unroll
                    for (int q = 0; q < 8; ++q)
                        row[q ^ (lane & 7)] = make_float4(__uint_as_float(r[4 * q]), __uint_as_float(r[4 * q + 1]),
                                                          __uint_as_float(r[4 * q + 2]), __uint_as_float(r[4 * q + 3]));
                    fence_proxy_async_smem();
                    __syncwarp();
                    if (lane == 0) {
                        tma_store_3d(&mapC, buf, n0 + c, m0 + quad * 32, splits == 1 ? 0 : z);
                        bulk_commit();
                    }
                    ++nst;
                } else {
#pragma unroll
                    for (int q = 0; q < 32; ++q) stage[lane * 33 + q] = __uint_as_float(r[q]);
                    __syncwarp();
                    const int64_t col = (int64_t)n0 + c + lane;
                    for (int rr = 0; rr < 32; ++rr) {
                        const int64_t row = (int64_t)m0 + quad * 32 + rr;
                        if (row < n && col < p) out[row * p + col] = stage[rr * 33 + lane];
                    }
                    __syncwarp();
                }
            }
        }
        if (TST && lane == 0) bulk_wait0();
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 1)
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "n"(2 * TC_TMEM_COLS)
                     : "memory");
}

// ------------------------------------------------------------------ host side

using EncodeTiledFn = CUresult (*)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                   const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                   CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static EncodeTiledFn encode_fn() {
    static EncodeTiledFn fn = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        void* p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<EncodeTiledFn>(p);
    });
    return fn;
}

static bool make_map(CUtensorMap* map, const void* base, int64_t rows, int64_t k, int box_rows) {
    EncodeTiledFn fn = encode_fn();
    if (!fn) return false;
    const cuuint64_t dims[2] = {(cuuint64_t)k, (cuuint64_t)rows};
    const cuuint64_t strides[1] = {(cuuint64_t)k * 2};
    const cuuint32_t box[2] = {(cuuint32_t)TC_BK, (cuuint32_t)box_rows};
    const cuuint32_t estr[2] = {1, 1};
    return fn(map, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims, strides, box, estr,
              CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
              CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// yss [m][p] (MN-major B): 64 (n) x 64 (k) boxes, 128-byte swizzle
static bool make_map_mn(CUtensorMap* map, const void* base, int64_t m, int64_t p) {
    EncodeTiledFn fn = encode_fn();
    if (!fn) return false;
    const cuuint64_t dims[2] = {(cuuint64_t)p, (cuuint64_t)m};
    const cuuint64_t strides[1] = {(cuuint64_t)p * 2};
    const cuuint32_t box[2] = {64, (cuuint32_t)TC_BK};
    const cuuint32_t estr[2] = {1, 1};
    return fn(map, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims, strides, box, estr,
              CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
              CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// fp32 output [splits][n][p] as a 3-D map, 32 x 32 boxes, 128-byte swizzle
static bool make_out_map(CUtensorMap* map, float* base, int64_t n, int64_t p, int splits) {
    EncodeTiledFn fn = encode_fn();
    if (!fn) return false;
    const cuuint64_t dims[3] = {(cuuint64_t)p, (cuuint64_t)n, (cuuint64_t)splits};
    const cuuint64_t strides[2] = {(cuuint64_t)p * 4, (cuuint64_t)(n * p * 4)};
    const cuuint32_t box[3] = {32, 32, 1};
    const cuuint32_t estr[3] = {1, 1, 1};
    return fn(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, base, dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
              CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_NONE,
              CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// TMA needs 16-byte-aligned bases and row pitches (m % 8 == 0 for bf16);
// everything else (ragged n, p, m) is covered by TMA zero-fill and masking.
bool tc_shape_ok(int64_t n, int64_t m, int64_t p, const void* A, const void* Bt) {
    return n > 0 && p > 0 && m >= 8 && m % 8 == 0 && ((uintptr_t)A % 16 == 0) && ((uintptr_t)Bt % 16 == 0) &&
           n < (1ll << 31) && p < (1ll << 31) && m < (1ll << 31) && encode_fn() != nullptr;
}

__global__ void mm_splitk_finalize(const float* __restrict__ part, float* __restrict__ C, int64_t outs, int splits) {
    for (int64_t o = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; o < outs; o += (int64_t)gridDim.x * blockDim.x) {
        float r = 0.f;
        for (int s = 0; s < splits; ++s) r += part[(int64_t)s * outs + o];
        C[o] = r;
    }
}

// splits: 1 = plain TOP tile; >1 = k split across CTAs (ws holds the partial
// tiles).  tc_splits() picks them: TOP only fills idle SMs (>= 8 k-tiles per
// split); FLAT (segred over all three levels) splits as far as 2 CTAs per SM.
int tc_splits(int64_t n, int64_t m, int64_t p, bool flat) {
    const int64_t tiles = ceil_div(n, TC_BM) * ceil_div(p, TC_BN);
    const int64_t nk = ceil_div(m, TC_BK);
    int64_t s = flat ? ceil_div((int64_t)296, tiles) : (int64_t)148 / tiles;
    const int64_t cap = flat ? nk : std::max<int64_t>(1, nk / 8);
    s = std::max<int64_t>(1, std::min(s, cap));
    const int64_t kps = ceil_div(nk, s);
    return (int)ceil_div(nk, kps);
}

bool tc_mn_ok(int64_t n, int64_t m, int64_t p, const void* A, const void* B) {
    return tc_shape_ok(n, m, p, A, B) && p % 8 == 0;  // yss rows: 16-byte pitch
}

cudaError_t launch_mm_top_tc(const void* A, const void* Bt, float* C, float* part, int64_t n, int64_t m, int64_t p,
                             int splits, cudaStream_t s, bool b_mn) {
    CUtensorMap ma, mb;
    if (!make_map(&ma, A, n, m, TC_BM) || !(b_mn ? make_map_mn(&mb, Bt, m, p) : make_map(&mb, Bt, p, m, TC_BN)))
        return cudaErrorInvalidValue;
    static std::once_flag once;
    std::call_once(once, [] {
        cudaFuncSetAttribute(mm_top_tc_kernel<true, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, TC_SMEM_P);
        cudaFuncSetAttribute(mm_top_tc_kernel<false, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, TC_SMEM_P);
        cudaFuncSetAttribute(mm_top_tc_kernel<true, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, TC_SMEM_P);
        cudaFuncSetAttribute(mm_top_tc_kernel<false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, TC_SMEM_P);
    });
    const int nk = (int)ceil_div(m, TC_BK);
    const int kps = (int)ceil_div(nk, splits);
    splits = (int)ceil_div(nk, kps);
    float* out = splits == 1 ? C : part;
    CUtensorMap mc;
    const bool tst = p % 4 == 0 && (uintptr_t)out % 16 == 0 && make_out_map(&mc, out, n, p, splits);
    const int64_t items = ceil_div(n, TC_BM) * ceil_div(p, TC_BN) * splits;
    static int sms = 0;
    if (!sms) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        if (sms <= 0) sms = 148;
    }
    const int grid = (int)std::min<int64_t>(items, sms);
    // rasterisation band: grouped only when the operands overflow L2 (B200,
    // 8192^3: 1.51 vs 1.36 PF, DRAM 1.3 vs 3.4 GB; 4096^3 is faster in row order)
    const int64_t opbytes = 2 * (n * m + p * m);
    const int group = opbytes > ((int64_t)96 << 20) ? IFL_TC_GROUP : 1;
    if (tst) {
        if (b_mn)
            mm_top_tc_kernel<true, true><<<grid, TC_THREADS, TC_SMEM_P, s>>>(ma, mb, mc, C, part, n, m, p, kps, splits,
                                                                            group);
        else
            mm_top_tc_kernel<true, false><<<grid, TC_THREADS, TC_SMEM_P, s>>>(ma, mb, mc, C, part, n, m, p, kps, splits,
                                                                             group);
    } else {
        if (b_mn)
            mm_top_tc_kernel<false, true><<<grid, TC_THREADS, TC_SMEM_P, s>>>(ma, mb, ma, C, part, n, m, p, kps, splits,
                                                                             group);
        else
            mm_top_tc_kernel<false, false><<<grid, TC_THREADS, TC_SMEM_P, s>>>(ma, mb, ma, C, part, n, m, p, kps,
                                                                              splits, group);
    }
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess || splits == 1) return e;
    const int64_t outs = n * p;
    mm_splitk_finalize<<<(unsigned)std::min<int64_t>(ceil_div(outs, 256), 148 * 16), 256, 0, s>>>(part, C, outs, splits);
    return cudaGetLastError();
}

}  // namespace ifl
