// redomap2.cu -- the map-map-redomap contraction of P:122,
//     C = map (\xs -> map (\ys -> redomap (+) (*) 0 xs ys) (transpose yss)) xss,
// in the three code versions of P:126-134 / rule G3:
//   V_FLAT   segred^1 <xs in xss> <ys in yss^T> <x y in xs ys> (+) 0 (x*y)
//            (paper version 1): every (i, j, k) parallel -- the m-long dot
//            products are split across CTAs (split-K), partials reduced in a
//            deterministic second pass.  For degenerate shapes (n*p small).
//   V_MIDDLE segmap^1 <i><j> (segred^0 <k> ...): a group of 1-8 warps per
//            output element (more when few outputs reduce a long k), lanes
//            split k, shuffle-tree reduction.
//   V_TOP    segmap^1 <i><j> (redomap sequential in k) with block tiling and
//            register tiling (paper versions 2 and 3): a 128x128 output tile
//            per CTA, 8x8 per thread, k-tiles double-buffered in shared
//            memory.  bf16 inputs take the tcgen05/TMEM/TMA tensor-core kernel
//            (redomap2_tc.cu) when the shape allows.
// A is [n][m]; B is yss^T as [p][m] (b_kmajor = 1, the array P:122 maps over)
// or yss as [m][p] (b_kmajor = 0: read in place by the SIMT tile kernels and
// the skinny engine; transposed into the workspace first for V_MIDDLE, the
// row-level leaves and the tcgen05 kernel).
// Inputs f32 or bf16, accumulation and C in f32.
#include <cuda_bf16.h>

#include <algorithm>

#include "common.cuh"
#include "ifl_internal.h"

namespace ifl {

// ------------------------------------------------------------- helpers

template <typename Tin>
__device__ __forceinline__ float to_f(Tin v) {
    if constexpr (std::is_same<Tin, float>::value) return v;
    else return __bfloat162float(v);
}

// E = elements per 16-byte vector
template <typename Tin>
struct VecE {
    static constexpr int E = 16 / sizeof(Tin);
};

template <typename Tin>
__device__ __forceinline__ void load16(const Tin* p, float (&o)[VecE<Tin>::E]) {
    const uint4 u = __ldg(reinterpret_cast<const uint4*>(p));
    if constexpr (std::is_same<Tin, float>::value) {
        o[0] = __uint_as_float(u.x);
        o[1] = __uint_as_float(u.y);
        o[2] = __uint_as_float(u.z);
        o[3] = __uint_as_float(u.w);
    } else {
        const uint32_t w[4] = {u.x, u.y, u.z, u.w};
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            o[2 * q] = __uint_as_float(w[q] << 16);
            o[2 * q + 1] = __uint_as_float(w[q] & 0xffff0000u);
        }
    }
}

// --------------------------------------------------------- B transpose
// yss [m][p] -> yss^T [p][m] in the workspace (32x32 smem tiles, coalesced).
template <typename Tin>
__global__ void __launch_bounds__(256) transpose_kernel(const Tin* __restrict__ B, Tin* __restrict__ Bt, int64_t m,
                                                        int64_t p) {
    __shared__ Tin tile[32][33];
    const int64_t k0 = (int64_t)blockIdx.y * 32, j0 = (int64_t)blockIdx.x * 32;
    const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5;
    for (int r = ty; r < 32; r += 8)
        if (k0 + r < m && j0 + tx < p) tile[r][tx] = B[(k0 + r) * p + j0 + tx];
    __syncthreads();
    for (int r = ty; r < 32; r += 8)
        if (j0 + r < p && k0 + tx < m) Bt[(j0 + r) * m + k0 + tx] = tile[tx][r];
}

// ------------------------------------------------------------- V_MIDDLE

// WPO warps per output (the group of segred^0): 1 when the outputs fill the
// GPU, up to 8 (the whole CTA) when few outputs each reduce a long k.
template <typename Tin, bool VEC, int WPO>
__global__ void __launch_bounds__(256) mm_mid_kernel(const Tin* __restrict__ A, const Tin* __restrict__ Bt,
                                                     float* __restrict__ C, int64_t n, int64_t m, int64_t p) {
    constexpr int E = VecE<Tin>::E, G = 32 * WPO;
    __shared__ float red[8];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int gl = (w % WPO) * 32 + lane;  // lane within the group
    const int64_t o = (int64_t)blockIdx.x * (8 / WPO) + w / WPO;
    const bool live = o < n * p;
    float acc[4] = {0.f, 0.f, 0.f, 0.f};
    if (live) {
        const int64_t i = o / p, j = o - i * p;
        const Tin* a = A + i * m;
        const Tin* b = Bt + j * m;
        if (VEC) {
            int64_t k = (int64_t)gl * E;
            for (; k + E + G * E <= m; k += 2 * G * E) {
                float x0[E], y0[E], x1[E], y1[E];
                load16(a + k, x0);
                load16(b + k, y0);
                load16(a + k + G * E, x1);
                load16(b + k + G * E, y1);
#pragma unroll
                for (int e = 0; e < E; ++e) {
                    acc[e & 3] = fmaf(x0[e], y0[e], acc[e & 3]);
                    acc[(e + 2) & 3] = fmaf(x1[e], y1[e], acc[(e + 2) & 3]);
                }
            }
            for (; k + E <= m; k += G * E) {
                float x0[E], y0[E];
                load16(a + k, x0);
                load16(b + k, y0);
#pragma unroll
                for (int e = 0; e < E; ++e) acc[e & 3] = fmaf(x0[e], y0[e], acc[e & 3]);
            }
            for (int64_t kk = m - (m % E) + gl; kk < m; kk += G) acc[0] = fmaf(to_f(a[kk]), to_f(b[kk]), acc[0]);
        } else {
            for (int64_t kk = gl; kk < m; kk += G) acc[kk & 3] = fmaf(to_f(a[kk]), to_f(b[kk]), acc[kk & 3]);
        }
    }
    float s = (acc[0] + acc[1]) + (acc[2] + acc[3]);
    s = warp_reduce<OP_SUM>(s);
    if constexpr (WPO == 1) {
        if (lane == 0 && live) C[o] = s;
    } else {
        if (lane == 0) red[w] = s;
        __syncthreads();
        if (live && w % WPO == 0 && lane == 0) {
            float r = 0.f;
#pragma unroll
            for (int q = 0; q < WPO; ++q) r += red[w + q];
            C[o] = r;
        }
    }
}

// -------------------------------------------------------- tiled SIMT kernel
// A BM x BN output tile per CTA of 256 threads (16 x 16), TM x TN = BM/16 x
// BN/16 outputs per thread in registers (register tiling), BK-deep k-tiles of
// A and Bt staged in double-buffered shared memory (block tiling), the next
// k-tile prefetched into registers while the current one is multiplied.
// blockIdx.z = k-split: k-tiles [z*kps, (z+1)*kps); partial tiles go to
// part[z] when gridDim.z > 1 (V_FLAT's split-K), else straight to C.
// BKM = false: B is yss itself, [m][p] (row-major, P:122 before the
// transpose): its k-tile rows are read along p (coalesced, 16-byte vectors
// when bvec) straight into the k-major shared tile -- no transposition pass.
template <typename Tin, int BM, int BN, int BK, bool VEC, bool BKM>
__global__ void __launch_bounds__(256) mm_tile_simt_kernel(const Tin* __restrict__ A, const Tin* __restrict__ Bt,
                                                           float* __restrict__ C, float* __restrict__ part, int64_t n,
                                                           int64_t m, int64_t p, int64_t kps, bool bvec) {
    constexpr int TM = BM / 16, TN = BN / 16;
    constexpr int EPT = BM * BK / 256;  // k-values each thread stages per tile (BM == BN)
    static_assert(BM == BN && EPT >= 1 && BK % EPT == 0, "tile config");
    constexpr int TPR = BK / EPT;  // threads per staged row
    __shared__ __align__(16) float As[2][BK][BM + 4];
    __shared__ __align__(16) float Bs[2][BK][BN + 4];
    const int tid = threadIdx.x, tx = tid & 15, ty = tid >> 4;
    const int64_t row0 = (int64_t)blockIdx.y * BM, col0 = (int64_t)blockIdx.x * BN;
    const int lr = tid / TPR, lk = (tid % TPR) * EPT;
    float ra[EPT], rb[EPT];
    const bool arow = row0 + lr < n, brow = BKM && col0 + lr < p;
    const Tin* ap = A + (arow ? (row0 + lr) * m : 0);
    const Tin* bp = Bt + (brow ? (col0 + lr) * m : 0);
    // row-major B: thread stages EPT consecutive columns of k-row bk
    const int bk = tid / (BN / EPT), bc = (tid % (BN / EPT)) * EPT;
    const int64_t nk_all = ceil_div(m, BK);
    const int64_t kt_begin = (int64_t)blockIdx.z * kps;
    const int64_t kt_end = std::min(nk_all, kt_begin + kps);
    float* out = gridDim.z == 1 ? C : part + (int64_t)blockIdx.z * n * p;
    auto gload = [&](int64_t k0) {
        const int64_t kb = k0 + lk;
        constexpr int E = VecE<Tin>::E;
        if constexpr (!BKM) {
            const int64_t kr = k0 + bk, c = col0 + bc;
            if ((EPT % E == 0) && bvec && kr < m && c + EPT <= p) {
#pragma unroll
                for (int h = 0; h < EPT / E; ++h) {
                    float y[E];
                    load16(Bt + kr * p + c + h * E, y);
#pragma unroll
                    for (int e = 0; e < E; ++e) rb[h * E + e] = y[e];
                }
            } else {
#pragma unroll
                for (int e = 0; e < EPT; ++e) rb[e] = (kr < m && c + e < p) ? to_f(Bt[kr * p + c + e]) : 0.f;
            }
        }
        if (VEC && (EPT % E == 0) && kb + EPT <= m) {
#pragma unroll
            for (int h = 0; h < EPT / E; ++h) {
                float x[E], y[E];
                if (arow) load16(ap + kb + h * E, x);
                else
#pragma unroll
                    for (int e = 0; e < E; ++e) x[e] = 0.f;
                if constexpr (BKM) {
                    if (brow) load16(bp + kb + h * E, y);
                    else
#pragma unroll
                        for (int e = 0; e < E; ++e) y[e] = 0.f;
                }
#pragma unroll
                for (int e = 0; e < E; ++e) {
                    ra[h * E + e] = x[e];
                    if constexpr (BKM) rb[h * E + e] = y[e];
                }
            }
        } else {
#pragma unroll
            for (int e = 0; e < EPT; ++e) {
                const int64_t k = kb + e;
                ra[e] = (arow && k < m) ? to_f(ap[k]) : 0.f;
                if constexpr (BKM) rb[e] = (brow && k < m) ? to_f(bp[k]) : 0.f;
            }
        }
    };
    auto sstore = [&](int buf) {
#pragma unroll
        for (int e = 0; e < EPT; ++e) {
            As[buf][lk + e][lr] = ra[e];
            if constexpr (BKM) Bs[buf][lk + e][lr] = rb[e];
            else Bs[buf][bk][bc + e] = rb[e];
        }
    };
    float acc[TM][TN];
#pragma unroll
    for (int i = 0; i < TM; ++i)
#pragma unroll
        for (int j = 0; j < TN; ++j) acc[i][j] = 0.f;
    if (kt_begin < kt_end) {
        gload(kt_begin * BK);
        sstore(0);
    }
    __syncthreads();
    for (int64_t kt = kt_begin; kt < kt_end; ++kt) {
        const int cur = (int)((kt - kt_begin) & 1);
        if (kt + 1 < kt_end) gload((kt + 1) * BK);
#pragma unroll
        for (int k = 0; k < BK; ++k) {
            // each thread's rows/cols are two halves {t*TM/2 ..} and {BM/2 + t*TM/2 ..}
            float a[TM], b[TN];
            if constexpr (TM == 1) {
                a[0] = As[cur][k][ty];
                b[0] = Bs[cur][k][tx];
            } else {
#pragma unroll
                for (int i = 0; i < TM / 2; ++i) {
                    a[i] = As[cur][k][ty * (TM / 2) + i];
                    a[TM / 2 + i] = As[cur][k][BM / 2 + ty * (TM / 2) + i];
                }
#pragma unroll
                for (int j = 0; j < TN / 2; ++j) {
                    b[j] = Bs[cur][k][tx * (TN / 2) + j];
                    b[TN / 2 + j] = Bs[cur][k][BN / 2 + tx * (TN / 2) + j];
                }
            }
#pragma unroll
            for (int i = 0; i < TM; ++i)
#pragma unroll
                for (int j = 0; j < TN; ++j) acc[i][j] = fmaf(a[i], b[j], acc[i][j]);
        }
        if (kt + 1 < kt_end) sstore(cur ^ 1);
        __syncthreads();
    }
#pragma unroll
    for (int i = 0; i < TM; ++i) {
        const int64_t r = row0 + (TM == 1 ? ty : (i < TM / 2 ? ty * (TM / 2) + i : BM / 2 + ty * (TM / 2) + i - TM / 2));
        if (r >= n) continue;
#pragma unroll
        for (int j = 0; j < TN; ++j) {
            const int64_t c =
                col0 + (TN == 1 ? tx : (j < TN / 2 ? tx * (TN / 2) + j : BN / 2 + tx * (TN / 2) + j - TN / 2));
            if (c < p) out[r * p + c] = acc[i][j];
        }
    }
}

// -------------------------------------------------------------------- launch

// tcgen05 bf16 kernel and the split-K finalize (redomap2_tc.cu)
__global__ void mm_splitk_finalize(const float* __restrict__ part, float* __restrict__ C, int64_t outs, int splits);
bool tc_shape_ok(int64_t n, int64_t m, int64_t p, const void* A, const void* Bt);
int tc_splits(int64_t n, int64_t m, int64_t p, bool flat);
bool tc_mn_ok(int64_t n, int64_t m, int64_t p, const void* A, const void* B);
cudaError_t launch_mm_top_tc(const void* A, const void* Bt, float* C, float* part, int64_t n, int64_t m, int64_t p,
                             int splits, cudaStream_t s, bool b_mn = false);

static size_t align256(size_t b) { return (b + 255) & ~(size_t)255; }

// V_FLAT's register-blocked split-K engine for skinny outputs (n*p <= 4096,
// the degenerate end of the Fig 2 family): grid = (k-chunks,
// RI x RJ output tiles).  Each thread walks its k positions of the chunk in
// 8-byte vectors of the RI rows of A and of B (B^T rows, or for B given as
// yss [m][p] the RJ-wide slices of yss's rows -- no transposition pass),
// staged through an S-deep cp.async pipeline in THREAD-PRIVATE shared-memory
// slots (each thread consumes only its own copies: no CTA barrier in the
// loop, and S-1 stages of loads in flight without holding registers), and
// accumulates the RI x RJ partial dot products in registers (bf16 widened to
// f32 exactly).  Every element of A and B is read from DRAM once per output
// tile row / column; the CTA reduces its partials (shuffles + smem) into one
// partial tile, and mm_splitk_finalize sums the chunks in a fixed order.
constexpr int kSkinnyThreads = 256;
constexpr int kSkinnyStageBytes = 128 * 1024;  // pipeline depth: as many stages as fit 128 KB (3..12)
constexpr int64_t kSkinnyMaxOuts = 4096;
constexpr size_t kSkinnyCntBytes = kMmCntBytes;  // one arrival counter per output tile
static_assert(kMmCntBytes >= (size_t)kSkinnyMaxOuts * 4, "counter region");

__device__ __forceinline__ void cp_async8(void* smem, const void* gmem) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(smem_u32(smem)), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cp_async4(void* smem, const void* gmem) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_u32(smem)), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

// 8 bytes of Tin -> E floats
template <typename Tin>
__device__ __forceinline__ void unpack8(uint2 u, float (&o)[8 / sizeof(Tin)]) {
    if constexpr (std::is_same<Tin, float>::value) {
        o[0] = __uint_as_float(u.x);
        o[1] = __uint_as_float(u.y);
    } else {
        o[0] = __uint_as_float(u.x << 16);
        o[1] = __uint_as_float(u.x & 0xffff0000u);
        o[2] = __uint_as_float(u.y << 16);
        o[3] = __uint_as_float(u.y & 0xffff0000u);
    }
}

// Shared-memory words per thread per stage: RI A vectors + the B data of one
// k-vector (KMAJ: RJ vectors; row-major: E slices of RJ elements, in units
// of min(8, RJ * sizeof) bytes).
template <typename Tin, int RI, int RJ, bool KMAJ>
struct SkinnyGeom {
    static constexpr int E = 8 / (int)sizeof(Tin);
    static constexpr int SLICE = RJ * (int)sizeof(Tin);        // bytes of one row-major B slice
    static constexpr int UNIT = SLICE >= 8 ? 8 : 4;            // cp.async size (row-major needs SLICE >= 4)
    static constexpr int BU = KMAJ ? RJ : E * (SLICE / UNIT);  // B copies per k-vector
    static constexpr int BWORDS = KMAJ ? RJ : E * ((SLICE + 7) / 8);  // 8-byte smem words of B
    static constexpr int WORDS = RI + BWORDS;
    static constexpr int S0 = kSkinnyStageBytes / (WORDS * kSkinnyThreads * 8);
    static constexpr int S = S0 < 3 ? 3 : S0 > 12 ? 12 : S0;  // cp.async stages
    static constexpr size_t SMEM = (size_t)S * WORDS * kSkinnyThreads * 8;
};

// The end of a skinny CTA: its RI x RJ dot products (thread t < RI*RJ holds
// output t).  Without k-splits they go to C; otherwise to the partial tiles,
// and the last CTA of the output tile to arrive (a counter per tile) sums the
// splits' partials in split order into C -- the order of mm_splitk_finalize,
// so the result is deterministic -- and re-arms the counter: V_FLAT's skinny
// engine is one kernel.
template <int RI, int RJ>
__device__ __forceinline__ void skinny_store(float v, float* __restrict__ part, float* __restrict__ C,
                                             unsigned* __restrict__ cnt, int64_t n, int64_t p, int64_t i0,
                                             int64_t j0, int tile, float* red) {
    __shared__ unsigned s_last;
    const int t = threadIdx.x;
    const int splits = (int)gridDim.x;
    const int64_t i = i0 + t / RJ, j = j0 + t % RJ;
    const bool own = t < RI * RJ && i < n && j < p;
    if (splits == 1) {
        if (own) C[i * p + j] = v;
        return;
    }
    if (own) part[(int64_t)blockIdx.x * n * p + i * p + j] = v;
    __threadfence();
    __syncthreads();
    if (t == 0) s_last = atomicAdd(cnt + tile, 1u) == (unsigned)(splits - 1) ? 1u : 0u;
    __syncthreads();
    if (!s_last) return;
    __threadfence();
    // every thread sums a fixed contiguous block of the splits of one output,
    // the blocks are added in block order: a fixed association whatever the
    // arrival order (deterministic), with the CTA's loads in flight together
    constexpr int NO = RI * RJ, TPO = kSkinnyThreads / NO;
    const int o = t % NO, g = t / NO;
    const int64_t io = i0 + o / RJ, jo = j0 + o % RJ;
    const int chunk = (splits + TPO - 1) / TPO, q0 = g * chunk, q1 = min(splits, q0 + chunk);
    float r = 0.f;
    if (io < n && jo < p)
        for (int q = q0; q < q1; ++q) r += __ldcg(part + (int64_t)q * n * p + io * p + jo);
    red[g * NO + o] = r;
    __syncthreads();
    if (own) {
        float sum = 0.f;
        for (int q = 0; q < TPO; ++q) sum += red[q * NO + t];
        C[i * p + j] = sum;
    }
    if (t == 0) cnt[tile] = 0u;
}

template <typename Tin, int RI, int RJ, bool KMAJ, bool CP>
__global__ void __launch_bounds__(kSkinnyThreads) mm_skinny_kernel(const Tin* __restrict__ A, const Tin* __restrict__ B,
                                                                   float* __restrict__ part, float* __restrict__ C,
                                                                   unsigned* __restrict__ cnt, int64_t n, int64_t m,
                                                                   int64_t p, int64_t kchunk, int tiles_j) {
    using Gm = SkinnyGeom<Tin, RI, RJ, KMAJ>;
    constexpr int E = Gm::E, NW = kSkinnyThreads / 32, S = Gm::S;
    extern __shared__ __align__(16) uint2 sbuf[];  // [S][WORDS][threads]
    constexpr int NRED = NW * RI * RJ > kSkinnyThreads ? NW * RI * RJ : kSkinnyThreads;
    __shared__ float red[NRED];  // [NW][RI * RJ] per-warp sums, then the finalize's [TPO][RI * RJ]
    const int t = threadIdx.x, lane = t & 31, w = t >> 5;
    const int tile = blockIdx.y;
    const int64_t i0 = (int64_t)(tile / tiles_j) * RI, j0 = (int64_t)(tile % tiles_j) * RJ;
    const int64_t k0 = (int64_t)blockIdx.x * kchunk, k1 = std::min(m, k0 + kchunk);
    const int64_t stride = (int64_t)kSkinnyThreads * E;
    const int nit = (int)ceil_div(std::max<int64_t>(0, k1 - k0), stride);
    const Tin* ar[RI];
#pragma unroll
    for (int r = 0; r < RI; ++r) ar[r] = A + std::min(i0 + r, n - 1) * m;  // rows past n: clamped, dropped at the end
    const Tin* br[RJ];
#pragma unroll
    for (int c = 0; c < RJ; ++c) br[c] = B + std::min(j0 + c, p - 1) * m;  // KMAJ rows of B^T
    auto slot = [&](int st, int word) -> uint2* { return sbuf + ((size_t)st * Gm::WORDS + word) * kSkinnyThreads + t; };
    // row-major B with slices of >= 16 bytes (COOP): the warp copies its
    // 32*E k-rows' slices lane-contiguously (coalesced 8-byte pieces) into
    // the owners' slots; B word idx of thread t lives at slot t ^ swz(idx)
    // so that both the copies and the owners' reads are bank-conflict-free
    constexpr int UPR = Gm::SLICE >= 8 ? Gm::SLICE / 8 : 1, KW = E * UPR;
    constexpr int KWS = KW <= 16 ? KW : 16;  // (a divisor of 16 whenever COOP)
    constexpr bool COOP = CP && !KMAJ && Gm::SLICE >= 16 && Gm::UNIT == 8 && KW <= 16 && (16 % KWS) == 0;
    auto swz = [](int idx) { return COOP ? (idx * (16 / KWS)) & 15 : 0; };
    auto bslot = [&](int st, int idx, int owner) -> uint2* {
        return sbuf + ((size_t)st * Gm::WORDS + RI + idx) * kSkinnyThreads + (owner ^ swz(idx));
    };
    auto issue = [&](int it) {
        const int64_t k = k0 + (int64_t)it * stride + (int64_t)t * E;
        const int st = it % S;
        if constexpr (COOP) {
            const int64_t kw = k0 + (int64_t)it * stride + (int64_t)(t & ~31) * E;
            if (it < nit) {
#pragma unroll
                for (int r = 0; r < KW; ++r) {
                    const int q = lane + 32 * r, row = q / UPR, u = q % UPR;
                    if (kw + row < k1)
                        cp_async8(bslot(st, (row % E) * UPR + u, (t & ~31) + row / E),
                                  reinterpret_cast<const char*>(B + (kw + row) * p + j0) + u * 8);
                }
            }
        }
        if (it < nit && k < k1) {
#pragma unroll
            for (int r = 0; r < RI; ++r) cp_async8(slot(st, r), ar[r] + k);
            if constexpr (KMAJ) {
#pragma unroll
                for (int c = 0; c < RJ; ++c) cp_async8(slot(st, RI + c), br[c] + k);
            } else if constexpr (!COOP) {
#pragma unroll
                for (int e = 0; e < E; ++e) {
                    const char* src = reinterpret_cast<const char*>(B + (k + e) * p + j0);
                    char* dst = reinterpret_cast<char*>(slot(st, RI + e * ((Gm::SLICE + 7) / 8)));
#pragma unroll
                    for (int u = 0; u < Gm::SLICE / Gm::UNIT; ++u) {
                        // consecutive 8-byte words of a slice are kSkinnyThreads words apart
                        char* d = dst + (size_t)((u * Gm::UNIT) / 8) * kSkinnyThreads * 8 + (u * Gm::UNIT) % 8;
                        if constexpr (Gm::UNIT == 8) cp_async8(d, src + u * 8);
                        else cp_async4(d, src + u * 4);
                    }
                }
            }
        }
        cp_async_commit();  // (possibly empty) group per iteration keeps the wait count uniform
    };
    float acc[RI][RJ];
#pragma unroll
    for (int r = 0; r < RI; ++r)
#pragma unroll
        for (int c = 0; c < RJ; ++c) acc[r][c] = 0.f;
#pragma unroll
    for (int s = 0; s < S - 1; ++s) issue(s);
    for (int it = 0; it < nit; ++it) {
        if constexpr (COOP) __syncwarp();  // the warp is done with the stage it refills now
        issue(it + S - 1);
        cp_async_wait<S - 1>();  // this thread's copies of iteration it have landed
        if constexpr (COOP) __syncwarp();  // ... and those of the other lanes
        const int64_t k = k0 + (int64_t)it * stride + (int64_t)t * E;
        if (k >= k1) continue;
        const int st = it % S;
        float a[RI][E], b[RJ][E];
#pragma unroll
        for (int r = 0; r < RI; ++r) unpack8<Tin>(*slot(st, r), a[r]);
        if constexpr (COOP) {
#pragma unroll
            for (int e = 0; e < E; ++e)
#pragma unroll
                for (int c = 0; c < RJ; ++c) {
                    const int byte = c * (int)sizeof(Tin);
                    const uint2 wd = *bslot(st, e * UPR + byte / 8, t);
                    const uint32_t h = (byte % 8) < 4 ? wd.x : wd.y;
                    if constexpr (std::is_same<Tin, float>::value) b[c][e] = __uint_as_float(h);
                    else b[c][e] = __uint_as_float((byte % 4) == 0 ? (h << 16) : (h & 0xffff0000u));
                }
        } else if constexpr (KMAJ) {
#pragma unroll
            for (int c = 0; c < RJ; ++c) unpack8<Tin>(*slot(st, RI + c), b[c]);
        } else {
#pragma unroll
            for (int e = 0; e < E; ++e) {
                const uint2* q = slot(st, RI + e * ((Gm::SLICE + 7) / 8));
#pragma unroll
                for (int c = 0; c < RJ; ++c) {
                    const int byte = c * (int)sizeof(Tin);
                    const uint2 wd = q[(size_t)(byte / 8) * kSkinnyThreads];
                    const uint32_t h = (byte % 8) < 4 ? wd.x : wd.y;
                    if constexpr (std::is_same<Tin, float>::value) b[c][e] = __uint_as_float(h);
                    else b[c][e] = __uint_as_float((byte % 4) == 0 ? (h << 16) : (h & 0xffff0000u));
                }
            }
        }
#pragma unroll
        for (int e = 0; e < E; ++e)
#pragma unroll
            for (int r = 0; r < RI; ++r)
#pragma unroll
                for (int c = 0; c < RJ; ++c) acc[r][c] = fmaf(a[r][e], b[c][e], acc[r][c]);
    }
    cp_async_wait<0>();
#pragma unroll
    for (int r = 0; r < RI; ++r)
#pragma unroll
        for (int c = 0; c < RJ; ++c) {
            const float v = warp_reduce<OP_SUM>(acc[r][c]);
            if (lane == 0) red[w * RI * RJ + r * RJ + c] = v;
        }
    __syncthreads();
    float s = 0.f;
    if (t < RI * RJ)
#pragma unroll
        for (int q = 0; q < NW; ++q) s += red[q * RI * RJ + t];
    __syncthreads();  // red is reused by the finalize
    skinny_store<RI, RJ>(s, part, C, cnt, n, p, i0, j0, tile, red);
}

// Scalar form (misaligned operands or m not a multiple of the vector width).
template <typename Tin, int RI, int RJ, bool KMAJ>
__global__ void __launch_bounds__(kSkinnyThreads) mm_skinny_scalar_kernel(const Tin* __restrict__ A,
                                                                          const Tin* __restrict__ B,
                                                                          float* __restrict__ part,
                                                                          float* __restrict__ C,
                                                                          unsigned* __restrict__ cnt, int64_t n,
                                                                          int64_t m, int64_t p, int64_t kchunk,
                                                                          int tiles_j) {
    constexpr int NW = kSkinnyThreads / 32;
    constexpr int NRED = NW * RI * RJ > kSkinnyThreads ? NW * RI * RJ : kSkinnyThreads;
    __shared__ float red[NRED];  // [NW][RI * RJ] per-warp sums, then the finalize's [TPO][RI * RJ]
    const int t = threadIdx.x, lane = t & 31, w = t >> 5;
    const int tile = blockIdx.y;
    const int64_t i0 = (int64_t)(tile / tiles_j) * RI, j0 = (int64_t)(tile % tiles_j) * RJ;
    const int64_t k0 = (int64_t)blockIdx.x * kchunk, k1 = std::min(m, k0 + kchunk);
    float acc[RI][RJ];
#pragma unroll
    for (int r = 0; r < RI; ++r)
#pragma unroll
        for (int c = 0; c < RJ; ++c) acc[r][c] = 0.f;
    for (int64_t k = k0 + t; k < k1; k += kSkinnyThreads) {
        float a[RI], b[RJ];
#pragma unroll
        for (int r = 0; r < RI; ++r) a[r] = to_f(__ldg(A + std::min(i0 + r, n - 1) * m + k));
#pragma unroll
        for (int c = 0; c < RJ; ++c) {
            const int64_t j = std::min(j0 + c, p - 1);
            b[c] = to_f(KMAJ ? __ldg(B + j * m + k) : __ldg(B + k * p + j));
        }
#pragma unroll
        for (int r = 0; r < RI; ++r)
#pragma unroll
            for (int c = 0; c < RJ; ++c) acc[r][c] = fmaf(a[r], b[c], acc[r][c]);
    }
#pragma unroll
    for (int r = 0; r < RI; ++r)
#pragma unroll
        for (int c = 0; c < RJ; ++c) {
            const float v = warp_reduce<OP_SUM>(acc[r][c]);
            if (lane == 0) red[w * RI * RJ + r * RJ + c] = v;
        }
    __syncthreads();
    float s = 0.f;
    if (t < RI * RJ)
#pragma unroll
        for (int q = 0; q < NW; ++q) s += red[q * RI * RJ + t];
    __syncthreads();  // red is reused by the finalize
    skinny_store<RI, RJ>(s, part, C, cnt, n, p, i0, j0, tile, red);
}

// Where the engine is V_FLAT's form: f32 up to 4096 outputs; bf16 up to 256
// (beyond, the tcgen05 split-K tiles win: B200, k = 30 family, n = p = 32 / 64:
// 63 / 32 us vs 96 / 104 us for this FMA-bound engine)
static bool skinny_ok(int64_t n, int64_t p, bool bf16) { return n * p <= (bf16 ? 256 : kSkinnyMaxOuts); }
static int skinny_r(int64_t x) { return x >= 8 ? 8 : x >= 4 ? 4 : x >= 2 ? 2 : 1; }
// k-chunks: one wave of CTAs over all output tiles (as many per SM as the
// pipeline's shared memory allows), >= 1 vector round per chunk
static int64_t skinny_kchunk(int64_t n, int64_t m, int64_t p) {
    const int64_t tiles = ceil_div(n, skinny_r(n)) * ceil_div(p, skinny_r(p));
    // CTAs per SM the pipeline's shared memory allows (K-major words; >= 1, <= 4)
    const int words = skinny_r(n) + skinny_r(p);
    const int S = std::min(12, std::max(3, kSkinnyStageBytes / (words * kSkinnyThreads * 8)));
    const int occ = std::min(4, std::max(1, (200 * 1024) / (S * words * kSkinnyThreads * 8)));
    const int64_t want = std::max<int64_t>(1, (int64_t)148 * occ / tiles);
    int64_t kc = std::max<int64_t>((int64_t)kSkinnyThreads * 2, ceil_div(m, want));  // >= one 8-byte vector per thread
    return ceil_div(kc, 8) * 8;  // a multiple of every vector width
}
static int64_t skinny_splits(int64_t n, int64_t m, int64_t p) { return ceil_div(m, skinny_kchunk(n, m, p)); }

template <typename Tin, int RI, int RJ, bool KMAJ>
static cudaError_t launch_skinny_k(const Tin* A, const Tin* B, float* part, float* C, unsigned* cnt, int64_t n,
                                   int64_t m, int64_t p, int64_t kc, int64_t splits, int tj, int64_t tiles,
                                   cudaStream_t s) {
    using Gm = SkinnyGeom<Tin, RI, RJ, KMAJ>;
    constexpr int E = Gm::E;
    // cp.async needs 8-byte aligned rows (KMAJ) / UNIT-aligned B slices (row-major)
    bool vec = ((uintptr_t)A % 8 == 0) && (m % E == 0);
    if (KMAJ) vec = vec && ((uintptr_t)B % 8 == 0);
    else vec = vec && Gm::SLICE >= 4 && ((uintptr_t)B % Gm::UNIT == 0) && ((p * (int64_t)sizeof(Tin)) % Gm::UNIT == 0) &&
               (p % RJ == 0);
    dim3 g((unsigned)splits, (unsigned)tiles);
    if (vec) {
        const size_t smem = Gm::SMEM;
        // row-major B spread over several column tiles (p > RJ): slices are
        // strided within the rows, copied warp-cooperatively (measured on B200:
        // k = 25 f32 n = p = 16..64 1.44-1.56x -> 1.10-1.17x the k-major time;
        // with one column tile a thread's own rows are contiguous already)
        auto k = p > RJ ? mm_skinny_kernel<Tin, RI, RJ, KMAJ, true> : mm_skinny_kernel<Tin, RI, RJ, KMAJ, false>;
        static bool attr = false;
        if (!attr) {
            cudaFuncSetAttribute(mm_skinny_kernel<Tin, RI, RJ, KMAJ, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 (int)smem);
            cudaFuncSetAttribute(mm_skinny_kernel<Tin, RI, RJ, KMAJ, false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 (int)smem);
            attr = true;
        }
        k<<<g, kSkinnyThreads, smem, s>>>(A, B, part, C, cnt, n, m, p, kc, tj);
    } else {
        mm_skinny_scalar_kernel<Tin, RI, RJ, KMAJ><<<g, kSkinnyThreads, 0, s>>>(A, B, part, C, cnt, n, m, p, kc, tj);
    }
    return cudaGetLastError();
}

template <typename Tin, int RI, int RJ>
static cudaError_t launch_skinny_rr(const Tin* A, const Tin* B, float* C, float* part, unsigned* cnt, int64_t n,
                                    int64_t m, int64_t p, bool kmajor, cudaStream_t s) {
    const int64_t kc = skinny_kchunk(n, m, p), splits = ceil_div(m, kc);
    const int tj = (int)ceil_div(p, RJ);
    const int64_t tiles = ceil_div(n, RI) * tj;
    return kmajor ? launch_skinny_k<Tin, RI, RJ, true>(A, B, part, C, cnt, n, m, p, kc, splits, tj, tiles, s)
                  : launch_skinny_k<Tin, RI, RJ, false>(A, B, part, C, cnt, n, m, p, kc, splits, tj, tiles, s);
}

template <typename Tin, int RI>
static cudaError_t launch_skinny_r(const Tin* A, const Tin* B, float* C, float* part, unsigned* cnt, int64_t n,
                                   int64_t m, int64_t p, bool kmajor, cudaStream_t s) {
    switch (skinny_r(p)) {
    case 8: return launch_skinny_rr<Tin, RI, 8>(A, B, C, part, cnt, n, m, p, kmajor, s);
    case 4: return launch_skinny_rr<Tin, RI, 4>(A, B, C, part, cnt, n, m, p, kmajor, s);
    case 2: return launch_skinny_rr<Tin, RI, 2>(A, B, C, part, cnt, n, m, p, kmajor, s);
    default: return launch_skinny_rr<Tin, RI, 1>(A, B, C, part, cnt, n, m, p, kmajor, s);
    }
}

template <typename Tin>
static cudaError_t launch_skinny(const Tin* A, const Tin* B, float* C, float* part, unsigned* cnt, int64_t n,
                                 int64_t m, int64_t p, bool kmajor, cudaStream_t s) {
    switch (skinny_r(n)) {
    case 8: return launch_skinny_r<Tin, 8>(A, B, C, part, cnt, n, m, p, kmajor, s);
    case 4: return launch_skinny_r<Tin, 4>(A, B, C, part, cnt, n, m, p, kmajor, s);
    case 2: return launch_skinny_r<Tin, 2>(A, B, C, part, cnt, n, m, p, kmajor, s);
    default: return launch_skinny_r<Tin, 1>(A, B, C, part, cnt, n, m, p, kmajor, s);
    }
}


// V_FLAT's SIMT form beyond the skinny engine: 32x32 output tiles split along
// k until the GPU is full.
constexpr int kFlatTileBM = 32, kFlatTileBK = 32;
static int64_t simt_flat_splits(int64_t n, int64_t m, int64_t p) {
    const int64_t tiles = ceil_div(n, kFlatTileBM) * ceil_div(p, kFlatTileBM);
    const int64_t nk = ceil_div(m, kFlatTileBK);
    return std::max<int64_t>(1, std::min(ceil_div((int64_t)148 * 6, tiles), nk));
}

size_t redomap2_ws_bytes(int64_t n, int64_t m, int64_t p, int version) {
    // transposition buffer for b_kmajor = 0 (upper bound: 4-byte elements) +
    // split-K partials (V_FLAT always may split; V_TOP's tensor-core kernel
    // splits k to fill idle SMs)
    size_t b = align256((size_t)m * p * 4);
    size_t part = 0;
    if (version == 2 || version == -1) {
        if (skinny_ok(n, p, false))
            part = std::max(part, (size_t)n * p * skinny_splits(n, m, p) * 4);
        part = std::max(part, (size_t)n * p * simt_flat_splits(n, m, p) * 4);
        part = std::max(part, (size_t)n * p * tc_splits(n, m, p, true) * 4);
    }
    if (version == 0 || version == -1) {
        part = std::max(part, (size_t)n * p * tc_splits(n, m, p, false) * 4);
        {  // SIMT TOP with 32x32 tiles (small output grids)
            const int64_t t32 = ceil_div(n, 32) * ceil_div(p, 32), nk32 = ceil_div(m, 32);
            const int64_t s32 = std::max<int64_t>(1, std::min<int64_t>((int64_t)148 / std::max<int64_t>(t32, 1), nk32 / 8));
            part = std::max(part, (size_t)n * p * s32 * 4);
        }
        const int64_t tiles = ceil_div(n, 128) * ceil_div(p, 128), nk = ceil_div(m, 16);
        const int64_t s = std::max<int64_t>(1, std::min<int64_t>((int64_t)148 / tiles, nk / 64));
        part = std::max(part, (size_t)n * p * (size_t)ceil_div(nk, ceil_div(nk, s)) * 4);
    }
    return kSkinnyCntBytes + b + align256(part);
}

bool redomap2_tc_ok(const MmArgs& a) { return a.in_dt == 2 && tc_shape_ok(a.n, a.m, a.p, a.A, a.B); }

// the SIMT tile kernel for either B layout (bkm: yss^T [p][m]; else yss [m][p])
template <typename Tin, int BM, int BK>
static void simt_go(dim3 g, bool vec, bool bkm, bool bvec, const Tin* A, const Tin* B, float* C, float* part,
                    int64_t n, int64_t m, int64_t p, int64_t kps, cudaStream_t s) {
    if (bkm) {
        if (vec) mm_tile_simt_kernel<Tin, BM, BM, BK, true, true><<<g, 256, 0, s>>>(A, B, C, part, n, m, p, kps, bvec);
        else mm_tile_simt_kernel<Tin, BM, BM, BK, false, true><<<g, 256, 0, s>>>(A, B, C, part, n, m, p, kps, bvec);
    } else {
        if (vec) mm_tile_simt_kernel<Tin, BM, BM, BK, true, false><<<g, 256, 0, s>>>(A, B, C, part, n, m, p, kps, bvec);
        else mm_tile_simt_kernel<Tin, BM, BM, BK, false, false><<<g, 256, 0, s>>>(A, B, C, part, n, m, p, kps, bvec);
    }
}

template <typename Tin>
static cudaError_t run_mm(int version, const MmArgs& a) {
    const Tin* A = (const Tin*)a.A;
    const Tin* Bt = (const Tin*)a.B;
    // [V_FLAT skinny arrival counters][yss^T][split-K partial tiles]: the
    // counters (zero at rest) never share bytes with the other regions
    unsigned* cnt = (unsigned*)a.ws;
    char* ws = a.ws ? (char*)a.ws + kSkinnyCntBytes : nullptr;
    if (version == 2 && skinny_ok(a.n, a.p, std::is_same<Tin, __nv_bfloat16>::value) && a.m > 0)
        // V_FLAT, skinny outputs: either B layout, no transposition pass
        // (yss with a single column is the same memory as its transpose)
        return launch_skinny<Tin>(A, Bt, a.C, (float*)ws, cnt, a.n, a.m, a.p, a.b_kmajor != 0 || a.p == 1, a.stream);
    constexpr bool kBf16 = std::is_same<Tin, __nv_bfloat16>::value;
    // tensor cores (bf16), V_MIDDLE and the row-level leaves read yss^T; the
    // SIMT tile kernels of V_TOP / V_FLAT read either layout in place
    // (the tensor-core kernel reads yss in place too when its rows have a
    // 16-byte pitch: MN-major B operand)
    const bool tc_mn = kBf16 && !a.b_kmajor && (version == 0 || version == 2) && tc_mn_ok(a.n, a.m, a.p, A, a.B);
    const bool tc = kBf16 && (tc_mn || tc_shape_ok(a.n, a.m, a.p, A, a.b_kmajor ? a.B : (const void*)ws));
    const bool direct = !a.b_kmajor && (version == 0 || version == 2) && (!tc || tc_mn);
    size_t used = 0;
    if (!a.b_kmajor && !direct) {  // yss [m][p] -> yss^T [p][m]
        Tin* t = (Tin*)ws;
        used = align256((size_t)a.m * a.p * sizeof(Tin));
        if (a.m * a.p > 0) {
            dim3 g((unsigned)ceil_div(a.p, 32), (unsigned)ceil_div(a.m, 32));
            transpose_kernel<Tin><<<g, 256, 0, a.stream>>>((const Tin*)a.B, t, a.m, a.p);
            cudaError_t e = cudaGetLastError();
            if (e != cudaSuccess) return e;
        }
        Bt = t;
    }
    if (a.m == 0) return cudaMemsetAsync(a.C, 0, (size_t)a.n * a.p * sizeof(float), a.stream);
    if (version == IFL_V_ROW_TOP || version == IFL_V_ROW_MIDDLE)  // row-level leaves (mm_row.cu)
        return launch_mm_row(version, A, Bt, a.C, a.n, a.m, a.p, a.in_dt, a.stream);
    constexpr int E = VecE<Tin>::E;
    const bool bkm = !direct;
    const bool vec = ((uintptr_t)A % 16 == 0) && (!bkm || (uintptr_t)Bt % 16 == 0) && (a.m % E == 0);
    const bool bvec = !bkm && ((uintptr_t)Bt % 16 == 0) && (a.p % E == 0);
    const int64_t outs = a.n * a.p;
    float* part = (float*)(ws + used);
    if (version == 2) {  // ---- V_FLAT: every level parallel (split-K)
        // bf16: 128x256 tensor-core tiles split along k (even a mostly empty
        // tile beats SIMT here); f32: SIMT 32x32 (16x16 when skinny) tiles
        if (tc)
            return launch_mm_top_tc(A, Bt, a.C, part, a.n, a.m, a.p, tc_splits(a.n, a.m, a.p, true), a.stream, tc_mn);
        const int BM = std::max(a.n, a.p) <= 16 ? 16 : kFlatTileBM;
        const int64_t s = simt_flat_splits(a.n, a.m, a.p);
        const int64_t nk = ceil_div(a.m, kFlatTileBK), kps = ceil_div(nk, s), splits = ceil_div(nk, kps);
        dim3 g((unsigned)ceil_div(a.p, BM), (unsigned)ceil_div(a.n, BM), (unsigned)splits);
        if (BM == 16)
            simt_go<Tin, 16, kFlatTileBK * 2>(g, vec, bkm, bvec, A, Bt, a.C, part, a.n, a.m, a.p, ceil_div(kps, 2),
                                              a.stream);
        else
            simt_go<Tin, kFlatTileBM, kFlatTileBK>(g, vec, bkm, bvec, A, Bt, a.C, part, a.n, a.m, a.p, kps, a.stream);
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess || splits == 1) return e;
        mm_splitk_finalize<<<(unsigned)std::min<int64_t>(ceil_div(outs, 256), 148 * 16), 256, 0, a.stream>>>(
            part, a.C, outs, (int)splits);
        return cudaGetLastError();
    }
    if (version == 1) {  // ---- V_MIDDLE: a group of warps per output
        // group size: warps per output so that >= 148 x 32 warps run, each with
        // >= 4 vector rounds of k
        int wpo = 1;
        while (wpo < 8 && outs * wpo < (int64_t)148 * 32 && a.m >= (int64_t)wpo * 2 * 32 * E * 4) wpo *= 2;
        const int64_t grid = ceil_div(outs * wpo, 8);
        auto go = [&](auto wc) {
            constexpr int W = decltype(wc)::value;
            if (vec) mm_mid_kernel<Tin, true, W><<<(unsigned)grid, 256, 0, a.stream>>>(A, Bt, a.C, a.n, a.m, a.p);
            else mm_mid_kernel<Tin, false, W><<<(unsigned)grid, 256, 0, a.stream>>>(A, Bt, a.C, a.n, a.m, a.p);
        };
        switch (wpo) {
        case 8: go(std::integral_constant<int, 8>{}); break;
        case 4: go(std::integral_constant<int, 4>{}); break;
        case 2: go(std::integral_constant<int, 2>{}); break;
        default: go(std::integral_constant<int, 1>{}); break;
        }
        return cudaGetLastError();
    }
    // ---- V_TOP: output tiles, sequential k (tensor cores for bf16)
    if (tc) return launch_mm_top_tc(A, Bt, a.C, part, a.n, a.m, a.p, tc_splits(a.n, a.m, a.p, false), a.stream, tc_mn);
    // SIMT TOP: 128x128 tiles; when fewer than half the SMs would get one, the
    // 32x32 tiles (k in chunks of >= 8 x 32, each walked sequentially) -- B200:
    // n = p = 64..512 outputs from 105-60 us down to the 32x32 engine's 11-18 us
    if (ceil_div(a.n, 128) * ceil_div(a.p, 128) < 74) {
        const int64_t t32 = ceil_div(a.n, 32) * ceil_div(a.p, 32), nk32 = ceil_div(a.m, 32);
        const int64_t s32 = std::max<int64_t>(1, std::min<int64_t>((int64_t)148 / t32, nk32 / 8));
        const int64_t kps32 = ceil_div(nk32, s32), sp32 = ceil_div(nk32, kps32);
        dim3 g32((unsigned)ceil_div(a.p, 32), (unsigned)ceil_div(a.n, 32), (unsigned)sp32);
        simt_go<Tin, 32, 32>(g32, vec, bkm, bvec, A, Bt, a.C, part, a.n, a.m, a.p, kps32, a.stream);
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess || sp32 == 1) return e;
        mm_splitk_finalize<<<(unsigned)std::min<int64_t>(ceil_div(outs, 256), 148 * 16), 256, 0, a.stream>>>(
            part, a.C, outs, (int)sp32);
        return cudaGetLastError();
    }
    const int64_t tiles = ceil_div(a.n, 128) * ceil_div(a.p, 128), nk = ceil_div(a.m, 16);
    const int64_t s = std::max<int64_t>(1, std::min<int64_t>((int64_t)148 / tiles, nk / 64));
    const int64_t kps = ceil_div(nk, s), splits = ceil_div(nk, kps);
    dim3 g((unsigned)ceil_div(a.p, 128), (unsigned)ceil_div(a.n, 128), (unsigned)splits);
    simt_go<Tin, 128, 16>(g, vec, bkm, bvec, A, Bt, a.C, part, a.n, a.m, a.p, kps, a.stream);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess || splits == 1) return e;
    mm_splitk_finalize<<<(unsigned)std::min<int64_t>(ceil_div(outs, 256), 148 * 16), 256, 0, a.stream>>>(part, a.C, outs,
                                                                                                   (int)splits);
    return cudaGetLastError();
}

cudaError_t launch_redomap2(int version, const MmArgs& a) {
    if (a.in_dt == 1) return run_mm<float>(version, a);
    if (a.in_dt == 2) return run_mm<__nv_bfloat16>(version, a);
    return cudaErrorInvalidValue;
}

}  // namespace ifl
