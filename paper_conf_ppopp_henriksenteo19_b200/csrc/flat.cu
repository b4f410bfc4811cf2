// flat.cu -- V_FLAT: the fully flattened segred^1 / segscan^1 over all n*m
// elements (rule G3's e_flat; Fig 6c version 3).
//
// The flat index space [0, n*m) is cut into tiles of kFlatTile = 256 x 20
// elements.  Segment starts are arithmetic (multiples of m): no flag array is
// read, and d is combined into every segment's first element.  The kernels
// are persistent (grid = resident CTAs) and stream tiles through a ring of
// shared-memory slots filled by the TMA engine (cp.async.bulk + mbarrier), so
// loads for the next tiles are in flight while a tile is processed.  Per tile:
//   * thread t takes its 20 consecutive elements (5 conflict-free LDS.128: the
//     80-byte stride is an odd multiple of 16 B).  A thread whose items hold
//     no segment boundary (the common case once m exceeds a few dozen) takes a
//     branch-free fast path; otherwise a sequential segmented scan;
//   * the CTA scans the (flag, value) thread aggregates with the segmented
//     operator (f1,v1).(f2,v2) = (f1|f2, f2 ? v2 : v1 (+) v2).
// segred (two passes, no inter-CTA waiting):
//   pass 1  complete segments are written to out directly; each tile leaves
//           head[t] (partial of the segment it starts inside) and tail[t]
//           (the open segment at its end, or the whole tile) in the workspace;
//   pass 2  every segment that crosses tiles ta < tb is
//           out = tail[ta] (+) tail[ta+1..tb-1] (+) head[tb]   (a tree reduce).
//   Rows of >= 8192 elements: uniform row pieces (flat_red_split_kernel).
// segscan:
//   * tiles that all begin at a segment start (m divides the tile): the
//     single-pass engine (flat_scan_dlb_kernel), no inter-tile dependence;
//   * otherwise the job-ring engine (flat_scan_jr_kernel): reduce-then-scan
//     desynchronised into jobs -- job k aggregates chunk k from DRAM and scans
//     chunk k - lag from L2 -- so no look-back ever waits on a status written
//     moments ago (under a saturated memory system a status store and the
//     poll that sees it take microseconds: DESIGN.md section 5).
//   Status words carry an epoch tag; the last CTA re-arms the workspace
//   (counter reset, epoch bump), so no per-call memset is needed.
// Workspace: [header 256 B][status: 8 B/tile][head: 4 B/tile][tail: 4 B/tile].
#include <string.h>

#include <algorithm>
#include <unordered_map>

#include "common.cuh"
#include "dispatch.cuh"
#include "ifl_internal.h"

namespace ifl {

constexpr int FB = kFlatThreads;
constexpr int FI = kFlatItems;
constexpr int FT = (int)kFlatTile;
static_assert(FI % 4 == 0 && (FI / 4) % 2 == 1, "odd number of 16-byte chunks per thread");

struct FlatHdr {
    uint32_t epoch;
    uint32_t tile_ctr;
    uint32_t done_ctr;
    uint32_t pad[61];
};
static_assert(sizeof(FlatHdr) == 256, "header size");

size_t flat_ws_bytes(int64_t total) {
    const int64_t tiles = ceil_div(total, kFlatTile);
    return sizeof(FlatHdr) + (size_t)tiles * 16;
}

// status word: [63:35] tag, [34:33] status (1 aggregate, 2 inclusive), [32] flag, [31:0] value
constexpr uint64_t ST_A = 1, ST_P = 2;

// The tag of a call's status words: the 32-bit epoch of the workspace header
// scrambled by an odd multiplier (a bijection on 29 bits), so that small
// integers left in the status region by an earlier call of another entry
// point (segred partials, user data) do not look like valid words of a young
// workspace whose epoch is itself a small integer.
__device__ __forceinline__ uint32_t status_tag(uint64_t hdr_word) {
    const uint32_t epoch = (uint32_t)(hdr_word >> 32);
    return (epoch * 0x9E3779B1u + 0x6A09E667u) & 0x1FFFFFFFu;
}
__device__ __forceinline__ uint64_t pack_status(uint32_t tag, uint64_t st, uint32_t flag, uint32_t val) {
    return ((uint64_t)tag << 35) | (st << 33) | ((uint64_t)flag << 32) | (uint64_t)val;
}

// Per-slot tile metadata, written by the producer thread when it claims a tile.
struct SlotMeta {
    int tile;
    int cnt;
    int64_t pos;  // (tile*FT) % m
    int64_t seg;  // (tile*FT) / m
};

__device__ __forceinline__ void fill_meta(SlotMeta& sm, int tile, int64_t N, int64_t m) {
    const int64_t base = (int64_t)tile * FT;
    sm.tile = tile;
    sm.cnt = (int)std::min((int64_t)FT, N - base);
    sm.pos = base % m;
    sm.seg = base / m;
}

// Thread view of a tile: position of its first item inside its segment.
struct ThreadPos {
    int nvalid, nx0, mi;
    int64_t seg;  // segment of the thread's first item
};

__device__ __forceinline__ ThreadPos thread_pos(const SlotMeta& sm, int64_t m) {
    ThreadPos p;
    const int off = threadIdx.x * FI;
    p.nvalid = max(0, min(FI, sm.cnt - off));
    int64_t pos;
    if (m > FT) {  // at most one boundary inside the tile: no division
        pos = sm.pos + off;
        p.seg = sm.seg;
        if (pos >= m) {
            pos -= m;
            p.seg += 1;
        }
    } else {  // m fits 32 bits
        const uint32_t q = (uint32_t)sm.pos + (uint32_t)off, mm = (uint32_t)m;
        pos = q % mm;
        p.seg = sm.seg + q / mm;
    }
    p.mi = (int)std::min(m, (int64_t)FI + 1);
    p.nx0 = (int)std::min(pos == 0 ? (int64_t)0 : m - pos, (int64_t)FI + 1);
    return p;
}

template <typename T>
__device__ __forceinline__ void load_items(const T* buf, T (&v)[FI]) {
    using V = typename Vec4<T>::type;
    const int o = threadIdx.x * FI;
#pragma unroll
    for (int c = 0; c < FI / 4; ++c) {
        V q = *reinterpret_cast<const V*>(&buf[o + 4 * c]);
        v[4 * c] = q.x; v[4 * c + 1] = q.y; v[4 * c + 2] = q.z; v[4 * c + 3] = q.w;
    }
}

template <typename T>
__device__ __forceinline__ void store_items(T* buf, const T (&v)[FI]) {
    using V = typename Vec4<T>::type;
    const int o = threadIdx.x * FI;
#pragma unroll
    for (int c = 0; c < FI / 4; ++c) {
        V q;
        q.x = v[4 * c]; q.y = v[4 * c + 1]; q.z = v[4 * c + 2]; q.w = v[4 * c + 3];
        *reinterpret_cast<V*>(&buf[o + 4 * c]) = q;
    }
}

// CTA-wide exclusive scan of the thread aggregates (fl, sv) under the
// segmented operator.  Returns the thread's exclusive prefix (exf, exv) and
// the tile aggregate (aggf, aggv).  Contains one __syncthreads.
// barrier among the FB consumer threads only (named barrier 1): used by the
// warp-specialised scan kernel, whose producer warp must not take part
__device__ __forceinline__ void consumer_sync() { asm volatile("bar.sync 1, %0;" ::"n"(FB) : "memory"); }

template <typename T, int OP, bool NAMED = false>
__device__ __forceinline__ void cta_seg_scan(uint32_t fl, T sv, uint32_t& exf, T& exv, uint32_t& aggf, T& aggv,
                                             T* s_wval, uint32_t* s_wflag) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
        const T ov = __shfl_up_sync(0xffffffffu, sv, off);
        const uint32_t of = __shfl_up_sync(0xffffffffu, fl, off);
        if (lane >= off) {
            if (!fl) sv = combine<OP>(ov, sv);
            fl |= of;
        }
    }
    if (lane == 31) {
        s_wval[w] = sv;
        s_wflag[w] = fl;
    }
    exv = __shfl_up_sync(0xffffffffu, sv, 1);
    exf = __shfl_up_sync(0xffffffffu, fl, 1);
    if (lane == 0) {
        exv = identity<OP, T>();
        exf = 0;
    }
    if (NAMED) consumer_sync();
    else __syncthreads();
    T pw = identity<OP, T>();
    uint32_t pf = 0;
    aggv = identity<OP, T>();
    aggf = 0;
#pragma unroll
    for (int k = 0; k < FB / 32; ++k) {
        const T wv = s_wval[k];
        const uint32_t wf = s_wflag[k];
        if (k < w) {
            pw = wf ? wv : combine<OP>(pw, wv);
            pf |= wf;
        }
        aggv = wf ? wv : combine<OP>(aggv, wv);
        aggf |= wf;
    }
    if (!exf) exv = combine<OP>(pw, exv);
    exf |= pf;
}

// ------------------------------------------------------------ ring helpers

template <typename T>
__device__ __forceinline__ void issue_tile_load(T* slot, const T* in, int tile, uint64_t* bar) {
    mbar_arrive_expect_tx(bar, FT * sizeof(T));
    bulk_g2s(slot, in + (int64_t)tile * FT, FT * sizeof(T), bar);
}

// Make tile data available in `slot`: wait for its TMA load (full tiles with
// an aligned input) or copy it cooperatively.
template <typename T>
__device__ __forceinline__ void acquire_tile(T* slot, const T* in, const SlotMeta& sm, bool tma, uint64_t* bar,
                                             uint32_t& phase_bits, int s) {
    if (tma && sm.cnt == FT) {
        mbar_wait(bar, (phase_bits >> s) & 1u);
        phase_bits ^= 1u << s;
    } else {
        const int64_t base = (int64_t)sm.tile * FT;
        for (int p = threadIdx.x; p < sm.cnt; p += FB) slot[p] = in[base + p];
        __syncthreads();
    }
}

// ------------------------------------------------------------ segred pass 1

// Warp-specialised like the scan: warp 8 is the producer (static round-robin
// tiles blockIdx + i*grid; waits for a ring slot to be released, writes its
// metadata, issues the TMA load); warps 0-7 consume.  A slot is released by
// each consumer warp as soon as its items are in registers (count-8 mbarrier),
// so the next load into it is issued while the tile is still being reduced.
#ifndef IFL_RED_SLOTS  // experiment overrides (tools/flat_probe.py with IFL_BUILD_TAG builds)
#define IFL_RED_SLOTS 3
#endif
#ifndef IFL_RED_MINB
#define IFL_RED_MINB 3
#endif
constexpr int kRedSlots = IFL_RED_SLOTS;

template <typename T, int OP, int F>
__global__ void __launch_bounds__(FB + 32, IFL_RED_MINB) flat_red_kernel(const T* in, T* out, int64_t N, int64_t m, T d, T* head,
                                                              T* tail, int num_tiles, bool tma) {
    extern __shared__ __align__(128) uint8_t smem_raw[];
    T* ring = reinterpret_cast<T*>(smem_raw);
    __shared__ alignas(8) uint64_t full[kRedSlots], empty[kRedSlots];
    __shared__ SlotMeta meta[kRedSlots];
    __shared__ T s_wval[2][FB / 32];
    __shared__ uint32_t s_wflag[2][FB / 32];
    const int t = threadIdx.x, lane = t & 31, w = t >> 5;
    const int G = gridDim.x;
    if (t == 0) {
        for (int q = 0; q < kRedSlots; ++q) {
            mbar_init(&full[q], 1);
            mbar_init(&empty[q], FB / 32);
        }
        fence_mbar_init();
    }
    __syncthreads();
    if (w == FB / 32) {  // ================= producer warp
        if (lane == 0) {
            for (int wv = 0;; ++wv) {
                const int tile = blockIdx.x + wv * G;
                if (tile >= num_tiles) break;
                const int sl = wv % kRedSlots;
                if (wv >= kRedSlots) mbar_wait(&empty[sl], ((wv / kRedSlots) - 1) & 1);
                fill_meta(meta[sl], tile, N, m);
                if (tma && meta[sl].cnt == FT) {
                    mbar_arrive_expect_tx(&full[sl], FT * sizeof(T));
                    bulk_g2s(ring + sl * FT, in + (int64_t)tile * FT, FT * sizeof(T), &full[sl]);
                } else {
                    mbar_arrive_expect_tx(&full[sl], 0);
                }
            }
        }
        return;
    }
    // ================= consumer warps 0-7
    uint32_t phase_bits = 0;
    for (int i = 0;; ++i) {
        const int tile0 = blockIdx.x + i * G;
        if (tile0 >= num_tiles) break;
        const int sl = i % kRedSlots;
        T* buf = ring + sl * FT;
        mbar_wait(&full[sl], (phase_bits >> sl) & 1u);
        phase_bits ^= 1u << sl;
        const SlotMeta sm = meta[sl];
        if (!(tma && sm.cnt == FT)) {
            const int64_t base = (int64_t)sm.tile * FT;
            for (int p = t; p < sm.cnt; p += FB) buf[p] = in[base + p];
            consumer_sync();
        }
        const ThreadPos tp = thread_pos(sm, m);
        T v[FI];
        load_items(buf, v);
        __syncwarp();
        if (lane == 0) mbar_arrive_expect_tx(&empty[sl], 0);  // this warp is done with the slot
        bool has_start = false, stash = false;
        T acc, stash_v = identity<OP, T>();
        if (tp.nx0 > tp.nvalid) {
            // no boundary among this thread's items: plain reduction, 4 chains
            T a4[4] = {identity<OP, T>(), identity<OP, T>(), identity<OP, T>(), identity<OP, T>()};
#pragma unroll
            for (int k = 0; k < FI; ++k)
                if (k < tp.nvalid) a4[k & 3] = combine<OP>(a4[k & 3], apply_map<F>(v[k]));
            acc = combine<OP>(combine<OP>(a4[0], a4[1]), combine<OP>(a4[2], a4[3]));
        } else {
            acc = identity<OP, T>();
            int nx = tp.nx0;
            int64_t sg = tp.seg;
#pragma unroll
            for (int k = 0; k < FI; ++k) {
                if (k < tp.nvalid) {
                    const T x = apply_map<F>(v[k]);
                    if (k == nx) {
                        acc = combine<OP>(d, x);
                        has_start = true;
                        nx += tp.mi;
                    } else {
                        acc = combine<OP>(acc, x);
                    }
                    if (k + 1 == nx) {  // item k ends segment sg
                        if (k < tp.nx0) {
                            stash = true;
                            stash_v = acc;
                        } else {
                            out[sg] = acc;
                        }
                        ++sg;
                    }
                }
            }
        }
        uint32_t exf, aggf;
        T exv, aggv;
        // double-buffered warp totals: no extra barrier between tiles
        cta_seg_scan<T, OP, true>(has_start ? 1u : 0u, acc, exf, exv, aggf, aggv, s_wval[i & 1], s_wflag[i & 1]);
        if (stash) {
            const T val = combine<OP>(exv, stash_v);
            if (exf) out[tp.seg] = val;  // began earlier in this tile: complete
            else head[sm.tile] = val;    // began before this tile: head partial
        }
        if (t == 0) tail[sm.tile] = aggv;
    }
}

// Pass 2: finish every segment that crosses a tile boundary,
//   out = tail[ta] (+) tail[ta+1..tb-1] (+) head[tb],   ta < tb.
// m < FT: a crossing segment spans exactly two tiles; one thread per tile
// boundary b (it is crossed iff b*FT is not a segment start).
template <typename T, int OP>
__global__ void __launch_bounds__(256) flat_red_fix_short(T* out, int64_t m, const T* head, const T* tail,
                                                          int num_tiles) {
    for (int b = 1 + blockIdx.x * blockDim.x + threadIdx.x; b < num_tiles; b += gridDim.x * blockDim.x) {
        const uint32_t rem = (uint32_t)(((uint64_t)b * FT) % (uint64_t)m);
        if (rem == 0) continue;
        const int64_t seg = ((int64_t)b * FT) / m;
        out[seg] = combine<OP>(tail[b - 1], head[b]);
    }
}

// m >= FT: one CTA per segment; the middle range of whole-tile partials is
// reduced with independent loads (8 in flight per thread) and a CTA tree.
template <typename T, int OP>
__global__ void __launch_bounds__(512) flat_red_fix_long(T* out, int64_t n, int64_t m, const T* head, const T* tail) {
    __shared__ T red[16];
    for (int64_t sgi = blockIdx.x; sgi < n; sgi += gridDim.x) {
        const int ta = (int)((sgi * m) / FT);
        const int tb = (int)(((sgi + 1) * m - 1) / FT);
        if (ta == tb) continue;  // segment inside one tile: pass 1 wrote it
        T a8[8];
#pragma unroll
        for (int q = 0; q < 8; ++q) a8[q] = identity<OP, T>();
        const int stride = blockDim.x;
        int u = ta + 1 + threadIdx.x;
        for (; u + 7 * stride < tb; u += 8 * stride) {
#pragma unroll
            for (int q = 0; q < 8; ++q) a8[q] = combine<OP>(a8[q], tail[u + q * stride]);
        }
        for (; u < tb; u += stride) a8[0] = combine<OP>(a8[0], tail[u]);
        T acc = a8[0];
#pragma unroll
        for (int q = 1; q < 8; ++q) acc = combine<OP>(acc, a8[q]);
        acc = warp_reduce<OP>(acc);
        if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = acc;
        __syncthreads();
        if (threadIdx.x == 0) {
            T r = tail[ta];
            for (int k = 0; k < (int)(blockDim.x >> 5); ++k) r = combine<OP>(r, red[k]);
            out[sgi] = combine<OP>(r, head[tb]);
        }
        __syncthreads();
    }
}

// Long rows (m >= kSplitMinM = 8192): the flattened reduction as uniform chunks.
// Row i is cut into P equal pieces (P*n ~ 2 CTAs per SM); a 512-thread CTA
// reduces one piece with 4 independent 128-bit loads per thread in flight
// (no ring, no staging: every element is read once, straight into
// registers), leaving one partial per piece; a second pass combines the P
// partials of each row and applies d.  Same two-pass structure as the tiled
// engine, without its per-tile segment bookkeeping.
constexpr int64_t kSplitMinM = 1 << 13;
constexpr int kSplitThreads = 512;

// CTA-wide reduction of f over src[a, b) (NT threads, 4 independent 128-bit
// loads per thread in flight); the total is valid in thread 0.
template <typename T, int OP, int F, int NT>
__device__ __forceinline__ T cta_piece_reduce(const T* __restrict__ src, int64_t a, int64_t b, T* red) {
    using V = typename Vec4<T>::type;
    T acc4[4] = {identity<OP, T>(), identity<OP, T>(), identity<OP, T>(), identity<OP, T>()};
    // scalar head up to 16-byte alignment, vector body, scalar tail
    int64_t h = (int64_t)(((16u - ((uint32_t)(uintptr_t)(src + a) & 15u)) & 15u) / sizeof(T));
    if (h > b - a) h = b - a;
    for (int64_t k = a + threadIdx.x; k < a + h; k += NT) acc4[0] = combine<OP>(acc4[0], apply_map<F>(__ldg(src + k)));
    const T* body = src + a + h;
    const int64_t nv = (b - a - h) >> 2;
    int64_t v = threadIdx.x;
    for (; v + 3 * NT < nv; v += 4 * NT) {
        V q[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) q[u] = ldg_stream4(body + 4 * (v + u * NT));
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            T e[4];
            unpack4<T>(q[u], e);
#pragma unroll
            for (int c = 0; c < 4; ++c) acc4[c] = combine<OP>(acc4[c], apply_map<F>(e[c]));
        }
    }
    for (; v < nv; v += NT) {
        T e[4];
        unpack4<T>(ldg_stream4(body + 4 * v), e);
#pragma unroll
        for (int c = 0; c < 4; ++c) acc4[c] = combine<OP>(acc4[c], apply_map<F>(e[c]));
    }
    for (int64_t k = a + h + 4 * nv + threadIdx.x; k < b; k += NT) acc4[1] = combine<OP>(acc4[1], apply_map<F>(__ldg(src + k)));
    T acc = warp_reduce<OP>(combine<OP>(combine<OP>(acc4[0], acc4[1]), combine<OP>(acc4[2], acc4[3])));
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = acc;
    __syncthreads();
    T r = identity<OP, T>();
    if (threadIdx.x < 32) {
        r = threadIdx.x < NT / 32 ? red[threadIdx.x] : identity<OP, T>();
        r = warp_reduce<OP>(r);
    }
    return r;
}

// DIRECT (P = 1, V_MIDDLE's one-CTA-per-row use of the same kernel): the
// CTA's result is final, part[row] = d (+) row total.
template <typename T, int OP, int F, bool DIRECT = false, int NT = kSplitThreads>
__global__ void __launch_bounds__(NT) flat_red_split_kernel(const T* __restrict__ in, int64_t m, int P,
                                                            T* __restrict__ part, T d) {
    __shared__ T red[NT / 32];
    const int64_t row = blockIdx.x / P;
    const int piece = blockIdx.x % P;
    const int64_t len = ceil_div(ceil_div(m, P), 4) * 4;  // piece length, a multiple of 4 elements
    const int64_t a = std::min(m, (int64_t)piece * len), b = std::min(m, a + len);
    const T r = cta_piece_reduce<T, OP, F, NT>(in + row * m, a, b, red);
    if (threadIdx.x == 0) part[blockIdx.x] = DIRECT ? combine<OP>(d, r) : r;
}

// V_MIDDLE on the thread-block-cluster level (P:346's hierarchy one level up,
// SURVEY 8(f) NEXT-4): when there are fewer rows than SMs, one CLUSTER of C
// CTAs is the group of a row -- each CTA reduces a piece, the C partials are
// combined through distributed shared memory by the cluster's rank-0 CTA,
// which writes d (+) row total.  Still one group per segment, no second pass.
template <typename T, int OP, int F, int NT>
__global__ void __launch_bounds__(NT) segred_cluster_kernel(const T* __restrict__ in, T* __restrict__ out, int64_t m,
                                                            T d) {
    __shared__ T red[NT / 32];
    __shared__ T cta_total;
    unsigned rank, csize;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(rank));
    asm volatile("mov.u32 %0, %%cluster_nctarank;" : "=r"(csize));
    const int64_t row = blockIdx.x / csize;
    const int64_t len = ceil_div(ceil_div(m, (int64_t)csize), 4) * 4;
    const int64_t a = std::min(m, (int64_t)rank * len), b = std::min(m, a + len);
    const T r = cta_piece_reduce<T, OP, F, NT>(in + row * m, a, b, red);
    if (threadIdx.x == 0) cta_total = r;
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
    if (rank == 0 && threadIdx.x == 0) {
        T t = d;
        const uint32_t local = (uint32_t)__cvta_generic_to_shared(&cta_total);
        for (unsigned q = 0; q < csize; ++q) {
            uint32_t remote;
            asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(remote) : "r"(local), "r"(q));
            uint32_t bits;
            asm volatile("ld.shared::cluster.u32 %0, [%1];" : "=r"(bits) : "r"(remote) : "memory");
            t = combine<OP>(t, from_bits<T>(bits));
        }
        out[row] = t;
    }
    // keep every CTA's shared memory alive until rank 0 has read it
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

static int sm_count();

// V_MIDDLE for rows of >= 8192 elements: a 512-thread CTA per row (the group
// size V_MIDDLE already uses there; 1024 threads when rows are fewer than two
// per SM), 4 independent 128-bit loads per thread.
cudaError_t launch_segred_rows512(const SegArgs& a) {
    return dispatch_all(a.dt, a.op, a.f, [&](auto tt, auto opc, auto fc) -> cudaError_t {
        using T = decltype(tt);
        constexpr int OP = decltype(opc)::value, F = decltype(fc)::value;
        if (a.n > 0x7fffffffLL) return cudaErrorInvalidValue;
        if (a.n < 2 * sm_count())
            flat_red_split_kernel<T, OP, F, true, 1024><<<(unsigned)a.n, 1024, 0, a.stream>>>(
                (const T*)a.in, a.m, 1, (T*)a.out, bits_to<T>(a.ne_bits));
        else
            flat_red_split_kernel<T, OP, F, true><<<(unsigned)a.n, kSplitThreads, 0, a.stream>>>(
                (const T*)a.in, a.m, 1, (T*)a.out, bits_to<T>(a.ne_bits));
        return cudaGetLastError();
    });
}

// ----------------------------------------------------------------- V_CLUSTER
// The thread-block cluster as a hardware level between the CTA and the grid
// (P:346's hierarchy extended): a cluster of C CTAs is the
// group of one segment, its CTAs combine through distributed shared memory.

// Cluster size for a segred row: a power of two <= 16 so that n*C CTAs fill
// the GPU with pieces of >= 4096 elements (B200: n = 2^5..2^8 rows of
// 2^18..2^21 elements at 6.4-6.6 TB/s; 16-CTA clusters only while 8-CTA ones
// leave over half the SMs idle: 16 rows x 16 CTAs 40.9 us vs x 8 48.1).
static int64_t cluster_size_red(int64_t n, int64_t m) {
    const int64_t target = (int64_t)sm_count() * 4;
    int64_t C = 1;
    while (C * 2 <= 8 && C * 2 * n <= target && C * 2 * 4096 <= m) C *= 2;
    if (C == 8 && 16 * n <= (int64_t)sm_count() * 2 && 16 * 4096 <= m) C = 16;
    return C;
}

template <typename K, typename... Args>
static cudaError_t launch_clustered(K kernel, int64_t rows, int64_t C, int threads, size_t smem, cudaStream_t st,
                                    Args... args) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)(rows * C));
    cfg.blockDim = dim3(threads);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = (unsigned)C;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    if (C > 8) cudaFuncSetAttribute(kernel, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);  // opt-in
    return cudaLaunchKernelEx(&cfg, kernel, args...);
}

cudaError_t launch_segred_cluster(const SegArgs& a) {
    return dispatch_all(a.dt, a.op, a.f, [&](auto tt, auto opc, auto fc) -> cudaError_t {
        using T = decltype(tt);
        constexpr int OP = decltype(opc)::value, F = decltype(fc)::value;
        int64_t C = cluster_size_red(a.n, a.m);
        if (a.n * C > 0x7fffffffLL) return cudaErrorInvalidValue;
        // very few rows (<= 4): 16-CTA clusters of 1024-thread CTAs (B200: n = 2 / 4
        // 145 / 79 us -> 83 / 51 us; n = 8 is faster with 512 threads: 49 vs 60 us)
        const bool big = C == 16 && a.n * 32 <= (int64_t)sm_count();
        auto kc = big ? segred_cluster_kernel<T, OP, F, 1024> : segred_cluster_kernel<T, OP, F, kSplitThreads>;
        cudaError_t e = launch_clustered(kc, a.n, C, big ? 1024 : kSplitThreads, 0, a.stream, (const T*)a.in,
                                         (T*)a.out, a.m, bits_to<T>(a.ne_bits));
        if (e != cudaSuccess && C > 8) {  // 16-CTA clusters refused: the portable size
            (void)cudaGetLastError();
            e = launch_clustered(kc, a.n, 8, big ? 1024 : kSplitThreads, 0, a.stream, (const T*)a.in, (T*)a.out, a.m,
                                 bits_to<T>(a.ne_bits));
        }
        return e;
    });
}

// segscan on the cluster level: CTA r of a row's cluster holds piece r of the
// row in shared memory (read once, f applied), reduces it, and after a cluster
// barrier takes its carry-in = d (+) totals of CTAs 0..r-1 through DSMEM; it
// then scans its piece from shared memory and stores it -- one read and one
// write per element.  Each thread scans a contiguous run of the piece (padded
// layout p + p/32: conflict-light strided runs).  Fit: a piece of at most
// kClPieceMax elements per CTA, 16 CTAs per cluster at most.
constexpr int kClThreads = 512;
constexpr int64_t kClPieceMax = 40960;  // 160 KB of f32 (+ padding) per CTA

__device__ __forceinline__ int clpad(int p) { return p + (p >> 5); }

template <typename T, int OP, int F>
__global__ void __launch_bounds__(kClThreads) segscan_cluster_kernel(const T* in, T* out, int64_t m, T d,
                                                                     const T* __restrict__ seed, bool rev) {
    extern __shared__ __align__(16) uint8_t cl_raw[];
    T* piece = reinterpret_cast<T*>(cl_raw);
    __shared__ T red[kClThreads / 32];
    __shared__ T cta_total, s_carry;
    unsigned rank, csize;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(rank));
    asm volatile("mov.u32 %0, %%cluster_nctarank;" : "=r"(csize));
    const int t = threadIdx.x, lane = t & 31, w = t >> 5;
    const int64_t row = blockIdx.x / csize;
    const int64_t len = ceil_div(ceil_div(m, (int64_t)csize), 4) * 4;
    const int64_t a = std::min(m, (int64_t)rank * len), b = std::min(m, a + len);
    const int L = (int)(b - a);
    const T* src = in + row * m;
    T* dst = out + row * m;
    using V = typename Vec4<T>::type;
    // 128-bit loads when the piece starts 16-byte aligned (pieces are multiples of 4 elements)
    const bool vec = !rev && (((uintptr_t)(src + a)) & 15u) == 0 && (L & 3) == 0;
    if (vec) {
        for (int q = t; q < (L >> 2); q += kClThreads) {
            T e[4];
            unpack4<T>(ld_coh4(src + a + 4 * q), e);
#pragma unroll
            for (int u = 0; u < 4; ++u) piece[clpad(4 * q + u)] = apply_map<F>(e[u]);
        }
    } else {
        for (int p = t; p < L; p += kClThreads) piece[clpad(p)] = apply_map<F>(src[rev ? m - 1 - (a + p) : a + p]);
    }
    __syncthreads();
    const int CL = (L + kClThreads - 1) / kClThreads;
    const int lo = min(L, t * CL), hi = min(L, lo + CL);
    T s = identity<OP, T>();
    for (int k = lo; k < hi; ++k) s = combine<OP>(s, piece[clpad(k)]);
    // CTA exclusive scan of the thread sums
    T inc = s;
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
        const T o = __shfl_up_sync(0xffffffffu, inc, off);
        if (lane >= off) inc = combine<OP>(o, inc);
    }
    if (lane == 31) red[w] = inc;
    T ex = __shfl_up_sync(0xffffffffu, inc, 1);
    if (lane == 0) ex = identity<OP, T>();
    __syncthreads();
    T before = identity<OP, T>(), tot = identity<OP, T>();
#pragma unroll
    for (int q = 0; q < kClThreads / 32; ++q) {
        if (q < w) before = combine<OP>(before, red[q]);
        tot = combine<OP>(tot, red[q]);
    }
    ex = combine<OP>(before, ex);
    if (t == 0) cta_total = tot;
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
    if (t == 0) {
        T c = seed ? seed[row] : d;
        const uint32_t local = (uint32_t)__cvta_generic_to_shared(&cta_total);
        for (unsigned q = 0; q < rank; ++q) {
            uint32_t remote, bits;
            asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(remote) : "r"(local), "r"(q));
            asm volatile("ld.shared::cluster.u32 %0, [%1];" : "=r"(bits) : "r"(remote) : "memory");
            c = combine<OP>(c, from_bits<T>(bits));
        }
        s_carry = c;
    }
    __syncthreads();
    T run = combine<OP>(s_carry, ex);
    for (int k = lo; k < hi; ++k) {
        run = combine<OP>(run, piece[clpad(k)]);
        piece[clpad(k)] = run;
    }
    __syncthreads();
    if (vec && (((uintptr_t)(dst + a)) & 15u) == 0) {
        for (int q = t; q < (L >> 2); q += kClThreads) {
            V o;
            o.x = piece[clpad(4 * q)];
            o.y = piece[clpad(4 * q + 1)];
            o.z = piece[clpad(4 * q + 2)];
            o.w = piece[clpad(4 * q + 3)];
            *reinterpret_cast<V*>(dst + a + 4 * q) = o;
        }
    } else {
        for (int p = t; p < L; p += kClThreads) dst[rev ? m - 1 - (a + p) : a + p] = piece[clpad(p)];
    }
    // keep every CTA's shared memory alive until the higher ranks have read its total
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

// Cluster size for a segscan row: the smallest power of two whose pieces fit,
// grown (<= 16) while the clusters leave SMs idle and pieces stay >= 2048.
// 0 = does not fit (m > 16 * kClPieceMax).
int64_t cluster_size_scan(int64_t n, int64_t m) {
    int64_t C = 1;
    while (C <= 16 && C * kClPieceMax < m) C *= 2;
    if (C > 16) return 0;
    while (C * 2 <= 16 && n * C < 2 * (int64_t)sm_count() && m / (C * 2) >= 2048) C *= 2;
    return C;
}

cudaError_t launch_segscan_cluster(const SegArgs& a) {
    const int64_t C = cluster_size_scan(a.n, a.m);
    if (C == 0) return cudaErrorNotSupported;
    if (a.n * C > 0x7fffffffLL) return cudaErrorInvalidValue;
    return dispatch_all(a.dt, a.op, a.f, [&](auto tt, auto opc, auto fc) -> cudaError_t {
        using T = decltype(tt);
        constexpr int OP = decltype(opc)::value, F = decltype(fc)::value;
        const int64_t len = ceil_div(ceil_div(a.m, C), 4) * 4;
        const size_t smem = (size_t)(len + len / 32 + 1) * sizeof(T);
        auto k = segscan_cluster_kernel<T, OP, F>;
        static bool attr = false;
        if (!attr) {
            cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 (int)((kClPieceMax + kClPieceMax / 32 + 1) * sizeof(T)));
            attr = true;
        }
        cudaError_t e = launch_clustered(k, a.n, C, kClThreads, smem, a.stream, (const T*)a.in, (T*)a.out, a.m,
                                         bits_to<T>(a.ne_bits), (const T*)a.seed, a.rev);
        if (e != cudaSuccess && C > 8) {  // 16-CTA clusters refused: this row does not fit 8 pieces
            (void)cudaGetLastError();
            if (8 * kClPieceMax < a.m) return cudaErrorNotSupported;
            const int64_t len8 = ceil_div(ceil_div(a.m, (int64_t)8), 4) * 4;
            e = launch_clustered(k, a.n, 8, kClThreads, (size_t)(len8 + len8 / 32 + 1) * sizeof(T), a.stream,
                                 (const T*)a.in, (T*)a.out, a.m, bits_to<T>(a.ne_bits), (const T*)a.seed, a.rev);
        }
        return e;
    });
}

// A warp per row combines its P piece partials (lanes stride over the pieces,
// a shuffle tree joins them): no single thread walks hundreds of partials.
template <typename T, int OP>
__global__ void __launch_bounds__(256) flat_red_split_fix(const T* __restrict__ part, T* __restrict__ out, int64_t n,
                                                          int P, T d) {
    const int lane = threadIdx.x & 31;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < n; i += nw) {
        T r = identity<OP, T>();
        for (int p = lane; p < P; p += 32) r = combine<OP>(r, part[i * P + p]);
        r = warp_reduce<OP>(r);
        if (lane == 0) out[i] = combine<OP>(d, r);
    }
}

// ------------------------------------------------------------------ segscan

// Thread-local segmented inclusive scan of the thread's items (in registers).
template <typename T, int OP, int F>
__device__ __forceinline__ void local_seg_scan(T (&v)[FI], const ThreadPos& tp, T d, bool& has_start, T& acc,
                                               const T* __restrict__ seed) {
    has_start = false;
    acc = identity<OP, T>();
    if (tp.nx0 > tp.nvalid) {  // no boundary: plain inclusive scan
#pragma unroll
        for (int k = 0; k < FI; ++k) {
            acc = combine<OP>(acc, apply_map<F>(v[k]));
            v[k] = acc;
        }
    } else {
        int nx = tp.nx0;
        int64_t ss = tp.seg + (tp.nx0 > 0 ? 1 : 0);  // segment the next start begins
#pragma unroll
        for (int k = 0; k < FI; ++k) {
            if (k < tp.nvalid) {
                const T x = apply_map<F>(v[k]);
                if (k == nx) {
                    acc = combine<OP>(seed ? seed[ss] : d, x);
                    ++ss;
                    has_start = true;
                    nx += tp.mi;
                } else {
                    acc = combine<OP>(acc, x);
                }
                v[k] = acc;
            }
        }
    }
}

constexpr int kScanThreads = FB + 32;  // 8 consumer warps + 1 producer warp

// Single-pass segmented scan with decoupled look-back over dynamically claimed
// tiles (one global read and one global write per element, no second pass).
// Warp 8 is the producer: it claims the next tile with an atomic counter (so
// tiles are claimed in index order and a tile's predecessors are always owned
// by running CTAs -- no co-residency requirement), writes the slot metadata
// and issues the TMA load.  Warps 0-7 consume a slot:
//   1. thread-local + CTA segmented scan of the tile (as the other engines);
//   2. publish the tile status at once: INCLUSIVE when the tile holds a
//      segment start (its carry-out no longer depends on predecessors),
//      AGGREGATE otherwise;
//   3. if the tile's first element continues a segment, a CTA-wide look-back:
//      the 256 consumer threads read the status words of the 256 preceding
//      tiles in one round trip (a window wide enough that the inclusive prefix
//      published one L2 round trip earlier lies inside it at full HBM rate),
//      fold the aggregates down to the nearest inclusive one, bounded
//      arithmetically by the tile holding the segment's start; then publish
//      the tile's own inclusive prefix;
//   4. apply the carry, store the tile from its slot with a TMA bulk store.
// The last CTA re-arms the workspace (tile counter 0, epoch + 1).

// CTA-wide look-back over status words [cs, pred], W words per thread
// (window NW*32*W per round trip): folds the aggregates from the nearest
// inclusive (or segment-start) word up to pred.  NAMED: the consumer warps
// synchronise on named barrier 1 (a producer warp does not take part).
template <typename T, int OP, int NW, int W, bool NAMED>
__device__ __forceinline__ T cta_lookback_w(const uint64_t* status, uint32_t tag, int pred, int cs, int* s_lbterm,
                                            T* s_lbval) {
    constexpr int NT = NW * 32;
    const int t = threadIdx.x, lane = t & 31, w = t >> 5;
    auto sync = [] {
        if (NAMED) asm volatile("bar.sync 1, %0;" ::"n"(NT) : "memory");
        else __syncthreads();
    };
    T carry = identity<OP, T>();
    while (true) {
        const int top = pred - t * W;  // this thread's newest word
        uint64_t wd[W];
#pragma unroll
        for (int q = 0; q < W; ++q) wd[q] = (top - q >= cs) ? ld_relaxed_u64(&status[top - q]) : 0;
        T tv = identity<OP, T>();
        bool tterm = false;
#pragma unroll
        for (int q = 0; q < W; ++q) {
            const int idx = top - q;
            if (!tterm) {
                if (idx < cs) {
                    tterm = true;
                } else {
                    while ((uint32_t)(wd[q] >> 35) != tag || ((wd[q] >> 33) & 3u) == 0)
                        wd[q] = ld_relaxed_u64(&status[idx]);
                    tv = combine<OP>(from_bits<T>((uint32_t)wd[q]), tv);  // older (+) newer
                    tterm = idx == cs || ((wd[q] >> 33) & 3u) == ST_P || ((wd[q] >> 32) & 1u);
                }
            }
        }
        const uint32_t tb = __ballot_sync(0xffffffffu, tterm);
        if (lane == 0) s_lbterm[w] = tb ? (w * 32 + __ffs(tb) - 1) : NT;
        sync();
        int stop = NT;
#pragma unroll
        for (int k = 0; k < NW; ++k) stop = min(stop, s_lbterm[k]);
        T val = t <= stop ? tv : identity<OP, T>();
#pragma unroll
        for (int off = 1; off < 32; off <<= 1) {  // ordered: higher lane = older words
            const T older = __shfl_down_sync(0xffffffffu, val, off);
            if (lane + off < 32) val = combine<OP>(older, val);
        }
        if (lane == 0) s_lbval[w] = val;
        sync();
        T win = identity<OP, T>();
#pragma unroll
        for (int k = NW - 1; k >= 0; --k) win = combine<OP>(win, s_lbval[k]);
        carry = combine<OP>(win, carry);
        sync();
        if (stop < NT) break;
        pred -= NT * W;
    }
    return carry;
}
#ifndef IFL_DLB_LBW
#define IFL_DLB_LBW 1
#endif
// Used for tile-aligned segments only (no look-back): 2 slots x 4 CTAs per SM
// (B200, n*m = 2^26 f32, m = 32..1024: 81-83 us = a copy's speed; 3 x 3: 82-91)
#ifndef IFL_DLB_SLOTS
#define IFL_DLB_SLOTS 2
#endif
#ifndef IFL_DLB_MINB
#define IFL_DLB_MINB 4
#endif
constexpr int kDlbSlots = IFL_DLB_SLOTS;

template <typename T, int OP, int F>
__global__ void __launch_bounds__(kScanThreads, IFL_DLB_MINB) flat_scan_dlb_kernel(const T* in, T* out, int64_t N, int64_t m, T d,
                                                                      uint8_t* ws, int num_tiles, bool tma_in,
                                                                      bool tma_out, const T* __restrict__ seed, bool rev) {
    extern __shared__ __align__(128) uint8_t smem_raw[];
    T* ring = reinterpret_cast<T*>(smem_raw);
    __shared__ alignas(8) uint64_t full[kDlbSlots], empty[kDlbSlots];
    __shared__ SlotMeta meta[kDlbSlots];
    __shared__ uint32_t s_tag;
    __shared__ T s_wval[2][FB / 32];
    __shared__ uint32_t s_wflag[2][FB / 32];
    __shared__ int s_lbterm[FB / 32];
    __shared__ T s_lbval[FB / 32];
    unsigned long long* ctr = reinterpret_cast<unsigned long long*>(ws);  // {epoch:32 | done:32}
    unsigned* tile_ctr = reinterpret_cast<unsigned*>(ws + 8);
    uint64_t* status = reinterpret_cast<uint64_t*>(ws + sizeof(FlatHdr));
    const int t = threadIdx.x, lane = t & 31, w = t >> 5;
    const int G = gridDim.x;
    if (t == 0) {
        s_tag = status_tag(ld_relaxed_u64(reinterpret_cast<const uint64_t*>(ctr)));
        for (int q = 0; q < kDlbSlots; ++q) {
            mbar_init(&full[q], 1);
            mbar_init(&empty[q], 1);
        }
        fence_mbar_init();
    }
    __syncthreads();

    if (w == FB / 32) {
        // ================= producer warp (one lane)
        if (lane == 0) {
            const uint64_t pol = policy_evict_first();
            for (int wv = 0;; ++wv) {
                const int sl = wv % kDlbSlots;
                if (wv >= kDlbSlots) mbar_wait(&empty[sl], ((wv / kDlbSlots) - 1) & 1);
                const int tile = (int)atomicAdd(tile_ctr, 1u);
                SlotMeta& sm = meta[sl];
                if (tile >= num_tiles) {
                    sm.tile = -1;
                    mbar_arrive_expect_tx(&full[sl], 0);
                    break;
                }
                fill_meta(sm, tile, N, m);
                if (tma_in && sm.cnt == FT) {
                    mbar_arrive_expect_tx(&full[sl], FT * sizeof(T));
                    bulk_g2s_hint(ring + sl * FT, in + (int64_t)tile * FT, FT * sizeof(T), &full[sl], pol);
                } else {
                    mbar_arrive_expect_tx(&full[sl], 0);  // consumers copy it themselves
                }
            }
        }
        return;
    }

    // ================= consumer warps 0-7
    const uint32_t tag = s_tag;
    uint32_t phase_bits = 0;
    int pend_slot = -1;  // slot whose bulk store may still be reading smem (thread 0)
    for (int i = 0;; ++i) {
        const int sl = i % kDlbSlots;
        T* buf = ring + sl * FT;
        mbar_wait(&full[sl], (phase_bits >> sl) & 1u);
        phase_bits ^= 1u << sl;
        const SlotMeta sm = meta[sl];
        if (t == 0 && pend_slot >= 0) {  // the previous tile's bulk store has long been issued
            bulk_wait_read0();
            mbar_arrive_expect_tx(&empty[pend_slot], 0);
            pend_slot = -1;
        }
        if (sm.tile < 0) break;
        const int64_t base = (int64_t)sm.tile * FT;
        if (!(tma_in && sm.cnt == FT)) {
            for (int p = t; p < sm.cnt; p += FB) buf[p] = in[rev ? N - 1 - (base + p) : base + p];
            consumer_sync();
        }
        const ThreadPos tp = thread_pos(sm, m);
        T v[FI];
        load_items(buf, v);
        bool hs;
        T acc;
        local_seg_scan<T, OP, F>(v, tp, d, hs, acc, seed);
        uint32_t exf, aggf;
        T exv, aggv;
        cta_seg_scan<T, OP, true>(hs ? 1u : 0u, acc, exf, exv, aggf, aggv, s_wval[i & 1], s_wflag[i & 1]);
        const bool carry_needed = sm.pos != 0;  // the tile's first element continues a segment
        if (t == 0)
            st_relaxed_u64(&status[sm.tile], pack_status(tag, (aggf || !carry_needed) ? ST_P : ST_A, aggf,
                                                         to_bits(aggv)));
        T carry = identity<OP, T>();
        if (carry_needed) {
            const int cs = (int)((base - sm.pos) / FT);  // tile holding the segment's start
            carry = cta_lookback_w<T, OP, FB / 32, IFL_DLB_LBW, true>(status, tag, sm.tile - 1, cs, s_lbterm, s_lbval);
            if (!aggf && t == 0)
                st_relaxed_u64(&status[sm.tile], pack_status(tag, ST_P, 0u, to_bits(combine<OP>(carry, aggv))));
        }
        {
            const T carry_t = exf ? exv : combine<OP>(carry, exv);
            const int lim = min(tp.nx0, tp.nvalid);
#pragma unroll
            for (int k = 0; k < FI; ++k)
                if (k < lim) v[k] = combine<OP>(carry_t, v[k]);
        }
        store_items(buf, v);
        const bool bulk = tma_out && sm.cnt == FT;
        if (bulk) fence_proxy_async_smem();
        consumer_sync();
        if (bulk) {
            if (t == 0) {
                bulk_s2g_hint(out + base, buf, FT * sizeof(T), policy_evict_first());
                bulk_commit();
                pend_slot = sl;
            }
        } else {
            for (int p = t; p < sm.cnt; p += FB) out[rev ? N - 1 - (base + p) : base + p] = buf[p];
            consumer_sync();
            if (t == 0) mbar_arrive_expect_tx(&empty[sl], 0);
        }
    }
    if (t == 0) {
        bulk_wait0();
        __threadfence();
        const unsigned long long old = atomicAdd(ctr, 1ull);
        if ((uint32_t)old == (uint32_t)G - 1) {  // every CTA has made its last claim: re-arm
            atomicExch(tile_ctr, 0u);
            atomicAdd(ctr, (1ull << 32) - (unsigned long long)G);
        }
    }
}

// ---------------------------------------------------------------------------
// "Job ring" engine (JR): reduce-then-scan desynchronised into jobs and
// streamed through one TMA ring per CTA.  Chunks of kJrChunkTiles tiles;
// job k (claimed in order from an atomic counter by a persistent CTA)
//   1. AGGREGATES chunk k: the tiles covering the part a successor needs
//      (after the chunk's last segment start; all of it for long segments)
//      are streamed from DRAM with L2::evict_last and reduced; the
//      segmented aggregate is published (an inclusive prefix when the chunk
//      holds a segment start);
//   2. SCANS chunk k - lag: the aggregates of its predecessors were
//      published `lag` jobs ago, so the CTA-wide look-back (2 words per
//      thread) ends in one round trip -- it never waits on a status written
//      moments ago, which under a saturated memory system takes microseconds
//      to become visible; the chunk's own inclusive prefix is published, and
//      its tiles -- pulled into L2 by step 1 -- are scanned with a running
//      carry and stored from their slots by TMA bulk stores.
// One producer warp feeds both steps through the same ring, so loads never
// pause between them; DRAM sees one read and one write per element.  A job's
// aggregation never waits on anything, so every claimed job completes
// (no co-residency requirement).
#ifndef IFL_JR_CHUNK_TILES
#define IFL_JR_CHUNK_TILES 4
#endif
#ifndef IFL_JR_LAG
#define IFL_JR_LAG 192
#endif
#ifndef IFL_JR_SLOTS
#define IFL_JR_SLOTS 3
#endif
#ifndef IFL_JR_MINB
#define IFL_JR_MINB 3
#endif
#ifndef IFL_JR_LBW
#define IFL_JR_LBW 2
#endif
constexpr int kJrChunkTiles = IFL_JR_CHUNK_TILES;
constexpr int kJrSlots = IFL_JR_SLOTS;

struct JrMeta {
    int tile;   // tile index
    int cnt;    // valid elements of the tile
    int kind;   // 0 aggregate, 1 scan, -1 no more work
    int chunk;
    int flags;  // agg: 1 = last tile of the chunk's range; scan: 1 = first tile of the chunk
    int a0, a1; // agg: range inside the tile
    int64_t pos, seg;  // scan: position of the tile's first element in its segment, segment index
};

__device__ __forceinline__ void mbar_arrive_cnt(uint64_t* bar, uint32_t cnt) {
    asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(cnt) : "memory");
}

template <typename T, int OP, int F>
__global__ void __launch_bounds__(kScanThreads, IFL_JR_MINB) flat_scan_jr_kernel(const T* in, T* out, int64_t N, int64_t m, T d,
                                                                    uint8_t* ws, int num_tiles, int num_chunks, int lag,
                                                                    bool tma_in, bool tma_out, const T* __restrict__ seed, bool rev) {
    extern __shared__ __align__(128) uint8_t smem_raw[];
    T* ring = reinterpret_cast<T*>(smem_raw);
    __shared__ alignas(8) uint64_t full[kJrSlots], empty[kJrSlots];
    __shared__ JrMeta meta[kJrSlots];
    __shared__ uint32_t s_tag;
    __shared__ T s_wval[2][FB / 32];
    __shared__ uint32_t s_wflag[2][FB / 32];
    __shared__ int s_lbterm[FB / 32];
    __shared__ T s_lbval[FB / 32];
    unsigned long long* ctr = reinterpret_cast<unsigned long long*>(ws);  // {epoch:32 | done:32}
    unsigned* job_ctr = reinterpret_cast<unsigned*>(ws + 8);
    uint64_t* status = reinterpret_cast<uint64_t*>(ws + sizeof(FlatHdr));
    const int t = threadIdx.x, lane = t & 31, w = t >> 5;
    const int G = gridDim.x;
    const int64_t CH = (int64_t)kJrChunkTiles * FT;
    constexpr uint32_t NCW = FB / 32;  // consumer warps: the empty barriers count their arrivals
    if (t == 0) {
        s_tag = status_tag(ld_relaxed_u64(reinterpret_cast<const uint64_t*>(ctr)));
        for (int q = 0; q < kJrSlots; ++q) {
            mbar_init(&full[q], 1);
            mbar_init(&empty[q], NCW);
        }
        fence_mbar_init();
    }
    __syncthreads();
    const uint32_t tag = s_tag;

    if (w == FB / 32) {
        // ================= producer warp (one lane)
        if (lane == 0) {
            const uint64_t pol_keep = policy_evict_last(), pol_stream = policy_evict_first();
            int wv = 0;
            auto slot = [&]() -> int {
                const int sl = wv % kJrSlots;
                if (wv >= kJrSlots) mbar_wait(&empty[sl], ((wv / kJrSlots) - 1) & 1);
                ++wv;
                return sl;
            };
            auto issue = [&](int sl, const JrMeta& jm, uint64_t pol) {
                meta[sl] = jm;
                if (tma_in && jm.cnt == FT) {
                    mbar_arrive_expect_tx(&full[sl], FT * sizeof(T));
                    bulk_g2s_hint(ring + sl * FT, in + (int64_t)jm.tile * FT, FT * sizeof(T), &full[sl], pol);
                } else {
                    mbar_arrive_expect_tx(&full[sl], 0);  // consumers read global memory themselves
                }
            };
            while (true) {
                const int k = (int)atomicAdd(job_ctr, 1u);
                if (k >= num_chunks + lag) {
                    const int sl = slot();
                    meta[sl].kind = -1;
                    mbar_arrive_expect_tx(&full[sl], 0);
                    break;
                }
                if (k < num_chunks) {  // 1. aggregate chunk k
                    const int64_t cb = (int64_t)k * CH, ce = std::min(N, cb + CH);
                    const int64_t ls = ((ce - 1) / m) * m;
                    const int64_t lo = ls >= cb ? ls : cb;
                    const int ta = (int)(lo / FT), tb = (int)((ce - 1) / FT);
                    for (int tile = ta; tile <= tb; ++tile) {
                        JrMeta jm;
                        jm.tile = tile;
                        jm.cnt = (int)std::min((int64_t)FT, N - (int64_t)tile * FT);
                        jm.kind = 0;
                        jm.chunk = k;
                        jm.flags = tile == tb ? 1 : 0;
                        jm.a0 = (int)std::max<int64_t>(0, lo - (int64_t)tile * FT);
                        jm.a1 = (int)std::min<int64_t>(jm.cnt, ce - (int64_t)tile * FT);
                        jm.pos = jm.seg = 0;
                        issue(slot(), jm, pol_keep);
                    }
                }
                const int c = k - lag;
                if (c >= 0) {  // 2. scan chunk c
                    const int t0 = c * kJrChunkTiles;
                    const int L = min(kJrChunkTiles, num_tiles - t0);
                    int64_t pos = ((int64_t)t0 * FT) % m, seg = ((int64_t)t0 * FT) / m;
                    for (int j = 0; j < L; ++j) {
                        JrMeta jm;
                        jm.tile = t0 + j;
                        jm.cnt = (int)std::min((int64_t)FT, N - (int64_t)jm.tile * FT);
                        jm.kind = 1;
                        jm.chunk = c;
                        jm.flags = j == 0 ? 1 : 0;
                        jm.a0 = jm.a1 = 0;
                        jm.pos = pos;
                        jm.seg = seg;
                        issue(slot(), jm, pol_stream);
                        pos += FT;
                        if (pos >= m) {
                            if (m > FT) {
                                pos -= m;
                                seg += 1;
                            } else {
                                seg += pos / m;
                                pos %= m;
                            }
                        }
                    }
                }
            }
        }
    } else {
        // ================= consumer warps 0-7
        uint32_t phase_bits = 0;
        int pend_slot = -1;
        T acc_a = identity<OP, T>();  // running aggregate of the chunk being aggregated
        T carry = identity<OP, T>();  // running carry of the chunk being scanned
        for (int i = 0;; ++i) {
            const int sl = i % kJrSlots;
            T* buf = ring + sl * FT;
            mbar_wait(&full[sl], (phase_bits >> sl) & 1u);
            phase_bits ^= 1u << sl;
            const JrMeta jm = meta[sl];
            if (t == 0 && pend_slot >= 0) {  // the previous scan tile's bulk store has been issued long ago
                bulk_wait_read0();
                mbar_arrive_cnt(&empty[pend_slot], NCW);
                pend_slot = -1;
            }
            if (jm.kind < 0) break;
            const int64_t base = (int64_t)jm.tile * FT;
            const bool in_smem = tma_in && jm.cnt == FT;
            if (jm.kind == 0) {
                // ---- aggregate: this tile's part of the chunk's needed range
                if (in_smem) {
                    for (int q = jm.a0 + t; q < jm.a1; q += FB) acc_a = combine<OP>(acc_a, apply_map<F>(buf[q]));
                } else {
                    for (int q = jm.a0 + t; q < jm.a1; q += FB) acc_a = combine<OP>(acc_a, apply_map<F>(in[rev ? N - 1 - (base + q) : base + q]));
                }
                consumer_sync();  // every consumer warp is done with the slot
                if (t == 0) mbar_arrive_cnt(&empty[sl], NCW);
                if (jm.flags & 1) {  // last tile of the range: CTA total, publish
                    T r = warp_reduce<OP>(acc_a);
                    if (lane == 0) s_lbval[w] = r;
                    consumer_sync();
                    if (t == 0) {
                        r = identity<OP, T>();
#pragma unroll
                        for (int q = 0; q < FB / 32; ++q) r = combine<OP>(r, s_lbval[q]);
                        const int64_t cb = (int64_t)jm.chunk * CH, ce = std::min(N, cb + CH);
                        const int64_t ls = ((ce - 1) / m) * m;
                        const bool flag = ls >= cb;
                        const T dseg = seed ? seed[ls / m] : d;
                        st_relaxed_u64(&status[jm.chunk], pack_status(tag, flag ? ST_P : ST_A, flag ? 1u : 0u,
                                                                      to_bits(flag ? combine<OP>(dseg, r) : r)));
                    }
                    consumer_sync();
                    acc_a = identity<OP, T>();
                }
                continue;
            }
            // ---- scan tile
            if (jm.flags & 1) {  // first tile of the chunk: carry-in
                const int c = jm.chunk;
                const int64_t cb = (int64_t)c * CH;
                carry = identity<OP, T>();
                if (cb % m != 0) {
                    const int cs = (int)(((cb / m) * m) / CH);  // chunk holding the segment's start
                    carry = cta_lookback_w<T, OP, FB / 32, IFL_JR_LBW, true>(status, tag, c - 1, cs, s_lbterm, s_lbval);
                }
                if (t == 0) {  // own aggregate: published (and so read) before this chunk is overwritten
                    uint64_t own;
                    do {
                        own = ld_relaxed_u64(&status[c]);
                    } while ((uint32_t)(own >> 35) != tag || ((own >> 33) & 3u) == 0);
                    if (((own >> 33) & 3u) != ST_P)
                        st_relaxed_u64(&status[c], pack_status(tag, ST_P, 0u,
                                                               to_bits(combine<OP>(carry, from_bits<T>((uint32_t)own)))));
                }
                consumer_sync();
            }
            if (!in_smem) {
                for (int p = t; p < jm.cnt; p += FB) buf[p] = in[rev ? N - 1 - (base + p) : base + p];
                consumer_sync();
            }
            SlotMeta smeta;
            smeta.tile = jm.tile;
            smeta.cnt = jm.cnt;
            smeta.pos = jm.pos;
            smeta.seg = jm.seg;
            const ThreadPos tp = thread_pos(smeta, m);
            T v[FI];
            load_items(buf, v);
            bool hs;
            T acc;
            local_seg_scan<T, OP, F>(v, tp, d, hs, acc, seed);
            uint32_t exf, aggf;
            T exv, aggv;
            cta_seg_scan<T, OP, true>(hs ? 1u : 0u, acc, exf, exv, aggf, aggv, s_wval[i & 1], s_wflag[i & 1]);
            {
                const T carry_t = exf ? exv : combine<OP>(carry, exv);
                const int lim = min(tp.nx0, tp.nvalid);
#pragma unroll
                for (int k = 0; k < FI; ++k)
                    if (k < lim) v[k] = combine<OP>(carry_t, v[k]);
            }
            carry = aggf ? aggv : combine<OP>(carry, aggv);
            store_items(buf, v);
            const bool bulk = tma_out && jm.cnt == FT;
            if (bulk) fence_proxy_async_smem();
            consumer_sync();
            if (bulk) {
                if (t == 0) {
                    bulk_s2g_hint(out + base, buf, FT * sizeof(T), policy_evict_first());
                    bulk_commit();
                    pend_slot = sl;
                }
            } else {
                for (int p = t; p < jm.cnt; p += FB) out[rev ? N - 1 - (base + p) : base + p] = buf[p];
                consumer_sync();
                if (t == 0) mbar_arrive_cnt(&empty[sl], NCW);
            }
        }
        if (t == 0) bulk_wait0();
    }
    if (t == 0) {
        __threadfence();
        const unsigned long long old = atomicAdd(ctr, 1ull);
        if ((uint32_t)old == (uint32_t)G - 1) {  // every CTA has made its last claim: re-arm
            atomicExch(job_ctr, 0u);
            atomicAdd(ctr, (1ull << 32) - (unsigned long long)G);
        }
    }
}

// ------------------------------------------------------------------ launch

static int sm_count() {
    static int n = 0;
    if (!n) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
        if (n <= 0) n = 148;
    }
    return n;
}

template <typename K>
static int resident_ctas(K kernel, size_t smem, int threads = FB) {
    static thread_local std::unordered_map<const void*, int> cache;
    auto it = cache.find((const void*)kernel);
    if (it != cache.end()) return it->second;
    cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    int per_sm = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kernel, threads, smem);
    if (per_sm < 1) per_sm = 1;
    const int n = per_sm * sm_count();
    cache[(const void*)kernel] = n;
    return n;
}

cudaError_t launch_flat(const SegArgs& a, bool scan) {
    const int64_t N = a.n * a.m;
    const int64_t tiles = ceil_div(N, kFlatTile);
    if (tiles > 0x3fffffffLL) return cudaErrorInvalidValue;
    // reverse scans: the flat index space mirrored (element k is physical n*m-1-k:
    // rows reversed, in reverse order -- the same regular segments), read and
    // written by the engines' cooperative (non-TMA) paths
    const bool tma_in = !a.rev && ((uintptr_t)a.in % 16) == 0;
    const bool tma_out = !a.rev && ((uintptr_t)a.out % 16) == 0;
    uint8_t* ws = (uint8_t*)a.ws;
    return dispatch_all(a.dt, a.op, a.f, [&](auto tt, auto opc, auto fc) -> cudaError_t {
        using T = decltype(tt);
        constexpr int OP = decltype(opc)::value, F = decltype(fc)::value;
        const T d = bits_to<T>(a.ne_bits);
        if (scan && FT % a.m == 0) {
            // every tile begins at a segment start: the tiles are independent, the
            // single-pass engine never looks back (B200, n*m = 2^26 f32, m = 1024:
            // 83 us, a copy's speed)
            auto k = flat_scan_dlb_kernel<T, OP, F>;
            const size_t smem_s = (size_t)kDlbSlots * FT * sizeof(T);
            const int grid = (int)std::min<int64_t>(tiles, resident_ctas(k, smem_s, kScanThreads));
            k<<<grid, kScanThreads, smem_s, a.stream>>>((const T*)a.in, (T*)a.out, N, a.m, d, ws, (int)tiles, tma_in,
                                                        tma_out, (const T*)a.seed, a.rev);
            return cudaGetLastError();
        }
        if (scan) {  // segments cross tiles: the job-ring engine
            auto k = flat_scan_jr_kernel<T, OP, F>;
            const size_t smem_s = (size_t)kJrSlots * FT * sizeof(T);
            const int chunks = (int)ceil_div(tiles, kJrChunkTiles);
            const int lag = std::min(IFL_JR_LAG, chunks);
            const int grid = (int)std::min<int64_t>(resident_ctas(k, smem_s, kScanThreads), chunks + lag);
            k<<<grid, kScanThreads, smem_s, a.stream>>>((const T*)a.in, (T*)a.out, N, a.m, d, ws, (int)tiles, chunks, lag,
                                                         tma_in, tma_out, (const T*)a.seed, a.rev);
            return cudaGetLastError();
        }
        T* head = reinterpret_cast<T*>(ws + sizeof(FlatHdr) + (size_t)tiles * 8);
        T* tail = head + tiles;
        if (a.m >= kSplitMinM) {
            // P pieces per row: n*P <= the resident CTAs of the GPU (a single wave, no
            // tail), pieces >= 8192 elements, so n*P <= tiles fits the head array
            auto ks = flat_red_split_kernel<T, OP, F>;
            const int64_t R = resident_ctas(ks, 0, kSplitThreads);
            const int P = (int)std::max<int64_t>(1, std::min<int64_t>(R / a.n, a.m / 8192));
            ks<<<(unsigned)(a.n * P), kSplitThreads, 0, a.stream>>>((const T*)a.in, a.m, P, head, d);
            cudaError_t e = cudaGetLastError();
            if (e != cudaSuccess) return e;
            const int g2 = (int)std::min<int64_t>(ceil_div(a.n, 8), (int64_t)sm_count() * 16);
            flat_red_split_fix<T, OP><<<g2, 256, 0, a.stream>>>(head, (T*)a.out, a.n, P, d);
            return cudaGetLastError();
        }
        auto k = flat_red_kernel<T, OP, F>;
        const size_t smem_r = (size_t)kRedSlots * FT * sizeof(T);
        const int grid = (int)std::min<int64_t>(tiles, resident_ctas(k, smem_r, FB + 32));
        k<<<grid, FB + 32, smem_r, a.stream>>>((const T*)a.in, (T*)a.out, N, a.m, d, head, tail, (int)tiles, tma_in);
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return e;
        if (a.m > FT) {
            const int g2 = (int)std::min<int64_t>(a.n, (int64_t)sm_count() * 4);
            flat_red_fix_long<T, OP><<<g2, 512, 0, a.stream>>>((T*)a.out, a.n, a.m, head, tail);
            e = cudaGetLastError();
        } else if (FT % a.m != 0 && tiles > 1) {
            const int g2 = (int)std::min<int64_t>(ceil_div(tiles, 256), (int64_t)sm_count() * 4);
            flat_red_fix_short<T, OP><<<g2, 256, 0, a.stream>>>((T*)a.out, a.m, head, tail, (int)tiles);
            e = cudaGetLastError();
        }
        return e;
    });
}

}  // namespace ifl

