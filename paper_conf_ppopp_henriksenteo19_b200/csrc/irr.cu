// irr.cu -- irregular nested parallelism: segred / segscan over segments
// given by an offset array (segment i = in[off[i] .. off[i+1]-1]), the
// paper's stated future work.  The same three G3
// versions, with an inspector measure of load imbalance in the
// guard ("inspectors can compute a measure of such properties, which
// can be integrated in the predicates"):
//   V_TOP     thread per segment, sequential walk (divergent and imbalanced
//             when lengths vary: its time is set by the longest segment);
//   V_MIDDLE  warp per segment: strided loads, shuffle reduce / warp scans
//             with a running carry;
//   V_FLAT    flattened over all elements: 4096-element tiles (256 threads x
//             16 items) with per-tile segment ranges, a CTA-wide segmented
//             scan of the thread pieces, and tile aggregates combined by a
//             single-CTA segmented scan over tiles:
//               pass 0  tile -> the segment holding its first element
//                       (each segment writes its tile starts; long ones with
//                       the whole warp); empty segments reduce to d;
//               pass 1  per tile: complete segments written; segred: the
//                       head / tail pieces of segments crossing tiles are
//                       combined into their outputs atomically (done);
//                       segscan: the tile's tail piece and flag recorded;
//               pass 2  (segscan) exclusive segmented scan of the tile tails;
//               pass 3  (segscan) the tile rescanned with its carry (two
//                       reads + one write per element).
#include <algorithm>

#include "common.cuh"
#include "dispatch.cuh"
#include "ifl_internal.h"

namespace ifl {

namespace {

constexpr int kIrrThreads = 256;
constexpr int kIrrItems = 16;
constexpr int64_t kIrrTile = (int64_t)kIrrThreads * kIrrItems;
constexpr int kIrrSmemOff = 2048;  // offsets of up to 2047 segments per tile staged in shared memory

// ------------------------------------------------------------ V_TOP

template <typename T, int OP, int F, bool SCAN>
__global__ void __launch_bounds__(256) irr_top_kernel(const T* __restrict__ in, T* __restrict__ out,
                                                      const int64_t* __restrict__ off, int64_t n, T d) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t a = off[i], b = off[i + 1];
        Acc<OP, T> acc(d);
#pragma unroll 4
        for (int64_t k = a; k < b; ++k) {
            acc.add(apply_map<F>(__ldg(in + k)));
            if constexpr (SCAN) out[k] = acc.get();
        }
        if constexpr (!SCAN) out[i] = acc.get();
    }
}

// ------------------------------------------------------------ V_MIDDLE

template <typename T, int OP, int F, bool SCAN>
__global__ void __launch_bounds__(256) irr_mid_kernel(const T* __restrict__ in, T* __restrict__ out,
                                                      const int64_t* __restrict__ off, int64_t n, T d) {
    const int lane = threadIdx.x & 31;
    const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t i = gw; i < n; i += nw) {
        const int64_t a = off[i], b = off[i + 1];
        if constexpr (!SCAN) {
            T acc[4] = {identity<OP, T>(), identity<OP, T>(), identity<OP, T>(), identity<OP, T>()};
            int64_t k = a + lane;
            for (; k + 96 < b; k += 128) {
                T x[4];
#pragma unroll
                for (int q = 0; q < 4; ++q) x[q] = __ldg(in + k + 32 * q);
#pragma unroll
                for (int q = 0; q < 4; ++q) acc[q] = combine<OP>(acc[q], apply_map<F>(x[q]));
            }
            for (; k < b; k += 32) acc[0] = combine<OP>(acc[0], apply_map<F>(__ldg(in + k)));
            T r = warp_reduce<OP>(combine<OP>(combine<OP>(acc[0], acc[1]), combine<OP>(acc[2], acc[3])));
            if (lane == 0) out[i] = combine<OP>(d, r);
        } else {
            Acc<OP, T> carry(d);
            for (int64_t base = a; base < b; base += 128) {  // 4 consecutive items per lane
                T x[4];
                const int64_t e0 = base + 4 * lane;
#pragma unroll
                for (int q = 0; q < 4; ++q) x[q] = e0 + q < b ? apply_map<F>(__ldg(in + e0 + q)) : identity<OP, T>();
#pragma unroll
                for (int q = 1; q < 4; ++q) x[q] = combine<OP>(x[q - 1], x[q]);
                T inc = x[3];
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const T y = __shfl_up_sync(0xffffffffu, inc, o);
                    if (lane >= o) inc = combine<OP>(y, inc);
                }
                T ex = __shfl_up_sync(0xffffffffu, inc, 1);
                if (lane == 0) ex = identity<OP, T>();
                const T tot = __shfl_sync(0xffffffffu, inc, 31);
                const T pre = combine<OP>(carry.get(), ex);
#pragma unroll
                for (int q = 0; q < 4; ++q)
                    if (e0 + q < b) out[e0 + q] = combine<OP>(pre, x[q]);
                carry.add(tot);
            }
        }
    }
}

// ------------------------------------------------------------ V_FLAT

// pass 0: every tile t learns the (non-empty) segment holding its first
// element: segment i writes tile_seg[t] for each tile start inside
// [off[i], off[i+1]) -- each tile exactly once, so no initialisation and no
// scan are needed.  A lane whose segment covers more than two tile starts
// hands it to its whole warp (ballot), so a long segment costs ~1/32 of its
// tiles per lane.  Empty segments reduce to d.
template <typename T, int OP, bool RED>
__global__ void __launch_bounds__(256) irr_claim_kernel(const int64_t* __restrict__ off, int64_t n,
                                                        int64_t* __restrict__ tile_seg, T* __restrict__ out, T d) {
    const int lane = threadIdx.x & 31;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    // uniform trip count per warp so the ballots see every lane
    const int64_t base0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) - lane;
    for (int64_t b0 = base0; b0 < n; b0 += stride) {
        const int64_t i = b0 + lane;
        int64_t t0 = 0, t1 = 0;  // tile starts [t0, t1) inside segment i
        if (i < n) {
            const int64_t a = off[i], b = off[i + 1];
            if (a == b) {
                if constexpr (RED) out[i] = d;
            } else {
                t0 = (a + kIrrTile - 1) / kIrrTile;
                t1 = (b + kIrrTile - 1) / kIrrTile;
                // a segment crossing tiles is assembled by atomic combines
                if constexpr (RED)
                    if (a / kIrrTile != (b - 1) / kIrrTile) out[i] = identity<OP, T>();
            }
        }
        const bool longseg = t1 - t0 > 2;
        if (!longseg)
            for (int64_t t = t0; t < t1; ++t) tile_seg[t] = i;
        unsigned ball = __ballot_sync(0xffffffffu, longseg);
        while (ball) {  // the warp writes each long segment's tiles together
            const int src = __ffs(ball) - 1;
            ball &= ball - 1;
            const int64_t s0 = __shfl_sync(0xffffffffu, t0, src), s1 = __shfl_sync(0xffffffffu, t1, src);
            for (int64_t t = s0 + lane; t < s1; t += 32) tile_seg[t] = b0 + src;
        }
    }
}

// CTA-wide exclusive scan of (flag, value) thread pieces under the segmented
// operator (f1,v1).(f2,v2) = (f1|f2, f2 ? v2 : v1 (+) v2).
template <typename T, int OP>
__device__ __forceinline__ void irr_cta_seg_scan(uint32_t fl, T v, uint32_t& exf, T& exv, uint32_t& aggf, T& aggv,
                                                 T* s_v, uint32_t* s_f) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const T ov = __shfl_up_sync(0xffffffffu, v, o);
        const uint32_t of = __shfl_up_sync(0xffffffffu, fl, o);
        if (lane >= o) {
            if (!fl) v = combine<OP>(ov, v);
            fl |= of;
        }
    }
    if (lane == 31) {
        s_v[w] = v;
        s_f[w] = fl;
    }
    exv = __shfl_up_sync(0xffffffffu, v, 1);
    exf = __shfl_up_sync(0xffffffffu, fl, 1);
    if (lane == 0) {
        exv = identity<OP, T>();
        exf = 0;
    }
    __syncthreads();
    T pw = identity<OP, T>();
    uint32_t pf = 0;
    aggv = identity<OP, T>();
    aggf = 0;
#pragma unroll
    for (int k = 0; k < kIrrThreads / 32; ++k) {
        const T wv = s_v[k];
        const uint32_t wf = s_f[k];
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

// Shared state of one tile: its segment range and the staged offsets.
struct IrrTile {
    int64_t base, s_lo, s_hi;
    int cnt;
    bool staged;
};

// largest i in [lo, hi] with off[i] <= e (off[lo] <= e holds)
__device__ __forceinline__ int64_t seg_search(const int64_t* o, int64_t lo, int64_t hi, int64_t e) {
    while (lo < hi) {
        const int64_t mid = (lo + hi + 1) >> 1;
        if (o[mid] <= e) lo = mid;
        else hi = mid - 1;
    }
    return lo;
}

// *addr = *addr (+) v, atomically: the pieces of a segment that crosses tiles
// are combined into its output in any order (every builtin (+) is associative
// and commutative; f32 sums may differ from run to run only by association,
// within the parity bound).
template <int OP, typename T>
__device__ __forceinline__ void atomic_combine(T* addr, T v) {
    if constexpr (std::is_same<T, int>::value) {
        if constexpr (OP == OP_SUM) { atomicAdd(addr, v); return; }
        if constexpr (OP == OP_MIN) { atomicMin(addr, v); return; }
        if constexpr (OP == OP_MAX) { atomicMax(addr, v); return; }
        if constexpr (OP == OP_AND) { atomicAnd(addr, v); return; }
        if constexpr (OP == OP_OR) { atomicOr(addr, v); return; }
        if constexpr (OP == OP_XOR) { atomicXor(addr, v); return; }
    } else {
        if constexpr (OP == OP_SUM) { atomicAdd(addr, v); return; }
    }
    // PROD (both types), f32 MIN / MAX: compare-and-swap on the bit pattern
    unsigned* a = reinterpret_cast<unsigned*>(addr);
    unsigned old = *a, assumed;
    do {
        assumed = old;
        const T cur = from_bits<T>(assumed);
        old = atomicCAS(a, assumed, to_bits<T>(combine<OP>(cur, v)));
    } while (old != assumed);
}

// Load the thread's 16 items of tile `tile` (identity past the end).
template <typename T, int OP>
__device__ __forceinline__ int irr_load(const T* __restrict__ in, int64_t total, int64_t tile, bool vec,
                                        T (&v)[kIrrItems]) {
    const int64_t e0 = tile * kIrrTile + (int64_t)threadIdx.x * kIrrItems;
    const int nval = (int)max((int64_t)0, min((int64_t)kIrrItems, total - e0));
    if (vec && nval == kIrrItems) {
#pragma unroll
        for (int c = 0; c < kIrrItems / 4; ++c) {
            T e[4];
            unpack4<T>(ldg_stream4(in + e0 + 4 * c), e);
#pragma unroll
            for (int q = 0; q < 4; ++q) v[4 * c + q] = e[q];
        }
    } else {
#pragma unroll
        for (int k = 0; k < kIrrItems; ++k) v[k] = k < nval ? __ldg(in + e0 + k) : identity<OP, T>();
    }
    return nval;
}

// One tile.  MODE 0: segred pass 1 (complete segments -> out, head / tail /
// flags); MODE 1: segscan pass 1 (tail / flags); MODE 2: segscan pass 3
// (rescan with the tile's carry, write out).
template <typename T, int OP, int F, int MODE>
__device__ __forceinline__ void irr_tile(int64_t tile, int64_t Tn, T (&v)[kIrrItems], int nval, T* __restrict__ out,
                                         const int64_t* __restrict__ off, int64_t n, int64_t total, T d,
                                         const int64_t* __restrict__ tile_seg, T* __restrict__ head,
                                         T* __restrict__ tail, uint32_t* __restrict__ tflag,
                                         const T* __restrict__ cin, bool vec, int64_t* s_off, T* s_v, uint32_t* s_f) {
    const int t = threadIdx.x;
    const int64_t base = tile * kIrrTile;
    const int cnt = (int)(total - base < kIrrTile ? total - base : kIrrTile);
    const int64_t e0 = base + (int64_t)t * kIrrItems;
    const int64_t s_lo = tile_seg[tile];
    const int64_t s_hi = tile + 1 < Tn ? tile_seg[tile + 1] : n - 1;
    const int64_t nseg = s_hi - s_lo + 2;  // offsets off[s_lo .. s_hi + 1]
    const bool staged = nseg <= kIrrSmemOff;
    __syncthreads();  // s_off / s_v of the previous tile are no longer read
    if (staged)
        for (int64_t k = threadIdx.x; k < nseg; k += kIrrThreads) s_off[k] = off[s_lo + k];
    __syncthreads();
    auto O = [&](int64_t i) -> int64_t { return staged ? s_off[i - s_lo] : off[i]; };
    // segment of the first item; the walk skips empty segments
    int64_t seg = s_lo, cur_start = 0, nxt = 0;
    if (nval > 0) {
        seg = staged ? s_lo + seg_search(s_off, 0, s_hi - s_lo, e0) : seg_search(off, s_lo, s_hi, e0);
        cur_start = O(seg);
        nxt = O(seg + 1);
    }
    bool has_start = false, stash = false;
    int first_start = kIrrItems;  // item index of the thread's first segment start
    int64_t stash_seg = -1;
    T acc = identity<OP, T>(), stash_v = identity<OP, T>();
    if (nval > 0 && e0 + nval <= nxt) {
        // fast path (long segments): every item lies in segment seg; at most
        // the first item starts it and at most the last one ends it
        const bool st = e0 == cur_start;
        if constexpr (MODE == 2) {
            T r = st ? d : identity<OP, T>();
#pragma unroll
            for (int k = 0; k < kIrrItems; ++k)
                if (k < nval) v[k] = r = combine<OP>(r, apply_map<F>(v[k]));
            acc = r;
        } else {
            T a4[4] = {identity<OP, T>(), identity<OP, T>(), identity<OP, T>(), identity<OP, T>()};
#pragma unroll
            for (int k = 0; k < kIrrItems; ++k)
                if (k < nval) a4[k & 3] = combine<OP>(a4[k & 3], apply_map<F>(v[k]));
            acc = combine<OP>(combine<OP>(a4[0], a4[1]), combine<OP>(a4[2], a4[3]));
            if (st) acc = combine<OP>(d, acc);
        }
        has_start = st;
        first_start = st ? 0 : kIrrItems;
        if (e0 + nval == nxt) {
            if (!st) {
                stash = true;
                stash_v = acc;
                stash_seg = seg;
            } else if constexpr (MODE == 0) {
                out[seg] = acc;
            }
        }
    } else
#pragma unroll
    for (int k = 0; k < kIrrItems; ++k) {
        if (k < nval) {
            const int64_t e = e0 + k;
            while (e >= nxt) {  // next non-empty segment
                ++seg;
                cur_start = nxt;
                nxt = O(seg + 1);
            }
            const T x = apply_map<F>(v[k]);
            if (e == cur_start) {
                acc = combine<OP>(d, x);
                if (!has_start) first_start = k;
                has_start = true;
            } else {
                acc = combine<OP>(acc, x);
            }
            if constexpr (MODE == 2) v[k] = acc;
            if (e + 1 == nxt) {  // item ends segment seg
                if (!has_start) {  // started before this thread
                    stash = true;
                    stash_v = acc;
                    stash_seg = seg;
                } else if constexpr (MODE == 0) {
                    out[seg] = acc;
                }
            }
        }
    }
    uint32_t exf, aggf;
    T exv, aggv;
    irr_cta_seg_scan<T, OP>(has_start ? 1u : 0u, acc, exf, exv, aggf, aggv, s_v, s_f);
    if constexpr (MODE == 0) {
        if (stash) {
            const T val = combine<OP>(exv, stash_v);
            if (exf) out[stash_seg] = val;                  // started earlier in this tile: complete
            else atomic_combine<OP>(out + stash_seg, val);  // the head piece of a crossing segment
        }
        if (t == 0) {
            // the open piece at the tile's end (from its last start, with d, or
            // the whole tile) belongs to a segment that continues past the tile
            const int64_t e_last = base + cnt - 1;
            const int64_t sl = staged ? s_lo + seg_search(s_off, 0, s_hi - s_lo, e_last) : seg_search(off, s_lo, s_hi, e_last);
            if (O(sl + 1) > e_last + 1) atomic_combine<OP>(out + sl, aggv);
        }
    } else if constexpr (MODE == 1) {
        if (t == 0) {
            tail[tile] = aggv;
            tflag[tile] = aggf ? 1u : 0u;
        }
    } else {
        // carry for the items before the thread's first start
        const T pre = exf ? exv : combine<OP>(cin[tile], exv);
#pragma unroll
        for (int k = 0; k < kIrrItems; ++k)
            if (k < first_start && k < nval) v[k] = combine<OP>(pre, v[k]);
        if (vec && nval == kIrrItems) {
#pragma unroll
            for (int c = 0; c < kIrrItems / 4; ++c) {
                typename Vec4<T>::type q;
                q.x = v[4 * c]; q.y = v[4 * c + 1]; q.z = v[4 * c + 2]; q.w = v[4 * c + 3];
                __stcs(reinterpret_cast<typename Vec4<T>::type*>(out + e0 + 4 * c), q);
            }
        } else {
#pragma unroll
            for (int k = 0; k < kIrrItems; ++k)
                if (k < nval) out[e0 + k] = v[k];
        }
    }
}

// kIrrTPB consecutive tiles per CTA; the next tile's items are loaded while
// the current one is processed.
constexpr int kIrrTPB = 1;

template <typename T, int OP, int F, int MODE>
__global__ void __launch_bounds__(kIrrThreads) irr_flat_kernel(const T* __restrict__ in, T* __restrict__ out,
                                                               const int64_t* __restrict__ off, int64_t n,
                                                               int64_t total, T d,
                                                               const int64_t* __restrict__ tile_seg,
                                                               T* __restrict__ head, T* __restrict__ tail,
                                                               uint32_t* __restrict__ tflag, const T* __restrict__ cin,
                                                               bool vec) {
    __shared__ int64_t s_off[kIrrSmemOff];
    __shared__ T s_v[kIrrThreads / 32];
    __shared__ uint32_t s_f[kIrrThreads / 32];
    const int64_t Tn = (total + kIrrTile - 1) / kIrrTile;
    const int64_t t0 = (int64_t)blockIdx.x * kIrrTPB;
    T v[kIrrItems], vn[kIrrItems];
    int nval = irr_load<T, OP>(in, total, t0, vec, v);
#pragma unroll
    for (int r = 0; r < kIrrTPB; ++r) {
        const int64_t tile = t0 + r;
        if (tile >= Tn) break;
        int nn = 0;
        if (r + 1 < kIrrTPB && tile + 1 < Tn) nn = irr_load<T, OP>(in, total, tile + 1, vec, vn);
        irr_tile<T, OP, F, MODE>(tile, Tn, v, nval, out, off, n, total, d, tile_seg, head, tail, tflag, cin, vec, s_off,
                                 s_v, s_f);
#pragma unroll
        for (int k = 0; k < kIrrItems; ++k) v[k] = vn[k];
        nval = nn;
    }
}

// pass 2: exclusive segmented scan over the tile tails, one CTA (chunks of
// 1024 x 8 tiles, loads in flight): cin[t] = the open segment's value
// entering tile t (from its start, with d).
template <typename T, int OP>
__global__ void __launch_bounds__(1024) irr_tile_scan_kernel(const T* __restrict__ tail,
                                                             const uint32_t* __restrict__ tflag, T* __restrict__ cin,
                                                             int64_t Tn) {
    __shared__ T s_v[32];
    __shared__ uint32_t s_f[32];
    constexpr int PT = 8;
    const int t = threadIdx.x, lane = t & 31, w = t >> 5;
    T carry = identity<OP, T>();
    for (int64_t c0 = 0; c0 < Tn; c0 += 1024 * PT) {
        const int64_t k0 = c0 + (int64_t)t * PT;
        T tv[PT];
        uint32_t tf[PT];
#pragma unroll
        for (int q = 0; q < PT; ++q) {
            const bool ok = k0 + q < Tn;
            tv[q] = ok ? tail[k0 + q] : identity<OP, T>();
            tf[q] = ok ? (tflag[k0 + q] & 1u) : 0u;
        }
        uint32_t f = 0;
        T v = identity<OP, T>();
#pragma unroll
        for (int q = 0; q < PT; ++q) {
            v = tf[q] ? tv[q] : combine<OP>(v, tv[q]);
            f |= tf[q];
        }
        uint32_t fl = f;
        T inc = v;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const T ov = __shfl_up_sync(0xffffffffu, inc, o);
            const uint32_t of = __shfl_up_sync(0xffffffffu, fl, o);
            if (lane >= o) {
                if (!fl) inc = combine<OP>(ov, inc);
                fl |= of;
            }
        }
        if (lane == 31) {
            s_v[w] = inc;
            s_f[w] = fl;
        }
        T ex = __shfl_up_sync(0xffffffffu, inc, 1);
        uint32_t exf = __shfl_up_sync(0xffffffffu, fl, 1);
        if (lane == 0) {
            ex = identity<OP, T>();
            exf = 0;
        }
        __syncthreads();
        T pw = carry, cv = carry;  // prefix of the warps before w / of the whole chunk, from the carry
        for (int k = 0; k < 32; ++k) {
            if (k < w) pw = s_f[k] ? s_v[k] : combine<OP>(pw, s_v[k]);
            cv = s_f[k] ? s_v[k] : combine<OP>(cv, s_v[k]);
        }
        T run = exf ? ex : combine<OP>(pw, ex);
#pragma unroll
        for (int q = 0; q < PT; ++q) {
            if (k0 + q < Tn) cin[k0 + q] = run;
            run = tf[q] ? tv[q] : combine<OP>(run, tv[q]);
        }
        carry = cv;
        __syncthreads();
    }
}

}  // namespace

int64_t irr_tiles(int64_t total) { return ceil_div(total, kIrrTile); }

// [tile_seg: 8 B][head: 4 B][tail: 4 B][cin: 4 B][tflag: 4 B] per tile
size_t irr_ws_bytes(int64_t total, int version) {
    if (version != IFL_V_FLAT && version != IFL_AUTO) return 0;
    const int64_t Tn = irr_tiles(total);
    return (size_t)Tn * 24 + 64;
}

cudaError_t launch_irr(const IrrArgs& a, bool scan, int version) {
    return dispatch_all(a.dt, a.op, a.f, [&](auto tt, auto opc, auto fc) -> cudaError_t {
        using T = decltype(tt);
        constexpr int OP = decltype(opc)::value, F = decltype(fc)::value;
        const T d = bits_to<T>(a.ne_bits);
        const T* in = (const T*)a.in;
        T* out = (T*)a.out;
        if (version == IFL_V_TOP || version == IFL_V_MIDDLE) {
            const int64_t threads = version == IFL_V_TOP ? a.n : a.n * 32;
            const unsigned grid = (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(threads, 256), 148 * 32));
            if (version == IFL_V_TOP) {
                if (scan) irr_top_kernel<T, OP, F, true><<<grid, 256, 0, a.stream>>>(in, out, a.off, a.n, d);
                else irr_top_kernel<T, OP, F, false><<<grid, 256, 0, a.stream>>>(in, out, a.off, a.n, d);
            } else {
                if (scan) irr_mid_kernel<T, OP, F, true><<<grid, 256, 0, a.stream>>>(in, out, a.off, a.n, d);
                else irr_mid_kernel<T, OP, F, false><<<grid, 256, 0, a.stream>>>(in, out, a.off, a.n, d);
            }
            return cudaGetLastError();
        }
        const int64_t Tn = irr_tiles(a.total);
        int64_t* tile_seg = (int64_t*)a.ws;
        T* head = (T*)(tile_seg + Tn);
        T* tail = head + Tn;
        T* cin = tail + Tn;
        uint32_t* tflag = (uint32_t*)(cin + Tn);
        cudaError_t e;
        const unsigned gs = (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(a.n, 256), 148 * 16));
        if (scan) irr_claim_kernel<T, OP, false><<<gs, 256, 0, a.stream>>>(a.off, a.n, tile_seg, out, d);
        else irr_claim_kernel<T, OP, true><<<gs, 256, 0, a.stream>>>(a.off, a.n, tile_seg, out, d);
        if ((e = cudaGetLastError()) != cudaSuccess) return e;
        const bool vec = ((uintptr_t)a.in % 16 == 0) && ((uintptr_t)a.out % 16 == 0);
        if (Tn > 0x7fffffffLL) return cudaErrorInvalidValue;
        if (scan)
            irr_flat_kernel<T, OP, F, 1><<<(unsigned)ceil_div(Tn, kIrrTPB), kIrrThreads, 0, a.stream>>>(
                in, out, a.off, a.n, a.total, d, tile_seg, head, tail, tflag, cin, vec);
        else
            irr_flat_kernel<T, OP, F, 0><<<(unsigned)ceil_div(Tn, kIrrTPB), kIrrThreads, 0, a.stream>>>(
                in, out, a.off, a.n, a.total, d, tile_seg, head, tail, tflag, cin, vec);
        if (!scan) return cudaGetLastError();  // crossing segments were combined atomically
        irr_tile_scan_kernel<T, OP><<<1, 1024, 0, a.stream>>>(tail, tflag, cin, Tn);
        if ((e = cudaGetLastError()) != cudaSuccess) return e;
        irr_flat_kernel<T, OP, F, 2><<<(unsigned)ceil_div(Tn, kIrrTPB), kIrrThreads, 0, a.stream>>>(
            in, out, a.off, a.n, a.total, d, tile_seg, head, tail, tflag, cin, vec);
        return cudaGetLastError();
    });
}

// Inspector: total, longest segment, validity of the descriptor.
__global__ void __launch_bounds__(256) irr_inspect_kernel(const int64_t* __restrict__ off, int64_t n,
                                                          unsigned long long* __restrict__ res) {
    int64_t mx = 0;
    bool bad = false;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t L = off[i + 1] - off[i];
        bad |= L < 0;
        mx = max(mx, L);
    }
    for (int o = 16; o > 0; o >>= 1) mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
    const unsigned ball = __ballot_sync(0xffffffffu, bad);
    if ((threadIdx.x & 31) == 0) {
        atomicMax(&res[0], (unsigned long long)mx);
        if (ball) atomicOr(&res[1], 1ull);
    }
    if (blockIdx.x == 0 && threadIdx.x == 0 && off[0] != 0) atomicOr(&res[1], 2ull);
}

cudaError_t launch_irr_inspect(const int64_t* off, int64_t n, void* res, cudaStream_t s) {
    cudaError_t e = cudaMemsetAsync(res, 0, 16, s);
    if (e != cudaSuccess) return e;
    const unsigned g = (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, 256), 148 * 16));
    irr_inspect_kernel<<<g, 256, 0, s>>>(off, n, (unsigned long long*)res);
    return cudaGetLastError();
}

}  // namespace ifl
