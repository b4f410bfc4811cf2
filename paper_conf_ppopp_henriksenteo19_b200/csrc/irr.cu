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
//   V_FLAT    flattened over segments and elements together (merge path:
//             tiles of 4096 merge items, see below).
#include <algorithm>

#include "common.cuh"
#include "dispatch.cuh"
#include "ifl_internal.h"

namespace ifl {

namespace {

constexpr int kIrrThreads = 256;
constexpr int kIrrItems = 16;
constexpr int64_t kIrrTile = (int64_t)kIrrThreads * kIrrItems;

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
// Merge-path decomposition (B200 design; the paper only names irregular
// nesting as future work): the n segment ends off[1..n] and the
// `total` element indices 0..total-1 are merged into one sequence of n + total
// items (an end off[i+1] comes before element j when off[i+1] <= j), and every
// tile takes kIrrTile consecutive merge items.  Every tile thus holds the same
// amount of work whatever the length mix -- empty segments, a mean of one
// element, or one segment of 12M elements.
//   partition  the (segment, element) coordinates of every tile start
//              (8 lanes per tile, 8-ary search over off);
//   segred     pass 1 (persistent CTAs, 3 per SM): the next tile's segment
//              ends and elements are copied into shared memory with cp.async
//              while the current one is walked -- each thread walks 16
//              consecutive items branch-free, a CTA-wide segmented scan of
//              the thread pieces gives each thread's carry, complete segments
//              are staged in place of their ends and stored coalesced; the
//              tile records its head piece (its first segment, when that began
//              in an earlier tile) and its open tail (flag: a segment starts
//              in the tile);
//              pass 2: segmented scan of the tile tails in two parallel
//              kernels (chunk aggregates; chunk scans seeded by the preceding
//              aggregates) that complete the head pieces, out[i] = carry (+)
//              head;
//   segscan    pass 1: per tile (a warp each), the reduce of its open tail
//              only (elements after the tile's last segment start: short
//              segments read almost nothing); pass 2: the segmented scan of
//              the tails (cin); pass 3: the merge walk again with the tile's
//              carry, the scanned elements staged in place and stored
//              coalesced (two reads + one write per element when segments are
//              long; one read + one write when they are short).

// Shared-memory staging (int32 ends relative to the tile's first element,
// elements), padded by one word per 32 so the thread-blocked walk (lanes ~16
// items apart) is bank-conflict-free.
constexpr int kMpSmem = (int)kIrrTile + (int)kIrrTile / 32 + 1;  // pd(kIrrTile) + 1
constexpr int kMpThreads = 128, kMpItems = 32, kMpItemsLog2 = 5;
static_assert(kMpThreads * kMpItems == kIrrTile && (1 << kMpItemsLog2) == kMpItems, "merge-path tile");
__device__ __forceinline__ int pd(int k) { return k + (k >> 5); }

__device__ __forceinline__ void mp_cp_async4(void* smem, const void* gmem) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_u32(smem)), "l"(gmem) : "memory");
}

// CTA-wide exclusive scan of (flag, value) thread pieces under the segmented
// operator (f1,v1).(f2,v2) = (f1|f2, f2 ? v2 : v1 (+) v2), seeded with an
// initial piece (init_f, init_v): exf/exv = everything before the thread,
// aggf/aggv = the whole CTA.  NT threads.
template <typename T, int OP, int NT>
__device__ __forceinline__ void irr_cta_seg_scan(uint32_t fl, T v, uint32_t init_f, T init_v, uint32_t& exf, T& exv,
                                                 uint32_t& aggf, T& aggv, T* s_v, uint32_t* s_f) {
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
    T pw = init_v;  // the initial piece, then the warps before w
    uint32_t pf = init_f;
    aggv = init_v;
    aggf = init_f;
#pragma unroll
    for (int k = 0; k < NT / 32; ++k) {
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

// partition: coord[b] = the number of segment ends among the first
// min(b*T, n+total) merge items.  P(i) = off[i+1] + i + 1 <= D is monotone
// (true then false): 8 lanes probe 8 evenly spaced i per round.  A CTA owns 32
// consecutive tile starts: two 8-lane groups first find the coordinates of
// its first and last start over the whole descriptor, then every start is
// searched only between them (a window of <= 32 tiles: fewer rounds, and the
// probes of one CTA share sectors in L2 instead of 32 random DRAM walks).
__device__ __forceinline__ int64_t mp_search8(const int64_t* __restrict__ off, int64_t D, int64_t lo, int64_t hi,
                                              bool live) {
    const int lane = threadIdx.x & 31, sub = lane & 7;
    const unsigned gmask = 0xffu << (lane & 24);
    if (!live) lo = hi;
    while (__any_sync(0xffffffffu, lo < hi)) {  // uniform trip count: the ballots need every lane
        const int64_t step = (hi - lo + 7) / 8;
        const int64_t p = lo + step * sub;
        const bool pr = lo < hi && p < hi && __ldg(off + p + 1) + p + 1 <= D;
        const int c = __popc(__ballot_sync(0xffffffffu, pr) & gmask);  // true probes: sub-lanes 0..c-1
        if (lo < hi) {
            if (c == 0) {
                hi = lo;  // P(lo) is false: the split is lo
            } else {
                hi = min(lo + step * c, hi);
                lo = lo + step * (c - 1) + 1;
            }
        }
    }
    return lo;
}

constexpr int kPartPerCta = 32;  // tile starts per CTA (8 lanes each: 256 threads)

__global__ void __launch_bounds__(256) irr_mp_partition_kernel(const int64_t* __restrict__ off, int64_t n,
                                                               int64_t total, int64_t Tn, int64_t* __restrict__ coord) {
    __shared__ int64_t s_bound[2];
    const int t = threadIdx.x, sub = t & 7, grp = t >> 3;
    const int64_t W = n + total;
    const int64_t b0 = (int64_t)blockIdx.x * kPartPerCta;
    const int64_t bl = min(b0 + kPartPerCta, Tn);  // the CTA's starts are b0 .. bl (bl inclusive)
    if (t < 32) {  // warp 0: groups 0 / 1 find the bounds (b0, bl) over the whole descriptor
        const int64_t bb = grp == 0 ? b0 : bl;
        const int64_t D = min(bb * kIrrTile, W);
        const int64_t r = mp_search8(off, D, max((int64_t)0, D - total), min(D, n), grp < 2);
        if (sub == 0 && grp < 2) s_bound[grp] = r;
    }
    __syncthreads();
    const int64_t b = b0 + grp;
    const bool live = b <= bl && b <= Tn;
    const int64_t D = live ? min(b * kIrrTile, W) : 0;
    const int64_t lo = max(s_bound[0], D - total), hi = min(s_bound[1], min(D, n));
    const int64_t r = mp_search8(off, D, lo, max(lo, hi), live);
    if (live && sub == 0) coord[b] = r;
}

// Elements-only segred tiles (no segment end: the tile lies inside one
// segment): a plain CTA reduction, float4 loads striped across the CTA from
// the tile's 16-byte-aligned base (no shared-memory staging).
template <typename T, int OP, int F>
__device__ __forceinline__ void mp_elems_red(const T* __restrict__ in, int64_t j0, uint32_t start_f, T init_v,
                                             int64_t b, T* __restrict__ tail, uint32_t* __restrict__ tflag, T* s_v,
                                             uint32_t* s_f) {
    const int t = threadIdx.x, R = (int)(j0 & 3);
    const T* base = in + (j0 - R);  // group g = elements [4g, 4g + 4) of base; the tile is [R, R + kIrrTile)
    T acc[4] = {identity<OP, T>(), identity<OP, T>(), identity<OP, T>(), identity<OP, T>()};
    constexpr int NG = (int)kIrrTile / 4 / kMpThreads;
    typename Vec4<T>::type u[NG];
#pragma unroll
    for (int q = 0; q < NG; ++q) u[q] = ldg_stream4(base + 4 * (t + kMpThreads * q));
#pragma unroll
    for (int q = 0; q < NG; ++q) {
        T e[4];
        unpack4<T>(u[q], e);
#pragma unroll
        for (int c = 0; c < 4; ++c) {
            const T m = apply_map<F>(e[c]);
            acc[c] = (q == 0 && t == 0 && c < R) ? acc[c] : combine<OP>(acc[c], m);
        }
    }
    if (R != 0 && t == 0) {  // the tile's last R elements: group kIrrTile / 4
        T e[4];
        unpack4<T>(ldg_stream4(base + kIrrTile), e);
#pragma unroll
        for (int c = 0; c < 4; ++c)
            if (c < R) acc[c] = combine<OP>(acc[c], apply_map<F>(e[c]));
    }
    uint32_t exf, aggf;
    T exv, aggv;
    irr_cta_seg_scan<T, OP, kMpThreads>(0u, combine<OP>(combine<OP>(acc[0], acc[1]), combine<OP>(acc[2], acc[3])),
                                        start_f, init_v, exf, exv, aggf, aggv, s_v, s_f);
    if (t == kMpThreads - 1) {
        tail[b] = aggv;
        tflag[b] = aggf;
    }
}

// Pass 1 of segred (SCAN = false) / pass 3 of segscan (SCAN = true), a tile
// per CTA of 128 threads x 32 items (twelve CTAs per SM).  The tile's ends
// (int32, relative to its first element) and elements share one padded
// shared-memory array: ends at [0, ns), elements at [ns, ns + ne).
// segscan: in may equal out (a tile reads and writes only its own elements;
// coherent loads).  Pass A scans only the elements after a thread's first
// segment start; pass B scans the thread's lead elements from its carry.
template <typename T, int OP, int F, bool SCAN>
__global__ void __launch_bounds__(kMpThreads) irr_mp_kernel(const T* in, T* out, const int64_t* __restrict__ off,
                                                            int64_t n, int64_t total, T d,
                                                            const int64_t* __restrict__ coord, T* __restrict__ tail,
                                                            uint32_t* __restrict__ tflag, T* __restrict__ head,
                                                            const T* __restrict__ cin, bool vec) {
    __shared__ int s_b[kMpSmem];  // ends (segred: then segment values), then elements (bit patterns)
    __shared__ T s_v[kMpThreads / 32];
    __shared__ uint32_t s_f[kMpThreads / 32];
    __shared__ int s_start[kMpThreads];
    __shared__ int s_skip0;
    const int t = threadIdx.x;
    const int64_t b = blockIdx.x;
    const int64_t D0 = b * kIrrTile, D1 = min(D0 + kIrrTile, n + total);
    const int64_t i0 = coord[b], i1 = coord[b + 1];
    const int64_t j0 = D0 - i0;
    const int ns = (int)(i1 - i0), ne = (int)((D1 - i1) - j0);
    const uint32_t start_f = __ldg(off + i0) >= j0 ? 1u : 0u;
    T init_v = start_f ? d : identity<OP, T>();
    if constexpr (SCAN) {
        if (!start_f) init_v = cin[b];
    } else {
        if (ns == 0 && ne == (int)kIrrTile && vec && (j0 & ~(int64_t)3) + kIrrTile + 4 <= total) {
            mp_elems_red<T, OP, F>(in, j0, start_f, init_v, b, tail, tflag, s_v, s_f);
            return;
        }
    }
    auto X = [&](int j) -> int& { return s_b[pd(ns + j)]; };
    // ---- staging.  Elements: asynchronous 4-byte copies, all in flight at
    // once without registers (a register-staged loop keeps ~8 loads per
    // thread in flight: four DRAM round trips per tile), issued first so the
    // ends' loads overlap them
#pragma unroll 8
    for (int k = t; k < ne; k += kMpThreads) mp_cp_async4(&X(k), in + j0 + k);
    asm volatile("cp.async.commit_group;" ::: "memory");
#pragma unroll 4
    for (int k = t; k < ns; k += kMpThreads) s_b[pd(k)] = (int)(__ldg(off + i0 + 1 + k) - j0);
    asm volatile("cp.async.wait_group 0;" ::: "memory");
    if (t == 0) s_skip0 = 0;
    __syncthreads();
    const int Wt = ns + ne;
    const int d0 = min(t * kMpItems, Wt), cnt = min(d0 + kMpItems, Wt) - d0;
    // thread starts without a search: end k sits at merge position
    // pos(k) = k + s_b[k] (strictly increasing), so the thread whose first
    // item is 32u (pos(k-1) < 32u <= pos(k)) starts at end k; threads past
    // the last end start at ns
    for (int k = t; k < ns; k += kMpThreads) {
        const int pk = k + s_b[pd(k)];
        const int pp = k == 0 ? -1 : (k - 1) + s_b[pd(k - 1)];
        for (int u = (pp >> kMpItemsLog2) + 1; u * kMpItems <= pk; ++u) s_start[u] = k;  // pp >= -1: floor
    }
    if (t * kMpItems > (ns == 0 ? -1 : (ns - 1) + s_b[pd(ns - 1)])) s_start[t] = ns;
    __syncthreads();  // (segred: also every read of the ends is done before segment values overwrite them)
    int i = s_start[t];
    const int ie = t + 1 < kMpThreads ? s_start[t + 1] : ns;
    const int j_s = d0 - i;
    T acc = identity<OP, T>();
    int first = -1;  // segred: the thread's first segment end
    int lead = 0;    // segscan: elements before the thread's first segment start
    if (ns * 32 > ne) {
        // ends-dense tiles (segments shorter than ~32): branch-free walk
        // (selects and predicated shared stores)
        int j = j_s;
        bool seen = false;
        int ce = i < ie ? s_b[pd(i)] : 0x7fffffff;
#pragma unroll
        for (int k = 0; k < kMpItems; ++k) {
            const bool valid = k < cnt;
            const bool end = valid && ce <= j;
            const bool elt = valid && !end;
            const T nacc = combine<OP>(acc, apply_map<F>(from_bits<T>((uint32_t)X(j))));  // j <= ne: inside
            if constexpr (SCAN) {
                if (elt && seen) X(j) = (int)to_bits<T>(nacc);  // lead elements are scanned in pass B
            } else {
                if (end) s_b[pd(i)] = (int)to_bits<T>(acc);
                first = (end && first < 0) ? i : first;
            }
            seen = seen || end;
            lead += (elt && !seen) ? 1 : 0;
            i += end ? 1 : 0;
            const int nc = s_b[pd(i)];  // read only when i < ie
            ce = end ? (i < ie ? nc : 0x7fffffff) : ce;
            acc = end ? d : (elt ? nacc : acc);
            j += elt ? 1 : 0;
        }
        if constexpr (SCAN) first = seen ? 0 : -1;
    } else
    {
        // element-dense tiles: the walk as runs of elements between segment
        // ends (a thread inside one segment is one run; divergent lanes cost
        // the longest run, not both paths)
        int j = j_s, rem = cnt;
        bool seen = false;
        while (rem > 0) {
            const int ce = i < ie ? s_b[pd(i)] : 0x7fffffff;
            const int run = min(ce - j, rem);  // elements before the next end
            if (SCAN && seen) {
#pragma unroll 4
                for (int q = 0; q < run; ++q) {
                    acc = combine<OP>(acc, apply_map<F>(from_bits<T>((uint32_t)X(j + q))));
                    X(j + q) = (int)to_bits<T>(acc);
                }
            } else {  // segred, or segscan's lead elements (scanned in pass B)
#pragma unroll 4
                for (int q = 0; q < run; ++q) acc = combine<OP>(acc, apply_map<F>(from_bits<T>((uint32_t)X(j + q))));
            }
            if (!seen) lead += run;
            j += run;
            rem -= run;
            if (rem > 0) {  // the end of segment i0 + i
                if constexpr (!SCAN) {
                    s_b[pd(i)] = (int)to_bits<T>(acc);
                    if (first < 0) first = i;
                }
                seen = true;
                acc = d;
                ++i;
                --rem;
            }
        }
        if constexpr (SCAN) first = seen ? 0 : -1;
    }
    uint32_t exf, aggf;
    T exv, aggv;
    irr_cta_seg_scan<T, OP, kMpThreads>(first >= 0 ? 1u : 0u, acc, start_f, init_v, exf, exv, aggf, aggv, s_v, s_f);
    if constexpr (SCAN) {
        // pass B: the elements before the thread's first segment start, scanned
        // from the thread's carry (pass A only reduced them)
        T a2 = exv;
        if (lead == kMpItems) {
#pragma unroll
            for (int k = 0; k < kMpItems; ++k) {
                a2 = combine<OP>(a2, apply_map<F>(from_bits<T>((uint32_t)X(j_s + k))));
                X(j_s + k) = (int)to_bits<T>(a2);
            }
        } else {
            for (int k = 0; k < lead; ++k) {
                a2 = combine<OP>(a2, apply_map<F>(from_bits<T>((uint32_t)X(j_s + k))));
                X(j_s + k) = (int)to_bits<T>(a2);
            }
        }
        __syncthreads();
#pragma unroll 8
        for (int k = t; k < ne; k += kMpThreads) __stcs(out + j0 + k, from_bits<T>((uint32_t)X(k)));
    } else {
        if (first >= 0) {
            const T v = combine<OP>(exv, from_bits<T>((uint32_t)s_b[pd(first)]));
            if (exf) {
                s_b[pd(first)] = (int)to_bits<T>(v);
            } else {  // segment i0 began in an earlier tile: its head piece
                head[b] = v;
                s_skip0 = 1;
            }
        }
        if (t == kMpThreads - 1) tail[b] = aggv;
        __syncthreads();
        if (t == 0) tflag[b] = aggf | (s_skip0 ? 2u : 0u);
        for (int k = t + s_skip0; k < ns; k += kMpThreads) __stcs(out + i0 + k, from_bits<T>((uint32_t)s_b[pd(k)]));
    }
}

// segscan pass 1 (a warp per tile): the open tail, from the start of the
// segment open at the tile's end (off[i1], with d) or the whole tile.
template <typename T, int OP, int F>
__global__ void __launch_bounds__(256) irr_mp_tail_kernel(const T* __restrict__ in, const int64_t* __restrict__ off,
                                                          int64_t n, int64_t total, T d,
                                                          const int64_t* __restrict__ coord, T* __restrict__ tail,
                                                          uint32_t* __restrict__ tflag, int64_t Tn) {
    const int lane = threadIdx.x & 31;
    const int64_t b = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    if (b >= Tn) return;
    const int64_t D1 = min((b + 1) * kIrrTile, n + total);
    const int64_t j0 = b * kIrrTile - coord[b], i1 = coord[b + 1], j1 = D1 - i1;
    const int64_t s = __ldg(off + i1);
    const bool started = s >= j0;
    const int64_t a = started ? s : j0;
    T acc[4] = {identity<OP, T>(), identity<OP, T>(), identity<OP, T>(), identity<OP, T>()};
    int64_t k = a + lane;
    for (; k + 96 < j1; k += 128) {
        T x[4];
#pragma unroll
        for (int q = 0; q < 4; ++q) x[q] = __ldg(in + k + 32 * q);
#pragma unroll
        for (int q = 0; q < 4; ++q) acc[q] = combine<OP>(acc[q], apply_map<F>(x[q]));
    }
    for (; k < j1; k += 32) acc[0] = combine<OP>(acc[0], apply_map<F>(__ldg(in + k)));
    const T r = warp_reduce<OP>(combine<OP>(combine<OP>(acc[0], acc[1]), combine<OP>(acc[2], acc[3])));
    if (lane == 0) {
        tail[b] = started ? combine<OP>(d, r) : r;
        tflag[b] = started ? 1u : 0u;
    }
}

// Segmented scan of the tile tails in two parallel kernels over chunks of
// kTsChunk tiles.  A: each chunk's aggregate (flag, value).
constexpr int kTsChunk = 256;

template <typename T, int OP>
__global__ void __launch_bounds__(kTsChunk) irr_mp_ts_agg_kernel(const T* __restrict__ tail,
                                                                 const uint32_t* __restrict__ tflag,
                                                                 T* __restrict__ cagg, uint32_t* __restrict__ cflag,
                                                                 int64_t Tn) {
    __shared__ T s_v[kTsChunk / 32];
    __shared__ uint32_t s_f[kTsChunk / 32];
    const int64_t k = (int64_t)blockIdx.x * kTsChunk + threadIdx.x;
    const bool ok = k < Tn;
    uint32_t exf, aggf;
    T exv, aggv;
    irr_cta_seg_scan<T, OP, kTsChunk>(ok ? (tflag[k] & 1u) : 0u, ok ? tail[k] : identity<OP, T>(), 0u,
                                      identity<OP, T>(), exf, exv, aggf, aggv, s_v, s_f);
    if (threadIdx.x == 0) {
        cagg[blockIdx.x] = aggv;
        cflag[blockIdx.x] = aggf;
    }
}

// B: chunk c's prefix = the segmented fold of chunks 0..c-1, then the chunk's
// exclusive scan: cin[k] (segscan) or the head fix-ups (segred).
template <typename T, int OP, bool SEGRED>
__global__ void __launch_bounds__(kTsChunk) irr_mp_ts_scan_kernel(const T* __restrict__ tail,
                                                                  const uint32_t* __restrict__ tflag,
                                                                  const T* __restrict__ cagg,
                                                                  const uint32_t* __restrict__ cflag,
                                                                  T* __restrict__ cin, const T* __restrict__ head,
                                                                  const int64_t* __restrict__ coord,
                                                                  T* __restrict__ out, int64_t Tn) {
    __shared__ T s_v[kTsChunk / 32];
    __shared__ uint32_t s_f[kTsChunk / 32];
    const int c = blockIdx.x, t = threadIdx.x;
    // prefix over chunks [0, c): thread t folds a contiguous block of them
    const int per = (c + kTsChunk - 1) / kTsChunk;
    uint32_t pf = 0;
    T pv = identity<OP, T>();
    for (int q = 0; q < per; ++q) {
        const int k = t * per + q;
        if (k < c) {
            const uint32_t f = cflag[k];
            const T v = cagg[k];
            pv = f ? v : combine<OP>(pv, v);
            pf |= f;
        }
    }
    uint32_t exf, aggf, pref_f;
    T exv, aggv, pref_v;
    irr_cta_seg_scan<T, OP, kTsChunk>(pf, pv, 0u, identity<OP, T>(), exf, exv, pref_f, pref_v, s_v, s_f);
    __syncthreads();  // s_v / s_f reused
    const int64_t k = (int64_t)c * kTsChunk + t;
    const bool ok = k < Tn;
    const uint32_t tf = ok ? tflag[k] : 0u;
    irr_cta_seg_scan<T, OP, kTsChunk>(tf & 1u, ok ? tail[k] : identity<OP, T>(), pref_f, pref_v, exf, exv, aggf,
                                      aggv, s_v, s_f);
    if (!ok) return;
    if constexpr (SEGRED) {
        if (tf & 2u) out[coord[k]] = combine<OP>(exv, head[k]);
    } else {
        cin[k] = exv;
    }
}

}  // namespace

int64_t irr_tiles(int64_t n, int64_t total) { return ceil_div(n + total, kIrrTile); }

// [coords: 8 B x (Tn + 1)][tail|flag|head|cin: 4 B x Tn each][chunk agg|flag: 4 B x chunks each]
size_t irr_ws_bytes(int64_t n, int64_t total, int version) {
    if (version != IFL_V_FLAT && version != IFL_AUTO) return 0;
    const int64_t Tn = irr_tiles(n, total), C = ceil_div(Tn, kTsChunk);
    return (size_t)(Tn + 1) * 8 + (size_t)Tn * 16 + (size_t)C * 8 + 64;
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
        const int64_t Tn = irr_tiles(a.n, a.total);
        if (Tn == 0) return cudaSuccess;
        if (Tn > 0x7fffffffLL) return cudaErrorInvalidValue;
        const int64_t C = ceil_div(Tn, kTsChunk);
        int64_t* coord = (int64_t*)a.ws;
        T* tail = (T*)(coord + Tn + 1);
        uint32_t* tflag = (uint32_t*)(tail + Tn);
        T* head = (T*)(tflag + Tn);
        T* cin = head + Tn;
        T* cagg = cin + Tn;
        uint32_t* cflag = (uint32_t*)(cagg + C);
        const bool vec = ((uintptr_t)a.in % 16 == 0) && ((uintptr_t)a.out % 16 == 0);
        cudaError_t e;
        irr_mp_partition_kernel<<<(unsigned)ceil_div(Tn + 1, kPartPerCta), 256, 0, a.stream>>>(a.off, a.n, a.total,
                                                                                                 Tn, coord);
        if ((e = cudaGetLastError()) != cudaSuccess) return e;
        if (!scan) {
            irr_mp_kernel<T, OP, F, false><<<(unsigned)Tn, kMpThreads, 0, a.stream>>>(
                in, out, a.off, a.n, a.total, d, coord, tail, tflag, head, cin, vec);
        } else {
            irr_mp_tail_kernel<T, OP, F><<<(unsigned)ceil_div(Tn * 32, 256), 256, 0, a.stream>>>(
                in, a.off, a.n, a.total, d, coord, tail, tflag, Tn);
        }
        if ((e = cudaGetLastError()) != cudaSuccess) return e;
        irr_mp_ts_agg_kernel<T, OP><<<(unsigned)C, kTsChunk, 0, a.stream>>>(tail, tflag, cagg, cflag, Tn);
        if ((e = cudaGetLastError()) != cudaSuccess) return e;
        if (!scan) {
            irr_mp_ts_scan_kernel<T, OP, true><<<(unsigned)C, kTsChunk, 0, a.stream>>>(tail, tflag, cagg, cflag, cin,
                                                                                       head, coord, out, Tn);
            return cudaGetLastError();
        }
        irr_mp_ts_scan_kernel<T, OP, false><<<(unsigned)C, kTsChunk, 0, a.stream>>>(tail, tflag, cagg, cflag, cin,
                                                                                    head, coord, out, Tn);
        if ((e = cudaGetLastError()) != cudaSuccess) return e;
        irr_mp_kernel<T, OP, F, true><<<(unsigned)Tn, kMpThreads, 0, a.stream>>>(in, out, a.off, a.n, a.total, d,
                                                                                  coord, tail, tflag, head, cin, vec);
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
