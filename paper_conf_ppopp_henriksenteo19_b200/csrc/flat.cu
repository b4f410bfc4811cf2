// flat.cu -- V_FLAT: the fully flattened segred^1 / segscan^1 over all n*m
// elements (rule G3's e_flat; Fig 6c version 3).
//
// One single-pass kernel serves both (SCAN writes every prefix, RED writes
// only the segment ends).  The flat index space [0, n*m) is cut into tiles of
// kFlatTile = 256 x 28 elements.  Per tile (one CTA, dynamic tile id):
//   1. the TMA engine copies the contiguous tile into shared memory
//      (cp.async.bulk, completion on an mbarrier);
//   2. thread t takes 28 consecutive elements (7 conflict-free LDS.128: the
//      112-byte stride is an odd multiple of 16 B) and runs a sequential
//      segmented scan; segment starts are arithmetic (multiples of m), so no
//      flag array is read -- d is combined into every segment's first element;
//   3. the CTA scans the (flag, value) thread aggregates with the segmented
//      operator (f1,v1).(f2,v2) = (f1|f2, f2 ? v2 : v1 (+) v2);
//   4. decoupled look-back over predecessor tiles' 64-bit status words
//      (aggregate / inclusive prefix, with the segment flag) gives the carry
//      into the tile; a tile that starts with a segment start skips it;
//   5. SCAN: results go back to shared memory and the TMA engine stores the
//      tile (cp.async.bulk shared -> global); RED: each segment end writes
//      out[segment].
// The workspace header carries a dynamic tile counter, a completion counter
// and an epoch; the last CTA resets the counters and bumps the epoch, and
// status words carry the epoch as a tag, so no memset is needed per call.
#include <string.h>

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
    return sizeof(FlatHdr) + (size_t)tiles * 8;
}

// status word: [63:35] tag, [34:33] status (1 aggregate, 2 inclusive), [32] flag, [31:0] value
constexpr uint64_t ST_A = 1, ST_P = 2;
__device__ __forceinline__ uint64_t pack_status(uint32_t tag, uint64_t st, uint32_t flag, uint32_t val) {
    return ((uint64_t)tag << 35) | (st << 33) | ((uint64_t)flag << 32) | (uint64_t)val;
}

template <typename T, int OP, int F, bool SCAN>
__global__ void __launch_bounds__(FB) flat_kernel(const T* in, T* out, int64_t N, int64_t m, T d, uint8_t* ws,
                                                  int num_tiles, bool tma_in, bool tma_out) {
    __shared__ alignas(128) T buf[FT];
    __shared__ alignas(8) uint64_t mbar;
    __shared__ int s_tile;
    __shared__ uint32_t s_tag;
    __shared__ T s_wval[FB / 32];
    __shared__ uint32_t s_wflag[FB / 32];
    __shared__ T s_carry;

    FlatHdr* hdr = reinterpret_cast<FlatHdr*>(ws);
    uint64_t* status = reinterpret_cast<uint64_t*>(ws + sizeof(FlatHdr));
    const int t = threadIdx.x, lane = t & 31, w = t >> 5;

    if (t == 0) {
        s_tile = (int)atomicAdd(&hdr->tile_ctr, 1u);
        s_tag = ld_relaxed_u32(&hdr->epoch) & 0x1FFFFFFFu;
        mbar_init(&mbar, 1);
        fence_mbar_init();
    }
    __syncthreads();
    const int tile = s_tile;
    const uint32_t tag = s_tag;
    const int64_t base = (int64_t)tile * FT;
    const int cnt = (int)min((int64_t)FT, N - base);
    const bool full = (cnt == FT);

    // ---- 1. stage the tile in shared memory
    if (full && tma_in) {
        if (t == 0) {
            mbar_arrive_expect_tx(&mbar, FT * sizeof(T));
            bulk_g2s(buf, in + base, FT * sizeof(T), &mbar);
        }
        mbar_wait(&mbar, 0);
    } else {
        for (int p = t; p < cnt; p += FB) buf[p] = in[base + p];
        __syncthreads();
    }

    // ---- 2. thread-local segmented scan over FI consecutive elements
    const int o = t * FI;
    T v[FI];
    {
        using V = typename Vec4<T>::type;
#pragma unroll
        for (int c = 0; c < FI / 4; ++c) {
            V q = *reinterpret_cast<const V*>(&buf[o + 4 * c]);
            v[4 * c] = q.x; v[4 * c + 1] = q.y; v[4 * c + 2] = q.z; v[4 * c + 3] = q.w;
        }
    }
    const int nvalid = max(0, min(FI, cnt - o));
    const int64_t g0 = base + o;
    const int64_t pos = (nvalid > 0) ? (g0 % m) : 0;
    const int mi = (int)min(m, (int64_t)FI + 1);                      // step between starts (capped)
    const int nx0 = (int)min(pos == 0 ? (int64_t)0 : m - pos, (int64_t)FI + 1);  // first start in thread
    bool has_start = false;
    T acc = identity<OP, T>();
    {
        int nx = nx0;
#pragma unroll
        for (int k = 0; k < FI; ++k) {
            if (k < nvalid) {
                const T x = apply_map<F>(v[k]);
                if (k == nx) {
                    acc = combine<OP>(d, x);
                    has_start = true;
                    nx += mi;
                } else {
                    acc = combine<OP>(acc, x);
                }
                v[k] = acc;
            }
        }
    }

    // ---- 3. CTA-wide exclusive segmented scan of (has_start, acc)
    uint32_t fl = has_start ? 1u : 0u;
    T sv = acc;
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
    T exv = __shfl_up_sync(0xffffffffu, sv, 1);
    uint32_t exf = __shfl_up_sync(0xffffffffu, fl, 1);
    if (lane == 0) {
        exv = identity<OP, T>();
        exf = 0;
    }
    __syncthreads();
    // prefix of the preceding warps, and the tile aggregate
    T pw = identity<OP, T>();
    uint32_t pf = 0;
    T aggv = identity<OP, T>();
    uint32_t aggf = 0;
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
    // thread exclusive = (warp prefix) . (in-warp exclusive)
    if (!exf) exv = combine<OP>(pw, exv);
    exf |= pf;

    // ---- 4. decoupled look-back (warp 0)
    const bool tile_starts = (base % m) == 0;  // first element starts a segment
    if (w == 0) {
        T carry = identity<OP, T>();
        if (tile == 0) {
            if (lane == 0) st_release_u64(&status[0], pack_status(tag, ST_P, aggf, to_bits(aggv)));
        } else {
            if (lane == 0)
                st_release_u64(&status[tile], pack_status(tag, aggf ? ST_P : ST_A, aggf, to_bits(aggv)));
            if (!tile_starts || !aggf) {
                int pred = tile - 1;
                T run = identity<OP, T>();
                while (true) {
                    const int idx = pred - lane;
                    uint64_t word = 0;
                    if (idx >= 0) {
                        do {
                            word = ld_acquire_u64(&status[idx]);
                        } while ((uint32_t)(word >> 35) != tag || ((word >> 33) & 3u) == 0);
                    }
                    const bool term = idx < 0 || ((word >> 33) & 3u) == ST_P || ((word >> 32) & 1u);
                    const uint32_t tm = __ballot_sync(0xffffffffu, term);
                    const int stop = tm ? (__ffs(tm) - 1) : 31;
                    T val = (lane <= stop && idx >= 0) ? from_bits<T>((uint32_t)word) : identity<OP, T>();
                    // ordered reduce: lane l+k is older than lane l
#pragma unroll
                    for (int off = 1; off < 32; off <<= 1) {
                        const T older = __shfl_down_sync(0xffffffffu, val, off);
                        if (lane + off < 32) val = combine<OP>(older, val);
                    }
                    val = __shfl_sync(0xffffffffu, val, 0);
                    run = combine<OP>(val, run);
                    if (tm) break;
                    pred -= 32;
                }
                carry = run;
                if (!aggf && lane == 0)
                    st_release_u64(&status[tile], pack_status(tag, ST_P, 0u, to_bits(combine<OP>(carry, aggv))));
            }
        }
        if (lane == 0) s_carry = carry;
    }
    __syncthreads();
    const T carry_t = exf ? exv : combine<OP>(s_carry, exv);

    // ---- 5. apply the carry to the elements before the thread's first start
    {
#pragma unroll
        for (int k = 0; k < FI; ++k)
            if (k < nx0 && k < nvalid) v[k] = combine<OP>(carry_t, v[k]);
    }
    if constexpr (SCAN) {
        using V = typename Vec4<T>::type;
#pragma unroll
        for (int c = 0; c < FI / 4; ++c) {
            V q;
            q.x = v[4 * c]; q.y = v[4 * c + 1]; q.z = v[4 * c + 2]; q.w = v[4 * c + 3];
            *reinterpret_cast<V*>(&buf[o + 4 * c]) = q;
        }
        if (full && tma_out) {
            fence_proxy_async_smem();
            __syncthreads();
            if (t == 0) {
                bulk_s2g(out + base, buf, FT * sizeof(T));
                bulk_commit();
                bulk_wait_read0();
            }
        } else {
            __syncthreads();
            for (int p = t; p < cnt; p += FB) out[base + p] = buf[p];
        }
    } else {
        // segment ends: global index g with (g + 1) % m == 0
        if (nvalid > 0) {
            int64_t seg = g0 / m;
            int nx = nx0;
#pragma unroll
            for (int k = 0; k < FI; ++k) {
                if (k < nvalid) {
                    if (k == nx) {
                        nx += mi;
                    }
                    if (k + 1 == nx) {
                        // the element ends segment `seg` (segment that contains g0 + k)
                        out[seg] = v[k];
                        ++seg;
                    }
                }
            }
        }
    }

    // ---- completion: the last CTA re-arms the workspace for the next call
    __syncthreads();
    if (t == 0) {
        __threadfence();
        const uint32_t old = atomicAdd(&hdr->done_ctr, 1u);
        if (old == (uint32_t)num_tiles - 1) {
            hdr->tile_ctr = 0;
            hdr->done_ctr = 0;
            hdr->epoch = hdr->epoch + 1;
            __threadfence();
        }
    }
}

cudaError_t launch_flat(const SegArgs& a, bool scan) {
    const int64_t N = a.n * a.m;
    const int64_t tiles = ceil_div(N, kFlatTile);
    if (tiles > 0x7fffffffLL) return cudaErrorInvalidValue;
    const bool tma_in = ((uintptr_t)a.in % 16) == 0;
    const bool tma_out = ((uintptr_t)a.out % 16) == 0;
    return dispatch_all(a.dt, a.op, a.f, [&](auto tt, auto opc, auto fc) -> cudaError_t {
        using T = decltype(tt);
        constexpr int OP = decltype(opc)::value, F = decltype(fc)::value;
        if (scan)
            flat_kernel<T, OP, F, true><<<(unsigned)tiles, FB, 0, a.stream>>>(
                (const T*)a.in, (T*)a.out, N, a.m, bits_to<T>(a.ne_bits), (uint8_t*)a.ws, (int)tiles, tma_in,
                tma_out);
        else
            flat_kernel<T, OP, F, false><<<(unsigned)tiles, FB, 0, a.stream>>>(
                (const T*)a.in, (T*)a.out, N, a.m, bits_to<T>(a.ne_bits), (uint8_t*)a.ws, (int)tiles, tma_in,
                tma_out);
        return cudaGetLastError();
    });
}

}  // namespace ifl
