// colred.cu -- axis-0 (column) segred / segscan of an [n][m] row-major array,
// the left-hand side of rule G4: reducing (or scanning) down the
// columns is segred/segscan of the transpose, but no transpose is
// materialised -- adjacent threads take adjacent columns, so every warp load
// is a contiguous row segment.
//
// The segments are the m columns (stride m, length n).  G3 gives the same
// three versions as for rows:
//   V_TOP     segmap^1 over columns, inner level sequential: a thread owns
//             VEC adjacent columns and walks all n rows (U rows in flight);
//   V_MIDDLE  a CTA per tile of 32*VEC columns: its 8 warps split the rows
//             (reduce: interleaved rows, smem combine; scan: chunks of 8*U
//             rows, per-warp local scans combined in smem, running carry);
//   V_FLAT    the rows are also split across CTAs (P row chunks): pass 1
//             per-chunk partials into the workspace, pass 2 combines them per
//             column (reduce: + d; scan: exclusive carries), and for the scan
//             pass 3 re-runs the chunk scan seeded with its carry ("at least
//             two, typically three, global accesses per element").
// d is applied exactly once per column (the reduce / exclusive carry of the
// first chunk starts from d).  f32 sum accumulators and carries are
// Kahan-compensated (long sequential chains: a column can hold 2^26 rows).
#include <algorithm>

#include "common.cuh"
#include "dispatch.cuh"
#include "ifl_internal.h"

namespace ifl {

namespace {

constexpr int kColThreads = 256;
constexpr int kColRG = 8;  // row groups (warps) of the V_MIDDLE / V_FLAT CTA

template <typename T, int VEC>
__device__ __forceinline__ void load_cols(const T* p, T (&v)[VEC]) {
    if constexpr (VEC == 4) {
        T e[4];
        unpack4<T>(ldg_stream4(p), e);
#pragma unroll
        for (int c = 0; c < 4; ++c) v[c] = e[c];
    } else {
        v[0] = __ldg(p);
    }
}

template <typename T, int VEC>
__device__ __forceinline__ void store_cols(T* p, const T (&v)[VEC]) {
    if constexpr (VEC == 4) {
        typename Vec4<T>::type q;
        q.x = v[0]; q.y = v[1]; q.z = v[2]; q.w = v[3];
        __stcs(reinterpret_cast<typename Vec4<T>::type*>(p), q);
    } else {
        p[0] = v[0];
    }
}

// Reduce rows [r0, r1) of a column tile.  A thread (cl, rg) owns columns
// c0 .. c0+VEC-1 and rows r0+rg, r0+rg+RG, ...; U loads in flight.  RG > 1:
// row groups combined in order through shared memory.  partial == nullptr:
// out[c] = d (+) column total; else partial[chunk][c] = chunk total (no d).
template <typename T, int OP, int F, int VEC, int RG>
__global__ void __launch_bounds__(kColThreads) col_red_kernel(const T* __restrict__ in, T* __restrict__ out,
                                                              int64_t n, int64_t m, T d, int64_t rows_per_chunk,
                                                              int ntiles, T* __restrict__ partial) {
    constexpr int CL = kColThreads / RG, W = CL * VEC, U = VEC == 4 ? 4 : 8;
    __shared__ T sred[RG > 1 ? RG : 1][RG > 1 ? W : 1];
    const int tile = blockIdx.x % ntiles;
    const int64_t chunk = blockIdx.x / ntiles;
    const int cl = threadIdx.x % CL, rg = threadIdx.x / CL;
    const int64_t c0 = (int64_t)tile * W + (int64_t)cl * VEC;
    const int64_t r0 = chunk * rows_per_chunk, r1 = std::min(n, r0 + rows_per_chunk);
    Acc<OP, T> acc[VEC];
#pragma unroll
    for (int v = 0; v < VEC; ++v) acc[v] = Acc<OP, T>(identity<OP, T>());
    if (c0 < m) {
        const T* col = in + c0;
        int64_t r = r0 + rg;
        for (; r + (U - 1) * RG < r1; r += U * RG) {
            T x[U][VEC];
#pragma unroll
            for (int u = 0; u < U; ++u) load_cols<T, VEC>(col + (r + u * RG) * m, x[u]);
#pragma unroll
            for (int u = 0; u < U; ++u)
#pragma unroll
                for (int v = 0; v < VEC; ++v) acc[v].add(apply_map<F>(x[u][v]));
        }
        for (; r < r1; r += RG) {
            T x[VEC];
            load_cols<T, VEC>(col + r * m, x);
#pragma unroll
            for (int v = 0; v < VEC; ++v) acc[v].add(apply_map<F>(x[v]));
        }
    }
    T tot[VEC];
#pragma unroll
    for (int v = 0; v < VEC; ++v) tot[v] = acc[v].get();
    if constexpr (RG > 1) {
#pragma unroll
        for (int v = 0; v < VEC; ++v) sred[rg][cl * VEC + v] = tot[v];
        __syncthreads();
        if (rg != 0) return;
#pragma unroll
        for (int v = 0; v < VEC; ++v) {
            Acc<OP, T> a(identity<OP, T>());
#pragma unroll
            for (int k = 0; k < RG; ++k) a.add(sred[k][cl * VEC + v]);
            tot[v] = a.get();
        }
    }
    if (c0 >= m) return;
    if (partial) {
        store_cols<T, VEC>(partial + chunk * m + c0, tot);
    } else {
#pragma unroll
        for (int v = 0; v < VEC; ++v) tot[v] = combine<OP>(d, tot[v]);
        store_cols<T, VEC>(out + c0, tot);
    }
}

// V_FLAT pass 2 when there are few chunks (wide arrays): one thread per
// column walks the P partials (SCAN: exclusive carries in place).
template <typename T, int OP, bool SCAN>
__global__ void __launch_bounds__(256) col_fix_kernel(T* __restrict__ partial, T* __restrict__ out, int64_t m,
                                                      int P, T d) {
    for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c < m; c += (int64_t)gridDim.x * blockDim.x) {
        Acc<OP, T> acc(d);
        for (int p = 0; p < P; ++p) {
            const T v = partial[(int64_t)p * m + c];
            if constexpr (SCAN) partial[(int64_t)p * m + c] = acc.get();
            acc.add(v);
        }
        if constexpr (!SCAN) out[c] = acc.get();
    }
}

// V_FLAT pass 2 over the per-chunk partials [P][mv] (mv = m, or 32 virtual
// columns in narrow mode, real column j = virtual c % m).  A CTA of 32 warps
// takes 32 real columns; warp w folds the chunks of its range of p, the
// warps' totals are combined in order in shared memory.  SCAN = false:
// out[j] = d (+) all chunk totals; SCAN = true: every chunk's (virtual)
// partials are replaced by its exclusive carry d (+) totals of chunks < p.
template <typename T, int OP, bool SCAN>
__global__ void __launch_bounds__(1024) col_carry_kernel(T* __restrict__ partial, T* __restrict__ out, int64_t m,
                                                         int64_t mv, int P, T d) {
    __shared__ T sw[32][33];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int64_t j = (int64_t)blockIdx.x * 32 + lane;
    const bool live = j < m;
    const int fold = (int)(mv / m);
    const int per = (P + 31) / 32, p0 = w * per, p1 = min(P, p0 + per);
    auto val = [&](int p) {
        T v = identity<OP, T>();
        for (int k = 0; k < fold; ++k) v = combine<OP>(v, partial[(int64_t)p * mv + j + (int64_t)k * m]);
        return v;
    };
    Acc<OP, T> a(identity<OP, T>());
    if (live)
        for (int p = p0; p < p1; p += 8) {  // 8 independent loads in flight
            T v[8];
#pragma unroll
            for (int q = 0; q < 8; ++q) v[q] = p + q < p1 ? val(p + q) : identity<OP, T>();
#pragma unroll
            for (int q = 0; q < 8; ++q) a.add(v[q]);
        }
    sw[w][lane] = a.get();
    __syncthreads();
    if constexpr (!SCAN) {
        if (w == 0 && live) {
            Acc<OP, T> t(d);
            for (int k = 0; k < 32; ++k) t.add(sw[k][lane]);
            out[j] = t.get();
        }
    } else {
        Acc<OP, T> c(d);
        for (int k = 0; k < w; ++k) c.add(sw[k][lane]);
        if (live)
            for (int p = p0; p < p1; ++p) {
                const T v = val(p);
                for (int k = 0; k < fold; ++k) partial[(int64_t)p * mv + j + (int64_t)k * m] = c.get();
                c.add(v);
            }
    }
}

// V_FLAT pass 2 in narrow mode (partials [P][vw], vw = 32 or 128 virtual
// columns, real column j = virtual c % m).  One CTA of 32 warps: warp w
// folds the chunks of its range of p.  Reduce: per virtual column, then the
// virtual columns of each real column in shared memory.  SCAN (m | 32): the
// vw/32 column groups and the lanes of a class (stride-m xor) are folded, and
// each chunk's virtual partials are replaced by its exclusive carry,
// replicated over every virtual column of the real column.
template <typename T, int OP, bool SCAN>
__global__ void __launch_bounds__(1024) col_narrow_fix_kernel(T* __restrict__ partial, T* __restrict__ out,
                                                              int m, int vw, int P, T d) {
    __shared__ T sv[32][129];
    __shared__ T vt[128];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int per = (P + 31) / 32, p0 = w * per, p1 = min(P, p0 + per);
    if constexpr (!SCAN) {
        for (int cg = 0; cg < vw; cg += 32) {
            Acc<OP, T> a(identity<OP, T>());
            for (int p = p0; p < p1; p += 8) {  // 8 independent loads in flight
                T v[8];
#pragma unroll
                for (int q = 0; q < 8; ++q) v[q] = p + q < p1 ? partial[(int64_t)(p + q) * vw + cg + lane] : identity<OP, T>();
#pragma unroll
                for (int q = 0; q < 8; ++q) a.add(v[q]);
            }
            sv[w][cg + lane] = a.get();
        }
        __syncthreads();
        if (threadIdx.x < vw) {
            Acc<OP, T> a(identity<OP, T>());
            for (int k = 0; k < 32; ++k) a.add(sv[k][threadIdx.x]);
            vt[threadIdx.x] = a.get();
        }
        __syncthreads();
        if (threadIdx.x < m) {
            Acc<OP, T> a(d);
            for (int c = threadIdx.x; c < vw; c += m) a.add(vt[c]);
            out[threadIdx.x] = a.get();
        }
    } else {
        // value of a chunk for this lane's real column class: fold the vw/32
        // virtual column groups, then the lanes of the class (stride m)
        const int ng = vw / 32;
        auto cls = [&](int p) {
            T v = identity<OP, T>();
            for (int g = 0; g < ng; ++g) {
                const int c = g * 32 + lane;
                if ((c % m) == (lane % m)) v = combine<OP>(v, partial[(int64_t)p * vw + c]);
            }
            for (int sft = m; sft < 32; sft <<= 1) v = combine<OP>(v, __shfl_xor_sync(0xffffffffu, v, sft));
            return v;
        };
        // the warp's chunk values stay in registers between the two walks (<= 48 chunks)
        constexpr int kMaxPer = 48;
        T v[kMaxPer];
#pragma unroll
        for (int q = 0; q < kMaxPer; ++q) v[q] = p0 + q < p1 ? cls(p0 + q) : identity<OP, T>();
        Acc<OP, T> a(identity<OP, T>());
#pragma unroll
        for (int q = 0; q < kMaxPer; ++q) a.add(v[q]);
        sv[w][lane] = a.get();
        __syncthreads();
        Acc<OP, T> c(d);
        for (int k = 0; k < w; ++k) c.add(sv[k][lane]);
#pragma unroll
        for (int q = 0; q < kMaxPer; ++q) {
            if (p0 + q < p1)
                for (int g = 0; g < ng; ++g) {
                    const int cc = g * 32 + lane;
                    partial[(int64_t)(p0 + q) * vw + cc] = c.get();  // every virtual column of the class
                }
            c.add(v[q]);
        }
    }
}

// Inclusive scan of rows [r0, r1) of a column tile, seeded per column with
// carry_in[chunk][c] (V_FLAT pass 3) or d.  Rows advance in chunks of RG*U:
// the thread scans its U consecutive rows in registers, the RG row-group
// totals are combined in order through shared memory, and the running carry
// (Kahan for f32 sums) moves to the next chunk.
//
// NARROW (V_FLAT pass 3 for m | 32, m < 32): the array is viewed as [n*m/32]
// virtual rows of 32 (one warp-wide 128-byte load each), virtual column l
// holding real column l % m; within a virtual row the real rows of one column
// are lanes l, l+m, l+2m, ..., combined by a stride-m warp scan (nm = m).
template <typename T, int OP, int F, int VEC, int RG, bool NARROW = false, int U = 4>
__global__ void __launch_bounds__(kColThreads) col_scan_kernel(const T* __restrict__ in, T* __restrict__ out,
                                                               int64_t n, int64_t m, T d, int64_t rows_per_chunk,
                                                               int ntiles, const T* __restrict__ carry_in,
                                                               int nm = 0) {
    constexpr int CL = kColThreads / RG, W = CL * VEC;
    __shared__ T stot[RG > 1 ? RG : 1][RG > 1 ? W : 1];
    const int tile = blockIdx.x % ntiles;
    const int64_t chunk = blockIdx.x / ntiles;
    const int cl = threadIdx.x % CL, rg = threadIdx.x / CL;
    const int64_t c0 = (int64_t)tile * W + (int64_t)cl * VEC;
    const bool live = c0 < m;
    const int64_t r0 = chunk * rows_per_chunk, r1 = std::min(n, r0 + rows_per_chunk);
    Acc<OP, T> carry[VEC];
#pragma unroll
    for (int v = 0; v < VEC; ++v)
        carry[v] = Acc<OP, T>((carry_in && live) ? carry_in[chunk * m + c0 + v] : d);
    for (int64_t base = r0; base < r1; base += (int64_t)RG * U) {
        const int64_t rb = base + (int64_t)rg * U;
        T x[U][VEC];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            if (live && rb + u < r1) {
                load_cols<T, VEC>(in + (rb + u) * m + c0, x[u]);
#pragma unroll
                for (int v = 0; v < VEC; ++v) x[u][v] = apply_map<F>(x[u][v]);
            } else {
#pragma unroll
                for (int v = 0; v < VEC; ++v) x[u][v] = identity<OP, T>();
            }
        }
        T ttot[VEC];  // the thread's total over its U rows
        if constexpr (NARROW) {
            // virtual row of 32*VEC elements: element e = lane*VEC + v holds real
            // column e % m.  Column slots of a lane: each component (m >= VEC), or
            // v % m (m = 1, 2 with VEC = 4: the lane holds 4/m rows of each
            // column, scanned in-lane first).  All register indices are static.
            const int lane = threadIdx.x & 31;
            const int q = nm >= VEC ? nm / VEC : 1;  // lane stride between rows of one column
            const int last = 32 - q + (lane % q);    // last lane of this lane's column class
            // inclusive stride-q warp scan of t: returns the exclusive prefix, rt = row total
            auto wscan = [&](T t, T& rt) {
                for (int sft = q; sft < 32; sft <<= 1) {
                    const T o = __shfl_up_sync(0xffffffffu, t, sft);
                    if (lane >= sft) t = combine<OP>(o, t);
                }
                rt = __shfl_sync(0xffffffffu, t, last);
                const T e = __shfl_up_sync(0xffffffffu, t, q);
                return lane >= q ? e : identity<OP, T>();
            };
            T acc[VEC];
#pragma unroll
            for (int c = 0; c < VEC; ++c) acc[c] = identity<OP, T>();
            if (VEC == 1 || nm >= VEC) {
#pragma unroll
                for (int u = 0; u < U; ++u)
#pragma unroll
                    for (int v = 0; v < VEC; ++v) {
                        T rt;
                        const T ex = wscan(x[u][v], rt);
                        x[u][v] = combine<OP>(combine<OP>(acc[v], ex), x[u][v]);
                        acc[v] = combine<OP>(acc[v], rt);
                    }
#pragma unroll
                for (int v = 0; v < VEC; ++v) ttot[v] = acc[v];
            } else if (nm == 2) {  // VEC == 4: slots {0, 2} and {1, 3}
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    x[u][VEC > 2 ? 2 : 0] = combine<OP>(x[u][0], x[u][VEC > 2 ? 2 : 0]);
                    x[u][VEC > 3 ? 3 : 0] = combine<OP>(x[u][VEC > 1 ? 1 : 0], x[u][VEC > 3 ? 3 : 0]);
                    T r0, r1;
                    const T e0 = wscan(x[u][VEC > 2 ? 2 : 0], r0), e1 = wscan(x[u][VEC > 3 ? 3 : 0], r1);
                    const T p0 = combine<OP>(acc[0], e0), p1 = combine<OP>(acc[VEC > 1 ? 1 : 0], e1);
#pragma unroll
                    for (int v = 0; v < VEC; ++v) x[u][v] = combine<OP>((v & 1) ? p1 : p0, x[u][v]);
                    acc[0] = combine<OP>(acc[0], r0);
                    acc[VEC > 1 ? 1 : 0] = combine<OP>(acc[VEC > 1 ? 1 : 0], r1);
                }
#pragma unroll
                for (int v = 0; v < VEC; ++v) ttot[v] = acc[(v & 1) && VEC > 1 ? 1 : 0];
            } else {  // nm == 1, VEC == 4: one column, the lane holds 4 consecutive rows
#pragma unroll
                for (int u = 0; u < U; ++u) {
#pragma unroll
                    for (int v = 1; v < VEC; ++v) x[u][v] = combine<OP>(x[u][v - 1], x[u][v]);
                    T r0;
                    const T p0 = combine<OP>(acc[0], wscan(x[u][VEC - 1], r0));
#pragma unroll
                    for (int v = 0; v < VEC; ++v) x[u][v] = combine<OP>(p0, x[u][v]);
                    acc[0] = combine<OP>(acc[0], r0);
                }
#pragma unroll
                for (int v = 0; v < VEC; ++v) ttot[v] = acc[0];
            }
        } else {
#pragma unroll
            for (int u = 1; u < U; ++u)
#pragma unroll
                for (int v = 0; v < VEC; ++v) x[u][v] = combine<OP>(x[u - 1][v], x[u][v]);
#pragma unroll
            for (int v = 0; v < VEC; ++v) ttot[v] = x[U - 1][v];
        }
        T pre[VEC], ctot[VEC];
        if constexpr (RG > 1) {
#pragma unroll
            for (int v = 0; v < VEC; ++v) stot[rg][cl * VEC + v] = ttot[v];
            __syncthreads();
#pragma unroll
            for (int v = 0; v < VEC; ++v) {
                T p = identity<OP, T>(), t = identity<OP, T>();
#pragma unroll
                for (int k = 0; k < RG; ++k) {
                    const T w = stot[k][cl * VEC + v];
                    if (k < rg) p = combine<OP>(p, w);
                    t = combine<OP>(t, w);
                }
                pre[v] = p;
                ctot[v] = t;
            }
            __syncthreads();  // stot is rewritten by the next chunk
        } else {
#pragma unroll
            for (int v = 0; v < VEC; ++v) {
                pre[v] = identity<OP, T>();
                ctot[v] = ttot[v];
            }
        }
#pragma unroll
        for (int v = 0; v < VEC; ++v) pre[v] = combine<OP>(carry[v].get(), pre[v]);
#pragma unroll
        for (int u = 0; u < U; ++u) {
            if (live && rb + u < r1) {
                T o[VEC];
#pragma unroll
                for (int v = 0; v < VEC; ++v) o[v] = combine<OP>(pre[v], x[u][v]);
                store_cols<T, VEC>(out + (rb + u) * m + c0, o);
            }
        }
#pragma unroll
        for (int v = 0; v < VEC; ++v) carry[v].add(ctot[v]);
    }
}

}  // namespace

// V_FLAT geometry: P row chunks so that tiles * P fills ~8 CTAs per SM, each
// chunk at least 64 rows (a multiple of the scan's RG*U rows).  Narrow mode
// (vw = 32 or 128): the [n][m] array viewed as [n*m/vw][vw] virtual rows,
// virtual column c holding real column c % m (m | vw).
ColGeom col_geom(int64_t n, int64_t m, int version, bool vec4, int vw) {
    ColGeom g;
    const int VEC = vec4 ? 4 : 1;
    const int RG = version == 0 ? 1 : kColRG;
    g.nv = vw ? n * m / vw : n;
    g.mv = vw ? vw : m;
    const int64_t W = (int64_t)(kColThreads / RG) * VEC;
    g.ntiles = ceil_div(g.mv, W);
    g.P = 1;
    g.rows_per_chunk = std::max<int64_t>(g.nv, 1);
    if (version == 2) {
        const int64_t want = ceil_div((int64_t)148 * 8, g.ntiles);
        const int64_t maxp = std::max<int64_t>(1, g.nv / 128);
        g.P = std::max<int64_t>(1, std::min(want, maxp));
        g.rows_per_chunk = ceil_div(ceil_div(g.nv, g.P), 128) * 128;
        g.P = ceil_div(g.nv, g.rows_per_chunk);
    }
    return g;
}

// Narrow-mode virtual width for V_FLAT: 128 (16-byte lanes) for the reduce
// when m | 128, 32 (one element per lane, stride-m warp scans) for the scan
// when m | 32; 0 = plain columns.
static int col_narrow(int64_t n, int64_t m, int version, bool scan, bool aligned16) {
    if (version != 2 || m <= 0) return 0;
    if (!scan && m < 128 && 128 % m == 0 && (n * m) % 128 == 0 && aligned16) return 128;
    if (scan && m < 32 && 32 % m == 0 && (n * m) % 128 == 0 && aligned16) return 128;
    if (scan && m < 32 && 32 % m == 0 && (n * m) % 32 == 0) return 32;
    return 0;
}

// 16-byte vectors for TOP whenever rows allow it; MIDDLE / FLAT only when a
// warp's 128 columns are all live (m >= 128), else one column per lane.
static bool col_vec4(const SegArgs& a, int version) {
    const bool ok = (a.m % 4 == 0) && ((uintptr_t)a.in % 16 == 0) && ((uintptr_t)a.out % 16 == 0);
    return ok && (version == 0 || a.m >= 128);
}

size_t col_ws_bytes(int64_t n, int64_t m, int version) {
    if (version != 2 && version != -1) return 0;
    if (n <= 0 || m <= 0) return 0;
    size_t mx = 0;
    for (int v4 = 0; v4 < 2; ++v4) {
        const ColGeom g = col_geom(n, m, 2, v4 != 0, 0);
        mx = std::max(mx, (size_t)g.P * (size_t)g.mv * 4);
    }
    for (int sc = 0; sc < 2; ++sc) {
        const int vw = col_narrow(n, m, 2, sc != 0, true);
        if (vw) {
            const ColGeom g = col_geom(n, m, 2, vw == 128, vw);
            mx = std::max(mx, (size_t)g.P * (size_t)g.mv * 4);
        }
    }
    return mx;
}

cudaError_t launch_col(const SegArgs& a, bool scan, int version) {
    const bool al16 = ((uintptr_t)a.in % 16 == 0) && ((uintptr_t)a.out % 16 == 0);
    const int vw = col_narrow(a.n, a.m, version, scan, al16);
    const bool vec4 = vw ? vw == 128 : col_vec4(a, version);
    const ColGeom g = col_geom(a.n, a.m, version, vec4, vw);
    if ((int64_t)g.ntiles * g.P > 0x7fffffffLL) return cudaErrorInvalidValue;
    const unsigned grid = (unsigned)(g.ntiles * g.P);
    return dispatch_all(a.dt, a.op, a.f, [&](auto tt, auto opc, auto fc) -> cudaError_t {
        using T = decltype(tt);
        constexpr int OP = decltype(opc)::value, F = decltype(fc)::value;
        const T d = bits_to<T>(a.ne_bits);
        const T* in = (const T*)a.in;
        T* out = (T*)a.out;
        T* part = (T*)a.ws;
        auto go = [&](auto vecc) -> cudaError_t {
            constexpr int VEC = decltype(vecc)::value;
            if (version == 0) {
                if (scan)
                    col_scan_kernel<T, OP, F, VEC, 1><<<grid, kColThreads, 0, a.stream>>>(in, out, a.n, a.m, d,
                                                                                         g.rows_per_chunk, (int)g.ntiles,
                                                                                         nullptr);
                else
                    col_red_kernel<T, OP, F, VEC, 1><<<grid, kColThreads, 0, a.stream>>>(in, out, a.n, a.m, d,
                                                                                        g.rows_per_chunk, (int)g.ntiles,
                                                                                        nullptr);
                return cudaGetLastError();
            }
            if (version == 1) {
                if (scan)
                    col_scan_kernel<T, OP, F, VEC, kColRG, false, VEC == 1 ? 16 : 4><<<grid, kColThreads, 0, a.stream>>>(
                        in, out, a.n, a.m, d, g.rows_per_chunk, (int)g.ntiles, nullptr);
                else
                    col_red_kernel<T, OP, F, VEC, kColRG><<<grid, kColThreads, 0, a.stream>>>(
                        in, out, a.n, a.m, d, g.rows_per_chunk, (int)g.ntiles, nullptr);
                return cudaGetLastError();
            }
            // V_FLAT: partials per row chunk -> combine over chunks -> (scan) seeded chunk scans
            col_red_kernel<T, OP, F, VEC, kColRG><<<grid, kColThreads, 0, a.stream>>>(
                in, out, g.nv, g.mv, d, g.rows_per_chunk, (int)g.ntiles, part);
            cudaError_t e = cudaGetLastError();
            if (e != cudaSuccess) return e;
            // pass 2: few chunks -> a thread per column; many -> 32 warps per 32 columns
            const bool wide = g.P < 64 && !vw;
            const unsigned g2 = wide ? (unsigned)std::min<int64_t>(ceil_div(a.m, 256), (int64_t)148 * 16)
                                     : (unsigned)ceil_div(a.m, 32);
            if (wide) {
                if (scan) col_fix_kernel<T, OP, true><<<g2, 256, 0, a.stream>>>(part, out, a.m, (int)g.P, d);
                else col_fix_kernel<T, OP, false><<<g2, 256, 0, a.stream>>>(part, out, a.m, (int)g.P, d);
            } else if (vw) {
                if (scan) col_narrow_fix_kernel<T, OP, true><<<1, 1024, 0, a.stream>>>(part, out, (int)a.m, vw, (int)g.P, d);
                else col_narrow_fix_kernel<T, OP, false><<<1, 1024, 0, a.stream>>>(part, out, (int)a.m, vw, (int)g.P, d);
            } else {
                if (scan) col_carry_kernel<T, OP, true><<<g2, 1024, 0, a.stream>>>(part, out, a.m, g.mv, (int)g.P, d);
                else col_carry_kernel<T, OP, false><<<g2, 1024, 0, a.stream>>>(part, out, a.m, g.mv, (int)g.P, d);
            }
            if ((e = cudaGetLastError()) != cudaSuccess || !scan) return e;
            if (vw) {  // narrow: virtual rows of 32*VEC, stride-m lane scans (16 KB per CTA chunk)
                col_scan_kernel<T, OP, F, VEC, kColRG, true, VEC == 1 ? 16 : 4><<<grid, kColThreads, 0, a.stream>>>(
                    in, out, g.nv, g.mv, d, g.rows_per_chunk, (int)g.ntiles, part, (int)a.m);
                return cudaGetLastError();
            }
            col_scan_kernel<T, OP, F, VEC, kColRG, false, VEC == 1 ? 16 : 4><<<grid, kColThreads, 0, a.stream>>>(
                in, out, a.n, a.m, d, g.rows_per_chunk, (int)g.ntiles, part);
            return cudaGetLastError();
        };
        return vec4 ? go(IC<4>{}) : go(IC<1>{});
    });
}

}  // namespace ifl
