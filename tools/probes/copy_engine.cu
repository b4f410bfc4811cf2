// Streaming-engine microbenchmark (not the product): how fast can a
// producer-warp + mbarrier ring + TMA bulk load/store structure copy 256 MiB
// on this GPU, versus a plain LDG/STG copy?  Variants differ in tile bytes,
// slots, CTAs per SM and the store path.  Prints one JSON line per variant.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mb_init(uint64_t* b, int c) { asm volatile("mbarrier.init.shared.b64 [%0], %1;" ::"r"(su32(b)), "r"(c)); }
__device__ __forceinline__ void mb_expect(uint64_t* b, uint32_t tx) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(b)), "r"(tx) : "memory");
}
__device__ __forceinline__ void mb_wait(uint64_t* b, uint32_t ph) {
    asm volatile("{\n.reg .pred P;\nW: mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n@!P bra W;\n}" ::"r"(su32(b)), "r"(ph) : "memory");
}
__device__ __forceinline__ void g2s(void* d, const void* s, uint32_t n, uint64_t* b) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(su32(d)), "l"(s), "r"(n), "r"(su32(b)) : "memory");
}
__device__ __forceinline__ void s2g(void* d, const void* s, uint32_t n) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(d), "r"(su32(s)), "r"(n) : "memory");
}

template <int TILE_F, int SLOTS, bool TMA_ST>
__global__ void engine(const float* __restrict__ in, float* __restrict__ out, int ntiles) {
    extern __shared__ __align__(128) float ring[];
    __shared__ alignas(8) uint64_t full[SLOTS], empty[SLOTS];
    const int t = threadIdx.x, w = t >> 5, lane = t & 31;
    if (t == 0) {
        for (int i = 0; i < SLOTS; ++i) { mb_init(&full[i], 1); mb_init(&empty[i], 1); }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const int G = gridDim.x;
    if (w == 8) {
        if (lane == 0) {
            int k = 0;
            for (int tile = blockIdx.x; tile < ntiles; tile += G, ++k) {
                const int sl = k % SLOTS;
                if (k >= SLOTS) mb_wait(&empty[sl], ((k / SLOTS) - 1) & 1);
                mb_expect(&full[sl], TILE_F * 4);
                g2s(ring + sl * TILE_F, in + (size_t)tile * TILE_F, TILE_F * 4, &full[sl]);
            }
        }
        return;
    }
    int k = 0, pend = -1;
    for (int tile = blockIdx.x; tile < ntiles; tile += G, ++k) {
        const int sl = k % SLOTS;
        float* buf = ring + sl * TILE_F;
        mb_wait(&full[sl], (k / SLOTS) & 1);
        // touch the data like a scan would: each thread rewrites its slice
        for (int i = t * 4; i < TILE_F; i += 256 * 4) {
            float4 v = *reinterpret_cast<float4*>(buf + i);
            v.x += 1.f; v.y += 1.f; v.z += 1.f; v.w += 1.f;
            if (TMA_ST) *reinterpret_cast<float4*>(buf + i) = v;
            else __stcs(reinterpret_cast<float4*>(out + (size_t)tile * TILE_F + i), v);
        }
        if (TMA_ST) asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        asm volatile("bar.sync 1, 256;" ::: "memory");
        if (t == 0) {
            if (TMA_ST) {
                s2g(out + (size_t)tile * TILE_F, buf, TILE_F * 4);
                asm volatile("cp.async.bulk.commit_group;" ::: "memory");
                if (pend >= 0) {
                    asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
                    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(&empty[pend])) : "memory");
                }
                pend = sl;
            } else {
                asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(&empty[sl])) : "memory");
            }
        }
    }
    if (t == 0 && TMA_ST) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

__global__ void plain_copy(const float4* __restrict__ in, float4* __restrict__ out, size_t n4) {
    for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += (size_t)gridDim.x * blockDim.x) {
        float4 v = __ldcs(in + i);
        v.x += 1.f;
        __stcs(out + i, v);
    }
}

template <int TILE_F, int SLOTS, bool TMA_ST>
void run(const char* name, const float* in, float* out, size_t N, int minb) {
    auto k = engine<TILE_F, SLOTS, TMA_ST>;
    const int smem = TILE_F * 4 * SLOTS;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    int per = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k, 288, smem);
    if (minb && per > minb) per = minb;
    const int ntiles = (int)(N / TILE_F);
    const int grid = per * 148;
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    for (int i = 0; i < 3; ++i) k<<<grid, 288, smem>>>(in, out, ntiles);
    cudaEventRecord(a);
    const int R = 10;
    for (int i = 0; i < R; ++i) k<<<grid, 288, smem>>>(in, out, ntiles);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    const double us = ms * 1e3 / R;
    printf("{\"variant\": \"%s\", \"tile_KB\": %d, \"slots\": %d, \"ctas_per_sm\": %d, \"us\": %.1f, \"GBps\": %.0f, \"err\": \"%s\"}\n",
           name, TILE_F * 4 / 1024, SLOTS, per, us, 8.0 * N / us / 1e3, cudaGetErrorString(cudaGetLastError()));
}

int main() {
    const size_t N = (size_t)1 << 26;
    float *in, *out;
    cudaMalloc(&in, N * 4);
    cudaMalloc(&out, N * 4);
    cudaMemset(in, 0, N * 4);
    {
        cudaEvent_t a, b;
        cudaEventCreate(&a);
        cudaEventCreate(&b);
        for (int i = 0; i < 3; ++i) plain_copy<<<148 * 8, 256>>>((const float4*)in, (float4*)out, N / 4);
        cudaEventRecord(a);
        for (int i = 0; i < 10; ++i) plain_copy<<<148 * 8, 256>>>((const float4*)in, (float4*)out, N / 4);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        printf("{\"variant\": \"plain_ldg_stg\", \"us\": %.1f, \"GBps\": %.0f}\n", ms * 100, 8.0 * N / (ms * 100) / 1e3);
    }
    run<5120, 3, true>("tma_ld_tma_st", in, out, N, 3);
    run<5120, 3, false>("tma_ld_stg", in, out, N, 3);
    run<5120, 4, true>("tma_ld_tma_st", in, out, N, 2);
    run<5120, 6, true>("tma_ld_tma_st", in, out, N, 2);
    run<2048, 4, true>("tma_ld_tma_st", in, out, N, 0);
    run<2048, 6, true>("tma_ld_tma_st", in, out, N, 0);
    run<4096, 4, true>("tma_ld_tma_st", in, out, N, 0);
    run<8192, 3, true>("tma_ld_tma_st", in, out, N, 0);
    run<8192, 6, true>("tma_ld_tma_st", in, out, N, 0);
    run<2048, 6, false>("tma_ld_stg", in, out, N, 0);
    run<4096, 6, false>("tma_ld_stg", in, out, N, 0);
    return 0;
}
