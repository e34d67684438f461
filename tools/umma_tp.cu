// umma_tp.cu -- tcgen05.mma kind::f16 (bf16) THROUGHPUT on one SM: cycles per instruction for
// 64 back-to-back M = 128, K = 16 instructions (one accumulator), by N and operand placement /
// layout: SS no-swizzle K-major, SS 128B-swizzle K-major, TS (A in TMEM) with B no-swizzle or
// 128B-swizzle.  Operand contents are irrelevant to the timing (zeros).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/umma_tp tools/umma_tp.cu
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t sa(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t desc(uint32_t a, uint32_t lbo, uint32_t sbo, uint32_t layout) {
    return (uint64_t)((a >> 4) & 0x3FFF) | ((uint64_t)((lbo >> 4) & 0x3FFF) << 16) |
           ((uint64_t)((sbo >> 4) & 0x3FFF) << 32) | (1ull << 46) | ((uint64_t)layout << 61);
}
__device__ __forceinline__ void mma_ss(uint32_t d, uint64_t a, uint64_t b, uint32_t id, uint32_t acc) {
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\ttcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d), "l"(a), "l"(b), "r"(id), "r"(acc));
}
__device__ __forceinline__ void mma_ts(uint32_t d, uint32_t a, uint64_t b, uint32_t id, uint32_t acc) {
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\ttcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}" ::"r"(d), "r"(a), "l"(b), "r"(id), "r"(acc));
}
template <int MODE, int N, int NACC>
__global__ void tp(long long *out, int reps) {
    extern __shared__ __align__(1024) unsigned char sm[];
    __shared__ uint64_t bar;
    __shared__ uint32_t tbase;
    const int t = threadIdx.x;
    for (int e = t; e < 160 * 1024 / 4; e += blockDim.x) reinterpret_cast<float *>(sm)[e] = 0.f;
    if (t < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(sa(&tbase)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (t == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sa(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    asm volatile("fence.proxy.async.shared::cta;");
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    const uint32_t tm = tbase;
    if (t < 32) {  // one warp issues (elect lane 0 inside)
        constexpr uint32_t id = (1u << 4) | (1u << 7) | (1u << 10) | (MODE == 4 ? (1u << 15) : 0u) | ((uint32_t)(N >> 3) << 17) | ((128u >> 4) << 24);
        const uint32_t s0 = sa(sm);
        const uint64_t a0 = MODE == 4 ? desc(s0, 1280, 128, 0) : ((MODE == 0 || MODE == 2) ? desc(s0, 128, 256, 0) : desc(s0, 16, 1024, 2));
        const uint64_t b0 = MODE == 4 ? desc(s0 + 65536, 128, 2048, 0) : ((MODE == 0 || MODE == 2) ? desc(s0 + 65536, 128, 256, 0) : desc(s0 + 65536, 16, 1024, 2));
        long long best = 1ll << 60;
        for (int rep = 0; rep < reps; ++rep) {
            __syncwarp();
            const long long c0 = clock64();
            if (t == 0) {
#pragma unroll
                for (int i = 0; i < 64; ++i) {
                    constexpr int DC = 256 / NACC > N ? N : 256 / NACC;
                    const uint32_t dcol = tm + 256 + (uint32_t)((i % NACC) * DC);
                    const uint64_t off = (MODE == 1 || MODE == 3) ? (uint64_t)((i & 3) * 2) : 0;
                    if (MODE < 2 || MODE == 4) mma_ss(dcol, a0 + (MODE == 4 ? (uint64_t)((i & 7) * 2 * 1280 >> 4) : off), b0 + (MODE == 4 ? (uint64_t)((i & 7) * 256 >> 4) : off), id, i >= NACC);
                    else mma_ts(dcol, tm + 8 * (i & 15), b0 + off, id, i >= NACC);
                }
                asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(sa(&bar)));
            }
            __syncwarp();
            uint32_t done = 0;
            while (!done)
                asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                             : "=r"(done) : "r"(sa(&bar)), "r"((unsigned)(rep & 1)));
            const long long c1 = clock64();
            if (c1 - c0 < best) best = c1 - c0;
        }
        if (t == 0) out[0] = best;
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    if (t < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tm));
}
template <int MODE, int N, int NACC> void run1(long long *d, const char *name) {
    long long h;
    cudaFuncSetAttribute(tp<MODE, N, NACC>, cudaFuncAttributeMaxDynamicSharedMemorySize, 160 * 1024);
    tp<MODE, N, NACC><<<1, 128, 160 * 1024>>>(d, 8);
    cudaError_t e = cudaDeviceSynchronize();
    cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost);
    printf("%-9s N=%3d acc=%d: %6.1f cycles/instr (%s)  ideal %5.1f\n", name, N, NACC, h / 64.0,
           cudaGetErrorString(e), 128.0 * N * 16 / 4096.0);
}
template <int MODE> void runm(long long *d, const char *name) {
    run1<MODE, 32, 1>(d, name); run1<MODE, 32, 4>(d, name); run1<MODE, 32, 8>(d, name);
    run1<MODE, 64, 1>(d, name); run1<MODE, 64, 4>(d, name);
    run1<MODE, 128, 1>(d, name); run1<MODE, 128, 2>(d, name); run1<MODE, 256, 1>(d, name);
}
// the K-means stage mix: 5 MMA1 (A in TMEM, N = 64, K-major B) + 8 MMA2 (A MN-major, N = 32)
__global__ void mix(long long *out, int reps) {
    extern __shared__ __align__(1024) unsigned char sm[];
    __shared__ uint64_t bar;
    __shared__ uint32_t tbase;
    const int t = threadIdx.x;
    for (int e = t; e < 160 * 1024 / 4; e += blockDim.x) reinterpret_cast<float *>(sm)[e] = 0.f;
    if (t < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(sa(&tbase)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (t == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sa(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    asm volatile("fence.proxy.async.shared::cta;");
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    const uint32_t tm = tbase;
    if (t < 32) {
        constexpr uint32_t id1 = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(64 >> 3) << 17) | ((128u >> 4) << 24);
        constexpr uint32_t id2 = (1u << 4) | (1u << 7) | (1u << 10) | (1u << 15) | ((uint32_t)(32 >> 3) << 17) | ((128u >> 4) << 24);
        const uint32_t s0 = sa(sm);
        const uint64_t b1 = desc(s0 + 65536, 128, 1536, 0);
        const uint64_t a2 = desc(s0, 1280, 128, 0), b2 = desc(s0 + 98304, 128, 2048, 0);
        long long best = 1ll << 60;
        for (int rep = 0; rep < reps; ++rep) {
            __syncwarp();
            const long long c0 = clock64();
            if (t == 0) {
#pragma unroll 1
                for (int st = 0; st < 16; ++st) {
#pragma unroll
                    for (int p = 0; p < 5; ++p) mma_ts(tm + 64 * (st & 3), tm + 384 + 8 * p, b1 + (uint64_t)(p * 256 >> 4), id1, p > 0);
#pragma unroll
                    for (int kk = 0; kk < 8; ++kk)
                        mma_ss(tm + 256 + 32 * (st & 1), a2 + (uint64_t)((kk * 2 * 1280) >> 4), b2 + (uint64_t)((kk * 256) >> 4), id2, 1);
                }
                asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(sa(&bar)));
            }
            __syncwarp();
            uint32_t done = 0;
            while (!done)
                asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                             : "=r"(done) : "r"(sa(&bar)), "r"((unsigned)(rep & 1)));
            const long long c1 = clock64();
            if (c1 - c0 < best) best = c1 - c0;
        }
        if (t == 0) out[0] = best;
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    if (t < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tm));
}
int main() {
    long long *d;
    cudaMalloc(&d, 8);
    runm<0>(d, "SS noswz"); runm<1>(d, "SS sw128"); runm<2>(d, "TS noswz"); runm<3>(d, "TS sw128");
    runm<4>(d, "SS A-MN");
    {
        long long h;
        cudaFuncSetAttribute(mix, cudaFuncAttributeMaxDynamicSharedMemorySize, 160 * 1024);
        mix<<<1, 128, 160 * 1024>>>(d, 8);
        cudaError_t e = cudaDeviceSynchronize();
        cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost);
        printf("k-means stage mix (5 MMA1 TS N=64 + 8 MMA2 SS N=32): %.1f cycles per stage (%s)\n", h / 16.0,
               cudaGetErrorString(e));
    }
    return 0;
}
