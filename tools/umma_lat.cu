// umma_lat.cu -- latency of the K-means step's tcgen05 MMA groups on one SM (cycles from
// the first issue to the commit's mbarrier arrival), for the operand placements in use.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t sa(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t desc(uint32_t a, uint32_t lbo, uint32_t sbo) {
    return (uint64_t)((a >> 4) & 0x3FFF) | ((uint64_t)((lbo >> 4) & 0x3FFF) << 16) | ((uint64_t)((sbo >> 4) & 0x3FFF) << 32) | (1ull << 46);
}
__device__ __forceinline__ void mma_ss(uint32_t d, uint64_t a, uint64_t b, uint32_t id, uint32_t acc) {
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\ttcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(d), "l"(a), "l"(b), "r"(id), "r"(acc));
}
__device__ __forceinline__ void mma_ts(uint32_t d, uint32_t a, uint64_t b, uint32_t id, uint32_t acc) {
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\ttcgen05.mma.cta_group::1.kind::tf32 [%0], [%1], %2, %3, p;\n\t}" ::"r"(d), "r"(a), "l"(b), "r"(id), "r"(acc));
}
__global__ void lat(long long *out, int mode, int reps) {
    extern __shared__ __align__(1024) unsigned char sm[];
    __shared__ uint64_t bar;
    __shared__ uint32_t tbase;
    const int t = threadIdx.x;
    for (int e = t; e < 96 * 1024 / 4; e += blockDim.x) reinterpret_cast<float *>(sm)[e] = 0.5f;
    if (t < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(sa(&tbase)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (t == 0) { asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sa(&bar))); asm volatile("fence.mbarrier_init.release.cluster;"); }
    asm volatile("fence.proxy.async.shared::cta;");
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    const uint32_t tm = tbase;
    if (t == 0) {
        const uint32_t id1 = (1u << 4) | (2u << 7) | (2u << 10) | ((32u >> 3) << 17) | ((128u >> 4) << 24);
        const uint32_t id2 = id1 | (1u << 15);
        const uint32_t s0 = sa(sm);
        long long best = 1ll << 60, tot = 0;
        for (int rep = 0; rep < reps; ++rep) {
            long long c0 = clock64();
            if (mode == 0) {          // MMA1, A from TMEM, 15 instructions
                for (int p = 0; p < 5; ++p) {
                    const uint64_t b = desc(s0 + 2 * p * 128, 128, 1280);
                    mma_ts(tm, tm + 192 + 8 * p, b, id1, p > 0);
                    mma_ts(tm, tm + 192 + 8 * p, b, id1, 1);
                    mma_ts(tm, tm + 232 + 8 * p, b, id1, 1);
                }
            } else if (mode == 1) {   // MMA1, A from smem K-major no swizzle, 15 instructions
                for (int p = 0; p < 5; ++p) {
                    const uint64_t a = desc(s0 + 8192 + 2 * p * 128, 128, 2560), b = desc(s0 + 2 * p * 128, 128, 1280);
                    mma_ss(tm, a, b, id1, p > 0); mma_ss(tm, a, b, id1, 1); mma_ss(tm, a, b, id1, 1);
                }
            } else if (mode == 2) {   // MMA2, A MN-major SW128_32B, B K-major, 16 instructions
                for (int kk = 0; kk < 16; ++kk)
                    mma_ss(tm + 96, desc(s0 + 8192 + kk * 3072, 512, 1536) | (1ull << 61), desc(s0 + 65536 + kk * 256, 128, 4096), id2, kk > 0);
            } else if (mode == 3) {   // MMA2-shaped but A K-major no swizzle (cost comparison only)
                for (int kk = 0; kk < 16; ++kk)
                    mma_ss(tm + 96, desc(s0 + 8192 + kk * 256, 128, 4096), desc(s0 + 65536 + kk * 256, 128, 4096), id1, kk > 0);
            } else if (mode == 4) {   // one single MMA1 instruction
                mma_ts(tm, tm + 192, desc(s0, 128, 1280), id1, 0);
            } else if (mode == 5) {   // 16 x N=32, four independent accumulators round-robin
                for (int kk = 0; kk < 16; ++kk)
                    mma_ss(tm + 32 * (kk & 3), desc(s0 + 8192 + kk * 256, 128, 4096), desc(s0 + 65536 + kk * 256, 128, 4096), id1, kk > 3);
            } else if (mode >= 6 && mode <= 8) {  // 16 x N = 64 / 128 / 256 (one accumulator)
                const uint32_t N = 64u << (mode - 6);
                const uint32_t idn = (1u << 4) | (2u << 7) | (2u << 10) | ((N >> 3) << 17) | ((128u >> 4) << 24);
                for (int kk = 0; kk < 16; ++kk)
                    mma_ss(tm, desc(s0 + 8192 + kk * 256, 128, 4096), desc(s0 + 65536 + kk * 256, 128, 256), idn, kk > 0);
            } else if (mode == 11) {  // K-means MMA1: bf16, A from TMEM, N = 64, 6 instructions
                const uint32_t idb = (1u << 4) | (1u << 7) | (1u << 10) | ((64u >> 3) << 17) | ((128u >> 4) << 24);
                for (int p = 0; p < 6; ++p)
                    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\ttcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}" ::"r"(tm), "r"(tm + 288 + 8 * p), "l"(desc(s0 + p * 256, 128, 1536)), "r"(idb), "r"((uint32_t)(p > 0)));
            } else if (mode == 12) {  // K-means MMA2: bf16, A MN-major (LBO 1280 K-groups, SBO 128), B K-major, N = 32, 8 instructions
                const uint32_t idb = (1u << 4) | (1u << 7) | (1u << 10) | (1u << 15) | ((32u >> 3) << 17) | ((128u >> 4) << 24);
                for (int kk = 0; kk < 8; ++kk)
                    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\ttcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tm + 192), "l"(desc(s0 + 8192 + kk * 2560, 1280, 128)), "l"(desc(s0 + 65536 + kk * 256, 128, 2048)), "r"(idb), "r"((uint32_t)(kk > 0)));
            } else if (mode == 13) {  // MMA1 + MMA2 back to back (one stage of the step)
                const uint32_t idb = (1u << 4) | (1u << 7) | (1u << 10) | ((64u >> 3) << 17) | ((128u >> 4) << 24);
                for (int p = 0; p < 6; ++p)
                    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\ttcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}" ::"r"(tm), "r"(tm + 288 + 8 * p), "l"(desc(s0 + p * 256, 128, 1536)), "r"(idb), "r"((uint32_t)(p > 0)));
                const uint32_t id2 = (1u << 4) | (1u << 7) | (1u << 10) | (1u << 15) | ((32u >> 3) << 17) | ((128u >> 4) << 24);
                for (int kk = 0; kk < 8; ++kk)
                    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\ttcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tm + 192), "l"(desc(s0 + 8192 + kk * 2560, 1280, 128)), "l"(desc(s0 + 65536 + kk * 256, 128, 2048)), "r"(id2), "r"((uint32_t)(kk > 0)));
            } else if (mode == 14) {  // MMA2 with M = 64: bf16 MN-major A, N = 32, 8 instructions
                const uint32_t idb = (1u << 4) | (1u << 7) | (1u << 10) | (1u << 15) | ((32u >> 3) << 17) | ((64u >> 4) << 24);
                for (int kk = 0; kk < 8; ++kk)
                    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\ttcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tm + 192), "l"(desc(s0 + 8192 + kk * 2560, 1280, 128)), "l"(desc(s0 + 65536 + kk * 256, 128, 2048)), "r"(idb), "r"((uint32_t)(kk > 0)));
            } else if (mode == 15) {  // MMA1 K = 80: 5 instructions
                const uint32_t idb = (1u << 4) | (1u << 7) | (1u << 10) | ((64u >> 3) << 17) | ((128u >> 4) << 24);
                for (int p = 0; p < 5; ++p)
                    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\ttcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}" ::"r"(tm), "r"(tm + 288 + 8 * p), "l"(desc(s0 + p * 256, 128, 1536)), "r"(idb), "r"((uint32_t)(p > 0)));
            } else {                  // kind::f16 (bf16) M128 N32 / N64 K16 x 8
                const uint32_t NB = mode == 9 ? 32u : 64u;
                const uint32_t idb = (1u << 4) | (1u << 7) | (1u << 10) | ((NB >> 3) << 17) | ((128u >> 4) << 24);
                for (int kk = 0; kk < 8; ++kk)
                    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\ttcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tm), "l"(desc(s0 + 8192 + kk * 256, 128, 4096)), "l"(desc(s0 + 65536 + kk * 256, 128, 4096)), "r"(idb), "r"((uint32_t)(kk > 0)));
            }
            asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(sa(&bar)));
            uint32_t done = 0;
            while (!done)
                asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}" : "=r"(done) : "r"(sa(&bar)), "r"(rep & 1));
            long long c1 = clock64() - c0;
            tot += c1;
            if (c1 < best) best = c1;
        }
        out[0] = best;
        out[1] = tot / reps;
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    if (t < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tm));
}
int main() {
    long long *o, h[2];
    cudaMalloc(&o, 16);
    cudaFuncSetAttribute(lat, cudaFuncAttributeMaxDynamicSharedMemorySize, 96 * 1024);
    const char *names[] = {"MMA1 TS x15", "MMA1 SS x15", "MMA2 MN-swz x16", "MMA2-shape K-major x16", "single MMA1 TS",
                           "x16 N32 4 accumulators", "x16 N64", "x16 N128", "x16 N256", "bf16 x8 N32 K16", "bf16 x8 N64 K16", "KM MMA1 bf16 TS N64 x6", "KM MMA2 bf16 MN x8", "KM stage (MMA1+MMA2)",
                           "MMA2 M64 x8", "MMA1 x5"};
    for (int m = 0; m < 16; ++m) {
        lat<<<1, 128, 96 * 1024>>>(o, m, 200);
        cudaError_t e = cudaDeviceSynchronize();
        if (e != cudaSuccess) { printf("%s: %s\n", names[m], cudaGetErrorString(e)); return 1; }
        cudaMemcpy(h, o, 16, cudaMemcpyDeviceToHost);
        printf("%-26s best %lld  avg %lld cycles\n", names[m], h[0], h[1]);
    }
    return 0;
}
