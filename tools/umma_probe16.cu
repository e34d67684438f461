// umma_probe16.cu -- pins the no-swizzle tcgen05 kind::f16 (bf16) operand layouts used by the
// K-means step: D[128 x N] = A[128 x 16] . B[16 x N] with small integers (exact in bf16).
//   A: K-major (core matrix 8 rows x 16 B = 8 k) or MN-major (8 k-rows x 16 B = 8 m), or TMEM
//   B: K-major
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#include <cuda_bf16.h>

__device__ __forceinline__ uint32_t sa(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t desc(uint32_t a, uint32_t lbo, uint32_t sbo) {
    return (uint64_t)((a >> 4) & 0x3FFF) | ((uint64_t)((lbo >> 4) & 0x3FFF) << 16) | ((uint64_t)((sbo >> 4) & 0x3FFF) << 32) | (1ull << 46);
}
__device__ float aval(int m, int k) { return (float)((m * 3 + k * 5) % 7 - 3); }
__device__ float bval(int n, int k) { return (float)((n * 2 + k * 3) % 5 - 2); }
// mode 0: A K-major smem; 1: A MN-major smem (LBO = K-group stride, SBO = M-group stride);
// 2: A MN-major with the two swapped; 3: A from TMEM (K-major)
__global__ void probe(int mode, int N, float *D) {
    __shared__ __align__(1024) __nv_bfloat16 As[128 * 16 * 2];
    __shared__ __align__(1024) __nv_bfloat16 Bs[64 * 16 * 2];
    __shared__ uint64_t bar;
    __shared__ uint32_t tbase;
    const int t = threadIdx.x;
    // A K-major: core (m/8, k/8): (m/8)*256 + (k/8)*128 + (m%8)*16 + (k%8)*2  (LBO k-chunk 128, SBO m-group 256)
    // A MN-major: core (m/8, k/8): (m/8)*128 + (k/8)*2048 + (k%8)*16 + (m%8)*2 (M-group 128, K-group 2048)
    for (int e = t; e < 128 * 16; e += 128) {
        int m = e / 16, k = e % 16;
        int o = mode == 0 || mode == 3 ? (m / 8) * 256 + (k / 8) * 128 + (m % 8) * 16 + (k % 8) * 2
                                       : (m / 8) * 128 + (k / 8) * 2048 + (k % 8) * 16 + (m % 8) * 2;
        As[o / 2] = __float2bfloat16(aval(m, k));
    }
    // B K-major: core (n/8, k/8): (n/8)*256 + (k/8)*128 + (n%8)*16 + (k%8)*2
    for (int e = t; e < 64 * 16; e += 128) {
        int n = e / 16, k = e % 16;
        Bs[((n / 8) * 256 + (k / 8) * 128 + (n % 8) * 16 + (k % 8) * 2) / 2] = __float2bfloat16(n < N ? bval(n, k) : 0.f);
    }
    if (t < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 128;" ::"r"(sa(&tbase)));
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
    const int w = t / 32;
    if (mode == 3) {  // A row t -> TMEM lane t, columns 64..71 (k pairs packed low = even k)
        uint32_t r[8];
        for (int c = 0; c < 8; ++c) {
            __nv_bfloat162 p = __floats2bfloat162_rn(aval(t, 2 * c), aval(t, 2 * c + 1));
            r[c] = *reinterpret_cast<uint32_t *>(&p);
        }
        asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"r"(tm + ((uint32_t)(w * 32) << 16) + 64),
                     "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]));
        asm volatile("tcgen05.wait::st.sync.aligned;");
        asm volatile("tcgen05.fence::before_thread_sync;");
        __syncthreads();
        asm volatile("tcgen05.fence::after_thread_sync;");
    }
    if (t == 0) {
        const uint32_t id = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(mode == 1 || mode == 2) << 15) | ((uint32_t)(N >> 3) << 17) | ((128u >> 4) << 24);
        const uint64_t db = desc(sa(Bs), 128, 256);
        if (mode == 3) {
            asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\ttcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}"
                         ::"r"(tm), "r"(tm + 64), "l"(db), "r"(id), "r"(0));
        } else {
            const uint64_t da = mode == 0 ? desc(sa(As), 128, 256) : mode == 1 ? desc(sa(As), 2048, 128) : desc(sa(As), 128, 2048);
            asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\ttcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}"
                         ::"r"(tm), "l"(da), "l"(db), "r"(id), "r"(0));
        }
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(sa(&bar)));
    }
    uint32_t done = 0;
    while (!done)
        asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n\tselp.u32 %0, 1, 0, p;\n\t}" : "=r"(done) : "r"(sa(&bar)));
    asm volatile("tcgen05.fence::after_thread_sync;");
    uint32_t r[32];
    for (int h = 0; h < N / 32; ++h) {
        asm volatile("tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
                     : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]), "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
                     : "r"(tm + ((uint32_t)(w * 32) << 16) + 32 * h));
        asm volatile("tcgen05.wait::ld.sync.aligned;");
        for (int c = 0; c < 32; ++c) D[t * 64 + 32 * h + c] = __uint_as_float(r[c]);
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    if (t < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 128;" ::"r"(tm));
}
static float ha(int m, int k) { return (float)((m * 3 + k * 5) % 7 - 3); }
static float hb(int n, int k) { return (float)((n * 2 + k * 3) % 5 - 2); }
int main() {
    float *D;
    cudaMalloc(&D, 128 * 64 * 4);
    static float h[128 * 64];
    const char *names[] = {"A K-major smem", "A MN-major (LBO=K, SBO=M)", "A MN-major (LBO=M, SBO=K)", "A TMEM"};
    for (int mode = 0; mode < 4; mode += (mode == 1 ? 2 : 1))
        for (int N = 32; N <= 64; N += 32) {
            cudaMemset(D, 0, sizeof(h));
            probe<<<1, 128>>>(mode, N, D);
            cudaError_t e = cudaDeviceSynchronize();
            if (e != cudaSuccess) { printf("%s N=%d: %s\n", names[mode], N, cudaGetErrorString(e)); return 1; }
            cudaMemcpy(h, D, sizeof(h), cudaMemcpyDeviceToHost);
            int bad = 0;
            for (int m = 0; m < 128; ++m)
                for (int n = 0; n < N; ++n) {
                    float s = 0;
                    for (int k = 0; k < 16; ++k) s += ha(m, k) * hb(n, k);
                    bad += h[m * 64 + n] != s;
                }
            printf("%-28s N=%d: %d / %d wrong\n", names[mode], N, bad, 128 * N);
        }
    return 0;
}
