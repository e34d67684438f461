// umma_probe.cu -- pins the no-swizzle tcgen05 (kind::tf32) operand layouts on the device:
// D[128 x 32] = A[128 x 8] . B[8 x 32] with small integers, A and B stored K-major or
// MN-major as core matrices of 8 x 16 bytes, with the LBO / SBO roles tried both ways.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t sa(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t desc(uint32_t a, uint32_t lbo, uint32_t sbo) {
    return (uint64_t)((a >> 4) & 0x3FFF) | ((uint64_t)((lbo >> 4) & 0x3FFF) << 16) | ((uint64_t)((sbo >> 4) & 0x3FFF) << 32) | (1ull << 46);
}
// element (m, k) of A / (k, n) of B -> byte offset, for major = 0 (K) / 1 (MN)
// K-major : core (mn/8, k/4) ; inside: (mn%8)*16 + (k%4)*4 ; core strides: mn-group G_mn, k-chunk G_k
// MN-major: core (mn/4, k/8) ; inside: (k%8)*16 + (mn%4)*4
__device__ int off(int major, int mn, int k, int Gmn, int Gk) {
    if (major == 2) return (mn / 32) * Gmn + (k / 4) * Gk + (k % 4) * 128 + ((((mn % 32) / 8) ^ (k % 4)) * 32) + (mn % 8) * 4;
    if (major == 0) return (mn / 8) * Gmn + (k / 4) * Gk + (mn % 8) * 16 + (k % 4) * 4;
    return (mn / 4) * Gmn + (k / 8) * Gk + (k % 8) * 16 + (mn % 4) * 4;
}
__global__ void probe(int amaj, int bmaj, int aswap, int bswap, float *D, int agk) {
    __shared__ __align__(1024) float As[128 * 8 * 4];
    __shared__ __align__(1024) float Bs[32 * 8 * 4];
    __shared__ uint64_t bar;
    __shared__ uint32_t tbase;
    const int t = threadIdx.x;
    // strides: A K-major: mn-group 256 B (2 chunks of 128), k-chunk 128; MN-major: mn-group 128, k-group 4096
    int AGmn = amaj == 0 ? 256 : 128, AGk = amaj == 0 ? 128 : 4096;
    int BGmn = bmaj == 0 ? 256 : 128, BGk = bmaj == 0 ? 128 : 1024;
    if (amaj == 2) { AGmn = 512; AGk = agk; }      // 4 MN atoms of 512 B, K groups at agk
    if (bmaj == 2) { BGmn = 512; BGk = 512; }
    for (int e = t; e < 128 * 8; e += 128) {
        int m = e / 8, k = e % 8;
        As[off(amaj, m, k, AGmn, AGk) / 4] = (float)((m * 3 + k * 5) % 7 - 3);
    }
    for (int e = t; e < 32 * 8; e += 128) {
        int n = e / 8, k = e % 8;
        Bs[off(bmaj, n, k, BGmn, BGk) / 4] = (float)((n * 2 + k * 3) % 5 - 2);
    }
    if (t < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 32;" ::"r"(sa(&tbase)));
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
    if (t == 0) {
        // descriptor LBO/SBO: per the cute mapping (swap = 0) K-major: LBO = k-chunk stride, SBO = mn-group
        // stride; MN-major: LBO = k-group stride, SBO = mn-group stride.  swap = 1 exchanges them.
        uint32_t al = AGk, as_ = AGmn, bl = BGk, bs = BGmn;
        if (aswap) { uint32_t x = al; al = as_; as_ = x; }
        if (bswap) { uint32_t x = bl; bl = bs; bs = x; }
        const uint32_t id = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(amaj != 0) << 15) | ((uint32_t)(bmaj != 0) << 16) | ((32u >> 3) << 17) | ((128u >> 4) << 24);
        const uint64_t da = desc(sa(As), al, as_) | (amaj == 2 ? (1ull << 61) : 0ull);
        const uint64_t db = desc(sa(Bs), bl, bs) | (bmaj == 2 ? (1ull << 61) : 0ull);
        asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\ttcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}"
                     ::"r"(tm), "l"(da), "l"(db), "r"(id), "r"(0));
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(sa(&bar)));
    }
    uint32_t done = 0;
    while (!done)
        asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n\tselp.u32 %0, 1, 0, p;\n\t}" : "=r"(done) : "r"(sa(&bar)));
    asm volatile("tcgen05.fence::after_thread_sync;");
    const int w = t / 32;
    uint32_t r[32];
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]), "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
                 : "r"(tm + ((uint32_t)(w * 32) << 16)));
    asm volatile("tcgen05.wait::ld.sync.aligned;");
    for (int c = 0; c < 32; ++c) D[t * 32 + c] = __uint_as_float(r[c]);
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    if (t < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 32;" ::"r"(tm));
}

int main() {
    float *D;
    cudaMalloc(&D, 128 * 32 * 4);
    static float h[128 * 32];
    struct Cfg { int amaj, bmaj, as, bs, agk; };
    Cfg cfgs[] = {{0,0,0,0,0}, {2,0,0,0,2048}, {2,0,1,0,2048}, {0,2,0,0,0}, {0,2,0,1,0}, {2,2,0,0,2048}, {2,2,1,1,2048},
                  {2,0,0,0,1536}, {2,0,1,0,1536}, {2,2,0,0,1536}, {2,2,0,0,2560}};
    for (const Cfg &c : cfgs) {
        cudaMemset(D, 0, 128 * 32 * 4);
        probe<<<1, 128>>>(c.amaj, c.bmaj, c.as, c.bs, D, c.agk);
        cudaError_t e = cudaDeviceSynchronize();
        if (e != cudaSuccess) { printf("amaj=%d bmaj=%d: %s\n", c.amaj, c.bmaj, cudaGetErrorString(e)); return 1; }
        cudaMemcpy(h, D, sizeof(h), cudaMemcpyDeviceToHost);
        int bad = 0;
        for (int m = 0; m < 128; ++m)
            for (int n = 0; n < 32; ++n) {
                float s = 0;
                for (int k = 0; k < 8; ++k) s += (float)((m * 3 + k * 5) % 7 - 3) * (float)((n * 2 + k * 3) % 5 - 2);
                bad += h[m * 32 + n] != s;
            }
        printf("A %d B %d aswap=%d bswap=%d agk=%d : %d / 4096 wrong (D[0..3] = %g %g %g %g)\n", c.amaj, c.bmaj, c.as, c.bs, c.agk, bad, h[0], h[1], h[2], h[3]);
    }
    return 0;
}
