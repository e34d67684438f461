// Microbenchmark: legacy warp-level mma.sync throughput on sm_100a (tf32 m16n8k8 and
// bf16 m16n8k16), register operands, 8 independent accumulators per warp.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o mma_micro tools/mma_micro.cu
#include <cstdio>
#include <cuda_runtime.h>
template <int TF32> __global__ void __launch_bounds__(256) kern(int iters, float *out) {
    unsigned a[4], b[2];
    float acc[8][4];
    for (int i = 0; i < 4; ++i) a[i] = __float_as_uint(1.0f + threadIdx.x * 1e-3f + i);
    for (int i = 0; i < 2; ++i) b[i] = __float_as_uint(0.5f + i);
    for (int u = 0; u < 8; ++u) for (int i = 0; i < 4; ++i) acc[u][i] = 0.f;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int u = 0; u < 8; ++u) {
            if (TF32)
                asm volatile("mma.sync.aligned.m16n8k8.row.col.f32.tf32.tf32.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};"
                             : "+f"(acc[u][0]), "+f"(acc[u][1]), "+f"(acc[u][2]), "+f"(acc[u][3])
                             : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b[0]), "r"(b[1]));
            else
                asm volatile("mma.sync.aligned.m16n8k16.row.col.f32.bf16.bf16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};"
                             : "+f"(acc[u][0]), "+f"(acc[u][1]), "+f"(acc[u][2]), "+f"(acc[u][3])
                             : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b[0]), "r"(b[1]));
        }
    }
    float s = 0;
    for (int u = 0; u < 8; ++u) for (int i = 0; i < 4; ++i) s += acc[u][i];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
int main() {
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    float *out; cudaMalloc(&out, sms * 8 * 256 * 4);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    const int iters = 4096;
    for (int t = 0; t < 2; ++t) for (int occ : {2, 4, 8}) {
        auto k = t ? kern<1> : kern<0>;
        k<<<sms * occ, 256>>>(iters, out);
        cudaEventRecord(a); k<<<sms * occ, 256>>>(iters, out); cudaEventRecord(b); cudaEventSynchronize(b);
        float ms; cudaEventElapsedTime(&ms, a, b);
        double mmas = (double)sms * occ * 8 * iters * 8;  // warps * iters * 8
        double flop = mmas * (t ? 16 * 8 * 8 : 16 * 8 * 16) * 2;
        printf("%s CTAs=%d/SM: %.3f ms  %.1f TFLOP/s  %.2f cycles/mma/SMSP\n", t ? "tf32 m16n8k8 " : "bf16 m16n8k16", occ, ms,
               flop / ms / 1e9, (ms * 1e-3 * 1.965e9) / (mmas / (sms * 4)));
    }
    printf("%s\n", cudaGetErrorString(cudaGetLastError()));
}
