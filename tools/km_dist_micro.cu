// Microbenchmark: throughput of the k-means assignment (argmin over K centroids of a
// D-dim squared distance) on CUDA cores, centroids in constant memory, no HBM traffic.
//   V1 direct  sum (x-c)^2, scalar FADD + FFMA
//   V2 direct  sum (x-c)^2, two centroids per FADD2/FFMA2 (f32x2)
//   V3 expand  |c|^2 - 2 x.c, scalar FFMA
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o km_dist_micro tools/km_dist_micro.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
constexpr int K = 32, D = 34;
__constant__ float cc[K * D];
__constant__ float cc2[D * K];      // [j][c] (pairs adjacent)
__constant__ float cnorm[K];

__device__ __forceinline__ void load_x(float (&x)[D], int64_t i) {
#pragma unroll
    for (int j = 0; j < D; ++j) x[j] = __int_as_float(0x3f000000 | (((unsigned)i * 2654435761u + j * 40503u) & 0x7fffff));
}

template <int V> __global__ void __launch_bounds__(256) kern(int64_t n, int *out) {
    int64_t stride = (int64_t)gridDim.x * blockDim.x;
    int acc_idx = 0;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += stride) {
        float x[D];
        load_x(x, i);
        float best = 3.4e38f;
        int bi = 0;
        if constexpr (V == 1) {
#pragma unroll
            for (int c = 0; c < K; ++c) {
                float a = 0.f;
#pragma unroll
                for (int j = 0; j < D; ++j) { float t = __fsub_rn(x[j], cc[c * D + j]); a = __fmaf_rn(t, t, a); }
                if (a < best) { best = a; bi = c; }
            }
        } else if constexpr (V == 2) {
#pragma unroll
            for (int c = 0; c < K; c += 2) {
                unsigned long long a = 0;
#pragma unroll
                for (int j = 0; j < D; ++j) {
                    unsigned long long cp = *reinterpret_cast<const unsigned long long *>(&cc2[j * K + c]);
                    unsigned long long xx, t;
                    asm("mov.b64 %0, {%1, %1};" : "=l"(xx) : "f"(x[j]));
                    asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(t) : "l"(xx), "l"(cp));
                    asm("fma.rn.f32x2 %0, %1, %1, %2;" : "=l"(a) : "l"(t), "l"(a));
                }
                float a0 = __int_as_float((int)(a & 0xffffffffu)), a1 = __int_as_float((int)(a >> 32));
                if (a0 < best) { best = a0; bi = c; }
                if (a1 < best) { best = a1; bi = c + 1; }
            }
        } else {
#pragma unroll
            for (int c = 0; c < K; ++c) {
                float a = 0.f;
#pragma unroll
                for (int j = 0; j < D; ++j) a = __fmaf_rn(x[j], cc[c * D + j], a);
                a = __fmaf_rn(-2.f, a, cnorm[c]);
                if (a < best) { best = a; bi = c; }
            }
        }
        acc_idx += bi;
    }
    out[blockIdx.x * blockDim.x + threadIdx.x] = acc_idx;
}

int main() {
    float h[K * D], h2[D * K], hn[K];
    for (int c = 0; c < K; ++c) { hn[c] = 0; for (int j = 0; j < D; ++j) { h[c * D + j] = 0.5f + 0.01f * ((c * 7 + j * 3) % 50); h2[j * K + c] = h[c * D + j]; hn[c] += h[c*D+j]*h[c*D+j]; } }
    cudaMemcpyToSymbol(cc, h, sizeof h); cudaMemcpyToSymbol(cc2, h2, sizeof h2); cudaMemcpyToSymbol(cnorm, hn, sizeof hn);
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    int grid = sms * 8; int *out; cudaMalloc(&out, grid * 256 * 4);
    int64_t n = 1ll << 26;
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    void (*ks[3])(int64_t, int *) = {kern<1>, kern<2>, kern<3>};
    const char *names[3] = {"V1 direct scalar", "V2 direct f32x2", "V3 expand scalar"};
    for (int v = 0; v < 3; ++v) {
        for (int occ : {4, 8}) {
            ks[v]<<<sms * occ, 256>>>(n, out);
            cudaEventRecord(a);
            for (int r = 0; r < 5; ++r) ks[v]<<<sms * occ, 256>>>(n, out);
            cudaEventRecord(b); cudaEventSynchronize(b);
            float ms; cudaEventElapsedTime(&ms, a, b);
            printf("%s grid=%d*SM: %.3f ms per 2^26 points (%.1f G pair-dists/s)\n", names[v], occ, ms / 5, n * (double)K / (ms / 5 * 1e6));
        }
    }
    printf("%s\n", cudaGetErrorString(cudaGetLastError()));
}
