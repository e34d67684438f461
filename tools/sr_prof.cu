// Driver for the -DFS_SR_PROFILE build: k-means stream_red n=2^26 d=34 k=32; prints
// cycles per 16-row stage spent waiting for the TMA ring vs computing.
#include <cstdio>
#include <cuda_runtime.h>
#include "futseg.h"
extern "C" void fs_sr_prof_ptr(void **p);
__global__ void fill(float *v, int *k, long n, long w) {
    for (long i = blockIdx.x * (long)blockDim.x + threadIdx.x; i < n * w; i += (long)gridDim.x * blockDim.x) {
        v[i] = (i % 977) * 0.001f;
        if (i < n) k[i] = (int)((i * 2654435761ull >> 7) % 32);
    }
}
int main() {
    const long n = 1l << 26, w = 34, k = 32;
    float *v, *sums; int *keys, *cnt; void *ws;
    cudaMalloc(&v, n * w * 4); cudaMalloc(&keys, n * 4); cudaMalloc(&sums, k * w * 4); cudaMalloc(&cnt, k * 4);
    fill<<<4096, 256>>>(v, keys, n, w);
    size_t wb; fs_stream_red_workspace(FS_F32, n, w, k, &wb);
    cudaMalloc(&ws, wb); cudaMemset(ws, 0, wb);
    for (int i = 0; i < 3; ++i) fs_stream_red(FS_F32, v, keys, n, w, k, sums, cnt, ws, wb, nullptr);
    cudaDeviceSynchronize();
    void *sym; fs_sr_prof_ptr(&sym); cudaMemset(sym, 0, 64);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    cudaEventRecord(a);
    int st = fs_stream_red(FS_F32, v, keys, n, w, k, sums, cnt, ws, wb, nullptr);
    cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    unsigned long long z[8]; cudaMemcpy(z, sym, 64, cudaMemcpyDeviceToHost);
    printf("status %d %.3f ms  stages %llu  wait %.1f cyc/stage  compute %.1f cyc/stage\n", st, ms, z[0],
           (double)z[1] / z[0], (double)z[2] / z[0]);
}
