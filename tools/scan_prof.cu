// Standalone driver for the -DFS_SCAN_PROFILE build of scan.cu: runs the f32 add
// scan over 2^28 elements and prints cycles per phase per iteration.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -DFS_SCAN_PROFILE \
//        -Iinclude -Ipaper_conf_pldi_henriksenseho17_b200/csrc tools/scan_prof.cu \
//        paper_conf_pldi_henriksenseho17_b200/csrc/{scan,api,redomap,colreduce,seg_reduce,stream_red,transpose}.cu -o scan_prof
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>
#include "futseg.h"
extern "C" void fs_scan_prof_ptr(void **p);

int main() {
    const int64_t n = 1ll << 28;
    float *x, *y; void *ws;
    cudaMalloc(&x, n * 4); cudaMalloc(&y, n * 4);
    cudaMemset(x, 0, n * 4);
    fs_opdesc op = {FS_ADD, FS_F32, 1};
    fs_mapdesc m = {FS_MAP_ID, 0, 0, 0};
    size_t wb; fs_scanomap_workspace(op, n, &wb);
    cudaMalloc(&ws, wb); cudaMemset(ws, 0, wb);
    const int64_t L = getenv("SEGLEN") ? atoll(getenv("SEGLEN")) : 0;
    auto run = [&]() {
        return L ? fs_seg_scan(op, x, n / L, L, FS_ROW_MAJOR, y, nullptr, ws, wb, nullptr)
                 : fs_scanomap(op, m, x, nullptr, n, y, nullptr, nullptr, nullptr, ws, wb, nullptr);
    };
    for (int i = 0; i < 3; ++i) run();
    cudaDeviceSynchronize();
    unsigned long long z[16] = {0};
    void *sym = nullptr; fs_scan_prof_ptr(&sym); cudaMemset(sym, 0, sizeof(z));
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    cudaEventRecord(a);
    int st = run();
    cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    cudaMemcpy(z, sym, sizeof(z), cudaMemcpyDeviceToHost);
    printf("status %d (%s) time %.3f ms  iterations %llu\n", st, cudaGetErrorString(cudaGetLastError()), ms, z[0]);
    const char *names[] = {"iters", "A: wait+reduce+publish", "C: wait+local scan", "C: look-back", "C: write",
                           "look-back steps"};
    for (int i = 1; i < 6; ++i) printf("%-20s %10.1f cycles/iter\n", names[i], (double)z[i] / (double)z[0]);
    return 0;
}
