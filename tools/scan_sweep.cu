// Standalone timing driver for scan.cu build-time knobs (tools/scan_sweep.sh):
// scanomap f32/i32 add over 2^28 and seg_scan f32 add (L = 1024, 33, 2^20),
// CUDA-event device time, median of 9 after 3 warm-ups; spot-checks the result.
#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <cuda_runtime.h>
#include "futseg.h"

int main(int argc, char **argv) {
    const char *tag = argc > 1 ? argv[1] : "default";
    const int64_t n = 1ll << 28;
    float *x, *y;
    void *ws;
    cudaMalloc(&x, n * 4);
    cudaMalloc(&y, n * 4);
    std::vector<float> h(1 << 20);
    for (size_t i = 0; i < h.size(); ++i) h[i] = (float)((i * 2654435761u) % 1000) / 1000.0f;
    for (int64_t o = 0; o < n; o += h.size()) cudaMemcpy(x + o, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
    size_t wb;
    fs_opdesc f32 = {FS_ADD, FS_F32, 1}, i32 = {FS_ADD, FS_I32, 1};
    fs_scanomap_workspace(f32, n, &wb);
    cudaMalloc(&ws, wb);
    cudaMemset(ws, 0, wb);
    fs_mapdesc m = {FS_MAP_ID, 0, 0, 0};
    struct Case { const char *name; int64_t L; fs_opdesc op; };
    Case cases[] = {{"scan_f32", 0, f32}, {"scan_i32", 0, i32}, {"seg_f32_L1024", 1024, f32},
                    {"seg_f32_L33", 33, f32}, {"seg_f32_L1M", 1 << 20, f32}};
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    printf("{\"tag\": \"%s\"", tag);
    for (auto &c : cases) {
        const int64_t nn = c.L ? (n / c.L) * c.L : n;
        auto run = [&]() {
            return c.L ? fs_seg_scan(c.op, x, nn / c.L, c.L, FS_ROW_MAJOR, y, nullptr, ws, wb, nullptr)
                       : fs_scanomap(c.op, m, x, nullptr, nn, y, nullptr, nullptr, nullptr, ws, wb, nullptr);
        };
        std::vector<float> t;
        int st = 0;
        for (int i = 0; i < 12; ++i) {
            cudaEventRecord(a);
            st |= run();
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms;
            cudaEventElapsedTime(&ms, a, b);
            if (i >= 3) t.push_back(ms);
        }
        std::sort(t.begin(), t.end());
        // spot check: last element of the first segment / of the whole scan (f32 only)
        double ok = 1;
        if (c.op.dtype == FS_F32) {
            const int64_t len = c.L ? c.L : nn;
            const int64_t chk = len < (1 << 22) ? len : (1 << 22);
            std::vector<float> yy(chk);
            cudaMemcpy(yy.data(), y, chk * 4, cudaMemcpyDeviceToHost);
            double s = 0;
            for (int64_t i = 0; i < chk; ++i) {
                s += h[i % h.size()];
                if (std::abs(yy[i] - s) > 1e-4 * s + 1e-6) { ok = 0; break; }
            }
        }
        printf(", \"%s\": {\"ms\": %.4f, \"GB_s\": %.1f, \"status\": %d, \"ok\": %d}", c.name, t[t.size() / 2],
               8.0 * nn / (t[t.size() / 2] * 1e6), st, (int)ok);
    }
    printf(", \"err\": \"%s\"}\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
