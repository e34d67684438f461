// internal.cuh -- host-side helpers shared by the kernel translation units and
// the C ABI (api.cu): device properties, occupancy-derived grid sizes, the
// (op, dtype) template dispatcher, and the per-primitive launchers.
#pragma once

#include <cuda_runtime.h>
#include <stddef.h>
#include <stdint.h>

#include "common.cuh"

namespace fs {

int sm_count();  // SMs of the current device (cached per device)
int max_blocks_per_sm(const void *kernel, int threads, size_t dyn_smem);  // cached
inline int resident_blocks(const void *kernel, int threads, size_t smem = 0) {
    return sm_count() * max_blocks_per_sm(kernel, threads, smem);
}
int forced_seg_regime();  // -1 = automatic
void note_regime(int r);   // the segmented regime the current call launched (fs_last_seg_regime)

// Segmented-regime IDs (include/futseg.h FS_REGIME_*): the one numbering shared by the
// dispatchers, fs_seg_regime and fs_last_seg_regime.
enum {
    RG_KG1 = 0, RG_KG2 = 1, RG_KG3 = 2, RG_KG4 = 3, RG_COL = 4, RG_KS_LOOKBACK = 5, RG_EMPTY = 6,
    RG_KS0 = 7, RG_KS1 = 8, RG_KS2 = 9, RG_KS0_BIG = 10, RG_KS3 = 11, RG_FLAT_ROW = 12
};
// Row-major seg_scan regime for n = nseg * L elements (nseg >= 1, L >= 1): the single plan both
// ScanRun (scan.cu) and fs_seg_regime use.  al16: in and out 16-byte aligned; co16: in and out
// share their 16-byte phase; elem: in and out aligned to the element size; plain: no carry-in
// and ibase 0 (every seg_scan call).
int seg_scan_plan(int op, int dt, int64_t n, int64_t L, bool al16, bool co16, bool elem, bool plain);

void note_launches(int n);  // counts kernels launched by this library (fs_launch_count)
inline fs_status launch_status(int kernels = 1) {
    note_launches(kernels);
    return cudaGetLastError() == cudaSuccess ? FS_OK : FS_ERR_CUDA;
}

inline int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

// (op, dtype) -> F<OP, T>::run(args...).  ops limited to ADD/MIN/MAX/ARGMIN.
template <template <int, typename> class F, typename T, typename... A>
fs_status dispatch_op(int op, A... a) {
    switch (op) {
    case FS_ADD: return F<kAdd, T>::run(a...);
    case FS_MIN: return F<kMin, T>::run(a...);
    case FS_MAX: return F<kMax, T>::run(a...);
    case FS_ARGMIN: return F<kArgmin, T>::run(a...);
    }
    return FS_ERR_UNSUPPORTED;
}
template <template <int, typename> class F, typename... A>
fs_status dispatch(int op, int dt, A... a) {
    switch (dt) {
    case FS_I32: return dispatch_op<F, int32_t>(op, a...);
    case FS_I64: return dispatch_op<F, int64_t>(op, a...);
    case FS_F32: return dispatch_op<F, float>(op, a...);
    }
    return FS_ERR_UNSUPPORTED;
}

inline size_t dtype_size(int dt) { return dt == FS_I64 ? 8 : 4; }
// bytes of one accumulator V for (op, dt)
inline size_t acc_size(int op, int dt) { return op == FS_ARGMIN ? 16 : dtype_size(dt); }

// ---- launchers (one per translation unit); arguments already validated ----
// redomap.cu
size_t redomap_ws(int op, int dt, int64_t n, bool nn);
fs_status redomap_run(int op, int dt, const fs_mapdesc &map, const void *in0, const void *in1, int64_t n,
                      void *out, int64_t *out_idx, void *ws, cudaStream_t st);
fs_status combine_run(int op, int dt, int64_t width, const void *parts, const int64_t *part_idx, int64_t P,
                      void *out, int64_t *out_idx, cudaStream_t st);
// colreduce.cu  ([m][w] row-major -> [w], any op; index = row)
size_t colreduce_ws(int op, int dt, int64_t m, int64_t w);
fs_status colreduce_run(int op, int dt, const void *in, int64_t m, int64_t w, void *out, int64_t *out_idx,
                        void *ws, cudaStream_t st);
// seg_reduce.cu (row-major regimes)
int seg_reduce_regime(int op, int dt, int64_t nseg, int64_t seglen);
size_t seg_reduce_ws(int op, int dt, int64_t nseg, int64_t seglen);
fs_status seg_reduce_run(int op, int dt, const void *in, int64_t nseg, int64_t seglen, void *out,
                         int64_t *out_idx, void *ws, cudaStream_t st);
fs_status fill_neutral_run(int op, int dt, int64_t count, void *out, int64_t *out_idx, cudaStream_t st);
// scan.cu
size_t scan_ws(int op, int dt, int64_t n);
fs_status scan_run(int op, int dt, const fs_mapdesc &map, const void *in0, const void *in1, int64_t n,
                   int64_t seglen, void *out, int64_t *out_idx, const void *carry, const int64_t *carry_idx,
                   void *ws, cudaStream_t st);
size_t colscan_ws(int op, int dt, int64_t m, int64_t w);
fs_status colscan_run(int op, int dt, const void *in, int64_t m, int64_t w, void *out, int64_t *out_idx,
                      void *ws, cudaStream_t st);
// stream_red.cu
size_t stream_red_ws(int dt, int64_t n, int64_t w, int64_t k);
fs_status stream_red_run(int dt, const void *vals, const int32_t *keys, int64_t n, int64_t w, int64_t k,
                         void *sums, int32_t *counts, void *ws, cudaStream_t st);
// knn.cu (NEXT-2)
size_t knn_ws(int64_t n);
fs_status knn_run(const float *lat, const float *lng, int64_t n, float q0, float q1, int64_t kk, float *out_dist,
                  int64_t *out_idx, void *ws, cudaStream_t st);
// kmeans.cu (NEXT-1)
size_t kmeans_ws(int64_t n, int64_t d, int64_t k);
fs_status kmeans_run(const float *pts, int64_t n, int64_t d, const float *cen, int64_t k, const int32_t *prev,
                     int32_t *membership, float *sums, int32_t *counts, float *new_cen, int64_t *delta, void *ws,
                     cudaStream_t st);
// seg_map_reduce.cu (NEXT-4)
size_t seg_map_reduce_ws(int op, int dt, int64_t nseg, int64_t L);
fs_status seg_map_reduce_run(int op, int dt, const void *in, int64_t nseg, int64_t L, int64_t ci, float cf, void *ymap,
                             void *out, int64_t *out_idx, void *ws, cudaStream_t st);
// scan_reduce.cu (NEXT-3)
size_t scan_reduce_ws(int dt);
fs_status scan_reduce_run(int red, int dt, const void *x, int64_t n, void *out, void *ws, cudaStream_t st);
fs_status kmeans_finish_run(const float *sums, const int32_t *counts, const float *cen, int64_t k, int64_t d,
                            float *new_cen, cudaStream_t st);
// exchange.cu (the multi-GPU layer's one-collective exchanges)
fs_status argmin_pack_run(int dt, const void *val, const int64_t *idx, int64_t n, int64_t *key, cudaStream_t st);
fs_status argmin_unpack_run(int dt, const int64_t *key, int64_t P, void *val, int64_t *idx, cudaStream_t st);
fs_status partials_pack_run(int dt, const void *sums, const int32_t *counts, const int64_t *extra, int64_t kw,
                            int64_t k, void *packed, cudaStream_t st);
fs_status partials_unpack_run(int dt, const void *packed, int64_t kw, int64_t k, void *sums, int32_t *counts,
                              int64_t *extra, cudaStream_t st);
fs_status copy_2d_run(int eb, const void *src, int64_t sld, int64_t rows, int64_t cols, void *dst, int64_t dld,
                      cudaStream_t st);
// transpose.cu
fs_status transpose_run(int dt, const void *in, int64_t rows, int64_t cols, void *out, cudaStream_t st);

}  // namespace fs
