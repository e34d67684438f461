// exchange.cu -- the per-GPU halves of the cross-GPU combine: the
// partial results of a rank are packed into ONE buffer of one NCCL-reducible type, so that every
// exchange of the multi-GPU layer is a single collective, and unpacked after it.
//
//   ARGMIN (i32 / f32 values): key = order(value) << 32 | (uint32) index, stored as a signed int64
//     with the top bit flipped so that signed MIN order equals the lexicographic (value, index)
//     order of reading R3 (smaller value first, then the smaller index; index -1, "no element", is
//     the largest).  One all_reduce MIN of the keys is the exact cross-GPU argmin; unpack decodes.
//   ARGMIN (i64 values): a record [value, index] (two int64); an all_gather of the P records and
//     an unpack that folds them in rank order with R3's operator.
//   partials (stream_red / kmeans_step sums, counts and an optional extra count such as delta):
//     f32 sums -> f64 (exact), counts -> f64 (exact below 2^53); integer sums -> int64 (i32
//     sign-extended; the SUM is taken modulo 2^64 and unpacked to the low 32 bits: reading R1's
//     wrap-around, bit-exact).  One all_reduce SUM of the packed buffer.
//   copy_2d: a strided 2-D copy (the column-block gather of the distributed transpose).
#include <type_traits>

#include "internal.cuh"

namespace fs {

__device__ __forceinline__ uint32_t order_bits(float v) {  // monotone map of f32 (no NaN) to u32
    const uint32_t b = v == 0.f ? 0u : __float_as_uint(v);  // -0 == +0 (R3 compares values)
    return (b & 0x80000000u) ? ~b : (b | 0x80000000u);
}
__device__ __forceinline__ float from_order_bits(uint32_t u) {
    return __uint_as_float((u & 0x80000000u) ? (u & 0x7FFFFFFFu) : ~u);
}
__device__ __forceinline__ uint32_t order_bits(int32_t v) { return (uint32_t)v ^ 0x80000000u; }

template <typename T>
__global__ void argmin_pack_kernel(const T *val, const int64_t *idx, int64_t n, int64_t *key) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        if constexpr (sizeof(T) == 8) {
            key[2 * i] = (int64_t)val[i];
            key[2 * i + 1] = idx[i];
        } else {
            // index -1 ("no element", R3's neutral) is the largest key whatever its value
            const uint64_t u = idx[i] < 0 ? ~0ull : ((uint64_t)order_bits(val[i]) << 32) | (uint64_t)(uint32_t)idx[i];
            key[i] = (int64_t)(u ^ 0x8000000000000000ull);
        }
    }
}

template <typename T>
__global__ void argmin_unpack_kernel(const int64_t *key, int64_t P, T *val, int64_t *idx) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    if constexpr (sizeof(T) == 8) {  // fold P records in rank order: (value, index) lexicographic, -1 = none
        int64_t bv = INT64_MAX, bi = -1;
        for (int64_t p = 0; p < P; ++p) {
            const int64_t v = key[2 * p], i = key[2 * p + 1];
            if (i < 0) continue;
            if (bi < 0 || v < bv || (v == bv && i < bi)) {
                bv = v;
                bi = i;
            }
        }
        *val = (T)bv;
        *idx = bi;
    } else {
        const uint64_t u = (uint64_t)key[0] ^ 0x8000000000000000ull;
        const uint32_t lo = (uint32_t)u;
        *idx = lo == 0xFFFFFFFFu ? -1 : (int64_t)lo;
        if constexpr (std::is_same<T, float>::value)
            *val = lo == 0xFFFFFFFFu ? __int_as_float(0x7f800000) : from_order_bits((uint32_t)(u >> 32));
        else
            *val = lo == 0xFFFFFFFFu ? INT32_MAX : (int32_t)((uint32_t)(u >> 32) ^ 0x80000000u);
    }
}

template <typename T>
__global__ void partials_pack_kernel(const T *sums, const int32_t *counts, const int64_t *extra, int64_t kw,
                                     int64_t k, void *packed) {
    const int64_t tot = kw + k + 1;
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < tot; e += (int64_t)gridDim.x * blockDim.x) {
        if constexpr (std::is_same<T, float>::value) {
            double *p = (double *)packed;
            p[e] = e < kw ? (double)sums[e] : (e < kw + k ? (counts ? (double)counts[e - kw] : 0.0)
                                                          : (extra ? (double)*extra : 0.0));
        } else {
            int64_t *p = (int64_t *)packed;
            p[e] = e < kw ? (int64_t)sums[e] : (e < kw + k ? (counts ? (int64_t)counts[e - kw] : 0) : (extra ? *extra : 0));
        }
    }
}

template <typename T>
__global__ void partials_unpack_kernel(const void *packed, int64_t kw, int64_t k, T *sums, int32_t *counts,
                                       int64_t *extra) {
    const int64_t tot = kw + k + 1;
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < tot; e += (int64_t)gridDim.x * blockDim.x) {
        if constexpr (std::is_same<T, float>::value) {
            const double v = ((const double *)packed)[e];
            if (e < kw) sums[e] = (float)v;
            else if (e < kw + k) { if (counts) counts[e - kw] = (int32_t)(int64_t)v; }
            else if (extra) *extra = (int64_t)v;
        } else {
            const int64_t v = ((const int64_t *)packed)[e];
            if (e < kw) sums[e] = (T)v;  // i32: the low 32 bits (sum modulo 2^32)
            else if (e < kw + k) { if (counts) counts[e - kw] = (int32_t)v; }
            else if (extra) *extra = v;
        }
    }
}

// dst[r * dld + c] = src[r * sld + c] for r < rows, c < cols, elements of eb bytes (4 or 8);
// 16-byte vectors when every row start is 16-byte aligned
template <typename W>
__global__ void copy_2d_kernel(const W *src, int64_t sld, int64_t rows, int64_t cols, W *dst, int64_t dld) {
    for (int64_t r = blockIdx.y; r < rows; r += gridDim.y)
        for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c < cols; c += (int64_t)gridDim.x * blockDim.x)
            dst[r * dld + c] = src[r * sld + c];
}

static int grid_for(int64_t n) {
    int64_t g = ceil_div(n > 0 ? n : 1, 256);
    return (int)(g > 4096 ? 4096 : g);
}

fs_status argmin_pack_run(int dt, const void *val, const int64_t *idx, int64_t n, int64_t *key, cudaStream_t st) {
    if (n == 0) return FS_OK;
    switch (dt) {
    case FS_I32: argmin_pack_kernel<int32_t><<<grid_for(n), 256, 0, st>>>((const int32_t *)val, idx, n, key); break;
    case FS_I64: argmin_pack_kernel<int64_t><<<grid_for(n), 256, 0, st>>>((const int64_t *)val, idx, n, key); break;
    default: argmin_pack_kernel<float><<<grid_for(n), 256, 0, st>>>((const float *)val, idx, n, key); break;
    }
    return launch_status();
}

fs_status argmin_unpack_run(int dt, const int64_t *key, int64_t P, void *val, int64_t *idx, cudaStream_t st) {
    switch (dt) {
    case FS_I32: argmin_unpack_kernel<int32_t><<<1, 32, 0, st>>>(key, P, (int32_t *)val, idx); break;
    case FS_I64: argmin_unpack_kernel<int64_t><<<1, 32, 0, st>>>(key, P, (int64_t *)val, idx); break;
    default: argmin_unpack_kernel<float><<<1, 32, 0, st>>>(key, P, (float *)val, idx); break;
    }
    return launch_status();
}

fs_status partials_pack_run(int dt, const void *sums, const int32_t *counts, const int64_t *extra, int64_t kw,
                            int64_t k, void *packed, cudaStream_t st) {
    const int g = grid_for(kw + k + 1);
    switch (dt) {
    case FS_I32: partials_pack_kernel<int32_t><<<g, 256, 0, st>>>((const int32_t *)sums, counts, extra, kw, k, packed); break;
    case FS_I64: partials_pack_kernel<int64_t><<<g, 256, 0, st>>>((const int64_t *)sums, counts, extra, kw, k, packed); break;
    default: partials_pack_kernel<float><<<g, 256, 0, st>>>((const float *)sums, counts, extra, kw, k, packed); break;
    }
    return launch_status();
}

fs_status partials_unpack_run(int dt, const void *packed, int64_t kw, int64_t k, void *sums, int32_t *counts,
                              int64_t *extra, cudaStream_t st) {
    const int g = grid_for(kw + k + 1);
    switch (dt) {
    case FS_I32: partials_unpack_kernel<int32_t><<<g, 256, 0, st>>>(packed, kw, k, (int32_t *)sums, counts, extra); break;
    case FS_I64: partials_unpack_kernel<int64_t><<<g, 256, 0, st>>>(packed, kw, k, (int64_t *)sums, counts, extra); break;
    default: partials_unpack_kernel<float><<<g, 256, 0, st>>>(packed, kw, k, (float *)sums, counts, extra); break;
    }
    return launch_status();
}

fs_status copy_2d_run(int eb, const void *src, int64_t sld, int64_t rows, int64_t cols, void *dst, int64_t dld,
                      cudaStream_t st) {
    if (rows == 0 || cols == 0) return FS_OK;
    const int64_t bytes = cols * eb;
    const bool v16 = ((uintptr_t)src % 16 == 0) && ((uintptr_t)dst % 16 == 0) && (sld * eb) % 16 == 0 &&
                     (dld * eb) % 16 == 0 && bytes % 16 == 0;
    dim3 grid;
    if (v16) {
        const int64_t w = bytes / 16;
        grid = dim3((unsigned)ceil_div(w, 256) > 64u ? 64u : (unsigned)ceil_div(w, 256),
                    (unsigned)(rows > 65535 ? 65535 : rows));
        copy_2d_kernel<int4><<<grid, 256, 0, st>>>((const int4 *)src, sld * eb / 16, rows, w, (int4 *)dst, dld * eb / 16);
    } else if (eb == 8) {
        grid = dim3((unsigned)ceil_div(cols, 256) > 64u ? 64u : (unsigned)ceil_div(cols, 256),
                    (unsigned)(rows > 65535 ? 65535 : rows));
        copy_2d_kernel<int64_t><<<grid, 256, 0, st>>>((const int64_t *)src, sld, rows, cols, (int64_t *)dst, dld);
    } else {
        grid = dim3((unsigned)ceil_div(cols, 256) > 64u ? 64u : (unsigned)ceil_div(cols, 256),
                    (unsigned)(rows > 65535 ? 65535 : rows));
        copy_2d_kernel<int32_t><<<grid, 256, 0, st>>>((const int32_t *)src, sld, rows, cols, (int32_t *)dst, dld);
    }
    return launch_status();
}

}  // namespace fs
