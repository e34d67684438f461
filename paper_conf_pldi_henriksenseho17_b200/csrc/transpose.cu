// transpose.cu -- KT1: out[j][i] = in[i][j]  (rearrange (1,0), L1389-1393; the
// manifest transposition behind as_column_major, L1426-1434, and G5's
// "at the expense of transposing the input", L1380-1381).
//
// A CTA moves a TILE x TILE block: coalesced row reads of the input into shared
// memory, then coalesced row writes of the output read down the shared tile's
// columns.  The shared tile is padded by one element per row so column reads
// hit 32 distinct banks.  Pure data movement: 2 x 4 (or 8) bytes per element.
#include "internal.cuh"

namespace fs {

constexpr int kTile = 32;
constexpr int kRowsPerPass = 8;

template <typename T>
__global__ void __launch_bounds__(kTile *kRowsPerPass)
transpose_kernel(const T *__restrict__ in, int64_t rows, int64_t cols, T *__restrict__ out,
                 int64_t tiles_c, int64_t ntiles) {
    __shared__ T tile[kTile][kTile + 1];
    const int tx = threadIdx.x, ty = threadIdx.y;
    for (int64_t tt = blockIdx.x; tt < ntiles; tt += gridDim.x) {
        const int64_t tr = tt / tiles_c, tc = tt - tr * tiles_c;
        const int64_t r0 = tr * kTile, c0 = tc * kTile;
        const int64_t c = c0 + tx;
        if (r0 + kTile <= rows && c0 + kTile <= cols) {
#pragma unroll
            for (int k = 0; k < kTile; k += kRowsPerPass) tile[ty + k][tx] = __ldg(in + (r0 + ty + k) * cols + c);
            __syncthreads();
#pragma unroll
            for (int k = 0; k < kTile; k += kRowsPerPass) out[(c0 + ty + k) * rows + r0 + tx] = tile[tx][ty + k];
        } else {
#pragma unroll
            for (int k = 0; k < kTile; k += kRowsPerPass)
                if (r0 + ty + k < rows && c < cols) tile[ty + k][tx] = __ldg(in + (r0 + ty + k) * cols + c);
            __syncthreads();
#pragma unroll
            for (int k = 0; k < kTile; k += kRowsPerPass)
                if (c0 + ty + k < cols && r0 + tx < rows) out[(c0 + ty + k) * rows + r0 + tx] = tile[tx][ty + k];
        }
        __syncthreads();
    }
}

template <typename T>
static fs_status transpose_t(const void *in, int64_t rows, int64_t cols, void *out, cudaStream_t st) {
    const int64_t tiles_r = ceil_div(rows, kTile), tiles_c = ceil_div(cols, kTile);
    const int64_t ntiles = tiles_r * tiles_c;
    if (ntiles == 0) return FS_OK;
    const int64_t cap = resident_blocks((const void *)transpose_kernel<T>, kTile * kRowsPerPass) * 4;
    const int64_t grid = ntiles < cap ? ntiles : cap;
    transpose_kernel<T><<<(unsigned)grid, dim3(kTile, kRowsPerPass), 0, st>>>(
        (const T *)in, rows, cols, (T *)out, tiles_c, ntiles);
    return launch_status();
}

fs_status transpose_run(int dt, const void *in, int64_t rows, int64_t cols, void *out, cudaStream_t st) {
    return dt == FS_I64 ? transpose_t<int64_t>(in, rows, cols, out, st) : transpose_t<int32_t>(in, rows, cols, out, st);
}

}  // namespace fs
