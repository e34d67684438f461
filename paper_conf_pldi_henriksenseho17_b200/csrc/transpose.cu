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

// 64 x 64 tiles, 256 threads, 16-byte vector loads and stores: each input row
// segment and each output row segment a CTA touches is 256 B (4-byte
// elements) / 512 B (8-byte) contiguous, so DRAM sees long runs on both sides.
// Shared memory is padded by one element per row; the transposed gather reads
// conflict at most 2-way.
constexpr int kTT = 64;            // tile edge (elements)
constexpr int kTThreads = 256;

template <typename T>
__global__ void __launch_bounds__(kTThreads)
transpose_kernel(const T *__restrict__ in, int64_t rows, int64_t cols, T *__restrict__ out, int64_t tiles_c,
                 int64_t ntiles) {
    constexpr int VEC = 16 / sizeof(T);
    constexpr int VPR = kTT / VEC;            // vectors per tile row
    constexpr int RPP = kTThreads / VPR;      // tile rows per pass
    __shared__ T tile[kTT][kTT + 1];
    const int t = threadIdx.x;
    const int vc = t % VPR, rr = t / VPR;
    for (int64_t tt = blockIdx.x; tt < ntiles; tt += gridDim.x) {
        const int64_t tr = tt / tiles_c, tc = tt - tr * tiles_c;
        const int64_t r0 = tr * kTT, c0 = tc * kTT;
        const bool interior = r0 + kTT <= rows && c0 + kTT <= cols && ((cols * sizeof(T)) & 15) == 0 &&
                              ((rows * sizeof(T)) & 15) == 0 && (((uintptr_t)in | (uintptr_t)out) & 15) == 0;
        if (interior) {
            int4 v[kTT / RPP];
#pragma unroll
            for (int p = 0; p < kTT / RPP; ++p)
                v[p] = ldg16(in + (r0 + rr + p * RPP) * cols + c0 + vc * VEC);
#pragma unroll
            for (int p = 0; p < kTT / RPP; ++p) {
                const Vec16<T> e = as_vec<T>(v[p]);
#pragma unroll
                for (int k = 0; k < VEC; ++k) tile[rr + p * RPP][vc * VEC + k] = e.e[k];
            }
            __syncthreads();
#pragma unroll
            for (int p = 0; p < kTT / RPP; ++p) {
                const int j = rr + p * RPP;  // output row within the tile (= input column)
                Vec16<T> o;
#pragma unroll
                for (int k = 0; k < VEC; ++k) o.e[k] = tile[vc * VEC + k][j];
                int4 ov;
                memcpy(&ov, &o, 16);
                *reinterpret_cast<int4 *>(out + (c0 + j) * rows + r0 + vc * VEC) = ov;
            }
        } else {
            for (int e = t; e < kTT * kTT; e += kTThreads) {
                const int i = e / kTT, j = e % kTT;
                if (r0 + i < rows && c0 + j < cols) tile[i][j] = in[(r0 + i) * cols + c0 + j];
            }
            __syncthreads();
            for (int e = t; e < kTT * kTT; e += kTThreads) {
                const int j = e / kTT, i = e % kTT;
                if (c0 + j < cols && r0 + i < rows) out[(c0 + j) * rows + r0 + i] = tile[i][j];
            }
        }
        __syncthreads();
    }
}

template <typename T>
static fs_status transpose_t(const void *in, int64_t rows, int64_t cols, void *out, cudaStream_t st) {
    const int64_t tiles_r = ceil_div(rows, kTT), tiles_c = ceil_div(cols, kTT);
    const int64_t ntiles = tiles_r * tiles_c;
    if (ntiles == 0) return FS_OK;
    const int64_t cap = resident_blocks((const void *)transpose_kernel<T>, kTThreads) * 8;
    const int64_t grid = ntiles < cap ? ntiles : cap;
    transpose_kernel<T><<<(unsigned)grid, kTThreads, 0, st>>>((const T *)in, rows, cols, (T *)out, tiles_c, ntiles);
    return launch_status();
}

fs_status transpose_run(int dt, const void *in, int64_t rows, int64_t cols, void *out, cudaStream_t st) {
    return dt == FS_I64 ? transpose_t<int64_t>(in, rows, cols, out, st) : transpose_t<int32_t>(in, rows, cols, out, st);
}

}  // namespace fs
