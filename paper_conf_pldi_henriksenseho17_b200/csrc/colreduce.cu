// colreduce.cu -- reduce with a vectorised operator over the rows of an
// [m][w] row-major array:  out[c] = x[0][c] (+) x[1][c] (+) ... (+) x[m-1][c].
//
// This is  reduce (map (+)) (replicate w 0(+))  (Fig 4b), i.e. the
// FS_VADD redomap, and -- by rule G5 (L1313-1319, L1375-1383) and the
// column-major representation of Sec. 5.2 (L1426-1434) -- also seg_reduce of
// an FS_COL_MAJOR [nseg][seglen] array (m = seglen rows of w = nseg columns):
// each thread owns a column (vector of columns) and walks down the rows, so
// consecutive threads read consecutive addresses (coalescing by
// transposition, without materialising the transpose).
//
// Grid: x = column tiles (CG vector-columns of VEC elements per CTA), y = row
// splits.  Threads of a CTA are (row-offset, vector-column) pairs, so narrow
// arrays (w = 5, 34, ...) still give every thread a coalesced load.  With
// several row splits, each CTA writes a partial row and the last CTA of a
// column tile (per-tile ticket) combines them in split order.
#include "internal.cuh"

namespace fs {

constexpr int kColThreads = 256;

template <int OP, typename T, int NT, int VEC, int U>
__global__ void __launch_bounds__(NT)
colreduce_kernel(const T *__restrict__ x, int64_t m, int64_t w, int CG, int64_t rows_per_split,
                 typename Op<OP, T>::V *partials, unsigned *tickets, T *out, int64_t *out_idx) {
    using O = Op<OP, T>;
    using V = typename O::V;
    __shared__ V part[NT * VEC];
    __shared__ bool last;
    const int t = threadIdx.x;
    const int RB = NT / CG;  // row offsets per CTA
    const int TCW = CG * VEC;  // columns per tile
    const int64_t col0 = (int64_t)blockIdx.x * TCW;
    const int64_t r0 = (int64_t)blockIdx.y * rows_per_split;
    const int64_t r1 = r0 + rows_per_split < m ? r0 + rows_per_split : m;

    V acc[VEC];
#pragma unroll
    for (int k = 0; k < VEC; ++k) acc[k] = O::id();
    const int cg = t % CG, roff = t / CG;
    const int64_t c = col0 + (int64_t)cg * VEC;
    if (roff < RB && c < w) {
        const T *base = x + c;
        int64_t r = r0 + roff;
        if (VEC > 1) {
            for (; r + (int64_t)(U - 1) * RB < r1; r += (int64_t)U * RB) {
                int4 v[U];
#pragma unroll
                for (int u = 0; u < U; ++u) v[u] = ldg16(base + (r + (int64_t)u * RB) * w);
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    const Vec16<T> e = as_vec<T>(v[u]);
#pragma unroll
                    for (int k = 0; k < VEC; ++k) acc[k] = O::fold(acc[k], e.e[k], r + (int64_t)u * RB);
                }
            }
            for (; r < r1; r += RB) {
                const Vec16<T> e = as_vec<T>(ldg16(base + r * w));
#pragma unroll
                for (int k = 0; k < VEC; ++k) acc[k] = O::fold(acc[k], e.e[k], r);
            }
        } else {
            for (; r + (int64_t)(U - 1) * RB < r1; r += (int64_t)U * RB) {
                T v[U];
#pragma unroll
                for (int u = 0; u < U; ++u) v[u] = __ldg(base + (r + (int64_t)u * RB) * w);
#pragma unroll
                for (int u = 0; u < U; ++u) acc[0] = O::fold(acc[0], v[u], r + (int64_t)u * RB);
            }
            for (; r < r1; r += RB) acc[0] = O::fold(acc[0], __ldg(base + r * w), r);
        }
    }
    // combine the RB row offsets of each column, in row-offset order
    if (roff < RB) {
#pragma unroll
        for (int k = 0; k < VEC; ++k) part[roff * TCW + cg * VEC + k] = acc[k];
    }
    __syncthreads();
    const bool single = gridDim.y == 1;
    for (int cc = t; cc < TCW; cc += NT) {
        V a = O::id();
        for (int q = 0; q < RB; ++q) a = O::comb(a, part[q * TCW + cc]);
        const int64_t col = col0 + cc;
        if (col < w) {
            if (single) store_out<O>(out, out_idx, col, a);
            else st_cg(partials + (int64_t)blockIdx.y * w + col, a);
        }
    }
    if (single) return;
    // the barrier orders the CTA's partial stores before thread 0's cumulative gpu fence
    __syncthreads();
    if (t == 0) {
        __threadfence();
        last = atomicAdd(tickets + blockIdx.x, 1u) == gridDim.y - 1;
        if (last) __threadfence();
    }
    __syncthreads();
    if (!last) return;
    // last CTA of this column tile: fold the gridDim.y partial rows (fixed order)
    const int Y = gridDim.y;
    const int tcw = (int)((w - col0) < TCW ? (w - col0) : TCW);
    if (tcw < NT) {
        const int YB = NT / tcw;
        const int cc = t % tcw, y0 = t / tcw;
        V a = O::id();
        if (y0 < YB) {
#pragma unroll 4
            for (int y = y0; y < Y; y += YB) a = O::comb(a, ld_cg(partials + (int64_t)y * w + col0 + cc));
        }
        __syncthreads();
        if (y0 < YB) part[y0 * tcw + cc] = a;
        __syncthreads();
        if (t < tcw) {
            V b = O::id();
            for (int q = 0; q < YB; ++q) b = O::comb(b, part[q * tcw + t]);
            store_out<O>(out, out_idx, col0 + t, b);
        }
    } else {
        for (int cc = t; cc < tcw; cc += NT) {
            V a = O::id();
#pragma unroll 4
            for (int y = 0; y < Y; ++y) a = O::comb(a, ld_cg(partials + (int64_t)y * w + col0 + cc));
            store_out<O>(out, out_idx, col0 + cc, a);
        }
    }
    if (t == 0) atomicExch(tickets + blockIdx.x, 0u);
}

// Many columns, few rows (one split): each thread owns one vector column and walks
// all m rows (U loads in flight), writing its outputs directly; a grid-stride loop
// over vector columns keeps the grid at the resident size instead of one CTA per
// 1024-column tile.
template <int OP, typename T, int NT, int VEC, int U>
__global__ void __launch_bounds__(NT)
colreduce_direct_kernel(const T *__restrict__ x, int64_t m, int64_t w, T *out, int64_t *out_idx) {
    using O = Op<OP, T>;
    using V = typename O::V;
    const int64_t WV = w / VEC;
    for (int64_t cv = (int64_t)blockIdx.x * NT + threadIdx.x; cv < WV; cv += (int64_t)gridDim.x * NT) {
        V acc[VEC];
#pragma unroll
        for (int k = 0; k < VEC; ++k) acc[k] = O::id();
        const T *base = x + cv * VEC;
        int64_t r = 0;
        for (; r + U <= m; r += U) {
            Vec16<T> e[U];
            T s1[U];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                if (VEC > 1) e[u] = as_vec<T>(ldg16(base + (r + u) * w));
                else s1[u] = __ldg(base + (r + u) * w);
            }
#pragma unroll
            for (int u = 0; u < U; ++u) {
#pragma unroll
                for (int k = 0; k < VEC; ++k) acc[k] = O::fold(acc[k], VEC > 1 ? e[u].e[k] : s1[u], r + u);
            }
        }
        for (; r < m; ++r) {
            if (VEC > 1) {
                const Vec16<T> e = as_vec<T>(ldg16(base + r * w));
#pragma unroll
                for (int k = 0; k < VEC; ++k) acc[k] = O::fold(acc[k], e.e[k], r);
            } else {
                acc[0] = O::fold(acc[0], __ldg(base + r * w), r);
            }
        }
#pragma unroll
        for (int k = 0; k < VEC; ++k) store_out<O>(out, out_idx, cv * VEC + k, acc[k]);
    }
}

struct ColPlan {
    int vec, CG;
    int64_t tiles, Y, rows_per_split;
};

static ColPlan col_plan(int dt, int64_t m, int64_t w, bool aligned, int op, int64_t resident) {
    ColPlan p;
    const int V = 16 / (int)dtype_size(dt);
    p.vec = (aligned && w % V == 0) ? V : 1;
    const int64_t wv = ceil_div(w, p.vec);
    p.CG = (int)(wv < kColThreads ? wv : kColThreads);
    if (p.CG < 1) p.CG = 1;
    // narrower column tiles when columns are few: enough tiles that each needs at most
    // ~64 row splits, so the last CTA of a tile folds few partial rows (a single CTA
    // folding hundreds of partial rows serialised the wide, short case)
    const int64_t want_tiles = resident / 64 > 1 ? resident / 64 : 1;
    while (p.CG > 32 && ceil_div(wv, p.CG) < want_tiles) p.CG /= 2;
    p.tiles = ceil_div(wv, p.CG);
    const int RB = kColThreads / p.CG;
    // row splits: fill the machine, keep >= 16 rows per thread-row, and keep the
    // partial rows below ~1% of the input bytes
    int64_t Y = resident / (p.tiles > 0 ? p.tiles : 1);
    if (p.tiles > kWsMaxTickets) Y = 1;  // per-tile tickets live in the workspace header
    const int64_t by_rows = m / ((int64_t)RB * 16);
    const int64_t by_bytes = (m * (int64_t)dtype_size(dt)) / (100 * (int64_t)acc_size(op, dt));
    if (Y > by_rows) Y = by_rows;
    if (Y > by_bytes) Y = by_bytes;
    if (Y > 65535) Y = 65535;
    if (Y < 1) Y = 1;
    p.rows_per_split = m > 0 ? ceil_div(m, Y) : 1;
    p.Y = m > 0 ? ceil_div(m, p.rows_per_split) : 1;
    return p;
}

template <int OP, typename T> struct ColRun {
    static fs_status run(const void *in, int64_t m, int64_t w, void *out, int64_t *out_idx, void *ws,
                         cudaStream_t st) {
        using V = typename Op<OP, T>::V;
        constexpr int VV = 16 / sizeof(T);
        const bool aligned = ((uintptr_t)in & 15) == 0;
        const int64_t resident = (int64_t)sm_count() * 8;
        const ColPlan p = col_plan(sizeof(T) == 8 ? FS_I64 : FS_I32, m, w, aligned, OP, resident);
        const int64_t WV = p.vec > 1 ? w / p.vec : w;
        if (p.Y == 1 && WV >= resident * kColThreads) {  // many columns, few rows
            const int64_t grid = ceil_div(WV, kColThreads) < resident * 2 ? ceil_div(WV, kColThreads) : resident * 2;
            if (p.vec > 1)
                colreduce_direct_kernel<OP, T, kColThreads, VV, 4><<<(unsigned)grid, kColThreads, 0, st>>>(
                    (const T *)in, m, w, (T *)out, out_idx);
            else
                colreduce_direct_kernel<OP, T, kColThreads, 1, 4><<<(unsigned)grid, kColThreads, 0, st>>>(
                    (const T *)in, m, w, (T *)out, out_idx);
            return launch_status();
        }
        char *wsb = (char *)ws;
        V *parts = (V *)(wsb + kWsHeader);
        unsigned *tickets = (unsigned *)(wsb + kWsTickets);  // p.Y > 1 implies p.tiles <= kWsMaxTickets
        const dim3 grid((unsigned)p.tiles, (unsigned)p.Y);
        if (p.vec > 1)
            colreduce_kernel<OP, T, kColThreads, VV, 4><<<grid, kColThreads, 0, st>>>(
                (const T *)in, m, w, p.CG, p.rows_per_split, parts, tickets, (T *)out, out_idx);
        else
            colreduce_kernel<OP, T, kColThreads, 1, 8><<<grid, kColThreads, 0, st>>>(
                (const T *)in, m, w, p.CG, p.rows_per_split, parts, tickets, (T *)out, out_idx);
        return launch_status();
    }
};

size_t colreduce_ws(int op, int dt, int64_t m, int64_t w) {
    // worst case over alignment: vec = 1 gives the most tiles; Y <= resident / tiles
    const int64_t resident = (int64_t)sm_count() * 8;
    const ColPlan p = col_plan(dt, m, w, false, op, resident);
    const ColPlan q = col_plan(dt, m, w, true, op, resident);
    const int64_t Y = p.Y > q.Y ? p.Y : q.Y;
    const int64_t tiles = p.tiles > q.tiles ? p.tiles : q.tiles;
    (void)tiles;
    return kWsHeader + align_up((size_t)Y * w * acc_size(op, dt), 256);
}

fs_status colreduce_run(int op, int dt, const void *in, int64_t m, int64_t w, void *out, int64_t *out_idx,
                        void *ws, cudaStream_t st) {
    return dispatch<ColRun>(op, dt, in, m, w, out, out_idx, ws, st);
}

}  // namespace fs
