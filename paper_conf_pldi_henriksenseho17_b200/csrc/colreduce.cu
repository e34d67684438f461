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

constexpr int kColGroup = 32;  // split rows folded per group (two-level combine)

// Fold partial rows [ya, yb) of the column tile [col0, col0 + tcw) (rows of stride w) in row
// order per thread-row, then across thread-rows; write the result to dst (a row, or the output).
// Eight loads in flight per thread.  Every thread of the CTA must call it.
template <typename O, typename T, int NT = kColThreads>
__device__ void col_fold_rows(const typename O::V *rows, int ya, int yb, int64_t w, int64_t col0, int tcw,
                              typename O::V *part, bool final, typename O::V *dst, T *out, int64_t *out_idx) {
    using V = typename O::V;
    const int t = threadIdx.x;
    const int YB = tcw < NT ? NT / tcw : 1;
    for (int cb = 0; cb < tcw; cb += NT) {
        const int cc = tcw < NT ? t % tcw : cb + t;
        const int y0 = tcw < NT ? t / tcw : 0;
        V a = O::id();
        if (y0 < YB && cc < tcw) {
            int y = ya + y0;
            for (; y + 7 * YB < yb; y += 8 * YB) {
                V v[8];
#pragma unroll
                for (int u = 0; u < 8; ++u) v[u] = ld_cg(rows + (int64_t)(y + u * YB) * w + col0 + cc);
#pragma unroll
                for (int u = 0; u < 8; ++u) a = O::comb(a, v[u]);
            }
            for (; y < yb; y += YB) a = O::comb(a, ld_cg(rows + (int64_t)y * w + col0 + cc));
        }
        if (YB > 1) {
            __syncthreads();
            if (y0 < YB) part[y0 * tcw + cc] = a;
            __syncthreads();
            if (t < tcw) {
                V b = O::id();
                for (int q = 0; q < YB; ++q) b = O::comb(b, part[q * tcw + t]);
                if (final) store_out<O>(out, out_idx, col0 + t, b);
                else st_cg(dst + col0 + t, b);
            }
        } else if (cc < tcw) {
            if (final) store_out<O>(out, out_idx, col0 + cc, a);
            else st_cg(dst + col0 + cc, a);
        }
    }
}

__host__ __device__ inline int tcw_of(int64_t w, int64_t col0, int TCW) {
    return (int)((w - col0) < TCW ? (w - col0) : TCW);
}

// After every CTA of split blockIdx.y has stored its partial row (columns [col0, col0 + tcw) of
// row blockIdx.y of `partials`, stride w) -- called by all threads of the CTA.
template <typename O, typename T>
__device__ void col_split_combine(typename O::V *partials, unsigned *tickets, int64_t w, int64_t col0, int tcw,
                                  typename O::V *part, bool *last, T *out, int64_t *out_idx) {
    using V = typename O::V;
    // Two-level combine of the Y partial rows: the last CTA of each group of kColGroup splits
    // (per-(tile, group) ticket) folds the group's rows into a group row; the last group
    // finisher of the tile (per-tile ticket) folds the group rows in group order.  A single
    // last CTA folding hundreds of partial rows (narrow w, m = 2^20..2^22) was a latency tail.
    const int t = threadIdx.x;
    const int Y = gridDim.y;
    const int ngroups = (Y + kColGroup - 1) / kColGroup;
    const int g = blockIdx.y / kColGroup;
    // the barrier orders the CTA's partial stores before thread 0's cumulative gpu fence
    __syncthreads();
    if (t == 0) {
        __threadfence();
        const int gsize = (g + 1) * kColGroup < Y ? kColGroup : Y - g * kColGroup;
        *last = atomicAdd(tickets + (int64_t)blockIdx.x * ngroups + g, 1u) == (unsigned)gsize - 1;
        if (*last) __threadfence();
    }
    __syncthreads();
    if (!*last) return;
    const int ya = g * kColGroup, yb = (ya + kColGroup < Y) ? ya + kColGroup : Y;
    if (ngroups == 1) {
        col_fold_rows<O, T>(partials, ya, yb, w, col0, tcw, part, true, partials, out, out_idx);
        if (t == 0) atomicExch(tickets + blockIdx.x, 0u);
        return;
    }
    V *grow = partials + (int64_t)Y * w;  // ngroups group rows after the Y split rows
    col_fold_rows<O, T>(partials, ya, yb, w, col0, tcw, part, false, grow + (int64_t)g * w, out, out_idx);
    __syncthreads();
    unsigned *tt = tickets + (int64_t)gridDim.x * ngroups;
    if (t == 0) {
        atomicExch(tickets + (int64_t)blockIdx.x * ngroups + g, 0u);
        __threadfence();
        *last = atomicAdd(tt + blockIdx.x, 1u) == (unsigned)ngroups - 1;
        if (*last) __threadfence();
    }
    __syncthreads();
    if (!*last) return;
    col_fold_rows<O, T>(grow, 0, ngroups, w, col0, tcw, part, true, partials, out, out_idx);
    if (t == 0) atomicExch(tt + blockIdx.x, 0u);
}

template <int OP, typename T, int NT, int VEC, int U>
__global__ void __launch_bounds__(NT, 2048 / NT)  // the plans assume 8 resident CTAs per SM
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
            if (r < r1) {  // the last partial batch: guarded loads issued together
                int4 v[U];
#pragma unroll
                for (int u = 0; u < U; ++u)
                    if (r + (int64_t)u * RB < r1) v[u] = ldg16(base + (r + (int64_t)u * RB) * w);
#pragma unroll
                for (int u = 0; u < U; ++u)
                    if (r + (int64_t)u * RB < r1) {
                        const Vec16<T> e = as_vec<T>(v[u]);
#pragma unroll
                        for (int k = 0; k < VEC; ++k) acc[k] = O::fold(acc[k], e.e[k], r + (int64_t)u * RB);
                    }
            }
        } else {
            for (; r + (int64_t)(U - 1) * RB < r1; r += (int64_t)U * RB) {
                T v[U];
#pragma unroll
                for (int u = 0; u < U; ++u) v[u] = __ldg(base + (r + (int64_t)u * RB) * w);
#pragma unroll
                for (int u = 0; u < U; ++u) acc[0] = O::fold(acc[0], v[u], r + (int64_t)u * RB);
            }
            if (r < r1) {  // the last partial batch: guarded loads issued together
                T v[U];
#pragma unroll
                for (int u = 0; u < U; ++u)
                    if (r + (int64_t)u * RB < r1) v[u] = __ldg(base + (r + (int64_t)u * RB) * w);
#pragma unroll
                for (int u = 0; u < U; ++u)
                    if (r + (int64_t)u * RB < r1) acc[0] = O::fold(acc[0], v[u], r + (int64_t)u * RB);
            }
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
    col_split_combine<O, T>(partials, tickets, w, col0, tcw_of(w, col0, TCW), part, &last, out, out_idx);
}

// Many columns, few rows (one split): each thread owns one vector column and walks
// all m rows (U loads in flight), writing its outputs directly; a grid-stride loop
// over vector columns keeps the grid at the resident size instead of one CTA per
// 1024-column tile.
template <int OP, typename T, int NT, int VEC, int U>
__global__ void __launch_bounds__(NT, 2048 / NT)  // the plans assume 8 resident CTAs per SM
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

// Narrow arrays (w <= kPeriodMaxW), 16-byte aligned base: the rows are read as ONE flat stream of
// 16-byte vectors.  P = R * rep rows (R * w a multiple of the vector width, rep copies so that a
// step is <= NT vectors) form a period whose vectors every step maps to the same columns, so a
// thread keeps VEC accumulators of fixed columns ((4q + k) mod w) and each CTA step reads P * w
// contiguous elements -- no partial-line rows, every thread busy, whatever w's phase.  Row
// splits (grid y) cover multiples of P rows; the split's leftover rows (< P) are folded per
// column; the splits combine two-level (col_split_combine).
constexpr int64_t kPeriodMaxW = 1024;

template <int OP, typename T, int NT, int U>
__global__ void __launch_bounds__(NT, 2048 / NT)
colreduce_period_kernel(const T *__restrict__ x, int64_t m, int64_t w, int P, int64_t rows_per_split,
                        typename Op<OP, T>::V *partials, unsigned *tickets, T *out, int64_t *out_idx) {
    using O = Op<OP, T>;
    using V = typename O::V;
    constexpr int VEC = 16 / sizeof(T);
    __shared__ V part[NT * VEC];
    __shared__ bool last;
    const int t = threadIdx.x;
    const int P4 = (int)((int64_t)P * w / VEC);  // vectors per period (<= NT)
    const int64_t r0 = (int64_t)blockIdx.y * rows_per_split;
    const int64_t r1 = r0 + rows_per_split < m ? r0 + rows_per_split : m;
    const int64_t rfull = r0 + (r1 - r0) / P * P;  // rows [r0, rfull) in whole periods
    V acc[VEC];
#pragma unroll
    for (int k = 0; k < VEC; ++k) acc[k] = O::id();
    int roff[VEC];  // row offset of each of this thread's elements within the period
#pragma unroll
    for (int k = 0; k < VEC; ++k) roff[k] = (int)(((int64_t)t * VEC + k) / w);
    if (t < P4) {
        const T *base = x + r0 * w + (int64_t)t * VEC;
        const int64_t step = (int64_t)P * w;
        int64_t r = r0;
        for (; r + (int64_t)U * P <= rfull; r += (int64_t)U * P) {
            int4 v[U];
#pragma unroll
            for (int u = 0; u < U; ++u) v[u] = ldg16(base + (r - r0 + (int64_t)u * P) * w);
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const Vec16<T> e = as_vec<T>(v[u]);
#pragma unroll
                for (int k = 0; k < VEC; ++k) acc[k] = O::fold(acc[k], e.e[k], r + (int64_t)u * P + roff[k]);
            }
        }
        for (; r < rfull; r += P) {
            const Vec16<T> e = as_vec<T>(ldg16(base + (r - r0) * w));
#pragma unroll
            for (int k = 0; k < VEC; ++k) acc[k] = O::fold(acc[k], e.e[k], r + roff[k]);
        }
        (void)step;
    }
    // per (period row, column) slot, then per column: the P slots in row order, then the leftover rows
    if (t < P4) {
#pragma unroll
        for (int k = 0; k < VEC; ++k) part[t * VEC + k] = acc[k];
    }
    __syncthreads();
    V colv[kPeriodMaxW / NT];
#pragma unroll
    for (int i = 0; i < (int)(kPeriodMaxW / NT); ++i) {
        const int64_t c = t + (int64_t)i * NT;
        V a = O::id();
        if (c < w) {
            for (int j = 0; j < P; ++j) a = O::comb(a, part[j * w + c]);
            for (int64_t r = rfull; r < r1; ++r) a = O::fold(a, __ldg(x + r * w + c), r);
        }
        colv[i] = a;
    }
    const bool single = gridDim.y == 1;
#pragma unroll
    for (int i = 0; i < (int)(kPeriodMaxW / NT); ++i) {
        const int64_t c = t + (int64_t)i * NT;
        if (c < w) {
            if (single) store_out<O>(out, out_idx, c, colv[i]);
            else st_cg(partials + (int64_t)blockIdx.y * w + c, colv[i]);
        }
    }
    if (single) return;
    __syncthreads();  // part[] is reused by the combine
    col_split_combine<O, T>(partials, tickets, w, 0, (int)w, part, &last, out, out_idx);
}

struct PeriodPlan {
    int P;
    int64_t Y, rows_per_split;
};

// P = R * rep: R the fewest rows whose elements fill whole vectors, rep the copies per step
static PeriodPlan period_plan(int dt, int op, int64_t m, int64_t w, int64_t resident) {
    PeriodPlan p;
    const int V = 16 / (int)dtype_size(dt);
    int R = 1;
    while ((R * w) % V) ++R;
    const int64_t per = R * w / V;  // vectors per R rows
    p.Y = 1;
    p.rows_per_split = 1;
    p.P = 0;  // not applicable: a period must fit one CTA step (<= kColThreads vectors)
    if (w > kPeriodMaxW || per > kColThreads) return p;
    const int64_t rep = kColThreads / per > 0 ? kColThreads / per : 1;
    p.P = (int)(R * rep);
    int64_t Y = resident;
    const int64_t by_rows = m / ((int64_t)p.P * 16);
    const int64_t by_bytes = (m * (int64_t)dtype_size(dt)) / (100 * (int64_t)acc_size(op, dt));
    if (Y > by_rows) Y = by_rows;
    if (Y > by_bytes) Y = by_bytes;
    while (Y > 1 && ceil_div(Y, kColGroup) + 1 > kWsMaxTickets) Y /= 2;
    if (Y < 1) Y = 1;
    p.rows_per_split = m > 0 ? ceil_div(ceil_div(m, Y), p.P) * p.P : p.P;
    p.Y = m > 0 ? ceil_div(m, p.rows_per_split) : 1;
    return p;
}

// Few rows (m <= 8), any column alignment: a thread owns 4 consecutive columns and issues all of
// its m x 4 loads at once (scalar loads; a warp's loads of one row are 512 contiguous bytes, so
// they coalesce whatever the row phase), then folds each column down the rows in order.  The
// column-major seg_reduce of short segments (seglen = 3, 7: an elementwise combine of m rows).
// VECIO (four-byte T, 16-byte aligned x and out, w % 4 == 0): every row's 4 columns arrive as
// one 16-byte load and the 4 results leave as one 16-byte store.
template <int OP, typename T, int MMAX, bool VECIO>
__global__ void __launch_bounds__(256)
colreduce_short_kernel(const T *__restrict__ x, int m, int64_t w, T *out, int64_t *out_idx) {
    using O = Op<OP, T>;
    using V = typename O::V;
    constexpr int C = 4;
    if constexpr (!VECIO) {
        // any row phase: a warp takes 32 x C consecutive columns, lane-interleaved (column
        // cw + lane + 32 k), so every load and store instruction touches 32 consecutive elements
        const int lane = threadIdx.x & 31;
        const int64_t nwb = (w + 32 * C - 1) / (32 * C);
        for (int64_t b = ((int64_t)blockIdx.x * 256 + threadIdx.x) >> 5; b < nwb; b += ((int64_t)gridDim.x * 256) >> 5) {
            const int64_t cw = b * 32 * C;
            T v[MMAX][C];
#pragma unroll
            for (int r = 0; r < MMAX; ++r)
#pragma unroll
                for (int k = 0; k < C; ++k)
                    if (r < m && cw + lane + 32 * k < w) v[r][k] = __ldg(x + (int64_t)r * w + cw + lane + 32 * k);
#pragma unroll
            for (int k = 0; k < C; ++k) {
                if (cw + lane + 32 * k >= w) continue;
                V a = O::id();
#pragma unroll
                for (int r = 0; r < MMAX; ++r)
                    if (r < m) a = O::fold(a, v[r][k], r);
                store_out<O>(out, out_idx, cw + lane + 32 * k, a);
            }
        }
        return;
    }
    const int64_t ng = (w + C - 1) / C;
    for (int64_t g = (int64_t)blockIdx.x * 256 + threadIdx.x; g < ng; g += (int64_t)gridDim.x * 256) {
        const int64_t c0 = g * C;
        T v[MMAX][C];
        if constexpr (VECIO) {
#pragma unroll
            for (int r = 0; r < MMAX; ++r)
                if (r < m) {
                    const Vec16<T> e = as_vec<T>(ldg16(x + (int64_t)r * w + c0));
#pragma unroll
                    for (int k = 0; k < C; ++k) v[r][k] = e.e[k];
                }
            Vec16<T> o;
#pragma unroll
            for (int k = 0; k < C; ++k) {
                V a = O::id();
#pragma unroll
                for (int r = 0; r < MMAX; ++r)
                    if (r < m) a = O::fold(a, v[r][k], r);
                o.e[k] = O::val(a);
            }
            int4 ov;
            memcpy(&ov, &o, 16);
            *reinterpret_cast<int4 *>(out + c0) = ov;
        } else {
#pragma unroll
            for (int r = 0; r < MMAX; ++r)
#pragma unroll
                for (int k = 0; k < C; ++k)
                    if (r < m && c0 + k < w) v[r][k] = __ldg(x + (int64_t)r * w + c0 + k);
#pragma unroll
            for (int k = 0; k < C; ++k) {
                if (c0 + k >= w) break;
                V a = O::id();
#pragma unroll
                for (int r = 0; r < MMAX; ++r)
                    if (r < m) a = O::fold(a, v[r][k], r);
                store_out<O>(out, out_idx, c0 + k, a);
            }
        }
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
    // (tile, group) tickets + per-tile tickets of the two-level combine must fit too
    while (Y > 1 && p.tiles * (ceil_div(Y, kColGroup) + 1) > kWsMaxTickets) Y /= 2;
    const int64_t by_rows = m / ((int64_t)RB * 16);
    // partial rows below ~1% of the input bytes -- ~4% for ARGMIN, whose 16-byte (value, index)
    // partials would otherwise cap the row splits at a quarter and leave most of the GPU idle
    // (col-major argmin L = 1024: 2 splits, 0.37 of HBM)
    const int64_t by_bytes = (m * (int64_t)dtype_size(dt)) / (100 * (int64_t)(op == FS_ARGMIN ? dtype_size(dt)
                                                                                             : acc_size(op, dt)));
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
        if (m <= 8 && w >= resident * 256) {  // few rows, many columns: elementwise, any alignment
            const int64_t ng = ceil_div(w, 4);
            const int64_t grid = ceil_div(ng, 256) < resident * 2 ? ceil_div(ng, 256) : resident * 2;
            if constexpr (sizeof(T) == 4 && OP != kArgmin) {
                if (aligned && ((uintptr_t)out & 15) == 0 && w % 4 == 0) {
                    if (m <= 4)
                        colreduce_short_kernel<OP, T, 4, true><<<(unsigned)grid, 256, 0, st>>>(
                            (const T *)in, (int)m, w, (T *)out, out_idx);
                    else
                        colreduce_short_kernel<OP, T, 8, true><<<(unsigned)grid, 256, 0, st>>>(
                            (const T *)in, (int)m, w, (T *)out, out_idx);
                    return launch_status();
                }
            }
            if (m <= 4)
                colreduce_short_kernel<OP, T, 4, false><<<(unsigned)grid, 256, 0, st>>>((const T *)in, (int)m, w,
                                                                                      (T *)out, out_idx);
            else
                colreduce_short_kernel<OP, T, 8, false><<<(unsigned)grid, 256, 0, st>>>((const T *)in, (int)m, w,
                                                                                      (T *)out, out_idx);
            return launch_status();
        }
        char *wsb = (char *)ws;
        V *parts = (V *)(wsb + kWsHeader);
        unsigned *tickets = (unsigned *)(wsb + kWsTickets);
        const PeriodPlan q = period_plan(sizeof(T) == 8 ? FS_I64 : FS_I32, OP, m, w, resident);
        if (aligned && q.P > 0 && m >= 4096) {  // narrow: one flat vector stream
            const dim3 grid(1u, (unsigned)q.Y);
            colreduce_period_kernel<OP, T, kColThreads, 4><<<grid, kColThreads, 0, st>>>(
                (const T *)in, m, w, q.P, q.rows_per_split, parts, tickets, (T *)out, out_idx);
            return launch_status();
        }
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
        // p.Y > 1 implies p.tiles <= kWsMaxTickets
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
    int64_t Y = p.Y > q.Y ? p.Y : q.Y;
    const PeriodPlan r = period_plan(dt, op, m, w, resident);
    if (r.P > 0 && r.Y > Y) Y = r.Y;
    const int64_t tiles = p.tiles > q.tiles ? p.tiles : q.tiles;
    (void)tiles;
    return kWsHeader + align_up((size_t)(Y + ceil_div(Y, kColGroup)) * w * acc_size(op, dt), 256);
}

fs_status colreduce_run(int op, int dt, const void *in, int64_t m, int64_t w, void *out, int64_t *out_idx,
                        void *ws, cudaStream_t st) {
    return dispatch<ColRun>(op, dt, in, m, w, out, out_idx, ws, st);
}

}  // namespace fs
