// seg_map_reduce.cu -- NEXT-4: the horizontally fused row nest of PAPER.md L247-252,
//
//     map (\row -> (map (\x -> x + c) row, reduce (+) 0 row)) matrix
//
// with the reduce taken from the operator table.  Both results come from ONE read of
// every row (the two inner SOACs share their input, so fusion makes them one pass,
// Sec. 4; the paper's flattening would otherwise run a map nest and a segmented
// reduction separately).  Per 16-byte vector: load once, store x + c, fold x.
//   short rows (L = 2^j <= 32 vectors, aligned): grid-stride over vectors; a row is G
//     consecutive lanes (or part of one vector), reduced with xor shuffles (as KG0);
//   long rows (L >= 8192) and enough of them: a CTA per row (a compact read window);
//   otherwise: a warp per (row, piece); a row longer than the machine's warps can cover
//     one per row is cut into C pieces whose partials the last piece (per-row ticket)
//     combines in piece order (deterministic), as KG4.
#include <type_traits>

#include "internal.cuh"

namespace fs {

template <typename T> __device__ __forceinline__ T map_add(T x, T c) { return wrap_add(x, c); }

template <int OP, typename T, int U>
__global__ void __launch_bounds__(256)
segmr_short_kernel(const T *__restrict__ x, int64_t n, int L, int G, T c, T *__restrict__ ymap, T *__restrict__ out,
                   int64_t *__restrict__ out_idx) {
    using O = Op<OP, T>;
    using V = typename O::V;
    constexpr int VEC = 16 / sizeof(T);
    const int lane = threadIdx.x & 31, lg = lane & (G - 1);
    const int64_t nvec = n / VEC;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t gid0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t iters = (nvec + stride - 1) / stride;  // warp-uniform
    for (int64_t it0 = 0; it0 < iters; it0 += U) {
        int4 r[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t v = gid0 + (it0 + u) * stride;
            if (it0 + u < iters && v < nvec) r[u] = ldg16(x + v * VEC);
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
            if (it0 + u >= iters) break;
            const int64_t v = gid0 + (it0 + u) * stride;
            const bool ok = v < nvec;
            const Vec16<T> e = as_vec<T>(r[u]);
            if (ok) {
                Vec16<T> o;
#pragma unroll
                for (int k = 0; k < VEC; ++k) o.e[k] = map_add(e.e[k], c);
                *reinterpret_cast<int4 *>(ymap + v * VEC) = *reinterpret_cast<const int4 *>(&o);
            }
            if (L <= VEC) {
                if (ok)
                    for (int sg = 0; sg < VEC / L; ++sg) {
                        V a = O::id();
                        for (int j = 0; j < L; ++j) a = O::fold(a, e.e[sg * L + j], j);
                        store_out<O>(out, out_idx, v * (VEC / L) + sg, a);
                    }
            } else {
                V a = O::id();
                if (ok)
#pragma unroll
                    for (int k = 0; k < VEC; ++k) a = O::fold(a, e.e[k], (int64_t)lg * VEC + k);
#pragma unroll 1
                for (int m = G >> 1; m >= 1; m >>= 1) a = O::comb(a, shfl_xor(a, m));
                if (ok && lg == 0) store_out<O>(out, out_idx, v / G, a);
            }
        }
    }
    // ragged tail (L < VEC, n not a multiple of VEC): whole rows, one per thread
    for (int64_t s = nvec * VEC / L + gid0; s * L < n; s += stride) {
        V a = O::id();
        for (int j = 0; j < L; ++j) {
            const T xv = x[s * L + j];
            ymap[s * L + j] = map_add(xv, c);
            a = O::fold(a, xv, j);
        }
        store_out<O>(out, out_idx, s, a);
    }
}

// a warp per (row s, piece p): elements [p*CS, min(L, (p+1)*CS)) of row s
template <int OP, typename T, int U>
__global__ void __launch_bounds__(256)
segmr_warp_kernel(const T *__restrict__ x, int64_t nseg, int64_t L, int64_t C, int64_t CS, T c, bool vstore,
                  T *__restrict__ ymap, typename Op<OP, T>::V *partials, unsigned *tickets, T *__restrict__ out,
                  int64_t *__restrict__ out_idx) {
    using O = Op<OP, T>;
    using V = typename O::V;
    constexpr int VEC = 16 / sizeof(T);
    const int lane = threadIdx.x & 31;
    const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t item = gw; item < nseg * C; item += nw) {
        const int64_t s = item / C, pc = item - s * C;
        const int64_t j0 = pc * CS, j1 = j0 + CS < L ? j0 + CS : L;
        const int64_t len = j1 > j0 ? j1 - j0 : 0;
        const T *p = x + s * L + j0;
        T *q = ymap + s * L + j0;
        int64_t head = (int64_t)(((16 - ((uintptr_t)p & 15)) & 15) / sizeof(T));
        if (head > len) head = len;
        const int64_t nvec = (len - head) / VEC, tail0 = head + nvec * VEC;
        V a = O::id();
        if (lane < head) {
            const T xv = __ldg(p + lane);
            q[lane] = map_add(xv, c);
            a = O::fold(a, xv, j0 + lane);
        }
        const int4 *pv = reinterpret_cast<const int4 *>(p + head);
        for (int64_t v = lane; v < nvec; v += U * 32) {
            int4 r[U];
#pragma unroll
            for (int u = 0; u < U; ++u)
                if (v + u * 32 < nvec) r[u] = ldg16(pv + v + u * 32);
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const int64_t vv = v + u * 32;
                if (vv >= nvec) break;
                const Vec16<T> e = as_vec<T>(r[u]);
                Vec16<T> o;
#pragma unroll
                for (int k = 0; k < VEC; ++k) o.e[k] = map_add(e.e[k], c);
                T *qo = q + head + vv * VEC;
                if (vstore) {
                    *reinterpret_cast<int4 *>(qo) = *reinterpret_cast<const int4 *>(&o);
                } else {
#pragma unroll
                    for (int k = 0; k < VEC; ++k) qo[k] = o.e[k];
                }
                const int64_t b = j0 + head + vv * VEC;
#pragma unroll
                for (int k = 0; k < VEC; ++k) a = O::fold(a, e.e[k], b + k);
            }
        }
        if (lane < len - tail0) {
            const T xv = __ldg(p + tail0 + lane);
            q[tail0 + lane] = map_add(xv, c);
            a = O::fold(a, xv, j0 + tail0 + lane);
        }
        a = group_reduce<O>(a);
        if (C == 1) {
            if (lane == 0) store_out<O>(out, out_idx, s, a);
            continue;
        }
        // several pieces per row: partial, per-row ticket, the last piece combines in order
        unsigned lastp = 0;
        if (lane == 0) {
            st_cg(partials + s * C + pc, a);
            __threadfence();
            lastp = atomicAdd(tickets + s, 1u) == (unsigned)(C - 1);
            if (lastp) __threadfence();
        }
        lastp = __shfl_sync(0xffffffffu, lastp, 0);
        if (lastp) {
            V t = O::id();
            for (int64_t k = lane; k < C; k += 32) t = O::comb(t, ld_cg(partials + s * C + k));
            t = group_reduce<O>(t);
            if (lane == 0) {
                store_out<O>(out, out_idx, s, t);
                tickets[s] = 0;
            }
        }
    }
}

// a CTA per long row (L >= 8192, rows enough to fill the machine): all 256 threads stream
// the same row, so the GPU reads a compact window of the matrix at any moment
template <int OP, typename T, int U>
__global__ void __launch_bounds__(256)
segmr_block_kernel(const T *__restrict__ x, int64_t nseg, int64_t L, T c, bool vstore, T *__restrict__ ymap,
                   T *__restrict__ out, int64_t *__restrict__ out_idx) {
    using O = Op<OP, T>;
    using V = typename O::V;
    constexpr int VEC = 16 / sizeof(T);
    __shared__ V sm[32];
    const int t = threadIdx.x;
    for (int64_t s = blockIdx.x; s < nseg; s += gridDim.x) {
        const T *p = x + s * L;
        T *q = ymap + s * L;
        int64_t head = (int64_t)(((16 - ((uintptr_t)p & 15)) & 15) / sizeof(T));
        if (head > L) head = L;
        const int64_t nvec = (L - head) / VEC, tail0 = head + nvec * VEC;
        V a = O::id();
        if (t < head) {
            const T xv = __ldg(p + t);
            q[t] = map_add(xv, c);
            a = O::fold(a, xv, t);
        }
        const int4 *pv = reinterpret_cast<const int4 *>(p + head);
        for (int64_t v = t; v < nvec; v += (int64_t)U * 256) {
            int4 r[U];
#pragma unroll
            for (int u = 0; u < U; ++u)
                if (v + u * 256 < nvec) r[u] = ldg16(pv + v + u * 256);
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const int64_t vv = v + u * 256;
                if (vv >= nvec) break;
                const Vec16<T> e = as_vec<T>(r[u]);
                Vec16<T> o;
#pragma unroll
                for (int k = 0; k < VEC; ++k) o.e[k] = map_add(e.e[k], c);
                T *qo = q + head + vv * VEC;
                if (vstore) {
                    *reinterpret_cast<int4 *>(qo) = *reinterpret_cast<const int4 *>(&o);
                } else {
#pragma unroll
                    for (int k = 0; k < VEC; ++k) qo[k] = o.e[k];
                }
                const int64_t b = head + vv * VEC;
#pragma unroll
                for (int k = 0; k < VEC; ++k) a = O::fold(a, e.e[k], b + k);
            }
        }
        if (t < L - tail0) {
            const T xv = __ldg(p + tail0 + t);
            q[tail0 + t] = map_add(xv, c);
            a = O::fold(a, xv, tail0 + t);
        }
        a = block_reduce<O, 256>(a, sm);
        if (t == 0) store_out<O>(out, out_idx, s, a);
        __syncthreads();  // sm reuse
    }
}

struct SegMrPlan {
    bool shortp, block;
    int64_t C, CS, grid;
};

static SegMrPlan segmr_plan(int dt, int64_t nseg, int64_t L, bool aligned) {
    SegMrPlan p;
    const int64_t vec = 16 / (int64_t)dtype_size(dt);
    p.shortp = aligned && nseg > 0 && L >= 1 && L <= 32 * vec && (L & (L - 1)) == 0;
    const int64_t warps = (int64_t)sm_count() * 64;
    p.block = !p.shortp && L >= 8192 && nseg >= 4 * (int64_t)sm_count();
    p.C = 1;
    if (!p.shortp && !p.block && nseg > 0 && nseg < 8 * warps && L > 2048) {  // >= ~8 items per warp: no tail
        p.C = ceil_div(8 * warps, nseg);
        const int64_t maxc = ceil_div(L, 2048);  // pieces of >= 2048 elements
        if (p.C > maxc) p.C = maxc;
        if (p.C < 1) p.C = 1;
    }
    p.CS = ceil_div(L > 0 ? L : 1, p.C);
    p.CS = ceil_div(p.CS, vec) * vec;  // pieces start on whole vectors of the row
    p.C = ceil_div(L > 0 ? L : 1, p.CS);
    return p;
}

size_t seg_map_reduce_ws(int op, int dt, int64_t nseg, int64_t L) {
    const SegMrPlan p = segmr_plan(dt, nseg, L, false);
    if (p.C <= 1) return kWsHeader;
    return kWsHeader + align_up((size_t)nseg * p.C * acc_size(op, dt), 256) + align_up((size_t)nseg * 4, 256);
}

template <int OP, typename T> struct SegMrRun {
    static fs_status run(const void *in, int64_t nseg, int64_t L, int64_t ci, float cf, void *ymap, void *out,
                         int64_t *out_idx, void *ws, cudaStream_t st) {
        using V = typename Op<OP, T>::V;
        T c;
        if constexpr (std::is_floating_point<T>::value) c = (T)cf;
        else c = (T)ci;
        const bool aligned = ((uintptr_t)in & 15) == 0 && ((uintptr_t)ymap & 15) == 0;
        SegMrPlan p = segmr_plan(sizeof(T) == 8 ? FS_I64 : FS_I32, nseg, L, aligned);
        constexpr int64_t VEC = 16 / sizeof(T);
        if (p.shortp) {
            auto k = segmr_short_kernel<OP, T, 4>;
            const int64_t nvec = nseg * L / VEC;
            int64_t grid = ceil_div(nvec > 0 ? nvec : 1, 256 * 4);
            const int64_t cap = resident_blocks((const void *)k, 256);
            grid = grid > cap ? cap : (grid < 1 ? 1 : grid);
            k<<<(unsigned)grid, 256, 0, st>>>((const T *)in, nseg * L, (int)L, L > VEC ? (int)(L / VEC) : 1, c, (T *)ymap,
                                              (T *)out, out_idx);
            return launch_status();
        }
        const bool vstore = ((((uintptr_t)in) ^ ((uintptr_t)ymap)) & 15) == 0;
        if (p.block) {
            auto kb = segmr_block_kernel<OP, T, 4>;
            int64_t grid = resident_blocks((const void *)kb, 256);
            grid = grid > nseg ? nseg : grid;
            kb<<<(unsigned)grid, 256, 0, st>>>((const T *)in, nseg, L, c, vstore, (T *)ymap, (T *)out, out_idx);
            return launch_status();
        }
        char *w = (char *)ws;
        V *parts = (V *)(w + kWsHeader);
        unsigned *tickets = (unsigned *)(w + kWsHeader + align_up((size_t)nseg * p.C * sizeof(V), 256));
        if (p.C > 1 && cudaMemsetAsync(tickets, 0, (size_t)nseg * 4, st) != cudaSuccess) return FS_ERR_CUDA;
        auto k = segmr_warp_kernel<OP, T, 4>;
        const int64_t items = nseg * p.C;
        int64_t grid = ceil_div(items, 8);  // 8 warps per CTA
        const int64_t cap = resident_blocks((const void *)k, 256);
        grid = grid > cap ? cap : (grid < 1 ? 1 : grid);
        k<<<(unsigned)grid, 256, 0, st>>>((const T *)in, nseg, L, p.C, p.CS, c, vstore, (T *)ymap, parts, tickets,
                                          (T *)out, out_idx);
        return launch_status();
    }
};

fs_status seg_map_reduce_run(int op, int dt, const void *in, int64_t nseg, int64_t L, int64_t ci, float cf, void *ymap,
                             void *out, int64_t *out_idx, void *ws, cudaStream_t st) {
    return dispatch<SegMrRun>(op, dt, in, nseg, L, ci, cf, ymap, out, out_idx, ws, st);
}

}  // namespace fs
