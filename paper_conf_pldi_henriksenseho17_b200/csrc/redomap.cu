// redomap.cu -- KR1: fused map + reduce over a flat array (PAPER.md L240-254:
// fold (+,0) g = reduce (+,0) . map g; rule F3 L1067-1068 turns the reduce into
// a stream_red whose chunks are folded sequentially and combined with (+)).
//
// B200 design: one persistent grid (resident CTAs = #SM x occupancy).  Each
// thread folds a grid-strided sequence of 16-byte vectors (U vectors in flight
// per thread, loaded through the non-coherent path with no L1 allocation), in
// increasing index order.  A CTA reduces its threads with warp butterflies and
// one shared-memory step; each CTA writes one partial, and the last CTA to
// arrive (atomic ticket) folds the partials in CTA order and writes the result
// -- the combine of sFold's chunk results (L259-260) without a second launch.
// The fused map (identity or the Rodinia NN distance) is applied in registers:
// the mapped array is never materialised (L1815-1817: fusion).
#include <stdlib.h>

#include "internal.cuh"

namespace fs {

constexpr int kRedThreads = 256;

// Fold a CTA's value into the grid result; the last CTA writes out/out_idx.
template <class O, int NT, typename T>
__device__ __forceinline__ void finish_grid(typename O::V acc, typename O::V *partials, unsigned *ticket, T *out,
                                            int64_t *out_idx, typename O::V *sm, int64_t ibase) {
    using V = typename O::V;
    __shared__ bool last;
    if (threadIdx.x == 0) {
        st_cg(partials + blockIdx.x, acc);
        __threadfence();
        unsigned t = atomicAdd(ticket, 1u);
        last = (t == gridDim.x - 1);
        if (last) __threadfence();  // acquire: one fence, ordered for the CTA by the barrier
    }
    __syncthreads();
    if (!last) return;
    V a = O::id();
    for (int i = threadIdx.x; i < (int)gridDim.x; i += NT) a = O::comb(a, ld_cg(partials + i));
    a = block_reduce<O, NT>(a, sm);
    if (threadIdx.x == 0) {
        store_out<O>(out, out_idx, 0, shift_idx(a, ibase));
        atomicExch(ticket, 0u);  // leave the workspace ready for the next call
    }
}

template <int OP, typename T, int NT, int U>
__global__ void __launch_bounds__(NT) redomap_id_kernel(const T *__restrict__ x, int64_t n,
                                                        typename Op<OP, T>::V *partials, unsigned *ticket,
                                                        T *out, int64_t *out_idx, int64_t ibase) {
    using O = Op<OP, T>;
    using V = typename O::V;
    constexpr int VEC = 16 / sizeof(T);
    __shared__ V sm[32];
    const int64_t gid = (int64_t)blockIdx.x * NT + threadIdx.x;
    const int64_t stride = (int64_t)gridDim.x * NT;
    int64_t head = (int64_t)(((16 - ((uintptr_t)x & 15)) & 15) / sizeof(T));
    if (head > n) head = n;
    const int64_t nvec = (n - head) / VEC;
    const int64_t tail0 = head + nvec * VEC;
    const int4 *xv = reinterpret_cast<const int4 *>(x + head);

    V acc = O::id();
    if (gid < head) acc = O::fold(acc, x[gid], gid);
    // a warp reads U consecutive 512-byte runs (one contiguous 2 KB block) per iteration and
    // the warps stride over the array by blocks; every thread's indices still increase
    const int lane = threadIdx.x & 31;
    const int64_t gw = gid >> 5, nw = stride >> 5;
    const int64_t nblk = nvec / (32 * U);  // whole blocks
    for (int64_t bk = gw; bk < nblk; bk += nw) {
        const int64_t v0 = bk * 32 * U + lane;
        int4 r[U];
#pragma unroll
        for (int u = 0; u < U; ++u) r[u] = ldg16(xv + v0 + u * 32);
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const Vec16<T> e = as_vec<T>(r[u]);
            const int64_t base = head + (v0 + u * 32) * VEC;
#pragma unroll
            for (int k = 0; k < VEC; ++k) acc = O::fold(acc, e.e[k], base + k);
        }
    }
    for (int64_t v = nblk * 32 * U + gid; v < nvec; v += stride) {  // vectors past the last block
        const Vec16<T> e = as_vec<T>(ldg16(xv + v));
        const int64_t base = head + v * VEC;
#pragma unroll
        for (int k = 0; k < VEC; ++k) acc = O::fold(acc, e.e[k], base + k);
    }
    if (gid < n - tail0) acc = O::fold(acc, x[tail0 + gid], tail0 + gid);
    acc = block_reduce<O, NT>(acc, sm);
    finish_grid<O, NT>(acc, partials, ticket, out, out_idx, sm, ibase);
}

// Rodinia NN distance (reading R5): every operation rounded to f32, no FMA.

template <int OP, int NT, int U, bool VECT>
__global__ void __launch_bounds__(NT) redomap_nn_kernel(const float *__restrict__ lat, const float *__restrict__ lng,
                                                        int64_t n, float q0, float q1,
                                                        typename Op<OP, float>::V *partials, unsigned *ticket,
                                                        float *out, int64_t *out_idx, int64_t ibase) {
    using O = Op<OP, float>;
    using V = typename O::V;
    __shared__ V sm[32];
    const int64_t gid = (int64_t)blockIdx.x * NT + threadIdx.x;
    const int64_t stride = (int64_t)gridDim.x * NT;
    V acc = O::id();
    if (VECT) {  // lat and lng share their misalignment (checked on the host)
        int64_t head = (int64_t)(((16 - ((uintptr_t)lat & 15)) & 15) / 4);
        if (head > n) head = n;
        const int64_t nvec = (n - head) / 4, tail0 = head + nvec * 4;
        const int4 *av = reinterpret_cast<const int4 *>(lat + head);
        const int4 *bv = reinterpret_cast<const int4 *>(lng + head);
        if (gid < head) acc = O::fold(acc, nn_distance(lat[gid], lng[gid], q0, q1), gid);
        int64_t v = gid;
        for (; v + (U - 1) * stride < nvec; v += U * stride) {
            int4 ra[U], rb[U];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                ra[u] = ldg16(av + v + u * stride);
                rb[u] = ldg16(bv + v + u * stride);
            }
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const Vec16<float> a = as_vec<float>(ra[u]), b = as_vec<float>(rb[u]);
                const int64_t base = head + (v + u * stride) * 4;
#pragma unroll
                for (int k = 0; k < 4; ++k) acc = O::fold(acc, nn_distance(a.e[k], b.e[k], q0, q1), base + k);
            }
        }
        for (; v < nvec; v += stride) {
            const Vec16<float> a = as_vec<float>(ldg16(av + v)), b = as_vec<float>(ldg16(bv + v));
#pragma unroll
            for (int k = 0; k < 4; ++k) acc = O::fold(acc, nn_distance(a.e[k], b.e[k], q0, q1), head + v * 4 + k);
        }
        if (gid < n - tail0) acc = O::fold(acc, nn_distance(lat[tail0 + gid], lng[tail0 + gid], q0, q1), tail0 + gid);
    } else {
        for (int64_t i = gid; i < n; i += stride) acc = O::fold(acc, nn_distance(lat[i], lng[i], q0, q1), i);
    }
    acc = block_reduce<O, NT>(acc, sm);
    finish_grid<O, NT>(acc, partials, ticket, out, out_idx, sm, ibase);
}

// fs_combine: fold P partial results in order (width 1).
template <int OP, typename T, int NT>
__global__ void __launch_bounds__(NT) combine_kernel(const T *__restrict__ parts, const int64_t *__restrict__ pidx,
                                                     int64_t P, T *out, int64_t *out_idx) {
    using O = Op<OP, T>;
    using V = typename O::V;
    __shared__ V sm[32];
    V a = O::id();
    for (int64_t p = threadIdx.x; p < P; p += NT) a = O::comb(a, O::lift(parts[p], pidx ? pidx[p] : p));
    a = block_reduce<O, NT>(a, sm);
    if (threadIdx.x == 0) store_out<O>(out, out_idx, 0, a);
}

// fs_combine for VADD: out[j] = sum_p parts[p][j] in p order.
template <typename T>
__global__ void vadd_combine_kernel(const T *__restrict__ parts, int64_t P, int64_t w, T *out) {
    for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < w; j += (int64_t)gridDim.x * blockDim.x) {
        T a = T(0);
        for (int64_t p = 0; p < P; ++p) a = wrap_add(a, parts[p * w + j]);
        out[j] = a;
    }
}

// ------------------------------------------------------------------ host side
constexpr int kRedU = 4;
constexpr int kNnU = 2;

template <int OP, typename T> struct RedomapId {
    static const void *kernel() { return (const void *)redomap_id_kernel<OP, T, kRedThreads, kRedU>; }
    static fs_status run(const void *in, int64_t n, void *out, int64_t *out_idx, int64_t ibase, void *ws,
                         cudaStream_t st) {
        using V = typename Op<OP, T>::V;
        const int64_t per_cta = (int64_t)kRedThreads * kRedU * (16 / sizeof(T));
        int64_t grid = ceil_div(n, per_cta);
        grid = grid < 1 ? 1 : grid;
        const int64_t cap = resident_blocks(kernel(), kRedThreads);
        grid = grid > cap ? cap : grid;
        char *w = (char *)ws;
        redomap_id_kernel<OP, T, kRedThreads, kRedU><<<(unsigned)grid, kRedThreads, 0, st>>>(
            (const T *)in, n, (V *)(w + kWsHeader), (unsigned *)(w + kWsTicket), (T *)out, out_idx, ibase);
        return launch_status();
    }
};

template <int OP, typename T> struct RedomapNN {
    static fs_status run(const float *lat, const float *lng, int64_t n, float q0, float q1, void *out,
                         int64_t *out_idx, int64_t ibase, void *ws, cudaStream_t st) {
        using V = typename Op<OP, float>::V;
        const bool vect = (((uintptr_t)lat ^ (uintptr_t)lng) & 15) == 0;
        const void *k = vect ? (const void *)redomap_nn_kernel<OP, kRedThreads, kNnU, true>
                             : (const void *)redomap_nn_kernel<OP, kRedThreads, kNnU, false>;
        // the distance map costs ~40 instructions per record: spread small inputs (NN's
        // 855,280 records) over the whole machine, kNnU 4-record vectors per thread, all of
        // them loaded before the first is folded (one DRAM round trip, not kNnU)
        const int64_t per_cta = (int64_t)kRedThreads * 4 * kNnU;
        int64_t grid = ceil_div(n, per_cta);
        grid = grid < 1 ? 1 : grid;
        const int64_t cap = resident_blocks(k, kRedThreads);
        grid = grid > cap ? cap : grid;
        char *w = (char *)ws;
        V *parts = (V *)(w + kWsHeader);
        unsigned *ticket = (unsigned *)(w + kWsTicket);
        if (vect)
            redomap_nn_kernel<OP, kRedThreads, kNnU, true>
                <<<(unsigned)grid, kRedThreads, 0, st>>>(lat, lng, n, q0, q1, parts, ticket, (float *)out, out_idx, ibase);
        else
            redomap_nn_kernel<OP, kRedThreads, kNnU, false>
                <<<(unsigned)grid, kRedThreads, 0, st>>>(lat, lng, n, q0, q1, parts, ticket, (float *)out, out_idx, ibase);
        return launch_status();
    }
};

template <int OP, typename T> struct Combine {
    static fs_status run(const void *parts, const int64_t *pidx, int64_t P, void *out, int64_t *out_idx,
                         cudaStream_t st) {
        combine_kernel<OP, T, 256><<<1, 256, 0, st>>>((const T *)parts, pidx, P, (T *)out, out_idx);
        return launch_status();
    }
};

size_t redomap_ws(int op, int dt, int64_t n, bool nn) {
    (void)n;
    (void)nn;
    // partials: at most one per resident CTA of the kernel with the highest occupancy
    const int cap = sm_count() * 32;
    return kWsHeader + align_up((size_t)cap * acc_size(op, dt), 256);
}

fs_status redomap_run(int op, int dt, const fs_mapdesc &map, const void *in0, const void *in1, int64_t n,
                      void *out, int64_t *out_idx, void *ws, cudaStream_t st) {
    if (map.kind == FS_MAP_NN_DIST) {
        switch (op) {
        case FS_ADD: return RedomapNN<kAdd, float>::run((const float *)in0, (const float *)in1, n, map.q0, map.q1, out, out_idx, map.ibase, ws, st);
        case FS_MIN: return RedomapNN<kMin, float>::run((const float *)in0, (const float *)in1, n, map.q0, map.q1, out, out_idx, map.ibase, ws, st);
        case FS_MAX: return RedomapNN<kMax, float>::run((const float *)in0, (const float *)in1, n, map.q0, map.q1, out, out_idx, map.ibase, ws, st);
        case FS_ARGMIN: return RedomapNN<kArgmin, float>::run((const float *)in0, (const float *)in1, n, map.q0, map.q1, out, out_idx, map.ibase, ws, st);
        }
        return FS_ERR_UNSUPPORTED;
    }
    return dispatch<RedomapId>(op, dt, in0, n, out, out_idx, map.ibase, ws, st);
}

fs_status combine_run(int op, int dt, int64_t width, const void *parts, const int64_t *part_idx, int64_t P,
                      void *out, int64_t *out_idx, cudaStream_t st) {
    if (op == FS_VADD) {
        const unsigned grid = (unsigned)(width <= 0 ? 1 : (ceil_div(width, 256) > 1024 ? 1024 : ceil_div(width, 256)));
        switch (dt) {
        case FS_I32: vadd_combine_kernel<int32_t><<<grid, 256, 0, st>>>((const int32_t *)parts, P, width, (int32_t *)out); break;
        case FS_I64: vadd_combine_kernel<int64_t><<<grid, 256, 0, st>>>((const int64_t *)parts, P, width, (int64_t *)out); break;
        case FS_F32: vadd_combine_kernel<float><<<grid, 256, 0, st>>>((const float *)parts, P, width, (float *)out); break;
        default: return FS_ERR_UNSUPPORTED;
        }
        return launch_status();
    }
    return dispatch<Combine>(op, dt, parts, part_idx, P, out, out_idx, st);
}

}  // namespace fs
