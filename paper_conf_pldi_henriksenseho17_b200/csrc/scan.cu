// scan.cu -- KS1 scanomap and KG5 seg_scan.
//
// scan (+) 0(+) [a1..an] = [a1, ..., a1 (+) ... (+) an]   (inclusive, L129-130)
//
// F5 (L1071-1074, explained L1024-1032) states the chunked form: scan every
// chunk independently and add the contribution a of the previous chunks.  On
// B200 this is a single pass with decoupled look-back: each CTA takes the next
// tile id from an atomic counter (so every predecessor tile is already owned by
// a running CTA), scans its tile in registers, publishes the tile aggregate,
// then looks back over its predecessors' published aggregates / inclusive
// prefixes (one warp, 32 predecessors per step) to obtain a = the exclusive
// prefix of the tile, publishes its own inclusive prefix, and writes
// a (+) local scan.  Every element is read once and written once (8 B/elem for
// 4-byte types).
//
// Segmented scan (footnote 5, L1230-1233: "a scan with a modified (associative)
// operator"): elements carry the implicit flag (i mod seglen == 0) and the
// operator is  (f1,v1) (+)s (f2,v2) = (f1|f2, f2 ? v2 : v1 (+) v2).  The same
// look-back kernel then scans every regular segment; a look-back stops at the
// first predecessor whose accumulated flag is set (segment start), so short
// segments never wait on far predecessors.
//
// Column-major seg_scan (segments are columns of an [m][w] row-major array):
// threads own (vector-column, row block) units and scan down their rows; row
// blocks are chained by a reduce / exclusive-scan-of-partials / rescan.
#include "internal.cuh"

namespace fs {

// ---------------------------------------------------------------- segmented value
template <class O> struct SOp {
    using V = typename O::V;
    struct S {
        V v;
        int f;
    };
    static __device__ __forceinline__ S id() { return S{O::id(), 0}; }
    // ordered: a is the left operand
    static __device__ __forceinline__ S comb(S a, S b) { return b.f ? b : S{O::comb(a.v, b.v), a.f}; }
};

template <class S> __device__ __forceinline__ S shfl_up_s(S a, int d) {
    S r;
    r.v = shfl_up(a.v, d);
    r.f = __shfl_up_sync(0xffffffffu, a.f, d);
    return r;
}
template <class S> __device__ __forceinline__ S shfl_down_s(S a, int d) {
    S r;
    r.v = shfl_down_v(a.v, d);
    r.f = __shfl_down_sync(0xffffffffu, a.f, d);
    return r;
}
template <class S> __device__ __forceinline__ S shfl_idx_s(S a, int l) {
    S r;
    r.v = shfl_idx(a.v, l);
    r.f = __shfl_sync(0xffffffffu, a.f, l);
    return r;
}

__device__ __forceinline__ unsigned ld_acquire(const unsigned *p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release(unsigned *p, unsigned v) {
    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

template <class S> __device__ __forceinline__ void st_payload(S *p, S a) {
    st_cg(&p->v, a.v);
    __stcg(&p->f, a.f);
}
template <class S> __device__ __forceinline__ S ld_payload(const S *p) {
    S a;
    a.v = ld_cg(&p->v);
    a.f = __ldcg(&p->f);
    return a;
}

__device__ __forceinline__ float nn_dist_s(float lat, float lng, float q0, float q1) {
    const float d0 = __fsub_rn(lat, q0), d1 = __fsub_rn(lng, q1);
    return __fsqrt_rn(__fadd_rn(__fmul_rn(d0, d0), __fmul_rn(d1, d1)));
}

constexpr int kScanThreads = 256;
constexpr int kScanRows = 4;  // 16-byte vectors per lane per tile
constexpr unsigned kStAgg = 1, kStIncl = 2;

// ws body layout (after the 256-byte header):
//   [0, 256)                 : tile counter
//   [256, 256 + st_bytes)    : status words (u32 per tile)
//   then aggregates S[ntiles], inclusive prefixes S[ntiles]
struct ScanWs {
    unsigned *counter, *status;
    void *aggs, *incls;
    size_t clear_bytes;
};
template <class S> static ScanWs scan_ws_layout(void *ws, int64_t ntiles) {
    char *b = (char *)ws + kWsHeader;
    ScanWs w;
    w.counter = (unsigned *)b;
    w.status = (unsigned *)(b + 256);
    const size_t st = align_up((size_t)ntiles * 4, 256);
    w.aggs = b + 256 + st;
    w.incls = b + 256 + st + align_up((size_t)ntiles * sizeof(S), 256);
    w.clear_bytes = 256 + st;
    return w;
}

template <int OP, typename T, bool NN, bool SEG, bool ALIGNED>
__global__ void __launch_bounds__(kScanThreads)
scan_lookback_kernel(const T *__restrict__ in0, const float *__restrict__ in1, int64_t n, int64_t L, float q0,
                     float q1, int64_t ibase, T *__restrict__ out, int64_t *__restrict__ out_idx, const T *carry,
                     const int64_t *carry_idx, unsigned *counter, unsigned *status,
                     typename SOp<Op<OP, T>>::S *aggs, typename SOp<Op<OP, T>>::S *incls, int64_t ntiles) {
    using O = Op<OP, T>;
    using SO = SOp<O>;
    using S = typename SO::S;
    constexpr int VEC = 16 / sizeof(T);
    constexpr int R = kScanRows;
    constexpr int NW = kScanThreads / 32;
    constexpr int64_t TILE = (int64_t)kScanThreads * R * VEC;
    __shared__ S s_wtot[NW];
    __shared__ S s_wex[NW];
    __shared__ S s_ex;
    __shared__ int64_t s_tile;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;

    while (true) {
        if (threadIdx.x == 0) s_tile = (int64_t)atomicAdd(counter, 1u);
        __syncthreads();
        const int64_t tile = s_tile;
        if (tile >= ntiles) break;
        const int64_t wbase = tile * TILE + (int64_t)warp * 32 * R * VEC;

        S loc[R][VEC];
        S pre[R];
        S carry_w = SO::id();
#pragma unroll
        for (int q = 0; q < R; ++q) {
            const int64_t p0 = wbase + ((int64_t)q * 32 + lane) * VEC;
            T x[VEC];
            if (ALIGNED && p0 + VEC <= n) {
                if (NN) {
                    const Vec16<float> a = as_vec<float>(ldg16((const float *)in0 + p0));
                    const Vec16<float> b = as_vec<float>(ldg16(in1 + p0));
#pragma unroll
                    for (int k = 0; k < VEC; ++k) x[k] = (T)nn_dist_s(a.e[k], b.e[k], q0, q1);
                } else {
                    const Vec16<T> a = as_vec<T>(ldg16(in0 + p0));
#pragma unroll
                    for (int k = 0; k < VEC; ++k) x[k] = a.e[k];
                }
            } else {
#pragma unroll
                for (int k = 0; k < VEC; ++k) {
                    if (p0 + k < n) {
                        if (NN) x[k] = (T)nn_dist_s(((const float *)in0)[p0 + k], in1[p0 + k], q0, q1);
                        else x[k] = in0[p0 + k];
                    } else {
                        x[k] = T(0);
                    }
                }
            }
            int64_t r = SEG ? (p0 % L) : 0;
            S run = SO::id();
#pragma unroll
            for (int k = 0; k < VEC; ++k) {
                S e;
                if (p0 + k < n) {
                    e.v = O::lift(x[k], SEG ? r : ibase + p0 + k);
                    e.f = SEG ? (r == 0) : 0;
                } else {
                    e = SO::id();
                }
                if (SEG) {
                    ++r;
                    if (r == L) r = 0;
                }
                run = SO::comb(run, e);
                loc[q][k] = run;
            }
            // ordered inclusive warp scan of the lane totals
            S a = run;
#pragma unroll
            for (int off = 1; off < 32; off <<= 1) {
                const S o = shfl_up_s(a, off);
                if (lane >= off) a = SO::comb(o, a);
            }
            S ex = shfl_up_s(a, 1);
            if (lane == 0) ex = SO::id();
            pre[q] = SO::comb(carry_w, ex);
            carry_w = SO::comb(carry_w, shfl_idx_s(a, 31));
        }
        if (lane == 0) s_wtot[warp] = carry_w;
        __syncthreads();
        if (warp == 0) {
            S a = lane < NW ? s_wtot[lane] : SO::id();
#pragma unroll
            for (int off = 1; off < 32; off <<= 1) {
                const S o = shfl_up_s(a, off);
                if (lane >= off) a = SO::comb(o, a);
            }
            S wex = shfl_up_s(a, 1);
            if (lane == 0) wex = SO::id();
            if (lane < NW) s_wex[lane] = wex;
            const S agg = shfl_idx_s(a, NW - 1);
            // ---- decoupled look-back
            S exc = SO::id();
            if (tile == 0) {
                if (carry) exc = S{O::lift(*carry, carry_idx ? *carry_idx : -1), 0};
                if (lane == 0) {
                    st_payload(incls, SO::comb(exc, agg));
                    __threadfence();
                    st_release(status, kStIncl);
                }
            } else {
                if (lane == 0) {
                    st_payload(aggs + tile, agg);
                    __threadfence();
                    st_release(status + tile, kStAgg);
                }
                int64_t j = tile - 1;
                while (true) {
                    const int64_t idx = j - lane;
                    unsigned st = kStIncl;
                    if (idx >= 0) {
                        st = ld_acquire(status + idx);
                        while (st == 0) st = ld_acquire(status + idx);
                    }
                    const unsigned m = __ballot_sync(0xffffffffu, idx >= 0 && st == kStIncl);
                    const int kk = m ? __ffs(m) - 1 : 31;
                    S v = SO::id();
                    if (lane <= kk && idx >= 0) v = (st == kStIncl) ? ld_payload(incls + idx) : ld_payload(aggs + idx);
                    // ordered reduction: higher lanes are further left
#pragma unroll
                    for (int off = 1; off < 32; off <<= 1) {
                        const S o = shfl_down_s(v, off);
                        if (lane + off < 32) v = SO::comb(o, v);
                    }
                    exc = SO::comb(shfl_idx_s(v, 0), exc);
                    if (m || exc.f) break;
                    j -= 32;
                }
                if (lane == 0) {
                    st_payload(incls + tile, SO::comb(exc, agg));
                    __threadfence();
                    st_release(status + tile, kStIncl);
                }
            }
            if (lane == 0) s_ex = exc;
        }
        __syncthreads();
        const S base = SO::comb(s_ex, s_wex[warp]);
#pragma unroll
        for (int q = 0; q < R; ++q) {
            const int64_t p0 = wbase + ((int64_t)q * 32 + lane) * VEC;
            const S P = SO::comb(base, pre[q]);
            T y[VEC];
            int64_t yi[VEC];
#pragma unroll
            for (int k = 0; k < VEC; ++k) {
                const S o = SO::comb(P, loc[q][k]);
                y[k] = O::val(o.v);
                yi[k] = O::idx(o.v);
            }
            if (ALIGNED && p0 + VEC <= n) {
                Vec16<T> w;
#pragma unroll
                for (int k = 0; k < VEC; ++k) w.e[k] = y[k];
                int4 wv;
                memcpy(&wv, &w, 16);
                *reinterpret_cast<int4 *>(out + p0) = wv;
            } else {
#pragma unroll
                for (int k = 0; k < VEC; ++k)
                    if (p0 + k < n) out[p0 + k] = y[k];
            }
            if (OP == kArgmin) {
#pragma unroll
                for (int k = 0; k < VEC; ++k)
                    if (p0 + k < n) out_idx[p0 + k] = yi[k];
            }
        }
        __syncthreads();  // s_tile / smem reuse
    }
}

template <int OP, typename T> struct ScanRun {
    template <bool NN, bool SEG, bool AL>
    static fs_status go(const void *in0, const void *in1, int64_t n, int64_t L, const fs_mapdesc &map, void *out,
                        int64_t *out_idx, const void *carry, const int64_t *carry_idx, void *ws, cudaStream_t st) {
        using S = typename SOp<Op<OP, T>>::S;
        const int64_t tile = (int64_t)kScanThreads * kScanRows * (16 / sizeof(T));
        const int64_t ntiles = ceil_div(n, tile);
        const ScanWs w = scan_ws_layout<S>(ws, ntiles);
        if (cudaMemsetAsync(w.counter, 0, w.clear_bytes, st) != cudaSuccess) return FS_ERR_CUDA;
        auto k = scan_lookback_kernel<OP, T, NN, SEG, AL>;
        const int64_t cap = resident_blocks((const void *)k, kScanThreads);
        const int64_t grid = ntiles < cap ? ntiles : cap;
        k<<<(unsigned)grid, kScanThreads, 0, st>>>((const T *)in0, (const float *)in1, n, L, map.q0, map.q1,
                                                   map.ibase, (T *)out, out_idx, (const T *)carry, carry_idx,
                                                   w.counter, w.status, (S *)w.aggs, (S *)w.incls, ntiles);
        return launch_status();
    }
    static fs_status run(const fs_mapdesc *map, const void *in0, const void *in1, int64_t n, int64_t L, void *out,
                         int64_t *out_idx, const void *carry, const int64_t *carry_idx, void *ws, cudaStream_t st) {
        const bool seg = L < n;
        bool al = ((uintptr_t)in0 & 15) == 0 && ((uintptr_t)out & 15) == 0;
        if (map->kind == FS_MAP_NN_DIST) {
            al = al && ((uintptr_t)in1 & 15) == 0;
            if constexpr (sizeof(T) == 4) {
                if (al) return go<true, false, true>(in0, in1, n, L, *map, out, out_idx, carry, carry_idx, ws, st);
                return go<true, false, false>(in0, in1, n, L, *map, out, out_idx, carry, carry_idx, ws, st);
            }
            return FS_ERR_UNSUPPORTED;
        }
        if (seg) {
            if (al) return go<false, true, true>(in0, in1, n, L, *map, out, out_idx, carry, carry_idx, ws, st);
            return go<false, true, false>(in0, in1, n, L, *map, out, out_idx, carry, carry_idx, ws, st);
        }
        if (al) return go<false, false, true>(in0, in1, n, L, *map, out, out_idx, carry, carry_idx, ws, st);
        return go<false, false, false>(in0, in1, n, L, *map, out, out_idx, carry, carry_idx, ws, st);
    }
};

size_t scan_ws(int op, int dt, int64_t n) {
    const int64_t tile = (int64_t)kScanThreads * kScanRows * (16 / (int64_t)dtype_size(dt));
    const int64_t ntiles = ceil_div(n, tile);
    const size_t s = align_up(acc_size(op, dt) + 4, 8);  // S = {V, int}, padded
    return kWsHeader + 256 + align_up((size_t)ntiles * 4, 256) + 2 * align_up((size_t)ntiles * (s + 8), 256);
}

fs_status scan_run(int op, int dt, const fs_mapdesc &map, const void *in0, const void *in1, int64_t n, int64_t L,
                   void *out, int64_t *out_idx, const void *carry, const int64_t *carry_idx, void *ws,
                   cudaStream_t st) {
    if (map.kind == FS_MAP_NN_DIST) dt = FS_F32;
    return dispatch<ScanRun>(op, dt, &map, in0, in1, n, L, out, out_idx, carry, carry_idx, ws, st);
}

// ================================================================ column-major seg_scan
// unit u = (vector-column cv, row block y): thread id -> (cv = id % WV, y = id / WV)
constexpr int kColScanThreads = 256;

template <int OP, typename T, int VEC>
__global__ void __launch_bounds__(kColScanThreads)
colscan_partial_kernel(const T *__restrict__ x, int64_t m, int64_t w, int64_t WV, int64_t Y, int64_t rpu,
                       typename Op<OP, T>::V *partials) {
    using O = Op<OP, T>;
    using V = typename O::V;
    const int64_t id = (int64_t)blockIdx.x * kColScanThreads + threadIdx.x;
    if (id >= WV * Y) return;
    const int64_t cv = id % WV, y = id / WV;
    const int64_t r0 = y * rpu, r1 = r0 + rpu < m ? r0 + rpu : m;
    V acc[VEC];
#pragma unroll
    for (int k = 0; k < VEC; ++k) acc[k] = O::id();
    const T *base = x + cv * VEC;
    for (int64_t r = r0; r < r1; ++r) {
        if (VEC > 1) {
            const Vec16<T> e = as_vec<T>(*reinterpret_cast<const int4 *>(base + r * w));
#pragma unroll
            for (int k = 0; k < VEC; ++k) acc[k] = O::fold(acc[k], e.e[k], r);
        } else {
            acc[0] = O::fold(acc[0], __ldg(base + r * w), r);
        }
    }
#pragma unroll
    for (int k = 0; k < VEC; ++k) partials[y * w + cv * VEC + k] = acc[k];
}

// exclusive scan over the Y row blocks of every column, in place
template <int OP, typename T>
__global__ void colscan_carry_kernel(typename Op<OP, T>::V *partials, int64_t w, int64_t Y) {
    using O = Op<OP, T>;
    using V = typename O::V;
    for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c < w; c += (int64_t)gridDim.x * blockDim.x) {
        V run = O::id();
        int64_t y = 0;
        for (; y + 4 <= Y; y += 4) {
            V p[4];
#pragma unroll
            for (int u = 0; u < 4; ++u) p[u] = partials[(y + u) * w + c];
#pragma unroll
            for (int u = 0; u < 4; ++u) {
                partials[(y + u) * w + c] = run;
                run = O::comb(run, p[u]);
            }
        }
        for (; y < Y; ++y) {
            const V p = partials[y * w + c];
            partials[y * w + c] = run;
            run = O::comb(run, p);
        }
    }
}

template <int OP, typename T, int VEC, bool CARRY>
__global__ void __launch_bounds__(kColScanThreads)
colscan_kernel(const T *__restrict__ x, int64_t m, int64_t w, int64_t WV, int64_t Y, int64_t rpu,
               const typename Op<OP, T>::V *carries, T *__restrict__ out, int64_t *__restrict__ out_idx) {
    using O = Op<OP, T>;
    using V = typename O::V;
    const int64_t id = (int64_t)blockIdx.x * kColScanThreads + threadIdx.x;
    if (id >= WV * Y) return;
    const int64_t cv = id % WV, y = id / WV;
    const int64_t r0 = y * rpu, r1 = r0 + rpu < m ? r0 + rpu : m;
    V acc[VEC];
#pragma unroll
    for (int k = 0; k < VEC; ++k) acc[k] = CARRY ? carries[y * w + cv * VEC + k] : O::id();
    const T *base = x + cv * VEC;
    T *obase = out + cv * VEC;
    for (int64_t r = r0; r < r1; ++r) {
        if (VEC > 1) {
            const Vec16<T> e = as_vec<T>(*reinterpret_cast<const int4 *>(base + r * w));
            Vec16<T> o;
#pragma unroll
            for (int k = 0; k < VEC; ++k) {
                acc[k] = O::comb(acc[k], O::lift(e.e[k], r));
                o.e[k] = O::val(acc[k]);
                if (OP == kArgmin) out_idx[r * w + cv * VEC + k] = O::idx(acc[k]);
            }
            int4 ov;
            memcpy(&ov, &o, 16);
            *reinterpret_cast<int4 *>(obase + r * w) = ov;
        } else {
            acc[0] = O::comb(acc[0], O::lift(__ldg(base + r * w), r));
            obase[r * w] = O::val(acc[0]);
            if (OP == kArgmin) out_idx[r * w + cv] = O::idx(acc[0]);
        }
    }
}

struct ColScanPlan {
    int vec;
    int64_t WV, Y, rpu;
};
static ColScanPlan colscan_plan(int dt, int64_t m, int64_t w, bool aligned) {
    ColScanPlan p;
    const int V = 16 / (int)dtype_size(dt);
    p.vec = (aligned && w % V == 0) ? V : 1;
    p.WV = ceil_div(w, p.vec);
    const int64_t threads = (int64_t)sm_count() * 2048;
    int64_t Y = ceil_div(threads, p.WV);
    const int64_t by_rows = m / 16;
    if (Y > by_rows) Y = by_rows;
    if (Y < 1) Y = 1;
    p.rpu = ceil_div(m, Y);
    p.Y = ceil_div(m, p.rpu);
    return p;
}

template <int OP, typename T> struct ColScanRun {
    template <int VEC>
    static fs_status go(const ColScanPlan &p, const T *x, int64_t m, int64_t w, T *out, int64_t *out_idx, void *ws,
                        cudaStream_t st) {
        using V = typename Op<OP, T>::V;
        V *parts = (V *)((char *)ws + kWsHeader);
        const int64_t units = p.WV * p.Y;
        const unsigned grid = (unsigned)ceil_div(units, kColScanThreads);
        if (p.Y == 1) {
            colscan_kernel<OP, T, VEC, false><<<grid, kColScanThreads, 0, st>>>(x, m, w, p.WV, 1, p.rpu, parts, out,
                                                                                out_idx);
            return launch_status();
        }
        colscan_partial_kernel<OP, T, VEC><<<grid, kColScanThreads, 0, st>>>(x, m, w, p.WV, p.Y, p.rpu, parts);
        int64_t g2 = ceil_div(w, 128);
        g2 = g2 > 4096 ? 4096 : g2;
        colscan_carry_kernel<OP, T><<<(unsigned)g2, 128, 0, st>>>(parts, w, p.Y);
        colscan_kernel<OP, T, VEC, true><<<grid, kColScanThreads, 0, st>>>(x, m, w, p.WV, p.Y, p.rpu, parts, out,
                                                                           out_idx);
        return launch_status(3);
    }
    static fs_status run(const void *in, int64_t m, int64_t w, void *out, int64_t *out_idx, void *ws, cudaStream_t st) {
        const bool aligned = ((uintptr_t)in & 15) == 0 && ((uintptr_t)out & 15) == 0;
        const ColScanPlan p = colscan_plan(sizeof(T) == 8 ? FS_I64 : FS_I32, m, w, aligned);
        if (p.vec > 1) return go<16 / sizeof(T)>(p, (const T *)in, m, w, (T *)out, out_idx, ws, st);
        return go<1>(p, (const T *)in, m, w, (T *)out, out_idx, ws, st);
    }
};

size_t colscan_ws(int op, int dt, int64_t m, int64_t w) {
    const ColScanPlan a = colscan_plan(dt, m, w, false), b = colscan_plan(dt, m, w, true);
    const int64_t Y = a.Y > b.Y ? a.Y : b.Y;
    return kWsHeader + align_up((size_t)Y * w * acc_size(op, dt), 256);
}

fs_status colscan_run(int op, int dt, const void *in, int64_t m, int64_t w, void *out, int64_t *out_idx, void *ws,
                      cudaStream_t st) {
    return dispatch<ColScanRun>(op, dt, in, m, w, out, out_idx, ws, st);
}

}  // namespace fs
