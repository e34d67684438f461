// scan_reduce.cu -- NEXT-3: the stream_seq fusion of Fig 10 (L1158-1227; rules F4, F5,
// F7 of Fig 9): reduce (red) (scan (+) x) without materialising the scan.
//
// F5 turns the scan into a stream_seq threading the running prefix a; F4 turns the
// reduce into a stream_seq threading its accumulator; F7 fuses the two, so a chunk is
// summarised by a PAIR and the whole array by folding pairs in index order:
//   (+, +)   : (A, R, L)  A = chunk sum, R = sum of the chunk's prefixes, L = length
//              (A1,R1,L1) . (A2,R2,L2) = (A1 + A2, R1 + R2 + L2*A1, L1 + L2)
//   (+, max) : (A, M)     M = max prefix:  (A1 + A2, max(M1, A1 + M2))   (likewise min)
// Both products are associative (not commutative), so chunks may run in parallel as
// long as they are combined in index order -- the q = 1 stream_seq of Fig 10c in every
// lane (registers only), then ordered shuffle trees, then warps in order.
//   lane : its 8 contiguous elements (two or four 16-byte vectors) of a tile, folded
//          sequentially;
//   warp : ordered tree over the 32 lanes, then the tile joins the warp's running pair;
//          a warp owns one contiguous chunk of tiles;
//   last CTA (ticket): the warps' pairs in order (f64 for f32) -> the result.
// One read of x, nothing written but the result (the scan is never materialised).
#include <type_traits>

#include "internal.cuh"

namespace fs {

template <typename C> struct SRPair {
    C A, R;
    int64_t L;
};
template <> struct Lim<double> {
    static __device__ double hi() { return __longlong_as_double(0x7ff0000000000000ll); }
    static __device__ double lo() { return __longlong_as_double((long long)0xfff0000000000000ull); }
};
__device__ __forceinline__ double wrap_add(double a, double b) { return a + b; }

__device__ __forceinline__ double shfl_down_v(double v, int d) { return __shfl_down_sync(0xffffffffu, v, d); }

template <typename T> __device__ __forceinline__ SRPair<T> ld_cg_pair(const SRPair<T> *p) {
    return {__ldcg(&p->A), __ldcg(&p->R), __ldcg(&p->L)};
}



// the fused operator for (scan +, reduce RED); C is the accumulation type
template <int RED, typename C> struct SRFuse;
template <typename C> struct SRFuse<kAdd, C> {
    static __device__ __forceinline__ SRPair<C> id() { return {C(0), C(0), 0}; }
    static __device__ __forceinline__ SRPair<C> comb(const SRPair<C> &a, const SRPair<C> &b) {
        // R1 + R2 + L2 * A1 (integers: wrap-around, in unsigned arithmetic)
        return {wrap_add(a.A, b.A), wrap_add(wrap_add(a.R, b.R), mulw(b.L, a.A)), a.L + b.L};
    }
    template <typename T> static __device__ __forceinline__ C mulw(int64_t l, T a) {
        if constexpr (std::is_floating_point<T>::value) return (C)((T)l * a);
        else return (C)((std::make_unsigned_t<T>)l * (std::make_unsigned_t<T>)a);
    }
};
template <int RED, typename C> struct SRFuseMinMax {
    template <typename T> static __device__ __forceinline__ C mulw(int64_t, T a) { return (C)a; }  // unused
    static __device__ __forceinline__ C pick(C a, C b) { return RED == kMax ? (a < b ? b : a) : (b < a ? b : a); }
    static __device__ __forceinline__ SRPair<C> id() {
        return {C(0), RED == kMax ? Lim<C>::lo() : Lim<C>::hi(), 0};
    }
    static __device__ __forceinline__ SRPair<C> comb(const SRPair<C> &a, const SRPair<C> &b) {
        if (b.L == 0) return a;
        if (a.L == 0) return b;
        return {wrap_add(a.A, b.A), pick(a.R, wrap_add(a.A, b.R)), a.L + b.L};
    }
};
template <typename C> struct SRFuse<kMax, C> : SRFuseMinMax<kMax, C> {};
template <typename C> struct SRFuse<kMin, C> : SRFuseMinMax<kMin, C> {};

template <typename C> __device__ __forceinline__ SRPair<C> sr_shfl_down(const SRPair<C> &p, int off) {
    return {shfl_down_v(p.A, off), shfl_down_v(p.R, off), shfl_down_v(p.L, off)};
}

// a lane's vector as a pair: sequential q = 1 stream_seq (Fig 10c)
template <int RED, typename T> __device__ __forceinline__ SRPair<T> sr_lift_vec(const Vec16<T> &e, int cnt) {
    using F = SRFuse<RED, T>;
    SRPair<T> p = F::id();
    for (int k = 0; k < cnt; ++k) p = F::comb(p, SRPair<T>{e.e[k], e.e[k], 1});
    return p;
}

template <int RED, typename T, int U>
__global__ void __launch_bounds__(256)
scan_reduce_kernel(const T *__restrict__ x, int64_t n, int64_t tiles_per_warp, SRPair<T> *wparts, unsigned *ticket,
                   T *out) {
    using F = SRFuse<RED, T>;
    using C = std::conditional_t<std::is_floating_point<T>::value, double, T>;
    using FC = SRFuse<RED, C>;
    constexpr int VEC = 16 / sizeof(T);
    constexpr int PV = 8 / VEC;             // 16-byte vectors per lane: 8 contiguous elements
    constexpr int E = PV * VEC;
    constexpr int64_t TILE = 32 * E;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int64_t gw = (int64_t)blockIdx.x * 8 + warp;
    const int64_t ntiles = (n + TILE - 1) / TILE;
    const int64_t t0 = gw * tiles_per_warp, t1 = min(ntiles, t0 + tiles_per_warp);
    SRPair<T> run = F::id();
    int4 r[U][PV], rn[U][PV];
    auto load = [&](int64_t tb, int4 (&dst)[U][PV]) {
#pragma unroll
        for (int u = 0; u < U; ++u)
#pragma unroll
            for (int v = 0; v < PV; ++v) {
                const int64_t e0 = (tb + u) * TILE + (int64_t)lane * E + v * VEC;
                if (tb + u < t1 && e0 + VEC <= n) dst[u][v] = ldg16(x + e0);
            }
    };
    if (t0 < t1) load(t0, r);
    for (int64_t t = t0; t < t1; t += U) {
        if (t + U < t1) load(t + U, rn);  // the next batch is in flight while this one folds
#pragma unroll
        for (int u = 0; u < U; ++u) {
            if (t + u >= t1) break;  // warp-uniform
            const int64_t e0 = (t + u) * TILE + (int64_t)lane * E;
            if ((t + u + 1) * TILE <= n) {
                // full tile: every lane holds E contiguous elements, so every block length in
                // the ordered tree is static -- the pair is (A, R) and L is implicit
                T a, rr;
#pragma unroll
                for (int v = 0; v < PV; ++v) {
                    const Vec16<T> ev = as_vec<T>(r[u][v]);
#pragma unroll
                    for (int k = 0; k < VEC; ++k) {
                        if (v == 0 && k == 0) {
                            a = rr = ev.e[0];
                        } else {
                            a = wrap_add(a, ev.e[k]);
                            rr = RED == kAdd ? wrap_add(rr, a)
                                             : (RED == kMax ? (rr < a ? a : rr) : (a < rr ? a : rr));
                        }
                    }
                }
#pragma unroll
                for (int off = 1; off < 32; off <<= 1) {
                    const T a2 = shfl_down_v(a, off), r2 = shfl_down_v(rr, off);
                    if ((lane & (2 * off - 1)) == 0) {
                        if (RED == kAdd) rr = wrap_add(wrap_add(rr, r2), F::mulw((int64_t)E * off, a));
                        else {
                            const T c = wrap_add(a, r2);
                            rr = RED == kMax ? (rr < c ? c : rr) : (c < rr ? c : rr);
                        }
                        a = wrap_add(a, a2);
                    }
                }
                run = F::comb(run, SRPair<T>{__shfl_sync(0xffffffffu, a, 0), __shfl_sync(0xffffffffu, rr, 0), TILE});
                continue;
            }
            // ragged end of the array: element by element
            SRPair<T> p = F::id();
            for (int k = 0; k < E; ++k)
                if (e0 + k < n) p = F::comb(p, SRPair<T>{x[e0 + k], x[e0 + k], 1});
            // ordered tree: lane i absorbs lane i + off (its right neighbour block)
#pragma unroll
            for (int off = 1; off < 32; off <<= 1) {
                const SRPair<T> o = sr_shfl_down(p, off);
                if ((lane & (2 * off - 1)) == 0) p = F::comb(p, o);
            }
            run = F::comb(run, SRPair<T>{__shfl_sync(0xffffffffu, p.A, 0), __shfl_sync(0xffffffffu, p.R, 0),
                                         __shfl_sync(0xffffffffu, p.L, 0)});
        }
#pragma unroll
        for (int u = 0; u < U; ++u)
#pragma unroll
            for (int v = 0; v < PV; ++v) r[u][v] = rn[u][v];
    }
    __shared__ bool last;
    if (lane == 0) wparts[gw] = run;
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence();
        last = atomicAdd(ticket, 1u) == gridDim.x - 1;
        if (last) __threadfence();
    }
    __syncthreads();
    if (!last) return;
    // the warps' pairs in index order: contiguous runs per thread, then an ordered tree
    const int64_t W = (int64_t)gridDim.x * 8;
    const int64_t per = (W + 255) / 256;
    SRPair<C> q = FC::id();
    const int64_t w0 = threadIdx.x * per, w1 = min(W, (threadIdx.x + 1) * per);
    for (int64_t w = w0; w < w1; w += 8) {  // 8 loads in flight, then the ordered folds
        SRPair<T> pw[8];
#pragma unroll
        for (int i = 0; i < 8; ++i)
            if (w + i < w1) pw[i] = ld_cg_pair(wparts + w + i);
#pragma unroll
        for (int i = 0; i < 8; ++i)
            if (w + i < w1) q = FC::comb(q, SRPair<C>{(C)pw[i].A, (C)pw[i].R, pw[i].L});
    }
    __shared__ SRPair<C> sq[256];
    sq[threadIdx.x] = q;
    __syncthreads();
    for (int off = 1; off < 256; off <<= 1) {
        SRPair<C> v = sq[threadIdx.x];
        const bool take = (threadIdx.x & (2 * off - 1)) == 0 && threadIdx.x + off < 256;
        if (take) v = FC::comb(v, sq[threadIdx.x + off]);
        __syncthreads();
        if (take) sq[threadIdx.x] = v;
        __syncthreads();
    }
    if (threadIdx.x == 0) {
        const SRPair<C> f = sq[0];
        *out = (T)f.R;
        atomicExch(ticket, 0u);
    }
}

size_t scan_reduce_ws(int dt) {
    (void)dt;
    return kWsHeader + align_up((size_t)sm_count() * 8 * 8 * 24, 256);  // one pair per warp
}

template <int RED, typename T>
static fs_status sr_launch(const void *x, int64_t n, void *out, void *ws, cudaStream_t st) {
    constexpr int64_t TILE = 32 * 8;  // 8 contiguous elements per lane
    const int64_t ntiles = ceil_div(n > 0 ? n : 1, TILE);
    // exactly the resident CTAs (one wave: every warp's chunk runs concurrently), <= 8 per SM
    int64_t G = resident_blocks((const void *)scan_reduce_kernel<RED, T, 2>, 256);
    if (G > (int64_t)sm_count() * 8) G = (int64_t)sm_count() * 8;
    int64_t tpw = ceil_div(ntiles, G * 8);
    if (tpw < 4) {  // small inputs: fewer warps, >= 4 tiles each
        tpw = 4;
        G = ceil_div(ceil_div(ntiles, tpw), 8);
    }
    char *w = (char *)ws;
    scan_reduce_kernel<RED, T, 2><<<(unsigned)G, 256, 0, st>>>((const T *)x, n, tpw, (SRPair<T> *)(w + kWsHeader),
                                                              (unsigned *)(w + kWsTicket), (T *)out);
    return launch_status();
}

fs_status scan_reduce_run(int red, int dt, const void *x, int64_t n, void *out, void *ws, cudaStream_t st) {
#define FS_SR(R)                                                              \
    switch (dt) {                                                             \
    case FS_I32: return sr_launch<R, int32_t>(x, n, out, ws, st);             \
    case FS_I64: return sr_launch<R, int64_t>(x, n, out, ws, st);             \
    case FS_F32: return sr_launch<R, float>(x, n, out, ws, st);               \
    }                                                                         \
    return FS_ERR_UNSUPPORTED;
    switch (red) {
    case FS_ADD: FS_SR(kAdd)
    case FS_MAX: FS_SR(kMax)
    case FS_MIN: FS_SR(kMin)
    }
#undef FS_SR
    return FS_ERR_UNSUPPORTED;
}

}  // namespace fs
