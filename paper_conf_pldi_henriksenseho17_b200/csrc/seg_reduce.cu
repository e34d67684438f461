// seg_reduce.cu -- segmented reduction over a regular FS_ROW_MAJOR
// [nseg][seglen] array: out[s] = reduce (+) 0(+) xss[s]   (footnote 5,
// L1230-1233: a map nest ending in a reduce; Fig 11's map-map-reduce nest).
//
// The paper's flattening has "no size that fits all" and proposes choosing
// between code versions at run time (L1411-1418).  This file is that choice,
// by segment length L (thresholds in seg_reduce_regime, calibrated by the
// seglen sweep in bench/ncu):
//   KG1  L small  : a CTA stages a tile of whole segments in shared memory
//                   with coalesced 16-byte loads, then groups of G lanes
//                   (G ~ L/4, a power of two) reduce one segment each.
//                   Shared memory is padded every 32 (4-byte) / 16 (8-byte)
//                   elements so strided per-segment reads do not conflict.
//   KG2  L medium : one warp per segment, 16-byte loads straight from HBM.
//   KG3  L large, many segments : one CTA per segment.
//   KG4  L large, few segments  : C CTAs per segment; each writes a partial
//                   and the last to arrive (per-segment ticket) combines the
//                   C partials in chunk order (the "second pass", fused).
#include <type_traits>

#include "internal.cuh"

namespace fs {

constexpr int kSegThreads = 256;
constexpr int kTileBytes = 32768;  // KG1 staged tile (before padding)

template <typename T> __device__ __forceinline__ int pad_pos(int e) {
    return sizeof(T) == 4 ? e + (e >> 5) : e + (e >> 4);
}
template <typename T> __host__ __device__ constexpr int tile_elems() { return kTileBytes / (int)sizeof(T); }
template <typename T> __host__ __device__ constexpr int tile_smem_bytes() {
    return (tile_elems<T>() + tile_elems<T>() / (sizeof(T) == 4 ? 32 : 16) + 4) * (int)sizeof(T);
}

// ---------------------------------------------------------------- KG1
template <int OP, typename T, int NT, int G>
__global__ void __launch_bounds__(NT)
seg_tile_kernel(const T *__restrict__ x, int64_t nseg, int L, int tile_segs, T *out, int64_t *out_idx) {
    using O = Op<OP, T>;
    using V = typename O::V;
    constexpr int VEC = 16 / sizeof(T);
    constexpr int U = 8;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    T *sm = reinterpret_cast<T *>(smem_raw);
    const int t = threadIdx.x;
    const bool vec_ok = (((uintptr_t)x & 15) == 0);  // host guarantees tile_segs*L*sizeof(T) % 16 == 0
    const int64_t ntiles = (nseg + tile_segs - 1) / tile_segs;
    for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
        const int64_t seg0 = tile * tile_segs;
        const int segs = (int)((nseg - seg0) < tile_segs ? (nseg - seg0) : tile_segs);
        const int ecount = segs * L;
        const T *src = x + seg0 * (int64_t)L;
        int done = 0;
        if (vec_ok) {
            const int nv = ecount / VEC;
            const int4 *sv = reinterpret_cast<const int4 *>(src);
            for (int v0 = t; v0 < nv; v0 += NT * U) {
                int4 r[U];
#pragma unroll
                for (int u = 0; u < U; ++u)
                    if (v0 + u * NT < nv) r[u] = ldg16(sv + v0 + u * NT);
#pragma unroll
                for (int u = 0; u < U; ++u)
                    if (v0 + u * NT < nv) {
                        const Vec16<T> e = as_vec<T>(r[u]);
                        const int b = (v0 + u * NT) * VEC;
#pragma unroll
                        for (int k = 0; k < VEC; ++k) sm[pad_pos<T>(b + k)] = e.e[k];
                    }
            }
            done = nv * VEC;
        }
        for (int e = done + t; e < ecount; e += NT) sm[pad_pos<T>(e)] = __ldg(src + e);
        __syncthreads();
        // reduce: group g of G lanes takes segment (base + g)
        constexpr int NG = NT / G;
        const int lg = t % G;
        for (int base = 0; base < segs; base += NG) {
            const int sl = base + t / G;
            V a = O::id();
            if (sl < segs) {
                const int off = sl * L;
                for (int j = lg; j < L; j += G) a = O::fold(a, sm[pad_pos<T>(off + j)], j);
            }
            a = group_reduce<O, G>(a);
            if (lg == 0 && sl < segs) store_out<O>(out, out_idx, seg0 + sl, a);
        }
        __syncthreads();
    }
}


// ---------------------------------------------------------------- KG1b (odd L <= 64)
// Short rows of odd length: tiles of R = 256 k whole rows (R L elements, <= ~32 KB) stream into a
// 2-slot shared-memory ring by 1-D TMA bulk copies (the next tile lands while this one is
// reduced), then thread t folds rows t, t + 256, ... in index order.  A row is L consecutive
// words: an odd stride, so the 32 lanes' loads fall in 32 distinct banks.  No padding, no
// staging instructions, one coalesced output store per row.
constexpr int kRowsTileElems = 8192;
__host__ __device__ inline int rows_tile_rows(int L) {
    const int k = kRowsTileElems / (256 * L);
    return 256 * (k > 1 ? k : 1);
}
template <int OP, typename T>
__global__ void __launch_bounds__(256)
seg_rows_odd_kernel(const T *__restrict__ x, int64_t nseg, int L, T *out, int64_t *out_idx) {
    using O = Op<OP, T>;
    using V = typename O::V;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    __shared__ __align__(8) uint64_t bars[2];
    const int t = threadIdx.x;
    const int R = rows_tile_rows(L);
    const int64_t ntiles = (nseg + R - 1) / R, nfull = nseg / R;
    const unsigned tile_bytes = (unsigned)(R * L * (int)sizeof(T));
    T *slot[2] = {reinterpret_cast<T *>(smem_raw), reinterpret_cast<T *>(smem_raw + tile_bytes)};
    if (t == 0) {
        mbar_init(&bars[0], 1);
        mbar_init(&bars[1], 1);
        fence_mbar_init();
    }
    __syncthreads();
    // tiles b, b + G, ...: the i-th of this CTA uses slot i & 1, phase (i >> 1) & 1
    auto issue = [&](int64_t tile, int sl) {
        if (tile < nfull) {
            mbar_expect_tx(&bars[sl], tile_bytes);
            tma_load_1d(slot[sl], x + tile * R * (int64_t)L, tile_bytes, &bars[sl]);
        }
    };
    if (t == 0) {
        issue(blockIdx.x, 0);
        issue(blockIdx.x + gridDim.x, 1);
    }
    int i = 0;
    for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x, ++i) {
        const int sl = i & 1;
        const int64_t r0 = tile * R;
        const int rows = (int)(nseg - r0 < R ? nseg - r0 : R);
        const bool full = tile < nfull;
        if (full) mbar_wait(&bars[sl], (unsigned)((i >> 1) & 1));
        const T *src = full ? slot[sl] : x + r0 * (int64_t)L;  // the ragged last tile from global memory
        for (int r = t; r < rows; r += 256) {
            const T *row = src + (int64_t)r * L;
            V a = O::id();
            for (int j = 0; j < L; ++j) a = O::fold(a, row[j], j);
            store_out<O>(out, out_idx, r0 + r, a);
        }
        __syncthreads();  // every thread is done with the slot before it is refilled
        if (t == 0) {
            fence_proxy_async();
            issue(tile + 2 * (int64_t)gridDim.x, sl);
        }
    }
}

// ---------------------------------------------------------------- KG0
// Power-of-two segments up to 32 vectors, 16-byte aligned base: no shared
// memory at all.  Each lane loads 16-byte vectors straight from HBM (coalesced,
// U in flight); a vector holds SPL = VEC/L whole segments (L < VEC) or a
// segment spans G = L/VEC lanes, reduced with log2(G) xor shuffles.
// a 16-byte vector holding VEC/LS whole segments of length LS (compile-time)
template <class O, typename T, int LS>
__device__ __forceinline__ void small_segs(const Vec16<T> &e, int64_t v, T *out, int64_t *out_idx) {
    constexpr int VEC = 16 / sizeof(T), SPL = VEC / LS;
    constexpr int OB = SPL * (int)sizeof(T);  // output bytes of one vector's segments
    if constexpr (!std::is_same<typename O::V, T>::value || (OB != 8 && OB != 16)) {
#pragma unroll
        for (int sg = 0; sg < SPL; ++sg) {
            typename O::V a = O::id();
#pragma unroll
            for (int k = 0; k < LS; ++k) a = O::fold(a, e.e[sg * LS + k], k);
            store_out<O>(out, out_idx, v * SPL + sg, a);
        }
    } else {  // the SPL results leave as ONE 8- or 16-byte store (L = 1, 2: a copy-like stream)
        T res[SPL];
#pragma unroll
        for (int sg = 0; sg < SPL; ++sg) {
            typename O::V a = O::id();
#pragma unroll
            for (int k = 0; k < LS; ++k) a = O::fold(a, e.e[sg * LS + k], k);
            res[sg] = a;
        }
        T *dst = out + v * SPL;
        if (((uintptr_t)dst & (OB - 1)) == 0) {
            if constexpr (OB == 16) {
                int4 w;
                memcpy(&w, res, 16);
                *reinterpret_cast<int4 *>(dst) = w;
            } else {
                int2 w;
                memcpy(&w, res, 8);
                *reinterpret_cast<int2 *>(dst) = w;
            }
        } else {
#pragma unroll
            for (int sg = 0; sg < SPL; ++sg) dst[sg] = res[sg];
        }
    }
}

template <int OP, typename T, int NT, int U>
__global__ void __launch_bounds__(NT, 4)
seg_vec_kernel(const T *__restrict__ x, int64_t nseg, int L, int G, T *out, int64_t *out_idx) {
    using O = Op<OP, T>;
    using V = typename O::V;
    constexpr int VEC = 16 / sizeof(T);
    const int lane = threadIdx.x & 31;
    const int64_t nvec = nseg * (int64_t)L / VEC;  // whole vectors
    const int64_t stride = (int64_t)gridDim.x * NT;
    const int lg = lane & (G - 1);
    const int64_t gid0 = (int64_t)blockIdx.x * NT + threadIdx.x;
    // every lane of a warp runs the same number of iterations (shuffles)
    const int64_t iters = (nvec + stride - 1) / stride;
    // software pipeline: the loads of batch b+1 are in flight while batch b is reduced
    int4 r[U], rn[U];
    auto load_batch = [&](int64_t it0, int4 (&dst)[U]) {
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t v = gid0 + (it0 + u) * stride;
            if (it0 + u < iters && v < nvec) dst[u] = ldg16(x + v * VEC);
        }
    };
    if (iters > 0) load_batch(0, r);
    for (int64_t it0 = 0; it0 < iters; it0 += U) {
        if (it0 + U < iters) load_batch(it0 + U, rn);
        if (L <= VEC) {
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const int64_t v = gid0 + (it0 + u) * stride;
                if (it0 + u < iters && v < nvec) {
                    const Vec16<T> e = as_vec<T>(r[u]);
                    if (L == 1) small_segs<O, T, 1>(e, v, out, out_idx);
                    else if (L == 2) small_segs<O, T, 2>(e, v, out, out_idx);
                    else small_segs<O, T, (VEC >= 4 ? 4 : VEC)>(e, v, out, out_idx);
                }
            }
        } else {
            // in-lane fold of each vector, then the xor-shuffle steps with the U vectors
            // interleaved (independent chains: the shuffle latency overlaps)
            V a[U];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const int64_t v = gid0 + (it0 + u) * stride;
                a[u] = O::id();
                if (it0 + u < iters && v < nvec) {
                    const Vec16<T> e = as_vec<T>(r[u]);
#pragma unroll
                    for (int k = 0; k < VEC; ++k) a[u] = O::fold(a[u], e.e[k], (int64_t)lg * VEC + k);
                }
            }
#pragma unroll 1
            for (int m = G >> 1; m >= 1; m >>= 1) {
#pragma unroll
                for (int u = 0; u < U; ++u) a[u] = O::comb(a[u], shfl_xor(a[u], m));
            }
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const int64_t v = gid0 + (it0 + u) * stride;
                if (it0 + u < iters && v < nvec && lg == 0) store_out<O>(out, out_idx, v / G, a[u]);
            }
        }
#pragma unroll
        for (int u = 0; u < U; ++u) r[u] = rn[u];
    }
    // ragged tail (L < VEC and nseg * L not a multiple of VEC): scalar, one segment per thread
    if (L < VEC) {
        const int64_t s0 = nvec * VEC / L;
        for (int64_t sgi = s0 + gid0; sgi < nseg; sgi += stride) {
            V a = O::id();
            for (int k = 0; k < L; ++k) a = O::fold(a, x[sgi * L + k], k);
            store_out<O>(out, out_idx, sgi, a);
        }
    }
}

// ---------------------------------------------------------------- KG0, wide lanes
// Power-of-two L >= UPL*VEC: each lane folds UPL consecutive 16-byte vectors
// (a 64-byte run) of one segment in registers, so a segment spans
// G = L / (UPL*VEC) lanes and needs log2(G) xor shuffles instead of
// log2(L/VEC).  A warp instruction reads 16 B per lane at a 64-B stride; the
// L1-allocating loads let the four instructions of a run share their sectors.
template <int OP, typename T, int NT, int U, int UPL>
__global__ void __launch_bounds__(NT, 4)
seg_vecw_kernel(const T *__restrict__ x, int64_t nseg, int L, int G, T *out, int64_t *out_idx) {
    using O = Op<OP, T>;
    using V = typename O::V;
    constexpr int VEC = 16 / sizeof(T);
    constexpr int RUN = UPL * VEC;  // elements per lane run
    const int lane = threadIdx.x & 31;
    const int64_t nrun = nseg * (int64_t)L / RUN;
    const int64_t stride = (int64_t)gridDim.x * NT;
    const int lg = lane & (G - 1);
    const int64_t gid0 = (int64_t)blockIdx.x * NT + threadIdx.x;
    const int64_t iters = (nrun + stride - 1) / stride;
    for (int64_t it0 = 0; it0 < iters; it0 += U) {
        int4 r[U][UPL];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t v = gid0 + (it0 + u) * stride;
            if (it0 + u < iters && v < nrun) {
                const int4 *p = reinterpret_cast<const int4 *>(x + v * RUN);
#pragma unroll
                for (int j = 0; j < UPL; ++j) r[u][j] = __ldg(p + j);
            }
        }
        V a[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t v = gid0 + (it0 + u) * stride;
            a[u] = O::id();
            if (it0 + u < iters && v < nrun) {
#pragma unroll
                for (int j = 0; j < UPL; ++j) {
                    const Vec16<T> e = as_vec<T>(r[u][j]);
#pragma unroll
                    for (int k = 0; k < VEC; ++k) a[u] = O::fold(a[u], e.e[k], (int64_t)lg * RUN + j * VEC + k);
                }
            }
        }
#pragma unroll 1
        for (int m = G >> 1; m >= 1; m >>= 1) {
#pragma unroll
            for (int u = 0; u < U; ++u) a[u] = O::comb(a[u], shfl_xor(a[u], m));
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t v = gid0 + (it0 + u) * stride;
            if (it0 + u < iters && v < nrun && lg == 0) store_out<O>(out, out_idx, v / G, a[u]);
        }
    }
}

// ---------------------------------------------------------------- KG2
template <int OP, typename T, int NT, int U>
__global__ void __launch_bounds__(NT)
seg_warp_kernel(const T *__restrict__ x, int64_t nseg, int64_t L, T *out, int64_t *out_idx) {
    using O = Op<OP, T>;
    using V = typename O::V;
    constexpr int VEC = 16 / sizeof(T);
    const int lane = threadIdx.x & 31;
    const int64_t gw = ((int64_t)blockIdx.x * NT + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * NT) >> 5;
    for (int64_t s = gw; s < nseg; s += nw) {
        const T *p = x + s * L;
        int64_t head = (int64_t)(((16 - ((uintptr_t)p & 15)) & 15) / sizeof(T));
        if (head > L) head = L;
        const int64_t nvec = (L - head) / VEC, tail0 = head + nvec * VEC;
        const int4 *pv = reinterpret_cast<const int4 *>(p + head);
        V a = O::id();
        if (lane < head) a = O::fold(a, __ldg(p + lane), lane);
        int64_t v = lane;
        for (; v + (U - 1) * 32 < nvec; v += U * 32) {
            int4 r[U];
#pragma unroll
            for (int u = 0; u < U; ++u) r[u] = ldg16(pv + v + u * 32);
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const Vec16<T> e = as_vec<T>(r[u]);
                const int64_t b = head + (v + u * 32) * VEC;
#pragma unroll
                for (int k = 0; k < VEC; ++k) a = O::fold(a, e.e[k], b + k);
            }
        }
        // the last partial batch: its (at most U) guarded loads issued together, one round trip
        if (v < nvec) {
            int4 r[U];
#pragma unroll
            for (int u = 0; u < U; ++u)
                if (v + u * 32 < nvec) r[u] = ldg16(pv + v + u * 32);
#pragma unroll
            for (int u = 0; u < U; ++u)
                if (v + u * 32 < nvec) {
                    const Vec16<T> e = as_vec<T>(r[u]);
                    const int64_t b = head + (v + u * 32) * VEC;
#pragma unroll
                    for (int k = 0; k < VEC; ++k) a = O::fold(a, e.e[k], b + k);
                }
        }
        if (lane < L - tail0) a = O::fold(a, __ldg(p + tail0 + lane), tail0 + lane);
        a = group_reduce<O>(a);
        if (lane == 0) store_out<O>(out, out_idx, s, a);
    }
}

// ---------------------------------------------------------------- KG3 / KG4
template <int OP, typename T, int NT, int U>
__global__ void __launch_bounds__(NT)
seg_block_kernel(const T *__restrict__ x, int64_t nseg, int64_t L, int64_t C, int64_t CS,
                 typename Op<OP, T>::V *partials, unsigned *tickets, T *out, int64_t *out_idx) {
    using O = Op<OP, T>;
    using V = typename O::V;
    constexpr int VEC = 16 / sizeof(T);
    __shared__ V sm[32];
    __shared__ bool last;
    const int t = threadIdx.x;
    const int64_t items = nseg * C;
    for (int64_t it = blockIdx.x; it < items; it += gridDim.x) {
        const int64_t s = it / C, c = it - s * C;
        const int64_t j0 = c * CS;
        const int64_t j1 = j0 + CS < L ? j0 + CS : L;
        const T *p = x + s * L + j0;
        const int64_t len = j1 > j0 ? j1 - j0 : 0;
        int64_t head = (int64_t)(((16 - ((uintptr_t)p & 15)) & 15) / sizeof(T));
        if (head > len) head = len;
        const int64_t nvec = (len - head) / VEC, tail0 = head + nvec * VEC;
        const int4 *pv = reinterpret_cast<const int4 *>(p + head);
        V a = O::id();
        if (t < head) a = O::fold(a, __ldg(p + t), j0 + t);
        int64_t v = t;
        for (; v + (int64_t)(U - 1) * NT < nvec; v += (int64_t)U * NT) {
            int4 r[U];
#pragma unroll
            for (int u = 0; u < U; ++u) r[u] = ldg16(pv + v + u * NT);
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const Vec16<T> e = as_vec<T>(r[u]);
                const int64_t b = j0 + head + (v + u * NT) * VEC;
#pragma unroll
                for (int k = 0; k < VEC; ++k) a = O::fold(a, e.e[k], b + k);
            }
        }
        for (; v < nvec; v += NT) {
            const Vec16<T> e = as_vec<T>(ldg16(pv + v));
#pragma unroll
            for (int k = 0; k < VEC; ++k) a = O::fold(a, e.e[k], j0 + head + v * VEC + k);
        }
        if (t < len - tail0) a = O::fold(a, __ldg(p + tail0 + t), j0 + tail0 + t);
        a = block_reduce<O, NT>(a, sm);
        if (C == 1) {
            if (t == 0) store_out<O>(out, out_idx, s, a);
            continue;
        }
        if (t == 0) {
            st_cg(partials + it, a);
            __threadfence();
            last = atomicAdd(tickets + s, 1u) == (unsigned)(C - 1);
            if (last) __threadfence();  // acquire, ordered for the CTA by the barrier
        }
        __syncthreads();
        if (last) {
            V b = O::id();
            for (int64_t q = t; q < C; q += NT) b = O::comb(b, ld_cg(partials + s * C + q));
            b = block_reduce<O, NT>(b, sm);
            if (t == 0) {
                store_out<O>(out, out_idx, s, b);
                atomicExch(tickets + s, 0u);
            }
        }
        __syncthreads();
    }
}

template <int OP, typename T>
__global__ void fill_neutral_kernel(int64_t count, T *out, int64_t *out_idx) {
    using O = Op<OP, T>;
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < count; k += (int64_t)gridDim.x * blockDim.x)
        store_out<O>(out, out_idx, k, O::id());
}

// ---------------------------------------------------------------- host
constexpr int64_t kWarpMaxL = 8192;    // KG2 upper bound (calibrated)
constexpr int64_t kMinChunk = 16384;   // KG4 smallest chunk (elements)

template <typename T> static int kg1_max_len() { return tile_elems<T>() / 4; }

int seg_reduce_regime(int op, int dt, int64_t nseg, int64_t L) {
    (void)op;
    if (nseg == 0 || L == 0) return 6;
    const int kg1max = dt == FS_I64 ? kg1_max_len<int64_t>() : kg1_max_len<int32_t>();
    const int forced = forced_seg_regime();
    if (forced >= 0 && forced <= 3) {
        if (forced == 0 && L > kg1max) return 1;
        return forced;
    }
    const int64_t vec = 16 / (int64_t)dtype_size(dt);
    if (L <= 64 || ((L & (L - 1)) == 0 && L <= 4 * 32 * vec / 2)) return 0;  // KG1 (KG0 when L is a power of two)
    if (L <= kWarpMaxL) return 1;
    const int64_t resident = (int64_t)sm_count() * 8;
    // KG3 (a CTA per row) from 3 x SMs rows: the C4 sweep, 2^28 f32 (profiles/r02_kg34.txt), KG3 vs KG4:
    // 4096 rows 0.95 / 0.90, 1024 0.94 / 0.89, 512 0.96 / 0.89, 256 0.80 / 0.92 (idle SMs)
    (void)resident;
    return nseg >= 3 * (int64_t)sm_count() ? 2 : 3;
}

struct BlockPlan {
    int64_t C, CS, items, grid;
};
static BlockPlan block_plan(int dt, int64_t nseg, int64_t L, int regime) {
    BlockPlan p;
    const int64_t resident = (int64_t)sm_count() * 8;
    const int64_t VEC = 16 / (int64_t)dtype_size(dt);
    p.C = 1;
    if (regime == 3) {
        const int64_t want = ceil_div(4 * resident, nseg);
        const int64_t maxc = ceil_div(L, kMinChunk);
        p.C = want < maxc ? want : maxc;
        if (p.C < 1 || nseg > kWsMaxTickets) p.C = 1;  // per-segment tickets live in the ws header
    }
    p.CS = ceil_div(ceil_div(L, p.C), VEC) * VEC;
    p.C = ceil_div(L, p.CS);
    p.items = nseg * p.C;
    p.grid = p.items < resident ? p.items : resident;
    return p;
}

#ifndef FS_SEG_UPL
// 16-byte vectors per lane run in KG0's wide-lane kernel: 2 (32-byte runs) measured 0.92-0.95 of
// HBM for L = 8..256 f32, 4 (64-byte runs) 0.80-0.87 (profiles/r02_seg_upl.txt)
#define FS_SEG_UPL 2
#endif
template <int OP, typename T> struct SegRun {
    static fs_status run(int regime, const void *in, int64_t nseg, int64_t L, void *out, int64_t *out_idx,
                         void *ws, cudaStream_t st) {
        using V = typename Op<OP, T>::V;
        const T *x = (const T *)in;
        constexpr int VEC = 16 / sizeof(T);
        const bool pow2 = (L & (L - 1)) == 0;
        constexpr int UPL = FS_SEG_UPL;
        if (regime == 0 && pow2 && L >= UPL * VEC && L <= 32 * UPL * VEC && ((uintptr_t)x & 15) == 0) {
            const int G = (int)(L / (UPL * VEC));
            const void *k = (const void *)seg_vecw_kernel<OP, T, kSegThreads, 2, UPL>;
            const int64_t nrun = nseg * L / (UPL * VEC);
            int64_t grid = ceil_div(nrun > 0 ? nrun : 1, (int64_t)kSegThreads * 2);
            const int64_t cap = resident_blocks(k, kSegThreads);
            grid = grid < cap ? grid : cap;
            seg_vecw_kernel<OP, T, kSegThreads, 2, UPL><<<(unsigned)grid, kSegThreads, 0, st>>>(x, nseg, (int)L, G,
                                                                                            (T *)out, out_idx);
            return launch_status();
        }
        if (regime == 0 && pow2 && L <= 32 * VEC && ((uintptr_t)x & 15) == 0) {
            const int G = L > VEC ? (int)(L / VEC) : 1;
            const void *k = (const void *)seg_vec_kernel<OP, T, kSegThreads, 4>;
            const int64_t nvec = nseg * L / VEC;
            int64_t grid = ceil_div(nvec > 0 ? nvec : 1, (int64_t)kSegThreads * 4);
            const int64_t cap = resident_blocks(k, kSegThreads);
            grid = grid < cap ? grid : cap;
            seg_vec_kernel<OP, T, kSegThreads, 4><<<(unsigned)grid, kSegThreads, 0, st>>>(x, nseg, (int)L, G,
                                                                                         (T *)out, out_idx);
            return launch_status();
        }
        if (regime == 0 && (L & 1) && L <= 64 && ((uintptr_t)x & 15) == 0 &&
            2 * rows_tile_rows((int)L) * L * (int64_t)sizeof(T) <= 160 * 1024) {
            const int R = rows_tile_rows((int)L);
            const int smem = 2 * R * (int)L * (int)sizeof(T);
            auto kr = seg_rows_odd_kernel<OP, T>;
            if (smem > 32 * 1024)
                cudaFuncSetAttribute((const void *)kr, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
            const int64_t ntiles = ceil_div(nseg, R);
            const int64_t cap = resident_blocks((const void *)kr, 256, (size_t)smem);
            const int64_t grid = ntiles < cap ? ntiles : cap;
            kr<<<(unsigned)(grid > 0 ? grid : 1), 256, smem, st>>>(x, nseg, (int)L, (T *)out, out_idx);
            return launch_status();
        }
        if (regime == 0) {
            const int maxe = tile_elems<T>();
            int tile_segs = maxe / (int)L;
            tile_segs &= ~3;  // L <= tile_elems/4: every tile start stays 16-byte aligned
            const int64_t ntiles = ceil_div(nseg, tile_segs);
            const int smem = tile_smem_bytes<T>();
            void (*k)(const T *, int64_t, int, int, T *, int64_t *);
            if (L < 8) k = seg_tile_kernel<OP, T, kSegThreads, 1>;
            else if (L < 16) k = seg_tile_kernel<OP, T, kSegThreads, 2>;
            else if (L < 32) k = seg_tile_kernel<OP, T, kSegThreads, 4>;
            else if (L < 64) k = seg_tile_kernel<OP, T, kSegThreads, 8>;
            else if (L < 128) k = seg_tile_kernel<OP, T, kSegThreads, 16>;
            else k = seg_tile_kernel<OP, T, kSegThreads, 32>;
            static bool attr_set = false;
            if (!attr_set) {
                cudaFuncSetAttribute((const void *)seg_tile_kernel<OP, T, kSegThreads, 1>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
                cudaFuncSetAttribute((const void *)seg_tile_kernel<OP, T, kSegThreads, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
                cudaFuncSetAttribute((const void *)seg_tile_kernel<OP, T, kSegThreads, 4>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
                cudaFuncSetAttribute((const void *)seg_tile_kernel<OP, T, kSegThreads, 8>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
                cudaFuncSetAttribute((const void *)seg_tile_kernel<OP, T, kSegThreads, 16>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
                cudaFuncSetAttribute((const void *)seg_tile_kernel<OP, T, kSegThreads, 32>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
                attr_set = true;
            }
            const int64_t cap = resident_blocks((const void *)k, kSegThreads, smem);
            const int64_t grid = ntiles < cap ? ntiles : cap;
            k<<<(unsigned)grid, kSegThreads, smem, st>>>(x, nseg, (int)L, tile_segs, (T *)out, out_idx);
            return launch_status();
        }
        if (regime == 1) {
            const void *k = (const void *)seg_warp_kernel<OP, T, kSegThreads, 4>;
            const int64_t cap = resident_blocks(k, kSegThreads);
            int64_t grid = ceil_div(nseg, kSegThreads / 32);
            grid = grid < cap ? grid : cap;
            seg_warp_kernel<OP, T, kSegThreads, 4><<<(unsigned)grid, kSegThreads, 0, st>>>(x, nseg, L, (T *)out, out_idx);
            return launch_status();
        }
        const BlockPlan p = block_plan(sizeof(T) == 8 ? FS_I64 : FS_I32, nseg, L, regime);
        char *w = (char *)ws;
        V *parts = (V *)(w + kWsHeader);
        unsigned *tickets = (unsigned *)(w + kWsTickets);
        seg_block_kernel<OP, T, kSegThreads, 4><<<(unsigned)p.grid, kSegThreads, 0, st>>>(
            x, nseg, L, p.C, p.CS, parts, tickets, (T *)out, out_idx);
        return launch_status();
    }
};

template <int OP, typename T> struct FillRun {
    static fs_status run(int64_t count, void *out, int64_t *out_idx, cudaStream_t st) {
        if (count <= 0) return FS_OK;
        int64_t grid = ceil_div(count, 256);
        grid = grid > 4096 ? 4096 : grid;
        fill_neutral_kernel<OP, T><<<(unsigned)grid, 256, 0, st>>>(count, (T *)out, out_idx);
        return launch_status();
    }
};

size_t seg_reduce_ws(int op, int dt, int64_t nseg, int64_t L) {
    const int r = seg_reduce_regime(op, dt, nseg, L);
    size_t body = 0;
    // KG3/KG4 may be forced for any length: size for the block plan of regime 3
    if (nseg > 0 && L > 0) {
        const BlockPlan p = block_plan(dt, nseg, L, 3);
        body = align_up((size_t)(p.C > 1 ? p.items : 0) * acc_size(op, dt), 256);
    }
    (void)r;
    return kWsHeader + body;
}

fs_status seg_reduce_run(int op, int dt, const void *in, int64_t nseg, int64_t L, void *out, int64_t *out_idx,
                         void *ws, cudaStream_t st) {
    const int regime = seg_reduce_regime(op, dt, nseg, L);
    note_regime(regime);
    if (regime == 6) return fill_neutral_run(op, dt, nseg, out, out_idx, st);
    return dispatch<SegRun>(op, dt, regime, in, nseg, L, out, out_idx, ws, st);
}

fs_status fill_neutral_run(int op, int dt, int64_t count, void *out, int64_t *out_idx, cudaStream_t st) {
    return dispatch<FillRun>(op, dt, count, out, out_idx, st);
}

}  // namespace fs
