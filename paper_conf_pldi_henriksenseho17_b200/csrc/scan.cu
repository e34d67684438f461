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
#include <stdlib.h>

#include <type_traits>

#include "internal.cuh"

namespace fs {

// ---------------------------------------------------------------- segmented value
// S = (value, flag).  Without SEG the flag is the constant 0 and vanishes.
template <class O, bool SEG> struct SOp {
    using V = typename O::V;
    struct S {
        V v;
        int f;
    };
    static __device__ __forceinline__ S id() { return S{O::id(), 0}; }
    // ordered: a is the left operand
    static __device__ __forceinline__ S comb(S a, S b) {
        if constexpr (SEG) return b.f ? b : S{O::comb(a.v, b.v), a.f};
        else return S{O::comb(a.v, b.v), 0};
    }
    static __device__ __forceinline__ S up(S a, int d) {
        return S{shfl_up(a.v, d), SEG ? __shfl_up_sync(0xffffffffu, a.f, d) : 0};
    }
    static __device__ __forceinline__ S down(S a, int d) {
        return S{shfl_down_v(a.v, d), SEG ? __shfl_down_sync(0xffffffffu, a.f, d) : 0};
    }
    static __device__ __forceinline__ S bcast(S a, int l) {
        return S{shfl_idx(a.v, l), SEG ? __shfl_sync(0xffffffffu, a.f, l) : 0};
    }
};

__device__ __forceinline__ unsigned ld_acquire(const unsigned *p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release(unsigned *p, unsigned v) {
    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ uint64_t ld_relaxed64(const uint64_t *p) {
    uint64_t v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_relaxed64(uint64_t *p, uint64_t v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint32_t to_bits(int32_t v) { return (uint32_t)v; }
__device__ __forceinline__ uint32_t to_bits(float v) { return __float_as_uint(v); }
template <typename V> __device__ __forceinline__ V from_bits(uint32_t b);
template <> __device__ __forceinline__ int32_t from_bits<int32_t>(uint32_t b) { return (int32_t)b; }
template <> __device__ __forceinline__ float from_bits<float>(uint32_t b) { return __uint_as_float(b); }

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

// Published per-tile state of the decoupled look-back.  Status: 0 = nothing,
// 1 = tile aggregate, 2 = inclusive prefix.
//  PACK (4-byte accumulators): one 64-bit word = value bits << 32 | flag << 2 |
//        status, written and read with single relaxed 64-bit accesses (the
//        value travels with its status: one L2 round trip per look-back step).
//  otherwise: a status word released after the payload is stored.
template <class S, bool PACK> struct TileState;
template <class S> struct TileState<S, true> {
    uint64_t *w;
    __device__ __forceinline__ void publish(int64_t t, S s, unsigned st) const {
        st_relaxed64(w + t, ((uint64_t)to_bits(s.v) << 32) | (s.f ? 4ull : 0ull) | st);
    }
    __device__ __forceinline__ unsigned poll(int64_t t, S &s) const {
        const uint64_t x = ld_relaxed64(w + t);
        s.v = from_bits<decltype(s.v)>((uint32_t)(x >> 32));
        s.f = (int)((x >> 2) & 1);
        return (unsigned)(x & 3);
    }
};
template <class S> struct TileState<S, false> {
    uint64_t *w;  // status words (u32) at w, then aggs S[ntiles], incls S[ntiles]
    S *aggs, *incls;
    __device__ __forceinline__ void publish(int64_t t, S s, unsigned st) const {
        st_payload((st == 1 ? aggs : incls) + t, s);
        st_release((unsigned *)w + t, st);
    }
    __device__ __forceinline__ unsigned poll(int64_t t, S &s) const {
        const unsigned st = ld_acquire((const unsigned *)w + t);
        if (st == 1) s = ld_payload(aggs + t);
        else if (st == 2) s = ld_payload(incls + t);
        return st;
    }
};

// 8-byte values (ring scan): value and status in ONE 16-byte word, stored and loaded with single
// 16-byte relaxed accesses (as CUB's tile state does), so a look-back step costs one L2 round
// trip as with PACK.  The status half also carries a 29-bit check of the value: a read that saw
// the new status with a stale value (were a 16-byte access ever split) fails the check and is
// treated as not yet published.
template <class S> struct TileStateW {
    uint64_t *w;  // 2 words per tile
    static __device__ __forceinline__ uint64_t chk(uint64_t v) {
        return (uint64_t)(((uint32_t)(v ^ (v >> 32)) * 0x9E3779B1u) >> 3);
    }
    __device__ __forceinline__ void publish(int64_t t, S s, unsigned st) const {
        const uint64_t lo = (uint64_t)s.v, hi = (chk(lo) << 3) | (s.f ? 4ull : 0ull) | st;
        asm volatile("st.relaxed.gpu.global.v2.u64 [%0], {%1, %2};" ::"l"(w + 2 * t), "l"(lo), "l"(hi) : "memory");
    }
    __device__ __forceinline__ unsigned poll(int64_t t, S &s) const {
        uint64_t lo, hi;
        asm volatile("ld.relaxed.gpu.global.v2.u64 {%0, %1}, [%2];" : "=l"(lo), "=l"(hi) : "l"(w + 2 * t) : "memory");
        unsigned st = (unsigned)(hi & 3);
        if (st && (hi >> 3) != chk(lo)) st = 0;
        s.v = (decltype(s.v))lo;
        s.f = (int)((hi >> 2) & 1);
        return st;
    }
};
// ARGMIN with 4-byte values (slab scan): value, index and status in ONE 16-byte word, like
// TileStateW: lo = value bits | (index + 1) bits 0..31 << 32, hi = (index + 1) bits 32..39 |
// flag << 8 | status << 9 | a 53-bit check of the rest.  Indices below 2^40 - 1.
template <class S> struct TileStateA {
    uint64_t *w;  // 2 words per tile
    static __device__ __forceinline__ uint64_t chk(uint64_t lo, uint64_t hb) {
        const uint64_t h = (lo ^ (hb << 40)) * 0x9E3779B97F4A7C15ull;
        return h >> 11;
    }
    __device__ __forceinline__ void publish(int64_t t, S s, unsigned st) const {
        const uint64_t ip = (uint64_t)(s.v.i + 1);
        const uint64_t lo = (uint64_t)to_bits(s.v.v) | (ip << 32), hb = (ip >> 32) & 0xFF;
        const uint64_t hi = hb | (s.f ? 256ull : 0ull) | ((uint64_t)st << 9) | (chk(lo, hb) << 11);
        asm volatile("st.relaxed.gpu.global.v2.u64 [%0], {%1, %2};" ::"l"(w + 2 * t), "l"(lo), "l"(hi) : "memory");
    }
    __device__ __forceinline__ unsigned poll(int64_t t, S &s) const {
        uint64_t lo, hi;
        asm volatile("ld.relaxed.gpu.global.v2.u64 {%0, %1}, [%2];" : "=l"(lo), "=l"(hi) : "l"(w + 2 * t) : "memory");
        const uint64_t hb = hi & 0xFF;
        unsigned st = (unsigned)((hi >> 9) & 3);
        if (st && (hi >> 11) != chk(lo, hb)) st = 0;
        s.v.v = from_bits<decltype(s.v.v)>((uint32_t)lo);
        s.v.i = (int64_t)((lo >> 32) | (hb << 32)) - 1;
        s.f = (int)((hi >> 8) & 1);
        return st;
    }
};

#ifndef FS_SCAN_R
#define FS_SCAN_R 4
#endif
#ifndef FS_SCAN_NT
#define FS_SCAN_NT 128  // swept on B200 (64/128/256 threads x R = 2/4/8): 128 x 4 fastest
#endif
constexpr int kScanThreads = FS_SCAN_NT;
constexpr unsigned kStAgg = 1, kStIncl = 2;


// 16-byte vectors per lane per tile: 8 for 8-byte (value, flag) pairs, 4 for wider ones
template <int OP, typename T> struct ScanShape {
    static constexpr bool PACK = OP != kArgmin && sizeof(T) == 4;
    static constexpr int R = (OP != kArgmin && sizeof(T) == 4) ? FS_SCAN_R : 2;
    static constexpr int VEC = 16 / sizeof(T);
    static constexpr int64_t TILE = (int64_t)kScanThreads * R * VEC;
    static constexpr unsigned TILE_BYTES = kScanThreads * R * 16;
};

// One pass: every CTA repeatedly takes the next tile id (atomic counter, so all
// predecessors are owned by running CTAs), prefetches the FOLLOWING tile with a
// TMA bulk copy into its second shared-memory buffer, scans the current tile,
// runs the decoupled look-back (warp 0) and writes the tile.  With TMA the next
// tile's HBM read overlaps this tile's scan, look-back and store.
template <int OP, typename T, bool NN, bool SEG, bool TMA>
__global__ void __launch_bounds__(kScanThreads, (TMA ? 768 : 512) / kScanThreads)
scan_kernel(const T *__restrict__ in0, const float *__restrict__ in1, int64_t n, int64_t L, float q0, float q1,
            int64_t ibase, T *__restrict__ out, int64_t *__restrict__ out_idx, const T *carry,
            const int64_t *carry_idx, unsigned *counter, TileState<typename SOp<Op<OP, T>, SEG>::S,
                                                                   ScanShape<OP, T>::PACK> ts,
            int64_t ntiles, bool aligned) {
    using O = Op<OP, T>;
    using SO = SOp<O, SEG>;
    using S = typename SO::S;
    using Sh = ScanShape<OP, T>;
    constexpr int VEC = Sh::VEC, R = Sh::R, NW = kScanThreads / 32;
    constexpr int64_t TILE = Sh::TILE;
    extern __shared__ __align__(128) unsigned char sbuf[];
    __shared__ uint64_t bars[2];
    __shared__ int64_t s_tile[2];
    __shared__ S s_wtot[NW], s_wex[NW], s_ex, s_lb_val[NW];
    __shared__ __align__(16) int s_lb_min[NW];  // aligned: the min over it is read with 16-byte loads
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    // offset in its segment of this lane's first element of row q: one 64-bit modulo per
    // tile, then steps of 32*VEC elements (rows of a lane's tile are 32*VEC apart)
    const int64_t seg_step = SEG ? ((int64_t)32 * VEC) % L : 0;
    int64_t seg_r0 = 0, seg_q0 = -1;
    auto seg_off = [&](int64_t p0, int q) -> int64_t {
        if (q == 0 || seg_q0 < 0) {
            seg_r0 = p0 % L;
        } else {
            seg_r0 += seg_step;
            if (seg_r0 >= L) seg_r0 -= L;
        }
        seg_q0 = q;
        return seg_r0;
    };

    if (threadIdx.x == 0) {
        if (TMA) {
            mbar_init(&bars[0], 1);
            mbar_init(&bars[1], 1);
            fence_mbar_init();
        }
        const int64_t t0 = (int64_t)atomicAdd(counter, 1u);
        s_tile[0] = t0;
        if (TMA && t0 < ntiles && (t0 + 1) * TILE <= n) {
            mbar_expect_tx(&bars[0], Sh::TILE_BYTES);
            tma_load_1d(sbuf, in0 + t0 * TILE, Sh::TILE_BYTES, &bars[0]);
        }
    }
    __syncthreads();
    for (int it = 0;; ++it) {
        const int b = it & 1;
        const int64_t tile = s_tile[b];
        if (tile >= ntiles) break;
        if (threadIdx.x == 0) {
            const int64_t t1 = (int64_t)atomicAdd(counter, 1u);
            s_tile[b ^ 1] = t1;
            if (TMA && t1 < ntiles && (t1 + 1) * TILE <= n) {
                fence_proxy_async();
                mbar_expect_tx(&bars[b ^ 1], Sh::TILE_BYTES);
                tma_load_1d(sbuf + (b ^ 1) * Sh::TILE_BYTES, in0 + t1 * TILE, Sh::TILE_BYTES, &bars[b ^ 1]);
            }
        }
        const bool full = (tile + 1) * TILE <= n;
        if (TMA && full) mbar_wait(&bars[b], (unsigned)(it >> 1) & 1u);
        const int64_t wbase = tile * TILE + (int64_t)warp * 32 * R * VEC;

        // phase A: lane totals per row (the tile stays in shared memory with TMA,
        // otherwise its (mapped) values stay in registers), ordered warp scans
        T xs[TMA ? 1 : R][VEC];
        S pre[R];
        S carry_w = SO::id();
#pragma unroll
        for (int q = 0; q < R; ++q) {
            const int64_t p0 = wbase + ((int64_t)q * 32 + lane) * VEC;
            T x[VEC];
            if (TMA && full) {
                const Vec16<T> a = *reinterpret_cast<const Vec16<T> *>(
                    sbuf + b * Sh::TILE_BYTES + (((warp * R + q) * 32 + lane) << 4));
#pragma unroll
                for (int k = 0; k < VEC; ++k) x[k] = a.e[k];
            } else if (aligned && p0 + VEC <= n) {
                if (NN) {
                    const Vec16<float> a = as_vec<float>(ldg16((const float *)in0 + p0));
                    const Vec16<float> c = as_vec<float>(ldg16(in1 + p0));
#pragma unroll
                    for (int k = 0; k < VEC; ++k) x[k] = (T)nn_distance(a.e[k], c.e[k], q0, q1);
                } else {
                    const Vec16<T> a = as_vec<T>(ldg16(in0 + p0));
#pragma unroll
                    for (int k = 0; k < VEC; ++k) x[k] = a.e[k];
                }
            } else {
#pragma unroll
                for (int k = 0; k < VEC; ++k) {
                    if (p0 + k < n) {
                        if (NN) x[k] = (T)nn_distance(((const float *)in0)[p0 + k], in1[p0 + k], q0, q1);
                        else x[k] = in0[p0 + k];
                    } else {
                        x[k] = T(0);
                    }
                }
            }
            if (!TMA) {
#pragma unroll
                for (int k = 0; k < VEC; ++k) xs[TMA ? 0 : q][k] = x[k];
            }
            int64_t r = SEG ? seg_off(p0, q) : 0;
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
            }
            // ordered inclusive warp scan of the lane totals
            S a = run;
#pragma unroll
            for (int off = 1; off < 32; off <<= 1) {
                const S o = SO::up(a, off);
                if (lane >= off) a = SO::comb(o, a);
            }
            S ex = SO::up(a, 1);
            if (lane == 0) ex = SO::id();
            pre[q] = SO::comb(carry_w, ex);
            carry_w = SO::comb(carry_w, SO::bcast(a, 31));
        }
        if (lane == 0) s_wtot[warp] = carry_w;
        __syncthreads();
        // block aggregate and per-warp exclusive prefixes (every warp computes them)
        S agg;
        {
            S a = lane < NW ? s_wtot[lane] : SO::id();
#pragma unroll
            for (int off = 1; off < 32; off <<= 1) {
                const S o = SO::up(a, off);
                if (lane >= off) a = SO::comb(o, a);
            }
            S wex = SO::up(a, 1);
            if (lane == 0) wex = SO::id();
            if (warp == 0 && lane < NW) s_wex[lane] = wex;
            agg = SO::bcast(a, NW - 1);
        }
        // ---- decoupled look-back with the whole CTA: 256 predecessors per step
        // (all CTAs start together, so the nearest published inclusive prefix is
        // about one wave of resident tiles back; one step covers most of it)
        S exc = SO::id();
        if (tile == 0) {
            if (carry) exc = S{O::lift(*carry, carry_idx ? *carry_idx : -1), 0};
            if (threadIdx.x == 0) ts.publish(0, SO::comb(exc, agg), kStIncl);
        } else {
            if (threadIdx.x == 0) ts.publish(tile, agg, kStAgg);
            int64_t j = tile - 1;
            while (true) {
                const int64_t idx = j - threadIdx.x;
                S v = SO::id();
                unsigned st = kStIncl;
                if (idx >= 0) {
                    do {
                        st = ts.poll(idx, v);
                    } while (st == 0);
                }
                // nearest predecessor holding an inclusive prefix
                const unsigned m = __ballot_sync(0xffffffffu, idx >= 0 && st == kStIncl);
                if (lane == 0) s_lb_min[warp] = m ? warp * 32 + __ffs(m) - 1 : 1 << 20;
                __syncthreads();
                int kk = 1 << 20;
#pragma unroll
                for (int q = 0; q < NW; ++q) kk = min(kk, s_lb_min[q]);
                if ((int)threadIdx.x > kk || idx < 0) v = SO::id();
                // ordered reduction: higher thread ids are further left
#pragma unroll
                for (int off = 1; off < 32; off <<= 1) {
                    const S o = SO::down(v, off);
                    if (lane + off < 32) v = SO::comb(o, v);
                }
                if (lane == 0) s_lb_val[warp] = v;
                __syncthreads();
                S P = SO::id();
#pragma unroll
                for (int q = NW - 1; q >= 0; --q) P = SO::comb(P, s_lb_val[q]);
                exc = SO::comb(P, exc);
                __syncthreads();  // s_lb_* reuse
                if (kk < (1 << 20) || exc.f) break;
                j -= kScanThreads;
            }
            if (threadIdx.x == 0) ts.publish(tile, SO::comb(exc, agg), kStIncl);
        }
        if (threadIdx.x == 0) s_ex = exc;
        __syncthreads();
        // phase C: re-derive every element's inclusive value from the tile prefix
        const S base = SO::comb(s_ex, s_wex[warp]);
#pragma unroll
        for (int q = 0; q < R; ++q) {
            const int64_t p0 = wbase + ((int64_t)q * 32 + lane) * VEC;
            T x[VEC];
            if (TMA && full) {
                const Vec16<T> a = *reinterpret_cast<const Vec16<T> *>(
                    sbuf + b * Sh::TILE_BYTES + (((warp * R + q) * 32 + lane) << 4));
#pragma unroll
                for (int k = 0; k < VEC; ++k) x[k] = a.e[k];
            } else if (TMA) {
#pragma unroll
                for (int k = 0; k < VEC; ++k) x[k] = p0 + k < n ? in0[p0 + k] : T(0);
            } else {
#pragma unroll
                for (int k = 0; k < VEC; ++k) x[k] = xs[TMA ? 0 : q][k];
            }
            S run = SO::comb(base, pre[q]);
            int64_t r = SEG ? seg_off(p0, q) : 0;
            T y[VEC];
            int64_t yi[VEC];
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
                y[k] = O::val(run.v);
                yi[k] = O::idx(run.v);
            }
            if (aligned && p0 + VEC <= n) {
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
        __syncthreads();  // smem buffers, s_tile and s_ex reuse
    }
}

// ---------------------------------------------------------------- warp-specialised slab scan
// The default path for 16-byte aligned inputs and outputs.  One CTA per SM.  The
// array is cut into tiles of TILE_BYTES and the tiles into slabs of `tps`
// consecutive tiles; CTA b owns slabs b, b+G, b+2G, ... (a "round" is G consecutive
// slabs).  Three warp roles run concurrently in every CTA:
//   A (4 warps)  REDUCE each slab as it streams from HBM through an STA-stage TMA
//                ring: the slab's look-back record is a commutative masked reduction
//                (for the segmented operator only elements at or after the slab's last
//                segment start count -- a closed form for regular segments), published
//                as soon as the slab has been read.
//   C (8 warps)  per slab: one decoupled look-back over the records of the preceding
//                slabs (window 256 >= G, one L2 round trip per slab), then scan the slab
//                tile by tile with a running carry from an STC-stage ring that re-reads
//                it from L2 (group A read it a moment ago), thread-contiguous R (odd)
//                vectors per thread (bank-conflict free), results written back in place.
//   P (1 warp)   the producer: issues every TMA load of both rings and the TMA bulk
//                store of every scanned tile, driven by mbarriers (A/C "slot consumed",
//                C "tile written back"); keeps group A at most DA slabs ahead of C so
//                the slabs between the two passes stay in L2 (G*(DA+1) slabs).
// HBM traffic is one read and one write per element.  This is F5 (L1071-1074) in
// B200 form: A computes the chunk aggregates, C the chunk scans with the carried
// prefix a, and the look-back composes the carries.
#ifndef FS_SCANW_R
#define FS_SCANW_R 7
#endif
#ifndef FS_SCANW_STA
#define FS_SCANW_STA 4
#endif
#ifndef FS_SCANW_STC
#define FS_SCANW_STC 3
#endif
#ifndef FS_SCANW_DA
#define FS_SCANW_DA 2
#endif
#ifndef FS_SCANW_TPS
#define FS_SCANW_TPS 4
#endif
#ifndef FS_SCANW_NC
#define FS_SCANW_NC 256
#endif
constexpr int kScanWA = 128, kScanWC = FS_SCANW_NC, kScanWThreads = kScanWA + kScanWC + 32;
template <int OP, typename T> struct ScanWShape {
    static constexpr bool PACK = OP != kArgmin && sizeof(T) == 4;
    static constexpr int R = FS_SCANW_R;  // C: 16-byte vectors per thread per tile
    static_assert(R % 2 == 1, "R must be odd (bank-conflict-free thread-contiguous vectors)");
    static constexpr int VEC = 16 / sizeof(T);
    static constexpr int E = R * VEC;
    static constexpr int64_t TILE = (int64_t)kScanWC * E;
    static constexpr unsigned TILE_BYTES = kScanWC * R * 16;
    static constexpr int RA = kScanWC * R / kScanWA;  // A: vectors per thread per tile
    static_assert(kScanWC * R % kScanWA == 0, "A threads split a tile evenly");
    static constexpr int STA = FS_SCANW_STA, STC = FS_SCANW_STC;
    static constexpr unsigned SMEM = (STA + STC) * TILE_BYTES;
};
template <int OP, typename T, bool SEG>
using WsState = typename std::conditional<
    ScanWShape<OP, T>::PACK, TileState<typename SOp<Op<OP, T>, SEG>::S, true>,
    typename std::conditional<OP == kArgmin && sizeof(T) == 4, TileStateA<typename SOp<Op<OP, T>, SEG>::S>,
                              TileState<typename SOp<Op<OP, T>, SEG>::S, false>>::type>::type;

__device__ __forceinline__ void named_bar(int id, int count) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(count) : "memory");
}
__device__ __forceinline__ bool mbar_test(uint64_t *bar, unsigned parity) {
    uint32_t done;
    asm volatile(
        "{\n\t.reg .pred p;\n\tmbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(done)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
    return done != 0;
}
__device__ __forceinline__ void mbar_arrive(uint64_t *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ uint64_t l2_policy_evict_last() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint64_t l2_policy_evict_first() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ void tma_load_1d_hint(void *dst, const void *src, unsigned bytes, uint64_t *bar,
                                                 uint64_t pol) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], "
        "%4;" ::"r"(smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol)
        : "memory");
}
__device__ __forceinline__ void tma_store_1d_hint(void *dst, const void *src, unsigned bytes, uint64_t pol) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group.L2::cache_hint [%0], [%1], %2, %3;" ::"l"(dst),
                 "r"(smem_u32(src)), "r"(bytes), "l"(pol)
                 : "memory");
}
__device__ __forceinline__ void bulk_wait_read_n(int n) {  // all but the n most recent groups have read
    if (n <= 0) bulk_wait_read<0>();
    else if (n == 1) bulk_wait_read<1>();
    else if (n == 2) bulk_wait_read<2>();
    else bulk_wait_read<3>();
}

template <int OP, typename T, bool SEG>
__global__ void __launch_bounds__(kScanWThreads, 1)
scan_ws_kernel(const T *__restrict__ in, int64_t n, int64_t L, int64_t ibase, T *__restrict__ out,
               int64_t *__restrict__ out_idx, const T *carry, const int64_t *carry_idx,
               WsState<OP, T, SEG> ts, int64_t ntiles, int tps) {
    using O = Op<OP, T>;
    using V = typename O::V;
    using SO = SOp<O, SEG>;
    using S = typename SO::S;
    using Sh = ScanWShape<OP, T>;
    constexpr int VEC = Sh::VEC, R = Sh::R, E = Sh::E, RA = Sh::RA, STA = Sh::STA, STC = Sh::STC;
    constexpr int NWA = kScanWA / 32, NWC = kScanWC / 32;
    constexpr int64_t TILE = Sh::TILE;
    constexpr unsigned TB = Sh::TILE_BYTES;
    extern __shared__ __align__(128) unsigned char sbuf[];
    unsigned char *ringA = sbuf, *ringC = sbuf + STA * TB;
    __shared__ uint64_t fullA[STA], emptyA[STA], fullC[STC], doneC[STC];
    __shared__ int s_c_slab;  // slab (local index) group C is working on (shared-memory atomics: a
                              // monotone progress flag read by the producer, no ordering needed)
    __shared__ V s_redA[NWA];
    __shared__ S s_wtot[2][NWC], s_lb_val[NWC];
    __shared__ __align__(16) int s_lb_min[NWC];  // 16-byte aligned: its vector loads stay inside it
    const int G = gridDim.x, b = blockIdx.x;
    const int64_t nslabs = (ntiles + tps - 1) / tps;
    const int my_slabs = (int)((nslabs - b + G - 1) / G);
    // tile sequence of this CTA: j -> (local slab j / tps, tile j % tps of it)
    auto slab_of = [&](int m) { return (int64_t)b + (int64_t)m * G; };
    auto tile_at = [&](int j) { return slab_of(j / tps) * tps + j % tps; };
    const int my_tiles = my_slabs == 0 ? 0 : (int)((my_slabs - 1) * (int64_t)tps +
                                                   (min((int64_t)tps, ntiles - slab_of(my_slabs - 1) * tps)));
    auto full_tile = [&](int64_t t) { return (t + 1) * TILE <= n; };
    const int tid = threadIdx.x;
    if (tid == 0) {
        for (int s = 0; s < STA; ++s) {
            mbar_init(&fullA[s], 1);
            mbar_init(&emptyA[s], kScanWA);
        }
        for (int s = 0; s < STC; ++s) {
            mbar_init(&fullC[s], 1);
            mbar_init(&doneC[s], kScanWC);
        }
        fence_mbar_init();
        s_c_slab = 0;
    }
    __syncthreads();

    if (tid >= kScanWA + kScanWC) {
        // ================================================================ P: producer
        if (tid != kScanWA + kScanWC) return;
        const uint64_t keep = l2_policy_evict_last(), stream = l2_policy_evict_first();
        int a_iss = 0, a_rel = 0, c_iss = 0, c_st = 0;
        while (c_st < my_tiles) {
            // A: a slot is released when all of group A has consumed its tile
            while (a_rel < a_iss && mbar_test(&emptyA[a_rel % STA], (unsigned)(a_rel / STA) & 1u)) ++a_rel;
            // A: issue while a slot is free and A stays within DA slabs of C
            while (a_iss < my_tiles && a_iss < a_rel + STA && a_iss / tps - FS_SCANW_DA <= atomicAdd(&s_c_slab, 0)) {
                const int64_t t = tile_at(a_iss);
                if (full_tile(t)) {
                    const int s = a_iss % STA;
                    mbar_expect_tx(&fullA[s], TB);
                    tma_load_1d_hint(ringA + s * TB, in + t * TILE, TB, &fullA[s], keep);
                }
                ++a_iss;
            }
            // C: store every tile group C has written back (in order)
            while (c_st < c_iss && mbar_test(&doneC[c_st % STC], (unsigned)(c_st / STC) & 1u)) {
                const int64_t t = tile_at(c_st);
                if (full_tile(t)) tma_store_1d_hint(out + t * TILE, ringC + (c_st % STC) * TB, TB, stream);
                bulk_commit();
                ++c_st;
            }
            // C: re-load (from L2) tiles group A has finished, into slots whose store has read them
            while (c_iss < my_tiles && c_iss < a_rel && c_iss < c_st + STC) {
                const int old = c_iss - STC;  // previous tile of this slot; its store is group `old`
                if (old >= 0) bulk_wait_read_n(c_st - 1 - old);
                const int64_t t = tile_at(c_iss);
                if (full_tile(t)) {
                    const int s = c_iss % STC;
                    fence_proxy_async();
                    mbar_expect_tx(&fullC[s], TB);
                    tma_load_1d_hint(ringC + s * TB, in + t * TILE, TB, &fullC[s], stream);
                }
                ++c_iss;
            }
        }
        bulk_wait<0>();
        return;
    }
    if (tid < kScanWA) {
        // ================================================================ A: slab records
        const int lane = tid & 31, warp = tid >> 5;
        int j = 0;
        for (int m = 0; m < my_slabs; ++m) {
            const int64_t slab = slab_of(m);
            const int64_t s0 = slab * tps * TILE, s1 = min(n, (slab + 1) * tps * TILE);
            // SEG: the record covers the slab's elements from its last segment start on (all
            // of them when no segment starts in it); they lie in ONE segment starting at `base`
            int64_t keep = s0, base = 0;
            int flag = 0;
            if (SEG) {
                const int64_t last_start = ((s1 - 1) / L) * L;
                flag = last_start >= s0;
                keep = flag ? last_start : s0;
                base = flag ? last_start : (s0 / L) * L;
            }
            V acc = O::id();
            const int64_t t_end = min(ntiles, (slab + 1) * tps);
            for (int64_t t = slab * tps; t < t_end; ++t, ++j) {
                const int s = j % STA;
                const bool full = full_tile(t);
                const int64_t t0 = t * TILE, t1 = t0 + TILE;
                if (full) mbar_wait(&fullA[s], (unsigned)(j / STA) & 1u);
                if (SEG && t1 <= keep) {
                    // entirely before the slab's last segment start: not part of the record
                } else if (full && (!SEG || t0 >= keep)) {
#pragma unroll
                    for (int q = 0; q < RA; ++q) {
                        const int vi = q * kScanWA + tid;
                        const int64_t p0 = t0 + (int64_t)vi * VEC;
                        const Vec16<T> a = *reinterpret_cast<const Vec16<T> *>(ringA + s * TB + vi * 16);
#pragma unroll
                        for (int k = 0; k < VEC; ++k)
                            acc = O::comb(acc, O::lift(a.e[k], SEG ? p0 + k - base : ibase + p0 + k));
                    }
                } else {
#pragma unroll
                    for (int q = 0; q < RA; ++q) {
                        const int vi = q * kScanWA + tid;
                        const int64_t p0 = t0 + (int64_t)vi * VEC;
                        T x[VEC];
                        if (full) {
                            const Vec16<T> a = *reinterpret_cast<const Vec16<T> *>(ringA + s * TB + vi * 16);
#pragma unroll
                            for (int k = 0; k < VEC; ++k) x[k] = a.e[k];
                        } else {
#pragma unroll
                            for (int k = 0; k < VEC; ++k) x[k] = p0 + k < n ? in[p0 + k] : T(0);
                        }
#pragma unroll
                        for (int k = 0; k < VEC; ++k) {
                            const int64_t pk = p0 + k;
                            if (pk < s1 && (!SEG || pk >= keep))
                                acc = O::comb(acc, O::lift(x[k], SEG ? pk - base : ibase + pk));
                        }
                    }
                }
                mbar_arrive(&emptyA[s]);
            }
            acc = group_reduce<O>(acc);
            if (lane == 0) s_redA[warp] = acc;
            named_bar(1, kScanWA);
            if (tid == 0) {
                V tot = O::id();
#pragma unroll
                for (int q = 0; q < NWA; ++q) tot = O::comb(tot, s_redA[q]);
                S agg{tot, flag};
                if (slab == 0) {
                    S c0 = SO::id();
                    if (carry) c0 = S{O::lift(*carry, carry_idx ? *carry_idx : -1), 0};
                    ts.publish(0, SO::comb(c0, agg), kStIncl);
                } else {
                    // a flagged record is already the inclusive prefix
                    ts.publish(slab, agg, (SEG && flag) ? kStIncl : kStAgg);
                }
            }
            named_bar(1, kScanWA);  // s_redA reuse
        }
        return;
    }
    // ==================================================================== C: look-back + scan
    const int ct = tid - kScanWA, lane = ct & 31, warp = ct >> 5;
    int j = 0;
    for (int m = 0; m < my_slabs; ++m) {
        const int64_t slab = slab_of(m);
        if (ct == 0) atomicExch(&s_c_slab, m);
        S exc = SO::id();
        if (slab == 0) {
            if (carry) exc = S{O::lift(*carry, carry_idx ? *carry_idx : -1), 0};
        } else if (!(SEG && (slab * tps * TILE) % L == 0)) {
            int64_t jj = slab - 1;
            while (true) {
                const int64_t idx = jj - ct;
                S v = SO::id();
                unsigned st = kStIncl;
                if (idx >= 0) {
                    do {
                        st = ts.poll(idx, v);
                    } while (st == 0);
                }
                const unsigned msk = __ballot_sync(0xffffffffu, idx >= 0 && st == kStIncl);
                if (lane == 0) s_lb_min[warp] = msk ? warp * 32 + __ffs(msk) - 1 : 1 << 30;
                named_bar(2, kScanWC);
                int kk = 1 << 30;
#pragma unroll
                for (int q = 0; q < NWC; ++q) kk = min(kk, s_lb_min[q]);
                if (ct > kk || idx < 0) v = SO::id();
                S w = v;
#pragma unroll
                for (int off = 1; off < 32; off <<= 1) {
                    const S o = SO::down(w, off);
                    if (lane + off < 32) w = SO::comb(o, w);
                }
                if (lane == 0) s_lb_val[warp] = w;
                named_bar(2, kScanWC);
                S P = SO::id(), left = SO::id();
#pragma unroll
                for (int q = NWC - 1; q >= 0; --q) {
                    if (q > warp) left = SO::comb(left, s_lb_val[q]);
                    P = SO::comb(P, s_lb_val[q]);
                }
                // help forward: records between here and the nearest inclusive prefix
                if (kk < (1 << 30) && idx >= 0 && ct < kk && st == kStAgg) ts.publish(idx, SO::comb(left, w), kStIncl);
                exc = SO::comb(P, exc);
                named_bar(2, kScanWC);  // s_lb_* reuse
                if (kk < (1 << 30) || exc.f || jj < kScanWC) break;
                jj -= kScanWC;
            }
        }
        S run_c = exc;
        const int64_t t_end = min(ntiles, (slab + 1) * tps);
        // offset in its segment of this thread's first element: one division per slab
        int64_t r0 = SEG ? (slab * tps * TILE + (int64_t)ct * E) % L : 0;
        for (int64_t t = slab * tps; t < t_end; ++t, ++j) {
            const int s = j % STC;
            const bool full = full_tile(t);
            const int64_t e0 = t * TILE + (int64_t)ct * E;
            unsigned char *sv = ringC + s * TB + ct * (R * 16);
            T x[E];
            if (full) {
                mbar_wait(&fullC[s], (unsigned)(j / STC) & 1u);
#pragma unroll
                for (int r = 0; r < R; ++r) {
                    const Vec16<T> a = *reinterpret_cast<const Vec16<T> *>(sv + r * 16);
#pragma unroll
                    for (int k = 0; k < VEC; ++k) x[r * VEC + k] = a.e[k];
                }
            } else {
#pragma unroll
                for (int i = 0; i < E; ++i) x[i] = e0 + i < n ? in[e0 + i] : T(0);
            }
            auto valid = [&](int i) { return full || e0 + i < n; };
            // SEG with L >= E: at most one segment start among a thread's E elements, at i0
            const bool one = SEG && L >= E;
            const int i0 = !SEG ? E : (r0 == 0 ? 0 : (L - r0 < E ? (int)(L - r0) : E));
            auto lifted = [&](int i, int64_t &r) {
                S e;
                if (valid(i)) {
                    e.v = O::lift(x[i], SEG ? r : ibase + e0 + i);
                    e.f = SEG ? (r == 0) : 0;
                } else {
                    e = SO::id();
                }
                if (SEG) {
                    ++r;
                    if (r == L) r = 0;
                }
                return e;
            };
            auto seg_idx = [&](int i) -> int64_t { return i < i0 ? r0 + i : i - i0; };  // one-start case
            S tot = SO::id();
            // fast path (a full tile, no segment start among this thread's elements): a plain
            // fold, no per-element validity or restart tests
            const bool plainrun = full && (!SEG || (one && i0 >= E));
            if (plainrun) {
                V acc = O::id();
#pragma unroll
                for (int i = 0; i < E; ++i) acc = O::comb(acc, O::lift(x[i], SEG ? r0 + i : ibase + e0 + i));
                tot = S{acc, 0};
            } else if (one) {
                V acc = O::id();
#pragma unroll
                for (int i = 0; i < E; ++i)
                    if (valid(i)) {
                        const V e = O::lift(x[i], seg_idx(i));
                        acc = i == i0 ? e : O::comb(acc, e);
                    }
                tot = S{acc, i0 < E};
            } else {
                int64_t r = r0;
#pragma unroll
                for (int i = 0; i < E; ++i) tot = SO::comb(tot, lifted(i, r));
            }
            S a = tot;
#pragma unroll
            for (int off = 1; off < 32; off <<= 1) {
                const S o = SO::up(a, off);
                if (lane >= off) a = SO::comb(o, a);
            }
            S tex = SO::up(a, 1);
            if (lane == 0) tex = SO::id();
            if (lane == 31) s_wtot[j & 1][warp] = a;
            named_bar(2, kScanWC);
            S bsc = lane < NWC ? s_wtot[j & 1][lane] : SO::id();
#pragma unroll
            for (int off = 1; off < NWC; off <<= 1) {
                const S o = SO::up(bsc, off);
                if (lane >= off) bsc = SO::comb(o, bsc);
            }
            S bex = SO::up(bsc, 1);
            if (lane == 0) bex = SO::id();
            const S wex = SO::bcast(bex, warp), tagg = SO::bcast(bsc, NWC - 1);
            S run = SO::comb(run_c, SO::comb(wex, tex));
            run_c = SO::comb(run_c, tagg);
            T y[E];
            if (plainrun) {
                V acc = run.v;
#pragma unroll
                for (int i = 0; i < E; ++i) {
                    acc = O::comb(acc, O::lift(x[i], SEG ? r0 + i : ibase + e0 + i));
                    y[i] = O::val(acc);
                    if (OP == kArgmin) out_idx[e0 + i] = O::idx(acc);
                }
            } else if (one) {
                V acc = run.v;
#pragma unroll
                for (int i = 0; i < E; ++i) {
                    if (valid(i)) {
                        const V e = O::lift(x[i], seg_idx(i));
                        acc = i == i0 ? e : O::comb(acc, e);
                    }
                    y[i] = O::val(acc);
                    if (OP == kArgmin && valid(i)) out_idx[e0 + i] = O::idx(acc);
                }
            } else {
                int64_t r = r0;
#pragma unroll
                for (int i = 0; i < E; ++i) {
                    run = SO::comb(run, lifted(i, r));
                    y[i] = O::val(run.v);
                    if (OP == kArgmin && valid(i)) out_idx[e0 + i] = O::idx(run.v);
                }
            }
            if (SEG) {
                r0 += TILE % L;
                if (r0 >= L) r0 -= L;
            }
            if (full) {
#pragma unroll
                for (int r = 0; r < R; ++r) {
                    Vec16<T> w;
#pragma unroll
                    for (int k = 0; k < VEC; ++k) w.e[k] = y[r * VEC + k];
                    *reinterpret_cast<Vec16<T> *>(sv + r * 16) = w;
                }
                fence_proxy_async();  // written back -> visible to the producer's bulk store
            } else {
#pragma unroll
                for (int i = 0; i < E; ++i)
                    if (e0 + i < n) out[e0 + i] = y[i];
            }
            mbar_arrive(&doneC[s]);
        }
        // the slab's inclusive prefix (group A may already have published an equal one)
        if (ct == 0) ts.publish(slab, run_c, kStIncl);
    }
    if (ct == 0) s_c_slab = 1 << 30;
}

static size_t scan_state_bytes(int64_t ntiles) { return align_up((size_t)ntiles * 8, 256); }

// ---------------------------------------------------------------- KS0: short power-of-two segments
// seg_scan for regular segments of length L = 2^j <= 32 * VEC with 16-byte aligned
// buffers.  A 16-byte vector never straddles a segment boundary unless L < VEC, and a
// segment of L > VEC elements is G = L / VEC consecutive vectors, i.e. G consecutive
// lanes of one warp (the grid-stride order maps vector v to lane v mod 32).  So the
// segmented scan needs no look-back and no segment flags at all: an in-register scan of
// the lane's vector, then an inclusive shuffle scan of the lane totals within each
// G-lane group (log2 G steps) and one (+) per element.  One read and one write per
// element, like a copy.
template <int OP, typename T, int U>
__global__ void __launch_bounds__(256)
segscan_vec_kernel(const T *__restrict__ x, int64_t n, int L, int G, T *__restrict__ out, int64_t *__restrict__ out_idx) {
    using O = Op<OP, T>;
    using V = typename O::V;
    constexpr int VEC = 16 / sizeof(T);
    const int lane = threadIdx.x & 31, lg = lane & (G - 1);
    const int64_t nvec = n / VEC;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t gid0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t iters = (nvec + stride - 1) / stride;  // warp-uniform: every lane shuffles
    // software pipeline: the next batch's loads are in flight while this batch is scanned
    int4 r[U], rn[U];
    auto load_batch = [&](int64_t i0, int4 (&dst)[U]) {
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t v = gid0 + (i0 + u) * stride;
            if (i0 + u < iters && v < nvec) dst[u] = ldg16(x + v * VEC);
        }
    };
    if (iters > 0) load_batch(0, r);
    for (int64_t it0 = 0; it0 < iters; it0 += U) {
        if (it0 + U < iters) load_batch(it0 + U, rn);
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t v = gid0 + (it0 + u) * stride;
            const bool ok = it0 + u < iters && v < nvec;
            if (it0 + u >= iters) break;  // warp-uniform
            const Vec16<T> e = as_vec<T>(r[u]);
            V a[VEC];
            if (L <= VEC) {  // whole segments inside the vector
#pragma unroll
                for (int k = 0; k < VEC; ++k) {
                    const int j = k & (L - 1);  // segment-local index
                    a[k] = j == 0 ? O::lift(e.e[k], 0) : O::fold(a[k > 0 ? k - 1 : 0], e.e[k], j);
                }
            } else {
                const int j0 = lg * VEC;  // segment-local index of the vector's first element
#pragma unroll
                for (int k = 0; k < VEC; ++k) a[k] = k == 0 ? O::lift(e.e[0], j0) : O::fold(a[k - 1], e.e[k], j0 + k);
                V incl = ok ? a[VEC - 1] : O::id();
#pragma unroll 1
                for (int dd = 1; dd < G; dd <<= 1) {
                    const V y = shfl_up(incl, dd);
                    if (lg >= dd) incl = O::comb(y, incl);
                }
                V ex = shfl_up(incl, 1);
                if (lg == 0) ex = O::id();
#pragma unroll
                for (int k = 0; k < VEC; ++k) a[k] = O::comb(ex, a[k]);
            }
            if (ok) {
                Vec16<T> o;
#pragma unroll
                for (int k = 0; k < VEC; ++k) o.e[k] = O::val(a[k]);
                *reinterpret_cast<int4 *>(out + v * VEC) = *reinterpret_cast<const int4 *>(&o);
                if (out_idx)
#pragma unroll
                    for (int k = 0; k < VEC; ++k) out_idx[v * VEC + k] = O::idx(a[k]);
            }
        }
#pragma unroll
        for (int u = 0; u < U; ++u) r[u] = rn[u];
    }
    // ragged tail (L < VEC and n not a multiple of VEC): whole segments, one per thread
    const int64_t t0 = nvec * VEC;
    for (int64_t sgi = t0 / L + gid0; sgi * L < n; sgi += stride) {
        V acc = O::id();
        for (int j = 0; j < L; ++j) {
            acc = j == 0 ? O::lift(x[sgi * L], 0) : O::fold(acc, x[sgi * L + j], j);
            out[sgi * L + j] = O::val(acc);
            if (out_idx) out_idx[sgi * L + j] = O::idx(acc);
        }
    }
}

// KS0 for rows that span 2..8 warps of a 256-thread CTA (32 * VEC < L <= 256 * VEC, L = 2^j):
// a CTA takes U chunks of 256 consecutive vectors (each chunk = 256 * VEC / L whole
// segments); every lane scans its vector in registers, every warp scans its lane totals
// with shuffles, and the warps of a segment combine their totals through shared memory
// (one barrier per U chunks).  No look-back, no flags: one read, one write per element.
// BIG: rows of 2..U chunks (256 * VEC < L <= U * 256 * VEC, U = 4 or 8); a row's warps then
// span chunks of one step, and warp 0 scans the U * 8 warp totals (segmented by row, U / 4
// totals per lane).
template <int OP, typename T, int U, bool BIG = false>
__global__ void __launch_bounds__(256)
segscan_blk_kernel(const T *__restrict__ x, int64_t n, int L, T *__restrict__ out, int64_t *__restrict__ out_idx) {
    using O = Op<OP, T>;
    using V = typename O::V;
    constexpr int VEC = 16 / sizeof(T);
    static_assert(!BIG || U == 4 || U == 8, "one warp scans the step's U * 8 warp totals, 1 or 2 per lane");
    __shared__ V wt[U][8];
    __shared__ V wx[BIG ? U * 8 : 1];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int WS = L / (32 * VEC);          // warps per segment (2, 4 or 8)
    const int wr = warp & (WS - 1);         // rank of this warp within its segment
    const int64_t nvec = n / VEC;  // whole segments are whole warps: a partial last chunk ends on a warp boundary
    const int64_t nchunk = (nvec + 255) / 256;
    for (int64_t c0 = (int64_t)blockIdx.x * U; c0 < nchunk; c0 += (int64_t)gridDim.x * U) {
        int4 r[U];
#pragma unroll
        for (int u = 0; u < U; ++u)
            if ((c0 + u) * 256 + threadIdx.x < nvec) r[u] = ldg16(x + ((c0 + u) * 256 + threadIdx.x) * VEC);
        V a[U][VEC], ex[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const Vec16<T> e = as_vec<T>(r[u]);
            const int wru = BIG ? ((u * 8 + warp) & (WS - 1)) : wr;
            const int j0 = (wru * 32 + lane) * VEC;  // segment-local index of the first element
#pragma unroll
            for (int k = 0; k < VEC; ++k)
                a[u][k] = k == 0 ? O::lift(e.e[0], j0) : O::fold(a[u][k - 1], e.e[k], j0 + k);
            V incl = a[u][VEC - 1];
#pragma unroll
            for (int dd = 1; dd < 32; dd <<= 1) {
                const V y = shfl_up(incl, dd);
                if (lane >= dd) incl = O::comb(y, incl);
            }
            ex[u] = shfl_up(incl, 1);
            if (lane == 0) ex[u] = O::id();
            if (lane == 31) wt[u][warp] = incl;
        }
        __syncthreads();
        if constexpr (BIG) {
            if (warp == 0) {
                constexpr int P = U / 4;           // warp totals per lane (a pair never straddles a row: WS >= 16)
                const int rk = lane & (WS / P - 1);  // rank of this lane's totals within their row
                const V t0 = (&wt[0][0])[lane * P];
                const V t1 = P == 2 ? (&wt[0][0])[lane * P + P - 1] : O::id();
                V incl = P == 2 ? O::comb(t0, t1) : t0;
#pragma unroll
                for (int dd = 1; dd < 32; dd <<= 1) {
                    const V y = shfl_up(incl, dd);
                    if (rk >= dd) incl = O::comb(y, incl);
                }
                V e = shfl_up(incl, 1);
                if (rk == 0) e = O::id();
                wx[lane * P] = e;
                if (P == 2) wx[lane * P + 1] = O::comb(e, t0);
            }
            __syncthreads();
#pragma unroll
            for (int u = 0; u < U; ++u) ex[u] = O::comb(wx[u * 8 + warp], ex[u]);
        } else {
#pragma unroll
            for (int u = 0; u < U; ++u) {
                V p = O::id();
                for (int q = warp - wr; q < warp; ++q) p = O::comb(p, wt[u][q]);
                ex[u] = O::comb(p, ex[u]);
            }
        }
        __syncthreads();  // wt / wx are reused by the next chunks
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t v = (c0 + u) * 256 + threadIdx.x;
            if (v >= nvec) break;
            Vec16<T> o;
#pragma unroll
            for (int k = 0; k < VEC; ++k) {
                const V z = O::comb(ex[u], a[u][k]);
                o.e[k] = O::val(z);
                if (out_idx) out_idx[v * VEC + k] = O::idx(z);
            }
            *reinterpret_cast<int4 *>(out + v * VEC) = *reinterpret_cast<const int4 *>(&o);
        }
    }
}

// KS3: rows of any length 32 < L <= 16384 (non-powers of two, whose 16-byte vectors straddle
// rows): a CTA takes R whole rows (R * L ~ 8192 elements) at a time, so no scan crosses a CTA
// and there is no look-back.  The rows are staged in shared memory by coalesced loads, each
// thread scans a contiguous piece sequentially (restarting at row heads), the CTA scans the
// 256 (head seen, total) piece summaries, each piece's first partial row takes its carry, and
// the rows leave by coalesced stores.  ADD/MIN/MAX (argmin's index output keeps the look-back).
constexpr int kRowsElems = 8192;
template <int OP, typename T>
__global__ void __launch_bounds__(256)
segscan_rows_kernel(const T *__restrict__ x, int64_t nseg, int64_t L, int64_t R, T *__restrict__ out) {
    using O = Op<OP, T>;
    extern __shared__ __align__(16) unsigned char smem_rows[];
    T *buf = reinterpret_cast<T *>(smem_rows);
    __shared__ T s_wa[8];
    __shared__ int s_wf[8];
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int64_t nchunk = (nseg + R - 1) / R;
    for (int64_t c = blockIdx.x; c < nchunk; c += gridDim.x) {
        const int64_t r0 = c * R, rows = (r0 + R < nseg ? r0 + R : nseg) - r0;
        const int cnt = (int)(rows * L);
        const T *src = x + r0 * L;
#pragma unroll 8
        for (int i = tid; i < cnt; i += 256) buf[i] = __ldcs(src + i);
        __syncthreads();
        const int E = ((cnt + 255) / 256) | 1;  // odd piece length: the lanes' strided reads hit distinct banks
        const int i0 = tid * E < cnt ? tid * E : cnt, i1 = i0 + E < cnt ? i0 + E : cnt;
        int j = (int)(i0 % L);  // position of element i0 in its row
        T acc = O::id();
        int f = 0;  // a row head lies in this piece
        for (int i = i0; i < i1; ++i) {
            const T v = buf[i];
            if (j == 0) {
                acc = v;
                f = 1;
            } else {
                acc = O::comb(acc, v);
            }
            buf[i] = acc;
            if (++j == L) j = 0;
        }
        // inclusive segmented scan of the (f, acc) piece summaries: (f1,a1).(f2,a2) = (f1|f2, f2 ? a2 : a1.a2)
        T a = acc;
        int fl = f;
#pragma unroll
        for (int dd = 1; dd < 32; dd <<= 1) {
            const T ya = shfl_up(a, dd);
            const int yf = __shfl_up_sync(0xffffffffu, fl, dd);
            if (lane >= dd) {
                if (!fl) a = O::comb(ya, a);
                fl |= yf;
            }
        }
        if (lane == 31) {
            s_wa[warp] = a;
            s_wf[warp] = fl;
        }
        __syncthreads();
        // exclusive prefix of this piece = (warps before, combined in order) . (lanes before in this warp)
        T ex = shfl_up(a, 1);
        int exf = __shfl_up_sync(0xffffffffu, fl, 1);
        if (lane == 0) {
            ex = O::id();
            exf = 0;
        }
        if (!exf) {
            T p = O::id();
            for (int q = 0; q < warp; ++q) p = s_wf[q] ? s_wa[q] : O::comb(p, s_wa[q]);
            ex = O::comb(p, ex);
        }
        // the piece's elements before its first row head continue the previous piece's row
        {
            int jj = (int)(i0 % L);
            for (int i = i0; i < i1 && jj != 0; ++i) {
                buf[i] = O::comb(ex, buf[i]);
                if (++jj == L) jj = 0;
            }
        }
        __syncthreads();
        T *dst = out + r0 * L;
#pragma unroll 8
        for (int i = tid; i < cnt; i += 256) __stcs(dst + i, buf[i]);
        __syncthreads();  // buf / s_wa reused by the next chunk
    }
}

// KS3 with TMA (16-byte aligned input and output): the same piece scan, but tiles of R whole
// rows (R * L * sizeof(T) a multiple of 16 bytes, <= 72 KB) arrive by TMA bulk copies into a
// 3-slot ring (the tile two ahead is in flight while this one is scanned) and leave by TMA bulk
// stores straight from shared memory; one CTA loop per resident slot.  Full tiles only: the
// nseg mod R leftover rows take segscan_rows_kernel.
template <int OP, typename T>
__global__ void __launch_bounds__(256)
segscan_rows_tma_kernel(const T *__restrict__ x, int64_t ntiles, int64_t L, int R, T *__restrict__ out) {
    using O = Op<OP, T>;
    extern __shared__ __align__(128) unsigned char smem_rt[];
    __shared__ uint64_t full[3];
    __shared__ T s_wa[8];
    __shared__ int s_wf[8];
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int cnt = (int)(R * L);
    const unsigned TB = (unsigned)cnt * sizeof(T);
    const int64_t G = gridDim.x;
    const int my = (int)((ntiles - blockIdx.x + G - 1) / G);
    auto issue = [&](int i) {  // thread 0: load this CTA's i-th tile into slot i % 3
        const int64_t tile = blockIdx.x + (int64_t)i * G;
        mbar_expect_tx(&full[i % 3], TB);
        tma_load_1d(smem_rt + (i % 3) * TB, x + tile * cnt, TB, &full[i % 3]);
    };
    if (tid == 0) {
        for (int q = 0; q < 3; ++q) mbar_init(&full[q], 1);
        fence_mbar_init();
        for (int i = 0; i < 2 && i < my; ++i) issue(i);
    }
    __syncthreads();
    const int E = ((cnt + 255) / 256) | 1;  // odd piece length: the lanes' strided reads hit distinct banks
    const int i0 = tid * E < cnt ? tid * E : cnt, i1 = i0 + E < cnt ? i0 + E : cnt;
    const int jstart = (int)(i0 % L);
    for (int it = 0; it < my; ++it) {
        const int64_t tile = blockIdx.x + (int64_t)it * G;
        T *buf = reinterpret_cast<T *>(smem_rt + (it % 3) * TB);
        mbar_wait(&full[it % 3], (unsigned)(it / 3) & 1u);
        int j = jstart;
        T acc = O::id();
        int f = 0;
        for (int i = i0; i < i1; ++i) {
            const T v = buf[i];
            if (j == 0) {
                acc = v;
                f = 1;
            } else {
                acc = O::comb(acc, v);
            }
            buf[i] = acc;
            if (++j == L) j = 0;
        }
        T a = acc;
        int fl = f;
#pragma unroll
        for (int dd = 1; dd < 32; dd <<= 1) {
            const T ya = shfl_up(a, dd);
            const int yf = __shfl_up_sync(0xffffffffu, fl, dd);
            if (lane >= dd) {
                if (!fl) a = O::comb(ya, a);
                fl |= yf;
            }
        }
        if (lane == 31) {
            s_wa[warp] = a;
            s_wf[warp] = fl;
        }
        __syncthreads();
        T ex = shfl_up(a, 1);
        int exf = __shfl_up_sync(0xffffffffu, fl, 1);
        if (lane == 0) {
            ex = O::id();
            exf = 0;
        }
        if (!exf) {
            T p = O::id();
            for (int q = 0; q < warp; ++q) p = s_wf[q] ? s_wa[q] : O::comb(p, s_wa[q]);
            ex = O::comb(p, ex);
        }
        {
            int jj = jstart;
            for (int i = i0; i < i1 && jj != 0; ++i) {
                buf[i] = O::comb(ex, buf[i]);
                if (++jj == L) jj = 0;
            }
        }
        fence_proxy_async();  // generic-proxy writes -> visible to the bulk store
        __syncthreads();
        if (tid == 0) {
            tma_store_1d(out + tile * cnt, buf, TB);
            bulk_commit();
            if (it + 2 < my) {
                if (it >= 1) bulk_wait_read<1>();  // the store of slot (it + 2) % 3 (iteration it - 1) has read it
                issue(it + 2);
            }
        }
    }
    if (tid == 0) bulk_wait_read<0>();
}

// KS2 with TMA (16-byte aligned buffers, seglen a multiple of the vector width): a CTA owns
// whole rows (rows b, b + G, ...) and streams each row through a 3-slot TMA ring in tiles of up
// to kRowStreamElems elements (the tile two ahead in flight), scans the tile in shared memory
// (odd-length thread pieces, a CTA scan of the piece totals, the row's running carry) and
// stores it with a TMA bulk store.  No look-back; every element crosses HBM once each way.
constexpr int kRowStreamElems = 8192;
template <int OP, typename T>
__global__ void __launch_bounds__(256)
segscan_rowstream_kernel(const T *__restrict__ x, int64_t nseg, int64_t L, T *__restrict__ out) {
    using O = Op<OP, T>;
    extern __shared__ __align__(128) unsigned char smem_rs[];
    __shared__ uint64_t full[3];
    __shared__ T s_wa[8];
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    constexpr int CH = kRowStreamElems;
    constexpr unsigned SLOT = CH * sizeof(T);
    const int64_t G = gridDim.x;
    const int64_t nch = (L + CH - 1) / CH;  // tiles per row
    const int64_t myrows = (nseg - blockIdx.x + G - 1) / G;
    const int64_t my = myrows * nch;
    auto item = [&](int64_t i, int64_t &row, int64_t &c) {
        row = blockIdx.x + (i / nch) * G;
        c = i % nch;
    };
    auto issue = [&](int64_t i) {  // thread 0: this CTA's i-th tile into slot i % 3
        int64_t row, c;
        item(i, row, c);
        const int64_t cnt = L - c * CH < CH ? L - c * CH : CH;
        mbar_expect_tx(&full[i % 3], (unsigned)(cnt * sizeof(T)));
        tma_load_1d(smem_rs + (i % 3) * SLOT, x + row * L + c * CH, (unsigned)(cnt * sizeof(T)), &full[i % 3]);
    };
    if (tid == 0) {
        for (int q = 0; q < 3; ++q) mbar_init(&full[q], 1);
        fence_mbar_init();
        for (int64_t i = 0; i < 2 && i < my; ++i) issue(i);
    }
    __syncthreads();
    T carry = O::id();
    for (int64_t it = 0; it < my; ++it) {
        int64_t row, c;
        item(it, row, c);
        const int cnt = (int)(L - c * CH < CH ? L - c * CH : CH);
        T *buf = reinterpret_cast<T *>(smem_rs + (it % 3) * SLOT);
        if (c == 0) carry = O::id();
        mbar_wait(&full[it % 3], (unsigned)(it / 3) & 1u);
        const int E = ((cnt + 255) / 256) | 1;  // odd: the lanes' strided reads hit distinct banks
        const int i0 = tid * E < cnt ? tid * E : cnt, i1 = i0 + E < cnt ? i0 + E : cnt;
        T acc = O::id();
        for (int i = i0; i < i1; ++i) {
            acc = O::comb(acc, buf[i]);
            buf[i] = acc;
        }
        T a = acc;  // inclusive warp scan of the piece totals
#pragma unroll
        for (int dd = 1; dd < 32; dd <<= 1) {
            const T y = shfl_up(a, dd);
            if (lane >= dd) a = O::comb(y, a);
        }
        if (lane == 31) s_wa[warp] = a;
        __syncthreads();
        T ex = shfl_up(a, 1);
        if (lane == 0) ex = O::id();
        T wp = carry, tot = carry;
#pragma unroll
        for (int q = 0; q < 8; ++q) {
            if (q < warp) wp = O::comb(wp, s_wa[q]);
            tot = O::comb(tot, s_wa[q]);
        }
        const T base = O::comb(wp, ex);
        for (int i = i0; i < i1; ++i) buf[i] = O::comb(base, buf[i]);
        carry = tot;
        fence_proxy_async();  // generic-proxy writes -> visible to the bulk store
        __syncthreads();      // (also: s_wa is rewritten only after every thread has read it)
        if (tid == 0) {
            tma_store_1d(out + row * L + c * CH, buf, (unsigned)(cnt * sizeof(T)));
            bulk_commit();
            if (it + 2 < my) {
                if (it >= 1) bulk_wait_read<1>();  // the store of slot (it + 2) % 3 has read it
                issue(it + 2);
            }
        }
    }
    if (tid == 0) bulk_wait_read<0>();
}

// rows per tile of the TMA KS3 path (R * L * es a multiple of 16 bytes, <= 72 KB), 0 if none
static int64_t ks3_tma_rows(int64_t L, int64_t es) {
    const int64_t VEC = 16 / es;
    int64_t g = VEC;  // gcd(L, VEC), VEC a power of two
    while (L % g) g >>= 1;
    const int64_t step = VEC / g;  // rows whose elements fill whole 16-byte vectors
    int64_t R = (kRowsElems / L) / step * step;
    if (R < step) R = step;
    if (R * L * es > 72 * 1024) return 0;  // 3 slots <= 216 KB
    return R;
}

// KS1: short rows of any length L <= 32 that are not powers of two (a 16-byte vector then
// straddles rows): a CTA stages 256 whole rows through shared memory with coalesced 16-byte
// loads (index padded every 32 elements), thread t scans row t sequentially in place, and
// the tile leaves with coalesced 16-byte stores.  No look-back, no per-element flags.
template <int OP, typename T>
__global__ void __launch_bounds__(256)
segscan_tile_kernel(const T *__restrict__ x, int64_t nseg, int L, T *__restrict__ out) {
    using O = Op<OP, T>;
    using V = typename O::V;
    constexpr int VEC = 16 / sizeof(T);
    extern __shared__ __align__(16) unsigned char tsm[];
    T *sm = reinterpret_cast<T *>(tsm);
    auto pad = [](int i) { return i + (i >> 5); };
    const int t = threadIdx.x;
    const int64_t ntile = (nseg + 255) / 256;
    for (int64_t tile = blockIdx.x; tile < ntile; tile += gridDim.x) {
        const int64_t s0 = tile * 256;
        const int rows = (int)min((int64_t)256, nseg - s0);
        const int te = rows * L;                  // elements of the tile
        const T *src = x + s0 * L;                // 16-byte aligned: 256 * L * sizeof(T) per tile
        const int nv = te / VEC;
        for (int v = t; v < nv; v += 256) {
            const Vec16<T> e = as_vec<T>(ldg16(src + (int64_t)v * VEC));
#pragma unroll
            for (int k = 0; k < VEC; ++k) sm[pad(v * VEC + k)] = e.e[k];
        }
        for (int i = nv * VEC + t; i < te; i += 256) sm[pad(i)] = src[i];
        __syncthreads();
        if (t < rows) {
            V a = O::id();
            for (int j = 0; j < L; ++j) {
                const int i = pad(t * L + j);
                a = j == 0 ? O::lift(sm[i], 0) : O::fold(a, sm[i], j);
                sm[i] = O::val(a);
            }
        }
        __syncthreads();
        T *dst = out + s0 * L;
        for (int v = t; v < nv; v += 256) {
            Vec16<T> o;
#pragma unroll
            for (int k = 0; k < VEC; ++k) o.e[k] = sm[pad(v * VEC + k)];
            *reinterpret_cast<int4 *>(dst + (int64_t)v * VEC) = *reinterpret_cast<const int4 *>(&o);
        }
        for (int i = nv * VEC + t; i < te; i += 256) dst[i] = sm[pad(i)];
        __syncthreads();
    }
}

// KS2: rows long enough that a CTA should own whole rows (L > 256 vectors) and numerous
// enough to fill the machine: a CTA scans its rows chunk by chunk with a running carry, so
// rows never wait on other CTAs (no look-back).  A chunk is 256 threads x R contiguous
// 16-byte vectors (thread-contiguous, R odd: conflict-free staging is not needed, the
// vectors stay in registers); the next chunk's loads are in flight while this one is
// scanned.  A misaligned row start is handled by a scalar head (thread 0), the ragged end
// by a scalar tail.
template <int OP, typename T, int R>
__global__ void __launch_bounds__(256)
segscan_cta_kernel(const T *__restrict__ x, int64_t nseg, int64_t L, T *__restrict__ out, int64_t *__restrict__ out_idx) {
    using O = Op<OP, T>;
    using V = typename O::V;
    constexpr int VEC = 16 / sizeof(T), E = R * VEC;
    constexpr int64_t CH = 256 * (int64_t)E;  // elements per chunk
    __shared__ V s_w[8];
    __shared__ V s_carry;
    const int t = threadIdx.x, lane = t & 31, warp = t >> 5;
    for (int64_t s = blockIdx.x; s < nseg; s += gridDim.x) {
        const T *p = x + s * L;
        T *q = out + s * L;
        int64_t head = (int64_t)(((16 - ((uintptr_t)p & 15)) & 15) / sizeof(T));
        if (head > L) head = L;
        const int64_t nch = (L - head) / CH;          // whole chunks
        const int64_t body_end = head + nch * CH;
        // head: scalar, thread 0, in order
        if (t == 0) {
            V c = O::id();
            for (int64_t j = 0; j < head; ++j) {
                c = j == 0 ? O::lift(p[0], 0) : O::fold(c, p[j], j);
                q[j] = O::val(c);
                if (out_idx) out_idx[s * L + j] = O::idx(c);
            }
            s_carry = c;
        }
        __syncthreads();
        V carry = s_carry;
        int4 r[R], rn[R];
        auto load = [&](int64_t ch, int4 (&dst)[R]) {
            const int4 *src = reinterpret_cast<const int4 *>(p + head + ch * CH) + (int64_t)t * R;
#pragma unroll
            for (int k = 0; k < R; ++k) dst[k] = ldg16(src + k);
        };
        if (nch > 0) load(0, r);
        for (int64_t ch = 0; ch < nch; ++ch) {
            if (ch + 1 < nch) load(ch + 1, rn);
            const int64_t j0 = head + ch * CH + (int64_t)t * E;  // row-local index of the thread's first element
            V a[E];
#pragma unroll
            for (int k = 0; k < R; ++k) {
                const Vec16<T> e = as_vec<T>(r[k]);
#pragma unroll
                for (int m = 0; m < VEC; ++m) {
                    const int i = k * VEC + m;
                    a[i] = i == 0 ? O::lift(e.e[0], j0) : O::fold(a[i - 1], e.e[m], j0 + i);
                }
            }
            // block exclusive scan of the thread totals
            V incl = a[E - 1];
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const V y = shfl_up(incl, o);
                if (lane >= o) incl = O::comb(y, incl);
            }
            V ex = shfl_up(incl, 1);
            if (lane == 0) ex = O::id();
            if (lane == 31) s_w[warp] = incl;
            __syncthreads();
            V wp = carry, tot = carry;
#pragma unroll
            for (int w = 0; w < 8; ++w) {
                if (w < warp) wp = O::comb(wp, s_w[w]);
                tot = O::comb(tot, s_w[w]);
            }
            __syncthreads();  // s_w is rewritten by the next chunk
            const V pre = O::comb(wp, ex);
            T *qo = q + head + ch * CH + (int64_t)t * E;
#pragma unroll
            for (int k = 0; k < R; ++k) {
                Vec16<T> o;
#pragma unroll
                for (int m = 0; m < VEC; ++m) {
                    const V z = O::comb(pre, a[k * VEC + m]);
                    o.e[m] = O::val(z);
                    if (out_idx) out_idx[s * L + j0 + k * VEC + m] = O::idx(z);
                }
                *reinterpret_cast<int4 *>(qo + k * VEC) = *reinterpret_cast<const int4 *>(&o);
            }
            carry = tot;
#pragma unroll
            for (int k = 0; k < R; ++k) r[k] = rn[k];
        }
        // ragged end: one partial chunk, element-guarded scalar loads, same block scan
        if (body_end < L) {
            const int64_t j0 = body_end + (int64_t)t * E;
            V a[E];
#pragma unroll
            for (int i = 0; i < E; ++i) {
                const bool ok = j0 + i < L;
                const V e = ok ? O::lift(p[j0 + i], j0 + i) : O::id();
                a[i] = i == 0 ? e : O::comb(a[i - 1], e);
            }
            V incl = a[E - 1];
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const V y = shfl_up(incl, o);
                if (lane >= o) incl = O::comb(y, incl);
            }
            V ex = shfl_up(incl, 1);
            if (lane == 0) ex = O::id();
            if (lane == 31) s_w[warp] = incl;
            __syncthreads();
            V wp = carry;
#pragma unroll
            for (int w = 0; w < 8; ++w)
                if (w < warp) wp = O::comb(wp, s_w[w]);
            const V pre = O::comb(wp, ex);
#pragma unroll
            for (int i = 0; i < E; ++i)
                if (j0 + i < L) {
                    const V z = O::comb(pre, a[i]);
                    q[j0 + i] = O::val(z);
                    if (out_idx) out_idx[s * L + j0 + i] = O::idx(z);
                }
        }
        __syncthreads();  // s_carry reuse
    }
}

// KS2 applies when every SM gets at least one row: the rows are then the unit of parallelism
// (seg sweep, profiles/r01_seg_sweep.json: at >= 1 row per SM KS2 beats the segmented look-back scan,
// 256-268 rows 3.8 -> 4.8 TB/s, 512 rows 3.8 -> 4.5; below one row per SM SMs idle: 128 rows 3.6, 32 rows 1.1)
#ifndef FS_KS2_MINF
// rows >= 1.7 x SMs (profiles/r02_scan_regimes.jsonl): KS2 0.94-0.98 of HBM from 256 rows up; at
// 128 rows of 2^21 KS2 0.78 vs the ring look-back scan 0.87
#define FS_KS2_MINF 170
#endif
static bool nseg_ok(int64_t n, int64_t L) { return L > 0 && n / L >= (int64_t)sm_count() * FS_KS2_MINF / 100; }
#ifndef FS_FLAT_ROW_MIN
#define FS_FLAT_ROW_MIN INT64_MAX
#endif
// rows at least this long: flat scan per row.  Off by default since the ring look-back scan
// (0.87 at 2 and 4 rows, one launch) beats one ring launch per row (0.86 / 0.78); forceable (12).
constexpr int64_t kFlatRowMin = FS_FLAT_ROW_MIN;
template <int OP, typename T> constexpr int ks2_rows() { return (sizeof(T) == 4 && OP != kArgmin) ? 3 : 1; }
template <typename T> constexpr int dt_of() {
    return sizeof(T) == 8 ? FS_I64 : (std::is_same<T, float>::value ? FS_F32 : FS_I32);
}

// The row-major seg_scan plan (internal.cuh).  Natural order: KS0 (power-of-two rows that fit one
// CTA step), KS0-BIG (power-of-two rows of 2-8 steps), KS2 (rows of >= 4 chunks, >= 1 row per SM),
// KS3 (32 < L <= 16384 staged in shared memory), KS1 (L <= 32 staged), the flat slab scan per
// row (rows >= kFlatRowMin, fewer than the SMs), else the segmented look-back scan.  A regime
// forced with fs_force_seg_regime is taken when its preconditions hold (the flat per-row scan
// then drops its length threshold).
int seg_scan_plan(int op, int dt, int64_t n, int64_t L, bool al16, bool co16, bool elem, bool plain) {
    if (L >= n) return RG_FLAT_ROW;  // one row: the unsegmented scan
    const int64_t es = (int64_t)dtype_size(dt), VEC = 16 / es;
    const bool pow2 = (L & (L - 1)) == 0;
    const int64_t ks2ch = 256 * VEC * ((es == 4 && op != FS_ARGMIN) ? 3 : 1);
    // (preconditions; a forced regime needs only these.  Preference:) the ring scan (regime 5
    // on 16-byte aligned buffers, add/min/max) beats KS3 above 4096
    // elements per row and KS2 wherever KS2 cannot stream rows by TMA (L not a multiple of the
    // vector): profiles/r02_scan_regimes_odd.jsonl (L = 8191: 0.57 -> 0.89, 65537: 0.75 -> 0.99)
    const bool ring = op != FS_ARGMIN && al16;
    const bool ok[13] = {
        false, false, false, false, false,
        true,                                                                         // 5 look-back
        false,
        al16 && plain && pow2 && L <= 256 * VEC,                                      // 7 KS0
        op != FS_ARGMIN && al16 && plain && L >= 2 && L <= 32,                        // 8 KS1
        plain && co16 && elem && L >= 4 * ks2ch && nseg_ok(n, L),                     // 9 KS2
        al16 && plain && pow2 && L > 256 * VEC && L <= 2048 * VEC,                    // 10 KS0-BIG
        op != FS_ARGMIN && plain && elem && L <= (es == 4 ? 16384 : 8192) &&          // 11 KS3
            (L > 32 || (L >= 2 && al16 && ks3_tma_rows(L, es) > 0)),
        al16 && plain && (L * es) % 16 == 0,                                          // 12 flat per row
    };
    const int f = forced_seg_regime();
    if (f >= 5 && f <= 12 && ok[f]) return f;
    if (ok[RG_KS0]) return RG_KS0;
    if (ok[RG_KS0_BIG]) return RG_KS0_BIG;
    if (ok[RG_KS2] && (!ring || L % VEC == 0)) return RG_KS2;
    if (ok[RG_KS3] && (!ring || L <= 4096)) return RG_KS3;
    if (ok[RG_KS1]) return RG_KS1;
    if (ok[RG_FLAT_ROW] && L >= kFlatRowMin) return RG_FLAT_ROW;
    return RG_KS_LOOKBACK;
}

// ---------------------------------------------------------------- ring scan (scanomap, long-row seg_scan)
// The single pass of F5 (L1071-1074) with every tile kept ON CHIP between its read
// and its write.  One CTA per SM streams tiles of 256 x kRingVPT 16-byte vectors
// (36 KB) through a ring of kRingStages shared-memory slots; warps are specialised:
//   producer warp  : tile ids from the atomic counter (increasing), taken kRingPf = 1 tile
//                    ahead and prefetched into L2 (cp.async.bulk.prefetch.L2) so that the
//                    1-D TMA load into a freed slot hits L2: the slot no longer waits on HBM
//                    latency (scanomap 0.89 -> 0.99 of the HBM peak; 2 or 4 ahead hold ids
//                    longer before their aggregates can be published: 0.97 / 0.91)
//   aggregate group: (4 warps, tiles in order) the tile aggregate as soon as the tile
//                    lands, published at once (status 1), so successors' look-backs
//                    never wait on a tile that is merely queued in a ring
//   consumer groups: (kRingNG x 8 warps, alternate tiles) scan the tile in registers
//                    (thread-contiguous odd vector runs: conflict-free 16-byte shared
//                    loads), warp 0 runs the decoupled look-back (32 x kRingEPL
//                    predecessors per step) and publishes the inclusive prefix, then
//                    prefix (+) local scan goes back into the slot and out with one TMA
//                    bulk store.
// Every element crosses HBM exactly once each way; nothing is re-read from L2.
// Other measured alternatives (tools/ring_trace.py, tools/scan_ab.py): separate look-back
// warps started at the aggregate (0.75 of HBM: they start before their predecessors
// are published and spin longer), wider look-back steps (worse), a third consumer
// group or a store warp (no gain); the ring's bytes / slot hold time is the limit.
// SEG: footnote 5's operator with the implicit flags i mod L == 0 (the look-back
// stops at the first flagged predecessor).  ADD / MIN / MAX (ARGMIN keeps
// scan_ws_kernel for its index output).
#ifndef FS_RING_VPT
#define FS_RING_VPT 9
#endif
#ifndef FS_RING_STAGES
#define FS_RING_STAGES 6
#endif
#ifndef FS_RING_NG
#define FS_RING_NG 2
#endif
#ifndef FS_RING_EPL
#define FS_RING_EPL 1
#endif
constexpr int kRingEPL = FS_RING_EPL;  // look-back predecessors per lane per step
#ifndef FS_RING_PF
#define FS_RING_PF 1
#endif
constexpr int kRingPf = FS_RING_PF;  // tile ids taken (and L2-prefetched) ahead of the ring
#ifndef FS_RING_SLEEP
#define FS_RING_SLEEP 0
#endif
constexpr int kRingSleep = FS_RING_SLEEP;  // ns between polls of an unpublished predecessor
constexpr int kRingVPT = FS_RING_VPT, kRingStages = FS_RING_STAGES, kRingG = 256, kRingA = 128, kRingNG = FS_RING_NG;
constexpr int kRingThreads = kRingNG * kRingG + kRingA + 32;
static_assert(kRingVPT % 2 == 1, "odd vectors per thread: conflict-free 16-byte shared loads");
template <int OP, typename T> struct RingShape {
    static constexpr bool PACK = sizeof(T) == 4 && OP != kArgmin;  // else 16-byte words (TileStateW / A)
    static constexpr int VEC = 16 / sizeof(T), E = kRingVPT * VEC;
    static constexpr int64_t TILE = (int64_t)kRingG * E;
    static constexpr unsigned TILE_BYTES = kRingG * kRingVPT * 16;
    static constexpr unsigned SMEM = kRingStages * TILE_BYTES;
};
template <int OP, typename T, bool SEG>
using RingState = typename std::conditional<
    OP == kArgmin, TileStateA<typename SOp<Op<OP, T>, SEG>::S>,
    typename std::conditional<RingShape<OP, T>::PACK, TileState<typename SOp<Op<OP, T>, SEG>::S, true>,
                              TileStateW<typename SOp<Op<OP, T>, SEG>::S>>::type>::type;

#ifdef FS_RING_TRACE
// per-tile event times (%globaltimer, ns): issued, landed, aggregate published, prefix
// published, written back, stored
constexpr int kRingTraceTiles = 65536;
__device__ unsigned long long g_ring_trace[kRingTraceTiles * 6];
__device__ __forceinline__ void ring_mark(int64_t t, int e) {
    unsigned long long v;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(v));
    if (t < kRingTraceTiles) g_ring_trace[t * 6 + e] = v;
}
extern "C" int fs_debug_ring_trace(void *host, size_t bytes) {
    return (int)cudaMemcpyFromSymbol(host, g_ring_trace, bytes < sizeof(g_ring_trace) ? bytes : sizeof(g_ring_trace));
}
#define RING_MARK(t, e) ring_mark(t, e)
#else
#define RING_MARK(t, e)
#endif

template <int OP, typename T, bool SEG>
__global__ void __launch_bounds__(kRingThreads, 1)
scan_ring_kernel(const T *__restrict__ in, int64_t n, int64_t L, int64_t ibase, T *__restrict__ out,
                 int64_t *__restrict__ out_idx, const T *carry, const int64_t *carry_idx, unsigned *counter,
                 RingState<OP, T, SEG> ts, int64_t ntiles) {
    // ARGMIN: an element's index is its offset in its row (SEG) or ibase + its position (flat);
    // out_idx receives the index of every prefix's minimum (16-byte aligned)
    using O = Op<OP, T>;
    using SO = SOp<O, SEG>;
    using S = typename SO::S;
    using Sh = RingShape<OP, T>;
    constexpr int VEC = Sh::VEC, E = Sh::E, NST = kRingStages, NWG = kRingG / 32, NG = kRingNG;
    constexpr int64_t TILE = Sh::TILE;
    constexpr int T_AGG = NG * kRingG, T_PROD = T_AGG + kRingA;
    constexpr int NMARK = NG;
    static_assert(NMARK <= NST, "the end markers fit in the ring");
    extern __shared__ __align__(128) unsigned char sbuf[];
    // full: tile landed (TMA tx); aggd: aggregate published; empty: the aggregate group is
    // done with the slot and the consumer's TMA store has read it
    __shared__ uint64_t full[NST], aggd[NST], empty[NST];
    __shared__ int64_t s_tid[NST];
    __shared__ S s_wtot[NG][NWG], s_wpre[NG][NWG];
    __shared__ typename O::V s_ared[2][kRingA / 32];
    const int tid = threadIdx.x, lane = tid & 31;
    if (tid == 0) {
        for (int s = 0; s < NST; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&aggd[s], 1);
            mbar_init(&empty[s], 2);
        }
        fence_mbar_init();
    }
    __syncthreads();
    auto tile_len = [&](int64_t t, int64_t &nv, int64_t &nbulk) {
        nv = (n - t * TILE) < TILE ? (n - t * TILE) : TILE;
        nbulk = ((nv * (int64_t)sizeof(T)) & ~(int64_t)15) / (int64_t)sizeof(T);
    };
    if (tid >= T_PROD) {  // ---- producer warp: tile ids in increasing order, TMA into the ring
        if (lane == 0) {
            int marks = 0;
            // kRingPf tile ids taken ahead and prefetched into L2 (the ring slot then waits on an
            // L2 hit instead of HBM latency)
            int64_t q[kRingPf > 0 ? kRingPf : 1];
            int qh = 0, qn = 0;
            bool dry = false;
            auto take = [&]() {
                if (dry) return;
                const int64_t u = (int64_t)atomicAdd(counter, 1u);
                if (u >= ntiles) {
                    dry = true;
                    return;
                }
                q[(qh + qn) % kRingPf] = u;
                ++qn;
                int64_t nv, nbulk;
                tile_len(u, nv, nbulk);
                if (nbulk) prefetch_l2_bulk(in + u * TILE, (unsigned)(nbulk * (int64_t)sizeof(T)));
            };
            if (kRingPf > 0)
                for (int i = 0; i < kRingPf; ++i) take();
            for (int64_t k = 0; marks < NMARK; ++k) {
                const int s = (int)(k % NST);
                if (k >= NST) mbar_wait(&empty[s], (unsigned)((k / NST) - 1) & 1u);
                int64_t t;
                if (kRingPf > 0) {
                    if (qn > 0) {
                        t = q[qh];
                        qh = (qh + 1) % kRingPf;
                        --qn;
                        take();
                    } else {
                        t = ntiles;
                    }
                } else {
                    t = marks ? ntiles : (int64_t)atomicAdd(counter, 1u);
                }
                if (t >= ntiles) {  // NMARK end markers in consecutive slots: every round-robin
                    s_tid[s] = -1;  // member of every role meets one
                    ++marks;
                    mbar_arrive(&full[s]);
                    continue;
                }
                s_tid[s] = t;
                RING_MARK(t, 0);
                int64_t nv, nbulk;
                tile_len(t, nv, nbulk);
                if (nbulk) {
                    mbar_expect_tx(&full[s], (unsigned)(nbulk * (int64_t)sizeof(T)));
                    tma_load_1d(sbuf + (size_t)s * Sh::TILE_BYTES, in + t * TILE,
                                (unsigned)(nbulk * (int64_t)sizeof(T)), &full[s]);
                } else {
                    mbar_arrive(&full[s]);
                }
            }
        }
        return;
    }
    if (tid >= T_AGG) {  // ---- aggregate group: every tile's aggregate as soon as it lands, in order
        const int at = tid - T_AGG, aw = at >> 5;
        for (int64_t k = 0, marks = 0; marks < NMARK; ++k) {
            const int s = (int)(k % NST);
            mbar_wait(&full[s], (unsigned)(k / NST) & 1u);
            const int64_t t = s_tid[s];
            if (t < 0) {
                ++marks;
                continue;
            }
            if (at == 0) RING_MARK(t, 1);
            const int64_t t0 = t * TILE;
            int64_t nv, nbulk;
            tile_len(t, nv, nbulk);
            const unsigned char *slot = sbuf + (size_t)s * Sh::TILE_BYTES;
            // SEG: the elements after the tile's last segment start (closed form), flag = a start exists
            int64_t lo = 0;
            int f = 0;
            if constexpr (SEG) {
                const int64_t r = t0 % L, i0 = r == 0 ? 0 : L - r;
                if (i0 < nv) {
                    lo = i0 + ((nv - 1 - i0) / L) * L;
                    f = 1;
                }
            }
            // ARGMIN: index of tile element p = ib + p (no start at or before p in the tile: ib =
            // the tile start's offset in its row, or ibase + t0 when flat) or p - lo (after the last start)
            int64_t ib = 0;
            if constexpr (OP == kArgmin) ib = SEG ? (f ? -lo : t0 % L) : ibase + t0;
            typename O::V acc = O::id();
            if (nv == TILE && lo == 0) {
#pragma unroll
                for (int j = 0; j < 2 * kRingVPT; ++j) {
                    const int e = (j * kRingA + at) * VEC;
                    const Vec16<T> a = as_vec<T>(*reinterpret_cast<const int4 *>(slot + ((j * kRingA + at) << 4)));
#pragma unroll
                    for (int q = 0; q < VEC; ++q) acc = O::comb(acc, O::lift(a.e[q], ib + e + q));
                }
            } else if (nv == TILE) {  // SEG, a start in the tile: the same vector loads, masked
#pragma unroll
                for (int j = 0; j < 2 * kRingVPT; ++j) {
                    const int e = (j * kRingA + at) * VEC;
                    const Vec16<T> a = as_vec<T>(*reinterpret_cast<const int4 *>(slot + ((j * kRingA + at) << 4)));
#pragma unroll
                    for (int q = 0; q < VEC; ++q)
                        if (e + q >= lo) acc = O::comb(acc, O::lift(a.e[q], ib + e + q));
                }
            } else {
                for (int j = 0; j < 2 * kRingVPT; ++j) {
                    const int64_t e = (int64_t)(j * kRingA + at) * VEC;
#pragma unroll
                    for (int q = 0; q < VEC; ++q) {
                        const int64_t p = e + q;
                        if (p >= lo && p < nv)
                            acc = O::comb(acc, O::lift(p < nbulk ? reinterpret_cast<const T *>(slot)[p] : in[t0 + p],
                                                       ib + p));
                    }
                }
            }
#pragma unroll
            for (int m = 16; m > 0; m >>= 1) acc = O::comb(acc, shfl_xor(acc, m));
            if ((at & 31) == 0) s_ared[k & 1][aw] = acc;
            named_bar(1 + NG, kRingA);
            if (at == 0) {
                S agg{s_ared[k & 1][0], f};
#pragma unroll
                for (int w = 1; w < kRingA / 32; ++w) agg.v = O::comb(agg.v, s_ared[k & 1][w]);
                if (t > 0) ts.publish(t, agg, kStAgg);
                RING_MARK(t, 2);
                mbar_arrive(&aggd[s]);
                mbar_arrive(&empty[s]);
            }
        }
        return;
    }
    // ---- consumer group g: tiles k = g, g + NG, ...
    const int g = tid / kRingG, gt = tid % kRingG, warp = gt >> 5;
    for (int64_t k = g;; k += NG) {
        const int s = (int)(k % NST);
        mbar_wait(&full[s], (unsigned)(k / NST) & 1u);
        const int64_t t = s_tid[s];
        if (t < 0) break;
        const int64_t t0 = t * TILE;
        int64_t nv, nbulk;
        tile_len(t, nv, nbulk);
        unsigned char *slot = sbuf + (size_t)s * Sh::TILE_BYTES;
        const int e0 = gt * E;  // this thread's first element in the tile
        // local inclusive scan of the thread's E contiguous elements, in registers
        T x[E];
        if (nv == TILE) {
#pragma unroll
            for (int j = 0; j < kRingVPT; ++j) {
                const Vec16<T> a = as_vec<T>(*reinterpret_cast<const int4 *>(slot + ((gt * kRingVPT + j) << 4)));
#pragma unroll
                for (int q = 0; q < VEC; ++q) x[j * VEC + q] = a.e[q];
            }
        } else {
#pragma unroll
            for (int i = 0; i < E; ++i) {
                const int64_t p = e0 + i;
                x[i] = p < nbulk ? reinterpret_cast<const T *>(slot)[p] : (p < nv ? in[t0 + p] : O::val(O::id()));
            }
        }
        int64_t r0 = 0;
        if constexpr (SEG) r0 = (t0 + e0) % L;
        // no segment start among this thread's elements: the plain scan (flag 0)
        const bool noflag = !SEG || (r0 != 0 && L - r0 >= E);
        // ARGMIN index of the thread's element i: xb + i (noflag or flat), else its row offset r
        const int64_t xb = SEG ? r0 : ibase + t0 + e0;
        S run = SO::id();
        if (noflag) {
#pragma unroll
            for (int i = 0; i < E; ++i) run.v = O::fold(run.v, x[i], xb + i);
        } else {
            int64_t r = r0;
#pragma unroll
            for (int i = 0; i < E; ++i) {
                S e;
                e.v = O::lift(x[i], r);
                e.f = SEG ? (r == 0) : 0;
                if (SEG) {
                    ++r;
                    if (r == L) r = 0;
                }
                run = SO::comb(run, e);
            }
        }
        // ordered inclusive warp scan of the thread totals
        S a = run;
#pragma unroll
        for (int off = 1; off < 32; off <<= 1) {
            const S o = SO::up(a, off);
            if (lane >= off) a = SO::comb(o, a);
        }
        S tex = SO::up(a, 1);
        if (lane == 0) tex = SO::id();
        if (lane == 31) s_wtot[g][warp] = a;
        named_bar(1 + g, kRingG);
        if (warp == 0) {
            S w = lane < NWG ? s_wtot[g][lane] : SO::id();
#pragma unroll
            for (int off = 1; off < NWG; off <<= 1) {
                const S o = SO::up(w, off);
                if (lane >= off) w = SO::comb(o, w);
            }
            S wex = SO::up(w, 1);
            if (lane == 0) wex = SO::id();
            const S agg = SO::bcast(w, NWG - 1);
            // decoupled look-back over the published predecessors
            S exc = SO::id();
            if (t == 0) {
                if (carry) exc = S{O::lift(*carry, carry_idx ? *carry_idx : -1), 0};
            } else {
                    // wide look-back: lane i polls predecessors j - EPL*i - 0 .. EPL-1 (all loads of a
                    // step in flight together: 32*EPL predecessors per L2 round trip)
                    constexpr int EPL = kRingEPL;
                    int64_t j = t - 1;
                    while (true) {
                        S v[EPL];
                        unsigned st[EPL];
    #pragma unroll
                        for (int e = 0; e < EPL; ++e) {
                            const int64_t idx = j - (int64_t)EPL * lane - e;
                            v[e] = SO::id();
                            st[e] = idx >= 0 ? ts.poll(idx, v[e]) : kStIncl;
                        }
    #pragma unroll
                        for (int e = 0; e < EPL; ++e) {
                            const int64_t idx = j - (int64_t)EPL * lane - e;
                            while (st[e] == 0) {
                                if (kRingSleep) __nanosleep(kRingSleep);
                                st[e] = ts.poll(idx, v[e]);
                            }
                        }
                        // this lane's nearest inclusive prefix (idx < 0 counts as one: nothing left)
                        int ne = EPL;
    #pragma unroll
                        for (int e = EPL - 1; e >= 0; --e)
                            if (st[e] == kStIncl) ne = e;
                        const unsigned m = __ballot_sync(0xffffffffu, ne < EPL);
                        const int kk = m ? __ffs(m) - 1 : 32;
                        // the lane's ordered fold of its entries up to (and including) its nearest
                        // inclusive prefix; entries further left are farther back
                        S a = SO::id();
    #pragma unroll
                        for (int e = EPL - 1; e >= 0; --e) {
                            const int64_t idx = j - (int64_t)EPL * lane - e;
                            if (e <= ne && idx >= 0) a = SO::comb(a, v[e]);
                        }
                        if (lane > kk) a = SO::id();
                        // ordered reduction: higher lanes are further left
    #pragma unroll
                        for (int off = 1; off < 32; off <<= 1) {
                            const S o = SO::down(a, off);
                            if (lane + off < 32) a = SO::comb(o, a);
                        }
                        exc = SO::comb(SO::bcast(a, 0), exc);
                        if (m || j < 32 * EPL || (SEG && exc.f)) break;
                        j -= 32 * EPL;
                    }
            }
            // (after the aggregate group's publish: never downgrade an inclusive prefix)
            mbar_wait(&aggd[s], (unsigned)(k / NST) & 1u);
            if (lane == 0) {
                ts.publish(t, SO::comb(exc, agg), kStIncl);
                RING_MARK(t, 3);
            }
            if (lane < NWG) s_wpre[g][lane] = SO::comb(exc, wex);
        }
        named_bar(1 + g, kRingG);
        const S p = SO::comb(s_wpre[g][warp], tex);
        // ARGMIN: the prefix minima's indices leave as they are produced, two per 16-byte store
        int64_t *oi = OP == kArgmin ? out_idx + t0 + e0 : nullptr;
        int64_t pend = 0;
        auto emit = [&](int i, int64_t idx) {
            if constexpr (OP == kArgmin) {
                if (nv == TILE) {
                    if (i & 1) {
                        longlong2 v2;
                        v2.x = pend;
                        v2.y = idx;
                        *reinterpret_cast<longlong2 *>(oi + i - 1) = v2;
                    } else {
                        pend = idx;
                    }
                } else if (e0 + i < nv) {
                    oi[i] = idx;
                }
            }
        };
        if (noflag) {
            typename O::V c = p.v;
#pragma unroll
            for (int i = 0; i < E; ++i) {
                c = O::comb(c, O::lift(x[i], xb + i));
                x[i] = O::val(c);
                emit(i, O::idx(c));
            }
        } else {
            S c = p;
            int64_t r = r0;
#pragma unroll
            for (int i = 0; i < E; ++i) {
                S e;
                e.v = O::lift(x[i], r);
                e.f = SEG ? (r == 0) : 0;
                if (SEG) {
                    ++r;
                    if (r == L) r = 0;
                }
                c = SO::comb(c, e);
                x[i] = O::val(c.v);
                emit(i, O::idx(c.v));
            }
        }
        if (nv == TILE) {
#pragma unroll
            for (int j = 0; j < kRingVPT; ++j) {
                Vec16<T> v;
#pragma unroll
                for (int q = 0; q < VEC; ++q) v.e[q] = x[j * VEC + q];
                int4 w;
                memcpy(&w, &v, 16);
                *reinterpret_cast<int4 *>(slot + ((gt * kRingVPT + j) << 4)) = w;
            }
        } else {
#pragma unroll
            for (int i = 0; i < E; ++i) {
                const int64_t q = e0 + i;
                if (q < nbulk) reinterpret_cast<T *>(slot)[q] = x[i];
                else if (q < nv) out[t0 + q] = x[i];
            }
        }
        fence_proxy_async();
        named_bar(1 + g, kRingG);
        if (gt == 0) {
            RING_MARK(t, 4);
            if (nbulk) {
                tma_store_1d(out + t0, slot, (unsigned)(nbulk * (int64_t)sizeof(T)));
                bulk_commit();
                bulk_wait_read<0>();
            }
            RING_MARK(t, 5);
            mbar_arrive(&empty[s]);
        }
    }
    if (gt == 0) bulk_wait<0>();
}

// FUTSEG_SCAN_KERNEL=ws selects the slab scan instead of the ring scan (A/B measurement only)
static bool scan_ring_disabled() {
    static const int v = [] {
        const char *e = getenv("FUTSEG_SCAN_KERNEL");
        return (e && e[0] == 'w' && e[1] == 's') ? 1 : 0;
    }();
    return v != 0;
}
template <int OP, typename T> struct ScanRun {
    template <bool NN, bool SEG, bool TMA>
    static fs_status go(const void *in0, const void *in1, int64_t n, int64_t L, const fs_mapdesc &map, void *out,
                        int64_t *out_idx, const void *carry, const int64_t *carry_idx, void *ws, bool aligned,
                        cudaStream_t st) {
        using Sh = ScanShape<OP, T>;
        using S = typename SOp<Op<OP, T>, SEG>::S;
        const int64_t ntiles = ceil_div(n, Sh::TILE);
        char *b = (char *)ws + kWsHeader;
        unsigned *counter = (unsigned *)b;
        TileState<S, Sh::PACK> ts;
        ts.w = (uint64_t *)(b + 256);
        if constexpr (!Sh::PACK) {
            ts.aggs = (S *)(b + 256 + scan_state_bytes(ntiles));
            ts.incls = ts.aggs + ntiles;
        }
        if constexpr (TMA && !NN && (OP != kArgmin || sizeof(T) == 4)) {  // the ring scan (16-byte aligned)
            if (!scan_ring_disabled() && (OP != kArgmin || ((uintptr_t)out_idx & 15) == 0)) {
                using ShR = RingShape<OP, T>;
                const int64_t ntr = ceil_div(n, ShR::TILE);
                // state words: 8 B per tile (PACK) or 16 B (TileStateW), zeroed per call
                const size_t stb = ShR::PACK ? scan_state_bytes(ntr) : 2 * scan_state_bytes(ntr);
                if (cudaMemsetAsync(counter, 0, 256 + stb, st) != cudaSuccess) return FS_ERR_CUDA;
                RingState<OP, T, SEG> tr;
                tr.w = ts.w;
                auto kr = scan_ring_kernel<OP, T, SEG>;
                static bool attr = false;
                if (!attr) {
                    cudaFuncSetAttribute((const void *)kr, cudaFuncAttributeMaxDynamicSharedMemorySize, ShR::SMEM);
                    attr = true;
                }
                const int64_t G0 = sm_count();
                const int64_t G = ntr < G0 ? ntr : G0;
                kr<<<(unsigned)(G > 0 ? G : 1), kRingThreads, ShR::SMEM, st>>>((const T *)in0, n, L, map.ibase,
                                                                               (T *)out, out_idx, (const T *)carry,
                                                                               carry_idx, counter, tr, ntr);
                return launch_status();
            }
        }
        if (cudaMemsetAsync(counter, 0, 256 + scan_state_bytes(ntiles), st) != cudaSuccess) return FS_ERR_CUDA;
        if constexpr (TMA && !NN) {  // the warp-specialised slab scan (16-byte aligned buffers)
            {
                using ShW = ScanWShape<OP, T>;
                const int64_t ntw = ceil_div(n, ShW::TILE);
                const int64_t G0 = sm_count();
                int64_t tps = ntw / (G0 * 4);
                tps = tps < 1 ? 1 : (tps > FS_SCANW_TPS ? FS_SCANW_TPS : tps);
                const int64_t nslabs = ceil_div(ntw, tps);
                const int64_t G = nslabs < G0 ? nslabs : G0;
                auto kw = scan_ws_kernel<OP, T, SEG>;
                cudaFuncSetAttribute((const void *)kw, cudaFuncAttributeMaxDynamicSharedMemorySize, ShW::SMEM);
                WsState<OP, T, SEG> tw;
                tw.w = ts.w;
                if constexpr (!ShW::PACK && !(OP == kArgmin && sizeof(T) == 4)) {
                    tw.aggs = ts.aggs;
                    tw.incls = ts.incls;
                }
                if constexpr (OP == kArgmin && sizeof(T) == 4) {  // 16 B per slab tile, zeroed
                    if (cudaMemsetAsync(ts.w, 0, 2 * scan_state_bytes(ntw), st) != cudaSuccess) return FS_ERR_CUDA;
                }
                kw<<<(unsigned)G, kScanWThreads, ShW::SMEM, st>>>((const T *)in0, n, L, map.ibase, (T *)out, out_idx,
                                                                  (const T *)carry, carry_idx, tw, ntw, (int)tps);
                return launch_status();
            }
        }
        auto k = scan_kernel<OP, T, NN, SEG, TMA>;
        const int smem = TMA ? 2 * (int)Sh::TILE_BYTES : 0;
        if (TMA) {
            static bool attr = false;
            if (!attr) {
                cudaFuncSetAttribute((const void *)k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
                attr = true;
            }
        }
        const int64_t cap = resident_blocks((const void *)k, kScanThreads, smem);
        const int64_t grid = ntiles < cap ? ntiles : cap;
        k<<<(unsigned)grid, kScanThreads, smem, st>>>((const T *)in0, (const float *)in1, n, L, map.q0, map.q1,
                                                      map.ibase, (T *)out, out_idx, (const T *)carry, carry_idx,
                                                      counter, ts, ntiles, aligned);
        return launch_status();
    }
    static fs_status run(const fs_mapdesc *map, const void *in0, const void *in1, int64_t n, int64_t L, void *out,
                         int64_t *out_idx, const void *carry, const int64_t *carry_idx, void *ws, cudaStream_t st) {
        const bool seg = L < n;
        bool al = ((uintptr_t)in0 & 15) == 0 && ((uintptr_t)out & 15) == 0;
        if (map->kind == FS_MAP_NN_DIST) {
            al = al && ((uintptr_t)in1 & 15) == 0;
            if constexpr (sizeof(T) == 4)
                return go<true, false, false>(in0, in1, n, L, *map, out, out_idx, carry, carry_idx, ws, al, st);
            return FS_ERR_UNSUPPORTED;
        }
        if (seg) {
            constexpr int64_t VEC = 16 / sizeof(T);
            const bool co16 = ((((uintptr_t)in0) ^ ((uintptr_t)out)) & 15) == 0;
            const bool elem = ((uintptr_t)in0 % sizeof(T)) == 0 && ((uintptr_t)out % sizeof(T)) == 0;
            const bool plain = !carry && map->ibase == 0;
            const int rg = seg_scan_plan(OP, dt_of<T>(), n, L, al, co16, elem, plain);
            note_regime(rg);
            if (rg == RG_KS0 && L <= 32 * VEC) {
                auto kv = segscan_vec_kernel<OP, T, 4>;
                const int64_t nvec = n / VEC;
                int64_t grid = ceil_div(nvec > 0 ? nvec : 1, 256 * 4);
                const int64_t cap = resident_blocks((const void *)kv, 256);
                grid = grid > cap ? cap : (grid < 1 ? 1 : grid);
                const int G = L > VEC ? (int)(L / VEC) : 1;
                kv<<<(unsigned)grid, 256, 0, st>>>((const T *)in0, n, (int)L, G, (T *)out, out_idx);
                return launch_status();
            }
            if (rg == RG_KS0) {
                auto kb = segscan_blk_kernel<OP, T, 2>;
                const int64_t nchunk = ceil_div(n / VEC, 256);
                int64_t grid = ceil_div(nchunk > 0 ? nchunk : 1, 2);
                const int64_t cap = resident_blocks((const void *)kb, 256);
                grid = grid > cap ? cap : (grid < 1 ? 1 : grid);
                kb<<<(unsigned)grid, 256, 0, st>>>((const T *)in0, n, (int)L, (T *)out, out_idx);
                return launch_status();
            }
            if (rg == RG_KS0_BIG) {
                const bool u8 = L > 1024 * VEC;
                auto kb = u8 ? segscan_blk_kernel<OP, T, 8, true> : segscan_blk_kernel<OP, T, 4, true>;
                const int64_t nchunk = ceil_div(n / VEC, 256);
                int64_t grid = ceil_div(nchunk > 0 ? nchunk : 1, u8 ? 8 : 4);
                const int64_t cap = resident_blocks((const void *)kb, 256);
                grid = grid > cap ? cap : (grid < 1 ? 1 : grid);
                kb<<<(unsigned)grid, 256, 0, st>>>((const T *)in0, n, (int)L, (T *)out, out_idx);
                return launch_status();
            }
            if constexpr (OP != kArgmin) {
                if (rg == RG_KS2 && al && L % VEC == 0) {  // whole rows streamed through a TMA ring
                    auto kr = segscan_rowstream_kernel<OP, T>;
                    const int smem = 3 * kRowStreamElems * (int)sizeof(T);
                    cudaFuncSetAttribute((const void *)kr, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
                    const int64_t nseg = n / L;
                    const int64_t cap = resident_blocks((const void *)kr, 256, (size_t)smem);
                    const int64_t k = ceil_div(nseg, cap);  // rows per CTA, equal for all CTAs
                    const int64_t grid = ceil_div(nseg, k);
                    kr<<<(unsigned)grid, 256, smem, st>>>((const T *)in0, nseg, L, (T *)out);
                    return launch_status();
                }
            }
            if (rg == RG_KS2) {
                constexpr int KS2R = ks2_rows<OP, T>();
                auto kc = segscan_cta_kernel<OP, T, KS2R>;
                const int64_t nseg = n / L;
                int64_t grid = resident_blocks((const void *)kc, 256);
                grid = grid > nseg ? nseg : grid;
                kc<<<(unsigned)grid, 256, 0, st>>>((const T *)in0, nseg, L, (T *)out, out_idx);
                return launch_status();
            }
            if constexpr (OP != kArgmin) {  // (argmin's index output keeps the look-back path)
                if (rg == RG_KS3 && al && ks3_tma_rows(L, sizeof(T)) > 0 && n / L >= ks3_tma_rows(L, sizeof(T))) {
                    const int64_t R = ks3_tma_rows(L, sizeof(T)), nseg = n / L, ntiles = nseg / R;
                    auto kt = segscan_rows_tma_kernel<OP, T>;
                    const int smem = (int)(3 * R * L * (int64_t)sizeof(T));
                    cudaFuncSetAttribute((const void *)kt, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
                    int64_t grid = resident_blocks((const void *)kt, 256, (size_t)smem);
                    grid = grid > ntiles ? ntiles : grid;
                    kt<<<(unsigned)grid, 256, smem, st>>>((const T *)in0, ntiles, L, (int)R, (T *)out);
                    const int64_t done = ntiles * R;
                    if (done < nseg) {  // leftover rows: the staged-load KS3
                        auto kr = segscan_rows_kernel<OP, T>;
                        const int64_t R2 = L >= kRowsElems ? 1 : kRowsElems / L;
                        const int sm2 = (int)(R2 * L * (int64_t)sizeof(T));
                        if (sm2 > 32 * 1024)
                            cudaFuncSetAttribute((const void *)kr, cudaFuncAttributeMaxDynamicSharedMemorySize, sm2);
                        const int64_t g2 = ceil_div(nseg - done, R2);
                        kr<<<(unsigned)g2, 256, sm2, st>>>((const T *)in0 + done * L, nseg - done, L, R2,
                                                          (T *)out + done * L);
                        return launch_status(2);
                    }
                    return launch_status();
                }
                if (rg == RG_KS3) {
                    auto kr = segscan_rows_kernel<OP, T>;
                    const int64_t nseg = n / L;
                    const int64_t R = L >= kRowsElems ? 1 : kRowsElems / L;
                    const int smem = (int)(R * L * (int64_t)sizeof(T));
                    // (the kernel's static shared words count against the 48 KB default too:
                    // L = 12288 f32 is exactly 48 KB dynamic)
                    if (smem > 32 * 1024)
                        cudaFuncSetAttribute((const void *)kr, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
                    int64_t grid = ceil_div(nseg, R);
                    const int64_t cap = resident_blocks((const void *)kr, 256, (size_t)smem);
                    grid = grid > cap ? cap : (grid < 1 ? 1 : grid);
                    kr<<<(unsigned)grid, 256, smem, st>>>((const T *)in0, nseg, L, R, (T *)out);
                    return launch_status();
                }
                if (rg == RG_KS1) {
                    auto kt = segscan_tile_kernel<OP, T>;
                    const int smem = (int)((256 * L + 256 * L / 32 + 1) * sizeof(T));
                    if (smem > 32 * 1024)
                        cudaFuncSetAttribute((const void *)kt, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
                    const int64_t nseg = n / L;
                    int64_t grid = ceil_div(nseg, 256);
                    const int64_t cap = resident_blocks((const void *)kt, 256, (size_t)smem);
                    grid = grid > cap ? cap : (grid < 1 ? 1 : grid);
                    kt<<<(unsigned)grid, 256, smem, st>>>((const T *)in0, nseg, (int)L, (T *)out);
                    return launch_status();
                }
            }
            // a few very long rows: each row is a flat scan (the unsegmented slab scan, one launch
            // per row, workspace reused in stream order) -- fewer rows than SMs leave KS2 idle
            // and the segmented look-back pays a head flag per tile
            if (rg == RG_FLAT_ROW) {
                for (int64_t s = 0; s < n / L; ++s) {
                    const fs_status r = go<false, false, true>((const T *)in0 + s * L, nullptr, L, L, *map,
                                                               (T *)out + s * L, out_idx ? out_idx + s * L : nullptr,
                                                               nullptr, nullptr, ws, true, st);
                    if (r != FS_OK) return r;
                }
                return FS_OK;
            }
            if (al) return go<false, true, true>(in0, in1, n, L, *map, out, out_idx, carry, carry_idx, ws, al, st);
            return go<false, true, false>(in0, in1, n, L, *map, out, out_idx, carry, carry_idx, ws, al, st);
        }
        note_regime(RG_FLAT_ROW);
        if (al) return go<false, false, true>(in0, in1, n, L, *map, out, out_idx, carry, carry_idx, ws, al, st);
        return go<false, false, false>(in0, in1, n, L, *map, out, out_idx, carry, carry_idx, ws, al, st);
    }
};

size_t scan_ws(int op, int dt, int64_t n) {
    const int R = (op != FS_ARGMIN && dtype_size(dt) == 4) ? FS_SCAN_R : 2;
    const int64_t tile = (int64_t)kScanThreads * R * (16 / (int64_t)dtype_size(dt));
    const int64_t ntiles = ceil_div(n, tile);
    return kWsHeader + 256 + scan_state_bytes(ntiles) + 2 * align_up((size_t)ntiles * 32, 256);
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
    constexpr int UR = 8;  // rows in flight per thread
    int64_t r = r0;
    for (; r + UR <= r1; r += UR) {
        Vec16<T> e[UR];
        T s1[UR];
#pragma unroll
        for (int u = 0; u < UR; ++u) {
            if (VEC > 1) e[u] = as_vec<T>(ldg16(base + (r + u) * w));
            else s1[u] = __ldg(base + (r + u) * w);
        }
#pragma unroll
        for (int u = 0; u < UR; ++u) {
            if (VEC > 1) {
#pragma unroll
                for (int k = 0; k < VEC; ++k) acc[k] = O::fold(acc[k], e[u].e[k], r + u);
            } else {
                acc[0] = O::fold(acc[0], s1[u], r + u);
            }
        }
    }
    for (; r < r1; ++r) {
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

// exclusive scan over the Y row blocks of ONE column per CTA (few columns, many
// row blocks): each thread folds a contiguous run of row blocks, the CTA scans the
// per-thread totals, then each thread rewrites its run with the carries
template <int OP, typename T>
__global__ void __launch_bounds__(256) colscan_carry_block_kernel(typename Op<OP, T>::V *partials, int64_t w, int64_t Y) {
    using O = Op<OP, T>;
    using V = typename O::V;
    __shared__ V s_tot[256];
    const int64_t c = blockIdx.x;
    const int t = threadIdx.x;
    const int64_t chunk = (Y + 255) / 256;
    const int64_t y0 = t * chunk, y1 = y0 + chunk < Y ? y0 + chunk : Y;
    V a = O::id();
    for (int64_t y = y0; y < y1; ++y) a = O::comb(a, partials[y * w + c]);
    s_tot[t] = a;
    __syncthreads();
    V run = O::id();
    for (int q = 0; q < t; ++q) run = O::comb(run, s_tot[q]);  // exclusive prefix of the runs
    for (int64_t y = y0; y < y1; ++y) {
        const V p = partials[y * w + c];
        partials[y * w + c] = run;
        run = O::comb(run, p);
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
    constexpr int UR = 8;  // rows loaded ahead per thread
    int64_t r = r0;
    for (; r + UR <= r1; r += UR) {
        Vec16<T> e[UR];
        T s1[UR];
#pragma unroll
        for (int u = 0; u < UR; ++u) {
            if (VEC > 1) e[u] = as_vec<T>(ldg16(base + (r + u) * w));
            else s1[u] = __ldg(base + (r + u) * w);
        }
#pragma unroll
        for (int u = 0; u < UR; ++u) {
            const int64_t rr = r + u;
            if (VEC > 1) {
                Vec16<T> o;
#pragma unroll
                for (int k = 0; k < VEC; ++k) {
                    acc[k] = O::comb(acc[k], O::lift(e[u].e[k], rr));
                    o.e[k] = O::val(acc[k]);
                    if (OP == kArgmin) out_idx[rr * w + cv * VEC + k] = O::idx(acc[k]);
                }
                int4 ov;
                memcpy(&ov, &o, 16);
                *reinterpret_cast<int4 *>(obase + rr * w) = ov;
            } else {
                acc[0] = O::comb(acc[0], O::lift(s1[u], rr));
                obase[rr * w] = O::val(acc[0]);
                if (OP == kArgmin) out_idx[rr * w + cv] = O::idx(acc[0]);
            }
        }
    }
    for (; r < r1; ++r) {
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

// ---------------------------------------------------------------- narrow column-major seg_scan
// Few columns (a row of w elements is WV <= 8 16-byte vectors, WV | 32): a WARP owns a block
// of rows and its lanes read 32 / WV consecutive rows at a time (lane l: row l / WV, vector
// column l % WV), so every warp load is one contiguous 512-byte run.  The per-thread
// (vector-column, row-block) units of the generic kernels above would give every lane its
// own row block and thrash L1 when rows are this short.  Partial: fold, then combine the
// row-lanes of each column with xor shuffles.  Scan: per 32/WV-row step, an inclusive shuffle
// scan down the row-lanes of each column plus the running carry.
template <int OP, typename T, bool CARRY, bool SCAN>
__global__ void __launch_bounds__(kColScanThreads)
colscan_narrow_kernel(const T *__restrict__ x, int64_t m, int64_t w, int WV, int64_t Y, int64_t rpu,
                      typename Op<OP, T>::V *parts, T *__restrict__ out, int64_t *__restrict__ out_idx) {
    using O = Op<OP, T>;
    using V = typename O::V;
    constexpr int VEC = 16 / sizeof(T);
    const int lane = threadIdx.x & 31;
    const int64_t y = ((int64_t)blockIdx.x * kColScanThreads + threadIdx.x) >> 5;  // warp = unit
    if (y >= Y) return;
    const int cv = lane % WV, ro = lane / WV, RPW = 32 / WV;
    const int64_t r0 = y * rpu, r1 = r0 + rpu < m ? r0 + rpu : m;
    V acc[VEC];
#pragma unroll
    for (int k = 0; k < VEC; ++k) acc[k] = CARRY ? parts[y * w + cv * VEC + k] : O::id();
    for (int64_t rb = r0; rb < r1; rb += RPW) {
        const int64_t r = rb + ro;
        const bool ok = r < r1;
        Vec16<T> e;
        if (ok) e = as_vec<T>(ldg16(x + r * w + cv * VEC));
        if constexpr (!SCAN) {
            if (ok)
#pragma unroll
                for (int k = 0; k < VEC; ++k) acc[k] = O::comb(acc[k], O::lift(e.e[k], r));
        } else {
            V v[VEC];
#pragma unroll
            for (int k = 0; k < VEC; ++k) v[k] = ok ? O::lift(e.e[k], r) : O::id();
#pragma unroll 1
            for (int dd = 1; dd < RPW; dd <<= 1) {
#pragma unroll
                for (int k = 0; k < VEC; ++k) {
                    const V o = shfl_up(v[k], dd * WV);
                    if (ro >= dd) v[k] = O::comb(o, v[k]);
                }
            }
            Vec16<T> o;
#pragma unroll
            for (int k = 0; k < VEC; ++k) {
                const V z = O::comb(acc[k], v[k]);
                o.e[k] = O::val(z);
                if (ok && OP == kArgmin) out_idx[r * w + cv * VEC + k] = O::idx(z);
                acc[k] = shfl_idx(z, (RPW - 1) * WV + cv);  // carry = the step's last row of this column
            }
            if (ok) *reinterpret_cast<int4 *>(out + r * w + cv * VEC) = *reinterpret_cast<const int4 *>(&o);
        }
    }
    if (!SCAN) {
        for (int dd = WV; dd < 32; dd <<= 1)
#pragma unroll
            for (int k = 0; k < VEC; ++k) acc[k] = O::comb(acc[k], shfl_xor(acc[k], dd));
        if (ro == 0)
#pragma unroll
            for (int k = 0; k < VEC; ++k) parts[y * w + cv * VEC + k] = acc[k];
    }
}

// ---------------------------------------------------------------- one-pass column-major seg_scan
// Column-major seg_scan with row splitting in ONE pass (one read and one write per element): a
// block is (column tile xt of CG vector-columns, row block y of RB thread-rows x K rows).  Each
// CTA takes the next block id from an atomic counter (row-block-major, so the block above is
// already owned by a running CTA), scans its K rows per thread in registers, combines the RB
// thread-row totals of every column (Hillis-Steele over shared memory), and then -- one thread
// per column -- runs a decoupled look-back up its column through the blocks above (published
// per-(block, column) aggregate / inclusive prefix, TileState), i.e. F5 (L1071-1074) with the
// chunks stacked down each column.  The three-kernel reduce / carry-scan / rescan above reads
// every element twice (12 B per element).
template <int OP, typename T, int VEC, int K>
__global__ void __launch_bounds__(256)
colscan_lb_kernel(const T *__restrict__ x, int64_t m, int64_t w, int CG, int64_t ntx, unsigned *counter,
                  TileState<typename SOp<Op<OP, T>, false>::S, ScanShape<OP, T>::PACK> ts, T *__restrict__ out,
                  int64_t *__restrict__ out_idx) {
    using O = Op<OP, T>;
    using V = typename O::V;
    using SO = SOp<O, false>;
    using S = typename SO::S;
    constexpr int NT = 256;
    __shared__ V sc[NT * VEC];
    __shared__ V s_carry[NT];
    __shared__ int64_t s_bid;
    const int t = threadIdx.x;
    const int RB = NT / CG, TCW = CG * VEC;
    if (t == 0) s_bid = atomicAdd(counter, 1u);
    __syncthreads();
    const int64_t bid = s_bid;
    const int64_t y = bid / ntx, xt = bid % ntx;
    const int cg = t % CG, roff = t / CG;
    const bool act = roff < RB;
    const int64_t c = (xt * CG + cg) * VEC;
    const bool colok = act && c < w;
    const int64_t rbase = y * (int64_t)RB * K + (int64_t)roff * K;
    V a[K][VEC];
    if (VEC > 1) {
        int4 raw[K];
#pragma unroll
        for (int j = 0; j < K; ++j)
            if (colok && rbase + j < m) raw[j] = ldg16(x + (rbase + j) * w + c);
#pragma unroll
        for (int j = 0; j < K; ++j) {
            const Vec16<T> e = as_vec<T>(raw[j]);
#pragma unroll
            for (int k = 0; k < VEC; ++k) a[j][k] = (colok && rbase + j < m) ? O::lift(e.e[k], rbase + j) : O::id();
        }
    } else {
        T raw[K];
#pragma unroll
        for (int j = 0; j < K; ++j)
            if (colok && rbase + j < m) raw[j] = __ldg(x + (rbase + j) * w + c);
#pragma unroll
        for (int j = 0; j < K; ++j) a[j][0] = (colok && rbase + j < m) ? O::lift(raw[j], rbase + j) : O::id();
    }
#pragma unroll
    for (int j = 1; j < K; ++j)
#pragma unroll
        for (int k = 0; k < VEC; ++k) a[j][k] = O::comb(a[j - 1][k], a[j][k]);
    if (act)
#pragma unroll
        for (int k = 0; k < VEC; ++k) sc[roff * TCW + cg * VEC + k] = a[K - 1][k];
    __syncthreads();
    for (int d = 1; d < RB; d <<= 1) {  // inclusive scan over the thread rows of every column
        V v[VEC];
        const bool up = act && roff >= d;
        if (up)
#pragma unroll
            for (int k = 0; k < VEC; ++k) v[k] = O::comb(sc[(roff - d) * TCW + cg * VEC + k], sc[roff * TCW + cg * VEC + k]);
        __syncthreads();
        if (up)
#pragma unroll
            for (int k = 0; k < VEC; ++k) sc[roff * TCW + cg * VEC + k] = v[k];
        __syncthreads();
    }
    if (t < TCW) {  // decoupled look-back up column t of the tile
        const S agg{sc[(RB - 1) * TCW + t], 0};
        S run = SO::id();
        if (y == 0) {
            ts.publish(bid * TCW + t, agg, kStIncl);
        } else {
            ts.publish(bid * TCW + t, agg, kStAgg);
            int64_t p = bid - ntx;
            while (true) {
                S s;
                const unsigned st = ts.poll(p * TCW + t, s);
                if (st == 0) continue;
                run = SO::comb(s, run);
                if (st == kStIncl) break;
                p -= ntx;
            }
            ts.publish(bid * TCW + t, SO::comb(run, agg), kStIncl);
        }
        s_carry[t] = run.v;
    }
    __syncthreads();
    if (!colok) return;
    V pre[VEC];
#pragma unroll
    for (int k = 0; k < VEC; ++k)
        pre[k] = roff > 0 ? O::comb(s_carry[cg * VEC + k], sc[(roff - 1) * TCW + cg * VEC + k]) : s_carry[cg * VEC + k];
#pragma unroll
    for (int j = 0; j < K; ++j) {
        const int64_t r = rbase + j;
        if (r >= m) break;
        if (VEC > 1) {
            Vec16<T> o;
#pragma unroll
            for (int k = 0; k < VEC; ++k) {
                const V z = O::comb(pre[k], a[j][k]);
                o.e[k] = O::val(z);
                if (OP == kArgmin) out_idx[r * w + c + k] = O::idx(z);
            }
            *reinterpret_cast<int4 *>(out + r * w + c) = *reinterpret_cast<const int4 *>(&o);
        } else {
            const V z = O::comb(pre[0], a[j][0]);
            out[r * w + c] = O::val(z);
            if (OP == kArgmin) out_idx[r * w + c] = O::idx(z);
        }
    }
}

// Few rows (m <= 8) of many columns, any alignment: a warp owns 4 x 32 consecutive columns, lane l
// the columns l, l + 32, l + 64, l + 96 (every load and store instruction of the warp is one
// contiguous 128-byte run), all m x 4 loads in flight, each column scanned down the rows.
template <int OP, typename T, int MMAX>
__global__ void __launch_bounds__(256)
colscan_short_kernel(const T *__restrict__ x, int m, int64_t w, T *__restrict__ out, int64_t *__restrict__ out_idx) {
    using O = Op<OP, T>;
    using V = typename O::V;
    constexpr int C = 4;
    const int lane = threadIdx.x & 31;
    const int64_t nw = (w + 32 * C - 1) / (32 * C);  // warp column groups
    const int64_t wstride = (int64_t)gridDim.x * 8;
    for (int64_t g = (int64_t)blockIdx.x * 8 + (threadIdx.x >> 5); g < nw; g += wstride) {
        const int64_t c0 = g * 32 * C + lane;
        T v[MMAX][C];
#pragma unroll
        for (int r = 0; r < MMAX; ++r)
#pragma unroll
            for (int k = 0; k < C; ++k)
                if (r < m && c0 + 32 * k < w) v[r][k] = __ldg(x + (int64_t)r * w + c0 + 32 * k);
#pragma unroll
        for (int k = 0; k < C; ++k) {
            const int64_t c = c0 + 32 * k;
            if (c >= w) break;
            V a = O::id();
#pragma unroll
            for (int r = 0; r < MMAX; ++r) {
                if (r >= m) break;
                a = O::comb(a, O::lift(v[r][k], r));
                out[(int64_t)r * w + c] = O::val(a);
                if (OP == kArgmin) out_idx[(int64_t)r * w + c] = O::idx(a);
            }
        }
    }
}

struct ColScanPlan {
    int vec;
    bool narrow;  // colscan_narrow_kernel: a warp per row block
    int64_t WV, Y, rpu;
    // one-pass look-back plan (taken whenever the rows must be split, Y > 1)
    int CG, K;
    int64_t ntx, nby, nblocks, nstate;
};
template <int OP, typename T> constexpr int colscan_lb_k() { return ScanShape<OP, T>::PACK ? 8 : 4; }
static ColScanPlan colscan_plan(int dt, int64_t m, int64_t w, bool aligned) {
    ColScanPlan p;
    const int V = 16 / (int)dtype_size(dt);
    p.vec = (aligned && w % V == 0) ? V : 1;
    p.WV = ceil_div(w, p.vec);
    p.narrow = p.vec > 1 && p.WV <= 8 && (32 % p.WV) == 0 && m >= 4096;
    if (p.narrow) {  // warps (units) of 32 / WV-row steps
        int64_t Y = (int64_t)sm_count() * (2048 / 32);
        const int64_t by_rows = m / 256;
        if (Y > by_rows) Y = by_rows;
        if (Y < 1) Y = 1;
        const int64_t step = 32 / p.WV;
        p.rpu = ceil_div(ceil_div(m, Y), step) * step;
        p.Y = ceil_div(m, p.rpu);
        return p;
    }
    const int64_t threads = (int64_t)sm_count() * 2048;
    int64_t Y = ceil_div(threads, p.WV);
    const int64_t by_rows = m / 16;
    if (Y > by_rows) Y = by_rows;
    if (Y < 1) Y = 1;
    p.rpu = ceil_div(m, Y);
    p.Y = ceil_div(m, p.rpu);
    return p;
}
static void colscan_lb_plan(ColScanPlan &p, int64_t m, int K) {
    p.K = K;
    p.CG = (int)(p.WV < 32 ? p.WV : 32);
    const int64_t RB = 256 / p.CG;
    p.ntx = ceil_div(p.WV, p.CG);
    p.nby = ceil_div(m, RB * K);
    p.nblocks = p.ntx * p.nby;
    p.nstate = p.nblocks * p.CG * p.vec;
}

template <int OP, typename T> struct ColScanRun {
    template <int VEC>
    static fs_status go(const ColScanPlan &p, const T *x, int64_t m, int64_t w, T *out, int64_t *out_idx, void *ws,
                        cudaStream_t st) {
        using V = typename Op<OP, T>::V;
        V *parts = (V *)((char *)ws + kWsHeader);
        if (p.Y > 1) {  // rows split: the one-pass look-back kernel
            ColScanPlan q = p;
            colscan_lb_plan(q, m, colscan_lb_k<OP, T>());
            using S = typename SOp<Op<OP, T>, false>::S;
            using Sh = ScanShape<OP, T>;
            char *b = (char *)ws + kWsHeader;
            unsigned *counter = (unsigned *)b;
            TileState<S, Sh::PACK> ts;
            ts.w = (uint64_t *)(b + 256);
            if constexpr (!Sh::PACK) {
                ts.aggs = (S *)(b + 256 + scan_state_bytes(q.nstate));
                ts.incls = ts.aggs + q.nstate;
            }
            if (cudaMemsetAsync(counter, 0, 256 + scan_state_bytes(q.nstate), st) != cudaSuccess) return FS_ERR_CUDA;
            colscan_lb_kernel<OP, T, VEC, colscan_lb_k<OP, T>()><<<(unsigned)q.nblocks, 256, 0, st>>>(
                x, m, w, q.CG, q.ntx, counter, ts, out, out_idx);
            return launch_status();
        }
        if (p.narrow) {
            const unsigned gn = (unsigned)ceil_div(p.Y * 32, kColScanThreads);
            const int wv = (int)p.WV;
            if (p.Y == 1) {
                colscan_narrow_kernel<OP, T, false, true><<<gn, kColScanThreads, 0, st>>>(x, m, w, wv, 1, p.rpu, parts,
                                                                                         out, out_idx);
                return launch_status();
            }
            colscan_narrow_kernel<OP, T, false, false><<<gn, kColScanThreads, 0, st>>>(x, m, w, wv, p.Y, p.rpu, parts,
                                                                                      out, out_idx);
            if (p.Y >= 256) {
                colscan_carry_block_kernel<OP, T><<<(unsigned)w, 256, 0, st>>>(parts, w, p.Y);
            } else {
                int64_t g2 = ceil_div(w, 128);
                colscan_carry_kernel<OP, T><<<(unsigned)(g2 > 4096 ? 4096 : g2), 128, 0, st>>>(parts, w, p.Y);
            }
            colscan_narrow_kernel<OP, T, true, true><<<gn, kColScanThreads, 0, st>>>(x, m, w, wv, p.Y, p.rpu, parts,
                                                                                    out, out_idx);
            return launch_status(3);
        }
        const int64_t units = p.WV * p.Y;
        const unsigned grid = (unsigned)ceil_div(units, kColScanThreads);
        if (p.Y == 1) {
            colscan_kernel<OP, T, VEC, false><<<grid, kColScanThreads, 0, st>>>(x, m, w, p.WV, 1, p.rpu, parts, out,
                                                                                out_idx);
            return launch_status();
        }
        colscan_partial_kernel<OP, T, VEC><<<grid, kColScanThreads, 0, st>>>(x, m, w, p.WV, p.Y, p.rpu, parts);
        if (p.Y >= 256) {  // few columns, many row blocks: one CTA per column
            colscan_carry_block_kernel<OP, T><<<(unsigned)w, 256, 0, st>>>(parts, w, p.Y);
        } else {
            int64_t g2 = ceil_div(w, 128);
            g2 = g2 > 4096 ? 4096 : g2;
            colscan_carry_kernel<OP, T><<<(unsigned)g2, 128, 0, st>>>(parts, w, p.Y);
        }
        colscan_kernel<OP, T, VEC, true><<<grid, kColScanThreads, 0, st>>>(x, m, w, p.WV, p.Y, p.rpu, parts, out,
                                                                           out_idx);
        return launch_status(3);
    }
    static fs_status run(const void *in, int64_t m, int64_t w, void *out, int64_t *out_idx, void *ws, cudaStream_t st) {
        const bool aligned = ((uintptr_t)in & 15) == 0 && ((uintptr_t)out & 15) == 0;
        const bool vec_ok = aligned && w % (16 / sizeof(T)) == 0;
        // few rows, many columns: the lane-interleaved short kernel for any phase, and for aligned
        // rows up to 2 (col L = 2: 0.70 -> 0.91; at 4 and 8 rows the vector kernels are faster)
        if (m <= 8 && (!vec_ok || m <= 2) && w >= (int64_t)sm_count() * 2048) {
            const int64_t ng = ceil_div(w, 4 * 256);
            const int64_t gmax = (int64_t)sm_count() * 16;
            const unsigned grid = (unsigned)(ng < gmax ? ng : gmax);
            if (m <= 4)
                colscan_short_kernel<OP, T, 4><<<grid, 256, 0, st>>>((const T *)in, (int)m, w, (T *)out, out_idx);
            else
                colscan_short_kernel<OP, T, 8><<<grid, 256, 0, st>>>((const T *)in, (int)m, w, (T *)out, out_idx);
            return launch_status();
        }
        const ColScanPlan p = colscan_plan(sizeof(T) == 8 ? FS_I64 : FS_I32, m, w, aligned);
        if (p.vec > 1) return go<16 / sizeof(T)>(p, (const T *)in, m, w, (T *)out, out_idx, ws, st);
        return go<1>(p, (const T *)in, m, w, (T *)out, out_idx, ws, st);
    }
};

size_t colscan_ws(int op, int dt, int64_t m, int64_t w) {
    ColScanPlan a = colscan_plan(dt, m, w, false), b = colscan_plan(dt, m, w, true);
    const int64_t Y = a.Y > b.Y ? a.Y : b.Y;
    // one-pass plan: counter, state words, and (not PACK) aggregate + inclusive payloads
    const bool pack = op != FS_ARGMIN && dtype_size(dt) == 4;
    const int K = pack ? 8 : 4;
    colscan_lb_plan(a, m, K);
    colscan_lb_plan(b, m, K);
    const int64_t ns = a.nstate > b.nstate ? a.nstate : b.nstate;
    const size_t pay = pack ? 0 : 2 * (size_t)ns * (acc_size(op, dt) + 8);
    const size_t lb = 256 + scan_state_bytes(ns) + pay;
    const size_t old = align_up((size_t)Y * w * acc_size(op, dt), 256);
    return kWsHeader + (lb > old ? lb : old);
}

fs_status colscan_run(int op, int dt, const void *in, int64_t m, int64_t w, void *out, int64_t *out_idx, void *ws,
                      cudaStream_t st) {
    return dispatch<ColScanRun>(op, dt, in, m, w, out, out_idx, ws, st);
}

}  // namespace fs
