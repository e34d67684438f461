// kmeans.cu -- NEXT-1: one fused iteration of Rodinia's K-means (Sec. 2.4,
// L445-531; L1628-1649; fusion F6 L1075-1090: the assignment map is fused into the
// stream_red that computes the new centres, so the points are read once and the
// membership array never has to be re-read).
//
//   membership[i] = argmin_c E(i, c), first c on ties            (readings R3, R18)
//   E(i, c)       = sum_j (x_ij - c_cj)^2, f32, j in order, acc = fma(t, t, acc)
//   sums, counts  = stream_red (map(+)) over the new membership  (Fig 4c)
//   new_centres   = sums / counts; an empty cluster keeps its centre     (R19)
//   delta         = #{ i : membership[i] != prev[i] }  (Rodinia's convergence test)
//
// B200 design: both contractions of the step run on the 5th-generation tensor cores
// (tcgen05.mma kind::tf32, accumulators in TMEM); the CUDA cores stage operands and
// take the per-row decision.  A stage is 128 consecutive points (one M = 128 tile); a
// CTA per SM streams its contiguous chunk of stages; warps are specialised:
//
//   producer  (1 warp)  1-D TMA bulk copies of the stages' rows into an NR-slot ring.
//   convert   (4 warps) thread r owns row r of a stage: reads it (conflict-free 8-byte
//             loads), computes |x|^2, splits every x into hi = x with the low 13 mantissa
//             bits cleared (exactly TF32) and lo = x - hi (exact), and writes
//               - hi | 1 1 (columns d, d+1) and lo into TMEM (tcgen05.st, TMEM lane r),
//                 the K-major A operand of MMA1, plus |x|^2 in one more column;
//               - hi[0..31], lo[0..31] and the extras (hi/lo of columns 32.., a 1.0 for
//                 the count) into shared memory as the MN-major A operand of MMA2
//                 (128B swizzle with 32-byte atoms: the layout tf32 MN-major needs).
//   MMA       (1 thread) MMA1: d~ = |c|^2 - 2 x.c for 128 rows x NC centres as three
//             TF32 products (hi.Bhi + hi.Blo + lo.Bhi; B = -2c split the same way, |c|^2
//             split in the augmented columns) -> TMEM D1.  MMA2: D2[j][c] += sum over the
//             stage's rows of X[row][j] * onehot[row][c] -> TMEM D2, 16 stages per buffer
//             (double-buffered).  It polls both queues so MMA1 runs ahead of decisions.
//   decide    (4 warps) thread r: one tcgen05.ld of its NC values, minimum m, candidates
//             d~_c <= m + 2 delta(x).  delta bounds |d~_c - (E_f32(x, c) - |x|^2)| (TF32
//             splitting 6 * 2^-20 |x||c|, the f32 |c|^2, the tensor core's f32
//             accumulation and the f32 rounding of R18's own E: all below 2^-15 (|x| +
//             |c|)^2 <= 2^-14 (|x|^2 + max|c|^2)), so R18's argmin is always a
//             candidate.  One candidate decides the row; several (rare) are re-evaluated
//             in R18's exact f32 order from x = hi + lo.  Writes the one-hot B operand of
//             MMA2 (K-major, one 1.0 per row, reset when the slot comes back),
//             membership and delta; every 16 stages moves D2 into registers (two-level
//             f32 accumulation).
// Chunk results combine CTA -> workspace -> last CTA, which divides by the counts.
#include <cuda_bf16.h>
#include <stdio.h>
#include <stdlib.h>

#include "internal.cuh"

namespace fs {

constexpr int kKmRows = 128;   // rows per stage (UMMA M)
constexpr int kKmRing = 5;     // TMA ring slots (at most)
constexpr int kKmCv = 2;       // convert groups of 4 warps; group g converts stages s = g (mod 2)
#ifndef FS_KM_NA
#define FS_KM_NA 4
#endif
constexpr int kKmNA = FS_KM_NA;  // TMEM stage slots (A operand, D1); 5 measured no faster than 4
constexpr int kKmDc = 2;       // decide groups of 4 warps; group g decides stages s = g (mod 2)
constexpr int kKmNXMax = 6;    // shared-memory stage slots (MMA2 operands), at most
constexpr int kKmThreads = (4 * kKmCv + 4 * kKmDc + 3) * 32;  // convert + decide + producer + 2 MMA warps
constexpr int kKmWarpDecide = 4 * kKmCv, kKmWarpProd = 4 * (kKmCv + kKmDc), kKmWarpMma = kKmWarpProd + 1;
// (MMA1 and MMA2 are issued by two warps, kKmWarpMma and kKmWarpMma + 1: a tcgen05.mma occupies
// its issuing thread for ~100+ cycles, one issuer alone could not keep up with both streams)
constexpr int kKmK = 32;       // max clusters
constexpr int kKmMaxD = 40;
constexpr int kKmSeg = 16;     // stages per D2 buffer


__device__ __forceinline__ uint32_t km_smem(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void km_arrive(uint64_t *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(km_smem(bar)) : "memory");
}
__device__ __forceinline__ void km_wait(uint64_t *bar, unsigned parity) {  // suspends in hardware while waiting
    uint32_t done = 0;
    while (!done) {
        asm volatile(
            "{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
            : "=r"(done)
            : "r"(km_smem(bar)), "r"(parity)
            : "memory");
    }
}
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
// no-swizzle UMMA shared-memory descriptor: start, leading (LBO) and stride (SBO) byte
// offsets >> 4, version 1 (sm_100), layout type 0 (SWIZZLE_NONE)
__device__ __forceinline__ uint64_t umma_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
    return (uint64_t)((saddr >> 4) & 0x3FFFu) | ((uint64_t)((lbo >> 4) & 0x3FFFu) << 16) |
           ((uint64_t)((sbo >> 4) & 0x3FFFu) << 32) | (1ull << 46);
}
// instruction descriptor, kind::f16 with bf16 A/B and f32 D, M = 128, N, majors (0 K, 1 MN)
__host__ __device__ constexpr uint32_t umma_idesc_bf16(int N, int a_mn, int b_mn) {
    return (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)a_mn << 15) | ((uint32_t)b_mn << 16) |
           ((uint32_t)(N >> 3) << 17) | ((uint32_t)(kKmRows >> 4) << 24);
}
// D[tmem] (+)= A[smem] . B[smem]
__device__ __forceinline__ void umma_bf16_ss(uint32_t dtmem, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(dtmem),
        "l"(a), "l"(b), "r"(idesc), "r"(acc)
        : "memory");
}
// D[tmem] (+)= A[tmem] (K-major) . B[smem]
__device__ __forceinline__ void umma_bf16_ts(uint32_t dtmem, uint32_t atmem, uint64_t b, uint32_t idesc, uint32_t acc) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}" ::"r"(dtmem),
        "r"(atmem), "l"(b), "r"(idesc), "r"(acc)
        : "memory");
}
__device__ __forceinline__ void umma_commit(uint64_t *bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(km_smem(bar))
                 : "memory");
}
// 32 lanes x 32 consecutive 32-bit columns: thread i of the warp gets lane (base + i)
__device__ __forceinline__ void tmem_ld32(uint32_t taddr, float (&v)[32]) {
    uint32_t r[32];
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,%18,"
        "%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]),
          "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]), "=r"(r[16]),
          "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]),
          "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
        : "r"(taddr)
        : "memory");
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
    for (int i = 0; i < 32; ++i) v[i] = __uint_as_float(r[i]);
}
__device__ __forceinline__ void km_tma_load(void *dst, const void *src, unsigned bytes, uint64_t *bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     km_smem(dst)),
                 "l"(src), "r"(bytes), "r"(km_smem(bar))
                 : "memory");
}
__device__ __forceinline__ void km_bar_sync(int id, int count) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(count) : "memory");
}
__device__ __forceinline__ uint32_t bf2(float lo, float hi) {  // packed bf16 pair, round to nearest even
    const __nv_bfloat162 p = __floats2bfloat162_rn(lo, hi);
    return *reinterpret_cast<const uint32_t *>(&p);
}
__device__ __forceinline__ float bfr(float x) { return __bfloat162float(__float2bfloat16_rn(x)); }
__device__ __forceinline__ float fmin3(float a, float b, float c) {
    float r;
    asm("min.f32 %0, %1, %2, %3;" : "=f"(r) : "f"(a), "f"(b), "f"(c));
    return r;
}
__device__ __forceinline__ void tmem_ld64(uint32_t taddr, float (&v)[64]) {
    float a[32], b[32];
    tmem_ld32(taddr, a);
    tmem_ld32(taddr + 32, b);
#pragma unroll
    for (int i = 0; i < 32; ++i) {
        v[i] = a[i];
        v[32 + i] = b[i];
    }
}
__device__ __forceinline__ bool km_test(uint64_t *bar, unsigned parity) {
    uint32_t done;
    asm volatile(
        "{\n\t.reg .pred p;\n\tmbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(done)
        : "r"(km_smem(bar)), "r"(parity)
        : "memory");
    return done != 0;
}
__device__ __forceinline__ void tmem_st8u(uint32_t taddr, const uint32_t (&v)[8]) {
    asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"r"(taddr), "r"(v[0]),
                 "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7])
                 : "memory");
}
__device__ __forceinline__ void tmem_st32(uint32_t taddr, const float (&v)[32]) {
    asm volatile(
        "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,%18,"
        "%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};" ::"r"(taddr),
        "f"(v[0]), "f"(v[1]), "f"(v[2]), "f"(v[3]), "f"(v[4]), "f"(v[5]), "f"(v[6]), "f"(v[7]), "f"(v[8]), "f"(v[9]),
        "f"(v[10]), "f"(v[11]), "f"(v[12]), "f"(v[13]), "f"(v[14]), "f"(v[15]), "f"(v[16]), "f"(v[17]), "f"(v[18]),
        "f"(v[19]), "f"(v[20]), "f"(v[21]), "f"(v[22]), "f"(v[23]), "f"(v[24]), "f"(v[25]), "f"(v[26]), "f"(v[27]),
        "f"(v[28]), "f"(v[29]), "f"(v[30]), "f"(v[31])
        : "memory");
}
__device__ __forceinline__ void tmem_st1(uint32_t taddr, float v) {
    asm volatile("tcgen05.st.sync.aligned.32x32b.x1.b32 [%0], {%1};" ::"r"(taddr), "r"(__float_as_uint(v)) : "memory");
}
__device__ __forceinline__ float tmem_ld1(uint32_t taddr) {
    uint32_t r;
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x1.b32 {%0}, [%1];" : "=r"(r) : "r"(taddr) : "memory");
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
    return __uint_as_float(r);
}
// E(x, c) exactly as reading R18 / the oracle: f32, j in order, one rounding per fma
__device__ __forceinline__ float km_exact(const float *x, const float *c, int d) {
    float acc = 0.f;
    for (int j = 0; j < d; ++j) {
        const float tt = __fsub_rn(__ldg(x + j), c[j]);
        acc = __fmaf_rn(tt, tt, acc);
    }
    return acc;
}



// Debug tracing (tools/km_trace.py): clock64 stamps of CTA 0's pipeline events per stage when
// FUTSEG_KM_TRACE is set; [stage][8]: convert begin / ready / end, decide begin / ready / end,
// MMA1 issue, MMA2 issue.
__device__ long long *g_km_trace = nullptr;
__device__ int g_km_trace_cta = 0;

#define KM_TRACE(s, e)                                                                   \
    do {                                                                                 \
        if (trace && (threadIdx.x & 127) == 0) trace[(s) * 16 + (e)] = clock64();         \
    } while (0)

struct KmBars {
    uint64_t raw_full[kKmRing], raw_empty[kKmRing];
    uint64_t a1full[kKmNA], d1full[kKmNA], slotfree[kKmNA];
    uint64_t ohfull[kKmNXMax], x2free[kKmNXMax];
    uint64_t d2full[2], d2free[2];
    uint32_t tmem_base;
    float cmax2;
    float nrm[kKmNA][kKmRows];  // |x|^2 of the rows of the stages in the TMEM slots
    short ohpos[kKmNXMax][kKmRows];  // the one-hot entry row r set in X slot q (-1: none), reset
                                     // by whichever decide group reuses the slot next
};
// running f32 totals of the D2 buffers ([128 M rows][NC]), after the barriers in shared memory

// Operand geometry for a given d (host and device):
//   KP  = bf16 columns of one A piece: d + 3 augmentation columns, padded to 16
//   JB  = first MMA2 row of the a2 piece (a1 rows 0..d-1, the count row d), padded to 8
//   NG  = MMA2 M-groups written (8 rows each): JB/8 + ceil(d/8)
struct KmGeom {
    int KP, JB, NG;
    __host__ __device__ KmGeom(int d) : KP((d + 3 + 15) / 16 * 16), JB((d + 1 + 7) / 8 * 8), NG(0) {
        NG = JB / 8 + (d + 7) / 8;
    }
    __host__ __device__ int x2_bytes() const { return 16 * NG * 128; }
};

__device__ __forceinline__ uint32_t cvt_bf2(float lo, float hi) {  // packed bf16 pair, round to nearest even
    uint32_t r;
    asm("cvt.rn.bf16x2.f32 %0, %1, %2;" : "=r"(r) : "f"(hi), "f"(lo));
    return r;
}

__device__ int g_km_skip = 0;  // debug: bit 0 skips the MMA2 instructions, bit 1 the MMA1 ones, bit 2 the
                               // A stores to TMEM, bit 3 the X stores to shared memory (timing only)
// One row of a stage -> the two bf16 pieces of every column, written as the MMA1 A operand (TMEM
// lane of the calling thread, K-major pairs: [a1 | 1 1 1 | 0..] then [a2 | 0..], KP columns each)
// and as the MMA2 A operand (shared memory, MN-major: the row is the K index, a1 rows 0..d-1, the
// count row d, a2 rows JB..JB+d-1).  Returns |x|^2 (f32).
// PK (even compile-time d): MMA1's A packed as [a1 (d) | a2 (d) | 1 1 1 | 0] in K1 = roundup16(2d + 3)
// columns (5 instructions at d = 34 instead of 6); otherwise [a1 | 1 1 1 | 0] [a2 | 0], KP each.
template <bool FULL, bool EVEN, int PK>
__device__ __forceinline__ float km_convert_row(const float *src, int d, bool valid, const KmGeom &G, int qd,
                                                uint32_t ta, unsigned char *xr, int skip) {
    float nrm = 0.f;
    uint32_t a2w[PK > 0 ? PK / 2 + 8 : 1];  // PK: the a2 pairs (+ the last a1 pairs), stored after the loop
#pragma unroll
    for (int q = 0; q < 3; ++q) {  // 16 columns per chunk (KP <= 48)
        if (16 * q < G.KP) {
            uint32_t w1[8], w2[8];
            const bool tail = q >= qd;  // the chunk holding column d (augmentation, count)
#pragma unroll
            for (int t = 0; t < 8; ++t) {
                const int j0 = 16 * q + 2 * t, j1 = j0 + 1;
                float x0, x1;
                if (EVEN && (!tail || j1 < d)) {
                    const float2 p2 = *reinterpret_cast<const float2 *>(src + j0);
                    x0 = p2.x;
                    x1 = p2.y;
                } else if (!tail) {
                    x0 = src[j0];
                    x1 = src[j1];
                } else {
                    x0 = j0 < d ? src[j0] : 0.f;
                    x1 = j1 < d ? src[j1] : 0.f;
                }
                if (!FULL && !valid) x0 = x1 = 0.f;
                nrm = __fmaf_rn(x0, x0, nrm);
                nrm = __fmaf_rn(x1, x1, nrm);
                w1[t] = cvt_bf2(x0, x1);
                w2[t] = cvt_bf2(__fsub_rn(x0, __uint_as_float(w1[t] << 16)),
                                __fsub_rn(x1, __uint_as_float(w1[t] & 0xFFFF0000u)));
            }
            uint32_t wt[8], wx[8];
#pragma unroll
            for (int t = 0; t < 8; ++t) {
                wt[t] = w1[t];
                wx[t] = w1[t];
            }
            if (tail) {  // MMA1 A: 1.0 in columns d, d+1, d+2; MMA2 A: the count at d
#pragma unroll
                for (int t = 0; t < 8; ++t) {
                    const int j0 = 16 * q + 2 * t, j1 = j0 + 1;
                    wt[t] |= ((j0 >= d && j0 <= d + 2) ? 0x3F80u : 0u) | ((j1 >= d && j1 <= d + 2) ? 0x3F800000u : 0u);
                    wx[t] |= ((j0 == d && valid) ? 0x3F80u : 0u) | ((j1 == d && valid) ? 0x3F800000u : 0u);
                }
            }
            if (PK > 0) {
#pragma unroll
                for (int t = 0; t < 8; ++t)
                    if (8 * q + t < PK / 2) a2w[8 * q + t] = w2[t];
                if (8 * q + 8 <= PK / 2) tmem_st8u(ta + 8 * q, w1);  // whole chunks of a1 pairs
            } else if (!(skip & 4)) {
                tmem_st8u(ta + 8 * q, wt);
                tmem_st8u(ta + G.KP / 2 + 8 * q, w2);
            }
            if (skip & 8) continue;
            if (16 * q < G.JB) *reinterpret_cast<uint4 *>(xr + (2 * q) * 128) = make_uint4(wx[0], wx[1], wx[2], wx[3]);
            if (16 * q + 8 < G.JB)
                *reinterpret_cast<uint4 *>(xr + (2 * q + 1) * 128) = make_uint4(wx[4], wx[5], wx[6], wx[7]);
            if (16 * q < d)
                *reinterpret_cast<uint4 *>(xr + (G.JB / 8 + 2 * q) * 128) = make_uint4(w2[0], w2[1], w2[2], w2[3]);
            if (16 * q + 8 < d)
                *reinterpret_cast<uint4 *>(xr + (G.JB / 8 + 2 * q + 1) * 128) = make_uint4(w2[4], w2[5], w2[6], w2[7]);
            if (PK > 0 && 8 * q + 8 > PK / 2 && 8 * q < PK / 2) {  // the chunk holding the last a1 pairs
#pragma unroll
                for (int t = 0; t < 8; ++t)
                    if (8 * q + t < PK / 2) a2w[PK / 2 + 1 + t] = w1[t];  // parked past the a2 pairs
            }
        }
    }
    if (PK > 0) {  // words [8 (PK/2 / 8), K1 / 2): remaining a1 pairs, a2 pairs, augmentation, zeros
        constexpr int H = PK / 2, W0 = H / 8 * 8, K1W = (2 * PK + 3 + 15) / 16 * 8;
#pragma unroll
        for (int w0 = W0; w0 < K1W; w0 += 8) {
            uint32_t v[8];
#pragma unroll
            for (int t = 0; t < 8; ++t) {
                const int w = w0 + t;
                v[t] = w < H ? a2w[H + 1 + (w - W0)] : (w < 2 * H ? a2w[w - H] : (w == 2 * H ? 0x3F803F80u : (w == 2 * H + 1 ? 0x3F80u : 0u)));
            }
            tmem_st8u(ta + w0, v);
        }
    }
    return nrm;
}

template <int NC, int DT>
__global__ void __launch_bounds__(kKmThreads, 1)
kmeans_tc_kernel(const float *__restrict__ pts, int64_t n, int d_rt, int NR, int NX, const float *__restrict__ cen,
                 int k, const int32_t *__restrict__ prev, int32_t *__restrict__ membership, int64_t rows_per_cta,
                 float *partials, int *pcounts, unsigned *ticket, unsigned long long *gdelta, float *sums,
                 int32_t *counts, float *new_cen, int64_t *delta_out) {
    extern __shared__ __align__(1024) unsigned char smem_raw[];
    unsigned char *smem =
        reinterpret_cast<unsigned char *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int d = DT > 0 ? DT : d_rt;  // DT > 0: the width is a compile-time constant (C3 / C5: 34)
    long long *const trace = (int)blockIdx.x == g_km_trace_cta ? g_km_trace : nullptr;  // debug tracing (normally null)
    const int skip = g_km_skip;                                        // debug timing switches (0)
    constexpr bool EVEN = DT > 0 && DT % 2 == 0;
    constexpr int PKD = EVEN ? DT : 0;  // packed MMA1 K layout (compile-time even d)
    const KmGeom G(d);
    const int K1 = PKD > 0 ? (2 * PKD + 3 + 15) / 16 * 16 : 2 * G.KP;  // MMA1 K
    constexpr int N1 = 2 * NC;  // MMA1 N: (centre, b piece)
    // ---- shared memory carve-up
    const uint32_t raw_bytes = (uint32_t)(kKmRows * d * 4);
    const uint32_t raw_slot = (raw_bytes + 1023u) & ~1023u;
    const uint32_t x2_bytes = (uint32_t)G.x2_bytes();
    constexpr uint32_t oh_bytes = NC / 8 * 2048;           // [centre group][16 row chunks][8 x 16 B]
    const uint32_t LB2 = (uint32_t)(G.NG * 128);           // MMA2 A: K-group (8 rows) stride
    const uint32_t SB1 = (uint32_t)(2 * G.KP / 8 * 128);  // MMA1 B: n-group stride (room for K1 <= 2 KP)
    unsigned char *raw = smem;                              // [NR][raw_slot]
    unsigned char *x2 = raw + NR * raw_slot;                // [NX][x2_bytes] + 1 KB (MMA2 M read-beyond)
    unsigned char *oh = x2 + NX * x2_bytes + 1024;          // [NX][oh_bytes]
    unsigned char *b1 = oh + NX * oh_bytes;                 // [N1/8][K1/8][8 x 16 B]
    float *cen_s = reinterpret_cast<float *>(b1 + (N1 / 8) * SB1);  // [NC][kKmMaxD]
    KmBars &B = *reinterpret_cast<KmBars *>(cen_s + NC * kKmMaxD);
    float *s_acc = reinterpret_cast<float *>(&B + 1);  // [128][NC]

    const int64_t i0 = (int64_t)blockIdx.x * rows_per_cta;
    const int64_t i1 = i0 + rows_per_cta < n ? i0 + rows_per_cta : n;
    const int64_t nrows = i1 > i0 ? i1 - i0 : 0;
    const int nfull = (int)(nrows / kKmRows);
    const int ns = nfull + ((nrows % kKmRows) ? 1 : 0);
    const int nseg2 = (ns + kKmSeg - 1) / kKmSeg;

    // ---- setup: barriers, TMEM, centre operand, zeroed MMA2 operands
    if (tid == 0) {
        for (int s = 0; s < NR; ++s) {
            mbar_init(&B.raw_full[s], 1);
            mbar_init(&B.raw_empty[s], 4);
        }
        for (int s = 0; s < kKmNA; ++s) {
            mbar_init(&B.a1full[s], 128);  // every convert thread (its |x|^2 store and TMEM rows)
            mbar_init(&B.d1full[s], 1);
            mbar_init(&B.slotfree[s], 128);  // every decide thread (its D1 row and |x|^2 read)
        }
        for (int s = 0; s < NX; ++s) {
            mbar_init(&B.ohfull[s], 4);
            mbar_init(&B.x2free[s], 1);
        }
        for (int s = 0; s < 2; ++s) {
            mbar_init(&B.d2full[s], 1);
            mbar_init(&B.d2free[s], 4);
        }
        fence_mbar_init();
    }
    if (warp == kKmWarpMma) {  // the MMA warp owns the TMEM allocation
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(km_smem(&B.tmem_base)),
                     "r"(512)
                     : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    for (int e = tid; e < NC * kKmMaxD; e += kKmThreads) {
        const int c = e / kKmMaxD, j = e - c * kKmMaxD;
        cen_s[e] = (c < k && j < d) ? cen[c * d + j] : 0.f;
    }
    for (int e = tid; e < (int)((NX * (x2_bytes + oh_bytes) + 1024) / 16); e += kKmThreads)
        reinterpret_cast<uint4 *>(x2)[e] = make_uint4(0u, 0u, 0u, 0u);
    for (int e = tid; e < kKmNXMax * kKmRows; e += kKmThreads) (&B.ohpos[0][0])[e] = -1;
    __syncthreads();
    // B1[n][k], K-major no swizzle: n < NC is centre n with the b1 piece of -2c and the |c|^2
    // pieces q1 q2 q3 in columns d, d+1, d+2 of the a1 half; n >= NC is centre n - NC with the b2
    // piece.  The a2 half of K (k >= KP) repeats the b piece without |c|^2.  Padding centres have
    // |c|^2 = 2^100 (finite: 0 * it stays 0), so they are never candidates.
    for (int e = tid; e < N1 * K1; e += kKmThreads) {
        const int nn = e / K1, kk = e - nn * K1;
        const int c = nn < NC ? nn : nn - NC, piece = nn < NC ? 0 : 1;
        // the x column (or augmentation slot) this K index multiplies
        int j, aug;
        if (PKD > 0) {
            j = kk < 2 * d ? (kk < d ? kk : kk - d) : -1;
            aug = kk >= 2 * d && kk <= 2 * d + 2 ? kk - 2 * d : -1;
        } else {
            const int jj = kk < G.KP ? kk : kk - G.KP;
            j = jj < d ? jj : -1;
            aug = (kk < G.KP && jj >= d && jj <= d + 2) ? jj - d : -1;
        }
        float v = 0.f;
        if (j >= 0) {
            const float b = c < k ? -2.f * cen_s[c * kKmMaxD + j] : 0.f;
            const float p1 = bfr(b);
            v = piece == 0 ? p1 : bfr(__fsub_rn(b, p1));
        } else if (aug >= 0 && piece == 0) {
            float c2 = 0x1p100f;
            if (c < k) {
                double sq = 0.0;
                for (int q = 0; q < d; ++q) sq += (double)cen_s[c * kKmMaxD + q] * (double)cen_s[c * kKmMaxD + q];
                c2 = (float)sq;
            }
            const float q1 = bfr(c2), q2 = bfr(__fsub_rn(c2, q1)), q3 = bfr(__fsub_rn(__fsub_rn(c2, q1), q2));
            v = aug == 0 ? q1 : (aug == 1 ? q2 : q3);
        }
        *reinterpret_cast<__nv_bfloat16 *>(b1 + (nn >> 3) * SB1 + (kk >> 3) * 128 + (nn & 7) * 16 + (kk & 7) * 2) =
            __float2bfloat16_rn(v);
    }
    if (tid < 32) {
        float m = 0.f;
        for (int c = lane; c < k; c += 32) {
            float sq = 0.f;
            for (int q = 0; q < d; ++q) sq = __fmaf_rn(cen_s[c * kKmMaxD + q], cen_s[c * kKmMaxD + q], sq);
            m = fmaxf(m, sq);
        }
        for (int o = 16; o; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
        if (lane == 0) B.cmax2 = m * 1.0001f;
    }
    fence_proxy_async();  // operands written by threads: visible to the tensor core
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = B.tmem_base;
    // TMEM columns: D1 slots [0, NA NC) (both b pieces accumulate into the same NC columns), D2
    // buffers (2 NC), A slots (KA each), D2 running totals (packed layout): 5 32 + 64 + 5 40 + 32 <= 512
    // A slots of KA columns: K1 / 2 with the packed layout (40 at d = 34), else KP; with the packed
    // layout the D2 running totals take the 32 columns after the A slots (TMEM, not shared memory)
    const int KA = PKD > 0 ? K1 / 2 : G.KP;
    const uint32_t tD1 = tmem, tD2 = tmem + kKmNA * NC, tA = tD2 + 2 * NC, tT = tA + kKmNA * KA;

    float *s_part = reinterpret_cast<float *>(x2);  // [128][NC] CTA partial (after the loop)
    if (warp < kKmWarpDecide) {
        // =============================== convert: row r -> bf16 pieces a1 = bf16(x), a2 = bf16(x - a1)
        // (x = a1 + a2 + O(2^-18 |x|)) in TMEM (MMA1 A, K-major) and shared memory (MMA2 A, MN-major)
        const int g = warp >> 2, wl = warp & 3, r = wl * 32 + lane;
        const uint32_t t_lane = (uint32_t)(wl * 32) << 16;
        const int qd = d >> 4;  // chunks of 16 columns that hold only data
        for (int s = g; s < ns; s += kKmCv) {
            const int64_t r0 = i0 + (int64_t)s * kKmRows;
            const bool full = s < nfull;
            const int nv = full ? kKmRows : (int)(i1 - r0);
            const bool valid = r < nv;
            const float *src;
            KM_TRACE(s, 0);
            if (full) {
                km_wait(&B.raw_full[s % NR], (unsigned)((s / NR) & 1));
                src = reinterpret_cast<const float *>(raw + (s % NR) * raw_slot) + (size_t)r * d;
            } else {
                src = pts + (r0 + (valid ? r : 0)) * d;
            }
            KM_TRACE(s, 12);
            const int sa = s % kKmNA, sx = s % NX;
            if (s >= kKmNA) km_wait(&B.slotfree[sa], (unsigned)(((s / kKmNA) - 1) & 1));  // decide read D1
            KM_TRACE(s, 13);
            if (s >= NX) km_wait(&B.x2free[sx], (unsigned)(((s / NX) - 1) & 1));         // MMA2 read X
            tc_fence_after();
            const uint32_t ta = tA + t_lane + (uint32_t)(sa * KA);
            unsigned char *xr = x2 + sx * x2_bytes + (r >> 3) * LB2 + (r & 7) * 16;
            KM_TRACE(s, 1);
            float nrm;
            if (full)
                nrm = km_convert_row<true, EVEN, PKD>(src, d, true, G, qd, ta, xr, skip);
            else
                nrm = km_convert_row<false, EVEN, PKD>(src, d, valid, G, qd, ta, xr, skip);
            B.nrm[sa][r] = nrm;
            asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
            fence_proxy_async();
            tc_fence_before();
            km_arrive(&B.a1full[sa]);
            __syncwarp();
            if (lane == 0 && full) km_arrive(&B.raw_empty[s % NR]);
            KM_TRACE(s, 2);
        }
    } else if (warp < kKmWarpProd) {
        // =============================== decide: candidates from the tensor-core ranking, exact R18
        // for near-ties; one-hot MMA2 operand; membership; delta; D2 buffers -> registers
        const int dg = (warp - kKmWarpDecide) >> 2, wl = warp & 3, r = wl * 32 + lane;
        const uint32_t t_lane = (uint32_t)(wl * 32) << 16;
        const float cmax2 = B.cmax2;
        float *acc_tot = s_acc + r;  // this thread's M row of the D2 totals (group 0): [c][128], conflict-free
        if (dg == 0) {
            if constexpr (PKD > 0) {  // totals in TMEM lane r, columns tT..tT+31
                float z[32];
#pragma unroll
                for (int c = 0; c < 32; ++c) z[c] = 0.f;
                tmem_st32(tT + t_lane, z);
                asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
            } else {
                for (int c = 0; c < NC; ++c) acc_tot[c * kKmRows] = 0.f;
            }
        }
        unsigned wdelta = 0;
        int flushed = 0;
        auto flush = [&]() {
            const int b2 = flushed & 1;
            km_wait(&B.d2full[b2], (unsigned)((flushed >> 1) & 1));
            tc_fence_after();
            float v[32];
            tmem_ld32(tD2 + t_lane + (uint32_t)(b2 * NC), v);
            if constexpr (PKD > 0) {
                float tt[32];
                tmem_ld32(tT + t_lane, tt);
#pragma unroll
                for (int c = 0; c < NC; ++c) tt[c] = __fadd_rn(tt[c], v[c]);
                tmem_st32(tT + t_lane, tt);
                asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
            } else {
#pragma unroll
                for (int c = 0; c < NC; ++c) acc_tot[c * kKmRows] = __fadd_rn(acc_tot[c * kKmRows], v[c]);
            }
            tc_fence_before();
            __syncwarp();
            if (lane == 0) km_arrive(&B.d2free[b2]);
            ++flushed;
        };
        for (int s = dg; s < ns; s += kKmDc) {
            const int64_t r0 = i0 + (int64_t)s * kKmRows;
            const int nv = s < nfull ? kKmRows : (int)(i1 - r0);
            const bool valid = r < nv;
            const int sa = s % kKmNA, sx = s % NX;
            const int pv = (prev && valid) ? __ldg(prev + r0 + r) : 0;  // in flight during the wait
            KM_TRACE(s, 3);
            km_wait(&B.d1full[sa], (unsigned)((s / kKmNA) & 1));
            km_wait(&B.a1full[sa], (unsigned)((s / kKmNA) & 1));  // (complete: orders the |x|^2 store)
            tc_fence_after();
            float dd[NC];
            {
                float v[32];  // (NC = 16: the upper 16 columns belong to the next slot, unused)
                tmem_ld32(tD1 + t_lane + (uint32_t)(sa * NC), v);
#pragma unroll
                for (int c = 0; c < NC; ++c) dd[c] = v[c];
            }
            const float nrm = B.nrm[sa][r];
            KM_TRACE(s, 4);
            tc_fence_before();
            km_arrive(&B.slotfree[sa]);
            float m1 = fminf(dd[0], dd[1]);
#pragma unroll
            for (int c = 2; c + 1 < NC; c += 2) m1 = fmin3(m1, dd[c], dd[c + 1]);
            const float thr = m1 + 2.f * 0x1p-14f * (nrm * 1.001f + cmax2);
            unsigned mask = 0;
#pragma unroll
            for (int c = 0; c < NC; ++c) {
                uint32_t le;
                asm("set.le.u32.f32 %0, %1, %2;" : "=r"(le) : "f"(dd[c]), "f"(thr));
                mask |= le & (1u << c);
            }
            int key = __ffs(mask) - 1;
            if ((mask & (mask - 1)) && valid) {  // several candidates: E in R18's exact f32 order
                const float *xgl = pts + (r0 + r) * d;
                float best = km_exact(xgl, cen_s + key * kKmMaxD, d);
                for (unsigned b = mask & (mask - 1); b; b &= b - 1) {
                    const int cc = __ffs(b) - 1;
                    const float e = km_exact(xgl, cen_s + cc * kKmMaxD, d);
                    if (e < best) {  // strict <: the first centre wins ties
                        best = e;
                        key = cc;
                    }
                }
            }
            if (valid) {
                if (membership) membership[r0 + r] = key;
                wdelta += (unsigned)(prev && pv != key);
            }
            // one-hot B operand of MMA2 (K-major bf16: [centre group][row chunk][8 x 16 B]); the
            // slot's previous MMA2 is complete (the convert of this stage waited for it)
            unsigned short *ohs = reinterpret_cast<unsigned short *>(oh + sx * oh_bytes);
            int op = B.ohpos[sx][r];
            if (op >= 0) ohs[op] = 0;
            op = valid ? ((key >> 3) * 2048 + (r >> 3) * 128 + (key & 7) * 16 + (r & 7) * 2) / 2 : -1;
            if (valid) ohs[op] = 0x3F80;  // bf16 1.0
            B.ohpos[sx][r] = (short)op;
            fence_proxy_async();
            __syncwarp();
            if (lane == 0) km_arrive(&B.ohfull[sx]);
            KM_TRACE(s, 5);
            // group 0 owns D2: move a finished buffer to the totals once its last MMA2 has completed
            // (tested, never waited for here -- a blocking wait stalled the pipeline every 16 stages)
            if (dg == 0 && flushed < nseg2 && (flushed + 1) * kKmSeg <= s &&
                km_test(&B.d2full[flushed & 1], (unsigned)((flushed >> 1) & 1)))
                flush();
        }
        if (dg == 0)
            while (flushed < nseg2) flush();
        wdelta = __reduce_add_sync(0xffffffffu, wdelta);
        if (lane == 0 && wdelta) atomicAdd(gdelta, (unsigned long long)wdelta);
        // every MMA has completed (the last D2 buffer follows every MMA2): the X slots may hold
        // the partial
        km_bar_sync(1, 4 * kKmDc * 32);
        if (dg == 0) {
            if constexpr (PKD > 0) {
                float tt[32];
                tmem_ld32(tT + t_lane, tt);
#pragma unroll
                for (int c = 0; c < NC; ++c) s_part[r * NC + c] = tt[c];
            } else {
                for (int c = 0; c < NC; ++c) s_part[r * NC + c] = acc_tot[c * kKmRows];
            }
        }
    } else if (warp == kKmWarpProd) {
        // =============================== producer: TMA bulk copies of full stages
        if (lane == 0) {
            for (int s = 0; s < nfull; ++s) {
                const int slot = s % NR;
                if (s >= NR) km_wait(&B.raw_empty[slot], (unsigned)(((s / NR) - 1) & 1));
                mbar_expect_tx(&B.raw_full[slot], raw_bytes);
                km_tma_load(raw + slot * raw_slot, pts + (i0 + (int64_t)s * kKmRows) * d, raw_bytes,
                            &B.raw_full[slot]);
            }
        }
    } else {
        // =============================== MMA issuers: one thread for MMA1, one for MMA2
        constexpr uint32_t id1 = umma_idesc_bf16(NC, 0, 0);  // N = NC: the b1 and b2 pieces in turn
        constexpr uint32_t id2 = umma_idesc_bf16(NC, 1, 0);  // A (X) MN-major, B (one-hot) K-major
        if (warp == kKmWarpMma && lane == 0) {
            const uint32_t b10 = km_smem(b1);
            const int K1S = K1 / 16;  // MMA1 instructions (K = 16 each)
            const uint64_t bdesc0 = umma_desc(b10, 128, SB1);                     // b1 rows n < NC
            const uint64_t bdesc1 = umma_desc(b10 + (uint32_t)(NC / 8) * SB1, 128, SB1);  // b2 rows
            for (int s1 = 0; s1 < ns; ++s1) {
                const int sa = s1 % kKmNA;
                km_wait(&B.a1full[sa], (unsigned)((s1 / kKmNA) & 1));  // (implies the D1 slot is free)
                if (trace) trace[s1 * 16 + 8] = clock64();
                tc_fence_after();
                const uint32_t ta = tA + (uint32_t)(sa * KA), dt = tD1 + (uint32_t)(sa * NC);
                for (int p = 0; p < ((skip & 2) ? 0 : K1S); ++p) {  // 8 TMEM columns (16 bf16) of A each
                    umma_bf16_ts(dt, ta + 8 * p, bdesc0 + (uint64_t)(p * 256 >> 4), id1, p > 0);
                    umma_bf16_ts(dt, ta + 8 * p, bdesc1 + (uint64_t)(p * 256 >> 4), id1, 1);
                }
                if (trace) trace[s1 * 16 + 9] = clock64();
                umma_commit(&B.d1full[sa]);
                if (trace) trace[s1 * 16 + 6] = clock64();
            }
        } else if (warp == kKmWarpMma + 1 && lane == 0) {
            const uint32_t x20 = km_smem(x2), oh0 = km_smem(oh);
            for (int s2 = 0; s2 < ns; ++s2) {
                const int sx = s2 % NX, seg = s2 / kKmSeg, b2 = seg & 1;
                const bool first = (s2 % kKmSeg) == 0;
                km_wait(&B.ohfull[sx], (unsigned)((s2 / NX) & 1));  // (implies MMA1 of the stage is done)
                if (first && seg >= 2) km_wait(&B.d2free[b2], (unsigned)(((seg >> 1) - 1) & 1));
                if (trace) trace[s2 * 16 + 10] = clock64();
                tc_fence_after();
                const uint64_t ad = umma_desc(x20 + sx * x2_bytes, LB2, 128);
                const uint64_t bd = umma_desc(oh0 + sx * oh_bytes, 128, 2048);
                const uint32_t dt = tD2 + (uint32_t)(b2 * NC);
#pragma unroll
                for (int kk = 0; kk < kKmRows / 16; ++kk)  // K = 16 rows per instruction
                    if (!(skip & 1))
                        umma_bf16_ss(dt, ad + (uint64_t)((kk * 2 * LB2) >> 4), bd + (uint64_t)((kk * 256) >> 4), id2,
                                     (first && kk == 0) ? 0u : 1u);
                if (trace) trace[s2 * 16 + 11] = clock64();
                umma_commit(&B.x2free[sx]);
                if (trace) trace[s2 * 16 + 7] = clock64();
                if ((s2 + 1) % kKmSeg == 0 || s2 + 1 == ns) umma_commit(&B.d2full[b2]);
            }
        }
    }
    tc_fence_before();
    __syncthreads();
    if (warp == kKmWarpMma) {
        tc_fence_after();
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(512) : "memory");
    }
    // ---- CTA partial: sums[c][j] = a1 row j + a2 row JB + j; counts = row d
    const int64_t kd = (int64_t)k * d;
    for (int64_t e = tid; e < kd; e += kKmThreads) {
        const int c = (int)(e / d), j = (int)(e - (int64_t)c * d);
        __stcg(partials + blockIdx.x * kd + e, __fadd_rn(s_part[j * NC + c], s_part[(G.JB + j) * NC + c]));
    }
    for (int c = tid; c < k; c += kKmThreads) __stcg(pcounts + blockIdx.x * k + c, (int)s_part[d * NC + c]);
    __shared__ bool last;
    __shared__ int s_cnt[kKmK];
    __syncthreads();
    if (tid == 0) {
        __threadfence();
        last = atomicAdd(ticket, 1u) == gridDim.x - 1;
        if (last) __threadfence();
    }
    __syncthreads();
    if (!last) return;
    const int NCTA = gridDim.x;
    // four interleaved accumulators (a fixed order): ~32 independent L2 loads in flight
    for (int cc = tid; cc < k; cc += kKmThreads) {
        unsigned a0 = 0, a1 = 0, a2 = 0, a3 = 0;
        int q = 0;
#pragma unroll 8
        for (; q + 4 <= NCTA; q += 4) {
            const int *p = pcounts + (int64_t)q * k + cc;
            a0 += (unsigned)__ldcg(p);
            a1 += (unsigned)__ldcg(p + k);
            a2 += (unsigned)__ldcg(p + 2 * k);
            a3 += (unsigned)__ldcg(p + 3 * k);
        }
        for (; q < NCTA; ++q) a0 += (unsigned)__ldcg(pcounts + (int64_t)q * k + cc);
        const unsigned a = a0 + a1 + a2 + a3;
        s_cnt[cc] = (int)a;
        counts[cc] = (int32_t)a;
    }
    __syncthreads();
    for (int64_t e = tid; e < kd; e += kKmThreads) {
        float a0 = 0.f, a1 = 0.f, a2 = 0.f, a3 = 0.f;
        int q = 0;
#pragma unroll 8
        for (; q + 4 <= NCTA; q += 4) {
            const float *p = partials + (int64_t)q * kd + e;
            a0 = __fadd_rn(a0, __ldcg(p));
            a1 = __fadd_rn(a1, __ldcg(p + kd));
            a2 = __fadd_rn(a2, __ldcg(p + 2 * kd));
            a3 = __fadd_rn(a3, __ldcg(p + 3 * kd));
        }
        for (; q < NCTA; ++q) a0 = __fadd_rn(a0, __ldcg(partials + (int64_t)q * kd + e));
        const float a = __fadd_rn(__fadd_rn(a0, a1), __fadd_rn(a2, a3));
        sums[e] = a;
        const int cc = (int)(e / d);
        if (new_cen) new_cen[e] = s_cnt[cc] > 0 ? __fdiv_rn(a, (float)s_cnt[cc]) : cen[e];
    }
    if (tid == 0) {
        if (delta_out) *delta_out = prev ? (int64_t)__ldcg(gdelta) : 0;
        *gdelta = 0;
        atomicExch(ticket, 0u);
    }
}

static size_t km_smem_bytes(int64_t d, int NC, int NR, int NX, bool pk) {
    const KmGeom G((int)d);
    const size_t raw_slot = align_up((size_t)kKmRows * d * 4, 1024);
    const size_t oh = (size_t)NC / 8 * 2048;
    const size_t b1 = (size_t)(2 * NC / 8) * (2 * G.KP / 8 * 128);
    return 1024 + NR * raw_slot + NX * ((size_t)G.x2_bytes() + oh) + 1024 + b1 + (size_t)NC * kKmMaxD * 4 +
           sizeof(KmBars) + (pk ? 0 : (size_t)kKmRows * NC * 4);  // (pk: the D2 totals live in TMEM)
}
// deepest rings that fit the 227 KB opt-in limit (+ the static shared words): X slots first
static void km_rings(int64_t d, int NC, bool pk, int &NR, int &NX) {
    if (const char *e = getenv("FUTSEG_KM_RINGS")) {  // "NX,NR": ring-depth experiments
        if (sscanf(e, "%d,%d", &NX, &NR) == 2 && NX >= 2 && NX <= kKmNXMax && NR >= 2 && NR <= kKmRing &&
            km_smem_bytes(d, NC, NR, NX, pk) + 2048 <= 227 * 1024)
            return;
    }
    // X slots first (the X-slot cycle convert -> MMA1 -> decide -> MMA2 is the critical loop),
    // then raw slots (3 measured as fast as 4; 2 is slower)
    for (NX = kKmNXMax; NX >= 2; --NX)
        for (NR = kKmRing; NR >= 3; --NR)
            if (km_smem_bytes(d, NC, NR, NX, pk) + 2048 <= 227 * 1024) return;
    NR = 2;
    NX = 2;
}
static int64_t km_grid(int64_t n) {
    const int64_t stages = ceil_div(n, kKmRows);
    int64_t g = sm_count();
    if (stages < g) g = stages;
    return g < 1 ? 1 : g;
}

size_t kmeans_ws(int64_t n, int64_t d, int64_t k) {
    const int64_t G = (int64_t)sm_count();  // >= km_grid(n)
    (void)n;
    return kWsHeader + align_up((size_t)G * k * d * 4, 256) + align_up((size_t)G * k * 4, 256);
}

template <int NC, int DT>
static fs_status km_launch(const float *pts, int64_t n, int d, const float *cen, int k, const int32_t *prev,
                           int32_t *membership, float *sums, int32_t *counts, float *new_cen, int64_t *delta,
                           void *ws, cudaStream_t st) {
    const int64_t G = km_grid(n);
    const int64_t rows = ceil_div(ceil_div(n > 0 ? n : 1, G), kKmRows) * kKmRows;  // whole stages per CTA
    char *w = (char *)ws;
    unsigned long long *gdelta = (unsigned long long *)(w + kWsCount2);  // zero between calls (header)
    float *parts = (float *)(w + kWsHeader);
    int *pcnt = (int *)(w + kWsHeader + align_up((size_t)G * k * d * 4, 256));
    int NR, NX;
    constexpr bool pk = DT > 0 && DT % 2 == 0;
    km_rings(d, NC, pk, NR, NX);
    {   // debug switches (tools/km_trace.py, tools/km_skip.py): set once per process and device,
        // only when requested (the device globals default to off: no copies on the product path)
        static const char *e = getenv("FUTSEG_KM_TRACE");
        static const int skip = getenv("FUTSEG_KM_SKIP") ? atoi(getenv("FUTSEG_KM_SKIP")) : 0;
        static long long *tr = nullptr;
        static unsigned done_dev = 0;
        int dev = 0;
        cudaGetDevice(&dev);
        if ((e || skip) && dev < 32 && !(done_dev & (1u << dev))) {
            if (e && !tr) cudaMalloc(&tr, 16 * 8 * 8192);
            long long *p = e ? tr : nullptr;
            const int cta = e ? atoi(e) : 0;
            cudaMemcpyToSymbol(g_km_trace, &p, sizeof(p));
            cudaMemcpyToSymbol(g_km_trace_cta, &cta, sizeof(cta));
            cudaMemcpyToSymbol(g_km_skip, &skip, sizeof(skip));
            done_dev |= 1u << dev;
        }
    }
    const size_t smem = km_smem_bytes(d, NC, NR, NX, pk);
    auto kern = kmeans_tc_kernel<NC, DT>;
    cudaFuncSetAttribute((const void *)kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    kern<<<(unsigned)G, kKmThreads, smem, st>>>(pts, n, d, NR, NX, cen, k, prev, membership, rows, parts, pcnt,
                                                 (unsigned *)(w + kWsTicket), gdelta, sums, counts, new_cen, delta);
    return launch_status();
}

// FUTSEG_KM_TRACE: copy CTA 0's stage stamps to the host (tools/km_trace.py)
extern "C" int fs_debug_km_trace(long long *host, int nstages) {
    long long *p = nullptr;
    if (cudaMemcpyFromSymbol(&p, g_km_trace, sizeof(p)) != cudaSuccess || !p) return 1;
    return cudaMemcpy(host, p, (size_t)nstages * 16 * 8, cudaMemcpyDeviceToHost) == cudaSuccess ? 0 : 1;
}

fs_status kmeans_run(const float *pts, int64_t n, int64_t d, const float *cen, int64_t k, const int32_t *prev,
                     int32_t *membership, float *sums, int32_t *counts, float *new_cen, int64_t *delta, void *ws,
                     cudaStream_t st) {
    // d = 34 (the kdd_cup width of C3 / C5) is compiled with the width known; others at run time
    if (k <= 16)
        return d == 34 ? km_launch<16, 34>(pts, n, (int)d, cen, (int)k, prev, membership, sums, counts, new_cen, delta,
                                           ws, st)
                       : km_launch<16, 0>(pts, n, (int)d, cen, (int)k, prev, membership, sums, counts, new_cen, delta,
                                          ws, st);
    return d == 34 ? km_launch<32, 34>(pts, n, (int)d, cen, (int)k, prev, membership, sums, counts, new_cen, delta, ws,
                                       st)
                   : km_launch<32, 0>(pts, n, (int)d, cen, (int)k, prev, membership, sums, counts, new_cen, delta, ws,
                                      st);
}

// new centres from (already combined) sums and counts: the last step of the iteration
// when the sums are reduced across GPUs first (dist.kmeans_step); R19 for empty clusters
__global__ void kmeans_finish_kernel(const float *sums, const int32_t *counts, const float *cen, int64_t k, int64_t d,
                                     float *new_cen) {
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < k * d; e += (int64_t)gridDim.x * blockDim.x) {
        const int32_t c = counts[e / d];
        new_cen[e] = c > 0 ? __fdiv_rn(sums[e], (float)c) : cen[e];
    }
}

fs_status kmeans_finish_run(const float *sums, const int32_t *counts, const float *cen, int64_t k, int64_t d,
                            float *new_cen, cudaStream_t st) {
    const int64_t kd = k * d;
    kmeans_finish_kernel<<<(unsigned)(kd > 0 ? ceil_div(kd, 256) : 1), 256, 0, st>>>(sums, counts, cen, k, d, new_cen);
    return launch_status();
}

}  // namespace fs
