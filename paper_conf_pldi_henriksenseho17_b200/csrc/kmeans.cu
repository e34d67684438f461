// kmeans.cu -- NEXT-1: one fused iteration of Rodinia's K-means (Sec. 2.4,
// L445-531; L1628-1649; fusion F6 L1075-1090: the assignment map is fused into the
// stream_red that computes the new centres, so the membership array never has to be
// re-read and the points are read once).
//
//   membership[i] = argmin_c E(i, c), first c on ties            (readings R3, R18)
//   E(i, c)       = sum_j (x_ij - c_cj)^2, f32, j in order, acc = fma(t, t, acc)
//   sums, counts  = stream_red (map(+)) over the new membership  (Fig 4c)
//   new_centres   = sums / counts; an empty cluster keeps its centre     (R19)
//   delta         = #{ i : membership[i] != prev[i] }  (Rodinia's convergence test)
//
// B200 design.  The distance computation is the one dense contraction on the path
// ([n][d] points x [d][k] centres), so it runs on the tensor cores: warp-level
// mma.sync m16n8k8 TF32 computes s = x . c for 16 rows x 32 centres per stage, and
// d~_c = |c|^2 - 2 s ranks the centres (|x|^2 is the same for every centre).  TF32
// is not the reading's f32 arithmetic, so the argmin is made EXACT by a bound: with
// both operands rounded to TF32 (cvt.rna, 2^-11 relative each),
//     | (E(i,c) - |x|^2) - d~_c |  <=  delta_c = 2^-9 (1 + 2^-7) |x| |c| + 2^-17 (|x| + |c|)^2
// (input rounding of the 2 x.c term, plus the f32 rounding of E itself and of the
// accumulation, generously).  Every centre with d~_c - delta_c <= min_c' (d~_c' +
// delta_c') is a candidate; the true argmin of E is always one.  A row with one
// candidate is decided; a row with several re-evaluates E exactly, in the reading's
// f32 order, for its candidates only (CUDA cores, from the staged row).  Rows are
// streamed through a per-warp TMA ring (as stream_red), the row norms come from the
// A-fragment loads, and the decided keys feed the stream_red accumulation of the same
// stage (lane-private shared-memory columns 0..31, cluster-owner registers for
// columns 32..d-1).  Chunk results combine warp -> CTA -> last CTA, which also
// divides by the counts.
#include "internal.cuh"

namespace fs {

constexpr int kKmThreads = 256;
constexpr int kKmWarps = kKmThreads / 32;
constexpr int kKmRS = 16;      // rows per stage = one m16 tile
constexpr int kKmStages = 2;
constexpr int kKmK = 32;       // max clusters (4 n-tiles of 8)
constexpr int kKmNT = kKmK / 8;
constexpr int kKmMaxD = 40;    // 5 k-steps of 8
constexpr int kKmXR = kKmMaxD - 32;  // extra columns (32..d-1) held by the cluster-owner lane
constexpr int kKmPairs = 128;        // per-warp scratch of (row, candidate) pairs for exact re-evaluation

__device__ __forceinline__ uint32_t to_tf32(float x) {
    uint32_t r;
    asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(r) : "f"(x));
    return r;
}

__device__ __forceinline__ void mma_tf32(float (&c)[4], uint32_t a0, uint32_t a1, uint32_t a2, uint32_t a3,
                                         uint32_t b0, uint32_t b1) {
    asm volatile(
        "mma.sync.aligned.m16n8k8.row.col.f32.tf32.tf32.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
        "{%0,%1,%2,%3};"
        : "+f"(c[0]), "+f"(c[1]), "+f"(c[2]), "+f"(c[3])
        : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
}

struct KmShared {  // per-CTA, after the per-warp regions
    float cen[kKmK * kKmMaxD];  // centres (f32, as given), rows >= k unused
    float csq[kKmK];            // |c|^2 (+inf for padding centres)
    float cn[kKmK];             // |c|
};

// E(x, c) exactly as reading R18 / the oracle: f32, j in order, one rounding per fma.
__device__ __forceinline__ float km_exact(const float *x, const float *c, int d) {
    float acc = 0.f;
    for (int j = 0; j < d; ++j) {
        const float t = __fsub_rn(x[j], c[j]);
        acc = __fmaf_rn(t, t, acc);
    }
    return acc;
}

template <int KS, int XR>
__global__ void __launch_bounds__(kKmThreads, 2)
kmeans_step_kernel(const float *__restrict__ pts, int64_t n, int d, const float *__restrict__ cen, int k,
                   const int32_t *__restrict__ prev, int32_t *__restrict__ membership, int64_t rows_per_warp,
                   float *partials, int *pcounts, unsigned *ticket, unsigned long long *gdelta, float *sums,
                   int32_t *counts, float *new_cen, int64_t *delta_out) {
    extern __shared__ __align__(128) unsigned char smem[];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int g = lane >> 2, t = lane & 3;
    const int XW = d > 32 ? d - 32 : 0;
    const unsigned vbytes = (unsigned)(kKmRS * d * 4);
    const unsigned slot = vbytes + kKmRS * 4;
    const size_t warp_bytes = (size_t)kKmStages * slot + kKmStages * 8 + (size_t)(kKmK + 1) * 32 * 4 + kKmPairs * 8;
    unsigned char *wbase = smem + (size_t)warp * warp_bytes;
    unsigned char *ring = wbase;
    uint64_t *bars = reinterpret_cast<uint64_t *>(wbase + kKmStages * slot);
    float *s_acc = reinterpret_cast<float *>(wbase + kKmStages * slot + kKmStages * 8);  // [K+1][32]
    unsigned *s_pair = reinterpret_cast<unsigned *>(s_acc + (kKmK + 1) * 32);          // [kKmPairs]
    float *s_e = reinterpret_cast<float *>(s_pair + kKmPairs);                          // [kKmPairs]
    KmShared &sh = *reinterpret_cast<KmShared *>(smem + (size_t)kKmWarps * warp_bytes);

    // ---- centres: shared copy, norms, TF32 B fragments (k permuted: logical t <-> column 2t,
    //      logical t+4 <-> column 2t+1 of each 8-column block, so A loads are column pairs)
    for (int e = threadIdx.x; e < kKmK * kKmMaxD; e += kKmThreads) {
        const int c = e / kKmMaxD, j = e - c * kKmMaxD;
        sh.cen[e] = (c < k && j < d) ? cen[c * d + j] : 0.f;
    }
    __syncthreads();
    if (threadIdx.x < kKmK) {
        const int c = threadIdx.x;
        float s = 0.f;
        for (int j = 0; j < d; ++j) s = __fmaf_rn(sh.cen[c * kKmMaxD + j], sh.cen[c * kKmMaxD + j], s);
        sh.csq[c] = c < k ? s : __int_as_float(0x7f800000);
        sh.cn[c] = c < k ? sqrtf(s) : 0.f;
    }
    for (int e = lane; e < (kKmK + 1) * 32; e += 32) s_acc[e] = 0.f;
    uint32_t bf[kKmNT][KS][2];
#pragma unroll
    for (int nt = 0; nt < kKmNT; ++nt)
#pragma unroll
        for (int ks = 0; ks < KS; ++ks) {
            const float *cr = sh.cen + (nt * 8 + g) * kKmMaxD + ks * 8 + 2 * t;
            bf[nt][ks][0] = to_tf32(cr[0]);
            bf[nt][ks][1] = to_tf32(cr[1]);
        }
    __syncthreads();
    // this thread's 8 centres (2 per n-tile): norms for the bound
    float ccsq[kKmNT][2], cmax = 0.f;
#pragma unroll
    for (int nt = 0; nt < kKmNT; ++nt)
#pragma unroll
        for (int h = 0; h < 2; ++h) ccsq[nt][h] = sh.csq[nt * 8 + 2 * t + h];
    for (int cc = 0; cc < k; ++cc) cmax = fmaxf(cmax, sh.cn[cc]);
    cmax *= 1.0001f;

    const int64_t gw = (int64_t)blockIdx.x * kKmWarps + warp;
    const int64_t i0 = gw * rows_per_warp;
    const int64_t i1 = i0 + rows_per_warp < n ? i0 + rows_per_warp : n;
    const int64_t nfull = i1 > i0 ? (i1 - i0) / kKmRS : 0;
    const int nst = (int)nfull + ((i1 > i0 && (i1 - i0) % kKmRS) ? 1 : 0);  // + one partial stage
    if (lane == 0) {
#pragma unroll
        for (int s = 0; s < kKmStages; ++s) mbar_init(bars + s, 1);
        fence_mbar_init();
        for (int s = 0; s < kKmStages && s < nfull; ++s) {
            mbar_expect_tx(bars + s, vbytes);
            tma_load_1d(ring + s * slot, pts + (i0 + (int64_t)s * kKmRS) * d, vbytes, bars + s);
        }
    }
    __syncwarp();
    float xa[XR > 0 ? XR : 1];
#pragma unroll
    for (int e = 0; e < (XR > 0 ? XR : 1); ++e) xa[e] = 0.f;
    unsigned wcnt = 0, wdelta = 0;
    int s = 0;
    unsigned phase = 0;
    constexpr float kE1 = 1.0f / 512.0f * (1.0f + 1.0f / 128.0f), kE2 = 1.0f / 131072.0f;
    for (int c = 0; c < nst; ++c) {
        const int64_t r0 = i0 + (int64_t)c * kKmRS;
        const bool full = c < nfull;
        const int nv = full ? kKmRS : (int)(i1 - r0);
        float *sv = reinterpret_cast<float *>(ring + s * slot);
        int *sk = reinterpret_cast<int *>(ring + s * slot + vbytes);
        if (full) {
            mbar_wait(bars + s, phase);
        } else {  // ragged tail of the chunk: plain loads into the (idle) slot, zero padding
            for (int e = lane; e < kKmRS * d; e += 32) sv[e] = e < nv * d ? __ldg(pts + r0 * d + e) : 0.f;
            __syncwarp();
        }
        // ---- assignment: s = x . c on the tensor cores, row norms from the same loads
        float acc[kKmNT][4];
#pragma unroll
        for (int nt = 0; nt < kKmNT; ++nt) acc[nt][0] = acc[nt][1] = acc[nt][2] = acc[nt][3] = 0.f;
        float nx0 = 0.f, nx1 = 0.f;
#pragma unroll
        for (int ks = 0; ks < KS; ++ks) {
            const int c0 = ks * 8 + 2 * t;
            const float x00 = c0 < d ? sv[g * d + c0] : 0.f, x01 = c0 + 1 < d ? sv[g * d + c0 + 1] : 0.f;
            const float x10 = c0 < d ? sv[(g + 8) * d + c0] : 0.f, x11 = c0 + 1 < d ? sv[(g + 8) * d + c0 + 1] : 0.f;
            nx0 = __fmaf_rn(x00, x00, __fmaf_rn(x01, x01, nx0));
            nx1 = __fmaf_rn(x10, x10, __fmaf_rn(x11, x11, nx1));
            const uint32_t a0 = to_tf32(x00), a1 = to_tf32(x10), a2 = to_tf32(x01), a3 = to_tf32(x11);
#pragma unroll
            for (int nt = 0; nt < kKmNT; ++nt) mma_tf32(acc[nt], a0, a1, a2, a3, bf[nt][ks][0], bf[nt][ks][1]);
        }
        nx0 += __shfl_xor_sync(0xffffffffu, nx0, 1);
        nx0 += __shfl_xor_sync(0xffffffffu, nx0, 2);
        nx1 += __shfl_xor_sync(0xffffffffu, nx1, 1);
        nx1 += __shfl_xor_sync(0xffffffffu, nx1, 2);
        nx0 = sqrtf(nx0) * 1.0001f;  // |x| (an upper bound up to f32 rounding)
        nx1 = sqrtf(nx1) * 1.0001f;
        // d~ = |c|^2 - 2 s for rows g, g+8 and centres 8nt + 2t + h; one bound per row with
        // the largest centre norm: candidates are d~_c <= min_c' d~_c' + 2 e(row)
        const float e0 = kE1 * nx0 * cmax + kE2 * (nx0 + cmax) * (nx0 + cmax);
        const float e1 = kE1 * nx1 * cmax + kE2 * (nx1 + cmax) * (nx1 + cmax);
        float dd0[kKmNT][2], dd1[kKmNT][2];
        float u0 = __int_as_float(0x7f800000), u1 = u0;
#pragma unroll
        for (int nt = 0; nt < kKmNT; ++nt)
#pragma unroll
            for (int h = 0; h < 2; ++h) {
                dd0[nt][h] = __fmaf_rn(-2.f, acc[nt][h], ccsq[nt][h]);
                dd1[nt][h] = __fmaf_rn(-2.f, acc[nt][2 + h], ccsq[nt][h]);
                u0 = fminf(u0, dd0[nt][h]);
                u1 = fminf(u1, dd1[nt][h]);
            }
        u0 = fminf(u0, __shfl_xor_sync(0xffffffffu, u0, 1));
        u0 = fminf(u0, __shfl_xor_sync(0xffffffffu, u0, 2));
        u1 = fminf(u1, __shfl_xor_sync(0xffffffffu, u1, 1));
        u1 = fminf(u1, __shfl_xor_sync(0xffffffffu, u1, 2));
        u0 += 2.f * e0;
        u1 += 2.f * e1;
        unsigned m0 = 0, m1 = 0;
#pragma unroll
        for (int nt = 0; nt < kKmNT; ++nt)
#pragma unroll
            for (int h = 0; h < 2; ++h) {
                m0 |= (dd0[nt][h] <= u0 ? 1u : 0u) << (nt * 8 + h);
                m1 |= (dd1[nt][h] <= u1 ? 1u : 0u) << (nt * 8 + h);
            }
        m0 <<= 2 * t;  // this thread's centres are 8nt + 2t + h
        m1 <<= 2 * t;
        m0 |= __shfl_xor_sync(0xffffffffu, m0, 1);
        m0 |= __shfl_xor_sync(0xffffffffu, m0, 2);
        m1 |= __shfl_xor_sync(0xffffffffu, m1, 1);
        m1 |= __shfl_xor_sync(0xffffffffu, m1, 2);
        // lane r < 16 decides row r
        const unsigned ma = __shfl_sync(0xffffffffu, m0, (lane & 7) * 4);
        const unsigned mb = __shfl_sync(0xffffffffu, m1, (lane & 7) * 4);
        const unsigned cm = lane < kKmRS ? (lane < 8 ? ma : mb) : 0u;
        int key = __ffs(cm) - 1;
        // rows with several candidates: E in the reading's exact f32 order, one (row,
        // candidate) pair per lane -- all of the stage's pairs in one 34-step pass
        const unsigned np = (cm & (cm - 1)) ? (unsigned)__popc(cm) : 0u;
        if (__any_sync(0xffffffffu, np)) {
            unsigned incl = np;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const unsigned v = __shfl_up_sync(0xffffffffu, incl, o);
                if (lane >= o) incl += v;
            }
            const unsigned total = __shfl_sync(0xffffffffu, incl, 31);
            if (total <= (unsigned)kKmPairs) {
                unsigned off = incl - np;
                for (unsigned b = np ? cm : 0u; b; b &= b - 1) s_pair[off++] = (lane << 8) | (__ffs(b) - 1);
                __syncwarp();
                for (unsigned p = lane; p < total; p += 32) {
                    const unsigned pr = s_pair[p];
                    s_e[p] = km_exact(sv + (pr >> 8) * d, sh.cen + (pr & 255) * kKmMaxD, d);
                }
                __syncwarp();
                if (np) {  // pairs are in ascending centre order: strict < keeps the first on ties
                    const unsigned o0 = incl - np;
                    float best = s_e[o0];
                    key = (int)(s_pair[o0] & 255);
                    for (unsigned p = o0 + 1; p < incl; ++p)
                        if (s_e[p] < best) {
                            best = s_e[p];
                            key = (int)(s_pair[p] & 255);
                        }
                }
                __syncwarp();
            } else if (np) {  // (rare) too many pairs for the scratch: each row on its own lane
                const float *xr = sv + lane * d;
                float best = km_exact(xr, sh.cen + key * kKmMaxD, d);
                for (unsigned b = cm & (cm - 1); b; b &= b - 1) {
                    const int cc = __ffs(b) - 1;
                    const float e = km_exact(xr, sh.cen + cc * kKmMaxD, d);
                    if (e < best) {
                        best = e;
                        key = cc;
                    }
                }
            }
        }
        if (lane < kKmRS) {
            if (lane >= nv) key = kKmK;  // padding row of the partial stage: trash row
            sk[lane] = key;
            if (lane < nv) {
                if (membership) membership[r0 + lane] = key;
                if (prev) wdelta += (unsigned)(__ldg(prev + r0 + lane) != key);
            }
        }
        __syncwarp();
        // ---- stream_red accumulation of the stage (as stream_red_tma_s_kernel)
        int kr[kKmRS];
#pragma unroll
        for (int q = 0; q < kKmRS / 4; ++q) {
            const int4 v4 = reinterpret_cast<const int4 *>(sk)[q];
            kr[4 * q] = v4.x;
            kr[4 * q + 1] = v4.y;
            kr[4 * q + 2] = v4.z;
            kr[4 * q + 3] = v4.w;
        }
        unsigned B = 0;
#pragma unroll
        for (int r = 0; r < kKmRS; ++r)
            if (kr[r] == lane) B |= 1u << r;
        wcnt += (unsigned)__popc(B);
        float v[kKmRS];
#pragma unroll
        for (int r = 0; r < kKmRS; ++r) v[r] = lane < d ? sv[r * d + lane] : 0.f;
#pragma unroll
        for (int r = 0; r < kKmRS; ++r) {
            float *p = s_acc + kr[r] * 32 + lane;
            *p = __fadd_rn(*p, v[r]);
        }
        if (XR > 0)
            for (unsigned b = B; b; b &= b - 1) {
                const float *xp = sv + (__ffs(b) - 1) * d + 32;
#pragma unroll
                for (int e = 0; e < (XR > 0 ? XR : 1); ++e)
                    if (e < XW) xa[e] = __fadd_rn(xa[e], xp[e]);
            }
        __syncwarp();
        if (full && lane == 0 && c + kKmStages < nfull) {
            fence_proxy_async();
            mbar_expect_tx(bars + s, vbytes);
            tma_load_1d(ring + s * slot, pts + (r0 + (int64_t)kKmStages * kKmRS) * d, vbytes, bars + s);
        }
        if (full && ++s == kKmStages) {
            s = 0;
            phase ^= 1u;
        }
    }
    // ---- chunk results -> CTA (warp order) -> workspace; last CTA -> outputs
    wdelta = __reduce_add_sync(0xffffffffu, wdelta);
    if (lane == 0 && wdelta) atomicAdd(gdelta, (unsigned long long)wdelta);
    __syncthreads();
    float *s_kw = reinterpret_cast<float *>(smem);  // [k][d] CTA sums (reuses warp 0's ring)
    int *s_cnt = reinterpret_cast<int *>(smem + align_up((size_t)kKmK * kKmMaxD * 4, 16));
    // each warp's region is still intact except warp 0's ring: combine through registers
    float colsum[kKmK];  // lane j: column j of every cluster, summed over warps in order
#pragma unroll
    for (int cc = 0; cc < kKmK; ++cc) colsum[cc] = 0.f;
    __syncthreads();
    if (warp == 0) {
        for (int q = 0; q < kKmWarps; ++q) {
            const float *qa = reinterpret_cast<const float *>(smem + (size_t)q * warp_bytes + kKmStages * slot +
                                                              kKmStages * 8);
#pragma unroll
            for (int cc = 0; cc < kKmK; ++cc) colsum[cc] = __fadd_rn(colsum[cc], qa[cc * 32 + lane]);
        }
    }
    __syncthreads();  // warp 0 has read every accumulator; the rings may now be reused
    // extras and counts: per-warp values held by the cluster-owner lanes -> shared, warp order
    float *s_x = reinterpret_cast<float *>(smem + align_up((size_t)kKmK * kKmMaxD * 4, 16) + 256);  // [W][K][XR]
    int *s_wc = reinterpret_cast<int *>(smem + align_up((size_t)kKmK * kKmMaxD * 4, 16) + 256 +
                                        (size_t)kKmWarps * kKmK * kKmXR * 4);  // [W][K]
#pragma unroll
    for (int e = 0; e < kKmXR; ++e) s_x[(warp * kKmK + lane) * kKmXR + e] = e < XR ? xa[e < XR ? e : 0] : 0.f;
    s_wc[warp * kKmK + lane] = (int)wcnt;
    if (warp == 0 && lane < d) {
#pragma unroll
        for (int cc = 0; cc < kKmK; ++cc)
            if (cc < k) s_kw[cc * d + lane] = colsum[cc];
    }
    __syncthreads();
    for (int e = threadIdx.x; e < k * d; e += kKmThreads) {
        const int cc = e / d, j = e - cc * d;
        if (j >= 32) {
            float a = 0.f;
            for (int q = 0; q < kKmWarps; ++q) a = __fadd_rn(a, s_x[(q * kKmK + cc) * kKmXR + (j - 32)]);
            s_kw[e] = a;
        }
    }
    if (threadIdx.x < k) {
        unsigned a = 0;
        for (int q = 0; q < kKmWarps; ++q) a += (unsigned)s_wc[q * kKmK + threadIdx.x];
        s_cnt[threadIdx.x] = (int)a;
    }
    __syncthreads();
    const int64_t kd = (int64_t)k * d;
    for (int64_t e = threadIdx.x; e < kd; e += kKmThreads) __stcg(partials + blockIdx.x * kd + e, s_kw[e]);
    for (int cc = threadIdx.x; cc < k; cc += kKmThreads) __stcg(pcounts + blockIdx.x * k + cc, s_cnt[cc]);
    __shared__ bool last;
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence();
        last = atomicAdd(ticket, 1u) == gridDim.x - 1;
        if (last) __threadfence();
    }
    __syncthreads();
    if (!last) return;
    const int G = gridDim.x;
    // four interleaved accumulators (a fixed order): ~32 independent L2 loads in flight
    for (int cc = threadIdx.x; cc < k; cc += kKmThreads) {
        unsigned a0 = 0, a1 = 0, a2 = 0, a3 = 0;
        int q = 0;
#pragma unroll 8
        for (; q + 4 <= G; q += 4) {
            const int *p = pcounts + (int64_t)q * k + cc;
            a0 += (unsigned)__ldcg(p);
            a1 += (unsigned)__ldcg(p + k);
            a2 += (unsigned)__ldcg(p + 2 * k);
            a3 += (unsigned)__ldcg(p + 3 * k);
        }
        for (; q < G; ++q) a0 += (unsigned)__ldcg(pcounts + (int64_t)q * k + cc);
        const unsigned a = a0 + a1 + a2 + a3;
        s_cnt[cc] = (int)a;
        counts[cc] = (int32_t)a;
    }
    __syncthreads();
    for (int64_t e = threadIdx.x; e < kd; e += kKmThreads) {
        float a0 = 0.f, a1 = 0.f, a2 = 0.f, a3 = 0.f;
        int q = 0;
#pragma unroll 8
        for (; q + 4 <= G; q += 4) {
            const float *p = partials + (int64_t)q * kd + e;
            a0 = __fadd_rn(a0, __ldcg(p));
            a1 = __fadd_rn(a1, __ldcg(p + kd));
            a2 = __fadd_rn(a2, __ldcg(p + 2 * kd));
            a3 = __fadd_rn(a3, __ldcg(p + 3 * kd));
        }
        for (; q < G; ++q) a0 = __fadd_rn(a0, __ldcg(partials + (int64_t)q * kd + e));
        const float a = __fadd_rn(__fadd_rn(a0, a1), __fadd_rn(a2, a3));
        sums[e] = a;
        const int cc = (int)(e / d);
        if (new_cen) new_cen[e] = s_cnt[cc] > 0 ? __fdiv_rn(a, (float)s_cnt[cc]) : cen[e];
    }
    if (threadIdx.x == 0) {
        if (delta_out) *delta_out = prev ? (int64_t)__ldcg(gdelta) : 0;
        *gdelta = 0;
        atomicExch(ticket, 0u);
    }
}

static size_t km_warp_bytes(int64_t d) {
    return (size_t)kKmStages * ((size_t)kKmRS * d * 4 + kKmRS * 4) + kKmStages * 8 + (size_t)(kKmK + 1) * 32 * 4 +
           kKmPairs * 8;
}
static size_t km_smem(int64_t d) {
    const size_t a = (size_t)kKmWarps * km_warp_bytes(d) + sizeof(KmShared);
    // combine scratch (carved from the start of the rings): sums, counts, extras, per-warp counts
    const size_t b = align_up((size_t)kKmK * kKmMaxD * 4, 16) + 256 + (size_t)kKmWarps * kKmK * kKmXR * 4 +
                     (size_t)kKmWarps * kKmK * 4;
    return a > b ? a : b;
}
static int64_t km_grid(int64_t n) {
    int64_t warps = ceil_div(n, 4 * kKmRS);  // at least 4 stages per warp
    const int64_t cap = (int64_t)sm_count() * 2 * kKmWarps;
    if (warps > cap) warps = cap;
    if (warps < 1) warps = 1;
    return ceil_div(warps, kKmWarps);
}

size_t kmeans_ws(int64_t n, int64_t d, int64_t k) {
    const int64_t G = (int64_t)sm_count() * 2;  // >= km_grid(n)
    (void)n;
    return kWsHeader + align_up((size_t)G * k * d * 4, 256) + align_up((size_t)G * k * 4, 256);
}

template <int KS, int XR>
static fs_status km_launch(const float *pts, int64_t n, int d, const float *cen, int k, const int32_t *prev,
                           int32_t *membership, float *sums, int32_t *counts, float *new_cen, int64_t *delta,
                           void *ws, cudaStream_t st) {
    const int64_t G = km_grid(n);
    const int64_t warps = G * kKmWarps;
    int64_t rows = n > 0 ? ceil_div(n, warps) : 0;
    rows = ceil_div(rows, kKmRS) * kKmRS;  // stages start 16-row (64d-byte) aligned
    char *w = (char *)ws;
    unsigned long long *gdelta = (unsigned long long *)(w + kWsCount2);  // zero between calls (header)
    float *parts = (float *)(w + kWsHeader);
    int *pcnt = (int *)(w + kWsHeader + align_up((size_t)G * k * d * 4, 256));
    const size_t smem = km_smem(d);
    cudaFuncSetAttribute((const void *)kmeans_step_kernel<KS, XR>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         (int)smem);
    kmeans_step_kernel<KS, XR><<<(unsigned)G, kKmThreads, smem, st>>>(pts, n, d, cen, k, prev, membership, rows, parts,
                                                                   pcnt, (unsigned *)(w + kWsTicket), gdelta, sums,
                                                                   counts, new_cen, delta);
    return launch_status();
}

fs_status kmeans_run(const float *pts, int64_t n, int64_t d, const float *cen, int64_t k, const int32_t *prev,
                     int32_t *membership, float *sums, int32_t *counts, float *new_cen, int64_t *delta, void *ws,
                     cudaStream_t st) {
#define FS_KM(KS, XR) return km_launch<KS, XR>(pts, n, (int)d, cen, (int)k, prev, membership, sums, counts, new_cen, delta, ws, st)
    if (d <= 8) FS_KM(1, 0);
    if (d <= 16) FS_KM(2, 0);
    if (d <= 24) FS_KM(3, 0);
    if (d <= 32) FS_KM(4, 0);
    if (d <= 34) FS_KM(5, 2);
    if (d <= 36) FS_KM(5, 4);
    if (d <= 40) FS_KM(5, 8);
#undef FS_KM
    return FS_ERR_UNSUPPORTED;
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
