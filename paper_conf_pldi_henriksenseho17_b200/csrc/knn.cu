// knn.cu -- NEXT-2: Rodinia NN's kk nearest neighbours (
// reading R16 in DESIGN.md).
//
// The paper's NN leaves "100 reduce operations for finding the nearest
// neighbors" to be run as 100 argmin reduces (value and index, L1654-1655),
// each excluding the record it found; the benchmark is "dominated by frequent
// launches of short kernels" (L1655-1656).  The kk rounds are, by definition,
// the kk smallest records under the ARGMIN order of reading R3: lexicographic
// (distance, index).  Distances are >= +0 (a square root), so that order is the
// unsigned order of the 64-bit key
//     key = (f32 bits of distance) << 32 | index        (index < 2^32)
// and keys are unique.  So ONE cooperative launch suffices (B200 design, not
// the paper's):
//   A. every CTA streams a contiguous chunk, maps records to keys in registers
//      (the distance map is never materialised) and histograms the top 12 key
//      bits (sign, exponent, 3 mantissa bits of the distance) in shared memory,
//      then adds its histogram into a global one;             -- grid barrier --
//   B. every CTA scans the global histogram to the first bin b* whose
//      cumulative count reaches kk, and appends the keys of its chunk in bins
//      <= b* to a global candidate buffer (about kk plus part of one bin);
//   C. the last CTA (atomic ticket) selects the kk smallest candidates (running
//      list + threshold filter + bitonic sort in shared memory) and writes them
//      in ascending order -- exactly the sequence of the kk argmin rounds --
//      then re-zeroes the histogram and counters for the next call.
#include "internal.cuh"

namespace fs {

constexpr int kKnnThreads = 512;
constexpr int kKnnPer = 4;                             // keys per thread per tile
constexpr int kKnnTile = kKnnThreads * kKnnPer;        // 2048 keys per tile
constexpr int kKnnCap = 8192;                          // shared sort capacity (64 KB of keys)
constexpr int64_t kKnnMaxK = 1024;                     // kk + kKnnTile <= kKnnCap
constexpr unsigned long long kKeyInf = ~0ull;

struct KnnState {
    int m;                  // running list S[0, m), ascending, m <= kk
    int cnt;                // buffered candidates S[m, m + cnt)
    unsigned long long T;   // keys >= T cannot enter (the kk-th smallest so far, or inf)
};

__device__ __forceinline__ unsigned long long knn_key(float d, uint32_t i) {
    return ((unsigned long long)__float_as_uint(d) << 32) | i;
}

// Ascending bitonic sort of S[0, P), P a power of two, whole block.
__device__ void knn_bitonic(unsigned long long *S, int P) {
    for (int k = 2; k <= P; k <<= 1)
        for (int j = k >> 1; j > 0; j >>= 1) {
            for (int t = threadIdx.x; t < (P >> 1); t += kKnnThreads) {
                const int lo = ((t & ~(j - 1)) << 1) | (t & (j - 1)), hi = lo + j;
                const bool up = (lo & k) == 0;
                const unsigned long long a = S[lo], b = S[hi];
                if ((a > b) == up) {
                    S[lo] = b;
                    S[hi] = a;
                }
            }
            __syncthreads();
        }
}

// Sort the running list and the buffer together; keep the kk smallest.
__device__ void knn_flush(unsigned long long *S, KnnState *st, int kk) {
    const int tot = st->m + st->cnt;
    int P = 2;
    while (P < tot) P <<= 1;
    for (int i = tot + threadIdx.x; i < P; i += kKnnThreads) S[i] = kKeyInf;
    __syncthreads();
    knn_bitonic(S, P);
    if (threadIdx.x == 0) {
        st->m = tot < kk ? tot : kk;
        st->cnt = 0;
        st->T = st->m == kk ? S[kk - 1] : kKeyInf;
    }
    __syncthreads();
}

// Offer this thread's kKnnPer keys (valid[u]) to the running selection.
__device__ void knn_push(unsigned long long *S, KnnState *st, int kk, const unsigned long long (&key)[kKnnPer],
                         const bool (&valid)[kKnnPer]) {
    if (st->m + st->cnt + kKnnTile > kKnnCap) knn_flush(S, st, kk);  // block-uniform (read after a barrier)
    const unsigned long long T = st->T;
    const int m0 = st->m;
    __syncthreads();  // every thread has read the state before any append moves st->cnt
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int u = 0; u < kKnnPer; ++u) {
        const bool in = valid[u] && key[u] < T;
        const unsigned mask = __ballot_sync(0xffffffffu, in);
        int off = 0;
        if (mask) {
            if (lane == 0) off = atomicAdd(&st->cnt, __popc(mask));
            off = __shfl_sync(0xffffffffu, off, 0);
        }
        if (in) S[m0 + off + __popc(mask & ((1u << lane) - 1u))] = key[u];
    }
    __syncthreads();
    if (st->m < kk && st->m + st->cnt >= kk) knn_flush(S, st, kk);  // first full list sets T
}

constexpr int kKnnBins = 4096;  // key >> 52: top 12 bits of the distance

struct KnnCtl {          // the workspace's self-resetting control words (zero between calls)
    unsigned *barrier;   // grid barrier arrivals            (kWsCount0)
    unsigned *ticket;    // CTAs done with phase B           (kWsTicket)
    unsigned long long *ncand;  // candidates appended       (kWsCount1)
};

__device__ __forceinline__ unsigned long long knn_record_key(const float *lat, const float *lng, int64_t i, float q0,
                                                             float q1) {
    return knn_key(nn_distance(__ldg(lat + i), __ldg(lng + i), q0, q1), (uint32_t)i);
}

__global__ void __launch_bounds__(kKnnThreads, 1)
knn_kernel(const float *__restrict__ lat, const float *__restrict__ lng, int64_t n, float q0, float q1, int kk,
           int64_t chunk, KnnCtl ctl, unsigned *ghist, unsigned long long *cand, float *out_dist,
           int64_t *out_idx) {
    extern __shared__ __align__(16) unsigned long long S[];
    unsigned *hist = reinterpret_cast<unsigned *>(S);  // phase A/B alias of the sort buffer
    __shared__ KnnState st;
    __shared__ bool last;
    __shared__ unsigned wsum[kKnnThreads / 32];
    __shared__ int bstar;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int64_t i0 = (int64_t)blockIdx.x * chunk;
    const int64_t i1 = i0 + chunk < n ? i0 + chunk : n;
    // ---- A. histogram of the top key bits
    for (int b = tid; b < kKnnBins; b += kKnnThreads) hist[b] = 0;
    __syncthreads();
    for (int64_t b = i0; b < i1; b += kKnnTile) {
#pragma unroll
        for (int u = 0; u < kKnnPer; ++u) {
            const int64_t i = b + u * kKnnThreads + tid;
            if (i < i1) atomicAdd(hist + (int)(knn_record_key(lat, lng, i, q0, q1) >> 52), 1u);
        }
    }
    __syncthreads();
    for (int b = tid; b < kKnnBins; b += kKnnThreads)
        if (hist[b]) atomicAdd(ghist + b, hist[b]);
    // grid barrier (cooperative launch: all CTAs are resident).  The CTA barrier orders the
    // block's writes before thread 0's cumulative gpu-scope fence (one fence per CTA, not
    // one per thread); the acquiring side mirrors it.
    __syncthreads();
    if (tid == 0) {
        __threadfence();
        atomicAdd(ctl.barrier, 1u);
        while (atomicAdd(ctl.barrier, 0u) < gridDim.x) __nanosleep(64);
        __threadfence();
    }
    __syncthreads();
    // ---- B. first bin whose cumulative count reaches kk; append the keys in bins <= b*
    const unsigned need = (unsigned)((int64_t)kk < n ? kk : n);
    constexpr int PER = kKnnBins / kKnnThreads;  // 8 bins per thread, contiguous
    unsigned c[PER], run = 0;
#pragma unroll
    for (int j = 0; j < PER; ++j) {
        c[j] = __ldcg(ghist + tid * PER + j);
        run += c[j];
    }
    unsigned incl = run;  // block-wide inclusive scan of the per-thread totals
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const unsigned t = __shfl_up_sync(0xffffffffu, incl, d);
        if (lane >= d) incl += t;
    }
    if (lane == 31) wsum[warp] = incl;
    if (tid == 0) bstar = kKnnBins - 1;
    __syncthreads();
    unsigned before = incl - run;
    for (int w = 0; w < warp; ++w) before += wsum[w];
    if (need > 0 && before < need && before + run >= need) {  // exactly one thread
        unsigned cum = before;
#pragma unroll
        for (int j = 0; j < PER; ++j) {
            cum += c[j];
            if (cum >= need) {
                bstar = tid * PER + j;
                break;
            }
        }
    }
    __syncthreads();
    const unsigned long long lim = bstar + 1 < kKnnBins ? (unsigned long long)(bstar + 1) << 52 : kKeyInf;  // keys < lim
    for (int64_t b = i0; b < i1; b += kKnnTile) {
#pragma unroll
        for (int u = 0; u < kKnnPer; ++u) {
            const int64_t i = b + u * kKnnThreads + tid;
            const unsigned long long key = i < i1 ? knn_record_key(lat, lng, i, q0, q1) : kKeyInf;
            const bool in = key < lim;
            const unsigned mask = __ballot_sync(0xffffffffu, in);
            unsigned long long off = 0;
            if (mask) {
                if (lane == 0) off = atomicAdd(ctl.ncand, (unsigned long long)__popc(mask));
                off = __shfl_sync(0xffffffffu, off, 0);
            }
            if (in) __stcg(cand + off + __popc(mask & ((1u << lane) - 1u)), key);
        }
    }
    __syncthreads();
    if (tid == 0) {
        __threadfence();
        last = atomicAdd(ctl.ticket, 1u) == gridDim.x - 1;
        if (last) __threadfence();
    }
    __syncthreads();
    if (!last) return;
    // ---- C. the last CTA: the kk smallest candidates, ascending
    if (tid == 0) {
        st.m = 0;
        st.cnt = 0;
        st.T = kKeyInf;
    }
    __syncthreads();
    const int64_t total = (int64_t)__ldcg(ctl.ncand);
    for (int64_t b = 0; b < total; b += kKnnTile) {
        unsigned long long key[kKnnPer];
        bool valid[kKnnPer];
#pragma unroll
        for (int u = 0; u < kKnnPer; ++u) {
            const int64_t e = b + u * kKnnThreads + tid;
            valid[u] = e < total;
            key[u] = valid[u] ? __ldcg(cand + e) : kKeyInf;
        }
        knn_push(S, &st, kk, key, valid);
    }
    if (st.cnt > 0) knn_flush(S, &st, kk);
    for (int i = tid; i < kk; i += kKnnThreads) {
        if (i < st.m) {
            out_dist[i] = __uint_as_float((unsigned)(S[i] >> 32));
            out_idx[i] = (int64_t)(S[i] & 0xffffffffull);
        } else {  // fewer than kk records: the argmin neutral element (R3/R4)
            out_dist[i] = __int_as_float(0x7f800000);
            out_idx[i] = -1;
        }
    }
    for (int b = tid; b < kKnnBins; b += kKnnThreads) ghist[b] = 0;  // leave the workspace reusable
    if (tid == 0) {
        *ctl.barrier = 0;
        *ctl.ticket = 0;
        *ctl.ncand = 0;
    }
}

// workspace body: [candidates: n u64]
size_t knn_ws(int64_t n) { return kWsHeader + align_up((size_t)(n > 0 ? n : 1) * 8, 256); }

fs_status knn_run(const float *lat, const float *lng, int64_t n, float q0, float q1, int64_t kk, float *out_dist,
                  int64_t *out_idx, void *ws, cudaStream_t st) {
    const size_t smem = (size_t)kKnnCap * 8;
    static bool attr = false;
    if (!attr) {
        cudaFuncSetAttribute((const void *)knn_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        attr = true;
    }
    int64_t G = ceil_div(n, kKnnTile);
    const int64_t cap = resident_blocks((const void *)knn_kernel, kKnnThreads, smem);
    if (G > cap) G = cap;
    if (G < 1) G = 1;
    int64_t chunk = n > 0 ? ceil_div(n, G) : 0;
    char *w = (char *)ws;
    // counters and histogram live in the workspace's zero-between-calls header (control
    // words; the 4096 self-resetting ticket slots hold the histogram), reset by the last CTA;
    // the body (candidates) is never assumed zero
    static_assert(kKnnBins == kWsMaxTickets, "histogram = the ticket slots");
    KnnCtl ctl{(unsigned *)(w + kWsCount0), (unsigned *)(w + kWsTicket), (unsigned long long *)(w + kWsCount1)};
    unsigned *ghist = (unsigned *)(w + kWsTickets);
    unsigned long long *cand = (unsigned long long *)(w + kWsHeader);
    int kki = (int)kk;
    void *args[] = {(void *)&lat, (void *)&lng, (void *)&n, (void *)&q0, (void *)&q1, (void *)&kki, (void *)&chunk,
                    (void *)&ctl, (void *)&ghist, (void *)&cand, (void *)&out_dist, (void *)&out_idx};
    if (cudaLaunchCooperativeKernel((const void *)knn_kernel, dim3((unsigned)G), dim3(kKnnThreads), args, smem, st) !=
        cudaSuccess) {
        cudaGetLastError();
        return FS_ERR_CUDA;
    }
    return launch_status();
}

}  // namespace fs
