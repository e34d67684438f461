// common.cuh -- device-side operator table and building blocks shared by the
// libfutseg kernels (sm_100a).  Nothing here is shared with oracle/.
//
// Operator table (include/futseg.h; a binary associative
// operator (+) with neutral element 0(+)):
//   ADD    : wrap-around integer add (unsigned arithmetic), f32 add
//   MIN/MAX: exact; neutral +inf/INT_MAX resp. -inf/INT_MIN
//   ARGMIN : lexicographic min of (value, index); neutral (MIN neutral, -1)
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include "futseg.h"

namespace fs {

constexpr int kAdd = FS_ADD, kMin = FS_MIN, kMax = FS_MAX, kArgmin = FS_ARGMIN;

// ------------------------------------------------------------------ limits
template <typename T> struct Lim;
template <> struct Lim<int32_t> {
    static __host__ __device__ constexpr int32_t hi() { return INT32_MAX; }
    static __host__ __device__ constexpr int32_t lo() { return INT32_MIN; }
};
template <> struct Lim<int64_t> {
    static __host__ __device__ constexpr int64_t hi() { return INT64_MAX; }
    static __host__ __device__ constexpr int64_t lo() { return INT64_MIN; }
};
template <> struct Lim<float> {
    static __device__ float hi() { return __int_as_float(0x7f800000); }
    static __device__ float lo() { return __int_as_float(0xff800000); }
};

__device__ __forceinline__ int32_t wrap_add(int32_t a, int32_t b) {
    return (int32_t)((uint32_t)a + (uint32_t)b);
}
__device__ __forceinline__ int64_t wrap_add(int64_t a, int64_t b) {
    return (int64_t)((uint64_t)a + (uint64_t)b);
}
__device__ __forceinline__ float wrap_add(float a, float b) { return __fadd_rn(a, b); }

// (value, index) pair: the ARGMIN carrier (zip of values and indices, L138-146)
template <typename T> struct AV {
    T v;
    int64_t i;
};

// ------------------------------------------------------------------ ops
// Each Op provides
//   V     : the accumulator type
//   id()  : 0(+)
//   comb(a, b) : a (+) b (associative, commutative)
//   fold(a, x, i) : a (+) lift(x, i), valid ONLY when every index already
//                   folded into `a` is smaller than i (a thread visiting its
//                   elements in increasing index order) -- it lets ARGMIN
//                   skip the index tie test.
//   val(a), idx(a): the parts written to out / out_idx.
template <int OP, typename T> struct Op;

template <typename T> struct Op<kAdd, T> {
    using V = T;
    static __device__ __forceinline__ V id() { return T(0); }
    static __device__ __forceinline__ V comb(V a, V b) { return wrap_add(a, b); }
    static __device__ __forceinline__ V fold(V a, T x, int64_t) { return wrap_add(a, x); }
    static __device__ __forceinline__ V lift(T x, int64_t) { return x; }
    static __device__ __forceinline__ T val(V a) { return a; }
    static __device__ __forceinline__ int64_t idx(V) { return -1; }
};

template <typename T> struct Op<kMin, T> {
    using V = T;
    static __device__ __forceinline__ V id() { return Lim<T>::hi(); }
    static __device__ __forceinline__ V comb(V a, V b) { return b < a ? b : a; }
    static __device__ __forceinline__ V fold(V a, T x, int64_t) { return x < a ? x : a; }
    static __device__ __forceinline__ V lift(T x, int64_t) { return x; }
    static __device__ __forceinline__ T val(V a) { return a; }
    static __device__ __forceinline__ int64_t idx(V) { return -1; }
};

template <typename T> struct Op<kMax, T> {
    using V = T;
    static __device__ __forceinline__ V id() { return Lim<T>::lo(); }
    static __device__ __forceinline__ V comb(V a, V b) { return a < b ? b : a; }
    static __device__ __forceinline__ V fold(V a, T x, int64_t) { return a < x ? x : a; }
    static __device__ __forceinline__ V lift(T x, int64_t) { return x; }
    static __device__ __forceinline__ T val(V a) { return a; }
    static __device__ __forceinline__ int64_t idx(V) { return -1; }
};

template <typename T> struct Op<kArgmin, T> {
    using V = AV<T>;
    static __device__ __forceinline__ V id() { return V{Lim<T>::hi(), -1}; }
    static __device__ __forceinline__ V comb(V a, V b) {
        if (a.i < 0) return b;
        if (b.i < 0) return a;
        return (b.v < a.v || (b.v == a.v && b.i < a.i)) ? b : a;
    }
    // increasing-index fold: a tie keeps the earlier (smaller) index
    static __device__ __forceinline__ V fold(V a, T x, int64_t i) {
        return (x < a.v || a.i < 0) ? V{x, i} : a;
    }
    static __device__ __forceinline__ V lift(T x, int64_t i) { return V{x, i}; }
    static __device__ __forceinline__ T val(V a) { return a.v; }
    static __device__ __forceinline__ int64_t idx(V a) { return a.i; }
};

// ------------------------------------------------------------------ shuffles
__device__ __forceinline__ int32_t shfl_xor(int32_t v, int m) { return __shfl_xor_sync(0xffffffffu, v, m); }
__device__ __forceinline__ int64_t shfl_xor(int64_t v, int m) {
    return (int64_t)__shfl_xor_sync(0xffffffffu, (long long)v, m);
}
__device__ __forceinline__ float shfl_xor(float v, int m) { return __shfl_xor_sync(0xffffffffu, v, m); }
template <typename T> __device__ __forceinline__ AV<T> shfl_xor(AV<T> a, int m) {
    return AV<T>{shfl_xor(a.v, m), shfl_xor(a.i, m)};
}
__device__ __forceinline__ int32_t shfl_up(int32_t v, int d) { return __shfl_up_sync(0xffffffffu, v, d); }
__device__ __forceinline__ int64_t shfl_up(int64_t v, int d) {
    return (int64_t)__shfl_up_sync(0xffffffffu, (long long)v, d);
}
__device__ __forceinline__ float shfl_up(float v, int d) { return __shfl_up_sync(0xffffffffu, v, d); }
template <typename T> __device__ __forceinline__ AV<T> shfl_up(AV<T> a, int d) {
    return AV<T>{shfl_up(a.v, d), shfl_up(a.i, d)};
}
__device__ __forceinline__ int32_t shfl_down_v(int32_t v, int d) { return __shfl_down_sync(0xffffffffu, v, d); }
__device__ __forceinline__ int64_t shfl_down_v(int64_t v, int d) {
    return (int64_t)__shfl_down_sync(0xffffffffu, (long long)v, d);
}
__device__ __forceinline__ float shfl_down_v(float v, int d) { return __shfl_down_sync(0xffffffffu, v, d); }
template <typename T> __device__ __forceinline__ AV<T> shfl_down_v(AV<T> a, int d) {
    return AV<T>{shfl_down_v(a.v, d), shfl_down_v(a.i, d)};
}
__device__ __forceinline__ int32_t shfl_idx(int32_t v, int l) { return __shfl_sync(0xffffffffu, v, l); }
__device__ __forceinline__ int64_t shfl_idx(int64_t v, int l) {
    return (int64_t)__shfl_sync(0xffffffffu, (long long)v, l);
}
__device__ __forceinline__ float shfl_idx(float v, int l) { return __shfl_sync(0xffffffffu, v, l); }
template <typename T> __device__ __forceinline__ AV<T> shfl_idx(AV<T> a, int l) {
    return AV<T>{shfl_idx(a.v, l), shfl_idx(a.i, l)};
}

// Butterfly reduction over aligned groups of G lanes (G a power of two <= 32);
// every lane of the group ends with the group's result.
template <class O, int G = 32> __device__ __forceinline__ typename O::V group_reduce(typename O::V a) {
#pragma unroll
    for (int m = G / 2; m >= 1; m >>= 1) a = O::comb(a, shfl_xor(a, m));
    return a;
}

// Block reduction; the result is valid in thread 0.  `sm` holds >= 32 V.
template <class O, int NT> __device__ __forceinline__ typename O::V block_reduce(typename O::V a, typename O::V *sm) {
    constexpr int NW = NT / 32;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    a = group_reduce<O>(a);
    if (NW == 1) return a;
    __syncthreads();  // sm may be reused by the caller between calls
    if (lane == 0) sm[wid] = a;
    __syncthreads();
    if (wid == 0) {
        a = lane < NW ? sm[lane] : O::id();
        a = group_reduce<O>(a);
    }
    return a;
}

// ------------------------------------------------------------------ loads
// 16-byte streaming load through the non-coherent path, no L1 allocation
// (each input byte is read exactly once).
__device__ __forceinline__ int4 ldg16(const void *p) {
    int4 r;
    asm("ld.global.nc.L1::no_allocate.v4.s32 {%0, %1, %2, %3}, [%4];"
        : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
        : "l"(p));
    return r;
}

template <typename T> struct Vec16 {
    static constexpr int N = 16 / sizeof(T);
    T e[N];
};
template <typename T> __device__ __forceinline__ Vec16<T> as_vec(int4 r) {
    Vec16<T> v;
    static_assert(sizeof(Vec16<T>) == 16, "vec");
    memcpy(&v, &r, 16);
    return v;
}

// global-scope loads that bypass L1 (data written by other CTAs in this launch)
template <typename T> __device__ __forceinline__ T ld_cg(const T *p) { return __ldcg(p); }
template <typename T> __device__ __forceinline__ AV<T> ld_cg(const AV<T> *p) {
    return AV<T>{__ldcg(&p->v), __ldcg(&p->i)};
}
template <typename T> __device__ __forceinline__ void st_cg(T *p, T v) { __stcg(p, v); }
template <typename T> __device__ __forceinline__ void st_cg(AV<T> *p, AV<T> v) {
    __stcg(&p->v, v.v);
    __stcg(&p->i, v.i);
}

// Shift an ARGMIN index by the global index of the first element (sharding);
// a no-op for the other operators and for the empty result (index -1).
template <typename V> __device__ __forceinline__ V shift_idx(V a, int64_t) { return a; }
template <typename T> __device__ __forceinline__ AV<T> shift_idx(AV<T> a, int64_t base) {
    if (a.i >= 0) a.i += base;
    return a;
}

// The NN distance map (reading R5): sqrt((lat-q0)^2 + (lng-q1)^2), every f32
// operation separately rounded (no FMA contraction), IEEE sqrt.
__device__ __forceinline__ float nn_distance(float lat, float lng, float q0, float q1) {
    const float d0 = __fsub_rn(lat, q0), d1 = __fsub_rn(lng, q1);
    return __fsqrt_rn(__fadd_rn(__fmul_rn(d0, d0), __fmul_rn(d1, d1)));
}

// Store the final value (and ARGMIN index) of accumulator `a` at position k.
template <class O, typename T>
__device__ __forceinline__ void store_out(T *out, int64_t *out_idx, int64_t k, typename O::V a) {
    out[k] = O::val(a);
    if (out_idx) out_idx[k] = O::idx(a);
}

// ------------------------------------------------------------------ TMA bulk copies + mbarriers
// 1-D bulk copies (cp.async.bulk, SASS UBLKCP) from global to shared memory,
// completion tracked by an mbarrier transaction count.  Used to stream
// contiguous tiles into shared memory without holding them in registers.
__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t *bar, unsigned count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() { asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, unsigned bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}
// dst, src 16-byte aligned; bytes a multiple of 16
__device__ __forceinline__ void tma_load_1d(void *dst, const void *src, unsigned bytes, uint64_t *bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_u32(dst)),
                 "l"(src), "r"(bytes), "r"(smem_u32(bar))
                 : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, unsigned parity) {
    uint32_t done = 0;
    const uint32_t a = smem_u32(bar);
    while (!done) {
        asm volatile(
            "{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
            : "=r"(done)
            : "r"(a), "r"(parity)
            : "memory");
    }
}

// L2 prefetch of a contiguous global range (no shared memory, no completion): issued a few
// stages ahead of the TMA load that will read it, it moves the HBM latency off the ring slot
__device__ __forceinline__ void prefetch_l2_bulk(const void *src, unsigned bytes) {
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(src), "r"(bytes) : "memory");
}

// 1-D bulk copy shared -> global (SASS UBLKCP), tracked by bulk async-groups of the
// issuing thread: commit after issuing, wait_group_read<N> before the source smem
// is overwritten (all but the N most recent groups have finished READING smem),
// wait_group<0> before exit (writes performed).
__device__ __forceinline__ void tma_store_1d(void *dst, const void *src, unsigned bytes) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(smem_u32(src)),
                 "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N> __device__ __forceinline__ void bulk_wait_read() {
    asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
template <int N> __device__ __forceinline__ void bulk_wait() {
    asm volatile("cp.async.bulk.wait_group %0;" ::"n"(N) : "memory");
}

// ------------------------------------------------------------------ workspace layout
// [0, 256)          : control words
//     u32 ticket   @ 0     (single-counter kernels; reset by the last CTA)
//     u32 err      @ 64    (device precondition flag, fs_check_device_error)
//     u64 counters @ 128, 136, 192 (nn_knn barrier and candidates, kmeans delta)
// [256, 16640)      : kWsMaxTickets u32 tickets (per column tile / per segment),
//                     each reset to 0 by the CTA that consumes it
// [16640, ...)      : per-primitive body (partials, scan tile states), never
//                     assumed zero
// The control words and tickets are never used as data by any primitive, so a
// zero-filled workspace stays valid across calls of different primitives.
constexpr size_t kWsTicket = 0;
constexpr size_t kWsErr = 64;
constexpr size_t kWsCount0 = 128;  // u64 counters, zero between calls (reset by their last CTA):
constexpr size_t kWsCount1 = 136;  //   nn_knn grid barrier / candidate count,
constexpr size_t kWsCount2 = 192;  //   kmeans_step delta
constexpr size_t kWsTickets = 256;
constexpr int64_t kWsMaxTickets = 4096;
constexpr size_t kWsHeader = kWsTickets + 4 * kWsMaxTickets;

__host__ __device__ constexpr size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

}  // namespace fs
