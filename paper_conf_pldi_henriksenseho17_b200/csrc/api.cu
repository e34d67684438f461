// api.cu -- the extern "C" boundary of libfutseg (include/futseg.h).
//
// Host-side argument validation happens here, before any launch, so an error
// status has no side effects (mirrors Futhark's hoisted dynamic shape and
// bounds checks, L429-432).  The launchers it calls live in the per-kernel
// translation units.
#include <atomic>
#include <mutex>
#include <stdlib.h>
#include <unordered_map>

#include "internal.cuh"

namespace fs {

// ------------------------------------------------------------ device queries
int sm_count() {
    static int cache[128] = {0};
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 128) return 148;
    if (cache[dev] == 0) {
        int v = 0;
        if (cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || v <= 0) v = 148;
        cache[dev] = v;
    }
    return cache[dev];
}

int max_blocks_per_sm(const void *kernel, int threads, size_t smem) {
    static std::mutex mu;
    static std::unordered_map<uint64_t, int> cache;
    const uint64_t key = (uint64_t)(uintptr_t)kernel * 1000003ull ^ ((uint64_t)threads << 40) ^ (uint64_t)smem;
    {
        std::lock_guard<std::mutex> g(mu);
        auto it = cache.find(key);
        if (it != cache.end()) return it->second;
    }
    int b = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, kernel, threads, smem) != cudaSuccess || b <= 0) {
        cudaGetLastError();
        b = 1;
    }
    std::lock_guard<std::mutex> g(mu);
    cache[key] = b;
    return b;
}

static std::atomic<unsigned long long> g_launches{0};
void note_launches(int n) { g_launches.fetch_add((unsigned long long)n, std::memory_order_relaxed); }

static int g_forced_regime = -2;
int forced_seg_regime() {
    if (g_forced_regime == -2) {
        const char *e = getenv("FUTSEG_FORCE_REGIME");
        g_forced_regime = e ? atoi(e) : -1;
    }
    return g_forced_regime;
}

static thread_local int g_last_regime = -1;
void note_regime(int r) { g_last_regime = r; }
int last_regime() { return g_last_regime; }

}  // namespace fs

using namespace fs;

namespace {

bool valid_dtype(int dt) { return dt == FS_I32 || dt == FS_I64 || dt == FS_F32; }
bool valid_scalar_op(int op) { return op == FS_ADD || op == FS_MIN || op == FS_MAX || op == FS_ARGMIN; }

// op descriptor check; allow_vadd only for redomap
fs_status check_op(const fs_opdesc &op, bool allow_vadd) {
    if (!valid_dtype(op.dtype)) return FS_ERR_UNSUPPORTED;
    if (op.op == FS_VADD) {
        if (!allow_vadd) return FS_ERR_UNSUPPORTED;
        if (op.width < 1) return FS_ERR_SIZE;
        return FS_OK;
    }
    if (!valid_scalar_op(op.op)) return FS_ERR_UNSUPPORTED;
    if (op.width > 1) return FS_ERR_UNSUPPORTED;
    return FS_OK;
}

bool mul_overflows(int64_t a, int64_t b) { return a != 0 && b > INT64_MAX / a; }

bool aligned_to(const void *p, size_t a) { return ((uintptr_t)p % a) == 0; }

// do [a, a+na) and [b, b+nb) overlap?
bool overlaps(const void *a, int64_t na, const void *b, int64_t nb) {
    if (!a || !b || na <= 0 || nb <= 0) return false;
    const uintptr_t x = (uintptr_t)a, y = (uintptr_t)b;
    return x < y + (uintptr_t)nb && y < x + (uintptr_t)na;
}

fs_status check_ws(void *ws, size_t have, size_t need) {
    if (need == 0) return FS_OK;
    if (!ws) return FS_ERR_WORKSPACE;
    if (have < need) return FS_ERR_WORKSPACE;
    if (!aligned_to(ws, 256)) return FS_ERR_WORKSPACE;
    return FS_OK;
}

cudaStream_t S(void *stream) { return (cudaStream_t)stream; }

#define FS_TRY(x)                           \
    do {                                    \
        fs_status _s = (x);                 \
        if (_s != FS_OK) return _s;         \
    } while (0)

// map descriptor + inputs for redomap/scanomap
fs_status check_map(const fs_opdesc &op, const fs_mapdesc &map, const void *in0, const void *in1, int64_t n) {
    if (map.kind == FS_MAP_ID) {
        if (in1) return FS_ERR_UNSUPPORTED;
        if (n > 0 && !in0) return FS_ERR_NULL;
        if (in0 && !aligned_to(in0, dtype_size(op.dtype))) return FS_ERR_UNSUPPORTED;
        return FS_OK;
    }
    if (map.kind == FS_MAP_NN_DIST) {
        if (op.dtype != FS_F32 || op.op == FS_VADD) return FS_ERR_UNSUPPORTED;
        if (n > 0 && (!in0 || !in1)) return FS_ERR_NULL;
        if ((in0 && !aligned_to(in0, 4)) || (in1 && !aligned_to(in1, 4))) return FS_ERR_UNSUPPORTED;
        return FS_OK;
    }
    return FS_ERR_UNSUPPORTED;
}

int64_t in_bytes(const fs_opdesc &op, const fs_mapdesc &map, int64_t n) {
    return n * (map.kind == FS_MAP_NN_DIST ? 4 : (int64_t)dtype_size(op.dtype) * (op.op == FS_VADD ? op.width : 1));
}

}  // namespace

extern "C" {

const char *fs_version(void) { return "libfutseg 0.1 (sm_100a)"; }

uint64_t fs_launch_count(void) { return (uint64_t)g_launches.load(std::memory_order_relaxed); }

const char *fs_status_string(fs_status s) {
    switch (s) {
    case FS_OK: return "FS_OK";
    case FS_ERR_NULL: return "FS_ERR_NULL: a required pointer is NULL";
    case FS_ERR_SIZE: return "FS_ERR_SIZE: negative or overflowing size";
    case FS_ERR_UNSUPPORTED: return "FS_ERR_UNSUPPORTED: (op, dtype, map, layout) not supported";
    case FS_ERR_ALIAS: return "FS_ERR_ALIAS: output overlaps an input";
    case FS_ERR_WORKSPACE: return "FS_ERR_WORKSPACE: workspace missing, misaligned or too small";
    case FS_ERR_CUDA: return "FS_ERR_CUDA: CUDA launch or runtime error";
    case FS_ERR_BOUNDS: return "FS_ERR_BOUNDS: device-side precondition violation (key out of range)";
    }
    return "unknown fs_status";
}

fs_status fs_force_seg_regime(int32_t regime) {
    // -1 automatic; 0..3 the seg_reduce regimes; 5, 7..12 the row-major seg_scan regimes
    // (applied only where their preconditions hold, see fs::seg_scan_plan)
    if (regime < -1 || regime == 4 || regime == 6 || regime > 12) return FS_ERR_UNSUPPORTED;
    g_forced_regime = regime;
    return FS_OK;
}

// ------------------------------------------------------------ workspace queries
fs_status fs_redomap_workspace(fs_opdesc op, int64_t n, size_t *bytes) {
    if (!bytes) return FS_ERR_NULL;
    FS_TRY(check_op(op, true));
    if (n < 0) return FS_ERR_SIZE;
    if (op.op == FS_VADD) {
        if (mul_overflows(n, op.width)) return FS_ERR_SIZE;
        *bytes = colreduce_ws(FS_ADD, op.dtype, n, op.width);
    } else {
        *bytes = redomap_ws(op.op, op.dtype, n, false);
    }
    return FS_OK;
}

fs_status fs_scanomap_workspace(fs_opdesc op, int64_t n, size_t *bytes) {
    if (!bytes) return FS_ERR_NULL;
    FS_TRY(check_op(op, false));
    if (n < 0) return FS_ERR_SIZE;
    *bytes = scan_ws(op.op, op.dtype, n);
    return FS_OK;
}

fs_status fs_seg_reduce_workspace(fs_opdesc op, int64_t nseg, int64_t seglen, int32_t layout, size_t *bytes) {
    if (!bytes) return FS_ERR_NULL;
    FS_TRY(check_op(op, false));
    if (nseg < 0 || seglen < 0 || mul_overflows(nseg, seglen)) return FS_ERR_SIZE;
    if (layout == FS_ROW_MAJOR || (layout == FS_COL_MAJOR && (nseg <= 1 || seglen <= 1)))
        *bytes = seg_reduce_ws(op.op, op.dtype, nseg, seglen);
    else if (layout == FS_COL_MAJOR) *bytes = colreduce_ws(op.op, op.dtype, seglen, nseg);
    else return FS_ERR_UNSUPPORTED;
    return FS_OK;
}

fs_status fs_seg_scan_workspace(fs_opdesc op, int64_t nseg, int64_t seglen, int32_t layout, size_t *bytes) {
    if (!bytes) return FS_ERR_NULL;
    FS_TRY(check_op(op, false));
    if (nseg < 0 || seglen < 0 || mul_overflows(nseg, seglen)) return FS_ERR_SIZE;
    if (layout == FS_ROW_MAJOR || (layout == FS_COL_MAJOR && (nseg <= 1 || seglen <= 1)))
        *bytes = scan_ws(op.op, op.dtype, nseg * seglen);
    else if (layout == FS_COL_MAJOR) *bytes = colscan_ws(op.op, op.dtype, seglen, nseg);
    else return FS_ERR_UNSUPPORTED;
    return FS_OK;
}

fs_status fs_stream_red_workspace(int32_t dtype, int64_t n, int64_t w, int64_t k, size_t *bytes) {
    if (!bytes) return FS_ERR_NULL;
    if (!valid_dtype(dtype)) return FS_ERR_UNSUPPORTED;
    if (n < 0 || w < 0 || k < 0 || mul_overflows(n, w) || mul_overflows(k, w)) return FS_ERR_SIZE;
    *bytes = stream_red_ws(dtype, n, w, k);
    return FS_OK;
}

// ------------------------------------------------------------ redomap
fs_status fs_redomap(fs_opdesc op, fs_mapdesc map, const void *in0, const void *in1, int64_t n, void *out,
                     int64_t *out_idx, void *ws, size_t ws_bytes, void *stream) {
    FS_TRY(check_op(op, true));
    if (n < 0) return FS_ERR_SIZE;
    if (op.op == FS_VADD && mul_overflows(n, op.width * (int64_t)dtype_size(op.dtype))) return FS_ERR_SIZE;
    FS_TRY(check_map(op, map, in0, in1, n));
    if (!out) return FS_ERR_NULL;
    if (op.op == FS_ARGMIN && !out_idx) return FS_ERR_NULL;
    if (!aligned_to(out, dtype_size(op.dtype)) || (out_idx && !aligned_to(out_idx, 8))) return FS_ERR_UNSUPPORTED;
    const int64_t ib = in_bytes(op, map, n);
    const int64_t ob = (op.op == FS_VADD ? op.width : 1) * (int64_t)dtype_size(op.dtype);
    if (overlaps(out, ob, in0, ib) || overlaps(out, ob, in1, ib) ||
        (op.op == FS_ARGMIN && (overlaps(out_idx, 8, in0, ib) || overlaps(out_idx, 8, in1, ib) ||
                                overlaps(out_idx, 8, out, ob))))
        return FS_ERR_ALIAS;
    size_t need = 0;
    FS_TRY(fs_redomap_workspace(op, n, &need));
    FS_TRY(check_ws(ws, ws_bytes, need));
    if (op.op == FS_VADD) {
        if (n == 0) return fill_neutral_run(FS_ADD, op.dtype, op.width, out, nullptr, S(stream));
        return colreduce_run(FS_ADD, op.dtype, in0, n, op.width, out, nullptr, ws, S(stream));
    }
    return redomap_run(op.op, op.dtype, map, in0, in1, n, out, op.op == FS_ARGMIN ? out_idx : nullptr, ws,
                       S(stream));
}

// ------------------------------------------------------------ scanomap
fs_status fs_scanomap(fs_opdesc op, fs_mapdesc map, const void *in0, const void *in1, int64_t n, void *out,
                      int64_t *out_idx, const void *carry, const int64_t *carry_idx, void *ws, size_t ws_bytes,
                      void *stream) {
    FS_TRY(check_op(op, false));
    if (n < 0) return FS_ERR_SIZE;
    FS_TRY(check_map(op, map, in0, in1, n));
    if (n > 0 && !out) return FS_ERR_NULL;
    if (n > 0 && op.op == FS_ARGMIN && !out_idx) return FS_ERR_NULL;
    if (carry && op.op == FS_ARGMIN && !carry_idx) return FS_ERR_NULL;
    if ((out && !aligned_to(out, dtype_size(op.dtype))) || (out_idx && !aligned_to(out_idx, 8)))
        return FS_ERR_UNSUPPORTED;
    const int64_t ib = in_bytes(op, map, n);
    const int64_t ob = n * (int64_t)dtype_size(op.dtype);
    if (overlaps(out, ob, in0, ib) || overlaps(out, ob, in1, ib) ||
        (op.op == FS_ARGMIN && (overlaps(out_idx, 8 * n, in0, ib) || overlaps(out_idx, 8 * n, in1, ib) ||
                                overlaps(out_idx, 8 * n, out, ob))))
        return FS_ERR_ALIAS;
    size_t need = 0;
    FS_TRY(fs_scanomap_workspace(op, n, &need));
    FS_TRY(check_ws(ws, ws_bytes, need));
    if (n == 0) return FS_OK;
    return scan_run(op.op, op.dtype, map, in0, in1, n, n, out, op.op == FS_ARGMIN ? out_idx : nullptr, carry,
                    op.op == FS_ARGMIN ? carry_idx : nullptr, ws, S(stream));
}

// ------------------------------------------------------------ combine
fs_status fs_combine(fs_opdesc op, const void *parts, const int64_t *part_idx, int64_t P, void *out,
                     int64_t *out_idx, void *stream) {
    FS_TRY(check_op(op, true));
    if (P < 0) return FS_ERR_SIZE;
    if (P > 0 && !parts) return FS_ERR_NULL;
    if (!out) return FS_ERR_NULL;
    if (op.op == FS_ARGMIN && (!out_idx || (P > 0 && !part_idx))) return FS_ERR_NULL;
    const int64_t w = op.op == FS_VADD ? op.width : 1;
    if (mul_overflows(P, w)) return FS_ERR_SIZE;
    const int64_t pb = P * w * (int64_t)dtype_size(op.dtype), ob = w * (int64_t)dtype_size(op.dtype);
    if (overlaps(out, ob, parts, pb) || overlaps(out, ob, part_idx, 8 * P)) return FS_ERR_ALIAS;
    return combine_run(op.op, op.dtype, w, parts, part_idx, P, out, op.op == FS_ARGMIN ? out_idx : nullptr,
                       S(stream));
}

// ------------------------------------------------------------ stream_red
fs_status fs_stream_red(int32_t dtype, const void *vals, const int32_t *keys, int64_t n, int64_t w, int64_t k,
                        void *sums, int32_t *counts, void *ws, size_t ws_bytes, void *stream) {
    if (!valid_dtype(dtype)) return FS_ERR_UNSUPPORTED;
    if (n < 0 || w < 0 || k < 0 || mul_overflows(n, w) || mul_overflows(k, w)) return FS_ERR_SIZE;
    if (n > 0 && (!keys || (w > 0 && !vals))) return FS_ERR_NULL;
    if (k > 0 && w > 0 && !sums) return FS_ERR_NULL;
    const int64_t es = (int64_t)dtype_size(dtype);
    if ((vals && !aligned_to(vals, es)) || (sums && !aligned_to(sums, es)) || (keys && !aligned_to(keys, 4)) ||
        (counts && !aligned_to(counts, 4)))
        return FS_ERR_UNSUPPORTED;
    const int64_t vb = n * w * es, kb = 4 * n, sb = k * w * es, cb = 4 * k;
    if (overlaps(sums, sb, vals, vb) || overlaps(sums, sb, keys, kb) || overlaps(counts, cb, vals, vb) ||
        overlaps(counts, cb, keys, kb) || overlaps(counts, cb, sums, sb))
        return FS_ERR_ALIAS;
    size_t need = 0;
    FS_TRY(fs_stream_red_workspace(dtype, n, w, k, &need));
    FS_TRY(check_ws(ws, ws_bytes, need));
    if (k == 0) return FS_OK;
    return stream_red_run(dtype, vals, keys, n, w, k, sums, counts, ws, S(stream));
}

// ------------------------------------------------------------ segmented
static fs_status seg_common(const fs_opdesc &op, const void *in, int64_t nseg, int64_t seglen, int32_t layout,
                            void *out, int64_t *out_idx, int64_t out_elems) {
    FS_TRY(check_op(op, false));
    if (nseg < 0 || seglen < 0 || mul_overflows(nseg, seglen) ||
        mul_overflows(nseg * seglen, (int64_t)sizeof(int64_t)))
        return FS_ERR_SIZE;
    if (layout != FS_ROW_MAJOR && layout != FS_COL_MAJOR) return FS_ERR_UNSUPPORTED;
    if (nseg * seglen > 0 && !in) return FS_ERR_NULL;
    if (out_elems > 0 && !out) return FS_ERR_NULL;
    if (out_elems > 0 && op.op == FS_ARGMIN && !out_idx) return FS_ERR_NULL;
    const int64_t es = (int64_t)dtype_size(op.dtype);
    if ((in && !aligned_to(in, es)) || (out && !aligned_to(out, es)) || (out_idx && !aligned_to(out_idx, 8)))
        return FS_ERR_UNSUPPORTED;
    const int64_t ib = nseg * seglen * es, ob = out_elems * es;
    if (overlaps(out, ob, in, ib) ||
        (op.op == FS_ARGMIN && (overlaps(out_idx, 8 * out_elems, in, ib) || overlaps(out_idx, 8 * out_elems, out, ob))))
        return FS_ERR_ALIAS;
    return FS_OK;
}

fs_status fs_seg_reduce(fs_opdesc op, const void *in, int64_t nseg, int64_t seglen, int32_t layout, void *out,
                        int64_t *out_idx, void *ws, size_t ws_bytes, void *stream) {
    FS_TRY(seg_common(op, in, nseg, seglen, layout, out, out_idx, nseg));
    size_t need = 0;
    FS_TRY(fs_seg_reduce_workspace(op, nseg, seglen, layout, &need));
    FS_TRY(check_ws(ws, ws_bytes, need));
    int64_t *oi = op.op == FS_ARGMIN ? out_idx : nullptr;
    note_regime(RG_EMPTY);
    if (nseg == 0) return FS_OK;
    if (seglen == 0) return fill_neutral_run(op.op, op.dtype, nseg, out, oi, S(stream));
    // with one segment, or segments of one element, both layouts are the same bytes
    note_regime(RG_COL);
    if (layout == FS_COL_MAJOR && nseg > 1 && seglen > 1)
        return colreduce_run(op.op, op.dtype, in, seglen, nseg, out, oi, ws, S(stream));
    return seg_reduce_run(op.op, op.dtype, in, nseg, seglen, out, oi, ws, S(stream));
}

fs_status fs_seg_scan(fs_opdesc op, const void *in, int64_t nseg, int64_t seglen, int32_t layout, void *out,
                      int64_t *out_idx, void *ws, size_t ws_bytes, void *stream) {
    FS_TRY(seg_common(op, in, nseg, seglen, layout, out, out_idx, nseg * seglen));
    size_t need = 0;
    FS_TRY(fs_seg_scan_workspace(op, nseg, seglen, layout, &need));
    FS_TRY(check_ws(ws, ws_bytes, need));
    int64_t *oi = op.op == FS_ARGMIN ? out_idx : nullptr;
    note_regime(RG_EMPTY);
    if (nseg * seglen == 0) return FS_OK;
    note_regime(RG_COL);
    if (layout == FS_COL_MAJOR && nseg > 1 && seglen > 1)
        return colscan_run(op.op, op.dtype, in, seglen, nseg, out, oi, ws, S(stream));
    const fs_mapdesc id = {FS_MAP_ID, 0.f, 0.f, 0};
    return scan_run(op.op, op.dtype, id, in, nullptr, nseg * seglen, seglen, out, oi, nullptr, nullptr, ws,
                    S(stream));
}

// ------------------------------------------------------------ transpose
fs_status fs_transpose_2d(int32_t dtype, const void *in, int64_t rows, int64_t cols, void *out, void *stream) {
    if (!valid_dtype(dtype)) return FS_ERR_UNSUPPORTED;
    if (rows < 0 || cols < 0 || mul_overflows(rows, cols) || mul_overflows(rows * cols, 8)) return FS_ERR_SIZE;
    if (rows * cols == 0) return FS_OK;
    if (!in || !out) return FS_ERR_NULL;
    const int64_t es = (int64_t)dtype_size(dtype);
    if (!aligned_to(in, es) || !aligned_to(out, es)) return FS_ERR_UNSUPPORTED;
    if (overlaps(out, rows * cols * es, in, rows * cols * es)) return FS_ERR_ALIAS;
    return transpose_run(dtype, in, rows, cols, out, S(stream));
}

// ------------------------------------------------------------ NEXT-2: nn_knn
fs_status fs_nn_knn_workspace(int64_t n, int64_t kk, size_t *bytes) {
    if (!bytes) return FS_ERR_NULL;
    if (n < 0 || n >= (int64_t(1) << 32) || kk < 0 || kk > 1024) return FS_ERR_SIZE;
    *bytes = knn_ws(n);
    return FS_OK;
}

fs_status fs_nn_knn(const float *lat, const float *lng, int64_t n, float q0, float q1, int64_t kk,
                    float *out_dist, int64_t *out_idx, void *ws, size_t ws_bytes, void *stream) {
    size_t need = 0;
    FS_TRY(fs_nn_knn_workspace(n, kk, &need));
    if (kk == 0) return FS_OK;
    if ((n > 0 && (!lat || !lng)) || !out_dist || !out_idx) return FS_ERR_NULL;
    if ((n > 0 && (!aligned_to(lat, 4) || !aligned_to(lng, 4))) || !aligned_to(out_dist, 4) ||
        !aligned_to(out_idx, 8))
        return FS_ERR_UNSUPPORTED;
    if (overlaps(out_dist, kk * 4, lat, n * 4) || overlaps(out_dist, kk * 4, lng, n * 4) ||
        overlaps(out_idx, kk * 8, lat, n * 4) || overlaps(out_idx, kk * 8, lng, n * 4) ||
        overlaps(out_idx, kk * 8, out_dist, kk * 4))
        return FS_ERR_ALIAS;
    FS_TRY(check_ws(ws, ws_bytes, need));
    return knn_run(lat, lng, n, q0, q1, kk, out_dist, out_idx, ws, S(stream));
}

// ------------------------------------------------------------ NEXT-1: kmeans_step
fs_status fs_kmeans_step_workspace(int64_t n, int64_t d, int64_t k, size_t *bytes) {
    if (!bytes) return FS_ERR_NULL;
    if (n < 0 || mul_overflows(n, d) || mul_overflows(n * (d > 0 ? d : 1), 4)) return FS_ERR_SIZE;
    if (k < 1 || k > 32 || d < 1 || d > 40) return FS_ERR_UNSUPPORTED;
    *bytes = kmeans_ws(n, d, k);
    return FS_OK;
}

fs_status fs_kmeans_step(const float *points, int64_t n, int64_t d, const float *centres, int64_t k,
                         const int32_t *prev, int32_t *membership, float *sums, int32_t *counts, float *new_centres,
                         int64_t *delta, void *ws, size_t ws_bytes, void *stream) {
    size_t need = 0;
    FS_TRY(fs_kmeans_step_workspace(n, d, k, &need));
    if ((n > 0 && !points) || !centres || !sums || !counts) return FS_ERR_NULL;
    if ((n > 0 && !aligned_to(points, 16)) || !aligned_to(centres, 4) || !aligned_to(sums, 4) ||
        !aligned_to(counts, 4) || (prev && !aligned_to(prev, 4)) || (membership && !aligned_to(membership, 4)) ||
        (new_centres && !aligned_to(new_centres, 4)) || (delta && !aligned_to(delta, 8)))
        return FS_ERR_UNSUPPORTED;
    const int64_t pb = n * d * 4, cb = k * d * 4;
    const void *ins[3] = {points, centres, prev};
    const int64_t inb[3] = {pb, cb, n * 4};
    void *outs[5] = {membership, sums, counts, new_centres, delta};
    const int64_t outb[5] = {n * 4, cb, k * 4, cb, 8};
    for (int o = 0; o < 5; ++o) {
        if (!outs[o]) continue;
        for (int i = 0; i < 3; ++i)
            if (ins[i] && overlaps(outs[o], outb[o], ins[i], inb[i])) return FS_ERR_ALIAS;
        for (int p = 0; p < o; ++p)
            if (outs[p] && overlaps(outs[o], outb[o], outs[p], outb[p])) return FS_ERR_ALIAS;
    }
    FS_TRY(check_ws(ws, ws_bytes, need));
    return kmeans_run(points, n, d, centres, k, prev, membership, sums, counts, new_centres, delta, ws, S(stream));
}

// ------------------------------------------------------------ NEXT-4: seg_map_reduce
fs_status fs_seg_map_reduce_workspace(fs_opdesc op, int64_t nseg, int64_t seglen, size_t *bytes) {
    if (!bytes) return FS_ERR_NULL;
    FS_TRY(check_op(op, false));
    if (nseg < 0 || seglen < 0 || mul_overflows(nseg, seglen) || mul_overflows(nseg * seglen, 8)) return FS_ERR_SIZE;
    *bytes = seg_map_reduce_ws(op.op, op.dtype, nseg, seglen);
    return FS_OK;
}

fs_status fs_seg_map_reduce(fs_opdesc op, const void *in, int64_t nseg, int64_t seglen, int64_t c_int, float c_f32,
                            void *out_map, void *out, int64_t *out_idx, void *ws, size_t ws_bytes, void *stream) {
    size_t need = 0;
    FS_TRY(fs_seg_map_reduce_workspace(op, nseg, seglen, &need));
    if (nseg == 0) return FS_OK;
    if (!out || (seglen > 0 && (!in || !out_map)) || (op.op == FS_ARGMIN && !out_idx)) return FS_ERR_NULL;
    const int64_t es = (int64_t)dtype_size(op.dtype), nb = nseg * seglen * es;
    if ((in && !aligned_to(in, es)) || (out_map && !aligned_to(out_map, es)) || !aligned_to(out, es) ||
        (out_idx && !aligned_to(out_idx, 8)))
        return FS_ERR_UNSUPPORTED;
    const int64_t ob = nseg * es, ib8 = out_idx ? nseg * 8 : 0;
    if (overlaps(out_map, nb, in, nb) || overlaps(out, ob, in, nb) || overlaps(out, ob, out_map, nb) ||
        (out_idx && (overlaps(out_idx, ib8, in, nb) || overlaps(out_idx, ib8, out_map, nb) ||
                     overlaps(out_idx, ib8, out, ob))))
        return FS_ERR_ALIAS;
    FS_TRY(check_ws(ws, ws_bytes, need));
    if (seglen == 0) return fill_neutral_run(op.op, op.dtype, nseg, out, op.op == FS_ARGMIN ? out_idx : nullptr,
                                             S(stream));
    return seg_map_reduce_run(op.op, op.dtype, in, nseg, seglen, c_int, c_f32, out_map, out,
                              op.op == FS_ARGMIN ? out_idx : nullptr, ws, S(stream));
}

fs_status fs_kmeans_finish(const float *sums, const int32_t *counts, const float *centres, int64_t k, int64_t d,
                           float *new_centres, void *stream) {
    if (k < 0 || d < 0 || mul_overflows(k, d)) return FS_ERR_SIZE;
    if (k * d == 0) return FS_OK;
    if (!sums || !counts || !centres || !new_centres) return FS_ERR_NULL;
    if (!aligned_to(sums, 4) || !aligned_to(counts, 4) || !aligned_to(centres, 4) || !aligned_to(new_centres, 4))
        return FS_ERR_UNSUPPORTED;
    const int64_t b = k * d * 4;
    if (overlaps(new_centres, b, sums, b) || overlaps(new_centres, b, centres, b) ||
        overlaps(new_centres, b, counts, k * 4))
        return FS_ERR_ALIAS;
    return kmeans_finish_run(sums, counts, centres, k, d, new_centres, S(stream));
}

// ------------------------------------------------------------ NEXT-3: scan_reduce
fs_status fs_scan_reduce_workspace(int32_t dtype, int64_t n, size_t *bytes) {
    if (!bytes) return FS_ERR_NULL;
    if (!valid_dtype(dtype)) return FS_ERR_UNSUPPORTED;
    if (n < 0 || mul_overflows(n, 8)) return FS_ERR_SIZE;
    *bytes = scan_reduce_ws(dtype);
    return FS_OK;
}

fs_status fs_scan_reduce(int32_t scan_op, int32_t red_op, int32_t dtype, const void *in, int64_t n, void *out,
                         void *ws, size_t ws_bytes, void *stream) {
    size_t need = 0;
    FS_TRY(fs_scan_reduce_workspace(dtype, n, &need));
    if (scan_op != FS_ADD || (red_op != FS_ADD && red_op != FS_MAX && red_op != FS_MIN)) return FS_ERR_UNSUPPORTED;
    if (!out || (n > 0 && !in)) return FS_ERR_NULL;
    const int64_t es = (int64_t)dtype_size(dtype);
    if ((in && !aligned_to(in, es)) || !aligned_to(out, es)) return FS_ERR_UNSUPPORTED;
    if (overlaps(out, es, in, n * es)) return FS_ERR_ALIAS;
    FS_TRY(check_ws(ws, ws_bytes, need));
    if (n > 0 && !aligned_to(in, 16)) return FS_ERR_UNSUPPORTED;  // 16-byte vector loads
    return scan_reduce_run(red_op, dtype, in, n, out, ws, S(stream));
}

// ------------------------------------------------------------ multi-GPU exchange helpers
fs_status fs_argmin_pack(int32_t dtype, const void *values, const int64_t *idx, int64_t n, int64_t *keys,
                         void *stream) {
    if (!valid_dtype(dtype)) return FS_ERR_UNSUPPORTED;
    if (n < 0) return FS_ERR_SIZE;
    if (n == 0) return FS_OK;
    if (!values || !idx || !keys) return FS_ERR_NULL;
    const int64_t es = (int64_t)dtype_size(dtype), kb = n * (dtype == FS_I64 ? 16 : 8);
    if (!aligned_to(values, es) || !aligned_to(idx, 8) || !aligned_to(keys, 8)) return FS_ERR_UNSUPPORTED;
    if (overlaps(keys, kb, values, n * es) || overlaps(keys, kb, idx, n * 8)) return FS_ERR_ALIAS;
    return argmin_pack_run(dtype, values, idx, n, keys, S(stream));
}

fs_status fs_argmin_unpack(int32_t dtype, const int64_t *keys, int64_t P, void *value, int64_t *idx, void *stream) {
    if (!valid_dtype(dtype)) return FS_ERR_UNSUPPORTED;
    if (P < 0 || (dtype != FS_I64 && P != 1)) return FS_ERR_SIZE;
    if ((P > 0 && !keys) || !value || !idx) return FS_ERR_NULL;
    const int64_t es = (int64_t)dtype_size(dtype), kb = P * (dtype == FS_I64 ? 16 : 8);
    if ((keys && !aligned_to(keys, 8)) || !aligned_to(value, es) || !aligned_to(idx, 8)) return FS_ERR_UNSUPPORTED;
    if (overlaps(value, es, keys, kb) || overlaps(idx, 8, keys, kb)) return FS_ERR_ALIAS;
    return argmin_unpack_run(dtype, keys, P, value, idx, S(stream));
}

fs_status fs_partials_pack(int32_t dtype, const void *sums, const int32_t *counts, const int64_t *extra, int64_t k,
                           int64_t w, void *packed, void *stream) {
    if (!valid_dtype(dtype)) return FS_ERR_UNSUPPORTED;
    if (k < 0 || w < 0 || mul_overflows(k, w)) return FS_ERR_SIZE;
    if (!packed || (k * w > 0 && !sums)) return FS_ERR_NULL;
    const int64_t es = (int64_t)dtype_size(dtype), pb = (k * w + k + 1) * 8;
    if ((sums && !aligned_to(sums, es)) || (counts && !aligned_to(counts, 4)) || (extra && !aligned_to(extra, 8)) ||
        !aligned_to(packed, 8))
        return FS_ERR_UNSUPPORTED;
    if (overlaps(packed, pb, sums, k * w * es) || overlaps(packed, pb, counts, k * 4) || overlaps(packed, pb, extra, 8))
        return FS_ERR_ALIAS;
    return partials_pack_run(dtype, sums, counts, extra, k * w, k, packed, S(stream));
}

fs_status fs_partials_unpack(int32_t dtype, const void *packed, int64_t k, int64_t w, void *sums, int32_t *counts,
                             int64_t *extra, void *stream) {
    if (!valid_dtype(dtype)) return FS_ERR_UNSUPPORTED;
    if (k < 0 || w < 0 || mul_overflows(k, w)) return FS_ERR_SIZE;
    if (!packed || (k * w > 0 && !sums)) return FS_ERR_NULL;
    const int64_t es = (int64_t)dtype_size(dtype), pb = (k * w + k + 1) * 8;
    if ((sums && !aligned_to(sums, es)) || (counts && !aligned_to(counts, 4)) || (extra && !aligned_to(extra, 8)) ||
        !aligned_to(packed, 8))
        return FS_ERR_UNSUPPORTED;
    if (overlaps(packed, pb, sums, k * w * es) || overlaps(packed, pb, counts, k * 4) || overlaps(packed, pb, extra, 8))
        return FS_ERR_ALIAS;
    return partials_unpack_run(dtype, packed, k * w, k, sums, counts, extra, S(stream));
}

fs_status fs_copy_2d(int32_t elem_bytes, const void *src, int64_t src_ld, int64_t rows, int64_t cols, void *dst,
                     int64_t dst_ld, void *stream) {
    if (elem_bytes != 4 && elem_bytes != 8) return FS_ERR_UNSUPPORTED;
    if (rows < 0 || cols < 0 || src_ld < cols || dst_ld < cols || mul_overflows(rows, src_ld) ||
        mul_overflows(rows, dst_ld))
        return FS_ERR_SIZE;
    if (rows * cols == 0) return FS_OK;
    if (!src || !dst) return FS_ERR_NULL;
    if (!aligned_to(src, elem_bytes) || !aligned_to(dst, elem_bytes)) return FS_ERR_UNSUPPORTED;
    const int64_t sb = ((rows - 1) * src_ld + cols) * elem_bytes, db = ((rows - 1) * dst_ld + cols) * elem_bytes;
    if (overlaps(dst, db, src, sb)) return FS_ERR_ALIAS;
    return copy_2d_run(elem_bytes, src, src_ld, rows, cols, dst, dst_ld, S(stream));
}

// ------------------------------------------------------------ utilities
fs_status fs_check_device_error(void *ws, void *stream) {
    if (!ws) return FS_ERR_NULL;
    if (cudaStreamSynchronize(S(stream)) != cudaSuccess) return FS_ERR_CUDA;
    unsigned err = 0;
    unsigned *p = (unsigned *)((char *)ws + kWsErr);
    if (cudaMemcpy(&err, p, sizeof(err), cudaMemcpyDeviceToHost) != cudaSuccess) return FS_ERR_CUDA;
    if (err) {
        if (cudaMemset(p, 0, sizeof(unsigned)) != cudaSuccess) return FS_ERR_CUDA;
        return FS_ERR_BOUNDS;
    }
    return FS_OK;
}

int32_t fs_seg_regime(int32_t prim_is_scan, fs_opdesc op, int64_t nseg, int64_t seglen, int32_t layout) {
    if (check_op(op, false) != FS_OK || nseg < 0 || seglen < 0 || mul_overflows(nseg, seglen)) return -1;
    if (layout != FS_ROW_MAJOR && layout != FS_COL_MAJOR) return -1;
    if (nseg == 0 || seglen == 0) return RG_EMPTY;
    if (layout == FS_COL_MAJOR && nseg > 1 && seglen > 1) return RG_COL;
    if (prim_is_scan)  // buffers from an allocator: 16-byte aligned, same phase
        return seg_scan_plan(op.op, op.dtype, nseg * seglen, seglen, true, true, true, true);
    return seg_reduce_regime(op.op, op.dtype, nseg, seglen);
}

int32_t fs_last_seg_regime(void) { return fs::last_regime(); }

}  // extern "C"
