/*
 * futseg.h -- C ABI of libfutseg, the B200 (sm_100a) hot path of Futhark's
 * compiled code (Henriksen et al., PLDI'17; /root/reference/PAPER.md = "L<n>").
 *
 * After fusion (Sec. 4) and flattening (Sec. 5) a Futhark program is a perfect
 * map nest whose innermost operator is a reduce, a scan or a stream_red.
 * This library implements those innermost operators as hand-written CUDA
 * kernels, over a fixed operator table:
 *
 *   op     : FS_ADD, FS_MIN, FS_MAX, FS_ARGMIN (value + index), FS_VADD (k-wide
 *            vector add, the map(+) operator of Fig 4b/4c and G5)
 *   dtype  : FS_I32, FS_I64, FS_F32
 *   map f  : FS_MAP_ID, FS_MAP_NN_DIST (Rodinia NN distance, see fs_mapdesc)
 *
 * Semantics (each a plain definition; the oracle in oracle/ is that definition):
 *   reduce (+) 0(+) [a1..an] = 0(+) (+) a1 (+) ... (+) an            L127-128
 *   scan   (+) 0(+) [a1..an] = [a1, ..., a1 (+) ... (+) an] (inclusive) L129-130
 *   redomap  = fold (+,0(+)) f = reduce (+) . map f                   L240-241, L254
 *   scanomap = scan (+) . map f   (name by analogy with redomap, L978)
 *   stream_red (map(+)) over chunks, each chunk folding into a fresh
 *   zero accumulator in place                       Fig 4c, Fig 8
 *   seg_reduce / seg_scan = map (reduce/scan) over the rows of a regular
 *   [nseg][seglen] array ("segmented" scan/reduce)  footnote 5 L1230-1233
 *   transpose_2d = rearrange (1,0) / as_column_major             L1389-1393, L1431
 *
 * Operator readings:
 *   - integer ADD wraps modulo 2^32 / 2^64 (two's complement);
 *   - neutral elements: ADD 0, MIN +inf / INT_MAX, MAX -inf / INT_MIN,
 *     ARGMIN (MIN's neutral, index -1);
 *   - ARGMIN is the lexicographic minimum of (value, index): among equal
 *     values the smallest index wins (first occurrence);
 *   - all operators are associative and commutative, so kernels may
 *     reassociate and reorder (footnote 4 L1020, L1137-1139); f32 ADD results
 *     are therefore equal to the exact sum only up to rounding;
 *   - inputs are NaN-free (results unspecified otherwise).
 *
 * Conventions for every entry point:
 *   - Ownership: the caller owns every buffer.  Pointers named in/out/ws are
 *     DEVICE pointers on the current CUDA device; the library never allocates
 *     or frees (allocation hoisting, L440-442).
 *   - Freshness: outputs are fresh (L705-708, L537-539): an output range that
 *     overlaps an input range is rejected with FS_ERR_ALIAS before any launch.
 *   - Asynchrony: every call enqueues its kernels on `stream` (a cudaStream_t,
 *     NULL = legacy default stream) and returns; results are valid in stream
 *     order.
 *   - Errors: FS_ERR_NULL / _SIZE / _UNSUPPORTED / _ALIAS / _WORKSPACE are
 *     detected on the host before any launch (no side effects).  FS_ERR_CUDA
 *     reports a failed launch.  Device-side precondition violations (a
 *     stream_red key outside [0,k)) set an error word in the workspace that
 *     fs_check_device_error() reports (L429-432: bounds checks).
 *   - Workspace: `ws` is a device buffer of at least the size the matching
 *     fs_*_workspace() query returns.  It must be zero-filled once before its
 *     first use; every successful call leaves it ready for the next one.  One
 *     workspace must not be used by two calls that may run concurrently.
 *   - Empty inputs are legal: n = 0 reduces to 0(+) (index -1); seglen = 0
 *     gives nseg copies of 0(+); a scan of nothing writes nothing.
 *   - Layout of a [nseg][seglen] input: FS_ROW_MAJOR puts element (s, j) at
 *     s*seglen + j; FS_COL_MAJOR at j*nseg + s (same type, other
 *     representation, L1429-1434).
 *   - ARGMIN outputs are zip/unzip split (L138-146): values in `out` (element
 *     dtype), int64 indices in `out_idx`.  Indices are global positions for
 *     redomap/scanomap and segment-local (0..seglen-1) for seg_*.
 */
#ifndef FUTSEG_H
#define FUTSEG_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum fs_dtype { FS_I32 = 0, FS_I64 = 1, FS_F32 = 2 } fs_dtype;

typedef enum fs_op { FS_ADD = 0, FS_MIN = 1, FS_MAX = 2, FS_ARGMIN = 3, FS_VADD = 4 } fs_op;

typedef enum fs_map_kind {
    FS_MAP_ID = 0,     /* f x = x                                               */
    FS_MAP_NN_DIST = 1 /* f (lat, lng) = sqrtf((lat-q0)^2 + (lng-q1)^2), every  */
                       /* f32 operation separately rounded (no FMA contraction). */
                       /* Rodinia NN (L1653-1656); inputs are SoA lat[], lng[]. */
} fs_map_kind;

typedef enum fs_layout { FS_ROW_MAJOR = 0, FS_COL_MAJOR = 1 } fs_layout;

typedef enum fs_status {
    FS_OK = 0,
    FS_ERR_NULL = 1,        /* a required pointer is NULL                        */
    FS_ERR_SIZE = 2,        /* negative size, or nseg*seglen / n*width overflows */
    FS_ERR_UNSUPPORTED = 3, /* (op, dtype, map, primitive) not in the table      */
    FS_ERR_ALIAS = 4,       /* an output range overlaps an input range           */
    FS_ERR_WORKSPACE = 5,   /* ws is NULL or smaller than the query's answer     */
    FS_ERR_CUDA = 6,        /* a CUDA launch or runtime call failed              */
    FS_ERR_BOUNDS = 7       /* device-side precondition violation (stream_red)   */
} fs_status;

/* Operator descriptor.  width = k for FS_VADD (vectors of k elements), else 1. */
typedef struct fs_opdesc {
    int32_t op;    /* fs_op    */
    int32_t dtype; /* fs_dtype */
    int64_t width;
} fs_opdesc;

/* Map descriptor for the fused map stage of redomap / scanomap. */
typedef struct fs_mapdesc {
    int32_t kind;  /* fs_map_kind */
    float q0, q1;  /* FS_MAP_NN_DIST query point (lat, lng); ignored otherwise */
    int64_t ibase; /* global index of in0[0]: ARGMIN indices are ibase + position */
                   /* (a shard of a larger array, see the multi-GPU layer); 0 */
                   /* for a whole array.                                        */
} fs_mapdesc;

/* ---------------------------------------------------------------- workspace */
/* Each query writes the workspace size (bytes) the matching call needs on the
 * CURRENT device (it depends on the SM count) for the given sizes. */
fs_status fs_redomap_workspace(fs_opdesc op, int64_t n, size_t *bytes);
fs_status fs_scanomap_workspace(fs_opdesc op, int64_t n, size_t *bytes);
fs_status fs_seg_reduce_workspace(fs_opdesc op, int64_t nseg, int64_t seglen, int32_t layout,
                                  size_t *bytes);
fs_status fs_seg_scan_workspace(fs_opdesc op, int64_t nseg, int64_t seglen, int32_t layout,
                                size_t *bytes);
fs_status fs_stream_red_workspace(int32_t dtype, int64_t n, int64_t w, int64_t k, size_t *bytes);

/* ---------------------------------------------------------------- redomap */
/* out = 0(+) (+) f(x_0) (+) ... (+) f(x_{n-1})       (fold, L240-241; F3 L1067)
 *   op.op in {ADD, MIN, MAX, ARGMIN, VADD}; op.dtype in {I32, I64, F32}.
 *   map.kind == FS_MAP_ID      : in0 = x, n elements of op.dtype (VADD: [n][width]
 *                                row-major, n rows); in1 must be NULL.
 *   map.kind == FS_MAP_NN_DIST : in0 = lat[n], in1 = lng[n] (f32); op.dtype must be
 *                                F32 and op.op in {ADD, MIN, MAX, ARGMIN}.
 *   out     : 1 element of op.dtype (VADD: width elements).
 *   out_idx : ARGMIN only, 1 int64 (global index of the first minimum; -1 if n == 0).
 * VADD(width) is the vectorised operator map(+) of Fig 4b; with op.op == VADD the
 * result is the column sums of the [n][width] input (G5, L1313-1319). */
fs_status fs_redomap(fs_opdesc op, fs_mapdesc map, const void *in0, const void *in1, int64_t n,
                     void *out, int64_t *out_idx, void *ws, size_t ws_bytes, void *stream);

/* ---------------------------------------------------------------- scanomap */
/* out[i] = c (+) f(x_0) (+) ... (+) f(x_i)  for i < n   (scan L129-130; F5 L1071-1074)
 *   Same op/map/input rules as fs_redomap, except op.op != VADD.
 *   out: n elements of op.dtype; out_idx: ARGMIN only, n int64.
 *   carry / carry_idx: optional DEVICE pointers to one element (and, for ARGMIN,
 *   one int64 index) folded in front of the scan: c.  NULL means c = 0(+).
 *   (Used to continue a scan across shards: F5's accumulator a.)
 * Single-pass chained scan with decoupled look-back (add/min/max on 16-byte aligned
 * buffers: the ring scan, every tile held in shared memory between its read and its
 * write); the workspace holds the per-tile status words and is re-initialised by every
 * call. */
fs_status fs_scanomap(fs_opdesc op, fs_mapdesc map, const void *in0, const void *in1, int64_t n,
                      void *out, int64_t *out_idx, const void *carry, const int64_t *carry_idx,
                      void *ws, size_t ws_bytes, void *stream);

/* ---------------------------------------------------------------- combine */
/* out = parts[0] (+) parts[1] (+) ... (+) parts[P-1], in that order.
 *   The final combine of per-chunk / per-GPU partial results (sFold's outer
 *   (+), L259-260; stream_red's reduction across chunks, L1004-1006).
 *   parts: P elements of op.dtype (VADD: [P][width]); part_idx: ARGMIN only, the
 *   P partial indices (global positions).  P = 0 gives 0(+).  No workspace. */
fs_status fs_combine(fs_opdesc op, const void *parts, const int64_t *part_idx, int64_t P, void *out,
                     int64_t *out_idx, void *stream);

/* ---------------------------------------------------------------- cross-GPU exchange */
/* The per-GPU halves of the multi-GPU combine (north_star "combined with one
 * NCCL allreduce"): a rank's partial results are packed into ONE buffer of one reducible type
 * so that each exchange of the multi-GPU layer is a single collective, then unpacked.
 *
 * fs_argmin_pack: for ARGMIN partials (value, global index) of dtype I32 / F32, keys[i] =
 *   int64 whose signed order is the lexicographic (value, index) order of reading R3 (index -1,
 *   "no element", orders last): one all_reduce MIN over the ranks is the exact global argmin.
 *   Requires -1 <= idx < 2^32 - 1.  For I64 values keys is [n][2] = (value, index) records,
 *   to be all_gathered.
 * fs_argmin_unpack: I32 / F32: decodes ONE reduced key (P must be 1) into value / idx (the
 *   neutral element (+inf or INT32_MAX, -1) when no rank had an element).  I64: folds the P
 *   gathered records in rank order with R3's operator.
 *   values, idx, keys: device pointers; no workspace; FS_ERR_SIZE, _NULL, _UNSUPPORTED, _ALIAS. */
fs_status fs_argmin_pack(int32_t dtype, const void *values, const int64_t *idx, int64_t n, int64_t *keys,
                         void *stream);
fs_status fs_argmin_unpack(int32_t dtype, const int64_t *keys, int64_t P, void *value, int64_t *idx,
                           void *stream);
/* fs_partials_pack: packed[0 .. k*w) = sums, [k*w .. k*w+k) = counts (0 when counts is NULL),
 *   packed[k*w+k] = *extra (0 when NULL, e.g. the k-means delta): 8-byte elements, f64 for
 *   F32 sums (exact widening; counts exact below 2^53) and int64 for I32 / I64 sums (I32
 *   sign-extended).  One all_reduce SUM of the packed buffer combines the ranks' partials
 *   (Fig 4c's map(+) across chunks, L526-531); integer sums stay exact modulo 2^32 / 2^64 (R1).
 * fs_partials_unpack: the inverse after the reduction: F32 sums rounded once from the f64
 *   total, I32 sums the low 32 bits, counts / extra converted back.  sums [k][w] of dtype,
 *   counts [k] int32, extra int64; counts / extra may be NULL. */
fs_status fs_partials_pack(int32_t dtype, const void *sums, const int32_t *counts, const int64_t *extra, int64_t k,
                           int64_t w, void *packed, void *stream);
fs_status fs_partials_unpack(int32_t dtype, const void *packed, int64_t k, int64_t w, void *sums, int32_t *counts,
                             int64_t *extra, void *stream);
/* fs_copy_2d: dst[r*dst_ld + c] = src[r*src_ld + c] for r < rows, c < cols, elements of
 *   elem_bytes (4 or 8): the column-block gather of the distributed transpose (rearrange (1,0)
 *   of a row-sharded matrix, L1389-1393).  src and dst must not overlap (FS_ERR_ALIAS). */
fs_status fs_copy_2d(int32_t elem_bytes, const void *src, int64_t src_ld, int64_t rows, int64_t cols, void *dst,
                     int64_t dst_ld, void *stream);

/* ---------------------------------------------------------------- stream_red */
/* The K-means centre update (Fig 4c; Sec. 2.4; L1649):
 *   sums[c][j] = sum of vals[i][j] over i with keys[i] == c      (c < k, j < w)
 *   counts[c]  = #{ i : keys[i] == c }
 * computed as stream_red (map(+)): the input is split into chunks; each chunk
 * folds its rows into a fresh zero [k][w] accumulator updated in place, and the
 * chunk results are combined with the vectorised add (L526-531).
 *   dtype in {I32, I64, F32} (vals and sums); keys are int32; counts int32 (wraps).
 *   vals: [n][w] row-major; sums: [k][w]; counts may be NULL.
 *   Outputs are overwritten (each chunk starts from the neutral zeros; no
 *   user-supplied initial accumulator).  A key outside [0, k) is skipped and
 *   raises the device error word (fs_check_device_error -> FS_ERR_BOUNDS). */
fs_status fs_stream_red(int32_t dtype, const void *vals, const int32_t *keys, int64_t n, int64_t w,
                        int64_t k, void *sums, int32_t *counts, void *ws, size_t ws_bytes,
                        void *stream);

/* ---------------------------------------------------------------- segmented */
/* out[s] = reduce (+) 0(+) xss[s]  for s < nseg  (footnote 5; G5; Fig 11)
 *   xss is the logical [nseg][seglen] array stored in `in` with `layout`.
 *   op.op in {ADD, MIN, MAX, ARGMIN}; out: nseg elements; out_idx: ARGMIN only
 *   (segment-local index).  The kernel is chosen by segment length
 *   (fs_seg_reduce_regime). */
fs_status fs_seg_reduce(fs_opdesc op, const void *in, int64_t nseg, int64_t seglen, int32_t layout,
                        void *out, int64_t *out_idx, void *ws, size_t ws_bytes, void *stream);

/* out = map (scan (+) 0(+)) xss: the inclusive scan of every row; out has the
 * shape and layout of in (footnote 5: a scan with a modified associative
 * operator).  op.op in {ADD, MIN, MAX, ARGMIN}; out_idx: ARGMIN only (nseg*seglen
 * int64, segment-local indices). */
fs_status fs_seg_scan(fs_opdesc op, const void *in, int64_t nseg, int64_t seglen, int32_t layout,
                      void *out, int64_t *out_idx, void *ws, size_t ws_bytes, void *stream);

/* ---------------------------------------------------------------- transpose */
/* out[j][i] = in[i][j] for an in : [rows][cols] row-major array of dtype
 * (4- or 8-byte elements); out : [cols][rows].  No workspace; no in-place. */
fs_status fs_transpose_2d(int32_t dtype, const void *in, int64_t rows, int64_t cols, void *out,
                          void *stream);

/* new_centres[c][j] = counts[c] > 0 ? sums[c][j] / counts[c] : centres[c][j] (R19): the
 * last step of fs_kmeans_step, on its own for sums and counts that were first combined
 * across GPUs (one all_reduce, multi-GPU layer).  k*d f32 / k int32, device pointers;
 * new_centres must not overlap the inputs.  No workspace. */
fs_status fs_kmeans_finish(const float *sums, const int32_t *counts, const float *centres, int64_t k, int64_t d,
                           float *new_centres, void *stream);

/* ---------------------------------------------------------------- NEXT-2: nn_knn */
/* Rodinia NN's kk nearest neighbours: "100 reduce operations for finding the
 * nearest neighbors", the reduce computing "both the minimal value and the
 * corresponding index" (L1653-1655; reading R16).  Defined as kk rounds of the
 * ARGMIN redomap over the NN distance map (R5), each round excluding the record
 * it found:
 *   (out_dist[r], out_idx[r]) = argmin over not-yet-chosen i of (dist(i), i)
 * i.e. the kk records with the smallest (distance, index), in ascending order.
 * Rounds beyond n give (+inf, -1) (the ARGMIN neutral element).
 *   lat, lng : n f32 records (device, 4-byte aligned); n < 2^32.
 *   out_dist : kk f32; out_idx : kk int64 (device); 0 <= kk <= 1024.
 * One launch (no host round trips between rounds).  Errors: FS_ERR_NULL,
 * FS_ERR_SIZE (n < 0, n >= 2^32, kk < 0 or kk > 1024), FS_ERR_ALIAS,
 * FS_ERR_WORKSPACE, FS_ERR_CUDA. */
fs_status fs_nn_knn_workspace(int64_t n, int64_t kk, size_t *bytes);
fs_status fs_nn_knn(const float *lat, const float *lng, int64_t n, float q0, float q1, int64_t kk,
                    float *out_dist, int64_t *out_idx, void *ws, size_t ws_bytes, void *stream);

/* ---------------------------------------------------------------- NEXT-1: kmeans_step */
/* One fused iteration of Rodinia's K-means (Sec. 2.4; the
 * assignment map fused into the centre stream_red, F6 L1075-1090):
 *   membership[i]  = argmin_c E(i, c), the first c on ties            (R3, R18)
 *   E(i, c)        = sum_j (x_ij - c_cj)^2 in f32, j in order, acc = fma(t, t, acc),
 *                    t = x_ij - c_cj (exactly this f32 sequence: membership is
 *                    bit-exact; the tensor-core ranking is certified by an error
 *                    bound and re-evaluated exactly for near-ties)
 *   sums[c][j]     = sum of x_ij over membership[i] == c, counts[c]   (Fig 4c)
 *   new_centres    = sums / counts; an empty cluster keeps its centre (R19)
 *   *delta         = #{ i : membership[i] != prev[i] } (0 when prev is NULL)
 *   points  : [n][d] f32 row-major, 16-byte aligned; centres : [k][d] f32.
 *   prev, membership, new_centres, delta : optional (NULL).
 *   1 <= k <= 32, 1 <= d <= 40 (else FS_ERR_UNSUPPORTED); n >= 0.
 * Outputs are overwritten; they must not overlap the inputs (FS_ERR_ALIAS). */
fs_status fs_kmeans_step_workspace(int64_t n, int64_t d, int64_t k, size_t *bytes);
fs_status fs_kmeans_step(const float *points, int64_t n, int64_t d, const float *centres, int64_t k,
                         const int32_t *prev, int32_t *membership, float *sums, int32_t *counts,
                         float *new_centres, int64_t *delta, void *ws, size_t ws_bytes, void *stream);

/* ---------------------------------------------------------------- NEXT-4: seg_map_reduce */
/* The horizontally fused row nest of L247-252,
 *     map (\row -> (map (\x -> x + c) row, reduce (+) 0 row)) matrix,
 * with the reduce from the operator table: for every row s of the row-major
 * [nseg][seglen] array `in`, in ONE read of the row,
 *   out_map[s][j] = in[s][j] + c          (I32/I64: c = c_int, wraps; F32: c = c_f32)
 *   out[s]        = reduce op 0(op) in[s] (the ORIGINAL row; ARGMIN: out_idx[s] is the
 *                                           row-local index, -1 for an empty row)
 *   op.op in {ADD, MIN, MAX, ARGMIN}; out_map has in's shape; no output may overlap an
 *   input or another output (FS_ERR_ALIAS). */
fs_status fs_seg_map_reduce_workspace(fs_opdesc op, int64_t nseg, int64_t seglen, size_t *bytes);
fs_status fs_seg_map_reduce(fs_opdesc op, const void *in, int64_t nseg, int64_t seglen, int64_t c_int, float c_f32,
                            void *out_map, void *out, int64_t *out_idx, void *ws, size_t ws_bytes, void *stream);

/* ---------------------------------------------------------------- NEXT-3: scan_reduce */
/* The stream_seq fusion of Fig 10 (L1158-1227; F4, F5, F7 of Fig 9):
 *     out = reduce red (scan (+) 0 x)
 * computed in ONE read without materialising the scan: chunks are summarised by the
 * fused (associative, non-commutative) pair operator and combined in index order.
 *   red in {FS_ADD (sum of the prefix sums), FS_MAX / FS_MIN (max / min prefix sum)};
 *   the scan operator is FS_ADD (others: FS_ERR_UNSUPPORTED); dtype I32/I64 or F32
 *   (reassociated; the cross-warp combine in f64).  out: 1 element of dtype; n = 0 gives
 *   red's neutral element.  Integer FS_ADD is exact under wrap-around; integer
 *   FS_MAX/FS_MIN are exact when no prefix sum overflows (precondition: the pair
 *   operator max(M1, A1 + M2) needs monotone addition). */
fs_status fs_scan_reduce_workspace(int32_t dtype, int64_t n, size_t *bytes);
fs_status fs_scan_reduce(int32_t scan_op, int32_t red_op, int32_t dtype, const void *in, int64_t n, void *out,
                         void *ws, size_t ws_bytes, void *stream);

/* ---------------------------------------------------------------- utilities */
/* Synchronises `stream`, reads and clears the device error word of `ws`.
 * Returns FS_ERR_BOUNDS if a kernel flagged a precondition violation. */
fs_status fs_check_device_error(void *ws, void *stream);

/* Run-time multi-versioning (the paper's future work, L1411-1418): the segmented
 * primitives pick a kernel by segment length.  Regime IDs (FS_REGIME_*):
 *   0 = KG0/KG1 short rows: power-of-two rows by in-lane + shuffle groups over
 *       16-byte loads (KG0), others thread/group per segment over a shared-memory
 *       tile (KG1)                                                     fs_seg_reduce
 *   1 = KG2 warp per segment                                            fs_seg_reduce
 *   2 = KG3 block per segment (at least 3 x SMs segments)              fs_seg_reduce
 *   3 = KG4 several blocks per segment, partials combined by the last   fs_seg_reduce
 *   4 = column kernels (FS_COL_MAJOR with nseg > 1 and seglen > 1)      both
 *   5 = single-pass segmented decoupled-look-back scan (the general case: argmin,
 *       carries, misaligned buffers, lengths no other regime takes).  add/min/max on
 *       16-byte aligned buffers run the ring scan (tiles held in a shared-memory TMA ring
 *       between read and write) and take every row longer than 4096 elements that KS2
 *       cannot stream by TMA (fewer than 1.7 x SMs rows, or L not a multiple of the
 *       16-byte vector); argmin runs the slab scan
 *   6 = empty input (nseg == 0 or seglen == 0: neutral fill / nothing)  both
 *   7 = KS0 power-of-two rows of <= 256 16-byte vectors (seglen <= 1024 f32/i32,
 *       512 i64), 16-byte aligned buffers: in-register + shuffle scan, a shared-memory
 *       combine across the warps of a CTA for rows longer than 32 vectors
 *   8 = KS1 rows of 2..32 elements that are not powers of two, op != ARGMIN, 16-byte
 *       aligned: 256 rows staged through shared memory, a thread scans a row.  Taken only
 *       when forced (fs_force_seg_regime): KS3's TMA ring is the plan's choice for these
 *       rows since round 2 (L = 3: 0.57 -> 0.83 of the HBM roofline)
 *   9 = KS2 rows of >= 4 chunks of 256 x R vectors (12288 f32/i32 add/min/max, 4096
 *       argmin, 2048 i64) when there are at least 1.7 x as many rows as SMs (in/out with
 *       the same 16-byte phase; add/min/max on aligned buffers only when L is a multiple
 *       of the vector, streamed by TMA): a CTA owns whole rows and scans them chunk by
 *       chunk with a running carry (no look-back)
 *  10 = KS0-BIG power-of-two rows of 2-8 CTA steps (256 < seglen/VEC <= 2048: 2048..8192
 *       f32/i32, 1024..4096 i64), 16-byte aligned: a CTA loads a whole row per step,
 *       warp 0 scans the warp totals
 *  11 = KS3 rows of 32 < seglen <= 16384 (8192 for i64; 4096 when the ring scan can run),
 *       op != ARGMIN, element-aligned,
 *       and rows of 2..32 elements (not powers of two) with 16-byte aligned input and
 *       output: R whole rows per CTA staged in shared memory (by TMA bulk copies through
 *       a 3-slot ring and TMA bulk stores when both buffers are 16-byte aligned and a tile
 *       of R rows is <= 72 KB), odd-length per-thread pieces, a CTA scan of the piece
 *       summaries (no look-back)
 *  12 = flat (unsegmented) scan per row: one row (nseg == 1); several rows only when
 *       forced (16-byte aligned; regime 5 is faster for a few long rows)
 * fs_seg_regime returns the regime a call with these sizes takes on the current device
 * when its buffers come from an allocator (16-byte aligned); misaligned views may take
 * 5 instead.  The row-major seg_scan plan is one function shared with the dispatcher.
 * Returns -1 for invalid arguments. */
int32_t fs_seg_regime(int32_t prim_is_scan, fs_opdesc op, int64_t nseg, int64_t seglen,
                      int32_t layout);

/* The regime the last fs_seg_reduce / fs_seg_scan call made BY THIS HOST THREAD actually
 * launched (-1 before any call).  Test aid: asserts that fs_seg_regime tells the truth. */
int32_t fs_last_seg_regime(void);

/* Testing / sweep aid: force a regime for subsequent calls in this process; -1
 * restores automatic selection.  0..3 force the FS_ROW_MAJOR seg_reduce regime;
 * 5 and 7..12 force a row-major seg_scan regime wherever its preconditions above hold
 * (elsewhere the automatic choice stands).
 * Also settable with the environment variable FUTSEG_FORCE_REGIME.  Returns
 * FS_ERR_UNSUPPORTED for other values. */
fs_status fs_force_seg_regime(int32_t regime);

const char *fs_status_string(fs_status s);
const char *fs_version(void);

/* Number of kernels this library has launched in this process (all devices,
 * all streams).  A benchmark reads it around its timed region. */
uint64_t fs_launch_count(void);

#ifdef __cplusplus
}
#endif
#endif /* FUTSEG_H */
