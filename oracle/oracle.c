/*
 * oracle/oracle.c -- sequential CPU oracle for the libfutseg hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.
 * It shares no code, header, table or constant with the CUDA path
 * (paper_conf_pldi_henriksenseho17_b200/csrc); it defines its own operator
 * table below.
 *
 * Every function is the plain definition of the SOAC it stands for, written
 * as a sequential left fold ("foldl") in index order:
 *   reduce  (+) 0 [a1..an] = 0 (+) a1 (+) ... (+) an          L127-128
 *   scan    (+) 0 [a1..an] = [a1, ..., a1 (+) ... (+) an]     L129-130 (inclusive)
 *   fold (+,0) g           = reduce (+,0) . map g             L240-241, L254
 *   stream_red for counts/sums (Fig 4a; Fig 4c)
 *   segmented reduce/scan  = map (reduce/scan) over rows      footnote 5 L1230-1233
 *   transpose / as_column_major                               L1389-1393, L1431
 * No blocking, fusion, chunking or reordering.
 *
 * Readings:
 *   R1 integer + wraps modulo 2^32 / 2^64 (computed in unsigned arithmetic).
 *   R2 f32 ADD accumulates in f64; the f64 result is returned (north_star:
 *      "within 1e-4 relative error of an f64-accumulated oracle").
 *   R3 ARGMIN is the lexicographic minimum of (value, index); index -1 means
 *      "no element" and is the neutral element's index.
 *   R4 neutral elements: ADD 0; MIN +inf / INT_MAX; MAX -inf / INT_MIN.
 *   R5 NN distance map: sqrtf((lat-q0)*(lat-q0) + (lng-q1)*(lng-q1)) with
 *      every operation separately rounded to f32 (built -ffp-contract=off).
 *
 * Build: gcc -O2 -ffp-contract=off -fno-fast-math -std=c11 -shared -fPIC (the
 * command is oracle/__init__.py build()).  -ffp-contract=off makes every a*b+c
 * below two roundings; the one fused multiply-add the oracle wants (R18,
 * orc_kmeans_step) is an explicit fmaf().  Status codes: 0 ok, 1 bad argument,
 * 2 key out of range.
 */
#include <math.h>
#include <stdint.h>
#include <string.h>

enum { ORC_I32 = 0, ORC_I64 = 1, ORC_F32 = 2 };
enum { ORC_ADD = 0, ORC_MIN = 1, ORC_MAX = 2, ORC_ARGMIN = 3 };
enum { ORC_ROW_MAJOR = 0, ORC_COL_MAJOR = 1 };

/* One accumulator value: `i` holds integer values (i32 sign-extended),
 * `f` holds f32 values widened exactly to double (and f64 sums), `idx` the
 * argmin index. */
typedef struct {
    int64_t i;
    double f;
    int64_t idx;
} val_t;

static int valid(int op, int dt) {
    return (dt == ORC_I32 || dt == ORC_I64 || dt == ORC_F32) &&
           (op == ORC_ADD || op == ORC_MIN || op == ORC_MAX || op == ORC_ARGMIN);
}

/* 0(+) for (op, dt): R4 / R3. */
static val_t neutral(int op, int dt) {
    val_t z;
    z.i = 0;
    z.f = 0.0;
    z.idx = -1;
    if (op == ORC_MIN || op == ORC_ARGMIN) {
        z.i = (dt == ORC_I32) ? INT32_MAX : INT64_MAX;
        z.f = INFINITY;
    } else if (op == ORC_MAX) {
        z.i = (dt == ORC_I32) ? INT32_MIN : INT64_MIN;
        z.f = -INFINITY;
    }
    return z;
}

static val_t load(int dt, const void *p, int64_t k, int64_t idx) {
    val_t v;
    v.i = 0;
    v.f = 0.0;
    v.idx = idx;
    if (dt == ORC_I32) v.i = ((const int32_t *)p)[k];
    else if (dt == ORC_I64) v.i = ((const int64_t *)p)[k];
    else v.f = (double)((const float *)p)[k];
    return v;
}

/* value comparison "a < b" in the element type */
static int less(int dt, val_t a, val_t b) {
    return (dt == ORC_F32) ? (a.f < b.f) : (a.i < b.i);
}

static int equal(int dt, val_t a, val_t b) {
    return (dt == ORC_F32) ? (a.f == b.f) : (a.i == b.i);
}

/* a (+) b for the operator table. */
static val_t combine(int op, int dt, val_t a, val_t b) {
    val_t r = a;
    switch (op) {
    case ORC_ADD:
        if (dt == ORC_I32) r.i = (int32_t)((uint32_t)a.i + (uint32_t)b.i);      /* R1 */
        else if (dt == ORC_I64) r.i = (int64_t)((uint64_t)a.i + (uint64_t)b.i); /* R1 */
        else r.f = a.f + b.f;                                                   /* R2 */
        return r;
    case ORC_MIN:
        return less(dt, b, a) ? b : a;
    case ORC_MAX:
        return less(dt, a, b) ? b : a;
    case ORC_ARGMIN: /* R3 */
        if (a.idx < 0) return b;
        if (b.idx < 0) return a;
        if (less(dt, b, a) || (equal(dt, b, a) && b.idx < a.idx)) return b;
        return a;
    }
    return r;
}

/* Output element type: f64 for f32 ADD (R2), else the element type. */
static void store(int op, int dt, void *out, int64_t k, val_t v, int64_t *out_idx) {
    if (dt == ORC_I32) ((int32_t *)out)[k] = (int32_t)v.i;
    else if (dt == ORC_I64) ((int64_t *)out)[k] = v.i;
    else if (op == ORC_ADD) ((double *)out)[k] = v.f;
    else ((float *)out)[k] = (float)v.f;
    if (op == ORC_ARGMIN && out_idx) out_idx[k] = v.idx;
}

/* reduce (+) 0(+) x  (L127-128): acc = 0(+); for i: acc = acc (+) x[i]. */
int orc_reduce(int op, int dt, const void *x, int64_t n, void *out, int64_t *out_idx) {
    if (!valid(op, dt) || n < 0 || (n > 0 && !x) || !out) return 1;
    val_t acc = neutral(op, dt);
    for (int64_t i = 0; i < n; ++i) acc = combine(op, dt, acc, load(dt, x, i, i));
    store(op, dt, out, 0, acc, out_idx);
    return 0;
}

/* scan (+) 0(+) x  (L129-130), inclusive: out[i] = x[0] (+) ... (+) x[i]. */
int orc_scan(int op, int dt, const void *x, int64_t n, void *out, int64_t *out_idx) {
    if (!valid(op, dt) || n < 0 || (n > 0 && (!x || !out))) return 1;
    val_t acc = neutral(op, dt);
    for (int64_t i = 0; i < n; ++i) {
        acc = combine(op, dt, acc, load(dt, x, i, i));
        store(op, dt, out, i, acc, out_idx);
    }
    return 0;
}

/* The NN map f (R5): out[i] = sqrtf((lat[i]-q0)^2 + (lng[i]-q1)^2) in f32. */
int orc_nn_dist(const float *lat, const float *lng, int64_t n, float q0, float q1, float *out) {
    if (n < 0 || (n > 0 && (!lat || !lng || !out))) return 1;
    for (int64_t i = 0; i < n; ++i) {
        float d0 = lat[i] - q0;
        float d1 = lng[i] - q1;
        float s0 = d0 * d0;
        float s1 = d1 * d1;
        float s = s0 + s1;
        out[i] = sqrtf(s);
    }
    return 0;
}

/* reduce (map (+)) (replicate w 0(+)) x over x : [m][w] row-major (Fig 4b
 * L474-480; G5 L1313-1319): acc[j] = acc[j] (+) (x[i][j], i) for i in order.
 * The argmin index is the row index i. */
int orc_vreduce(int op, int dt, const void *x, int64_t m, int64_t w, void *out, int64_t *out_idx) {
    if (!valid(op, dt) || m < 0 || w < 0 || (m > 0 && w > 0 && !x) || (w > 0 && !out)) return 1;
    for (int64_t j = 0; j < w; ++j) {
        val_t acc = neutral(op, dt);
        for (int64_t i = 0; i < m; ++i) acc = combine(op, dt, acc, load(dt, x, i * w + j, i));
        store(op, dt, out, j, acc, out_idx);
    }
    return 0;
}

/* Position of logical element (s, j) of a [nseg][seglen] array under the
 * representation `layout` (L1429-1434: column major changes the
 * representation, not the type). */
static int64_t pos(int layout, int64_t nseg, int64_t seglen, int64_t s, int64_t j) {
    return layout == ORC_ROW_MAJOR ? s * seglen + j : j * nseg + s;
}

/* map (reduce (+) 0(+)) xss  (footnote 5 L1230-1233; example L247-252).
 * The argmin index is segment-local (j). */
int orc_seg_reduce(int op, int dt, const void *x, int64_t nseg, int64_t seglen, int layout,
                   void *out, int64_t *out_idx) {
    if (!valid(op, dt) || nseg < 0 || seglen < 0 || (layout != ORC_ROW_MAJOR && layout != ORC_COL_MAJOR))
        return 1;
    if (nseg > 0 && (!out || (seglen > 0 && !x))) return 1;
    for (int64_t s = 0; s < nseg; ++s) {
        val_t acc = neutral(op, dt);
        for (int64_t j = 0; j < seglen; ++j)
            acc = combine(op, dt, acc, load(dt, x, pos(layout, nseg, seglen, s, j), j));
        store(op, dt, out, s, acc, out_idx);
    }
    return 0;
}

/* map (scan (+) 0(+)) xss; the output has the input's shape and layout. */
int orc_seg_scan(int op, int dt, const void *x, int64_t nseg, int64_t seglen, int layout,
                 void *out, int64_t *out_idx) {
    if (!valid(op, dt) || nseg < 0 || seglen < 0 || (layout != ORC_ROW_MAJOR && layout != ORC_COL_MAJOR))
        return 1;
    if (nseg > 0 && seglen > 0 && (!x || !out)) return 1;
    for (int64_t s = 0; s < nseg; ++s) {
        val_t acc = neutral(op, dt);
        for (int64_t j = 0; j < seglen; ++j) {
            int64_t k = pos(layout, nseg, seglen, s, j);
            acc = combine(op, dt, acc, load(dt, x, k, j));
            store(op, dt, out, k, acc, out_idx);
        }
    }
    return 0;
}

/* stream_red (map (+)) over one chunk = the sequential loop of Fig 4a
 * (L469-471) generalised from counts to per-cluster sums of w-vectors
 * (K-means new centres, L447-453, L1649):
 *   counts = replicate k 0; sums = replicate k (replicate w 0)
 *   for i < n: c = keys[i]; counts[c] += 1; sums[c][j] += vals[i][j]
 * f32 sums accumulate in f64 (R2) and are returned as f64; integer sums wrap
 * (R1).  A key outside [0,k) violates the precondition: returns 2.  */
int orc_stream_red(int dt, const void *vals, const int32_t *keys, int64_t n, int64_t w, int64_t k,
                   void *sums, int32_t *counts) {
    if (dt != ORC_I32 && dt != ORC_I64 && dt != ORC_F32) return 1;
    if (n < 0 || w < 0 || k < 0) return 1;
    if (n > 0 && (!keys || (w > 0 && !vals))) return 1;
    for (int64_t c = 0; c < k; ++c) {
        if (counts) counts[c] = 0;
        for (int64_t j = 0; j < w; ++j) {
            if (dt == ORC_I32) ((int32_t *)sums)[c * w + j] = 0;
            else if (dt == ORC_I64) ((int64_t *)sums)[c * w + j] = 0;
            else ((double *)sums)[c * w + j] = 0.0;
        }
    }
    for (int64_t i = 0; i < n; ++i) {
        int64_t c = keys[i];
        if (c < 0 || c >= k) return 2;
        if (counts) counts[c] = (int32_t)((uint32_t)counts[c] + 1u);
        for (int64_t j = 0; j < w; ++j) {
            if (dt == ORC_I32) {
                int32_t *s = &((int32_t *)sums)[c * w + j];
                *s = (int32_t)((uint32_t)*s + (uint32_t)((const int32_t *)vals)[i * w + j]);
            } else if (dt == ORC_I64) {
                int64_t *s = &((int64_t *)sums)[c * w + j];
                *s = (int64_t)((uint64_t)*s + (uint64_t)((const int64_t *)vals)[i * w + j]);
            } else {
                ((double *)sums)[c * w + j] += (double)((const float *)vals)[i * w + j];
            }
        }
    }
    return 0;
}

/* rearrange (1,0) / transpose (L1389-1393): out[j][i] = in[i][j]. */
int orc_transpose(int64_t esize, const void *in, int64_t rows, int64_t cols, void *out) {
    if (esize <= 0 || rows < 0 || cols < 0) return 1;
    if (rows > 0 && cols > 0 && (!in || !out)) return 1;
    const char *src = (const char *)in;
    char *dst = (char *)out;
    for (int64_t i = 0; i < rows; ++i)
        for (int64_t j = 0; j < cols; ++j)
            memcpy(dst + (j * rows + i) * esize, src + (i * cols + j) * esize, (size_t)esize);
    return 0;
}

/* NEXT-2, Rodinia NN's "100 reduce operations for finding the nearest
 * neighbors" (L1653-1655; reading R16): kk rounds of the argmin reduce of
 * R3 over the distance map of R5, each round excluding the record it found.
 *   round r: (out_dist[r], out_idx[r]) = argmin over not-yet-chosen i of
 *            (dist[i], i), first occurrence among equal distances;
 *   rounds beyond n give (+inf, -1) (the argmin neutral element, R3/R4).
 * O(kk * n) by design: this is the repeated reduce the paper describes, not
 * a selection algorithm.  dist_scratch: n floats; chosen_scratch: n bytes. */
int orc_nn_knn(const float *lat, const float *lng, int64_t n, float q0, float q1, int64_t kk,
               float *out_dist, int64_t *out_idx, float *dist_scratch, unsigned char *chosen_scratch) {
    if (n < 0 || kk < 0 || (n > 0 && (!lat || !lng || !dist_scratch || !chosen_scratch)) ||
        (kk > 0 && (!out_dist || !out_idx)))
        return 1;
    orc_nn_dist(lat, lng, n, q0, q1, dist_scratch);
    memset(chosen_scratch, 0, (size_t)n);
    for (int64_t r = 0; r < kk; ++r) {
        float best = INFINITY;
        int64_t bi = -1;
        for (int64_t i = 0; i < n; ++i) {
            if (chosen_scratch[i]) continue;
            if (bi < 0 || dist_scratch[i] < best) {  /* strict <: first occurrence wins ties */
                best = dist_scratch[i];
                bi = i;
            }
        }
        out_dist[r] = best;
        out_idx[r] = bi;
        if (bi >= 0) chosen_scratch[bi] = 1;
    }
    return 0;
}

/* NEXT-1, one iteration of Rodinia's K-means (Sec. 2.4; Fig 4; L1628-1649):
 *   assignment  membership[i] = argmin_c E(i, c), the first c on ties (R3), with
 *               E(i, c) = sum over j = 0..d-1, in order, of (x_ij - c_cj)^2 computed
 *               in f32 as acc = fmaf(t, t, acc), t = x_ij - c_cj (reading R18:
 *               Rodinia's squared Euclidean distance, one rounding per fma);
 *   new centres sums[c][j] = sum of x_ij over membership[i] == c (f64, R2),
 *               counts[c]; new_centres[c][j] = sums/counts when counts > 0, else
 *               the old centre (reading R19) -- the segmented reduction of L1649;
 *   delta       #{ i : membership[i] != prev[i] } (Rodinia's convergence test),
 *               only if prev != NULL.
 * Straight loops in index order; sums/new_centres are f64.  */
int orc_kmeans_step(const float *x, int64_t n, int64_t d, const float *cen, int64_t k, const int32_t *prev,
                    int32_t *membership, double *sums, int32_t *counts, double *new_cen, int64_t *delta) {
    if (n < 0 || d < 1 || k < 1 || (n > 0 && (!x || !membership)) || !cen || !sums || !counts || !new_cen)
        return 1;
    int64_t changed = 0;
    for (int64_t c = 0; c < k; ++c) {
        counts[c] = 0;
        for (int64_t j = 0; j < d; ++j) sums[c * d + j] = 0.0;
    }
    for (int64_t i = 0; i < n; ++i) {
        float best = 0.0f;
        int32_t bc = -1;
        for (int64_t c = 0; c < k; ++c) {
            float acc = 0.0f;
            for (int64_t j = 0; j < d; ++j) {
                const float t = x[i * d + j] - cen[c * d + j];
                acc = fmaf(t, t, acc);
            }
            if (bc < 0 || acc < best) { /* strict <: first centre wins ties */
                best = acc;
                bc = (int32_t)c;
            }
        }
        membership[i] = bc;
        if (prev && prev[i] != bc) ++changed;
        counts[bc] += 1;
        for (int64_t j = 0; j < d; ++j) sums[bc * d + j] += (double)x[i * d + j];
    }
    for (int64_t c = 0; c < k; ++c)
        for (int64_t j = 0; j < d; ++j)
            new_cen[c * d + j] = counts[c] > 0 ? sums[c * d + j] / (double)counts[c] : (double)cen[c * d + j];
    if (delta) *delta = prev ? changed : 0;
    return 0;
}

/* NEXT-4, the horizontally fused row nest of L247-252:
 *     map (\row -> (map (\x -> x + c) row, reduce (+) 0 row)) matrix
 * generalised to the operator table for the reduce: for every row s of the
 * row-major [nseg][seglen] x,
 *     out_map[s][j] = x[s][j] + c    (i32/i64: wraps, R1; f32: one f32 add)
 *     out_red[s]    = reduce op 0(op) x[s]   (over the ORIGINAL row, as in L250)
 * c is ci for integer types and cf for f32.  Straight loops, no fusion. */
int orc_seg_map_reduce(int op, int dt, const void *x, int64_t nseg, int64_t seglen, int64_t ci, float cf,
                       void *out_map, void *out_red, int64_t *out_idx) {
    if (!valid(op, dt) || nseg < 0 || seglen < 0) return 1;
    if (nseg > 0 && seglen > 0 && (!x || !out_map)) return 1;
    for (int64_t e = 0; e < nseg * seglen; ++e) {
        if (dt == ORC_F32) {
            ((float *)out_map)[e] = ((const float *)x)[e] + cf;
        } else if (dt == ORC_I32) {
            ((int32_t *)out_map)[e] = (int32_t)((uint32_t)((const int32_t *)x)[e] + (uint32_t)ci);
        } else {
            ((int64_t *)out_map)[e] = (int64_t)((uint64_t)((const int64_t *)x)[e] + (uint64_t)ci);
        }
    }
    return orc_seg_reduce(op, dt, x, nseg, seglen, ORC_ROW_MAJOR, out_red, out_idx);
}

/* NEXT-3, Fig 10a (L1158-1170) with g = id: the scan is materialised and reduced,
 *     y = scan (scan_op) x;   out = reduce (red_op) y
 * exactly the unfused program (F5 and F4 fuse it into one stream_seq, F7; the
 * library computes the fused form).  f32 in f64 (R2; the result is returned as a
 * double), integers wrap (R1). */
int orc_scan_reduce(int scan_op, int red_op, int dt, const void *x, int64_t n, void *out) {
    if (!valid(scan_op, dt) || !valid(red_op, dt) || scan_op == ORC_ARGMIN || red_op == ORC_ARGMIN || n < 0 ||
        !out || (n > 0 && !x))
        return 1;
    val_t s = neutral(scan_op, dt), r = neutral(red_op, dt);
    for (int64_t i = 0; i < n; ++i) {
        s = combine(scan_op, dt, s, load(dt, x, i, i));  /* y[i] */
        val_t y = s;
        y.idx = i;
        r = combine(red_op, dt, r, y);
    }
    if (dt == ORC_F32) ((double *)out)[0] = r.f;  /* f64 for f32 (R2), whatever red_op */
    else store(red_op, dt, out, 0, r, 0);
    return 0;
}
