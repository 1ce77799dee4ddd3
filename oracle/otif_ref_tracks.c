/*
 * otif_ref_tracks.c — CPU ORACLE for NEXT-4, track refinement.
 *
 * TEST INFRASTRUCTURE ONLY (see otif_ref.h).  Plain C99, single-threaded, following the
 * paper's paragraph on refinement step by step:
 *   1. resample every track to N evenly spaced points,
 *   2. d(s1, s2) = mean Euclidean distance between corresponding points,
 *   3. DBSCAN over S* with that distance,
 *   4. cluster centres = per-index mean point,
 *   5. per query: centres passing close to d1 and dn, the k = 10 closest, and start/end =
 *      the size-weighted median of their start/end points.
 * Readings where the paragraph is silent: DESIGN.md R20–R25.  Built with
 * -ffp-contract=off so every float/double operation is one IEEE rounding, in the order
 * written here; decisions (d <= eps, the k nearest) are taken in fp32, the kernel's
 * precision.  The "spatial index" of P:L200 is a speed device, not a result: here it is
 * the plain predicate it evaluates (reading R24).
 */
#include "otif_ref.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>

/* ------------------------------------------------------------------------- */
/* Step 1 — P:L196: "we compute N points evenly spaced along each track".
 * Reading R21: evenly spaced in arc length along the polyline through the detections,
 * both endpoints included.  cum_0 = 0, cum_{j+1} = cum_j + |p_{j+1} − p_j| (fp64, in
 * order); L = cum_{n−1}; point i (0 < i < N−1) sits at s = (L·i)/(N−1) on the first
 * segment j with cum_{j+1} >= s, at t = min((s − cum_j)/seg_j, 1); point 0 is p_0 and
 * point N−1 is p_{n−1}.  A single-detection or zero-length track repeats p_0.         */
static void resample_one(const float *p, int64_t n, int32_t N, float *out) {
    double *seg = (double *)malloc((size_t)(n > 1 ? n - 1 : 1) * sizeof(double));
    double *cum = (double *)malloc((size_t)n * sizeof(double));
    cum[0] = 0.0;
    for (int64_t j = 0; j + 1 < n; j++) {
        double dx = (double)p[2 * (j + 1)] - (double)p[2 * j];
        double dy = (double)p[2 * (j + 1) + 1] - (double)p[2 * j + 1];
        seg[j] = sqrt(dx * dx + dy * dy);
        cum[j + 1] = cum[j] + seg[j];
    }
    double L = cum[n - 1];
    for (int32_t i = 0; i < N; i++) {
        if (n == 1 || L == 0.0 || i == 0) {
            out[2 * i] = p[0];
            out[2 * i + 1] = p[1];
            continue;
        }
        if (i == N - 1) {
            out[2 * i] = p[2 * (n - 1)];
            out[2 * i + 1] = p[2 * (n - 1) + 1];
            continue;
        }
        double s = (L * (double)i) / (double)(N - 1);
        int64_t j = 0;
        while (cum[j + 1] < s) j++;
        double t = (s - cum[j]) / seg[j];
        if (t > 1.0) t = 1.0;
        double x = (double)p[2 * j] + t * ((double)p[2 * (j + 1)] - (double)p[2 * j]);
        double y = (double)p[2 * j + 1] + t * ((double)p[2 * (j + 1) + 1] - (double)p[2 * j + 1]);
        out[2 * i] = (float)x;
        out[2 * i + 1] = (float)y;
    }
    free(seg);
    free(cum);
}

int otif_ref_track_resample(const float *pts, const int64_t *offsets, int64_t n, int32_t npts, float *out) {
    if (n < 0 || npts < 2) return -1;
    for (int64_t t = 0; t < n; t++) {
        int64_t len = offsets[t + 1] - offsets[t];
        if (len < 1) return -1;
        resample_one(pts + 2 * offsets[t], len, npts, out + (size_t)t * npts * 2);
    }
    return 0;
}

/* ------------------------------------------------------------------------- */
/* Step 2 — P:L196: d(s1, s2) = (1/N) Σ_{i=1..N} eucl(P(s1)[i], P(s2)[i]).  Reading R22:
 * fp32, eucl = sqrt(dx² + dy²), summed in index order, then divided by N.             */
float otif_ref_track_distance(const float *a, const float *b, int32_t npts) {
    float sum = 0.0f;
    for (int32_t i = 0; i < npts; i++) {
        float dx = a[2 * i] - b[2 * i];
        float dy = a[2 * i + 1] - b[2 * i + 1];
        float e = sqrtf(dx * dx + dy * dy);
        sum = sum + e;
    }
    return sum / (float)npts;
}

/* ------------------------------------------------------------------------- */
/* Step 3 — P:L198: "we begin by clustering the tracks in S* using DBSCAN".  Reading
 * R23 (the classic algorithm, processed in index order): eps-neighbourhoods include the
 * track itself; a core track has >= min_pts neighbours; a cluster is started at the
 * lowest-index unlabelled core track and grown through core tracks; a non-core track
 * with a core neighbour is a border track of the earliest such cluster; else noise. */
int32_t otif_ref_dbscan(const float *P, int64_t n, int32_t npts, float eps, int32_t min_pts, int32_t *labels,
                        uint8_t *core_out) {
    if (n < 0 || npts < 2 || min_pts < 1) return -1;
    size_t stride = (size_t)npts * 2;
    uint8_t *core = (uint8_t *)calloc((size_t)(n > 0 ? n : 1), 1);
    int64_t *queue = (int64_t *)malloc((size_t)(n > 0 ? n : 1) * sizeof(int64_t));
    for (int64_t i = 0; i < n; i++) {
        int64_t cnt = 0;
        for (int64_t j = 0; j < n; j++)
            if (otif_ref_track_distance(P + i * stride, P + j * stride, npts) <= eps) cnt++;
        core[i] = cnt >= min_pts;
        labels[i] = -1;
    }
    int32_t nc = 0;
    for (int64_t i = 0; i < n; i++) {
        if (!core[i] || labels[i] != -1) continue;
        int64_t head = 0, tail = 0;
        labels[i] = nc;
        queue[tail++] = i;
        while (head < tail) {
            int64_t u = queue[head++];
            for (int64_t v = 0; v < n; v++) {
                if (!core[v] || labels[v] != -1) continue;
                if (otif_ref_track_distance(P + u * stride, P + v * stride, npts) <= eps) {
                    labels[v] = nc;
                    queue[tail++] = v;
                }
            }
        }
        nc++;
    }
    for (int64_t i = 0; i < n; i++) {
        if (core[i]) continue;
        int32_t best = -1;
        for (int64_t j = 0; j < n; j++) {
            if (!core[j]) continue;
            if (otif_ref_track_distance(P + i * stride, P + j * stride, npts) <= eps &&
                (best < 0 || labels[j] < best))
                best = labels[j];
        }
        labels[i] = best;
    }
    if (core_out) memcpy(core_out, core, (size_t)n);
    free(core);
    free(queue);
    return nc;
}

/* ------------------------------------------------------------------------- */
/* Step 4 — P:L198: centre of a cluster c = the path of N points p_i = mean of
 * {P(s)[i] | s ∈ c}.  fp64 sum over members in index order, / count, rounded to fp32. */
int otif_ref_track_centers(const float *P, const int32_t *labels, int64_t n, int32_t npts, int32_t nc,
                           float *centers, int32_t *sizes) {
    if (n < 0 || npts < 2 || nc < 0) return -1;
    size_t stride = (size_t)npts * 2;
    double *sum = (double *)malloc(stride * sizeof(double));
    for (int32_t c = 0; c < nc; c++) {
        int64_t cnt = 0;
        for (size_t q = 0; q < stride; q++) sum[q] = 0.0;
        for (int64_t i = 0; i < n; i++) {
            if (labels[i] != c) continue;
            cnt++;
            for (size_t q = 0; q < stride; q++) sum[q] = sum[q] + (double)P[i * stride + q];
        }
        sizes[c] = (int32_t)cnt;
        for (size_t q = 0; q < stride; q++)
            centers[(size_t)c * stride + q] = cnt ? (float)(sum[q] / (double)cnt) : 0.0f;
    }
    free(sum);
    return 0;
}

/* ------------------------------------------------------------------------- */
/* Step 5 — P:L200.  eucl in fp32 as in step 2.                                       */
static float eucl32(float ax, float ay, float bx, float by) {
    float dx = ax - bx;
    float dy = ay - by;
    return sqrtf(dx * dx + dy * dy);
}

/* "several cluster centers that pass close to d1 and dn" (reading R24): some point of
 * the centre within rho of d1 and some point within rho of dn.                        */
static int passes_close(const float *center, int32_t npts, float x, float y, float rho) {
    for (int32_t i = 0; i < npts; i++)
        if (eucl32(center[2 * i], center[2 * i + 1], x, y) <= rho) return 1;
    return 0;
}

typedef struct { float d; int32_t c; } cand_t;
typedef struct { float v; int32_t w; } wval_t;

static int cmp_cand(const void *a, const void *b) {
    const cand_t *x = (const cand_t *)a, *y = (const cand_t *)b;
    if (x->d < y->d) return -1;
    if (x->d > y->d) return 1;
    return (x->c > y->c) - (x->c < y->c);
}

static int cmp_wval(const void *a, const void *b) {
    const wval_t *x = (const wval_t *)a, *y = (const wval_t *)b;
    return (x->v > y->v) - (x->v < y->v);
}

/* Reading R25: the lower weighted median — sort by value, the first value whose
 * cumulative weight reaches half the total (2·cum >= total).                          */
static float weighted_median(wval_t *vals, int32_t cnt) {
    qsort(vals, (size_t)cnt, sizeof(wval_t), cmp_wval);
    int64_t total = 0, cum = 0;
    for (int32_t l = 0; l < cnt; l++) total += vals[l].w;
    for (int32_t l = 0; l < cnt; l++) {
        cum += vals[l].w;
        if (2 * cum >= total) return vals[l].v;
    }
    return vals[cnt - 1].v;
}

int otif_ref_track_refine(const float *pts, const int64_t *offsets, int64_t m, int32_t npts, const float *centers,
                          const int32_t *sizes, int32_t nc, int32_t k, float rho, float *out, int32_t *used) {
    if (m < 0 || npts < 2 || nc < 0 || k < 1) return -1;
    size_t stride = (size_t)npts * 2;
    float *Pq = (float *)malloc(stride * sizeof(float));
    cand_t *cand = (cand_t *)malloc((size_t)(nc > 0 ? nc : 1) * sizeof(cand_t));
    wval_t *vals = (wval_t *)malloc((size_t)k * sizeof(wval_t));
    for (int64_t q = 0; q < m; q++) {
        int64_t len = offsets[q + 1] - offsets[q];
        if (len < 1) { free(Pq); free(cand); free(vals); return -1; }
        const float *p = pts + 2 * offsets[q];
        float x1 = p[0], y1 = p[1], xn = p[2 * (len - 1)], yn = p[2 * (len - 1) + 1];
        resample_one(p, len, npts, Pq);
        int32_t nk = 0;
        for (int32_t c = 0; c < nc; c++) {
            const float *cc = centers + (size_t)c * stride;
            if (rho > 0.0f && !(passes_close(cc, npts, x1, y1, rho) && passes_close(cc, npts, xn, yn, rho)))
                continue;
            cand[nk].d = otif_ref_track_distance(Pq, cc, npts);
            cand[nk].c = c;
            nk++;
        }
        qsort(cand, (size_t)nk, sizeof(cand_t), cmp_cand);
        if (nk > k) nk = k;
        used[q] = nk;
        if (nk == 0) {
            out[4 * q] = x1; out[4 * q + 1] = y1; out[4 * q + 2] = xn; out[4 * q + 3] = yn;
            continue;
        }
        for (int e = 0; e < 4; e++) {
            /* e = 0,1: start x, y (centre point 0); e = 2,3: end x, y (centre point N−1) */
            size_t off = (e < 2) ? (size_t)(e & 1) : (size_t)(2 * (npts - 1) + (e & 1));
            for (int32_t l = 0; l < nk; l++) {
                vals[l].v = centers[(size_t)cand[l].c * stride + off];
                vals[l].w = sizes[cand[l].c];
            }
            out[4 * q + e] = weighted_median(vals, nk);
        }
    }
    free(Pq);
    free(cand);
    free(vals);
    return 0;
}
