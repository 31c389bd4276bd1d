/*
 * oracle.c — CPU ORACLE: TEST INFRASTRUCTURE ONLY (see oracle.h).
 *
 * Plain serial evaluation of the original stencil program, written to be
 * checked against PAPER.md by eye.  No blocking, no fusion, no reordering:
 *
 *   for each statement S in program order           (OEG order, §3.2.3;
 *                                                     statement-wise = kernel-wise
 *                                                     under reading R3)
 *     for k, j, i over the interior (∩ box)          (R1, R2)
 *                 ∩ the statement's loop bounds      (R2': kernels with shorter loops)
 *       acc = T(S.term[0]); acc = acc + T(S.term[t]) (R4: fixed left-to-right order)
 *       S.out[i,j,k] = acc
 *
 * Build: gcc -O2 -ffp-contract=off -fPIC -shared (no -ffast-math).
 */
#include "oracle.h"

#include <stddef.h>

typedef struct {
    long sx, sy, sz; /* element strides: 1, row, plane */
    long base;       /* offset of interior point (0,0,0) */
} or_layout;

static or_layout layout_of(const or_grid *g) {
    or_layout L;
    L.sx = 1;
    L.sy = g->nx + 2L * g->hx;
    L.sz = L.sy * (g->ny + 2L * g->hy);
    L.base = (long)g->hz * L.sz + (long)g->hy * L.sy + (long)g->hx;
    return L;
}

/* A tap may reach at most the ghost width (the caller allocated nothing beyond). */
static int tap_ok(const or_grid *g, int n_arrays, const or_tap *t) {
    if (t->arr < 0 || t->arr >= n_arrays) return 0;
    if (t->dx < -g->hx || t->dx > g->hx) return 0;
    if (t->dy < -g->hy || t->dy > g->hy) return 0;
    if (t->dz < -g->hz || t->dz > g->hz) return 0;
    return 1;
}

static int program_ok(const or_grid *g, int n_arrays, int n_stmts, const or_stmt *stmts) {
    for (int s = 0; s < n_stmts; ++s) {
        if (stmts[s].out < 0 || stmts[s].out >= n_arrays || stmts[s].n_terms < 1) return 0;
        for (int t = 0; t < stmts[s].n_terms; ++t) {
            const or_term *tm = &stmts[s].terms[t];
            if (!tap_ok(g, n_arrays, &tm->a)) return 0;
            if (tm->has_b && !tap_ok(g, n_arrays, &tm->b)) return 0;
        }
    }
    return 1;
}

static void clip_box(const or_grid *g, const long *box, long r[6]) {
    long full[6] = {0, g->nx, 0, g->ny, 0, g->nz};
    for (int d = 0; d < 3; ++d) {
        long lo = full[2 * d], hi = full[2 * d + 1];
        if (box) {
            if (box[2 * d] > lo) lo = box[2 * d];
            if (box[2 * d + 1] < hi) hi = box[2 * d + 1];
        }
        r[2 * d] = lo;
        r[2 * d + 1] = hi;
    }
}

/* Built with -fopenmp (liboracle_omp.so, the parallel CPU baseline of SURVEY.md
 * §8(d)) the planes of one statement are split across threads; every point is
 * still evaluated by the same expression in the same order (points of one
 * statement are independent, reading R3), so the result is identical. */
#ifdef _OPENMP
#define OR_PARALLEL_FOR _Pragma("omp parallel for schedule(static)")
#else
#define OR_PARALLEL_FOR
#endif

/* One generic body per storage type; REAL is the arithmetic type.
 * T(term) = coef * a[p+oa]  or  (coef * a[p+oa]) * b[p+ob]            (R4) */
#define OR_DEFINE(NAME, STORE, REAL)                                                   \
    static int NAME(const or_grid *g, const long *box, int n_arrays,                   \
                    STORE *const *arrays, int n_stmts, const or_stmt *stmts) {         \
        if (!program_ok(g, n_arrays, n_stmts, stmts)) return -1;                       \
        or_layout L = layout_of(g);                                                    \
        long r[6];                                                                     \
        clip_box(g, box, r);                                                           \
        for (int s = 0; s < n_stmts; ++s) {                                            \
            const or_stmt *S = &stmts[s];                                              \
            STORE *out = arrays[S->out];                                               \
            long q[6]; /* points evaluated: interior, box, statement loop bounds */    \
            for (int d = 0; d < 6; ++d) q[d] = r[d];                                   \
            if (S->has_box)                                                            \
                for (int d = 0; d < 3; ++d) {                                          \
                    if (S->box[2 * d] > q[2 * d]) q[2 * d] = S->box[2 * d];            \
                    if (S->box[2 * d + 1] < q[2 * d + 1]) q[2 * d + 1] = S->box[2 * d + 1]; \
                }                                                                      \
            OR_PARALLEL_FOR                                                            \
            for (long k = q[4]; k < q[5]; ++k)                                         \
                for (long j = q[2]; j < q[3]; ++j)                                     \
                    for (long i = q[0]; i < q[1]; ++i) {                               \
                        long p = L.base + k * L.sz + j * L.sy + i * L.sx;              \
                        REAL acc = 0;                                                  \
                        for (int t = 0; t < S->n_terms; ++t) {                         \
                            const or_term *tm = &S->terms[t];                          \
                            REAL c = (REAL)tm->coef;                                   \
                            long pa = p + tm->a.dz * L.sz + tm->a.dy * L.sy + tm->a.dx;\
                            REAL v = c * (REAL)arrays[tm->a.arr][pa];                  \
                            if (tm->has_b) {                                           \
                                long pb = p + tm->b.dz * L.sz + tm->b.dy * L.sy +      \
                                          tm->b.dx;                                    \
                                v = v * (REAL)arrays[tm->b.arr][pb];                   \
                            }                                                          \
                            acc = (t == 0) ? v : acc + v;                              \
                        }                                                              \
                        out[p] = (STORE)acc;                                           \
                    }                                                                  \
        }                                                                              \
        return 0;                                                                      \
    }

/* Note: a statement reading its own output array at a non-zero offset would
 * observe partially updated values in this in-place loop; the program model
 * forbids such statements (reading R3), and the harness validates programs
 * before calling the oracle. */

OR_DEFINE(run_f64, double, double)
OR_DEFINE(run_f32, float, float)
OR_DEFINE(run_f32_in_f64, float, double)

int oracle_run_f64(const or_grid *g, int n, double *const *a, int ns, const or_stmt *s) {
    return run_f64(g, NULL, n, a, ns, s);
}
int oracle_run_f32(const or_grid *g, int n, float *const *a, int ns, const or_stmt *s) {
    return run_f32(g, NULL, n, a, ns, s);
}
int oracle_run_box_f64(const or_grid *g, const long box[6], int n, double *const *a, int ns,
                       const or_stmt *s) {
    return run_f64(g, box, n, a, ns, s);
}
int oracle_run_box_f32(const or_grid *g, const long box[6], int n, float *const *a, int ns,
                       const or_stmt *s) {
    return run_f32(g, box, n, a, ns, s);
}
int oracle_run_f32_in_f64(const or_grid *g, int n, float *const *a, int ns, const or_stmt *s) {
    return run_f32_in_f64(g, NULL, n, a, ns, s);
}
