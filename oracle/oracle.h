/*
 * oracle.h — CPU ORACLE: TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
 * reference legs may load this library.  The product (paper_conf_hpdc_wahibm15_b200)
 * never includes, links or calls it, and this file shares no code with it.
 *
 * What it computes (Wahib & Maruyama HPDC'15, PAPER.md):
 *   The method is an exact program transformation: "Output of the automated
 *   method was verified against the output of the original code base for every
 *   single run" (§6.1.2).  The oracle is therefore the ORIGINAL program:
 *   every kernel, in host invocation order (the OEG total order, §3.2.3),
 *   every statement of the kernel in order (reading R3 in DESIGN.md), every
 *   interior point of the grid inside the kernel's loop bounds (R1/R2/R2'),
 *   accumulating the statement's terms left
 *   to right (R4):
 *       acc = T(term0);  acc = acc + T(term_t) for t = 1..;   out[p] = acc
 *       T(term) = coef * a[p+oa]            or   (coef * a[p+oa]) * b[p+ob]
 *   Ghost cells are read, never written (R1).
 *
 * Layout: each array is dense [nz+2hz][ny+2hy][nx+2hx], x fastest; point
 * (i,j,k) (interior: 0 <= i < nx ...) lives at
 *     ((k+hz)*(ny+2hy) + (j+hy))*(nx+2hx) + (i+hx).
 *
 * Precision: the program dtype (binary64, or binary32 for fp32 programs —
 * reading R4), round-to-nearest, no FMA contraction (built with
 * -ffp-contract=off, no -ffast-math).  Coefficients are converted to the
 * program dtype once, as the product does at create time.
 *
 * Box variants: statements are evaluated only at points of the interior that
 * also lie inside box = [i0,i1) x [j0,j1) x [k0,k1).  With a window of a larger
 * grid as "the grid" and the global interior (in window coordinates) as the
 * box, the centre of a window wider than the program's accumulated reach is
 * exact: this is how single output points are checked at full size.
 */
#ifndef SF_ORACLE_H
#define SF_ORACLE_H
#ifdef __cplusplus
extern "C" {
#endif

typedef struct { int arr, dx, dy, dz; } or_tap;
typedef struct { double coef; or_tap a; int has_b; or_tap b; } or_term;
/* has_box: the statement's kernel iterates only box = [i0,i1) x [j0,j1) x [k0,k1)
 * of the interior (its loop bounds, §5.5.2 "shorter loops";
 * reading R2' in DESIGN.md): points outside it are not written. */
typedef struct { int out; int n_terms; const or_term *terms; int has_box; long box[6]; } or_stmt;
typedef struct { long nx, ny, nz; int hx, hy, hz; } or_grid;

/* Runs n_stmts statements (kernels flattened in program order) over the grid.
 * arrays[a] points to array a's dense padded storage.  Returns 0, or -1 if a
 * tap reaches beyond the ghost width or an array index is invalid (nothing is
 * written in that case). */
int oracle_run_f64(const or_grid *g, int n_arrays, double *const *arrays,
                   int n_stmts, const or_stmt *stmts);
int oracle_run_f32(const or_grid *g, int n_arrays, float *const *arrays,
                   int n_stmts, const or_stmt *stmts);
int oracle_run_box_f64(const or_grid *g, const long box[6], int n_arrays,
                       double *const *arrays, int n_stmts, const or_stmt *stmts);
int oracle_run_box_f32(const or_grid *g, const long box[6], int n_arrays,
                       float *const *arrays, int n_stmts, const or_stmt *stmts);

/* The same program evaluated in binary64 on binary32 storage: operands are
 * widened, every statement result is rounded to binary32 when stored.  Used
 * only to bound the fp32 path's rounding error (never as the parity oracle). */
int oracle_run_f32_in_f64(const or_grid *g, int n_arrays, float *const *arrays,
                          int n_stmts, const or_stmt *stmts);

#ifdef __cplusplus
}
#endif
#endif
