/*
 * oracle.h -- plain, slow, obviously-correct CPU oracle for the Paraprox
 * Stencil & Partition approximation (Samadi et al., ASPLOS'14, PAPER.md
 * §3.2).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load or call this.
 * It shares no code, header, table or helper with the CUDA library under
 * paper_conf_asplos_samadijlm14_b200/ and include/; neither includes or links
 * the other.
 *
 * Arithmetic: inputs and weights are fp32; every sum is accumulated in fp64
 * and outputs are fp64 (the paper never states a precision, S9).
 * Loops follow the paper's definitions in order; no folding, blocking or
 * reordering.  Frames are [n, h, w] row-major, contiguous.
 *
 * Parity status: every function below is pinned by tests/test_oracle_*.py
 * (scipy library routines, hand tables, closed forms, brute force); none is
 * "parity unpinned".  The index map for tiles larger than 5x5 follows reading
 * S5 (lattice of anchors); parity with the paper there rests on that reading.
 */
#ifndef PARAPROX_ORACLE_H
#define PARAPROX_ORACLE_H

#ifdef __cplusplus
extern "C" {
#endif

/* schemes and metrics use the oracle's own numbering (same meaning as the
 * library's, defined independently) */
enum { OR_EXACT = 0, OR_ROW = 1, OR_COL = 2, OR_CENTER = 3,
       OR_SKIP_ROW = 4, OR_SKIP_COL = 5, OR_SKIP_BOTH = 6 /* reduction approximation */ };
enum { OR_MRE = 0, OR_L2 = 1, OR_PSNR = 2 };

/* Reaching-distance rule for one axis of a tile of radius r (PAPER.md
 * L1196-1218 §3.2.3): m[i + r] = offset whose value stands in for offset i,
 * i in [-r, r].  Returns 0, or -1 on bad arguments. */
int oracle_index_map(int r, int d, int* m);

/* Scheme -> per-axis reaching distances (reading S3/S4 of DESIGN.md):
 * exact (0,0), row (d,0), column (0,d), centre (d,d). */
int oracle_scheme_reaches(int scheme, int reach, int* dy, int* dx);

/* Exact stencil, the plain definition:
 * E(y,x) = sum_i sum_j w[i][j] * X(clamp(y+i), clamp(x+j)). */
int oracle_stencil_exact(const float* x, int n, int h, int w,
                         const float* wgt, int ky, int kx, double* out);

/* Approximate stencil by literal per-window substitution (L1144-1148,
 * L1196-1218): build the tile W_p, replace each element by the element at
 * its index-mapped offset, then apply the filter to the substituted tile. */
int oracle_stencil_approx(const float* x, int n, int h, int w,
                          const float* wgt, int ky, int kx,
                          int dy, int dx, double* out);

/* Separable filter w = wy (outer) wx: horizontal pass then vertical pass,
 * each with the substituted (dy, dx) windows, fp64 intermediate. */
int oracle_stencil_sep(const float* x, int n, int h, int w,
                       const float* wy, int ky, const float* wx, int kx,
                       int dy, int dx, double* out);

/* Output quality of approx against exact over `count` elements (Table 1,
 * L1644-1664; §4.2).  MRE / L2 -> 1 - error; PSNR -> dB. */
int oracle_quality(const double* e, const double* a, long long count,
                   int metric, double* quality);

/* Tuner candidates in cost order (O7).  Writes up to `cap`
 * (scheme, reach) pairs, returns the count (or -1). */
int oracle_tune_candidates(int ky, int kx, int separable, int cap,
                           int* schemes, int* reaches);

/* TOQ tuner (L572-592 §2; L1220-1226 §3.2.4; L1620-1628 §4.1): run the exact
 * kernel once and each candidate in cost order on the training frames; the
 * first whose quality >= toq wins, else (EXACT, 0, 1.0).  Outputs are rounded
 * to fp32 ("what the user gets") before the quality is taken.  Per-candidate
 * qualities (in candidate order, up to the decision) go to `qualities` when
 * non-NULL (capacity `cap`); `*n_evaluated` receives their count. */
int oracle_tune(const float* x, int n, int h, int w, int separable,
                const float* wgt_or_wy, int ky, const float* wx, int kx,
                double toq, int metric, int cap, double* qualities,
                int* n_evaluated, int* scheme, int* reach, double* quality);

/* Global-lattice reading of the stencil approximation (DESIGN.md reading
 * G): "Paraprox accesses a subset of values in the
 * input array and replicates that subset to construct an approximate version
 * of the array".  Per axis of length len and reach d:
 * the accessed coordinates are the multiples of s = 2d+1; every coordinate
 * reads the nearest accessed one, and coordinates past the last accessed
 * one read the last:  g[t] = min(s*floor(t/s + 1/2), s*floor((len-1)/s)).
 * d = 0 is the identity.  Returns 0, or -1 on bad arguments. */
int oracle_lattice_map(int len, int d, int* g);

/* The approximate array X~(y,x) = X(g_y(y), g_x(x)) (reaches dy, dx), then
 * the exact stencil (dense, or the separable two passes) applied to X~. */
int oracle_stencil_lattice(const float* x, int n, int h, int w,
                           const float* wgt, int ky, int kx,
                           int dy, int dx, double* out);
int oracle_stencil_lattice_sep(const float* x, int n, int h, int w,
                               const float* wy, int ky, const float* wx, int kx,
                               int dy, int dx, double* out);

/* Lattice tuner: exact once, then the row lattice with reach 4, 3, 2, 1
 * (fewest HBM bytes first); the first with quality >= toq, else EXACT.  The
 * four qualities go to qualities4 when non-NULL. */
int oracle_tune_lattice(const float* x, int n, int h, int w, int separable,
                        const float* wgt_or_wy, int ky, const float* wx, int kx,
                        double toq, int metric, double* qualities4,
                        int* scheme, int* reach, double* quality);

/* Reduction approximation of the stencil loops (§3.3.3;
 * NEXT-3): the filter-row loop executes every ny-th iteration from its first
 * (i = -r_y, -r_y+ny, ...) and the filter-column loop every nx-th, each loop
 * summing into a zero-initialised temporary that is multiplied by its
 * skipping rate after the loop.  Rates above the trip count saturate to it.
 * Schemes: skip-row (N, 1), skip-col (1, N), skip-both (N, N). */
int oracle_scheme_skips(int scheme, int rate, int* ny, int* nx);
int oracle_stencil_skip(const float* x, int n, int h, int w, const float* wgt, int ky, int kx,
                        int ny, int nx, double* out);
int oracle_stencil_skip_sep(const float* x, int n, int h, int w, const float* wy, int ky,
                            const float* wx, int kx, int ny, int nx, double* out);

/* Extended tuner: flags bit 0 = stencil schemes, bit 1 = reduction schemes
 * (rates 2..r+1), one cost order over both (O7 + S24). */
int oracle_tune_candidates_ex(int ky, int kx, int separable, int flags, int cap, int* schemes, int* rates);
int oracle_tune_ex(const float* x, int n, int h, int w, int separable,
                   const float* wgt_or_wy, int ky, const float* wx, int kx, int flags,
                   double toq, int metric, int cap, double* qualities,
                   int* n_evaluated, int* scheme, int* rate, double* quality);

/* HotSpot (Table 1; 3x3 tiles L1916-1920; NEXT-4): `iterations`
 * explicit thermal steps T' = T + c (P + (T_N + T_S - 2T) gy + (T_E + T_W -
 * 2T) gx + (Tamb - T) gz) on n independent [h, w] grids, the 3x3 tile of T
 * substituted through the index maps (dy, dx) before each update. */
int oracle_hotspot(const float* temp, const float* power, int n, int h, int w,
                   double c, double gx, double gy, double gz, double tamb,
                   int dy, int dx, int iterations, double* out);

/* Runtime loop (§2, §5;
 * readings DESIGN.md R1-R4).
 * oracle_runtime_ladder: from the m candidates' training qualities (cost
 * order), rung 0 = the first with q >= toq, then every later candidate whose
 * q is strictly above all earlier rungs, then EXACT (written as -1).  Writes
 * up to cap candidate indices to rungs; returns the rung count (or -1).
 * oracle_runtime_trace: the rung each of t_count invocations runs on, given
 * q[t * rungs + k] = the quality a check of invocation t would measure on
 * rung k.  Invocation t is checked when check_every > 0, t % check_every ==
 * 0 and the rung is not EXACT (the last); a check below toq moves one rung
 * down before invocation t + 1.  checked[t] (optional) flags the checks. */
int oracle_runtime_ladder(int m, const double* train_q, double toq, int cap, int* rungs);
int oracle_runtime_trace(int rungs, int check_every, double toq, int t_count, const double* q,
                         int* rung_used, int* checked, long long* checks, long long* backoffs);

#ifdef __cplusplus
}
#endif
#endif
