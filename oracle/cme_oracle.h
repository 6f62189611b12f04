/*
 * cme_oracle.h -- TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, obviously-correct CPU oracle for the CME steady-state Jacobi
 * hot path of Maggioni, Berger-Wolf & Liang (IPDPS-W 2013).  Citations
 * "P:Lnn" refer to /root/reference/PAPER.md line nn.  Only tests/,
 * __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs
 * may load this library.  It shares no code, header, table or helper with the
 * CUDA library under paper_conf_ipps_maggionibl13_b200/ -- both are written
 * from the paper and the readings in DESIGN.md independently.
 *
 * Every array returned through a `**` out-parameter is malloc()ed here and
 * must be released with oracle_free().  Functions return 0 on success or one
 * of the ORACLE_* codes below (numbered like the product's cme_status so the
 * tests can compare error behaviour).
 */
#ifndef CME_ORACLE_H
#define CME_ORACLE_H
#include <stdint.h>

#define ORACLE_OK 0
#define ORACLE_INVALID_ARG 1
#define ORACLE_NEGATIVE_RATE 2
#define ORACLE_ZERO_OUTFLOW 3
#define ORACLE_OOM 5
#define ORACLE_NOT_CONVERGED 8
#define ORACLE_STAGNATED 9
#define ORACLE_NUMERIC 10

void oracle_free(void* p);

/* Reachable microstates by recursive-DFS preorder from x0 ([17];
 * reading: SURVEY App. A / DESIGN.md R7-R10), zero-outflow states pruned to a
 * fixpoint, then one off-diagonal COO triplet (row = target, col = source,
 * rate = propensity) per (kept state j ascending, enabled reaction k
 * ascending).  Propensity A_k(x_j) = r_k * prod_i C(x_i, c_ki) (eq. 1). */
int oracle_enumerate(int m, const int32_t* x0, int R, const int32_t* reac, const int32_t* change,
                     const double* rates, const int32_t* w, int64_t cap,
                     int64_t* n_out, int64_t* nnz_out, int32_t** states_out,
                     int32_t** row_out, int32_t** col_out, double** rate_out);

/* COO -> CSR of the off-diagonal part (rows = incoming), duplicates
 * summed in input order (eq. 2); diag d_j = -(sum of column j in
 * ascending row order) (eq. 4) unless diag_given. */
int oracle_ingest(int64_t n, int64_t nnz, const int32_t* row, const int32_t* col, const double* rate,
                  int diag_given, int64_t** row_ptr_out, int32_t** col_out, double** val_out,
                  double** diag_out);

/* Orderings (R11, R12): new_to_old permutation. */
int oracle_order_dfs(int64_t n, const int64_t* row_ptr, const int32_t* col, int64_t root,
                     int32_t* new_to_old);
int oracle_order_rcm(int64_t n, const int64_t* row_ptr, const int32_t* col, int32_t* new_to_old);

/* Symmetric permutation: new row r = old row new_to_old[r]; columns sorted. */
int oracle_permute(int64_t n, const int64_t* row_ptr, const int32_t* col, const double* val,
                   const double* diag, const int32_t* new_to_old, int64_t** rp_out,
                   int32_t** col_out, double** val_out, double** diag_out);

/* Directed period test: gcd over edges u->v of |lvl(u)+1-lvl(v)| (R1). */
int64_t oracle_period(int64_t n, const int64_t* row_ptr, const int32_t* col, int64_t root);

/* Packed DIAG + warp-grained sliced ELL (layout v0). */
typedef struct {
    int64_t n, n_slots, n_slices, n_ell; /* n_ell = total ELL slots incl. padding  */
    int32_t band_on;
    int32_t window;
    double* lo;       /* [n_slots] slot order, 0 if band off                      */
    double* up;       /* [n_slots]                                                 */
    double* inv_d;    /* [n_slots] 1/(-a_ii)                                       */
    int32_t* row_of;  /* [n_slots] row of each slot; pad slots hold their slot id  */
    int64_t* slice_off; /* [n_slices+1]                                            */
    int32_t* slice_w;   /* [n_slices]                                              */
    double* val;      /* [n_ell]                                                   */
    int32_t* col;     /* [n_ell]                                                   */
} oracle_packed;
/* band: 0 AUTO (+-1 density >= 2/3), 1 ALWAYS, 2 NEVER.  window <= 1 = off.
 * group: slices sharing one width -- 1 warp-grained sliced ELL,
 * 8 = 256-row block-sliced ELL ([5]), 0 = one global width (plain ELL). */
int oracle_pack(int64_t n, const int64_t* row_ptr, const int32_t* col, const double* val,
                const double* diag, int32_t window, int32_t band, int32_t group,
                oracle_packed* out);
void oracle_packed_free(oracle_packed* p);

/* One damped-Jacobi application (eq. 8 with relaxation omega, R1):
 * y_i = (1-omega) x_i + omega * (sum_{j!=i} a_ij x_j) / (-a_ii). */
int oracle_jacobi_step(int64_t n, const int64_t* row_ptr, const int32_t* col, const double* val,
                       const double* diag, double omega, const double* x, double* y);

/* Jacobi solve: checks every C, deferred L1
 * normalisation, stop on delta = |y-x|_1/|x|_1 <= tol (stop_mode 0) or the
 * paper's normalised inf-residual (stop_mode 1), stagnation per
 * DESIGN.md R3.  nthreads <= 1 serial; otherwise OpenMP with identical bits. */
int oracle_jacobi_solve(int64_t n, const int64_t* row_ptr, const int32_t* col, const double* val,
                        const double* diag, const double* p0, double omega, double tol,
                        int64_t C, int64_t max_iter, int stop_mode, double stag_tol,
                        int nthreads, double* p_out, int64_t* iters_out, double* delta_out,
                        double* resid_out);

/* Transient landscape p(t) = exp(A t) p0 by uniformization (the paper's
 * future work; R22): Lambda = max_i |a_ii|, P = I + A/Lambda,
 * p(t) = sum_{k=0}^{K} Pois(k; Lambda t) P^k p0 with K the smallest k whose
 * cumulative Poisson weight reaches 1 - eps.  p0 NULL = all mass on state 0. */
int oracle_transient(int64_t n, const int64_t* row_ptr, const int32_t* col, const double* val,
                     const double* diag, const double* p0, double t, double eps, double* p_out,
                     int64_t* terms_out, double* lambda_out);

/* Dense GEPP null-space solve of A p = 0, sum p = 1 (last row of A replaced by
 * ones, rhs e_n), n <= 4096. */
int oracle_lu_steady(int64_t n, const int64_t* row_ptr, const int32_t* col, const double* val,
                     const double* diag, double* p_out);

#endif
