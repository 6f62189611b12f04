/*
 * cme.h -- C ABI of libcme: B200-native (sm_100a) steady-state solver for the
 * Chemical Master Equation, after Maggioni, Berger-Wolf & Liang, "GPU-based
 * Steady-State Solution of the Chemical Master Equation" (IPDPS-W 2013).
 *
 * Citations "P:Lnn" are lines of the paper's text (/root/reference/PAPER.md in
 * the build container); "Rn" are the readings recorded in DESIGN.md section 3.
 *
 * Problem: A is the sparse reaction-rate matrix, A_ij >= 0 for
 * i != j is the rate of the transition x_j -> x_i (eqs. 1-2),
 * A_jj = -sum_{i != j} A_ij (eq. 4, zero column sums).  The steady
 * state is the probability vector p with A p = 0, p >= 0, ||p||_1 = 1
 * (P:L63-67, L125).  It is computed by the (damped) Jacobi iteration
 *     x^(k+1) = (1 - omega) x^(k) + omega * (-D^-1 (L + U) x^(k))
 * (eqs. 6, 8; omega per R1), L1-renormalised every check
 * (P:L125), with the convergence test every `check_every` iterations.
 *
 * Conventions for every entry point
 *  - All functions return a cme_status; no C++ exception crosses the ABI.
 *  - Ownership: create functions COPY their inputs (the caller keeps them);
 *    a cme_matrix owns all of its host and device buffers until
 *    cme_matrix_destroy.  Output vectors are caller-allocated.
 *  - Vectors passed to the solver (p0, p_out, x, y) may be host or device
 *    pointers (CUDA unified addressing decides); device pointers must be on
 *    the matrix's device.  They are always in ORIGINAL state order (the order
 *    of the COO/CSR input), whatever reordering was applied.
 *  - Call order: create -> [cme_reorder] -> cme_pack -> [cme_matrix_distribute]
 *    -> solve/spmv.  Anything else returns CME_ERR_BAD_STATE.
 *  - Threads: one handle per host thread at a time.
 *  - Indices are int32 (n < 2^31 states); counts are int64.
 */
#ifndef CME_H
#define CME_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum cme_status {
    CME_OK = 0,
    CME_ERR_INVALID_ARG = 1,   /* bad size/index/pointer/option, NaN/Inf rate, i==j without CME_DIAG_GIVEN */
    CME_ERR_NEGATIVE_RATE = 2, /* an off-diagonal rate < 0 (all off-diagonals are positive) */
    CME_ERR_ZERO_OUTFLOW = 3,  /* a state with no outflow: A_jj = 0, Jacobi undefined */
    CME_ERR_BAD_STATE = 4,     /* wrong call order */
    CME_ERR_OOM = 5,           /* host or device allocation failed */
    CME_ERR_CUDA = 6,          /* CUDA runtime error (see cme_last_error) */
    CME_ERR_NCCL = 7,          /* NCCL error or NCCL library not loadable */
    CME_NOT_CONVERGED = 8,     /* solve hit max_iter (p_out still written, normalised) */
    CME_STAGNATED = 9,         /* delta stopped changing (R3), p_out written */
    CME_ERR_NUMERIC = 10,      /* NaN/Inf or zero mass in the iterate */
    CME_ERR_NO_DEVICE = 11,    /* no CUDA device visible */
    CME_ERR_TIMEOUT = 12       /* a bounded device-side wait expired: a peer rank's flag barrier
                                  (peer-memory transport) or a resident-kernel dependency
                                  (CME_RES_TIMEOUT_MS); the solve stopped instead of hanging */
} cme_status;

typedef struct cme_matrix_s* cme_matrix; /* opaque */
typedef struct cme_comm_s* cme_comm;     /* opaque; wraps an NCCL communicator */

/* ---- creation ------------------------------------------------ */

#define CME_DIAG_FROM_COLSUMS 0u /* default: input holds off-diagonals only; A_jj = -colsum */
#define CME_DIAG_GIVEN 1u        /* input may hold i==j entries (negative a_jj); checked against colsums */

/* COO triplets (row[e], col[e], rate[e]), e < nnz: rate of x_col -> x_row.
 * Duplicates are summed in input order (eq. 2); entries whose sum is
 * exactly 0 are dropped; A_jj = -(sum of column j in ascending row order).
 * Host pointers only.  Errors: INVALID_ARG, NEGATIVE_RATE, ZERO_OUTFLOW, OOM. */
cme_status cme_matrix_create_coo(int64_t n, int64_t nnz, const int32_t* row, const int32_t* col,
                                 const double* rate, uint32_t flags, cme_matrix* out);

/* Batched parameter sweep ("the study of the same reaction network
 * under different conditions"): `batch` rate sets on ONE COO
 * pattern, rates[b*nnz + e] for member b.  batch in {1, 2, 4, 8}.  An entry is
 * stored if any member's summed rate is non-zero; every member must have
 * outflow from every state.  Column indices are stored once; values, the
 * diagonal and the iterate are member-minor on the device, so one gather
 * fetches all members.  For a batch handle every vector argument below
 * (p0, p_out, x, y) holds batch*n doubles, member-major (member b at
 * [b*n, (b+1)*n)), and the solve stops when every member is converged or
 * stagnated (per-member results: cme_get_batch_report).  The CSR ablation
 * format takes batch 1 only. */
cme_status cme_matrix_create_coo_batch(int64_t n, int64_t nnz, const int32_t* row, const int32_t* col,
                                       const double* rates, int32_t batch, uint32_t flags, cme_matrix* out);

/* CSR by rows (row_ptr[n+1], col[row_ptr[n]], rate) -- same semantics as COO. */
cme_status cme_matrix_create_csr(int64_t n, const int64_t* row_ptr, const int32_t* col,
                                 const double* rate, uint32_t flags, cme_matrix* out);

/* ---- ordering (R11, R12) ---------------------------------------- */
enum { CME_ORDER_NONE = 0, CME_ORDER_DFS = 1, CME_ORDER_RCM = 2 };
/* DFS: preorder of the transition graph j -> i (A_ij != 0), out-neighbours in
 * ascending index, from `root`, restarting at the smallest unvisited state.
 * RCM: reverse Cuthill-McKee of the pattern of A + A^T, George-Liu
 * pseudo-peripheral start per component (root ignored).  Host-only work. */
cme_status cme_reorder(cme_matrix h, int method, int64_t root);
/* A caller-chosen ordering (e.g. a seeded random permutation, the locality
 * stress test of P:L225): new_to_old must be a permutation of 0..n-1. */
cme_status cme_set_permutation(cme_matrix h, const int32_t* new_to_old);

/* ---- packing ----------------------------------------------- */
enum { CME_FMT_DIAG_SELL = 0, CME_FMT_ELL = 1, CME_FMT_CSR = 2, CME_FMT_SELL256 = 3 };
enum { CME_BAND_AUTO = 0, CME_BAND_ALWAYS = 1, CME_BAND_NEVER = 2 };
#define CME_DEVICE_HOST_ONLY (-2)
typedef struct cme_pack_opts {
    int32_t slice;  /* rows per slice; must be 32 (= warp)                   */
    int32_t window; /* local-rearrangement window in rows; <= 1 disables        */
    int32_t band;   /* CME_BAND_*: DIA {-1,+1} band, AUTO = on iff +-1 density >= 2/3 */
    int32_t device; /* CUDA device ordinal; -1 = current device; CME_DEVICE_HOST_ONLY = build
                       the host layout only (inspection/tests; solving then returns BAD_STATE) */
} cme_pack_opts;
/* Builds the packed layout on the host, runs the directed
 * period test (R1), uploads to device memory.  opts == NULL: {32, 256, AUTO, -1}.
 * Ablation arms (Tables II-III): CME_FMT_ELL = one global width
 * (+DIA band per opts.band), CME_FMT_SELL256 = sliced ELL with 256-row slices
 * ([5], slice = CTA), both without rearrangement; CME_FMT_CSR = plain CSR.
 * window may be any size (window >= n = the global nnz reordering, pJDS [20]).
 * Errors: INVALID_ARG, BAD_STATE, OOM, CUDA, NO_DEVICE. */
cme_status cme_pack(cme_matrix h, int format, const cme_pack_opts* opts);

/* ---- solver -------------------------------------------------------------- */
enum { CME_STOP_DELTA_L1 = 0, CME_STOP_PAPER_RESID = 1 };
typedef struct cme_solver_opts {
    double omega;        /* (0,1]; 0 = auto: 1.0 if period == 1 else 0.9 (R1)             */
    int64_t check_every; /* C >= 1, default 100 (R4)                               */
    int32_t stop;        /* CME_STOP_DELTA_L1: ||y-x||_1/||x||_1 <= tol (R2);
                            CME_STOP_PAPER_RESID: ||r||_inf/(||A||_inf ||x||_inf) <= tol */
    double stag_tol;     /* STAGNATED if |delta_k - delta_{k-C}| <= stag_tol*delta_{k-C} (R3); 0 disables; default 1e-10 */
    void* stream;        /* cudaStream_t for all device work; NULL = the handle's own stream */
} cme_solver_opts;
/* NULL restores defaults {0, 100, DELTA_L1, 1e-10, NULL}. */
cme_status cme_set_solver_opts(cme_matrix h, const cme_solver_opts* o);

/* Full solve.  p0 (n doubles, >= 0, positive sum) or NULL for uniform 1/n (R6);
 * p_out (n doubles) receives the L1-normalised landscape; *iters_out (may be
 * NULL) the iterations done.  Synchronous.  Returns CME_OK (converged),
 * CME_NOT_CONVERGED, CME_STAGNATED, CME_ERR_NUMERIC (p_out written in all
 * four cases) or an error.  Under a communicator every rank calls it and every
 * rank receives the full p_out. */
cme_status cme_jacobi_solve(cme_matrix h, const double* p0, double tol, int64_t max_iter,
                            double* p_out, int64_t* iters_out);

/* Transient landscape p(t) = exp(A t) p0 (dP/dt = A P) by
 * uniformization -- the paper's stated future work, on the same
 * fused step (I + A/Lambda is a Jacobi step with per-row omega = |a_ii|/Lambda):
 * Lambda = max_i |a_ii|, p(t) = sum_{k<=K} w_k (I + A/Lambda)^k p0 with the
 * Poisson(Lambda t) weights of reading R22 (normalised on k <= ceil(mu +
 * 10 sqrt(mu) + 40), right tail <= eps cut).  p0 (n doubles, used as given) or
 * NULL = all mass on original state 0 (the enumeration's initial microstate).
 * *terms_out = K + 1 fused steps.  Batch 1, SELL formats.  Synchronous. */
cme_status cme_transient(cme_matrix h, const double* p0, double t, double eps, double* p_out,
                         int64_t* terms_out);

typedef struct cme_report {
    int32_t status;    /* cme_status of the last solve                                 */
    int64_t iters;     /* iterations done                                              */
    double delta;      /* last ||y - x||_1 / ||x||_1                                    */
    double resid;      /* last ||A x||_inf / (||A||_inf ||x||_inf)             */
    double mass;       /* last sum(y) before normalisation                            */
    double omega;      /* effective omega                                              */
    double seconds;    /* device time of the iteration loop (CUDA events)              */
} cme_report;
cme_status cme_get_report(cme_matrix h, cme_report* r);
/* Per-member reports of the last solve of a batch handle (count <= batch):
 * status = CME_OK / CME_STAGNATED / CME_NOT_CONVERGED / CME_ERR_NUMERIC of
 * that member, iters = the iteration at which its status was decided. */
cme_status cme_get_batch_report(cme_matrix h, cme_report* reports, int32_t count);

/* One application y = M_omega x = (1-omega) x - omega D^-1 (L+U) x, no
 * normalisation (test hook for per-SpMV parity).  x, y: n doubles. */
cme_status cme_spmv(cme_matrix h, const double* x, double* y);

/* Resident-iterate API (what a time-stepping caller and bench.py use):
 *   load: x <- p0 / sum(p0) (or uniform) into the device iterate;
 *   run:  enqueue `blocks` blocks of check_every iterations (last one of each
 *         block checks + normalises), no stop decision, asynchronous;
 *   fetch: write the normalised iterate to p_out (original order), sync. */
cme_status cme_solver_load(cme_matrix h, const double* p0);
cme_status cme_solver_run(cme_matrix h, int64_t blocks);
cme_status cme_solver_fetch(cme_matrix h, double* p_out);

/* ---- introspection ------------------------------------------------------ */
typedef struct cme_info {
    int64_t n, nnz, nnz_offdiag;  /* nnz counts the diagonal (Table I)       */
    int64_t bandwidth;            /* max |i - j| over A_ij != 0 in the current order  */
    double band_density;          /* (#A_{i,i-1} != 0 + #A_{i,i+1} != 0)/(2n-2)       */
    double band_density3;         /* d{-1,0,+1} of Table I: band nnz incl. diag/(3n-2) */
    double ell_efficiency;        /* e = ELL nonzeros / stored ELL slots    */
    int32_t format, order, band_on, window;
    int64_t period;               /* directed period (R1), 0 = undetermined          */
    double norm_inf;              /* ||A||_inf                                       */
    double omega;                 /* omega the solver will use                       */
    int64_t n_slots, n_slices, n_ell;
    int64_t packed_bytes;         /* device bytes of the packed matrix              */
    int64_t bytes_alg;            /* 12 nnz + 16 n: algorithmic bytes / iteration    */
    int64_t bytes_fmt;            /* compulsory bytes / iteration of this layout     */
    int32_t rank, nranks;         /* 0/1 unless distributed                         */
    int64_t row_begin, row_end;   /* local rows in the reordered numbering          */
    int64_t halo_begin, halo_end; /* local x span [halo_begin, halo_end)             */
    int32_t kernel;               /* step kernel: 0 register SELL, 1 TMA-staged SELL, 2 CSR,
                                     3 SMEM-resident persistent SELL (matrix in shared memory,
                                     neighbour-flag sync; problems that fit), -1 none */
    int32_t tma_warps, tma_stages;/* TMA kernel: consumer warps per CTA, smem stages */
    int32_t grid;                 /* CTAs per step launch                            */
    int32_t batch;                /* rate sets sharing the pattern (1 = single matrix) */
    int32_t compact;              /* 1: the TMA kernel streams the compact encoding (rows of
                                     M = |D|^-1 O, int16 column and uint8 row offsets,
                                     DESIGN.md sec. 5b); 2: its value-indexed form (sec. 5c);
                                     bytes_fmt/packed_bytes count it */
    int32_t records;              /* 1: the value-indexed encoding is streamed as one
                                     contiguous record per tile (sell_vi2_kernel, sec. 5d) */
    int32_t wf_steps;             /* s > 1: check blocks run as wavefront passes of s steps
                                     (sell_wf_kernel, sec. 5e; the records re-read from L2);
                                     0: one launch per step */
    int32_t wf_lag;               /* wavefront lag L in tiles (0 when wf_steps = 0)     */
    int32_t halo_fused;           /* 1: row-sharded over peer memory with the halo ordered
                                     inside the step kernel (no per-step barrier, sec. 8) */
    int32_t xwin_kb;              /* > 0: the step kernel reads the iterate from a shared-memory
                                     x window of this many KB per CTA, streamed with the tile
                                     records (sec. 5f); 0: x gathers through L1/L2 */
} cme_info;
cme_status cme_get_info(cme_matrix h, cme_info* info);

/* new_to_old[r] = original index of reordered state r (n int32). */
cme_status cme_get_permutation(cme_matrix h, int32_t* new_to_old);

/* Host copies of the packed arrays (library-owned, valid until destroy or the
 * next pack/distribute) -- for bit-exact tests against the oracle.  For a
 * distributed matrix: the local part, columns in local x-span coordinates. */
typedef struct cme_packed_view {
    int64_t n, n_slots, n_slices, n_ell;
    int32_t band_on, window, batch, pad_;   /* val/lo/up/inv_d hold batch values per entry/slot */
    const double* lo;        /* [n_slots] slot order                         */
    const double* up;        /* [n_slots]                                    */
    const double* inv_d;     /* [n_slots] 1/(-A_ii)                          */
    const int32_t* row_of;   /* [n_slots] local row of slot; pad = slot id   */
    const int64_t* slice_off;/* [n_slices+1]                                 */
    const int32_t* slice_w;  /* [n_slices]                                   */
    const double* val;       /* [n_ell]                                      */
    const int32_t* col;      /* [n_ell]                                      */
    const int64_t* csr_row_ptr; /* CME_FMT_CSR only (else NULL): [n+1]       */
} cme_packed_view;
cme_status cme_export_packed(cme_matrix h, cme_packed_view* v);

/* Compact encoding of the current SELL pack (what the TMA
 * kernel streams when cme_info.compact = 1): the rows of M = |D|^-1 O, the
 * matrix of the Jacobi iteration (eq. 8), plus offsets instead of
 * indices.  val[e] = a_rj / (-a_rr) (one IEEE division), lo/up likewise;
 * col16[e] = j - r (x-span column minus the entry's own row, int16); row8[s]
 * = r - (s >> win_shift << win_shift) (row inside its rearrangement window).
 * Pad entries: val 0, col16 0; pad slots: all 0.  A batch (B rate sets on one
 * pattern) has the offsets and the value index of its entries' B-tuples only.  Library-owned host arrays,
 * valid until destroy or the next pack/distribute; computed on demand when
 * the device does not use it (so host-only packs can be checked too).
 * Errors: BAD_STATE before cme_pack; INVALID_ARG when the pack does not
 * qualify (CSR format, window not a power of two <= 256, or an offset outside
 * int16). */
typedef struct cme_compact_view {
    int64_t n, n_slots, n_slices, n_ell;
    int32_t band_on, win_shift;
    const double* val;       /* [n_ell]                                      */
    const int16_t* col16;    /* [n_ell]                                      */
    const uint8_t* row8;     /* [n_slots], NULL when win_shift == 0          */
    const double* lo;        /* [n_slots], NULL when the band is off         */
    const double* up;        /* [n_slots], NULL when the band is off         */
    /* Value-indexed form (CSR-VI style): dict = the distinct
     * values of layout v0's val (all n_ell entries, pads included) and, band on,
     * lo/up, ascending; vidx[e] / loi[s] / upi[s] = their positions in dict.
     * n_dict = 0 and NULL pointers when there are more than 65536. */
    int64_t n_dict;
    const double* dict;      /* [n_dict * batch]: tuples, member-minor         */
    const uint16_t* vidx;    /* [n_ell]                                      */
    const uint16_t* loi;     /* [n_slots], NULL when the band is off         */
    const uint16_t* upi;     /* [n_slots], NULL when the band is off         */
    int32_t batch, pad_;     /* rate sets B; for B > 1 `val`/`lo`/`up` are NULL (only the
                                offsets and the value index of the B-tuples are built)     */
} cme_compact_view;
cme_status cme_export_compact(cme_matrix h, cme_compact_view* v);

/* Directed period of the ingested graph from `root` (R1); host-only. */
cme_status cme_period(cme_matrix h, int64_t root, int64_t* period_out);

/* The x-window plan of a packed single-GPU DIAG_SELL
 * matrix (B = 1; a CME_DEVICE_HOST_ONLY pack suffices) for tiles of `ncw`
 * slices with `stages` records in flight -- host logic exported for tests.
 * Iterate chunk k = local rows [256 k - 1, 256 k + 255).  plan[2 t], plan[2 t + 1]
 * (caller-allocated, 2 * tiles int32, tiles = ceil(n_slices / ncw)) receive tile
 * t's chunk range [first, end): every row, band neighbour and gathered column of
 * the tile lies in it; both ends are non-decreasing in t.  *need = the ring
 * chunks a CTA needs (max over t of end(t) - first(t - stages + 1)), *span =
 * the widest tile's chunk count.  BAD_STATE before pack or when distributed. */
cme_status cme_export_xw_plan(cme_matrix h, int32_t ncw, int32_t stages, int64_t tiles, int32_t* plan,
                              int64_t* need, int64_t* span);

/* ---- multi-GPU -------------------------------------------- */
/* Rank 0 creates the id; it is broadcast over the caller's process group
 * (torch.distributed) and every rank calls cme_comm_init.  NCCL is loaded
 * with dlopen (the copy torch already loaded, else libnccl.so.2). */
cme_status cme_comm_unique_id(uint8_t id[128]);
cme_status cme_comm_init(int nranks, int rank, const uint8_t id[128], int device, cme_comm* out);
/* Peer-memory transport (NEXT-4; no NCCL on the iteration path): an
 * in-process group of nranks communicators on devices[r] (distinct GPUs with
 * NVLink/NVSwitch peer access, or the same GPU repeated).  After
 * cme_matrix_distribute every step kernel stores the halo rows its
 * neighbours need straight into their iterate buffers (st.global to peer
 * memory), and a one-thread flag kernel (st.release.sys / ld.acquire.sys,
 * bounded spin) orders consecutive steps; check records and the output are
 * exchanged the same way.  Each rank's handle must be driven by its own host
 * thread; comms_out[nranks]; nranks <= 9. */
cme_status cme_comm_init_local(int nranks, const int* devices, cme_comm* comms_out);
/* The same transport across processes (one per GPU): cme_comm_init_ipc for
 * this rank, cme_matrix_distribute, then cme_matrix_ipc_export fills this
 * rank's CME_IPC_BLOB_BYTES blob (CUDA IPC handles of its iterate buffers,
 * flags, gather and staging arrays); the caller all-gathers the blobs in rank
 * order (e.g. torch.distributed) and passes them to cme_matrix_ipc_attach.
 * Until attach, solving returns BAD_STATE.  Before cme_matrix_destroy the
 * caller barriers the ranks (peers map this rank's memory). */
#define CME_IPC_BLOB_BYTES 512
cme_status cme_comm_init_ipc(int nranks, int rank, int device, cme_comm* out);
cme_status cme_matrix_ipc_export(cme_matrix h, uint8_t blob[CME_IPC_BLOB_BYTES]);
cme_status cme_matrix_ipc_attach(cme_matrix h, const uint8_t* blobs /* [nranks][CME_IPC_BLOB_BYTES] */);
/* Host-only partition plan for (nranks, rank): contiguous reordered rows cut
 * at window boundaries, balanced by packed bytes; local layout with columns
 * remapped to the local x span.  cme_matrix_distribute = plan + upload. */
cme_status cme_matrix_plan_partition(cme_matrix h, int nranks, int rank);
cme_status cme_matrix_distribute(cme_matrix h, cme_comm c);
typedef struct cme_halo_view {
    int32_t nranks, rank;
    const int64_t* row_begin; /* [nranks+1] global row cut points             */
    const int64_t* span;      /* [2*nranks] x-span [lo_r, hi_r) of every rank  */
    /* this rank's per-iteration exchange: send x-span[off, off+cnt) (own rows)
     * to peer; receive peer's rows into x-span[off, off+cnt) (halo)          */
    int32_t n_send, n_recv;
    const int32_t* send_peer; const int64_t* send_off; const int64_t* send_cnt;
    const int32_t* recv_peer; const int64_t* recv_off; const int64_t* recv_cnt;
} cme_halo_view;
cme_status cme_export_halo(cme_matrix h, cme_halo_view* v);

/* For a handle distributed over a peer-memory (cme_comm_init_local) group,
 * destroy is collective: it returns when every rank has called it. */
void cme_matrix_destroy(cme_matrix h);
void cme_comm_destroy(cme_comm c);

/* ---- misc ---------------------------------------------------------------- */
const char* cme_status_string(cme_status s);
const char* cme_last_error(void);          /* thread-local detail of the last error */
int cme_abi_version(void);                 /* 1 */

/* ---- network enumerator ([17]; separate from the solve path) ------ */
/* Reachable microstates of a finitely buffered network by recursive-DFS
 * preorder from x0 (R7-R10); zero-outflow states pruned to a fixpoint; one
 * COO triplet per (kept state j, enabled reaction k).  reac/change are R x m
 * row-major; w.x <= cap is the buffer.  Result arrays are owned by the
 * returned object and read with cme_coo_get; free with cme_coo_destroy. */
typedef struct cme_coo_s* cme_coo;
cme_status cme_network_enumerate(int m, const int32_t* x0, int R, const int32_t* reac,
                                 const int32_t* change, const double* rates, const int32_t* w,
                                 int64_t cap, cme_coo* out);
/* GPU enumerator: the same reachable set, rates and
 * zero-outflow pruning as cme_network_enumerate (eq. 1, R7-R10),
 * computed on CUDA device `device` (-1: current) by a level-synchronous BFS
 * over a 128-bit-key hash table (16 bits per species).  States are numbered in
 * LEXICOGRAPHIC order of (x_0, ..., x_{m-1}) -- deterministic -- instead of
 * DFS preorder; triplets are emitted per source state in reaction order, rates
 * bit-identical to the host enumerator's.  Limits: m <= 8 species, R <= 64
 * reactions, counts <= 65534 (CME_ERR_INVALID_ARG otherwise: use
 * cme_network_enumerate).  CME_ERR_NO_DEVICE / CME_ERR_OOM / CME_ERR_CUDA on
 * device failures.  Output object and ownership as cme_network_enumerate. */
cme_status cme_network_enumerate_gpu(int m, const int32_t* x0, int R, const int32_t* reac,
                                     const int32_t* change, const double* rates, const int32_t* w,
                                     int64_t cap, int device, cme_coo* out);
cme_status cme_coo_get(cme_coo c, int64_t* n, int64_t* nnz, int32_t m[1], const int32_t** states,
                       const int32_t** row, const int32_t** col, const double** rate);
void cme_coo_destroy(cme_coo c);

#ifdef __cplusplus
}
#endif
#endif /* CME_H */
