/* nitro.h — C ABI of the B200-native Nitro SpMV code-variant hot path.
 *
 * The paper (Muralidharan et al., "Nitro: A Framework for Adaptive Code
 * Variant Tuning", IPDPS 2014) is cited as P:L<n> = line n of its text
 * (/root/reference/PAPER.md on the build box; the citations are restated in
 * DESIGN.md so the GPU box never needs the file).
 *
 * Two layers:
 *  1. the generic Nitro layer (Fig. 2): a context, code variants
 *     with cost-returning variant functions, feature functions, constraints,
 *     training inputs, offline training (exhaustive search + RBF-SVM)
 *     and selection;
 *  2. the SpMV layer (the hot path, BASELINE north_star): a matrix handle over
 *     a borrowed device CSR, the GPU feature pass, the CSR->ELL/DIA/HYB
 *     converters, the five SpMV variants, timing, and a registration helper
 *     that plugs the five variants + features + constraints into layer 1.
 *  3. the multi-GPU row-partitioned SpMV (x all-gathered or halo-exchanged
 *     with NCCL, or over the single-GPU loopback transport; the solver-loop
 *     mode with the exchange fused into the SpMV epilogue).
 *  4. the histogram code-variant family (a second workload).
 *
 * Conventions (all functions):
 *  - extern "C"; return nitro_status_t (NITRO_OK = 0); never throw or abort.
 *    nitro_last_error() returns a thread-local message for the last failure.
 *  - Handles are opaque.  Device arrays passed in are BORROWED: the caller
 *    keeps them alive while the handle uses them.  Formats produced by
 *    conversion are OWNED by the handle and freed by *_destroy.
 *  - `stream` arguments are cudaStream_t passed as void*; NULL = legacy default.
 *    GPU work is enqueued on the handle's stream.  Only calls that return host
 *    results (features, allowed, time, select, call, train, export) synchronise it.
 *  - Sizes are int64_t element counts unless named *_bytes.
 */
#ifndef NITRO_H
#define NITRO_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef int nitro_status_t;
enum {
  NITRO_OK = 0,
  NITRO_E_INVALID_ARG = 1, /* null pointer, bad enum, size mismatch */
  NITRO_E_BAD_MATRIX = 2,  /* non-canonical CSR (see nitro_spmv_feat) */
  NITRO_E_STATE = 3,       /* select before train/load, mutation after train */
  NITRO_E_CONSTRAINT = 4,  /* explicit run of a variant its constraint rules out */
  NITRO_E_OOM = 5,         /* device or host allocation failed */
  NITRO_E_CUDA = 6,        /* CUDA runtime error (message has the CUDA string) */
  NITRO_E_NCCL = 7,        /* NCCL error */
  NITRO_E_IO = 8,          /* model file read/write */
  NITRO_E_UNSUPPORTED = 9  /* configuration outside what this build handles */
};

const char *nitro_last_error(void);
const char *nitro_version(void);

/* ========================================================================
 * 1. Generic Nitro layer (Fig. 2 L71-124; autotuner P:L136-190)
 * ======================================================================== */
typedef struct nitro_context nitro_context; /* global state shared by variants */
typedef struct nitro_cv nitro_cv;           /* code_variant<Policy, ArgTuple> */

/* Variant body: runs the variant on `input`, returns its
 * cost (default: elapsed seconds; +INFINITY = failed).  Lower is better. */
typedef double (*nitro_variant_fn)(void *input, void *user);
/* Feature function: same argument as the variant, returns a double. */
typedef double (*nitro_feature_fn)(const void *input, void *user);
/* Fused feature group: fills out[0..n) in one pass (replaces n feature calls;
 * on the GPU one kernel computes every SpMV feature).  Returns 0 on success. */
typedef int (*nitro_feature_group_fn)(const void *input, double *out, int n, void *user);
/* Constraint: nonzero = the variant may run on this input. */
typedef int (*nitro_constraint_fn)(const void *input, void *user);

nitro_status_t nitro_context_create(nitro_context **out);
void nitro_context_destroy(nitro_context *ctx);

/* name: copied.  The cv keeps a pointer to ctx (must outlive it). */
nitro_status_t nitro_cv_create(nitro_context *ctx, const char *name, nitro_cv **out);
void nitro_cv_destroy(nitro_cv *cv);

/* add_variant: label = insertion index 0..|V|-1. */
nitro_status_t nitro_cv_add_variant(nitro_cv *cv, const char *name, nitro_variant_fn fn, void *user, int *out_id);
/* set_default: fallback when a predicted variant is ruled out. */
nitro_status_t nitro_cv_set_default(nitro_cv *cv, int variant_id);
/* add_input_feature: appended to the feature table. */
nitro_status_t nitro_cv_add_feature(nitro_cv *cv, const char *name, nitro_feature_fn fn, void *user, int *out_id);
/* n features filled by one call (names copied). */
nitro_status_t nitro_cv_add_feature_group(nitro_cv *cv, const char *const *names, int n,
                                          nitro_feature_group_fn fn, void *user);
/* add_constraint(&variant, &constraint).  Several may be
 * added per variant; all must hold. */
nitro_status_t nitro_cv_add_constraint(nitro_cv *cv, int variant_id, nitro_constraint_fn fn, void *user);
/* Feature transform of the model.  Default (and the paper's reading):
 * none = libSVM's svm-scale min-max to [-1, 1].  EXTENSION (R11x,
 * not from the paper): features j with bit j of log_mask set are replaced by
 * log1p(x) (they must be >= 0) before the [-1, 1] min-max scaling; clip != 0
 * clips scaled inputs to [-1, 1], so inputs beyond the training range are
 * treated as the nearest training extreme instead of extrapolated by the RBF
 * kernel.  Before training (NITRO_E_STATE after); saved in the model file.
 * The registration helpers leave the paper's plain scaling in place. */
nitro_status_t nitro_cv_set_feature_transform(nitro_cv *cv, uint32_t log_mask, int clip);
/* set_training_args.  `input` is borrowed until train returns. */
nitro_status_t nitro_cv_add_training_input(nitro_cv *cv, void *input);

/* Training options (Table II of the paper is absent from the text; these are
 * the readings of DESIGN.md "Readings" R10-R12). */
typedef struct {
  int folds;                      /* CV folds (default 5) */
  uint64_t seed;                  /* fold shuffling seed (default 0) */
  double tol;                     /* SMO stopping tolerance (default 1e-6) */
  int log2c_lo, log2c_hi, log2c_step; /* default -5, 15, 2   (libSVM grid.py) */
  int log2g_lo, log2g_hi, log2g_step; /* default -15, 3, 2 */
  int verbose;                    /* 0 = silent */
  double timeout_factor;          /* training timeout: while an input is labelled, a
                                     variant may stop timing once its cost exceeds this factor x the
                                     best cost seen so far on that input (default 20; <= 0 = off) */
} nitro_train_opts;
void nitro_train_opts_default(nitro_train_opts *o);
/* For variant functions: the cost above which the input's exhaustive search
 * no longer needs an exact value (timeout_factor x the best cost so far on
 * the input being labelled); +INFINITY outside training or when off.  A
 * variant may stop measuring once it is sure to exceed it and return the
 * cost measured so far (the SpMV variants stop their reps, >= 3 run). */
double nitro_cv_cost_cutoff(void);

/* Offline training: for every training input evaluate features,
 * run every variant (constraint false => cost +INF), label = argmin
 * (ties -> lowest id); scale features to [-1,1]; CV grid over (C, gamma);
 * fit the RBF C-SVC (one-vs-one) on all inputs.  Freezes the cv (later
 * add_* calls return NITRO_E_STATE). */
nitro_status_t nitro_cv_train(nitro_cv *cv, const nitro_train_opts *opts);
/* Fit from an externally measured table (same steps after labelling).
 * feat[n_in * n_feat], cost[n_in * n_var] (row-major). */
nitro_status_t nitro_cv_train_from_table(nitro_cv *cv, int n_in, const double *feat, const double *cost,
                                         const nitro_train_opts *opts);
/* Incremental tuning: features of every training input are
 * computed first (they are cheap); then only a subset is labelled by
 * exhaustive search: `init` inputs in a seeded order (extended until two
 * labels are present), then one input per iteration chosen by the
 * Best-vs-Second-Best rule (smallest gap between the two largest class
 * probabilities of the current model, P:L188 [20]), refitting after each.
 * Stops after `iters` picks ("iter") or once the accuracy on the
 * labelled test set reaches `acc` ("acc"), or when the pool is empty. */
typedef struct {
  int init;                 /* initial labelled inputs (default: number of variants) */
  int iters;                /* max BvSB picks; <= 0 = until the pool is exhausted */
  double acc;               /* target test accuracy in (0,1]; 0 = off */
  uint64_t seed;            /* order of the initial picks */
  int prob_folds;           /* Platt CV folds (default 5) */
  int n_test;               /* optional labelled test set (0 = none) */
  const double *test_feat;  /* [n_test * n_feat] raw features */
  const double *test_cost;  /* [n_test * n_var] costs (+INF = ruled out); label = argmin */
} nitro_itune_opts;
void nitro_itune_opts_default(nitro_itune_opts *o);
nitro_status_t nitro_cv_itune(nitro_cv *cv, const nitro_train_opts *train, const nitro_itune_opts *it);
/* One entry per refit: labelled count, input picked after it (-1 = none),
 * test accuracy and test performance (mean t_best / t_selected), NaN without a test set. */
nitro_status_t nitro_cv_itune_history(const nitro_cv *cv, int *n_steps, int *n_labelled, int *picked,
                                      double *test_acc, double *test_perf);
/* Copies out the training table; any pointer may be NULL.  Sizes: cost
 * [n_in*n_var], feat [n_in*n_feat], label [n_in]. */
nitro_status_t nitro_cv_training_table(const nitro_cv *cv, int *n_in, double *cost, double *feat, int *label);
/* Model facts: chosen C, gamma, CV accuracy, #support vectors. */
nitro_status_t nitro_cv_model_info(const nitro_cv *cv, double *C, double *gamma, double *cv_acc, int *n_sv);
nitro_status_t nitro_cv_save_model(const nitro_cv *cv, const char *path);
nitro_status_t nitro_cv_load_model(nitro_cv *cv, const char *path);
nitro_status_t nitro_cv_num_features(const nitro_cv *cv, int *n);
nitro_status_t nitro_cv_num_variants(const nitro_cv *cv, int *n);

/* Deployment: evaluate features, predict, check the
 * predicted variant's constraints (fail => default).  select does not run the
 * variant; call runs it and returns its cost.  out_feat (nullable) receives
 * the raw feature vector. */
nitro_status_t nitro_cv_select(nitro_cv *cv, const void *input, int *out_variant, double *out_feat);
nitro_status_t nitro_cv_call(nitro_cv *cv, void *input, int *out_variant, double *out_cost);
/* Select from an already-computed raw feature vector and allowed mask. */
nitro_status_t nitro_cv_predict(nitro_cv *cv, const double *feat, const int *allowed /*nullable*/, int *out_variant);

/* Host SVM primitives (the learning step of P:L61-62, L179), exposed so the
 * host logic can be checked against libSVM without a GPU.
 * X row-major [n*d] (already scaled), y labels >= 0. */
typedef struct nitro_svm nitro_svm;
nitro_status_t nitro_svm_fit(int n, int d, const double *X, const int *y, double C, double gamma, double tol,
                             nitro_svm **out);
nitro_status_t nitro_svm_predict(const nitro_svm *m, int n, const double *X, int *out_labels);
/* one-vs-one decision values, pairs (i<j) in ascending class order [n * n_pairs] */
nitro_status_t nitro_svm_decision(const nitro_svm *m, int n, const double *X, double *out, int *n_pairs);
/* dual coefficients y_i*alpha_i of pair p for training sample ids (dense [n_train]) and rho */
nitro_status_t nitro_svm_pair_dual(const nitro_svm *m, int p, double *coef_dense, double *rho);
void nitro_svm_destroy(nitro_svm *m);
/* Probability model (libSVM's method, used by BvSB active learning):
 * per pair a Platt sigmoid fitted on decision values of an internal `folds`-fold
 * CV (deterministic stratified folds from `seed`), then pairwise coupling. */
nitro_status_t nitro_svm_fit_prob(int n, int d, const double *X, const int *y, double C, double gamma, double tol,
                                  int folds, uint64_t seed, nitro_svm **out);
/* class probabilities [n * n_classes] in ascending-label order */
nitro_status_t nitro_svm_probability(const nitro_svm *m, int n, const double *X, double *out, int *n_classes);
nitro_status_t nitro_svm_pair_sigmoid(const nitro_svm *m, int p, double *A, double *B);
/* deterministic stratified folds (R12) */
nitro_status_t nitro_svm_fold_assign(int n, const int *y, int k, uint64_t seed, int *out_fold);
nitro_status_t nitro_svm_cv_accuracy(int n, int d, const double *X, const int *y, double C, double gamma,
                                     double tol, int folds, uint64_t seed, double *out_acc);

/* ========================================================================
 * 2. SpMV layer — the hot path (BASELINE north_star)
 * ======================================================================== */
typedef enum {
  NITRO_CSR_SCALAR = 0, /* thread per row */
  NITRO_CSR_VECTOR = 1, /* V lanes (2..32) per row, "a warp to each row" P:L209 */
  NITRO_ELL = 2,        /* column-major padded ELL */
  NITRO_DIA = 3,        /* padded diagonals */
  NITRO_HYB = 4,        /* ELL(K) + atomic-free COO tail */
  NITRO_NUM_VARIANTS = 5
} nitro_spmv_variant;

/* Features (P:L97-101 nnz, num_rows; P:L200, L209 AvgNZPerRow, RL-SD,
 * MaxDeviation, DIA-Fill, ELL-Fillin).  Integer moments are exact; the
 * doubles follow DESIGN.md R4's finishing expression bit for bit. */
typedef struct {
  int64_t rows, cols, nnz;
  uint64_t sum_len, sum_len2; /* sum L_i, sum L_i^2 */
  int64_t max_row, ndiag;     /* Lmax, number of occupied diagonals */
  int32_t canonical, pad_;
  double mean, sd, max_dev, dia_fill, ell_fill;
} nitro_spmv_feat;

/* Format facts after prepare. */
typedef struct {
  int64_t ld;         /* padded row pitch of ELL/DIA/HYB-ELL (multiple of 32);
                         CSR-vector stream mode: hot x values staged in shared memory (0 = none);
                         CSR-vector row mode: 1 = the vector-load kernel K6v, 0 = K6 */
  int64_t width;      /* ELL: K = Lmax; DIA: ndiag; HYB: K_hyb; CSR-vector: lanes per row (0 = stream mode) */
  int64_t tail;       /* HYB: COO tail entries; CSR-vector: long-row segments (row mode) or chunks (stream mode) */
  int64_t bytes;      /* device bytes owned for this format */
  double compulsory_bytes; /* algorithmic bytes of one multiply */
} nitro_format_info;

typedef struct nitro_spmv nitro_spmv;

/* Borrow a device CSR (rowptr int32 or int64 [rows+1], colidx int32 [nnz],
 * vals fp32 or fp64 [nnz]).  Columns must be < 2^31.  Structure is checked in
 * the feature pass, not here. */
nitro_status_t nitro_spmv_create(int device, void *stream, int64_t rows, int64_t cols, int64_t nnz,
                                 const void *d_rowptr, int rowptr_is_64, const int32_t *d_colidx,
                                 const void *d_vals, int is_fp64, nitro_spmv **out);
nitro_status_t nitro_spmv_set_stream(nitro_spmv *A, void *stream);
/* GPU feature pass (one pass over rowptr + colidx) + host finishing.  Syncs.
 * A non-canonical matrix (rowptr not monotone from 0 to nnz, columns not
 * strictly increasing in a row, or out of [0, cols)) returns
 * NITRO_E_BAD_MATRIX with out->canonical = 0.  Cached. */
nitro_status_t nitro_spmv_features(nitro_spmv *A, nitro_spmv_feat *out);
/* Cheaper feature level (the Fig. 8 overhead study): one pass over
 * rowptr only -> rows, cols, nnz, sum_len, sum_len2, max_row, mean, sd,
 * max_dev, ell_fill exactly as nitro_spmv_features (bit-identical); the
 * column-dependent fields are not evaluated: ndiag = -1, dia_fill = -1.0,
 * canonical = -1 (rowptr monotonicity is still checked: a broken rowptr
 * returns NITRO_E_BAD_MATRIX).  Not cached; does not satisfy constraints.
 * Syncs the handle's stream. */
nitro_status_t nitro_spmv_row_features(nitro_spmv *A, nitro_spmv_feat *out);
/* fix_inputs analogue: enqueue the feature pass now, on the
 * handle's stream, without waiting; the next features/allowed/select waits. */
nitro_status_t nitro_spmv_features_async(nitro_spmv *A);
/* Constraints (R9): DIA needs dia_fill <= 3 and
 * its padded bytes <= budget; ELL likewise with ell_fill; others always. */
nitro_status_t nitro_spmv_allowed(nitro_spmv *A, int variant, int *out_allowed);
/* budget for padded formats in bytes (default: 40% of free HBM at first use) */
nitro_status_t nitro_spmv_set_budget(nitro_spmv *A, double bytes);
/* Kernel implementation of the two CSR variants (DESIGN.md §6 K5/K6/K6s):
 * NITRO_CSR_IMPL_AUTO (default) = the direct kernels, and for CSR-vector the
 * nnz-split stream kernel (K6s) when the row lengths are skewed (row-length
 * SD > mean: power-law rows); the TMA row-tile pipeline measured slower on
 * every class, so AUTO uses it only when the environment sets
 * NITRO_CSR_STAGED=1.  _DIRECT = the direct row-oriented kernels; _STAGED =
 * the TMA row-tile pipeline for every matrix (tiles that do not fit the
 * shared-memory stage are computed from global memory); _STREAM = the
 * nnz-split stream kernel for CSR-vector (CSR-scalar keeps the direct
 * kernel); _VEC4 = the vector-load CSR-vector kernel (K6v: V lanes per row,
 * 4 consecutive entries per lane per step by 128-bit loads; needs 16-byte
 * aligned col / val, else the direct kernel runs), which AUTO also picks for
 * rows of similar length when the build's default says so.
 * Within a mode the result is deterministic; the row-oriented
 * implementations are bit-identical to each other, the stream mode sums each
 * row in fp64 in a different association (within the R2 tolerance).
 * Returns NITRO_E_INVALID_ARG for any other value.  Takes effect at the next
 * run (the CSR-vector format is rebuilt if its mode changes). */
enum { NITRO_CSR_IMPL_AUTO = 0, NITRO_CSR_IMPL_DIRECT = 1, NITRO_CSR_IMPL_STAGED = 2, NITRO_CSR_IMPL_STREAM = 3,
       NITRO_CSR_IMPL_VEC4 = 4 };
nitro_status_t nitro_spmv_set_csr_impl(nitro_spmv *A, int impl);
/* Build the variant's format (cached; conversions are amortised). */
nitro_status_t nitro_spmv_prepare(nitro_spmv *A, int variant);
nitro_status_t nitro_spmv_format_info(nitro_spmv *A, int variant, nitro_format_info *out);
/* y[rows] = A * x[cols] (overwrite), async on the handle's stream.  Prepares
 * the format if needed (which may sync).  d_x and d_y must not alias. */
nitro_status_t nitro_spmv_run(nitro_spmv *A, int variant, const void *d_x, void *d_y);
/* End-to-end call with HOST buffers: copies x in, multiplies, copies y out,
 * synchronises.  h_x / h_y should be pinned for full speed. */
nitro_status_t nitro_spmv_run_host(nitro_spmv *A, int variant, const void *h_x, void *h_y);
/* Timing (a variant's cost is its elapsed time): warmup runs, then
 * `reps` runs each preceded (if flush_l2) by an L2-evicting read of 3x the L2 size, CUDA events
 * around the SpMV kernels only; returns the median in seconds.  out_all
 * (nullable) receives all reps. */
nitro_status_t nitro_spmv_time(nitro_spmv *A, int variant, const void *d_x, void *d_y, int warmup, int reps,
                               int flush_l2, double *out_median_s, double *out_all);
/* Evict L2: a streaming read of a scratch buffer of 3x the L2 size (clean
 * lines, so no write-back lands in the next timed region), on the handle's stream. */
nitro_status_t nitro_spmv_flush_l2(nitro_spmv *A);
/* Number of kernel launches one nitro_spmv_run of `variant` issues. */
nitro_status_t nitro_spmv_launches(nitro_spmv *A, int variant, int *out);

/* Export converted arrays to host (bit-exact tests).  part:
 *  0 ELL col (int32 [K*ld]), 1 ELL val ([K*ld]),
 *  2 DIA offsets (int32 [D]), 3 DIA val ([D*ld]),
 *  4 HYB ELL col, 5 HYB ELL val, 6 HYB tail row (int32 [Zt]), 7 tail col, 8 tail val,
 *  9 diagonal offsets from the feature pass (int32 [ndiag], ascending).
 * needed receives the byte size; copies only if cap >= needed.  Syncs. */
nitro_status_t nitro_spmv_export(nitro_spmv *A, int part, void *host_buf, size_t cap, size_t *needed);
/* The caller changed the borrowed CSR contents in place: drop the cached
 * features and every converted format (buffers are kept for reuse).  The
 * next features/prepare/run recomputes them. */
nitro_status_t nitro_spmv_invalidate(nitro_spmv *A);
/* Free one variant's format (variant = -1: all). */
nitro_status_t nitro_spmv_release(nitro_spmv *A, int variant);
void nitro_spmv_destroy(nitro_spmv *A);

/* Input record consumed by the registered SpMV variants of a nitro_cv. */
typedef struct {
  nitro_spmv *A;
  const void *d_x;
  void *d_y;
  int warmup, reps, flush_l2; /* timing protocol for the variant cost */
} nitro_spmv_input;

/* Register on a fresh cv: the 5 variants (ids = nitro_spmv_variant), the fused
 * feature group {nnz, rows, mean, sd, max_dev, dia_fill, ell_fill}, the DIA and
 * ELL constraints, and default = CSR-vector (Fig. 2).  Inputs passed to
 * train/select/call are nitro_spmv_input*. */
nitro_status_t nitro_spmv_register(nitro_cv *cv);

/* ========================================================================
 * 3. Multi-GPU row-partitioned SpMV (north_star; one process per GPU)
 * ======================================================================== */
typedef struct nitro_dist nitro_dist;
/* 128-byte NCCL unique id, created on rank 0 and broadcast by the caller. */
nitro_status_t nitro_dist_unique_id(void *out128);
nitro_status_t nitro_dist_init(const void *id128, int rank, int nranks, int device, nitro_dist **out);
void nitro_dist_destroy(nitro_dist *D);
/* nnz-balanced contiguous partition: rank r owns rows [bounds[r], bounds[r+1]),
 * bounds[r] = first row i with rowptr[i] >= ceil(r*nnz/P) (host rowptr). */
nitro_status_t nitro_dist_partition(int64_t rows, const int64_t *h_rowptr, int nranks, int64_t *bounds);
/* Per-rank matrix: this rank's row block of a SQUARE global matrix (x is
 * partitioned like y), with GLOBAL column ids < global_rows (checked by the
 * feature pass: NITRO_E_BAD_MATRIX), borrowed like nitro_spmv_create.  bounds[nranks+1] is the global
 * row partition (x is distributed the same way).  Splits interior rows (all
 * columns owned locally) from boundary rows and remaps columns into the
 * gathered-x layout (block r at r*B, B = max block rows). */
nitro_status_t nitro_dist_spmv_create(nitro_dist *D, int64_t global_rows, const int64_t *bounds,
                                      int64_t local_nnz, const void *d_rowptr, int rowptr_is_64,
                                      const int32_t *d_colidx, const void *d_vals, int is_fp64,
                                      nitro_spmv **out_local);
/* Same, choosing the x exchange: -1 auto (halo when the largest per-rank halo
 * is < 1/4 of the all-gather volume), 0 all-gather (layout: P*B padded
 * blocks), 1 halo (layout: [x[halo < lo] | x_local | x[halo >= hi]], monotone in the global column; grouped send/recv of
 * only the referenced remote entries).  Collective when the
 * handle has a communicator (every rank must call it). */
nitro_status_t nitro_dist_spmv_create_ex(nitro_dist *D, int64_t global_rows, const int64_t *bounds,
                                         int64_t local_nnz, const void *d_rowptr, int rowptr_is_64,
                                         const int32_t *d_colidx, const void *d_vals, int is_fp64, int exchange,
                                         nitro_spmv **out_local);
/* Exchange facts: mode (0 all-gather, 1 halo), x layout length, halo entries
 * this rank receives, entries it sends. */
nitro_status_t nitro_dist_exchange_info(nitro_spmv *A_local, int *mode, int64_t *layout_len, int64_t *halo_len,
                                        int64_t *send_len);
/* The sorted global column ids of the halo (host array of halo_len entries). */
nitro_status_t nitro_dist_halo_cols(nitro_spmv *A_local, int32_t *h_out);
/* Device address where this rank's x block lives inside the exchange layout:
 * passing it as d_x_local to nitro_dist_spmv_run (e.g. a solver writing its
 * next x there directly) skips the per-multiply copy. */
nitro_status_t nitro_dist_x_local(nitro_spmv *A_local, void **ptr);
/* y_local = A_local * x (x exchanged with NCCL on a side stream — all-gather or
 * halo send/recv; interior rows overlap the exchange, boundary rows follow). */
nitro_status_t nitro_dist_spmv_run(nitro_dist *D, nitro_spmv *A_local, int variant, const void *d_x_local,
                                   void *d_y_local);
/* Same multiply from an x that is already exchanged into this handle's layout
 * (all-gather: block q at q*B, B = max block rows, length nranks*B; halo:
 * [x[halo below] | x_local | x[halo above]]; padding entries must be finite, e.g. 0, because
 * padded formats multiply zero slots by them): no communication.
 * Used when the caller owns the exchange (e.g. a solver that writes y straight
 * into the next x), and to check every rank's part on one GPU. */
nitro_status_t nitro_dist_spmv_run_gathered(nitro_dist *D, nitro_spmv *A_local, int variant,
                                            const void *d_x_gathered, void *d_y_local);
/* Format facts of this rank's multiply (prepares the parts' formats):
 * bytes / tail summed over the rank's row parts, width / ld their maximum,
 * compulsory_bytes = the parts' matrix + y bytes (DESIGN.md §6 formulas) + the
 * exchanged x layout read once.  A part whose constraint rules the variant
 * out is counted with the default (CSR-vector), as nitro_dist_spmv_run runs it. */
nitro_status_t nitro_dist_format_info(nitro_spmv *A_local, int variant, nitro_format_info *out);
/* Padded block size B and this rank's [i0, i1) interior row run (rows that
 * read only local x and overlap the all-gather). */
nitro_status_t nitro_dist_layout(nitro_spmv *A_local, int64_t *B, int64_t *i0, int64_t *i1);
/* A communicator-less handle for (rank, nranks): everything but the NCCL
 * calls works (partition, remap, parts, run_gathered); run/features with
 * nranks > 1 return NITRO_E_STATE.  For single-GPU checks of multi-rank logic. */
nitro_status_t nitro_dist_init_local(int rank, int nranks, int device, nitro_dist **out);
/* Global features from per-rank feature passes: S1, S2 all-reduced (sum),
 * Lmax and the non-canonical flag all-reduced (max), and D = |union of the
 * ranks' occupied diagonals|, each rank contributing its compacted sorted
 * offset list through one all-gather.  Identical (bit for bit)
 * to the single-GPU features of the whole matrix.  Collective; syncs. */
nitro_status_t nitro_dist_features(nitro_dist *D, nitro_spmv *A_local, nitro_spmv_feat *out);

/* Solver-loop mode: in loops where the y of one
 * multiply is the x of the next (power iteration, Krylov-type methods), the
 * SpMV epilogue stores every y_i straight into EVERY rank's next x layout
 * (all-gather layout, block r at r*B): through NCCL symmetric-memory windows
 * (ncclMemAlloc + ncclCommWindowRegister, peer addresses from the NCCL device
 * API, one LSA barrier per step) on NCCL ranks, through the group's buffers
 * on the loopback transport.  No separate all-gather runs: the exchange is
 * spread over the multiply.  Two layouts alternate (x_k is read from one,
 * x_{k+1} written into the other).  CSR-scalar, ELL and DIA have the fused
 * epilogue; other variants compute the rank's block and push it with a copy
 * kernel.  Requires a handle created with the all-gather exchange
 * (NITRO_E_UNSUPPORTED otherwise) and, on NCCL, every rank in one NVLink
 * domain.  create / start / step are collective (all ranks, same order). */
typedef struct nitro_dist_loop nitro_dist_loop;
nitro_status_t nitro_dist_loop_create(nitro_dist *D, nitro_spmv *A_local, nitro_dist_loop **out);
void nitro_dist_loop_destroy(nitro_dist_loop *L);
/* Device address of this rank's block of the CURRENT x (write x_0 here before start). */
nitro_status_t nitro_dist_loop_x(nitro_dist_loop *L, void **d_x_local);
/* Exchange x_0 once (all-gather into every rank's current layout). */
nitro_status_t nitro_dist_loop_start(nitro_dist_loop *L);
/* One multiply y = A x_k; x_{k+1} = y on every rank (fused epilogue +
 * barrier); d_y_local (nullable) also receives this rank's y block. */
nitro_status_t nitro_dist_loop_step(nitro_dist_loop *L, int variant, void *d_y_local);

/* LOOPBACK transport: P rank handles inside ONE process on ONE GPU, each
 * driven by its own host thread.  Every collective of nitro_dist_* (the
 * exchange-plan all-gather and send/recv in create, the per-multiply x
 * all-gather or halo send/recv, the feature reductions) meets at a host
 * barrier and moves data with device copies ordered on the callers' streams
 * — the same pack / send-list / receive-offset / layout code as NCCL, so the
 * P > 1 paths run (and are tested) on a single GPU.  Each rank's thread calls
 * nitro_dist_init_loopback(L, rank) and then the ordinary nitro_dist_* calls
 * in the same order as the other ranks (as with NCCL).  The group object must
 * outlive its rank handles. */
typedef struct nitro_loopback nitro_loopback;
nitro_status_t nitro_dist_loopback_create(int nranks, int device, nitro_loopback **out);
void nitro_dist_loopback_destroy(nitro_loopback *L);
nitro_status_t nitro_dist_init_loopback(nitro_loopback *L, int rank, nitro_dist **out);

/* ========================================================================
 * 4. Histogram code-variant family: a second workload
 *    through the same generic layer.  PAPER.md P:L216-217 (Fig. 4 row
 *    "Histogram": Sort-ES / Sort-Dynamic, Shared-Atomic-ES /
 *    Shared-Atomic-Dynamic; features N, N/#bins, SubSampleSD), P:L226 (the
 *    CUB variants: "three variants and two grid-mapping strategies thus giving
 *    rise to six code variants"), P:L254 (results), P:L269 (sub-sample size).
 * ======================================================================== */
typedef enum {
  NITRO_HIST_SORT_ES = 0,      /* per tile: sort bin ids in shared memory, run-length -> atomics (default) */
  NITRO_HIST_SORT_DYN = 1,     /* same, tiles from a global atomic queue */
  NITRO_HIST_SHARED_ES = 2,    /* per-CTA shared-memory histogram, merged at the end */
  NITRO_HIST_SHARED_DYN = 3,
  NITRO_HIST_GLOBAL_ES = 4,    /* one global atomic per sample */
  NITRO_HIST_GLOBAL_DYN = 5
} nitro_hist_variant;
#define NITRO_HIST_NUM_VARIANTS 6
typedef struct nitro_hist nitro_hist;
/* An even histogram of n uint32 samples (device array, borrowed; 16-byte
 * alignment enables 128-bit loads):
 *   h[b] = #{ i : s_i < range, floor(s_i * nbins / range) = b },  b < nbins,
 * 1 <= nbins <= 65536, 1 <= range <= 2^32; samples >= range are not counted.
 * All work is enqueued on `stream`. */
nitro_status_t nitro_hist_create(int device, void *stream, int64_t n, const uint32_t *d_samples, int32_t nbins,
                                 uint64_t range, nitro_hist **out);
void nitro_hist_destroy(nitro_hist *H);
/* out3 = {N, N / nbins, SubSampleSD}: SubSampleSD = population standard
 * deviation of s[floor(j*N/k)], j < k, k = min(ceil(N/4), 10000),
 * from exact integer moments: sqrt((double)(k*S2 - S1^2) / ((double)k*k)),
 * 0 for N = 0.  Syncs the stream; cached. */
nitro_status_t nitro_hist_features(nitro_hist *H, double *out3);
/* Constraint: the shared-atomic variants need nbins <= 49152 (192 KB of
 * shared counters per CTA); the others are always allowed. */
nitro_status_t nitro_hist_allowed(nitro_hist *H, int variant, int *out_allowed);
/* d_hist (uint32[nbins], device) = the histogram; async on the stream.
 * NITRO_E_CONSTRAINT for a shared-atomic variant with nbins > 49152.
 * Kernels are launched cooperatively (all CTAs resident: CTA 0 zeroes d_hist
 * and the others wait on a per-handle epoch flag), so the calls of one handle
 * must stay ordered on its stream (no concurrent calls on one handle). */
nitro_status_t nitro_hist_run(nitro_hist *H, int variant, uint32_t *d_hist);
/* Median of reps CUDA-event timings of nitro_hist_run (L2 flushed before
 * each when flush_l2), after warmup untimed runs.  Syncs. */
nitro_status_t nitro_hist_time(nitro_hist *H, int variant, uint32_t *d_hist, int warmup, int reps, int flush_l2,
                               double *out_median_s);
/* Input record of the registered histogram variants. */
typedef struct {
  nitro_hist *H;
  uint32_t *d_hist;
  int warmup, reps, flush_l2;
} nitro_hist_input;
/* Register on a fresh cv: the 6 variants (ids = nitro_hist_variant), the
 * feature group {n, n_per_bin, subsample_sd} (plain [-1, 1] scaling), the
 * shared-memory constraints, default = SORT_ES (always allowed; robust to
 * skewed inputs, where atomics contend). */
nitro_status_t nitro_hist_register(nitro_cv *cv);

#ifdef __cplusplus
}
#endif
#endif /* NITRO_H */
