/* oracle/oracle.c — the CPU oracle of the Nitro SpMV hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.
 * The product (paper_conf_ipps_muralidharanshgc14_b200/, libnitro.so) never
 * links, imports or calls it, and shares no code or header with it.
 *
 * Plain, slow, obviously correct: fp64, sequential loops, no blocking, no
 * fusion, no reordering beyond the written definitions.  Build with
 * -ffp-contract=off so no FMA contraction changes a rounding.
 *
 * Citations: PAPER.md = /root/reference/PAPER.md line numbers (P:L<n>);
 * SURVEY.md §8(c) rows C1..C9 give the readings adopted where the paper is
 * silent (also listed in DESIGN.md "Readings").
 */
#include <math.h>
#include <omp.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

/* ------------------------------------------------------------------ C1 SpMV
 * PAPER.md §II: "for(i = 0; i < nnz; i++) y[row[i]] += A[i]*x[col[i]];"
 * read as y <- A.x (y starts at zero; empty rows give 0), entries summed in
 * storage order k = rowptr[i] .. rowptr[i+1]-1.  r_i = sum_k |A_ik x_col| is
 * the magnitude used by the acceptance tolerance (BASELINE north_star). */
void oracle_spmv(int64_t N, const int64_t *rowptr, const int32_t *col, const double *val,
                 const double *x, double *y, double *r) {
  for (int64_t i = 0; i < N; ++i) {
    double s = 0.0, a = 0.0;
    for (int64_t k = rowptr[i]; k < rowptr[i + 1]; ++k) {
      double p = val[k] * x[col[k]];
      s = s + p;
      a = a + fabs(p);
    }
    y[i] = s;
    if (r) r[i] = a;
  }
}

/* The same loop with the rows split over host threads (OpenMP, static
 * schedule): every row is still summed sequentially in storage order, so y and
 * r are bit-identical to oracle_spmv.  Used only by bench.py's all-core CPU
 * baseline leg (the north star asks for the oracle timed on the box's host
 * cores).  Returns the number of threads that ran. */
int oracle_spmv_threads(int64_t N, const int64_t *rowptr, const int32_t *col, const double *val,
                        const double *x, double *y, double *r, int nthreads) {
  int used = 1;
#pragma omp parallel num_threads(nthreads > 0 ? nthreads : 1)
  {
#pragma omp single
    used = omp_get_num_threads();
#pragma omp for schedule(static)
    for (int64_t i = 0; i < N; ++i) {
      double s = 0.0, a = 0.0;
      for (int64_t k = rowptr[i]; k < rowptr[i + 1]; ++k) {
        double p = val[k] * x[col[k]];
        s = s + p;
        a = a + fabs(p);
      }
      y[i] = s;
      if (r) r[i] = a;
    }
  }
  return used;
}

/* ------------------------------------------------------------------ C4 features
 * PAPER.md §IV L200 (features: average non-zeros per row, standard deviation of
 * the row lengths, deviation of the longest row from the average, DIA and ELL
 * fill-in) and Fig. 2 L97-101 (nnz, num_rows).  Readings:
 * population SD; MaxDeviation = Lmax - mean; fill = stored slots / nnz with
 * DIA slots counted as ndiag*rows; exact integer moments then one fixed fp64
 * finishing expression. */
typedef struct {
  int64_t rows, cols, nnz;
  uint64_t sum_len, sum_len2;
  int64_t max_row, ndiag;
  int32_t canonical, pad_;
  double mean, sd, max_dev, dia_fill, ell_fill;
} oracle_features_t;

/* C3 canonical CSR: rowptr[0]=0, non-decreasing, rowptr[N]=Z, columns strictly
 * increasing within each row, 0 <= col < M. */
int oracle_is_canonical(int64_t N, int64_t M, int64_t Z, const int64_t *rowptr, const int32_t *col) {
  if (rowptr[0] != 0 || rowptr[N] != Z) return 0;
  for (int64_t i = 0; i < N; ++i) {
    if (rowptr[i + 1] < rowptr[i]) return 0;
    for (int64_t k = rowptr[i]; k < rowptr[i + 1]; ++k) {
      if (col[k] < 0 || (int64_t)col[k] >= M) return 0;
      if (k > rowptr[i] && col[k] <= col[k - 1]) return 0;
    }
  }
  return 1;
}

/* The finishing step of C4 on given exact integers (also used alone where the
 * integers come from closed forms, e.g. configs[4] whose CSR does not fit the
 * host): fp64, round-to-nearest, no contraction; all doubles 0 when N = 0.
 * Leaves canonical as it finds it. */
void oracle_finish_features(int64_t N, int64_t M, int64_t Z, uint64_t s1, uint64_t s2, int64_t lmax, int64_t D,
                            oracle_features_t *f) {
  f->rows = N;
  f->cols = M;
  f->nnz = Z;
  f->sum_len = s1;
  f->sum_len2 = s2;
  f->max_row = lmax;
  f->ndiag = D;
  f->mean = f->sd = f->max_dev = f->dia_fill = f->ell_fill = 0.0;
  if (N == 0) return;
  __int128 num = (__int128)N * (__int128)s2 - (__int128)s1 * (__int128)s1;
  int64_t Zc = Z > 1 ? Z : 1;
  f->mean = (double)s1 / (double)N;
  double var = (double)num / ((double)N * (double)N);
  f->sd = sqrt(var);
  f->max_dev = (double)lmax - f->mean;
  f->dia_fill = (double)D * (double)N / (double)Zc;
  f->ell_fill = (double)lmax * (double)N / (double)Zc;
}

/* offsets_out (nullable, capacity N+M-1) receives the distinct diagonal offsets
 * d = col - row in ascending order.  Returns 0. */
int oracle_features(int64_t N, int64_t M, const int64_t *rowptr, const int32_t *col,
                    oracle_features_t *f, int32_t *offsets_out) {
  memset(f, 0, sizeof(*f));
  f->rows = N;
  f->cols = M;
  f->nnz = rowptr[N] - rowptr[0];
  f->canonical = oracle_is_canonical(N, M, f->nnz, rowptr, col);
  if (N == 0) return 0;
  /* exact integer moments of the row lengths */
  uint64_t s1 = 0, s2 = 0;
  int64_t lmax = 0;
  for (int64_t i = 0; i < N; ++i) {
    int64_t L = rowptr[i + 1] - rowptr[i];
    s1 += (uint64_t)L;
    s2 += (uint64_t)L * (uint64_t)L;
    if (L > lmax) lmax = L;
  }
  /* occupied diagonals: mark offset d = col - row at index d + (N-1) */
  int64_t span = N + M - 1;
  unsigned char *seen = (unsigned char *)calloc((size_t)(span > 0 ? span : 1), 1);
  if (!seen) return -1;
  for (int64_t i = 0; i < N; ++i)
    for (int64_t k = rowptr[i]; k < rowptr[i + 1]; ++k) {
      int64_t d = (int64_t)col[k] - i;
      if (d >= -(N - 1) && d <= M - 1) seen[d + (N - 1)] = 1;
    }
  int64_t D = 0;
  for (int64_t t = 0; t < span; ++t)
    if (seen[t]) {
      if (offsets_out) offsets_out[D] = (int32_t)(t - (N - 1));
      ++D;
    }
  free(seen);
  oracle_finish_features(N, M, f->nnz, s1, s2, lmax, D, f);
  return 0;
}

/* ------------------------------------------------------------------ C5 CSR->ELL
 * Column-major, ld >= N rows, width K = Lmax.  Slot (k, i) at k*ld + i holds the
 * k-th entry of row i, else col = -1, val = 0.  (Layout reading: SURVEY C5.) */
int oracle_csr_to_ell(int64_t N, const int64_t *rowptr, const int32_t *col, const double *val,
                      int64_t K, int64_t ld, int32_t *ecol, double *eval) {
  for (int64_t t = 0; t < K * ld; ++t) { ecol[t] = -1; eval[t] = 0.0; }
  for (int64_t i = 0; i < N; ++i) {
    int64_t L = rowptr[i + 1] - rowptr[i];
    if (L > K) return -1;
    for (int64_t k = 0; k < L; ++k) {
      ecol[k * ld + i] = col[rowptr[i] + k];
      eval[k * ld + i] = val[rowptr[i] + k];
    }
  }
  return 0;
}

/* ELL -> CSR (for round trips): row i's entries are its slots k = 0..K-1 with
 * col != -1, in slot order.  rowptr_out[N+1]; returns nnz. */
int64_t oracle_ell_to_csr(int64_t N, int64_t K, int64_t ld, const int32_t *ecol, const double *eval,
                          int64_t *rowptr_out, int32_t *col_out, double *val_out) {
  int64_t z = 0;
  rowptr_out[0] = 0;
  for (int64_t i = 0; i < N; ++i) {
    for (int64_t k = 0; k < K; ++k)
      if (ecol[k * ld + i] != -1) {
        if (col_out) { col_out[z] = ecol[k * ld + i]; val_out[z] = eval[k * ld + i]; }
        ++z;
      }
    rowptr_out[i + 1] = z;
  }
  return z;
}

/* ------------------------------------------------------------------ C6 CSR->DIA
 * PAPER.md L87/L126 (dia_type, "Diagonal [15]").  offsets[D] ascending;
 * slot (d, i) at d*ld + i holds a(i, i+off_d) when stored, else 0
 * (also for out-of-range i+off_d and rows N..ld-1).  Indexed by row. */
int oracle_csr_to_dia(int64_t N, int64_t M, const int64_t *rowptr, const int32_t *col, const double *val,
                      int64_t D, const int32_t *offsets, int64_t ld, double *dval) {
  (void)M;
  for (int64_t t = 0; t < D * ld; ++t) dval[t] = 0.0;
  for (int64_t i = 0; i < N; ++i)
    for (int64_t k = rowptr[i]; k < rowptr[i + 1]; ++k) {
      int64_t off = (int64_t)col[k] - i;
      int64_t d = -1;
      for (int64_t t = 0; t < D; ++t)          /* plain linear search */
        if (offsets[t] == off) { d = t; break; }
      if (d < 0) return -1;
      dval[d * ld + i] = val[k];
    }
  return 0;
}

/* DIA -> CSR: row i emits (i, i+off_d) for every in-range slot with a nonzero
 * value, in ascending column (= ascending offset) order. */
int64_t oracle_dia_to_csr(int64_t N, int64_t M, int64_t D, const int32_t *offsets, int64_t ld,
                          const double *dval, int64_t *rowptr_out, int32_t *col_out, double *val_out) {
  int64_t z = 0;
  rowptr_out[0] = 0;
  for (int64_t i = 0; i < N; ++i) {
    for (int64_t d = 0; d < D; ++d) {
      int64_t j = i + offsets[d];
      if (j < 0 || j >= M) continue;
      double v = dval[d * ld + i];
      if (v != 0.0) {
        if (col_out) { col_out[z] = (int32_t)j; val_out[z] = v; }
        ++z;
      }
    }
    rowptr_out[i + 1] = z;
  }
  return z;
}

/* ------------------------------------------------------------------ C7 CSR->HYB
 * Not in the paper (HYB is in the north star, from the CUSP family P:L47).
 * K_hyb = first k in [0, Lmax) with 3*R_k < N or R_k < 4096, where
 * R_k = |{i : L_i > k}|; else Lmax.  Written as the literal count per k. */
int64_t oracle_hyb_width(int64_t N, const int64_t *rowptr) {
  int64_t lmax = 0;
  for (int64_t i = 0; i < N; ++i)
    if (rowptr[i + 1] - rowptr[i] > lmax) lmax = rowptr[i + 1] - rowptr[i];
  for (int64_t k = 0; k < lmax; ++k) {
    int64_t Rk = 0;
    for (int64_t i = 0; i < N; ++i)
      if (rowptr[i + 1] - rowptr[i] > k) ++Rk;
    if (3 * Rk < N || Rk < 4096) return k;
  }
  return lmax;
}

/* Tail length for width K. */
int64_t oracle_hyb_tail_len(int64_t N, const int64_t *rowptr, int64_t K) {
  int64_t t = 0;
  for (int64_t i = 0; i < N; ++i) {
    int64_t L = rowptr[i + 1] - rowptr[i];
    if (L > K) t += L - K;
  }
  return t;
}

/* ELL part = first min(L_i, K) entries of each row (C5 layout, width K);
 * tail = the remaining entries as (row, col, val) in CSR order. */
int oracle_csr_to_hyb(int64_t N, const int64_t *rowptr, const int32_t *col, const double *val,
                      int64_t K, int64_t ld, int32_t *ecol, double *eval,
                      int32_t *trow, int32_t *tcol, double *tval) {
  for (int64_t t = 0; t < K * ld; ++t) { ecol[t] = -1; eval[t] = 0.0; }
  int64_t z = 0;
  for (int64_t i = 0; i < N; ++i) {
    int64_t L = rowptr[i + 1] - rowptr[i];
    for (int64_t k = 0; k < L; ++k) {
      int64_t src = rowptr[i] + k;
      if (k < K) {
        ecol[k * ld + i] = col[src];
        eval[k * ld + i] = val[src];
      } else {
        trow[z] = (int32_t)i;
        tcol[z] = col[src];
        tval[z] = val[src];
        ++z;
      }
    }
  }
  return 0;
}

/* HYB -> CSR: row i = its ELL slots (slot order) followed by its tail entries
 * (tail order).  Two plain passes: count, then emit. */
int64_t oracle_hyb_to_csr(int64_t N, int64_t K, int64_t ld, const int32_t *ecol, const double *eval,
                          int64_t Zt, const int32_t *trow, const int32_t *tcol, const double *tval,
                          int64_t *rowptr_out, int32_t *col_out, double *val_out) {
  int64_t *cnt = (int64_t *)calloc((size_t)N + 1, sizeof(int64_t));
  if (!cnt) return -1;
  for (int64_t i = 0; i < N; ++i)
    for (int64_t k = 0; k < K; ++k)
      if (ecol[k * ld + i] != -1) cnt[i]++;
  for (int64_t t = 0; t < Zt; ++t) cnt[trow[t]]++;
  rowptr_out[0] = 0;
  for (int64_t i = 0; i < N; ++i) rowptr_out[i + 1] = rowptr_out[i] + cnt[i];
  if (col_out) {
    for (int64_t i = 0; i < N; ++i) cnt[i] = rowptr_out[i];
    for (int64_t i = 0; i < N; ++i)
      for (int64_t k = 0; k < K; ++k)
        if (ecol[k * ld + i] != -1) { col_out[cnt[i]] = ecol[k * ld + i]; val_out[cnt[i]] = eval[k * ld + i]; cnt[i]++; }
    for (int64_t t = 0; t < Zt; ++t) { col_out[cnt[trow[t]]] = tcol[t]; val_out[cnt[trow[t]]] = tval[t]; cnt[trow[t]]++; }
  }
  int64_t z = rowptr_out[N];
  free(cnt);
  return z;
}

/* ------------------------------------------------------------------ C9 constraints
 * PAPER.md §II-B L134 (constraints rule a variant out; L105-106 dia_cutoff).
 * Readings: fill cutoff 3.0 and a memory budget (bytes) for the padded format. */
int oracle_dia_allowed(const oracle_features_t *f, int64_t ld, int64_t sv, double budget_bytes) {
  return f->dia_fill <= 3.0 && (double)f->ndiag * (double)ld * (double)sv <= budget_bytes;
}
int oracle_ell_allowed(const oracle_features_t *f, int64_t ld, int64_t sv, double budget_bytes) {
  return f->ell_fill <= 3.0 && (double)f->max_row * (double)ld * (double)(sv + 4) <= budget_bytes;
}

int oracle_features_size(void) { return (int)sizeof(oracle_features_t); }
