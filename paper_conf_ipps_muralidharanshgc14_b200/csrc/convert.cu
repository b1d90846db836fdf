// convert.cu — A5: CSR -> ELL / DIA / HYB(ELL + COO tail), and the CSR-vector
// long-row segment table.  Conversions are cached per matrix and excluded from
// variant time (their cost is amortised over repeated SpMVs).
//
// Layouts (R5-R7): column-major, pitch ld = round_up(N, 32) rows so
// every (slot, 4-row group) is 16-byte aligned for 128-bit loads; ELL padding
// col = -1, val = 0; DIA indexed by row (val[d*ld + i] = a(i, i+off_d));
// HYB = ELL of width K_hyb + tail (row, col, val) in CSR order.
#include "nitro_internal.h"
#include "util.cuh"

#include <algorithm>
#include <vector>

namespace nitro {
namespace {

constexpr int64_t kTailThread = 64, kTailPiece = 4096;

template <typename IT, typename VT>
__global__ void k_fill_ell(const IT *__restrict__ rowptr, const int32_t *__restrict__ col, const VT *__restrict__ val,
                           int64_t N, int64_t K, int64_t ld, int32_t *__restrict__ ecol, VT *__restrict__ eval,
                           const int64_t *__restrict__ toff, int32_t *__restrict__ trow, int32_t *__restrict__ tcol,
                           VT *__restrict__ tval) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < ld; i += (int64_t)gridDim.x * blockDim.x) {
    int64_t a = 0, L = 0;
    if (i < N) { a = (int64_t)rowptr[i]; L = (int64_t)rowptr[i + 1] - a; }
    for (int64_t k = 0; k < K; ++k) {
      const bool in = k < L;
      ecol[k * ld + i] = in ? col[a + k] : -1;
      eval[k * ld + i] = in ? val[a + k] : (VT)0;
    }
    if (toff && L > K && L - K <= kTailThread) {  // longer tails: k_fill_tail_tasks
      int64_t o = toff[i];
      for (int64_t k = K; k < L; ++k, ++o) {
        trow[o] = (int32_t)i;
        tcol[o] = col[a + k];
        tval[o] = val[a + k];
      }
    }
  }
}

// HYB tails longer than kTailThread entries are copied by whole warps, in
// (row, piece of kTailPiece entries) tasks spread over the grid (an R-MAT hub
// row's 1.5e5-entry tail would serialise one thread for milliseconds)
template <typename IT>
__global__ void k_tail_tasks_count(const IT *__restrict__ rowptr, int64_t N, int64_t K, int64_t *__restrict__ cnt) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < N; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t t = (int64_t)rowptr[i + 1] - (int64_t)rowptr[i] - K;
    cnt[i] = t > kTailThread ? (t + kTailPiece - 1) / kTailPiece : 0;
  }
}
__global__ void k_tail_tasks_emit(const int64_t *__restrict__ off, int64_t N, int2 *__restrict__ tasks) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < N; i += (int64_t)gridDim.x * blockDim.x)
    for (int64_t t = off[i]; t < off[i + 1]; ++t) tasks[t] = make_int2((int)i, (int)(t - off[i]));
}
template <typename IT, typename VT>
__global__ void k_fill_tail_tasks(const IT *__restrict__ rowptr, const int32_t *__restrict__ col,
                                  const VT *__restrict__ val, int64_t K, const int64_t *__restrict__ toff,
                                  const int2 *__restrict__ tasks, int64_t ntask, int32_t *__restrict__ trow,
                                  int32_t *__restrict__ tcol, VT *__restrict__ tval) {
  const int lane = threadIdx.x & 31;
  const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t t = gw; t < ntask; t += nw) {
    const int2 tk = tasks[t];
    const int64_t a = (int64_t)rowptr[tk.x], b = (int64_t)rowptr[tk.x + 1];
    const int64_t st = a + K + (int64_t)tk.y * kTailPiece, en = st + kTailPiece < b ? st + kTailPiece : b;
    const int64_t o = toff[tk.x] + (int64_t)tk.y * kTailPiece - st;
#pragma unroll 4
    for (int64_t e = st + lane; e < en; e += 32) {
      trow[o + e] = tk.x;
      tcol[o + e] = col[e];
      tval[o + e] = val[e];
    }
  }
}

// HYB fixup plan: the carry slots a tail multiply fills are fixed by the
// structure — slot 2c = row of chunk c's first entry, slot 2c+1 = row of its
// last (left empty by the tail kernel when it equals the first).  With
// eff[2c+1] = that last row either way, slots of one row are a contiguous run.
__global__ void k_fix_eff(const int32_t *__restrict__ trow, int64_t Zt, int64_t CH, int64_t nch,
                          int32_t *__restrict__ eff) {
  for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c < nch; c += (int64_t)gridDim.x * blockDim.x) {
    const int64_t s0 = c * CH, e1 = (s0 + CH < Zt ? s0 + CH : Zt) - 1;
    eff[2 * c] = trow[s0];
    eff[2 * c + 1] = trow[e1];
  }
}
__global__ void k_fix_heads(const int32_t *__restrict__ eff, int64_t n, int64_t *__restrict__ h) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x)
    h[j] = (j == 0 || eff[j] != eff[j - 1]) ? 1 : 0;
}
__global__ void k_fix_emit(const int32_t *__restrict__ eff, const int64_t *__restrict__ pos, int64_t n,
                           int32_t *__restrict__ seg) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x)
    if (j == 0 || eff[j] != eff[j - 1]) seg[pos[j]] = (int32_t)j;
  if (blockIdx.x == 0 && threadIdx.x == 0) seg[pos[n]] = (int32_t)n;
}
__global__ void k_fix_long(const int32_t *__restrict__ seg, int64_t S, int32_t *__restrict__ lst,
                           unsigned long long *__restrict__ cnt) {
  for (int64_t s = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; s < S; s += (int64_t)gridDim.x * blockDim.x)
    if (seg[s + 1] - seg[s] > 32) lst[atomicAdd(cnt, 1ull)] = (int32_t)s;
}

// tail count per row (HYB): max(L_i - K, 0)
template <typename IT>
__global__ void k_tail_counts(const IT *__restrict__ rowptr, int64_t N, int64_t K, int64_t *__restrict__ cnt) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < N; i += (int64_t)gridDim.x * blockDim.x) {
    int64_t L = (int64_t)rowptr[i + 1] - (int64_t)rowptr[i];
    cnt[i] = L > K ? L - K : 0;
  }
}

// histogram of row lengths over the window [k0, k0 + W): bins[t] = #rows with
// L == k0 + t, bins[W] = #rows with L >= k0 + W.
template <typename IT, int W>
__global__ void __launch_bounds__(256) k_len_hist(const IT *__restrict__ rowptr, int64_t N, int64_t k0,
                                                  unsigned long long *__restrict__ bins) {
  __shared__ unsigned s[W + 1];
  for (int t = threadIdx.x; t <= W; t += blockDim.x) s[t] = 0;
  __syncthreads();
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < N; i += (int64_t)gridDim.x * blockDim.x) {
    int64_t L = (int64_t)rowptr[i + 1] - (int64_t)rowptr[i];
    int64_t t = L - k0;
    if (t < 0) continue;
    int b = t >= W ? W : (int)t;
    // warp-aggregated increment: lanes with the same bin add once
    unsigned grp = __match_any_sync(__activemask(), b);
    if ((int)(__ffs(grp) - 1) == (int)(threadIdx.x & 31)) atomicAdd(&s[b], (unsigned)__popc(grp));
  }
  __syncthreads();
  for (int t = threadIdx.x; t <= W; t += blockDim.x)
    if (s[t]) atomicAdd(&bins[t], (unsigned long long)s[t]);
}

// DIA offsets: popcount per tile of 1024 bitmap words, then emit ascending
__global__ void __launch_bounds__(256) k_popc_tiles(const uint32_t *__restrict__ bm, int64_t nwords,
                                                    int64_t *__restrict__ cnt) {
  int64_t base = (int64_t)blockIdx.x * 1024;
  int64_t s = 0;
  for (int t = threadIdx.x; t < 1024; t += 256)
    if (base + t < nwords) s += __popc(bm[base + t]);
  s = block_sum_i64<256>(s);
  if (threadIdx.x == 0) cnt[blockIdx.x] = s;
}
__global__ void __launch_bounds__(256) k_emit_offsets(const uint32_t *__restrict__ bm, int64_t nwords,
                                                      const int64_t *__restrict__ tile_off, int64_t G,
                                                      int32_t *__restrict__ out) {
  int64_t base = (int64_t)blockIdx.x * 1024 + threadIdx.x * 4;
  uint32_t w[4];
  int64_t c = 0;
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    w[q] = base + q < nwords ? bm[base + q] : 0u;
    c += __popc(w[q]);
  }
  int64_t agg;
  int64_t o = tile_off[blockIdx.x] + block_exclusive_i64<256>(c, agg);
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    uint32_t v = w[q];
    while (v) {
      int b = __ffs(v) - 1;
      v &= v - 1;
      out[o++] = (int32_t)((base + q) * 32 + b - G);
    }
  }
}

template <typename IT, typename VT>
__global__ void k_fill_dia(const IT *__restrict__ rowptr, const int32_t *__restrict__ col, const VT *__restrict__ val,
                           int64_t N, int64_t row0, const int32_t *__restrict__ offs, int64_t D, int64_t ld,
                           VT *__restrict__ dval) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < N; i += (int64_t)gridDim.x * blockDim.x) {
    int64_t a = (int64_t)rowptr[i], b = (int64_t)rowptr[i + 1];
    if (a == b) continue;
    // binary search the first entry's offset, then walk (offsets ascend with columns)
    int64_t off0 = (int64_t)col[a] - (row0 + i);
    int64_t lo = 0, hi = D;
    while (lo < hi) {
      int64_t mid = (lo + hi) >> 1;
      if ((int64_t)__ldg(offs + mid) < off0) lo = mid + 1; else hi = mid;
    }
    int64_t d = lo;
    for (int64_t k = a; k < b; ++k) {
      int64_t off = (int64_t)col[k] - (row0 + i);
      while (d < D && (int64_t)__ldg(offs + d) < off) ++d;
      dval[d * ld + i] = val[k];
    }
  }
}

// CSR-vector long rows: flag rows with L > T, then emit row ids ascending
template <typename IT>
__global__ void k_long_flags(const IT *__restrict__ rowptr, int64_t N, int64_t T, int64_t S,
                             int64_t *__restrict__ nseg) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < N; i += (int64_t)gridDim.x * blockDim.x) {
    int64_t L = (int64_t)rowptr[i + 1] - (int64_t)rowptr[i];
    nseg[i] = L > T ? (L + S - 1) / S : 0;
  }
}
// segment table: seg_row[s], seg_first[s] (index of the row's first segment),
// seg_count[s]; segments of a row are consecutive.
template <typename IT>
__global__ void k_long_emit(const IT *__restrict__ rowptr, int64_t N, const int64_t *__restrict__ segoff,
                            int32_t *__restrict__ seg_row, int32_t *__restrict__ seg_k) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < N; i += (int64_t)gridDim.x * blockDim.x) {
    int64_t s0 = segoff[i], s1 = segoff[i + 1];
    for (int64_t s = s0; s < s1; ++s) {
      seg_row[s] = (int32_t)i;
      seg_k[s] = (int32_t)(s - s0);  // segment ordinal within its row
    }
  }
}

unsigned grid_of(int64_t n, int threads = 256) {
  int64_t g = (n + threads - 1) / threads;
  int64_t cap = (int64_t)num_sms() * 16;
  if (g > cap) g = cap;
  return (unsigned)(g < 1 ? 1 : g);
}

template <typename IT, typename VT>
nitro_status_t fill_ell_t(nitro_spmv *A, int64_t K, int64_t ld, int32_t *ecol, VT *eval, const int64_t *toff,
                          int32_t *trow, int32_t *tcol, VT *tval) {
  k_fill_ell<IT, VT><<<grid_of(ld), 256, 0, A->stream>>>((const IT *)A->rowptr, A->col, (const VT *)A->val, A->N, K,
                                                         ld, ecol, eval, toff, trow, tcol, tval);
  NITRO_CUDA(cudaGetLastError());
  return NITRO_OK;
}

nitro_status_t fill_ell(nitro_spmv *A, int64_t K, int64_t ld, void *ecol, void *eval, const int64_t *toff,
                        void *trow, void *tcol, void *tval) {
  if (A->rp64) {
    if (A->fp64) return fill_ell_t<int64_t, double>(A, K, ld, (int32_t *)ecol, (double *)eval, toff, (int32_t *)trow, (int32_t *)tcol, (double *)tval);
    return fill_ell_t<int64_t, float>(A, K, ld, (int32_t *)ecol, (float *)eval, toff, (int32_t *)trow, (int32_t *)tcol, (float *)tval);
  }
  if (A->fp64) return fill_ell_t<int32_t, double>(A, K, ld, (int32_t *)ecol, (double *)eval, toff, (int32_t *)trow, (int32_t *)tcol, (double *)tval);
  return fill_ell_t<int32_t, float>(A, K, ld, (int32_t *)ecol, (float *)eval, toff, (int32_t *)trow, (int32_t *)tcol, (float *)tval);
}

}  // namespace

// ------------------------------------------------------------------ ELL (C5)
nitro_status_t prepare_ell(nitro_spmv *A) {
  if (A->ell.ready) return NITRO_OK;
  NITRO_TRY(features_finish(A));
  const int64_t K = A->feat.max_row, ld = round_up(A->N, 32), sv = A->fp64 ? 8 : 4;
  NITRO_TRY(A->ell.col.alloc((size_t)std::max<int64_t>(K * ld, 1) * 4));
  NITRO_TRY(A->ell.val.alloc((size_t)std::max<int64_t>(K * ld, 1) * sv));
  if (K > 0) NITRO_TRY(fill_ell(A, K, ld, A->ell.col.p, A->ell.val.p, nullptr, nullptr, nullptr, nullptr));
  A->ell.K = K;
  A->ell.ld = ld;
  A->ell.ready = true;
  return NITRO_OK;
}

// ------------------------------------------------------------------ DIA (C6)
nitro_status_t prepare_dia(nitro_spmv *A) {
  if (A->dia.ready) return NITRO_OK;
  NITRO_TRY(features_finish(A));
  cudaStream_t s = A->stream;
  const int64_t D = A->feat.ndiag, ld = round_up(A->N, 32), sv = A->fp64 ? 8 : 4;
  const int64_t G = diag_shift(A);
  const int64_t span = A->N > 0 ? G + A->M : 0, nwords = (span + 31) / 32;
  NITRO_TRY(A->dia.off.alloc((size_t)std::max<int64_t>(D, 1) * 4));
  if (D > 0) {
    const int64_t nt = (nwords + 1023) / 1024;
    DevBuf cnt;
    NITRO_TRY(cnt.alloc((size_t)(2 * nt + 2) * 8));
    int64_t *tile_cnt = cnt.as<int64_t>(), *tile_off = tile_cnt + nt + 1;
    k_popc_tiles<<<(unsigned)nt, 256, 0, s>>>(A->bitmap.as<uint32_t>(), nwords, tile_cnt);
    NITRO_TRY(exclusive_scan_i64(tile_cnt, tile_off, nt, A->scratch, s));
    k_emit_offsets<<<(unsigned)nt, 256, 0, s>>>(A->bitmap.as<uint32_t>(), nwords, tile_off, G, A->dia.off.as<int32_t>());
    NITRO_CUDA(cudaGetLastError());
  }
  NITRO_TRY(A->dia.val.alloc((size_t)std::max<int64_t>(D * ld, 1) * sv));
  if (D > 0) {
    NITRO_CUDA(cudaMemsetAsync(A->dia.val.p, 0, (size_t)(D * ld * sv), s));
    const unsigned g = grid_of(A->N);
    if (A->rp64) {
      if (A->fp64) k_fill_dia<int64_t, double><<<g, 256, 0, s>>>((const int64_t *)A->rowptr, A->col, (const double *)A->val, A->N, A->row0, A->dia.off.as<int32_t>(), D, ld, A->dia.val.as<double>());
      else k_fill_dia<int64_t, float><<<g, 256, 0, s>>>((const int64_t *)A->rowptr, A->col, (const float *)A->val, A->N, A->row0, A->dia.off.as<int32_t>(), D, ld, A->dia.val.as<float>());
    } else {
      if (A->fp64) k_fill_dia<int32_t, double><<<g, 256, 0, s>>>((const int32_t *)A->rowptr, A->col, (const double *)A->val, A->N, A->row0, A->dia.off.as<int32_t>(), D, ld, A->dia.val.as<double>());
      else k_fill_dia<int32_t, float><<<g, 256, 0, s>>>((const int32_t *)A->rowptr, A->col, (const float *)A->val, A->N, A->row0, A->dia.off.as<int32_t>(), D, ld, A->dia.val.as<float>());
    }
    NITRO_CUDA(cudaGetLastError());
  }
  // in-range slots (compulsory bytes): sum_d |{i : 0 <= row0+i+off_d < M}|
  std::vector<int32_t> h(D);
  if (D > 0) {
    NITRO_CUDA(cudaMemcpyAsync(h.data(), A->dia.off.p, (size_t)D * 4, cudaMemcpyDeviceToHost, s));
    NITRO_CUDA(cudaStreamSynchronize(s));
  }
  int64_t inr = 0;
  for (int64_t d = 0; d < D; ++d) {
    int64_t lo = std::max<int64_t>(0, -(A->row0 + h[d])), hi = std::min<int64_t>(A->N, A->M - A->row0 - h[d]);
    if (hi > lo) inr += hi - lo;
  }
  A->dia.off_min = D > 0 ? h[0] : 0;
  A->dia.off_max = D > 0 ? h[D - 1] : 0;
  A->dia.D = D;
  A->dia.ld = ld;
  A->dia.inrange = inr;
  A->dia.ready = true;
  return NITRO_OK;
}

int hyb_windows(size_t sv) {
  static int env = [] {
    const char *e = getenv("NITRO_HYB_W");
    return e ? atoi(e) : 0;
  }();
  if (env == 4 || env == 8) return env;
  return sv == 8 ? 4 : 8;
}

// ------------------------------------------------------------------ HYB (C7)
nitro_status_t prepare_hyb(nitro_spmv *A) {
  if (A->hyb.ready) return NITRO_OK;
  NITRO_TRY(features_finish(A));
  cudaStream_t s = A->stream;
  const int64_t N = A->N, lmax = A->feat.max_row, ld = round_up(N, 32), sv = A->fp64 ? 8 : 4;
  // K_hyb = first k in [0, Lmax) with 3 R_k < N or R_k < 4096 (R_k = #rows with L > k); else Lmax
  constexpr int W = 1024;
  int64_t K = lmax, Rk_at_K = 0;
  {
    DevBuf bins;
    NITRO_TRY(bins.alloc((W + 1) * sizeof(unsigned long long)));
    std::vector<unsigned long long> hb(W + 1);
    bool found = false;
    // R_{k0-1} = #rows with L >= k0; start with R_{-1} = N
    for (int64_t k0 = 0; k0 < lmax && !found; k0 += W) {
      NITRO_CUDA(cudaMemsetAsync(bins.p, 0, bins.bytes, s));
      if (A->rp64) k_len_hist<int64_t, W><<<grid_of(N), 256, 0, s>>>((const int64_t *)A->rowptr, N, k0, bins.as<unsigned long long>());
      else k_len_hist<int32_t, W><<<grid_of(N), 256, 0, s>>>((const int32_t *)A->rowptr, N, k0, bins.as<unsigned long long>());
      NITRO_CUDA(cudaGetLastError());
      NITRO_CUDA(cudaMemcpyAsync(hb.data(), bins.p, bins.bytes, cudaMemcpyDeviceToHost, s));
      NITRO_CUDA(cudaStreamSynchronize(s));
      // rows with L >= k0
      int64_t ge = 0;
      for (int t = 0; t <= W; ++t) ge += (int64_t)hb[t];
      for (int t = 0; t < W && k0 + t < lmax; ++t) {
        ge -= (int64_t)hb[t];  // now ge = #rows with L > k0 + t = R_{k0+t}
        if (3 * ge < N || ge < 4096) { K = k0 + t; Rk_at_K = ge; found = true; break; }
      }
    }
  }
  A->hyb.tail_rows = Rk_at_K;  // rows with L > K (0 when K = Lmax)
  DevBuf cnt;
  NITRO_TRY(cnt.alloc((size_t)(2 * N + 2) * 8));
  int64_t *c = cnt.as<int64_t>(), *toff = c + N + 1;
  int64_t Zt = 0;
  if (N > 0) {
    if (A->rp64) k_tail_counts<int64_t><<<grid_of(N), 256, 0, s>>>((const int64_t *)A->rowptr, N, K, c);
    else k_tail_counts<int32_t><<<grid_of(N), 256, 0, s>>>((const int32_t *)A->rowptr, N, K, c);
    NITRO_TRY(exclusive_scan_i64(c, toff, N, A->scratch, s));
    NITRO_CUDA(cudaMemcpyAsync(&Zt, toff + N, 8, cudaMemcpyDeviceToHost, s));
    NITRO_CUDA(cudaStreamSynchronize(s));
  }
  NITRO_TRY(A->hyb.col.alloc((size_t)std::max<int64_t>(K * ld, 1) * 4));
  NITRO_TRY(A->hyb.val.alloc((size_t)std::max<int64_t>(K * ld, 1) * sv));
  NITRO_TRY(A->hyb.trow.alloc((size_t)std::max<int64_t>(Zt, 1) * 4));
  NITRO_TRY(A->hyb.tcol.alloc((size_t)std::max<int64_t>(Zt, 1) * 4));
  NITRO_TRY(A->hyb.tval.alloc((size_t)std::max<int64_t>(Zt, 1) * sv));
  A->hyb.W = hyb_windows((size_t)sv);
  const int64_t chunk = 32 * A->hyb.W;
  const int64_t nch = (Zt + chunk - 1) / chunk;
  NITRO_TRY(A->hyb.carry_row.alloc((size_t)std::max<int64_t>(2 * nch, 1) * 4));
  NITRO_TRY(A->hyb.carry_val.alloc((size_t)std::max<int64_t>(2 * nch, 1) * 8));
  if (N > 0)
    NITRO_TRY(fill_ell(A, K, ld, A->hyb.col.p, A->hyb.val.p, Zt > 0 ? toff : nullptr, A->hyb.trow.p, A->hyb.tcol.p,
                       A->hyb.tval.p));
  if (Zt > 0 && lmax - K > kTailThread) {
    // long tails: (row, piece) tasks, one warp each
    DevBuf tc;
    NITRO_TRY(tc.alloc((size_t)(2 * N + 2) * 8));
    int64_t *tcnt = tc.as<int64_t>(), *tof = tcnt + N + 1;
    if (A->rp64) k_tail_tasks_count<int64_t><<<grid_of(N), 256, 0, s>>>((const int64_t *)A->rowptr, N, K, tcnt);
    else k_tail_tasks_count<int32_t><<<grid_of(N), 256, 0, s>>>((const int32_t *)A->rowptr, N, K, tcnt);
    NITRO_TRY(exclusive_scan_i64(tcnt, tof, N, A->scratch, s));
    int64_t ntask = 0;
    NITRO_CUDA(cudaMemcpyAsync(&ntask, tof + N, 8, cudaMemcpyDeviceToHost, s));
    NITRO_CUDA(cudaStreamSynchronize(s));
    DevBuf tk;
    NITRO_TRY(tk.alloc((size_t)std::max<int64_t>(ntask, 1) * sizeof(int2)));
    k_tail_tasks_emit<<<grid_of(N), 256, 0, s>>>(tof, N, tk.as<int2>());
    const unsigned gt = (unsigned)std::max<int64_t>(1, std::min<int64_t>((ntask + 7) / 8, (int64_t)num_sms() * 8));
#define NITRO_TT(IT, VT)                                                                                        \
  k_fill_tail_tasks<IT, VT><<<gt, 256, 0, s>>>((const IT *)A->rowptr, A->col, (const VT *)A->val, K, toff,    \
                                              tk.as<int2>(), ntask, A->hyb.trow.as<int32_t>(),                \
                                              A->hyb.tcol.as<int32_t>(), A->hyb.tval.as<VT>())
    if (A->rp64) { if (A->fp64) NITRO_TT(int64_t, double); else NITRO_TT(int64_t, float); }
    else { if (A->fp64) NITRO_TT(int32_t, double); else NITRO_TT(int32_t, float); }
#undef NITRO_TT
    NITRO_CUDA(cudaGetLastError());
    NITRO_CUDA(cudaStreamSynchronize(s));  // tc / tk are freed on return
  }
  // fixup plan (see k_fix_eff)
  A->hyb.fix_S = A->hyb.fix_nlong = 0;
  if (Zt > 0) {
    const int64_t nslot = 2 * nch;
    DevBuf fx;
    NITRO_TRY(fx.alloc((size_t)nslot * 4 + (size_t)(2 * nslot + 2) * 8 + 8));
    int32_t *eff = fx.as<int32_t>();
    int64_t *hd = reinterpret_cast<int64_t *>(fx.as<char>() + round_up(nslot * 4, 8)), *pos = hd + nslot + 1;
    k_fix_eff<<<grid_of(nch), 256, 0, s>>>(A->hyb.trow.as<int32_t>(), Zt, chunk, nch, eff);
    k_fix_heads<<<grid_of(nslot), 256, 0, s>>>(eff, nslot, hd);
    NITRO_TRY(exclusive_scan_i64(hd, pos, nslot, A->scratch, s));
    int64_t S = 0;
    NITRO_CUDA(cudaMemcpyAsync(&S, pos + nslot, 8, cudaMemcpyDeviceToHost, s));
    NITRO_CUDA(cudaStreamSynchronize(s));
    NITRO_TRY(A->hyb.fix_seg.alloc((size_t)(S + 1) * 4));
    NITRO_TRY(A->hyb.fix_long.alloc((size_t)std::max<int64_t>(S, 1) * 4));
    k_fix_emit<<<grid_of(nslot), 256, 0, s>>>(eff, pos, nslot, A->hyb.fix_seg.as<int32_t>());
    DevBuf lc;
    NITRO_TRY(lc.alloc(8));
    NITRO_CUDA(cudaMemsetAsync(lc.p, 0, 8, s));
    k_fix_long<<<grid_of(S), 256, 0, s>>>(A->hyb.fix_seg.as<int32_t>(), S, A->hyb.fix_long.as<int32_t>(),
                                          lc.as<unsigned long long>());
    NITRO_CUDA(cudaGetLastError());
    unsigned long long nl = 0;
    NITRO_CUDA(cudaMemcpyAsync(&nl, lc.p, 8, cudaMemcpyDeviceToHost, s));
    NITRO_CUDA(cudaStreamSynchronize(s));
    A->hyb.fix_S = S;
    A->hyb.fix_nlong = (int64_t)nl;
  }
  NITRO_CUDA(cudaStreamSynchronize(s));  // cnt is freed on return
  A->hyb.K = K;
  A->hyb.ld = ld;
  A->hyb.Zt = Zt;
  A->hyb.nchunks = nch;
  A->hyb.ready = true;
  return NITRO_OK;
}

bool csrv_stream_mode(const nitro_spmv *A) {
  static int env = [] {
    const char *e = getenv("NITRO_CSRV_STREAM");
    return e ? atoi(e) : -1;
  }();
  if (A->csr_impl == NITRO_CSR_IMPL_STREAM) return true;
  if (A->csr_impl != NITRO_CSR_IMPL_AUTO) return false;
  if (env == 0 || env == 1) return env == 1;
  return A->feat_ready && A->feat.sd > A->feat.mean;
}

// K6v (vector-load CSR-vector) for regular rows: explicit NITRO_CSR_IMPL_VEC4,
// or AUTO when not in stream mode, the longest row is at most 16 steps of 4V
// entries, and col / val are 16-byte aligned (NITRO_CSRV_VEC=0 / 1 overrides
// the AUTO choice)
bool csrv_vec_mode(const nitro_spmv *A) {
  static int env = [] {
    const char *e = getenv("NITRO_CSRV_VEC");
    return e ? atoi(e) : -1;
  }();
  const bool aligned = ((reinterpret_cast<uintptr_t>(A->col) | reinterpret_cast<uintptr_t>(A->val)) & 15) == 0;
  if (!aligned || !A->csrv.ready || A->csrv.stream) return false;
  if (A->csr_impl == NITRO_CSR_IMPL_VEC4) return true;
  if (A->csr_impl != NITRO_CSR_IMPL_AUTO || env == 0) return false;
  const bool bounded = A->feat_ready && A->feat.max_row <= 16LL * 4 * A->csrv.V;
  return bounded && (env == 1 || kCsrvVecDefault);
}

// NITRO_CSRV_HOT=0 disables the hot-x staging of K6s; =2 skips its benefit
// test (small matrices: tools/sanitize_run.py exercises the kernel that way)
int csrv_hot_env() {
  static int env = [] {
    const char *e = getenv("NITRO_CSRV_HOT");
    return e ? atoi(e) : 1;
  }();
  return env;
}
bool csrv_hot_on() { return csrv_hot_env() != 0; }
// NITRO_CSRV_HOT_KB: shared memory for the hot x values per CTA (KB, 8-96).
// Default 48 (6144 fp64): two CTAs then fit the 132 KB shared carveout and
// keep 124 KB of L1 for the other gathers; B200, configs[2] R-MAT: 16 KB 0.671,
// 32 KB 0.663, 48 KB 0.654, 56 KB 0.695 (the 164 KB carveout), 64 KB 0.688,
// 80 KB 0.861 ms; forcing the max-shared carveout: 1.73 ms (L1 starved)
int csrv_hot_kb() {
  static int kb = [] {
    const char *e = getenv("NITRO_CSRV_HOT_KB");
    const int v = e ? atoi(e) : 48;
    return v < 8 ? 8 : v > 96 ? 96 : v;
  }();
  return kb;
}
bool csrv_hot_forced() { return csrv_hot_env() == 2; }

// ------------------------------------------------------------------ CSR-vector stream mode (K6s)
// chunk_row[c] = the row holding entry c*CH (the last row whose start <= c*CH),
// chunk_row[nch] = N; eff[2c] / eff[2c+1] = rows of the chunk's first / last
// entry (the carry slots' rows, grouped into the fixup plan like HYB's)
template <typename IT>
__global__ void k_stream_rows(const IT *__restrict__ rowptr, int64_t N, int64_t Z, int64_t CH, int64_t nch,
                              int32_t *__restrict__ chunk_row, int32_t *__restrict__ eff) {
  auto row_of = [&](int64_t e) {  // last r with rowptr[r] <= e
    int64_t lo = 0, hi = N;        // rowptr[lo] <= e < rowptr[hi] (rowptr[N] = Z > e)
    while (hi - lo > 1) {
      const int64_t m = (lo + hi) >> 1;
      if ((int64_t)rowptr[m] <= e) lo = m; else hi = m;
    }
    return (int32_t)lo;
  };
  for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c <= nch; c += (int64_t)gridDim.x * blockDim.x) {
    if (c == nch) { chunk_row[c] = (int32_t)N; continue; }
    const int64_t s0 = c * CH, e1 = (s0 + CH < Z ? s0 + CH : Z) - 1;
    const int32_t r0 = row_of(s0);
    chunk_row[c] = r0;
    eff[2 * c] = r0;
    eff[2 * c + 1] = row_of(e1);
  }
}

// ------------------------------------------------------------------ K6s hot-x staging
__global__ void k_col_deg(const int32_t *__restrict__ col, int64_t Z, unsigned *__restrict__ deg) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < Z; e += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(deg + col[e], 1u);
}
// bins[b] = #columns with floor(log2(deg)) == b (deg >= 1), b < 32
__global__ void k_deg_hist(const unsigned *__restrict__ deg, int64_t M, unsigned long long *__restrict__ bins) {
  __shared__ unsigned long long sb[32];
  if (threadIdx.x < 32) sb[threadIdx.x] = 0;
  __syncthreads();
  for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c < M; c += (int64_t)gridDim.x * blockDim.x)
    if (deg[c]) atomicAdd(&sb[31 - __clz(deg[c])], 1ull);
  __syncthreads();
  if (threadIdx.x < 32 && sb[threadIdx.x]) atomicAdd(bins + threadIdx.x, sb[threadIdx.x]);
}
__global__ void k_deg_count(const unsigned *__restrict__ deg, int64_t M, unsigned t,
                            unsigned long long *__restrict__ out) {
  unsigned long long c = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < M; i += (int64_t)gridDim.x * blockDim.x)
    c += deg[i] >= t;
  for (int o = 16; o > 0; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
  if ((threadIdx.x & 31) == 0 && c) atomicAdd(out, c);
}
__global__ void k_hot_flags(const unsigned *__restrict__ deg, int64_t M, unsigned thr, int64_t *__restrict__ f,
                            unsigned long long *__restrict__ covered) {
  unsigned long long cv = 0;
  for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c < M; c += (int64_t)gridDim.x * blockDim.x) {
    const bool h = deg[c] >= thr;
    f[c] = h ? 1 : 0;
    if (h) cv += deg[c];
  }
  for (int o = 16; o > 0; o >>= 1) cv += __shfl_xor_sync(0xffffffffu, cv, o);
  if ((threadIdx.x & 31) == 0 && cv) atomicAdd(covered, cv);
}
// hot column c -> slot pos[c]: hot_cols[slot] = c, and slot_of[c] = slot (else -1)
__global__ void k_hot_emit(const int64_t *__restrict__ f, const int64_t *__restrict__ pos, int64_t M,
                           int32_t *__restrict__ hot_cols, int32_t *__restrict__ slot_of) {
  for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c < M; c += (int64_t)gridDim.x * blockDim.x) {
    if (f[c]) { hot_cols[pos[c]] = (int32_t)c; slot_of[c] = (int32_t)pos[c]; }
    else slot_of[c] = -1;
  }
}
__global__ void k_hot_remap(const int32_t *__restrict__ col, int64_t Z, const int32_t *__restrict__ slot_of,
                            int32_t *__restrict__ hcol) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < Z; e += (int64_t)gridDim.x * blockDim.x) {
    const int32_t c = col[e], sl = slot_of[c];
    hcol[e] = sl >= 0 ? ~sl : c;
  }
}

// The hot set: the columns of degree >= T for the smallest T >= kHotMinDeg
// that keeps at most cap of them; used when they cover >= kHotMinShare of the
// nonzeros.
constexpr unsigned kHotMinDeg = 16;
constexpr double kHotMinShare = 0.10;
nitro_status_t prepare_hot(nitro_spmv *A, int64_t cap) {
  cudaStream_t s = A->stream;
  const int64_t M = A->M, Z = A->Z;
  A->csrv.nhot = 0;
  A->csrv.hot_share = 0.0;
  if (M <= 0 || Z <= 0 || cap <= 0) return NITRO_OK;
  DevBuf deg, aux;
  NITRO_TRY(deg.alloc((size_t)M * 4));
  NITRO_TRY(aux.alloc(34 * 8));
  unsigned long long *bins = aux.as<unsigned long long>(), *covered = bins + 32;
  NITRO_CUDA(cudaMemsetAsync(deg.p, 0, (size_t)M * 4, s));
  NITRO_CUDA(cudaMemsetAsync(aux.p, 0, 34 * 8, s));
  k_col_deg<<<grid_of(Z), 256, 0, s>>>(A->col, Z, deg.as<unsigned>());
  k_deg_hist<<<grid_of(M), 256, 0, s>>>(deg.as<unsigned>(), M, bins);
  unsigned long long hb[32];
  NITRO_CUDA(cudaMemcpyAsync(hb, bins, sizeof(hb), cudaMemcpyDeviceToHost, s));
  NITRO_CUDA(cudaStreamSynchronize(s));
  // the smallest degree threshold T >= kHotMinDeg with #{c : deg(c) >= T} <= cap
  // (bisection over T, one counting pass per step; the log2 histogram bounds it)
  int top = 31;
  while (top > 0 && hb[top] == 0) --top;
  unsigned lo = kHotMinDeg, hi = top >= 31 ? 0xffffffffu : (2u << top);  // count(hi) == 0
  if (hi <= lo) return NITRO_OK;
  DevBuf cntb;
  NITRO_TRY(cntb.alloc(8));
  auto count_ge = [&](unsigned t, int64_t &out) -> nitro_status_t {
    NITRO_CUDA(cudaMemsetAsync(cntb.p, 0, 8, s));
    k_deg_count<<<grid_of(M), 256, 0, s>>>(deg.as<unsigned>(), M, t, cntb.as<unsigned long long>());
    unsigned long long h = 0;
    NITRO_CUDA(cudaMemcpyAsync(&h, cntb.p, 8, cudaMemcpyDeviceToHost, s));
    NITRO_CUDA(cudaStreamSynchronize(s));
    out = (int64_t)h;
    return NITRO_OK;
  };
  int64_t c_lo = 0;
  NITRO_TRY(count_ge(lo, c_lo));
  unsigned thr = lo;
  if (c_lo > cap) {  // bisection: count(lo) > cap >= count(hi)
    while (hi - lo > 1) {
      const unsigned mid = lo + (hi - lo) / 2;
      int64_t cm = 0;
      NITRO_TRY(count_ge(mid, cm));
      if (cm > cap) lo = mid; else hi = mid;
    }
    thr = hi;
  }
  DevBuf fl;
  NITRO_TRY(fl.alloc((size_t)(2 * M + 2) * 8));
  int64_t *f = fl.as<int64_t>(), *pos = f + M + 1;
  k_hot_flags<<<grid_of(M), 256, 0, s>>>(deg.as<unsigned>(), M, thr, f, covered);
  NITRO_TRY(exclusive_scan_i64(f, pos, M, A->scratch, s));
  int64_t nh = 0;
  unsigned long long cov = 0;
  NITRO_CUDA(cudaMemcpyAsync(&nh, pos + M, 8, cudaMemcpyDeviceToHost, s));
  NITRO_CUDA(cudaMemcpyAsync(&cov, covered, 8, cudaMemcpyDeviceToHost, s));
  NITRO_CUDA(cudaStreamSynchronize(s));
  const double share = (double)cov / (double)Z;
  if (nh == 0 || nh > cap || share < kHotMinShare) return NITRO_OK;
  // every persistent CTA loads the nh hot values once: worth it only when the
  // gathers it saves are several times that (small power-law matrices lost to
  // it: a 2^16-row one saves ~0.3 M gathers against ~2.4 M staged loads)
  if ((double)cov < 4.0 * 2.0 * (double)num_sms() * (double)nh && !csrv_hot_forced()) return NITRO_OK;
  NITRO_TRY(A->csrv.hot_cols.alloc((size_t)nh * 4));
  NITRO_TRY(A->csrv.hcol.alloc((size_t)Z * 4));
  DevBuf slot;
  NITRO_TRY(slot.alloc((size_t)M * 4));
  k_hot_emit<<<grid_of(M), 256, 0, s>>>(f, pos, M, A->csrv.hot_cols.as<int32_t>(), slot.as<int32_t>());
  k_hot_remap<<<grid_of(Z), 256, 0, s>>>(A->col, Z, slot.as<int32_t>(), A->csrv.hcol.as<int32_t>());
  NITRO_CUDA(cudaGetLastError());
  NITRO_CUDA(cudaStreamSynchronize(s));  // deg / fl / slot are freed on return
  A->csrv.nhot = nh;
  A->csrv.hot_share = share;
  return NITRO_OK;
}

// ------------------------------------------------------------------ CSR-vector (C8)
// V = lanes per row from the mean row length; rows longer than 8V are split
// into segments of kCsrvSeg entries, each reduced by one warp (see spmv.cu).
nitro_status_t prepare_csrv(nitro_spmv *A) {
  if (A->csrv.ready) return NITRO_OK;
  NITRO_TRY(features_finish(A));
  cudaStream_t s = A->stream;
  const int64_t N = A->N;
  const int64_t q = N > 0 ? A->Z / N : 0;
  // ~2-4 entries per lane (B200 sweep: V = mean/4 beat CUSP's V = mean by
  // 1.3-1.6x on stencils and sparse bands — more loads in flight per lane);
  // NITRO_CSRV_RULE=cusp restores V = 2/4/8/16/32 for q <= 2/4/8/16/else
  static const bool cusp = [] {
    const char *e = getenv("NITRO_CSRV_RULE");
    return e && std::string(e) == "cusp";
  }();
  int V = cusp ? (q <= 2 ? 2 : q <= 4 ? 4 : q <= 8 ? 8 : q <= 16 ? 16 : 32)
               : (q <= 8 ? 2 : q <= 16 ? 4 : q <= 32 ? 8 : q <= 64 ? 16 : 32);
  // tuning hook: NITRO_CSRV_SHIFT=k divides V by 2^k (more entries per lane)
  static int shift = [] {
    const char *e = getenv("NITRO_CSRV_SHIFT");
    return e ? atoi(e) : 0;
  }();
  for (int k = 0; k < shift && V > 2; ++k) V >>= 1;
  A->csrv.V = V;
  A->csrv.stream = csrv_stream_mode(A);
  if (A->csrv.stream && A->Z > 0) {
    // entries per lane: B200 A/B on c2b (fp64) EP 4 vs 8: 0.716 vs 0.753 ms; on
    // fp32 (c2a) 8 beats 4: 1.297 vs 1.462 ms
    const int EP = A->fp64 ? 4 : 8;
    const int64_t CH = 32LL * EP, nch = (A->Z + CH - 1) / CH, nslot = 2 * nch;
    A->csrv.EP = EP;
    A->csrv.nch = nch;
    NITRO_TRY(A->csrv.chunk_row.alloc((size_t)(nch + 1) * 4));
    NITRO_TRY(A->csrv.carry_row.alloc((size_t)nslot * 4));
    NITRO_TRY(A->csrv.carry_val.alloc((size_t)nslot * 8));
    DevBuf fx;
    NITRO_TRY(fx.alloc((size_t)nslot * 4 + (size_t)(2 * nslot + 2) * 8 + 8));
    int32_t *eff = fx.as<int32_t>();
    int64_t *hd = reinterpret_cast<int64_t *>(fx.as<char>() + round_up(nslot * 4, 8)), *pos = hd + nslot + 1;
    if (A->rp64) k_stream_rows<int64_t><<<grid_of(nch + 1), 256, 0, s>>>((const int64_t *)A->rowptr, N, A->Z, CH, nch, A->csrv.chunk_row.as<int32_t>(), eff);
    else k_stream_rows<int32_t><<<grid_of(nch + 1), 256, 0, s>>>((const int32_t *)A->rowptr, N, A->Z, CH, nch, A->csrv.chunk_row.as<int32_t>(), eff);
    k_fix_heads<<<grid_of(nslot), 256, 0, s>>>(eff, nslot, hd);
    NITRO_TRY(exclusive_scan_i64(hd, pos, nslot, A->scratch, s));
    int64_t S = 0;
    NITRO_CUDA(cudaMemcpyAsync(&S, pos + nslot, 8, cudaMemcpyDeviceToHost, s));
    NITRO_CUDA(cudaStreamSynchronize(s));
    NITRO_TRY(A->csrv.fix_seg.alloc((size_t)(S + 1) * 4));
    NITRO_TRY(A->csrv.fix_long.alloc((size_t)std::max<int64_t>(S, 1) * 4));
    k_fix_emit<<<grid_of(nslot), 256, 0, s>>>(eff, pos, nslot, A->csrv.fix_seg.as<int32_t>());
    DevBuf lc;
    NITRO_TRY(lc.alloc(8));
    NITRO_CUDA(cudaMemsetAsync(lc.p, 0, 8, s));
    k_fix_long<<<grid_of(S), 256, 0, s>>>(A->csrv.fix_seg.as<int32_t>(), S, A->csrv.fix_long.as<int32_t>(),
                                          lc.as<unsigned long long>());
    NITRO_CUDA(cudaGetLastError());
    unsigned long long nl = 0;
    NITRO_CUDA(cudaMemcpyAsync(&nl, lc.p, 8, cudaMemcpyDeviceToHost, s));
    NITRO_CUDA(cudaStreamSynchronize(s));
    A->csrv.fix_S = S;
    A->csrv.fix_nlong = (int64_t)nl;
    A->csrv.n_long = 0;
    // hot-x staging: up to 48 KB of x values per CTA (6144 fp64, csrv_hot_kb);
    // measured on fp64 only (configs[2] R-MAT) — the fp32 form (one 768-thread
    // CTA per SM, 56 registers) is not used
    if (csrv_hot_on() && A->fp64) NITRO_TRY(prepare_hot(A, (int64_t)csrv_hot_kb() * 1024 / 8));
    else A->csrv.nhot = 0;
    A->csrv.ready = true;
    return NITRO_OK;
  }
  const int64_t T = 8LL * V, S = kCsrvSeg;
  A->csrv.n_long = 0;
  if (A->feat.max_row > T) {
    DevBuf cnt;
    NITRO_TRY(cnt.alloc((size_t)(2 * N + 2) * 8));
    int64_t *c = cnt.as<int64_t>(), *off = c + N + 1;
    if (A->rp64) k_long_flags<int64_t><<<grid_of(N), 256, 0, s>>>((const int64_t *)A->rowptr, N, T, S, c);
    else k_long_flags<int32_t><<<grid_of(N), 256, 0, s>>>((const int32_t *)A->rowptr, N, T, S, c);
    NITRO_TRY(exclusive_scan_i64(c, off, N, A->scratch, s));
    int64_t nseg = 0;
    NITRO_CUDA(cudaMemcpyAsync(&nseg, off + N, 8, cudaMemcpyDeviceToHost, s));
    NITRO_CUDA(cudaStreamSynchronize(s));
    // layout: seg_row[nseg] | seg_k[nseg] | seg partials (double)[nseg] | row counters (uint)[nseg]
    NITRO_TRY(A->csrv.long_rows.alloc((size_t)std::max<int64_t>(nseg, 1) * (4 + 4 + 8 + 4) + 16));
    int32_t *seg_row = A->csrv.long_rows.as<int32_t>();
    int32_t *seg_k = seg_row + nseg;
    if (A->rp64) k_long_emit<int64_t><<<grid_of(N), 256, 0, s>>>((const int64_t *)A->rowptr, N, off, seg_row, seg_k);
    else k_long_emit<int32_t><<<grid_of(N), 256, 0, s>>>((const int32_t *)A->rowptr, N, off, seg_row, seg_k);
    NITRO_CUDA(cudaGetLastError());
    // zero the per-row completion counters (indexed by a row's first segment)
    char *base = (char *)A->csrv.long_rows.p;
    size_t ctr_off = (size_t)nseg * 16;
    NITRO_CUDA(cudaMemsetAsync(base + ctr_off, 0, (size_t)std::max<int64_t>(nseg, 1) * 4, s));
    NITRO_CUDA(cudaStreamSynchronize(s));
    A->csrv.n_long = nseg;
  }
  A->csrv.ready = true;
  return NITRO_OK;
}

}  // namespace nitro
