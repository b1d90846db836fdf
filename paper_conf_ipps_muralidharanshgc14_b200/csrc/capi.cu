// capi.cu — the SpMV layer of the C ABI (include/nitro.h §2) + shared plumbing.
#include "nitro_internal.h"

#include <algorithm>
#include <cmath>
#include <cstring>
#include <new>
#include <vector>

namespace nitro {

static thread_local std::string g_err;

void set_error(const std::string &msg) { g_err = msg; }
nitro_status_t fail(nitro_status_t code, const std::string &msg) {
  g_err = msg;
  return code;
}
nitro_status_t cuda_fail(cudaError_t e, const char *where) {
  g_err = std::string("CUDA error ") + cudaGetErrorName(e) + " (" + cudaGetErrorString(e) + ") at " + where;
  return e == cudaErrorMemoryAllocation ? NITRO_E_OOM : NITRO_E_CUDA;
}

nitro_status_t DevBuf::alloc(size_t n) {
  if (n <= bytes && p) return NITRO_OK;
  release();
  if (n == 0) n = 16;
  cudaError_t e = cudaMalloc(&p, n);
  if (e != cudaSuccess) {
    p = nullptr;
    bytes = 0;
    (void)cudaGetLastError();
    return cuda_fail(e, "cudaMalloc");
  }
  bytes = n;
  return NITRO_OK;
}
void DevBuf::release() {
  if (p) cudaFree(p);
  p = nullptr;
  bytes = 0;
}

int num_sms() {
  static int cached[64] = {0};
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 0 || dev >= 64) dev = 0;
  if (!cached[dev]) {
    int n = 0;
    if (cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || n <= 0) n = 148;
    cached[dev] = n;
  }
  return cached[dev];
}

namespace {

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur = -1;
    if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
  }
};

bool valid_variant(int v) { return v >= 0 && v < NITRO_NUM_VARIANTS; }

nitro_status_t ensure_budget(nitro_spmv *A) {
  if (A->budget >= 0) return NITRO_OK;
  size_t fr = 0, tot = 0;
  NITRO_CUDA(cudaMemGetInfo(&fr, &tot));
  A->budget = 0.4 * (double)fr;
  return NITRO_OK;
}

// C9 constraints (R9)
nitro_status_t allowed_impl(nitro_spmv *A, int v, int *out) {
  NITRO_TRY(features_finish(A));
  NITRO_TRY(ensure_budget(A));
  const double ld = (double)round_up(A->N, 32), sv = A->fp64 ? 8 : 4;
  const nitro_spmv_feat &f = A->feat;
  switch (v) {
    case NITRO_DIA: *out = f.dia_fill <= 3.0 && (double)f.ndiag * ld * sv <= A->budget; break;
    case NITRO_ELL: *out = f.ell_fill <= 3.0 && (double)f.max_row * ld * (sv + 4) <= A->budget; break;
    default: *out = 1;
  }
  return NITRO_OK;
}

nitro_status_t prepare_impl(nitro_spmv *A, int v) {
  int ok = 0;
  NITRO_TRY(allowed_impl(A, v, &ok));
  if (!ok) return fail(NITRO_E_CONSTRAINT, "variant ruled out by its constraint for this matrix");
  switch (v) {
    case NITRO_CSR_SCALAR: return NITRO_OK;
    case NITRO_CSR_VECTOR: return prepare_csrv(A);
    case NITRO_ELL: return prepare_ell(A);
    case NITRO_DIA: return prepare_dia(A);
    case NITRO_HYB: return prepare_hyb(A);
  }
  return fail(NITRO_E_INVALID_ARG, "bad variant");
}

bool is_ready(const nitro_spmv *A, int v) {
  switch (v) {
    case NITRO_CSR_SCALAR: return A->feat_ready && A->feat.canonical;
    case NITRO_CSR_VECTOR: return A->csrv.ready;
    case NITRO_ELL: return A->ell.ready;
    case NITRO_DIA: return A->dia.ready;
    case NITRO_HYB: return A->hyb.ready;
  }
  return false;
}

}  // namespace
}  // namespace nitro

using namespace nitro;

#define NITRO_GUARD_BEGIN try {
#define NITRO_GUARD_END                                              \
  }                                                                  \
  catch (const std::bad_alloc &) {                                   \
    return fail(NITRO_E_OOM, "host allocation failed");             \
  }                                                                  \
  catch (...) {                                                      \
    return fail(NITRO_E_INVALID_ARG, "unexpected exception");       \
  }

extern "C" {

const char *nitro_last_error(void) { return g_err.c_str(); }
const char *nitro_version(void) { return "nitro-b200 0.1 (sm_100a)"; }

nitro_status_t nitro_spmv_create(int device, void *stream, int64_t rows, int64_t cols, int64_t nnz,
                                 const void *d_rowptr, int rowptr_is_64, const int32_t *d_colidx, const void *d_vals,
                                 int is_fp64, nitro_spmv **out) {
  NITRO_GUARD_BEGIN
  if (!out) return fail(NITRO_E_INVALID_ARG, "out is NULL");
  *out = nullptr;
  if (rows < 0 || cols < 0 || nnz < 0) return fail(NITRO_E_INVALID_ARG, "negative size");
  if (!d_rowptr) return fail(NITRO_E_INVALID_ARG, "rowptr is NULL");
  if (nnz > 0 && (!d_colidx || !d_vals)) return fail(NITRO_E_INVALID_ARG, "colidx/vals NULL with nnz > 0");
  if (cols > 2147483647LL || rows > 2147483647LL) return fail(NITRO_E_UNSUPPORTED, "rows/cols must be < 2^31");
  if (!rowptr_is_64 && nnz > 2147483647LL) return fail(NITRO_E_INVALID_ARG, "nnz >= 2^31 needs a 64-bit rowptr");
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev)
    return fail(NITRO_E_CUDA, "no such CUDA device");
  nitro_spmv *A = new nitro_spmv();
  A->device = device;
  A->stream = (cudaStream_t)stream;
  A->N = rows; A->M = cols; A->Z = nnz;
  A->rowptr = d_rowptr; A->rp64 = rowptr_is_64 != 0;
  A->col = d_colidx; A->val = d_vals; A->fp64 = is_fp64 != 0;
  *out = A;
  return NITRO_OK;
  NITRO_GUARD_END
}

nitro_status_t nitro_spmv_set_stream(nitro_spmv *A, void *stream) {
  if (!A) return fail(NITRO_E_INVALID_ARG, "NULL handle");
  A->stream = (cudaStream_t)stream;
  return NITRO_OK;
}

nitro_status_t nitro_spmv_features(nitro_spmv *A, nitro_spmv_feat *out) {
  NITRO_NVTX("nitro_spmv_features");
  NITRO_GUARD_BEGIN
  if (!A || !out) return fail(NITRO_E_INVALID_ARG, "NULL argument");
  DeviceGuard g(A->device);
  nitro_status_t st = features_finish(A);
  if (A->feat_ready) *out = A->feat;
  return st;
  NITRO_GUARD_END
}

nitro_status_t nitro_spmv_row_features(nitro_spmv *A, nitro_spmv_feat *out) {
  NITRO_GUARD_BEGIN
  if (!A || !out) return fail(NITRO_E_INVALID_ARG, "NULL argument");
  DeviceGuard g(A->device);
  return row_features(A, out);
  NITRO_GUARD_END
}

nitro_status_t nitro_spmv_features_async(nitro_spmv *A) {
  NITRO_NVTX("nitro_spmv_features_async");
  NITRO_GUARD_BEGIN
  if (!A) return fail(NITRO_E_INVALID_ARG, "NULL handle");
  DeviceGuard g(A->device);
  return features_launch(A);
  NITRO_GUARD_END
}

nitro_status_t nitro_spmv_allowed(nitro_spmv *A, int variant, int *out_allowed) {
  NITRO_GUARD_BEGIN
  if (!A || !out_allowed || !valid_variant(variant)) return fail(NITRO_E_INVALID_ARG, "bad argument");
  DeviceGuard g(A->device);
  return allowed_impl(A, variant, out_allowed);
  NITRO_GUARD_END
}

nitro_status_t nitro_spmv_set_budget(nitro_spmv *A, double bytes) {
  if (!A || !(bytes >= 0)) return fail(NITRO_E_INVALID_ARG, "bad argument");
  A->budget = bytes;
  return NITRO_OK;
}

nitro_status_t nitro_spmv_set_csr_impl(nitro_spmv *A, int impl) {
  if (!A || impl < NITRO_CSR_IMPL_AUTO || impl > NITRO_CSR_IMPL_VEC4) return fail(NITRO_E_INVALID_ARG, "bad argument");
  A->csr_impl = impl;
  // the CSR-vector format depends on the mode (stream chunks vs long-row segments)
  if (A->csrv.ready && A->csrv.stream != csrv_stream_mode(A)) A->csrv.ready = false;
  return NITRO_OK;
}

nitro_status_t nitro_spmv_prepare(nitro_spmv *A, int variant) {
  NITRO_NVTX("nitro_spmv_prepare");
  NITRO_GUARD_BEGIN
  if (!A || !valid_variant(variant)) return fail(NITRO_E_INVALID_ARG, "bad argument");
  DeviceGuard g(A->device);
  if (is_ready(A, variant)) return NITRO_OK;
  return prepare_impl(A, variant);
  NITRO_GUARD_END
}

nitro_status_t nitro_spmv_format_info(nitro_spmv *A, int variant, nitro_format_info *out) {
  NITRO_GUARD_BEGIN
  if (!A || !out || !valid_variant(variant)) return fail(NITRO_E_INVALID_ARG, "bad argument");
  DeviceGuard g(A->device);
  if (!is_ready(A, variant)) NITRO_TRY(prepare_impl(A, variant));
  memset(out, 0, sizeof(*out));
  switch (variant) {
    case NITRO_CSR_SCALAR: out->width = 1; break;
    case NITRO_CSR_VECTOR:
      out->width = A->csrv.stream ? 0 : A->csrv.V;  // 0: nnz-split stream mode (K6s)
      out->tail = A->csrv.stream ? A->csrv.nch : A->csrv.n_long;
      out->bytes = (int64_t)(A->csrv.long_rows.bytes + A->csrv.chunk_row.bytes + A->csrv.carry_row.bytes +
                             A->csrv.carry_val.bytes + A->csrv.fix_seg.bytes + A->csrv.fix_long.bytes +
                             A->csrv.hot_cols.bytes + A->csrv.hcol.bytes);
      // stream mode: hot x values staged in shared memory (0 = none); row
      // mode: 1 when the vector-load kernel K6v runs, else 0
      out->ld = A->csrv.stream ? A->csrv.nhot : (csrv_vec_mode(A) ? 1 : 0);
      break;
    case NITRO_ELL: out->ld = A->ell.ld; out->width = A->ell.K; out->bytes = (int64_t)(A->ell.col.bytes + A->ell.val.bytes); break;
    case NITRO_DIA: out->ld = A->dia.ld; out->width = A->dia.D; out->bytes = (int64_t)(A->dia.off.bytes + A->dia.val.bytes); break;
    case NITRO_HYB:
      out->ld = A->hyb.ld; out->width = A->hyb.K; out->tail = A->hyb.Zt;
      out->bytes = (int64_t)(A->hyb.col.bytes + A->hyb.val.bytes + A->hyb.trow.bytes + A->hyb.tcol.bytes +
                             A->hyb.tval.bytes + A->hyb.carry_row.bytes + A->hyb.carry_val.bytes);
      break;
  }
  out->compulsory_bytes = compulsory_bytes(A, variant);
  return NITRO_OK;
  NITRO_GUARD_END
}

nitro_status_t nitro_spmv_run(nitro_spmv *A, int variant, const void *d_x, void *d_y) {
  NITRO_NVTX("nitro_spmv_run");
  NITRO_GUARD_BEGIN
  if (!A || !valid_variant(variant)) return fail(NITRO_E_INVALID_ARG, "bad argument");
  if ((A->M > 0 && !d_x) || (A->N > 0 && !d_y)) return fail(NITRO_E_INVALID_ARG, "x or y is NULL");
  DeviceGuard g(A->device);
  if (!is_ready(A, variant)) NITRO_TRY(prepare_impl(A, variant));
  return launch_spmv(A, variant, d_x, d_y, A->stream);
  NITRO_GUARD_END
}

}  // extern "C"

namespace {
// Row chunks of the pipelined host-buffer call: the row-separable variants
// (CSR-scalar, ELL, DIA) of matrices of >= 2^18 rows; NITRO_RUN_HOST_CHUNKS
// overrides the count (1 = no pipeline).
int run_host_chunks(const nitro_spmv *A, int variant) {
  static int env = [] {
    const char *e = getenv("NITRO_RUN_HOST_CHUNKS");
    return e ? atoi(e) : 0;
  }();
  if (variant != NITRO_CSR_SCALAR && variant != NITRO_ELL && variant != NITRO_DIA) return 1;
  // about one chunk per 32 MB of x, 4 to 16: B200, pinned buffers, DIA —
  // configs[1] (x 8 MB, ms per call) 1 chunk 0.372, 2 0.320, 4 0.313, 8 0.340,
  // 16 0.410 (smaller copies lose more to per-copy setup than the finer overlap
  // gains); configs[4] (x 537 MB) 1: 21.5, 4: 15.1, 8: 13.6, 16: 13.3, 32: 13.4
  // (81 GB/s of H2D + D2H, the PCIe limit with both directions busy).  A
  // CUDA-graph capture of the enqueue made no difference (copies, not the host, bound it)
  const double xmb = (double)A->M * (A->fp64 ? 8 : 4) / (32.0 * 1048576.0);
  const int want = env > 0 ? env : (int)std::max(4.0, std::min(16.0, std::ceil(xmb)));
  if (want <= 1 || A->N < (int64_t)want * 32768) return 1;
  return want;
}

// x arrives in column pieces on s_in, chunk c's multiply (rows [r_c, r_c+1))
// starts on the handle's stream as soon as the columns its rows reference are
// in, and its y rows leave on s_out while later chunks compute: the two copy
// directions overlap each other and the kernels.
nitro_status_t run_host_pipelined(nitro_spmv *A, int variant, const void *h_x, void *h_y, int nch) {
  const size_t sv = A->fp64 ? 8 : 4;
  if (!A->s_in) NITRO_CUDA(cudaStreamCreateWithFlags(&A->s_in, cudaStreamNonBlocking));
  if (!A->s_out) NITRO_CUDA(cudaStreamCreateWithFlags(&A->s_out, cudaStreamNonBlocking));
  const size_t nev = (size_t)(2 * nch + 2);
  while (A->ev_pipe.size() < nev) {
    cudaEvent_t e;
    NITRO_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    A->ev_pipe.push_back(e);
  }
  // chunk ends: multiples of 1024 rows
  std::vector<int64_t> ends(nch);
  const int64_t step = round_up((A->N + nch - 1) / nch, 1024);
  for (int c = 0; c < nch; ++c) ends[c] = std::min<int64_t>(A->N, (int64_t)(c + 1) * step);
  ends[nch - 1] = A->N;
  // columns each chunk needs: DIA from its offsets (+8: the aligned x windows
  // may touch a few entries past the last one used), else from the rows
  std::vector<int64_t> xhi(nch);
  if (variant == NITRO_DIA) {
    for (int c = 0; c < nch; ++c)
      xhi[c] = std::min<int64_t>(A->M, std::max<int64_t>(0, A->row0 + ends[c] + A->dia.off_max + 8));
  } else {
    if (!A->xhi_ready || A->csr_xhi.size() != (size_t)nch) {
      NITRO_TRY(csr_chunk_xhi(A, ends, A->csr_xhi));
      A->xhi_ready = true;
    }
    xhi = A->csr_xhi;
  }
  xhi[nch - 1] = A->M;  // everything in by the last chunk
  cudaEvent_t *ev_in = A->ev_pipe.data(), *ev_k = ev_in + nch, ev_start = ev_in[2 * nch], ev_done = ev_in[2 * nch + 1];
  // order after earlier work on the handle's stream
  NITRO_CUDA(cudaEventRecord(ev_start, A->stream));
  NITRO_CUDA(cudaStreamWaitEvent(A->s_in, ev_start, 0));
  NITRO_CUDA(cudaStreamWaitEvent(A->s_out, ev_start, 0));
  int64_t lo = 0;
  for (int c = 0; c < nch; ++c) {
    const int64_t hi = std::max(lo, xhi[c]);
    if (hi > lo)
      NITRO_CUDA(cudaMemcpyAsync(A->xbuf.as<char>() + lo * sv, (const char *)h_x + lo * sv, (size_t)(hi - lo) * sv,
                                 cudaMemcpyHostToDevice, A->s_in));
    NITRO_CUDA(cudaEventRecord(ev_in[c], A->s_in));
    lo = hi;
  }
  int64_t r0 = 0;
  for (int c = 0; c < nch; ++c) {
    NITRO_CUDA(cudaStreamWaitEvent(A->stream, ev_in[c], 0));
    NITRO_TRY(launch_spmv_rows(A, variant, A->xbuf.p, A->ybuf.p, A->stream, r0, ends[c]));
    NITRO_CUDA(cudaEventRecord(ev_k[c], A->stream));
    NITRO_CUDA(cudaStreamWaitEvent(A->s_out, ev_k[c], 0));
    if (ends[c] > r0)
      NITRO_CUDA(cudaMemcpyAsync((char *)h_y + r0 * sv, A->ybuf.as<char>() + r0 * sv, (size_t)(ends[c] - r0) * sv,
                                 cudaMemcpyDeviceToHost, A->s_out));
    r0 = ends[c];
  }
  NITRO_CUDA(cudaEventRecord(ev_done, A->s_out));
  NITRO_CUDA(cudaStreamWaitEvent(A->stream, ev_done, 0));
  NITRO_CUDA(cudaStreamSynchronize(A->stream));
  return NITRO_OK;
}
}  // namespace

extern "C" {

nitro_status_t nitro_spmv_run_host(nitro_spmv *A, int variant, const void *h_x, void *h_y) {
  NITRO_NVTX("nitro_spmv_run_host");
  NITRO_GUARD_BEGIN
  if (!A || !valid_variant(variant)) return fail(NITRO_E_INVALID_ARG, "bad argument");
  if ((A->M > 0 && !h_x) || (A->N > 0 && !h_y)) return fail(NITRO_E_INVALID_ARG, "x or y is NULL");
  DeviceGuard g(A->device);
  if (!is_ready(A, variant)) NITRO_TRY(prepare_impl(A, variant));
  const size_t sv = A->fp64 ? 8 : 4;
  NITRO_TRY(A->xbuf.alloc(std::max<size_t>(A->M * sv, 16)));
  NITRO_TRY(A->ybuf.alloc(std::max<size_t>(A->N * sv, 16)));
  const int nch = run_host_chunks(A, variant);
  if (nch > 1) return run_host_pipelined(A, variant, h_x, h_y, nch);
  if (A->M) NITRO_CUDA(cudaMemcpyAsync(A->xbuf.p, h_x, A->M * sv, cudaMemcpyHostToDevice, A->stream));
  NITRO_TRY(launch_spmv(A, variant, A->xbuf.p, A->ybuf.p, A->stream));
  if (A->N) NITRO_CUDA(cudaMemcpyAsync(h_y, A->ybuf.p, A->N * sv, cudaMemcpyDeviceToHost, A->stream));
  NITRO_CUDA(cudaStreamSynchronize(A->stream));
  return NITRO_OK;
  NITRO_GUARD_END
}

nitro_status_t nitro_spmv_flush_l2(nitro_spmv *A) {
  NITRO_GUARD_BEGIN
  if (!A) return fail(NITRO_E_INVALID_ARG, "NULL handle");
  DeviceGuard g(A->device);
  return launch_flush(A, A->stream);
  NITRO_GUARD_END
}

nitro_status_t nitro_spmv_time(nitro_spmv *A, int variant, const void *d_x, void *d_y, int warmup, int reps,
                               int flush_l2, double *out_median_s, double *out_all) {
  NITRO_NVTX("nitro_spmv_time");
  NITRO_GUARD_BEGIN
  if (!A || !valid_variant(variant) || reps < 1 || warmup < 0 || !out_median_s)
    return fail(NITRO_E_INVALID_ARG, "bad argument");
  return nitro::time_variant(A, variant, d_x, d_y, warmup, reps, flush_l2, INFINITY, out_median_s, out_all, nullptr);
  NITRO_GUARD_END
}

nitro_status_t nitro_spmv_launches(nitro_spmv *A, int variant, int *out) {
  NITRO_GUARD_BEGIN
  if (!A || !out || !valid_variant(variant)) return fail(NITRO_E_INVALID_ARG, "bad argument");
  DeviceGuard g(A->device);
  if (!is_ready(A, variant)) NITRO_TRY(prepare_impl(A, variant));
  *out = launches_of(A, variant);
  return NITRO_OK;
  NITRO_GUARD_END
}

nitro_status_t nitro_spmv_export(nitro_spmv *A, int part, void *host_buf, size_t cap, size_t *needed) {
  NITRO_GUARD_BEGIN
  if (!A || !needed) return fail(NITRO_E_INVALID_ARG, "NULL argument");
  DeviceGuard g(A->device);
  const size_t sv = A->fp64 ? 8 : 4;
  const void *src = nullptr;
  size_t n = 0;
  DevBuf tmp;
  if (part <= 1) {
    NITRO_TRY(nitro_spmv_prepare(A, NITRO_ELL));
    n = (size_t)(A->ell.K * A->ell.ld) * (part == 0 ? 4 : sv);
    src = part == 0 ? A->ell.col.p : A->ell.val.p;
  } else if (part <= 3) {
    NITRO_TRY(nitro_spmv_prepare(A, NITRO_DIA));
    n = part == 2 ? (size_t)A->dia.D * 4 : (size_t)(A->dia.D * A->dia.ld) * sv;
    src = part == 2 ? A->dia.off.p : A->dia.val.p;
  } else if (part <= 8) {
    NITRO_TRY(nitro_spmv_prepare(A, NITRO_HYB));
    const size_t ke = (size_t)(A->hyb.K * A->hyb.ld), zt = (size_t)A->hyb.Zt;
    switch (part) {
      case 4: n = ke * 4; src = A->hyb.col.p; break;
      case 5: n = ke * sv; src = A->hyb.val.p; break;
      case 6: n = zt * 4; src = A->hyb.trow.p; break;
      case 7: n = zt * 4; src = A->hyb.tcol.p; break;
      default: n = zt * sv; src = A->hyb.tval.p; break;
    }
  } else if (part == 9) {
    // ascending diagonal offsets of the feature pass (same emit as DIA prepare)
    NITRO_TRY(features_finish(A));
    if (!A->dia.ready) {
      // emit without building DIA values: reuse prepare_dia only when allowed, else emit directly
      int ok = 0;
      NITRO_TRY(allowed_impl(A, NITRO_DIA, &ok));
      if (ok) NITRO_TRY(prepare_dia(A));
    }
    if (A->dia.ready) {
      n = (size_t)A->dia.D * 4;
      src = A->dia.off.p;
    } else {
      return fail(NITRO_E_CONSTRAINT, "diagonal list is only materialised for DIA-allowed matrices");
    }
  } else {
    return fail(NITRO_E_INVALID_ARG, "bad part");
  }
  *needed = n;
  if (host_buf && cap >= n && n > 0) {
    NITRO_CUDA(cudaMemcpyAsync(host_buf, src, n, cudaMemcpyDeviceToHost, A->stream));
    NITRO_CUDA(cudaStreamSynchronize(A->stream));
  }
  return NITRO_OK;
  NITRO_GUARD_END
}

nitro_status_t nitro_spmv_invalidate(nitro_spmv *A) {
  if (!A) return fail(NITRO_E_INVALID_ARG, "NULL handle");
  DeviceGuard g(A->device);
  NITRO_CUDA(cudaStreamSynchronize(A->stream));
  A->feat_ready = A->feat_pending = false;
  A->ell.ready = A->dia.ready = A->hyb.ready = A->csrv.ready = false;
  A->xhi_ready = false;
  return NITRO_OK;
}

nitro_status_t nitro_spmv_release(nitro_spmv *A, int variant) {
  if (!A) return fail(NITRO_E_INVALID_ARG, "NULL handle");
  DeviceGuard g(A->device);
  cudaStreamSynchronize(A->stream);
  if (variant == -1 || variant == NITRO_ELL) { A->ell.col.release(); A->ell.val.release(); A->ell.ready = false; }
  if (variant == -1 || variant == NITRO_DIA) { A->dia.off.release(); A->dia.val.release(); A->dia.ready = false; }
  if (variant == -1 || variant == NITRO_HYB) {
    A->hyb.col.release(); A->hyb.val.release(); A->hyb.trow.release(); A->hyb.tcol.release();
    A->hyb.tval.release(); A->hyb.carry_row.release(); A->hyb.carry_val.release();
    A->hyb.fix_seg.release(); A->hyb.fix_long.release(); A->hyb.ready = false;
  }
  if (variant == -1 || variant == NITRO_CSR_VECTOR) {
    A->csrv.long_rows.release();
    A->csrv.chunk_row.release(); A->csrv.carry_row.release(); A->csrv.carry_val.release();
    A->csrv.fix_seg.release(); A->csrv.fix_long.release();
    A->csrv.hot_cols.release(); A->csrv.hcol.release(); A->csrv.nhot = 0;
    A->csrv.ready = false;
  }
  return NITRO_OK;
}

void nitro_spmv_destroy(nitro_spmv *A) {
  if (!A) return;
  {
    DeviceGuard g(A->device);
    cudaStreamSynchronize(A->stream);
    nitro_spmv_release(A, -1);
    if (A->h_acc) cudaFreeHost(A->h_acc);
    if (A->feat_done) cudaEventDestroy(A->feat_done);
    for (auto e : A->ev_pipe) cudaEventDestroy(e);
    if (A->s_in) cudaStreamDestroy(A->s_in);
    if (A->s_out) cudaStreamDestroy(A->s_out);
    A->feat_acc.release(); A->bitmap.release(); A->offsets.release(); A->scratch.release();
    A->flush.release(); A->xbuf.release(); A->ybuf.release();
    if (A->dist_free && A->dist_state) A->dist_free(A->dist_state);
  }
  delete A;
}

}  // extern "C"

namespace nitro {
// Median of `reps` CUDA-event timings (L2 flushed before each when flush_l2).
// cutoff_s finite (the training timeout of SURVEY §5): after every rep from
// the third on, stop once the median so far exceeds cutoff_s — a variant 20x
// slower than the input's current best is ranked by the reps it has run.
nitro_status_t time_variant(nitro_spmv *A, int variant, const void *d_x, void *d_y, int warmup, int reps,
                            int flush_l2, double cutoff_s, double *out_median_s, double *out_all, int *out_reps) {
  DeviceGuard g(A->device);
  if (!is_ready(A, variant)) NITRO_TRY(prepare_impl(A, variant));
  cudaStream_t s = A->stream;
  for (int w = 0; w < warmup; ++w) NITRO_TRY(launch_spmv(A, variant, d_x, d_y, s));
  const bool early = std::isfinite(cutoff_s);
  std::vector<cudaEvent_t> ev(2 * reps, nullptr);
  for (auto &e : ev) NITRO_CUDA(cudaEventCreate(&e));
  std::vector<double> t;
  nitro_status_t st = NITRO_OK;
  auto collect = [&](int upto) {  // rep times [t.size(), upto)
    cudaError_t e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) return cuda_fail(e, "cudaStreamSynchronize");
    for (int r = (int)t.size(); r < upto; ++r) {
      float ms = 0.f;
      cudaEventElapsedTime(&ms, ev[2 * r], ev[2 * r + 1]);
      t.push_back(ms * 1e-3);
    }
    return (nitro_status_t)NITRO_OK;
  };
  auto median = [](std::vector<double> v) {
    std::sort(v.begin(), v.end());
    const size_t n = v.size();
    return n % 2 ? v[n / 2] : 0.5 * (v[n / 2 - 1] + v[n / 2]);
  };
  int done = 0;
  for (int r = 0; r < reps && st == NITRO_OK; ++r) {
    if (flush_l2) st = launch_flush(A, s);
    if (st == NITRO_OK) {
      cudaEventRecord(ev[2 * r], s);
      st = launch_spmv(A, variant, d_x, d_y, s);
      cudaEventRecord(ev[2 * r + 1], s);
    }
    done = r + 1;
    if (st == NITRO_OK && early && done >= 3 && done < reps) {
      st = collect(done);
      if (st == NITRO_OK && median(t) > cutoff_s) break;
    }
  }
  if (st == NITRO_OK) st = collect(done);
  for (auto &x : ev) cudaEventDestroy(x);
  if (st != NITRO_OK) return st;
  if (out_all) {
    std::copy(t.begin(), t.end(), out_all);
    std::fill(out_all + t.size(), out_all + reps, std::numeric_limits<double>::quiet_NaN());
  }
  *out_median_s = median(t);
  if (out_reps) *out_reps = (int)t.size();
  return NITRO_OK;
}
}  // namespace nitro
