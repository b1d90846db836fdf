// dist.cu — A13: multi-GPU row-partitioned SpMV (include/nitro.h §3).
//
// One process per GPU.  Rank r owns the contiguous, nnz-balanced row block
// [bounds[r], bounds[r+1]) (R14) and the matching block of x.
// Every multiply all-gathers x with NCCL (in place, into a padded layout where
// block r starts at r*B, B = max block rows); columns are remapped once to that
// layout.  Local rows are split into head [0,i0) / interior [i0,i1) / tail
// [i1,n): interior rows only touch locally owned columns, so they run on the
// compute stream while the all-gather is in flight on the comm stream; head
// and tail rows run after it.  Each part is an ordinary nitro_spmv over a
// rebased CSR slice, so every variant (and its constraint) works unchanged.
// Global features: per-rank K1 over a global-offset bitmap, integer moments
// all-reduced (sum / max), occupied diagonals unioned (max over u8 flags).
#include <nccl.h>

#include <algorithm>
#include <vector>

#include "nitro_internal.h"

struct nitro_dist {
  ncclComm_t comm = nullptr;
  int rank = 0, nranks = 1, device = 0;
  cudaStream_t comm_stream = nullptr;
  cudaEvent_t ev_x = nullptr, ev_g = nullptr;
};

namespace nitro {
namespace {

#define NITRO_NCCL(call)                                                                    \
  do {                                                                                      \
    ncclResult_t r_ = (call);                                                               \
    if (r_ != ncclSuccess) return fail(NITRO_E_NCCL, std::string("NCCL: ") + ncclGetErrorString(r_) + " at " #call); \
  } while (0)

struct DistState {
  nitro_dist *D = nullptr;
  int64_t global_rows = 0, B = 0, n = 0, row_begin = 0, i0 = 0, i1 = 0;
  std::vector<int64_t> bounds;
  DevBuf colmap, rp_part[3], xfull, flags;
  nitro_spmv *part[3] = {nullptr, nullptr, nullptr};
  nitro_spmv *feat = nullptr;  // original global columns, for global features
  int64_t part_begin[3] = {0, 0, 0};
};

void free_state(void *p) {
  DistState *st = (DistState *)p;
  if (!st) return;
  for (auto *h : st->part) if (h) nitro_spmv_destroy(h);
  if (st->feat) nitro_spmv_destroy(st->feat);
  delete st;
}

__global__ void k_remap(const int32_t *__restrict__ col, int64_t Z, const int64_t *__restrict__ bounds, int P,
                        int64_t B, int32_t *__restrict__ out) {
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < Z; k += (int64_t)gridDim.x * blockDim.x) {
    const int64_t c = col[k];
    int lo = 0, hi = P - 1;  // owner = last r with bounds[r] <= c
    while (lo < hi) {
      int mid = (lo + hi + 1) >> 1;
      if (bounds[mid] <= c) lo = mid; else hi = mid - 1;
    }
    out[k] = (int32_t)((int64_t)lo * B + (c - bounds[lo]));
  }
}

template <typename IT>
__global__ void k_interior(const IT *__restrict__ rowptr, const int32_t *__restrict__ col, int64_t n, int64_t lo,
                           int64_t hi, uint8_t *__restrict__ flag) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    uint8_t f = 1;
    for (int64_t k = (int64_t)rowptr[i]; k < (int64_t)rowptr[i + 1]; ++k)
      if (col[k] < lo || col[k] >= hi) { f = 0; break; }
    flag[i] = f;
  }
}

template <typename IT>
__global__ void k_rebase(const IT *__restrict__ rowptr, int64_t s, int64_t cnt, int32_t *__restrict__ out) {
  const int64_t base = (int64_t)rowptr[s];
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i <= cnt; i += (int64_t)gridDim.x * blockDim.x)
    out[i] = (int32_t)((int64_t)rowptr[s + i] - base);
}

__global__ void k_bits_to_flags(const uint32_t *__restrict__ bm, int64_t nbits, uint8_t *__restrict__ f) {
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < nbits; t += (int64_t)gridDim.x * blockDim.x)
    f[t] = (bm[t >> 5] >> (t & 31)) & 1u;
}
__global__ void k_count_flags(const uint8_t *__restrict__ f, int64_t n, unsigned long long *out) {
  unsigned long long s = 0;
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < n; t += (int64_t)gridDim.x * blockDim.x)
    s += f[t] != 0;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  if ((threadIdx.x & 31) == 0 && s) atomicAdd(out, s);
}
__global__ void k_pack_acc(const FeatAcc *a, unsigned long long *sum2, unsigned long long *max2) {
  sum2[0] = a->s1; sum2[1] = a->s2; max2[0] = a->lmax; max2[1] = a->bad;
}

unsigned grid_n(int64_t n) {
  int64_t g = (n + 255) / 256, cap = (int64_t)num_sms() * 16;
  return (unsigned)std::max<int64_t>(1, std::min(g, cap));
}

}  // namespace
}  // namespace nitro

using namespace nitro;

extern "C" {

nitro_status_t nitro_dist_unique_id(void *out128) {
  if (!out128) return fail(NITRO_E_INVALID_ARG, "NULL out");
  ncclUniqueId id;
  NITRO_NCCL(ncclGetUniqueId(&id));
  static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId size");
  memcpy(out128, &id, 128);
  return NITRO_OK;
}

nitro_status_t nitro_dist_init(const void *id128, int rank, int nranks, int device, nitro_dist **out) {
  if (!id128 || !out || nranks < 1 || rank < 0 || rank >= nranks) return fail(NITRO_E_INVALID_ARG, "bad argument");
  NITRO_CUDA(cudaSetDevice(device));
  nitro_dist *D = new nitro_dist();
  D->rank = rank; D->nranks = nranks; D->device = device;
  ncclUniqueId id;
  memcpy(&id, id128, 128);
  ncclResult_t r = ncclCommInitRank(&D->comm, nranks, id, rank);
  if (r != ncclSuccess) {
    delete D;
    return fail(NITRO_E_NCCL, std::string("ncclCommInitRank: ") + ncclGetErrorString(r));
  }
  NITRO_CUDA(cudaStreamCreateWithFlags(&D->comm_stream, cudaStreamNonBlocking));
  NITRO_CUDA(cudaEventCreateWithFlags(&D->ev_x, cudaEventDisableTiming));
  NITRO_CUDA(cudaEventCreateWithFlags(&D->ev_g, cudaEventDisableTiming));
  *out = D;
  return NITRO_OK;
}

void nitro_dist_destroy(nitro_dist *D) {
  if (!D) return;
  cudaSetDevice(D->device);
  if (D->comm) ncclCommDestroy(D->comm);
  if (D->comm_stream) cudaStreamDestroy(D->comm_stream);
  if (D->ev_x) cudaEventDestroy(D->ev_x);
  if (D->ev_g) cudaEventDestroy(D->ev_g);
  delete D;
}

nitro_status_t nitro_dist_partition(int64_t rows, const int64_t *h_rowptr, int nranks, int64_t *bounds) {
  if (rows < 0 || !h_rowptr || nranks < 1 || !bounds) return fail(NITRO_E_INVALID_ARG, "bad argument");
  const int64_t Z = h_rowptr[rows];
  bounds[0] = 0;
  for (int r = 1; r < nranks; ++r) {
    const __int128 t = ((__int128)r * Z + nranks - 1) / nranks;  // ceil(r Z / P)
    const int64_t target = (int64_t)t;
    int64_t lo = 0, hi = rows;  // first i with rowptr[i] >= target
    while (lo < hi) {
      int64_t mid = (lo + hi) / 2;
      if (h_rowptr[mid] < target) lo = mid + 1; else hi = mid;
    }
    bounds[r] = std::max(lo, bounds[r - 1]);
  }
  bounds[nranks] = rows;
  return NITRO_OK;
}

nitro_status_t nitro_dist_spmv_create(nitro_dist *D, int64_t global_rows, const int64_t *bounds, int64_t local_nnz,
                                      const void *d_rowptr, int rowptr_is_64, const int32_t *d_colidx,
                                      const void *d_vals, int is_fp64, nitro_spmv **out_local) {
  try {
    if (!D || !bounds || !d_rowptr || !out_local || local_nnz < 0) return fail(NITRO_E_INVALID_ARG, "bad argument");
    *out_local = nullptr;
    const int P = D->nranks, r = D->rank;
    for (int q = 0; q < P; ++q)
      if (bounds[q + 1] < bounds[q]) return fail(NITRO_E_INVALID_ARG, "bounds not monotone");
    if (bounds[0] != 0 || bounds[P] != global_rows) return fail(NITRO_E_INVALID_ARG, "bounds must span [0, rows]");
    NITRO_CUDA(cudaSetDevice(D->device));
    DistState *st = new DistState();
    st->D = D;
    st->global_rows = global_rows;
    st->bounds.assign(bounds, bounds + P + 1);
    st->row_begin = bounds[r];
    st->n = bounds[r + 1] - bounds[r];
    for (int q = 0; q < P; ++q) st->B = std::max(st->B, bounds[q + 1] - bounds[q]);
    if ((int64_t)P * st->B > 2147483647LL) { free_state(st); return fail(NITRO_E_UNSUPPORTED, "P*B must be < 2^31"); }
    const size_t sv = is_fp64 ? 8 : 4;
    cudaStream_t s = nullptr;
    auto bail = [&](nitro_status_t code) { free_state(st); return code; };
    // features handle over the original columns (global rows start at row_begin)
    nitro_status_t rc = nitro_spmv_create(D->device, nullptr, st->n, global_rows, local_nnz, d_rowptr, rowptr_is_64,
                                          d_colidx, d_vals, is_fp64, &st->feat);
    if (rc) return bail(rc);
    st->feat->row0 = st->row_begin;
    st->feat->feat_G = global_rows - 1;
    // remapped columns
    if ((rc = st->colmap.alloc(std::max<int64_t>(local_nnz, 1) * 4))) return bail(rc);
    DevBuf dbounds;
    if ((rc = dbounds.alloc((P + 1) * 8))) return bail(rc);
    NITRO_CUDA(cudaMemcpy(dbounds.p, bounds, (P + 1) * 8, cudaMemcpyHostToDevice));
    if (local_nnz > 0)
      k_remap<<<grid_n(local_nnz), 256, 0, s>>>(d_colidx, local_nnz, dbounds.as<int64_t>(), P, st->B,
                                                 st->colmap.as<int32_t>());
    // interior rows (all columns inside this rank's block) -> contiguous run [i0, i1)
    std::vector<uint8_t> hf(st->n);
    if (st->n > 0) {
      if ((rc = st->flags.alloc(st->n))) return bail(rc);
      if (rowptr_is_64)
        k_interior<int64_t><<<grid_n(st->n), 256, 0, s>>>((const int64_t *)d_rowptr, d_colidx, st->n, bounds[r],
                                                          bounds[r + 1], st->flags.as<uint8_t>());
      else
        k_interior<int32_t><<<grid_n(st->n), 256, 0, s>>>((const int32_t *)d_rowptr, d_colidx, st->n, bounds[r],
                                                          bounds[r + 1], st->flags.as<uint8_t>());
      NITRO_CUDA(cudaGetLastError());
      NITRO_CUDA(cudaMemcpy(hf.data(), st->flags.p, st->n, cudaMemcpyDeviceToHost));
    }
    int64_t i0 = 0;
    while (i0 < st->n && !hf[i0]) ++i0;
    int64_t i1 = i0;
    while (i1 < st->n && hf[i1]) ++i1;
    st->i0 = i0;
    st->i1 = i1;
    // three part handles over rebased CSR slices with remapped columns
    const int64_t beg[3] = {0, i0, i1}, end[3] = {i0, i1, st->n};
    std::vector<int64_t> hrp(4, 0);
    for (int k = 0; k < 3; ++k) {
      const int64_t cnt = end[k] - beg[k];
      st->part_begin[k] = beg[k];
      if (cnt <= 0) continue;
      int64_t ab[2];
      if (rowptr_is_64) {
        NITRO_CUDA(cudaMemcpy(&ab[0], (const int64_t *)d_rowptr + beg[k], 8, cudaMemcpyDeviceToHost));
        NITRO_CUDA(cudaMemcpy(&ab[1], (const int64_t *)d_rowptr + end[k], 8, cudaMemcpyDeviceToHost));
      } else {
        int32_t t[2];
        NITRO_CUDA(cudaMemcpy(&t[0], (const int32_t *)d_rowptr + beg[k], 4, cudaMemcpyDeviceToHost));
        NITRO_CUDA(cudaMemcpy(&t[1], (const int32_t *)d_rowptr + end[k], 4, cudaMemcpyDeviceToHost));
        ab[0] = t[0]; ab[1] = t[1];
      }
      const int64_t pz = ab[1] - ab[0];
      if (pz > 2147483647LL) return bail(fail(NITRO_E_UNSUPPORTED, "a rank part needs < 2^31 nonzeros"));
      if ((rc = st->rp_part[k].alloc((cnt + 1) * 4))) return bail(rc);
      if (rowptr_is_64)
        k_rebase<int64_t><<<grid_n(cnt + 1), 256, 0, s>>>((const int64_t *)d_rowptr, beg[k], cnt, st->rp_part[k].as<int32_t>());
      else
        k_rebase<int32_t><<<grid_n(cnt + 1), 256, 0, s>>>((const int32_t *)d_rowptr, beg[k], cnt, st->rp_part[k].as<int32_t>());
      NITRO_CUDA(cudaGetLastError());
      rc = nitro_spmv_create(D->device, nullptr, cnt, (int64_t)P * st->B, pz, st->rp_part[k].p, 0,
                             st->colmap.as<int32_t>() + ab[0], (const char *)d_vals + ab[0] * sv, is_fp64,
                             &st->part[k]);
      if (rc) return bail(rc);
      st->part[k]->row0 = (int64_t)r * st->B + beg[k];  // rows in the remapped space keep diagonal offsets
    }
    if ((rc = st->xfull.alloc(std::max<int64_t>((int64_t)P * st->B, 1) * sv))) return bail(rc);
    // padding rows of every block stay 0: padded formats (DIA) multiply their
    // zero slots by x there, so it must be finite
    NITRO_CUDA(cudaMemset(st->xfull.p, 0, st->xfull.bytes));
    NITRO_CUDA(cudaDeviceSynchronize());
    // the returned handle: the whole local block over remapped columns
    nitro_spmv *A = nullptr;
    rc = nitro_spmv_create(D->device, nullptr, st->n, (int64_t)P * st->B, local_nnz, d_rowptr, rowptr_is_64,
                           st->colmap.as<int32_t>(), d_vals, is_fp64, &A);
    if (rc) return bail(rc);
    A->row0 = (int64_t)r * st->B;
    A->dist = D;
    A->dist_state = st;
    A->dist_free = free_state;
    *out_local = A;
    return NITRO_OK;
  } catch (...) {
    return fail(NITRO_E_OOM, "host allocation failed");
  }
}

static nitro_status_t run_part(DistState *st, int k, int variant, cudaStream_t s, const void *xg, void *y,
                               size_t sv) {
  nitro_spmv *P = st->part[k];
  if (!P) return NITRO_OK;
  P->stream = s;
  int ok = 0, v = variant;
  NITRO_TRY(nitro_spmv_allowed(P, v, &ok));
  if (!ok) v = NITRO_CSR_VECTOR;  // part-level constraint fallback
  return nitro_spmv_run(P, v, xg, (char *)y + (size_t)st->part_begin[k] * sv);
}

nitro_status_t nitro_dist_spmv_run(nitro_dist *D, nitro_spmv *A, int variant, const void *d_x_local, void *d_y_local) {
  if (!D || !A || !A->dist_state || variant < 0 || variant >= NITRO_NUM_VARIANTS)
    return fail(NITRO_E_INVALID_ARG, "bad argument");
  if (!D->comm && D->nranks > 1) return fail(NITRO_E_STATE, "communicator-less handle: use run_gathered");
  DistState *st = (DistState *)A->dist_state;
  NITRO_CUDA(cudaSetDevice(D->device));
  const size_t sv = A->fp64 ? 8 : 4;
  cudaStream_t s = A->stream;
  char *xfull = st->xfull.as<char>();
  char *mine = xfull + (size_t)D->rank * st->B * sv;
  if (st->n > 0) NITRO_CUDA(cudaMemcpyAsync(mine, d_x_local, st->n * sv, cudaMemcpyDeviceToDevice, s));
  NITRO_CUDA(cudaEventRecord(D->ev_x, s));
  NITRO_CUDA(cudaStreamWaitEvent(D->comm_stream, D->ev_x, 0));
  if (D->nranks > 1)
    NITRO_NCCL(ncclAllGather(mine, xfull, (size_t)st->B, A->fp64 ? ncclFloat64 : ncclFloat32, D->comm,
                             D->comm_stream));
  NITRO_CUDA(cudaEventRecord(D->ev_g, D->comm_stream));
  NITRO_TRY(run_part(st, 1, variant, s, xfull, d_y_local, sv));  // interior: overlaps the all-gather
  NITRO_CUDA(cudaStreamWaitEvent(s, D->ev_g, 0));
  NITRO_TRY(run_part(st, 0, variant, s, xfull, d_y_local, sv));
  NITRO_TRY(run_part(st, 2, variant, s, xfull, d_y_local, sv));
  return NITRO_OK;
}

nitro_status_t nitro_dist_spmv_run_gathered(nitro_dist *D, nitro_spmv *A, int variant, const void *d_xg,
                                            void *d_y_local) {
  if (!D || !A || !A->dist_state || !d_xg || variant < 0 || variant >= NITRO_NUM_VARIANTS)
    return fail(NITRO_E_INVALID_ARG, "bad argument");
  DistState *st = (DistState *)A->dist_state;
  NITRO_CUDA(cudaSetDevice(D->device));
  const size_t sv = A->fp64 ? 8 : 4;
  for (int k = 0; k < 3; ++k) NITRO_TRY(run_part(st, k, variant, A->stream, d_xg, d_y_local, sv));
  return NITRO_OK;
}

nitro_status_t nitro_dist_layout(nitro_spmv *A, int64_t *B, int64_t *i0, int64_t *i1) {
  if (!A || !A->dist_state) return fail(NITRO_E_INVALID_ARG, "not a dist handle");
  DistState *st = (DistState *)A->dist_state;
  if (B) *B = st->B;
  if (i0) *i0 = st->i0;
  if (i1) *i1 = st->i1;
  return NITRO_OK;
}

nitro_status_t nitro_dist_init_local(int rank, int nranks, int device, nitro_dist **out) {
  if (!out || nranks < 1 || rank < 0 || rank >= nranks) return fail(NITRO_E_INVALID_ARG, "bad argument");
  NITRO_CUDA(cudaSetDevice(device));
  nitro_dist *D = new nitro_dist();
  D->rank = rank; D->nranks = nranks; D->device = device;
  NITRO_CUDA(cudaStreamCreateWithFlags(&D->comm_stream, cudaStreamNonBlocking));
  NITRO_CUDA(cudaEventCreateWithFlags(&D->ev_x, cudaEventDisableTiming));
  NITRO_CUDA(cudaEventCreateWithFlags(&D->ev_g, cudaEventDisableTiming));
  *out = D;
  return NITRO_OK;
}

nitro_status_t nitro_dist_features(nitro_dist *D, nitro_spmv *A, nitro_spmv_feat *out) {
  if (!D || !A || !A->dist_state || !out) return fail(NITRO_E_INVALID_ARG, "bad argument");
  if (!D->comm && D->nranks > 1) return fail(NITRO_E_STATE, "communicator-less handle");
  DistState *st = (DistState *)A->dist_state;
  NITRO_CUDA(cudaSetDevice(D->device));
  nitro_spmv *F = st->feat;
  F->stream = A->stream;
  cudaStream_t s = A->stream;
  if (!F->feat_pending && !F->feat_ready) NITRO_TRY(features_launch(F));
  NITRO_CUDA(cudaEventSynchronize(F->feat_done));
  // integer moments: sum (s1, s2), max (lmax, bad)
  DevBuf red;
  NITRO_TRY(red.alloc(5 * 8));
  unsigned long long *sum2 = red.as<unsigned long long>(), *max2 = sum2 + 2, *dcnt = sum2 + 4;
  k_pack_acc<<<1, 1, 0, s>>>(F->feat_acc.as<FeatAcc>(), sum2, max2);
  // occupied diagonals: union of the per-rank bitmaps over the global offset range
  const int64_t span = st->global_rows > 0 ? st->global_rows - 1 + F->M : 0;
  NITRO_TRY(st->flags.alloc(std::max<int64_t>(span, 1)));
  if (span > 0 && F->N > 0)
    k_bits_to_flags<<<grid_n(span), 256, 0, s>>>(F->bitmap.as<uint32_t>(), span, st->flags.as<uint8_t>());
  else if (span > 0)
    NITRO_CUDA(cudaMemsetAsync(st->flags.p, 0, span, s));  // empty block: contributes no diagonal
  NITRO_CUDA(cudaGetLastError());
  if (D->nranks > 1) {
    NITRO_NCCL(ncclGroupStart());
    NITRO_NCCL(ncclAllReduce(sum2, sum2, 2, ncclUint64, ncclSum, D->comm, s));
    NITRO_NCCL(ncclAllReduce(max2, max2, 2, ncclUint64, ncclMax, D->comm, s));
    if (span > 0) NITRO_NCCL(ncclAllReduce(st->flags.p, st->flags.p, span, ncclUint8, ncclMax, D->comm, s));
    NITRO_NCCL(ncclGroupEnd());
  }
  NITRO_CUDA(cudaMemsetAsync(dcnt, 0, 8, s));
  if (span > 0) k_count_flags<<<grid_n(span), 256, 0, s>>>(st->flags.as<uint8_t>(), span, dcnt);
  unsigned long long h[5];
  NITRO_CUDA(cudaMemcpyAsync(h, sum2, 5 * 8, cudaMemcpyDeviceToHost, s));
  NITRO_CUDA(cudaStreamSynchronize(s));
  finish_features(st->global_rows, F->M, (int64_t)h[0], h[0], h[1], (int64_t)h[2], (int64_t)h[4], out);
  out->canonical = h[3] == 0;
  return out->canonical ? NITRO_OK : fail(NITRO_E_BAD_MATRIX, "non-canonical CSR on some rank");
}

}  // extern "C"
