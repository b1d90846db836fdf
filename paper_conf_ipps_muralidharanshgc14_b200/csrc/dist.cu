// dist.cu — A13: multi-GPU row-partitioned SpMV (include/nitro.h §3).
//
// One process per GPU.  Rank r owns the contiguous, nnz-balanced row block
// [bounds[r], bounds[r+1]) (R14) and the matching block of x.  Two
// x-exchange modes, fixed when the handle is created:
//  * all-gather: every multiply all-gathers x in place with NCCL into a padded
//    layout where block q starts at q*B (B = max block rows);
//  * halo: only the x entries this rank's rows reference on
//    other ranks are exchanged (grouped ncclSend/ncclRecv of packed lists),
//    into a layout [x_local (n) | halo (nh)] — for stencil/banded partitions a
//    few planes instead of the whole vector.  Chosen automatically when the
//    largest halo is under a quarter of the all-gather volume.
// Columns are remapped once to the chosen layout.  Local rows are split into
// head [0,i0) / interior [i0,i1) / tail [i1,n): interior rows only touch
// locally owned columns, so they run on the compute stream while the exchange
// is in flight on the comm stream; head and tail rows run after it.  Each part
// is an ordinary nitro_spmv over a rebased CSR slice, so every variant (and
// its constraint) works unchanged.  Global features: per-rank K1 over a
// global-offset bitmap, integer moments all-reduced (sum / max), occupied
// diagonals as each rank's compacted sorted offset list, all-gathered and
// unioned.
//
// Transport: every exchange goes through four operations (all-gather,
// u64 all-reduce, grouped send/recv) implemented either with NCCL (one
// process per GPU) or with the LOOPBACK transport: P rank handles of one
// process on one GPU (one host thread each) whose collectives meet at a host
// barrier and move data with stream-ordered device copies.  The loopback runs
// the same pack / send-list / receive-offset / layout code as NCCL for any P
// on a single GPU, so the P > 1 paths are testable without a second device.
#include <nccl.h>

#include <algorithm>
#include <condition_variable>
#include <mutex>
#include <vector>

#include "nitro_internal.h"
#include "util.cuh"

#include "dist_internal.h"

namespace nitro {
namespace {


// ---------------------------------------------------------------- transport
// All four are collective: every rank of the handle's group calls them in the
// same order.  Work is ordered on stream s.
nitro_status_t t_allgather(nitro_dist *D, const void *send, void *recv, size_t bytes, cudaStream_t s) {
  if (D->nranks == 1) {
    if (send != recv && bytes) NITRO_CUDA(cudaMemcpyAsync(recv, send, bytes, cudaMemcpyDeviceToDevice, s));
    return NITRO_OK;
  }
  if (D->comm) {
    NITRO_NCCL(ncclAllGather(send, recv, bytes, ncclInt8, D->comm, s));
    return NITRO_OK;
  }
  nitro_loopback *L = D->lb;
  auto &me = L->slot[D->rank];
  me.send = send;
  me.recv = recv;
  me.bytes = bytes;
  NITRO_CUDA(cudaEventRecord(me.ready, s));
  L->barrier();
  char *rb = (char *)recv;
  for (int q = 0; q < D->nranks; ++q) {
    const void *src = q == D->rank ? send : L->slot[q].send;
    char *dst = rb + (size_t)q * bytes;
    if (q != D->rank) NITRO_CUDA(cudaStreamWaitEvent(s, L->slot[q].ready, 0));
    if (src != dst && bytes) NITRO_CUDA(cudaMemcpyAsync(dst, src, bytes, cudaMemcpyDeviceToDevice, s));
  }
  NITRO_CUDA(cudaEventRecord(me.done, s));
  L->barrier();
  for (int q = 0; q < D->nranks; ++q)  // nobody reuses its send buffer before every copy of it is done
    if (q != D->rank) NITRO_CUDA(cudaStreamWaitEvent(s, L->slot[q].done, 0));
  L->barrier();  // slots may be re-posted
  return NITRO_OK;
}

// in-place u64 all-reduce (sum or max) of a small device array; syncs s
nitro_status_t t_allreduce_u64(nitro_dist *D, unsigned long long *dbuf, int n, bool is_max, cudaStream_t s) {
  if (D->nranks == 1) return NITRO_OK;
  if (D->comm) {
    NITRO_NCCL(ncclAllReduce(dbuf, dbuf, n, ncclUint64, is_max ? ncclMax : ncclSum, D->comm, s));
    NITRO_CUDA(cudaStreamSynchronize(s));
    return NITRO_OK;
  }
  nitro_loopback *L = D->lb;
  auto &me = L->slot[D->rank];
  me.host.assign(n, 0ull);
  NITRO_CUDA(cudaMemcpyAsync(me.host.data(), dbuf, (size_t)n * 8, cudaMemcpyDeviceToHost, s));
  NITRO_CUDA(cudaStreamSynchronize(s));
  L->barrier();
  std::vector<unsigned long long> r(L->slot[0].host);
  for (int q = 1; q < D->nranks; ++q)
    for (int i = 0; i < n; ++i) r[i] = is_max ? std::max(r[i], L->slot[q].host[i]) : r[i] + L->slot[q].host[i];
  L->barrier();
  NITRO_CUDA(cudaMemcpyAsync(dbuf, r.data(), (size_t)n * 8, cudaMemcpyHostToDevice, s));
  NITRO_CUDA(cudaStreamSynchronize(s));
  return NITRO_OK;
}

// grouped point-to-point: the k-th send to q pairs with q's k-th receive from me
nitro_status_t t_sendrecv(nitro_dist *D, const std::vector<Msg> &sends, const std::vector<Msg> &recvs,
                          cudaStream_t s) {
  if (D->nranks == 1) return NITRO_OK;
  if (D->comm) {
    NITRO_NCCL(ncclGroupStart());
    for (const Msg &m : sends)
      if (m.bytes) NITRO_NCCL(ncclSend(m.src, m.bytes, ncclInt8, m.peer, D->comm, s));
    for (const Msg &m : recvs)
      if (m.bytes) NITRO_NCCL(ncclRecv(m.dst, m.bytes, ncclInt8, m.peer, D->comm, s));
    NITRO_NCCL(ncclGroupEnd());
    return NITRO_OK;
  }
  nitro_loopback *L = D->lb;
  auto &me = L->slot[D->rank];
  me.sends = sends;
  NITRO_CUDA(cudaEventRecord(me.ready, s));
  L->barrier();
  std::vector<int> used(D->nranks, 0);
  for (const Msg &m : recvs) {
    const auto &ps = L->slot[m.peer].sends;
    int k = used[m.peer]++, seen = 0;
    const Msg *src = nullptr;
    for (const Msg &t : ps)
      if (t.peer == D->rank && seen++ == k) { src = &t; break; }
    if (!src || src->bytes != m.bytes) return fail(NITRO_E_STATE, "loopback send/recv mismatch");
    NITRO_CUDA(cudaStreamWaitEvent(s, L->slot[m.peer].ready, 0));
    if (m.bytes) NITRO_CUDA(cudaMemcpyAsync(m.dst, src->src, m.bytes, cudaMemcpyDeviceToDevice, s));
  }
  NITRO_CUDA(cudaEventRecord(me.done, s));
  L->barrier();
  for (int q = 0; q < D->nranks; ++q)
    if (q != D->rank) NITRO_CUDA(cudaStreamWaitEvent(s, L->slot[q].done, 0));
  L->barrier();
  return NITRO_OK;
}


void free_state(void *p) {
  DistState *st = (DistState *)p;
  if (!st) return;
  for (auto *h : st->part) if (h) nitro_spmv_destroy(h);
  if (st->feat) nitro_spmv_destroy(st->feat);
  delete st;
}

unsigned grid_n(int64_t n) {
  int64_t g = (n + 255) / 256, cap = (int64_t)num_sms() * 16;
  return (unsigned)std::max<int64_t>(1, std::min(g, cap));
}

// all-gather layout: owner(c) * B + (c - bounds[owner])
__global__ void k_remap_ag(const int32_t *__restrict__ col, int64_t Z, const int64_t *__restrict__ bounds, int P,
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

// halo layout [x[H_below] | x_local | x[H_above]] (monotone in the global
// column, so remapped rows stay sorted): c < lo -> its position k in the sorted
// halo list H; local c -> nb + (c - lo); c >= hi -> n + k  (nb = |H_below|)
__global__ void k_remap_halo(const int32_t *__restrict__ col, int64_t Z, int64_t lo, int64_t hi, int64_t n,
                             int64_t nb, const int32_t *__restrict__ H, int64_t nh, int32_t *__restrict__ out) {
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < Z; k += (int64_t)gridDim.x * blockDim.x) {
    const int64_t c = col[k];
    if (c >= lo && c < hi) { out[k] = (int32_t)(nb + c - lo); continue; }
    int64_t a = 0, b = nh;
    while (a < b) {
      const int64_t m = (a + b) >> 1;
      if ((int64_t)H[m] < c) a = m + 1; else b = m;
    }
    out[k] = (int32_t)(c < lo ? a : n + a);
  }
}

// mark remote columns in a bitmap over the global columns
__global__ void k_mark_remote(const int32_t *__restrict__ col, int64_t Z, int64_t lo, int64_t hi,
                              uint32_t *__restrict__ bm) {
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < Z; k += (int64_t)gridDim.x * blockDim.x) {
    const int64_t c = col[k];
    if (c < lo || c >= hi) {
      const uint32_t bit = 1u << (c & 31);
      if (!(__ldcg(bm + (c >> 5)) & bit)) atomicOr(bm + (c >> 5), bit);
    }
  }
}
__global__ void __launch_bounds__(256) k_bm_tile_counts(const uint32_t *__restrict__ bm, int64_t nwords,
                                                        int64_t *__restrict__ cnt) {
  const int64_t base = (int64_t)blockIdx.x * 1024;
  int64_t s = 0;
  for (int t = threadIdx.x; t < 1024; t += 256)
    if (base + t < nwords) s += __popc(bm[base + t]);
  s = block_sum_i64<256>(s);
  if (threadIdx.x == 0) cnt[blockIdx.x] = s;
}
__global__ void __launch_bounds__(256) k_bm_emit(const uint32_t *__restrict__ bm, int64_t nwords,
                                                 const int64_t *__restrict__ tile_off, int32_t *__restrict__ out) {
  const int64_t base = (int64_t)blockIdx.x * 1024 + threadIdx.x * 4;
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
      const int b = __ffs(v) - 1;
      v &= v - 1;
      out[o++] = (int32_t)((base + q) * 32 + b);
    }
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

template <typename IT, typename OT>
__global__ void k_rebase(const IT *__restrict__ rowptr, int64_t s, int64_t cnt, OT *__restrict__ out) {
  const int64_t base = (int64_t)rowptr[s];
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i <= cnt; i += (int64_t)gridDim.x * blockDim.x)
    out[i] = (OT)((int64_t)rowptr[s + i] - base);
}

__global__ void k_to_local(int32_t *__restrict__ ids, int64_t n, int64_t lo) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    ids[i] = (int32_t)((int64_t)ids[i] - lo);
}

template <typename VT>
__global__ void k_pack(const VT *__restrict__ xl, const int32_t *__restrict__ idx, int64_t n, VT *__restrict__ out) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    out[i] = xl[idx[i]];
}

__global__ void k_set_bits(const int32_t *__restrict__ idx, int64_t n, uint32_t *__restrict__ bm) {
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < n; t += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t i = (uint32_t)idx[t];
    atomicOr(bm + (i >> 5), 1u << (i & 31));
  }
}
__global__ void k_popc_sum(const uint32_t *__restrict__ bm, int64_t nwords, unsigned long long *out) {
  unsigned long long c = 0;
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < nwords; t += (int64_t)gridDim.x * blockDim.x)
    c += __popc(bm[t]);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
  if ((threadIdx.x & 31) == 0 && c) atomicAdd(out, c);
}
__global__ void k_pack_acc(const FeatAcc *a, unsigned long long *sum2, unsigned long long *max2) {
  sum2[0] = a->s1; sum2[1] = a->s2; max2[0] = a->lmax; max2[1] = a->bad;
}

// sorted list of the remote global columns referenced by this rank's rows
nitro_status_t halo_list(DistState *st, const int32_t *col, int64_t Z, DevBuf &out, int64_t &nh) {
  const int64_t M = st->global_rows, nwords = (M + 31) / 32, nt = (nwords + 1023) / 1024;
  DevBuf bm, cnt, scratch;
  NITRO_TRY(bm.alloc((size_t)std::max<int64_t>(nwords, 1) * 4));
  NITRO_CUDA(cudaMemset(bm.p, 0, (size_t)std::max<int64_t>(nwords, 1) * 4));
  if (Z > 0) k_mark_remote<<<grid_n(Z), 256>>>(col, Z, st->bounds[st->D->rank], st->bounds[st->D->rank + 1],
                                               bm.as<uint32_t>());
  NITRO_TRY(cnt.alloc((size_t)(2 * nt + 2) * 8));
  int64_t *tc = cnt.as<int64_t>(), *to = tc + nt + 1;
  nh = 0;
  if (nt > 0) {
    k_bm_tile_counts<<<(unsigned)nt, 256>>>(bm.as<uint32_t>(), nwords, tc);
    NITRO_TRY(exclusive_scan_i64(tc, to, nt, scratch, nullptr));
    NITRO_CUDA(cudaMemcpy(&nh, to + nt, 8, cudaMemcpyDeviceToHost));
  }
  NITRO_TRY(out.alloc((size_t)std::max<int64_t>(nh, 1) * 4));
  if (nh > 0) k_bm_emit<<<(unsigned)nt, 256>>>(bm.as<uint32_t>(), nwords, to, out.as<int32_t>());
  NITRO_CUDA(cudaGetLastError());
  NITRO_CUDA(cudaDeviceSynchronize());
  return NITRO_OK;
}

// halo plan: what to receive from each owner, and (via NCCL) what to send to each requester
nitro_status_t halo_plan(DistState *st) {
  nitro_dist *D = st->D;
  const int P = D->nranks, me = D->rank;
  std::vector<int32_t> H(st->nh);
  if (st->nh) NITRO_CUDA(cudaMemcpy(H.data(), st->halo_cols.p, st->nh * 4, cudaMemcpyDeviceToHost));
  st->recv_off.assign(P + 1, 0);
  for (int q = 0, k = 0; q < P; ++q) {
    while (k < (int)st->nh && H[k] < st->bounds[q + 1]) ++k;
    st->recv_off[q + 1] = k;
  }
  st->nb = st->recv_off[me];  // halo entries owned by lower ranks (columns < lo)
  st->send_off.assign(P + 1, 0);
  st->ns = 0;
  if (!D->has_transport() || P == 1) return NITRO_OK;  // communicator-less: the caller supplies the layout
  // need matrix: row r = counts rank r receives from each owner
  DevBuf need;
  NITRO_TRY(need.alloc((size_t)P * P * 8));
  std::vector<int64_t> mine(P), all((size_t)P * P);
  for (int q = 0; q < P; ++q) mine[q] = st->recv_off[q + 1] - st->recv_off[q];
  NITRO_CUDA(cudaMemcpy(need.as<int64_t>() + (size_t)me * P, mine.data(), P * 8, cudaMemcpyHostToDevice));
  NITRO_TRY(t_allgather(D, need.as<int64_t>() + (size_t)me * P, need.p, (size_t)P * 8, D->comm_stream));
  NITRO_CUDA(cudaStreamSynchronize(D->comm_stream));
  NITRO_CUDA(cudaMemcpy(all.data(), need.p, (size_t)P * P * 8, cudaMemcpyDeviceToHost));
  for (int r = 0; r < P; ++r) st->send_off[r + 1] = st->send_off[r] + all[(size_t)r * P + me];
  st->ns = st->send_off[P];
  NITRO_TRY(st->send_idx.alloc((size_t)std::max<int64_t>(st->ns, 1) * 4));
  // requesters send me the global ids they need from me
  std::vector<Msg> sends, recvs;
  for (int q = 0; q < P; ++q) {
    if (q == me) continue;
    const int64_t rc = st->recv_off[q + 1] - st->recv_off[q];
    const int64_t sc = st->send_off[q + 1] - st->send_off[q];
    if (rc > 0) sends.push_back({q, st->halo_cols.as<int32_t>() + st->recv_off[q], nullptr, (size_t)rc * 4});
    if (sc > 0) recvs.push_back({q, nullptr, st->send_idx.as<int32_t>() + st->send_off[q], (size_t)sc * 4});
  }
  NITRO_TRY(t_sendrecv(D, sends, recvs, D->comm_stream));
  NITRO_CUDA(cudaStreamSynchronize(D->comm_stream));
  if (st->ns > 0) k_to_local<<<grid_n(st->ns), 256>>>(st->send_idx.as<int32_t>(), st->ns, st->bounds[me]);
  NITRO_CUDA(cudaDeviceSynchronize());
  return NITRO_OK;
}

nitro_status_t run_part(DistState *st, int k, int variant, cudaStream_t s, const void *xg, void *y, size_t sv) {
  nitro_spmv *P = st->part[k];
  if (!P) return NITRO_OK;
  P->stream = s;
  int ok = 0, v = variant;
  NITRO_TRY(nitro_spmv_allowed(P, v, &ok));
  if (!ok) v = NITRO_CSR_VECTOR;  // part-level constraint fallback
  return nitro_spmv_run(P, v, xg, (char *)y + (size_t)st->part_begin[k] * sv);
}

}  // namespace

nitro_status_t dist_allgather(nitro_dist *D, const void *send, void *recv, size_t bytes, cudaStream_t s) {
  return t_allgather(D, send, recv, bytes, s);
}
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

nitro_status_t nitro_dist_spmv_create_ex(nitro_dist *D, int64_t global_rows, const int64_t *bounds, int64_t local_nnz,
                                         const void *d_rowptr, int rowptr_is_64, const int32_t *d_colidx,
                                         const void *d_vals, int is_fp64, int exchange, nitro_spmv **out_local) {
  try {
    if (!D || !bounds || !d_rowptr || !out_local || local_nnz < 0 || exchange < -1 || exchange > 1)
      return fail(NITRO_E_INVALID_ARG, "bad argument");
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
    const size_t sv = is_fp64 ? 8 : 4;
    auto bail = [&](nitro_status_t code) { free_state(st); return code; };
    // features handle over the original columns (global rows start at row_begin)
    nitro_status_t rc = nitro_spmv_create(D->device, nullptr, st->n, global_rows, local_nnz, d_rowptr, rowptr_is_64,
                                          d_colidx, d_vals, is_fp64, &st->feat);
    if (rc) return bail(rc);
    st->feat->row0 = st->row_begin;
    st->feat->feat_G = global_rows - 1;
    // ---- exchange mode: halo when the largest halo is < 1/4 of the all-gather volume
    if ((rc = halo_list(st, d_colidx, local_nnz, st->halo_cols, st->nh))) return bail(rc);
    int64_t max_nh = st->nh;
    if (D->has_transport() && P > 1) {
      DevBuf t;
      if ((rc = t.alloc(8))) return bail(rc);
      NITRO_CUDA(cudaMemcpy(t.p, &max_nh, 8, cudaMemcpyHostToDevice));
      if ((rc = t_allreduce_u64(D, t.as<unsigned long long>(), 1, true, D->comm_stream))) return bail(rc);
      NITRO_CUDA(cudaMemcpy(&max_nh, t.p, 8, cudaMemcpyDeviceToHost));
    }
    st->mode = exchange == -1 ? (4 * max_nh < (int64_t)(P - 1) * st->B || P == 1 ? kHalo : kAllGather) : exchange;
    if (st->mode == kAllGather && (int64_t)P * st->B > 2147483647LL)
      return bail(fail(NITRO_E_UNSUPPORTED, "all-gather layout needs P*B < 2^31"));
    if (st->mode == kHalo) {
      if (st->n + st->nh > 2147483647LL) return bail(fail(NITRO_E_UNSUPPORTED, "n + halo must be < 2^31"));
      if ((rc = halo_plan(st))) return bail(rc);
      if ((rc = st->sendbuf.alloc((size_t)std::max<int64_t>(st->ns, 1) * sv))) return bail(rc);
    }
    // remapped columns
    if ((rc = st->colmap.alloc(std::max<int64_t>(local_nnz, 1) * 4))) return bail(rc);
    if (local_nnz > 0) {
      if (st->mode == kHalo) {
        k_remap_halo<<<grid_n(local_nnz), 256>>>(d_colidx, local_nnz, bounds[r], bounds[r + 1], st->n, st->nb,
                                                 st->halo_cols.as<int32_t>(), st->nh, st->colmap.as<int32_t>());
      } else {
        DevBuf dbounds;
        if ((rc = dbounds.alloc((P + 1) * 8))) return bail(rc);
        NITRO_CUDA(cudaMemcpy(dbounds.p, bounds, (P + 1) * 8, cudaMemcpyHostToDevice));
        k_remap_ag<<<grid_n(local_nnz), 256>>>(d_colidx, local_nnz, dbounds.as<int64_t>(), P, st->B,
                                               st->colmap.as<int32_t>());
        NITRO_CUDA(cudaDeviceSynchronize());
      }
    }
    // interior rows (all columns inside this rank's block) -> contiguous run [i0, i1)
    std::vector<uint8_t> hf(st->n);
    if (st->n > 0) {
      if ((rc = st->flags.alloc(st->n))) return bail(rc);
      if (rowptr_is_64)
        k_interior<int64_t><<<grid_n(st->n), 256>>>((const int64_t *)d_rowptr, d_colidx, st->n, bounds[r],
                                                    bounds[r + 1], st->flags.as<uint8_t>());
      else
        k_interior<int32_t><<<grid_n(st->n), 256>>>((const int32_t *)d_rowptr, d_colidx, st->n, bounds[r],
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
    const int64_t Mx = st->layout_len(), xoff = st->x_offset();
    // three part handles over rebased CSR slices with remapped columns
    const int64_t beg[3] = {0, i0, i1}, end[3] = {i0, i1, st->n};
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
      const bool p64 = pz > 2147483647LL;  // parts of >= 2^31 nonzeros keep 64-bit row pointers
      if ((rc = st->rp_part[k].alloc((cnt + 1) * (p64 ? 8 : 4)))) return bail(rc);
      if (rowptr_is_64) {
        if (p64) k_rebase<int64_t, int64_t><<<grid_n(cnt + 1), 256>>>((const int64_t *)d_rowptr, beg[k], cnt, st->rp_part[k].as<int64_t>());
        else k_rebase<int64_t, int32_t><<<grid_n(cnt + 1), 256>>>((const int64_t *)d_rowptr, beg[k], cnt, st->rp_part[k].as<int32_t>());
      } else {
        k_rebase<int32_t, int32_t><<<grid_n(cnt + 1), 256>>>((const int32_t *)d_rowptr, beg[k], cnt, st->rp_part[k].as<int32_t>());
      }
      NITRO_CUDA(cudaGetLastError());
      rc = nitro_spmv_create(D->device, nullptr, cnt, Mx, pz, st->rp_part[k].p, p64 ? 1 : 0,
                             st->colmap.as<int32_t>() + ab[0], (const char *)d_vals + ab[0] * sv, is_fp64, &st->part[k]);
      if (rc) return bail(rc);
      st->part[k]->row0 = xoff + beg[k];  // local row i sits at layout index xoff + i: diagonal offsets kept
    }
    if ((rc = st->xbuf.alloc(std::max<int64_t>(Mx, 1) * sv))) return bail(rc);
    // padding / not-yet-exchanged entries stay 0: padded formats (DIA) multiply
    // their zero slots by x there, so it must be finite
    NITRO_CUDA(cudaMemset(st->xbuf.p, 0, st->xbuf.bytes));
    NITRO_CUDA(cudaDeviceSynchronize());
    // the returned handle: the whole local block over remapped columns
    nitro_spmv *A = nullptr;
    rc = nitro_spmv_create(D->device, nullptr, st->n, Mx, local_nnz, d_rowptr, rowptr_is_64, st->colmap.as<int32_t>(),
                           d_vals, is_fp64, &A);
    if (rc) return bail(rc);
    A->row0 = xoff;
    A->dist = D;
    A->dist_state = st;
    A->dist_free = free_state;
    *out_local = A;
    return NITRO_OK;
  } catch (...) {
    return fail(NITRO_E_OOM, "host allocation failed");
  }
}

nitro_status_t nitro_dist_spmv_create(nitro_dist *D, int64_t global_rows, const int64_t *bounds, int64_t local_nnz,
                                      const void *d_rowptr, int rowptr_is_64, const int32_t *d_colidx,
                                      const void *d_vals, int is_fp64, nitro_spmv **out_local) {
  return nitro_dist_spmv_create_ex(D, global_rows, bounds, local_nnz, d_rowptr, rowptr_is_64, d_colidx, d_vals,
                                   is_fp64, -1, out_local);
}

nitro_status_t nitro_dist_spmv_run(nitro_dist *D, nitro_spmv *A, int variant, const void *d_x_local, void *d_y_local) {
  NITRO_NVTX("nitro_dist_spmv_run");
  if (!D || !A || !A->dist_state || variant < 0 || variant >= NITRO_NUM_VARIANTS)
    return fail(NITRO_E_INVALID_ARG, "bad argument");
  if (!D->has_transport() && D->nranks > 1) return fail(NITRO_E_STATE, "communicator-less handle: use run_gathered");
  DistState *st = (DistState *)A->dist_state;
  NITRO_CUDA(cudaSetDevice(D->device));
  const size_t sv = A->fp64 ? 8 : 4;
  cudaStream_t s = A->stream;
  char *xb = st->xbuf.as<char>();
  char *mine = xb + (size_t)st->x_offset() * sv;
  if (st->n > 0 && d_x_local != mine)  // callers that write x in place (nitro_dist_x_local) skip this copy
    NITRO_CUDA(cudaMemcpyAsync(mine, d_x_local, st->n * sv, cudaMemcpyDeviceToDevice, s));
  if (st->mode == kHalo && st->ns > 0) {
    if (A->fp64) k_pack<double><<<grid_n(st->ns), 256, 0, s>>>((const double *)mine, st->send_idx.as<int32_t>(), st->ns, st->sendbuf.as<double>());
    else k_pack<float><<<grid_n(st->ns), 256, 0, s>>>((const float *)mine, st->send_idx.as<int32_t>(), st->ns, st->sendbuf.as<float>());
    NITRO_CUDA(cudaGetLastError());
  }
  NITRO_CUDA(cudaEventRecord(D->ev_x, s));
  NITRO_CUDA(cudaStreamWaitEvent(D->comm_stream, D->ev_x, 0));
  if (D->nranks > 1) {
    if (st->mode == kAllGather) {
      NITRO_TRY(t_allgather(D, mine, xb, (size_t)st->B * sv, D->comm_stream));
    } else {
      std::vector<Msg> sends, recvs;
      for (int q = 0; q < D->nranks; ++q) {
        if (q == D->rank) continue;
        const int64_t sc = st->send_off[q + 1] - st->send_off[q], rc = st->recv_off[q + 1] - st->recv_off[q];
        if (sc > 0) sends.push_back({q, st->sendbuf.as<char>() + (size_t)st->send_off[q] * sv, nullptr, (size_t)sc * sv});
        if (rc > 0) recvs.push_back({q, nullptr, xb + (size_t)st->halo_dest(st->recv_off[q]) * sv, (size_t)rc * sv});
      }
      NITRO_TRY(t_sendrecv(D, sends, recvs, D->comm_stream));
    }
  }
  NITRO_CUDA(cudaEventRecord(D->ev_g, D->comm_stream));
  NITRO_TRY(run_part(st, 1, variant, s, xb, d_y_local, sv));  // interior: overlaps the exchange
  NITRO_CUDA(cudaStreamWaitEvent(s, D->ev_g, 0));
  NITRO_TRY(run_part(st, 0, variant, s, xb, d_y_local, sv));
  NITRO_TRY(run_part(st, 2, variant, s, xb, d_y_local, sv));
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

nitro_status_t nitro_dist_format_info(nitro_spmv *A, int variant, nitro_format_info *out) {
  if (!A || !A->dist_state || !out || variant < 0 || variant >= NITRO_NUM_VARIANTS)
    return fail(NITRO_E_INVALID_ARG, "bad argument");
  DistState *st = (DistState *)A->dist_state;
  const double sv = A->fp64 ? 8 : 4;
  memset(out, 0, sizeof(*out));
  double cb = (double)st->layout_len() * sv;  // the exchanged x layout, read once
  for (nitro_spmv *P : st->part) {
    if (!P) continue;
    int ok = 0, v = variant;
    NITRO_TRY(nitro_spmv_allowed(P, v, &ok));
    if (!ok) v = NITRO_CSR_VECTOR;  // as run_part
    nitro_format_info fi;
    NITRO_TRY(nitro_spmv_format_info(P, v, &fi));
    cb += fi.compulsory_bytes - (double)P->M * sv;  // each part's matrix + y bytes
    out->bytes += fi.bytes;
    out->tail += fi.tail;
    out->width = std::max(out->width, fi.width);
    out->ld = std::max(out->ld, fi.ld);
  }
  out->compulsory_bytes = cb;
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

nitro_status_t nitro_dist_exchange_info(nitro_spmv *A, int *mode, int64_t *layout_len, int64_t *halo_len,
                                        int64_t *send_len) {
  if (!A || !A->dist_state) return fail(NITRO_E_INVALID_ARG, "not a dist handle");
  DistState *st = (DistState *)A->dist_state;
  if (mode) *mode = st->mode;
  if (layout_len) *layout_len = st->layout_len();
  if (halo_len) *halo_len = st->nh;
  if (send_len) *send_len = st->ns;
  return NITRO_OK;
}

nitro_status_t nitro_dist_halo_cols(nitro_spmv *A, int32_t *h_out) {
  if (!A || !A->dist_state) return fail(NITRO_E_INVALID_ARG, "not a dist handle");
  DistState *st = (DistState *)A->dist_state;
  if (h_out && st->nh) NITRO_CUDA(cudaMemcpy(h_out, st->halo_cols.p, st->nh * 4, cudaMemcpyDeviceToHost));
  return NITRO_OK;
}

nitro_status_t nitro_dist_x_local(nitro_spmv *A, void **ptr) {
  if (!A || !A->dist_state || !ptr) return fail(NITRO_E_INVALID_ARG, "not a dist handle");
  DistState *st = (DistState *)A->dist_state;
  *ptr = st->xbuf.as<char>() + (size_t)st->x_offset() * (A->fp64 ? 8 : 4);
  return NITRO_OK;
}

nitro_status_t nitro_dist_features(nitro_dist *D, nitro_spmv *A, nitro_spmv_feat *out) {
  NITRO_NVTX("nitro_dist_features");
  if (!D || !A || !A->dist_state || !out) return fail(NITRO_E_INVALID_ARG, "bad argument");
  if (!D->has_transport() && D->nranks > 1) return fail(NITRO_E_STATE, "communicator-less handle");
  DistState *st = (DistState *)A->dist_state;
  NITRO_CUDA(cudaSetDevice(D->device));
  nitro_spmv *F = st->feat;
  F->stream = A->stream;
  cudaStream_t s = A->stream;
  const int P = D->nranks;
  if (!F->feat_pending && !F->feat_ready) NITRO_TRY(features_launch(F));
  NITRO_CUDA(cudaEventSynchronize(F->feat_done));
  // integer moments: sum (s1, s2), max (lmax, bad)
  DevBuf red;
  NITRO_TRY(red.alloc(5 * 8));
  unsigned long long *sum2 = red.as<unsigned long long>(), *max2 = sum2 + 2, *dcnt = sum2 + 4;
  k_pack_acc<<<1, 1, 0, s>>>(F->feat_acc.as<FeatAcc>(), sum2, max2);
  NITRO_CUDA(cudaGetLastError());
  NITRO_TRY(t_allreduce_u64(D, sum2, 2, false, s));
  NITRO_TRY(t_allreduce_u64(D, max2, 2, true, s));
  // occupied diagonals: this rank's sorted distinct offsets,
  // compacted from its bitmap over the global offset range [0, span), are
  // all-gathered (padded to the largest count) and unioned into one bitmap
  const int64_t span = st->global_rows > 0 ? st->global_rows - 1 + F->M : 0;
  const int64_t nwords = (span + 31) / 32, nt = (nwords + 1023) / 1024;
  int64_t cnt = 0;
  DevBuf tiles, scratch, mylist;
  if (nt > 0 && F->N > 0) {
    NITRO_TRY(tiles.alloc((size_t)(2 * nt + 2) * 8));
    int64_t *tc = tiles.as<int64_t>(), *to = tc + nt + 1;
    k_bm_tile_counts<<<(unsigned)nt, 256, 0, s>>>(F->bitmap.as<uint32_t>(), nwords, tc);
    NITRO_TRY(exclusive_scan_i64(tc, to, nt, scratch, s));
    NITRO_CUDA(cudaMemcpyAsync(&cnt, to + nt, 8, cudaMemcpyDeviceToHost, s));
    NITRO_CUDA(cudaStreamSynchronize(s));
    NITRO_TRY(mylist.alloc((size_t)std::max<int64_t>(cnt, 1) * 4));
    if (cnt > 0) k_bm_emit<<<(unsigned)nt, 256, 0, s>>>(F->bitmap.as<uint32_t>(), nwords, to, mylist.as<int32_t>());
    NITRO_CUDA(cudaGetLastError());
  }
  DevBuf counts;
  NITRO_TRY(counts.alloc((size_t)P * 8));
  NITRO_CUDA(cudaMemcpyAsync(counts.as<int64_t>() + D->rank, &cnt, 8, cudaMemcpyHostToDevice, s));
  NITRO_TRY(t_allgather(D, counts.as<int64_t>() + D->rank, counts.p, 8, s));
  std::vector<int64_t> hc(P);
  NITRO_CUDA(cudaMemcpyAsync(hc.data(), counts.p, (size_t)P * 8, cudaMemcpyDeviceToHost, s));
  NITRO_CUDA(cudaStreamSynchronize(s));
  const int64_t maxc = *std::max_element(hc.begin(), hc.end());
  NITRO_CUDA(cudaMemsetAsync(dcnt, 0, 8, s));
  if (maxc > 0) {
    DevBuf all, bm;
    NITRO_TRY(all.alloc((size_t)P * maxc * 4));
    int32_t *mine = all.as<int32_t>() + (size_t)D->rank * maxc;
    if (cnt > 0) NITRO_CUDA(cudaMemcpyAsync(mine, mylist.p, (size_t)cnt * 4, cudaMemcpyDeviceToDevice, s));
    NITRO_TRY(t_allgather(D, mine, all.p, (size_t)maxc * 4, s));
    NITRO_TRY(bm.alloc((size_t)nwords * 4));
    NITRO_CUDA(cudaMemsetAsync(bm.p, 0, (size_t)nwords * 4, s));
    for (int q = 0; q < P; ++q)
      if (hc[q] > 0)
        k_set_bits<<<grid_n(hc[q]), 256, 0, s>>>(all.as<int32_t>() + (size_t)q * maxc, hc[q], bm.as<uint32_t>());
    k_popc_sum<<<grid_n(nwords), 256, 0, s>>>(bm.as<uint32_t>(), nwords, dcnt);
    NITRO_CUDA(cudaGetLastError());
    unsigned long long h[5];
    NITRO_CUDA(cudaMemcpyAsync(h, sum2, 5 * 8, cudaMemcpyDeviceToHost, s));
    NITRO_CUDA(cudaStreamSynchronize(s));
    finish_features(st->global_rows, F->M, (int64_t)h[0], h[0], h[1], (int64_t)h[2], (int64_t)h[4], out);
    out->canonical = h[3] == 0;
  } else {
    unsigned long long h[5];
    NITRO_CUDA(cudaMemcpyAsync(h, sum2, 5 * 8, cudaMemcpyDeviceToHost, s));
    NITRO_CUDA(cudaStreamSynchronize(s));
    finish_features(st->global_rows, F->M, (int64_t)h[0], h[0], h[1], (int64_t)h[2], 0, out);
    out->canonical = h[3] == 0;
  }
  return out->canonical ? NITRO_OK : fail(NITRO_E_BAD_MATRIX, "non-canonical CSR on some rank");
}

nitro_status_t nitro_dist_loopback_create(int nranks, int device, nitro_loopback **out) {
  if (!out || nranks < 1) return fail(NITRO_E_INVALID_ARG, "bad argument");
  NITRO_CUDA(cudaSetDevice(device));
  nitro_loopback *L = new nitro_loopback();
  L->nranks = nranks;
  L->device = device;
  L->slot.resize(nranks);
  for (auto &sl : L->slot) {
    NITRO_CUDA(cudaEventCreateWithFlags(&sl.ready, cudaEventDisableTiming));
    NITRO_CUDA(cudaEventCreateWithFlags(&sl.done, cudaEventDisableTiming));
  }
  *out = L;
  return NITRO_OK;
}

void nitro_dist_loopback_destroy(nitro_loopback *L) {
  if (!L) return;
  cudaSetDevice(L->device);
  for (auto &sl : L->slot) {
    if (sl.ready) cudaEventDestroy(sl.ready);
    if (sl.done) cudaEventDestroy(sl.done);
  }
  delete L;
}

nitro_status_t nitro_dist_init_loopback(nitro_loopback *L, int rank, nitro_dist **out) {
  if (!L || !out || rank < 0 || rank >= L->nranks) return fail(NITRO_E_INVALID_ARG, "bad argument");
  NITRO_TRY(nitro_dist_init_local(rank, L->nranks, L->device, out));
  (*out)->lb = L;
  return NITRO_OK;
}

}  // extern "C"
