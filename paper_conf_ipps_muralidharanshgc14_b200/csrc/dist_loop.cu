// dist_loop.cu — SURVEY §8(f) f3 (ii): the solver-loop mode of the multi-GPU
// SpMV with the y -> x exchange FUSED into the SpMV epilogue.
//
// In a solver-style loop (power iteration, Krylov-type methods without a
// global reduction between multiplies) the y block a rank computes is the x
// block every rank reads in the next multiply.  A13 computes y, then
// all-gathers it (a separate NCCL collective, x ingress floor 0.52 ms at P = 8
// on configs[4]).  Here the multiply's own store epilogue writes each y_i
// straight into every rank's NEXT x layout (all-gather layout: block r at
// r*B), so the exchange is spread over the whole kernel instead of following
// it, and one cross-rank barrier closes the step:
//  * NCCL ranks: the two x layouts live in symmetric memory (ncclMemAlloc +
//    ncclCommWindowRegister, NCCL_WIN_COLL_SYMMETRIC); peer addresses come
//    from the NCCL device API (ncclGetPeerPointer on the window), the barrier
//    is an LSA barrier session (ncclDevCommCreate with one LSA barrier) in a
//    one-CTA kernel ordered after the multiply on the stream;
//  * loopback ranks (one GPU): the layouts are device buffers whose addresses
//    the ranks exchange through the group; the barrier is the group's host
//    barrier after a stream synchronise.
// The multiply reads x_k from buffer k%2 and writes x_{k+1} into buffer
// (k+1)%2, so no rank overwrites what a peer may still be reading.  CSR-scalar,
// ELL and DIA carry the fused epilogue (launch_spmv_fused: the same kernels,
// bit-identical values); a rank part running another variant (CSR-vector,
// HYB, or a constraint fallback) writes its block of the next layout locally
// and pushes it to the peers with a copy kernel.
#include <nccl.h>
#include <nccl_device.h>

#include <algorithm>
#include <vector>

#include "dist_internal.h"
#include "util.cuh"

struct nitro_dist_loop {
  nitro_dist *D = nullptr;
  nitro_spmv *A = nullptr;
  nitro::DistState *st = nullptr;
  size_t sv = 4, layout_bytes = 0, my_off = 0;  // my block's byte offset in a layout
  void *xb[2] = {nullptr, nullptr};
  bool nccl_mem = false;
  ncclWindow_t win[2] = {nullptr, nullptr};
  ncclDevComm devcomm{};
  bool devcomm_ok = false;
  nitro::DevBuf own[2];     // loopback: the layouts
  nitro::DevBuf table;      // [2][P] device pointers: rank q's layout b + my_off
  int cur = 0;              // the buffer holding x_k
};

namespace nitro {
namespace {

__global__ void k_peer_table(ncclWindow_t w0, ncclWindow_t w1, size_t off, int P, void **table) {
  for (int q = threadIdx.x; q < P; q += blockDim.x) {
    table[q] = ncclGetPeerPointer(w0, off, q);
    table[P + q] = ncclGetPeerPointer(w1, off, q);
  }
}

// cross-rank barrier of one step: every rank's stores of this step (earlier
// kernels on the stream) are released system-wide before it arrives
__global__ void k_lsa_barrier(ncclDevComm comm) {
  __threadfence_system();
  ncclLsaBarrierSession<ncclCoopCta> bar(ncclCoopCta(), comm, ncclTeamTagLsa(), 0);
  bar.sync(ncclCoopCta(), cuda::memory_order_acq_rel);
}

// fallback push of this rank's block [0, n) of the next layout to every peer
template <typename VT>
__global__ void k_push(const VT *__restrict__ src, int64_t n, void *const *__restrict__ dst, int64_t off, int P,
                       int self) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const VT v = src[i];
    for (int q = 0; q < P; ++q)
      if (q != self) reinterpret_cast<VT *>(dst[q])[off + i] = v;
  }
}

bool fusable(int v) { return v == NITRO_CSR_SCALAR || v == NITRO_ELL || v == NITRO_DIA; }

nitro_status_t loop_barrier(nitro_dist_loop *L, cudaStream_t s) {
  nitro_dist *D = L->D;
  if (D->nranks == 1 && !D->comm) return NITRO_OK;
  if (D->comm) {
    k_lsa_barrier<<<1, 128, 0, s>>>(L->devcomm);
    NITRO_CUDA(cudaGetLastError());
    return NITRO_OK;
  }
  NITRO_CUDA(cudaStreamSynchronize(s));  // my stores (into every rank's layout) are done
  D->lb->barrier();
  return NITRO_OK;
}

}  // namespace
}  // namespace nitro

using namespace nitro;

extern "C" {

nitro_status_t nitro_dist_loop_create(nitro_dist *D, nitro_spmv *A, nitro_dist_loop **out) {
  if (!D || !A || !A->dist_state || !out) return fail(NITRO_E_INVALID_ARG, "bad argument");
  DistState *st = (DistState *)A->dist_state;
  if (st->mode != kAllGather) return fail(NITRO_E_UNSUPPORTED, "solver-loop mode needs the all-gather layout");
  if (!D->has_transport() && D->nranks > 1) return fail(NITRO_E_STATE, "communicator-less handle");
  NITRO_CUDA(cudaSetDevice(D->device));
  const int P = D->nranks;
  nitro_dist_loop *L = new nitro_dist_loop();
  L->D = D;
  L->A = A;
  L->st = st;
  L->sv = A->fp64 ? 8 : 4;
  L->layout_bytes = (size_t)P * (size_t)st->B * L->sv;
  L->my_off = (size_t)D->rank * (size_t)st->B * L->sv;
  const size_t bytes = std::max<size_t>(L->layout_bytes, 4096);
  auto bail = [&](nitro_status_t rc) {
    nitro_dist_loop_destroy(L);
    return rc;
  };
  nitro_status_t rc = L->table.alloc((size_t)2 * P * sizeof(void *));
  if (rc) return bail(rc);
  if (D->comm) {
    ncclTeam_t lsa = ncclTeamLsa(D->comm);
    if (lsa.nRanks != P) return bail(fail(NITRO_E_UNSUPPORTED, "solver-loop mode needs every rank in one NVLink (LSA) domain"));
    for (int b = 0; b < 2; ++b) {
      ncclResult_t r = ncclMemAlloc(&L->xb[b], bytes);
      if (r != ncclSuccess) return bail(fail(NITRO_E_OOM, std::string("ncclMemAlloc: ") + ncclGetErrorString(r)));
      r = ncclCommWindowRegister(D->comm, L->xb[b], bytes, &L->win[b], NCCL_WIN_COLL_SYMMETRIC);
      if (r != ncclSuccess) return bail(fail(NITRO_E_NCCL, std::string("ncclCommWindowRegister: ") + ncclGetErrorString(r)));
    }
    L->nccl_mem = true;
    ncclDevCommRequirements reqs;
    memset(&reqs, 0, sizeof(reqs));
    reqs.lsaBarrierCount = 1;
    ncclResult_t r = ncclDevCommCreate(D->comm, &reqs, &L->devcomm);
    if (r != ncclSuccess) return bail(fail(NITRO_E_NCCL, std::string("ncclDevCommCreate: ") + ncclGetErrorString(r)));
    L->devcomm_ok = true;
    k_peer_table<<<1, 32>>>(L->win[0], L->win[1], L->my_off, P, L->table.as<void *>());
    NITRO_CUDA(cudaGetLastError());
  } else {
    for (int b = 0; b < 2; ++b) {
      if ((rc = L->own[b].alloc(bytes))) return bail(rc);
      L->xb[b] = L->own[b].p;
    }
    std::vector<void *> tab((size_t)2 * P);
    if (D->lb) {  // exchange the layout addresses through the group
      nitro_loopback *G = D->lb;
      G->slot[D->rank].send = L->xb[0];
      G->slot[D->rank].recv = L->xb[1];
      G->barrier();
      for (int q = 0; q < P; ++q) {
        tab[q] = (char *)const_cast<void *>(G->slot[q].send) + L->my_off;
        tab[P + q] = (char *)G->slot[q].recv + L->my_off;
      }
      G->barrier();
    } else {  // one rank without a communicator
      tab[0] = (char *)L->xb[0] + L->my_off;
      tab[1] = (char *)L->xb[1] + L->my_off;
    }
    NITRO_CUDA(cudaMemcpy(L->table.p, tab.data(), tab.size() * sizeof(void *), cudaMemcpyHostToDevice));
  }
  // padding entries are read by padded formats (zero slots x padding): keep them finite
  for (int b = 0; b < 2; ++b) NITRO_CUDA(cudaMemset(L->xb[b], 0, bytes));
  NITRO_CUDA(cudaDeviceSynchronize());
  if (D->lb) D->lb->barrier();  // every rank's layouts are zeroed before anyone writes into them
  *out = L;
  return NITRO_OK;
}

void nitro_dist_loop_destroy(nitro_dist_loop *L) {
  if (!L) return;
  cudaSetDevice(L->D->device);
  cudaDeviceSynchronize();
  if (L->devcomm_ok) ncclDevCommDestroy(L->D->comm, &L->devcomm);
  for (int b = 0; b < 2; ++b) {
    if (L->win[b]) ncclCommWindowDeregister(L->D->comm, L->win[b]);
    if (L->nccl_mem && L->xb[b]) ncclMemFree(L->xb[b]);
  }
  delete L;
}

nitro_status_t nitro_dist_loop_x(nitro_dist_loop *L, void **d_x_local) {
  if (!L || !d_x_local) return fail(NITRO_E_INVALID_ARG, "bad argument");
  *d_x_local = (char *)L->xb[L->cur] + L->my_off;
  return NITRO_OK;
}

nitro_status_t nitro_dist_loop_start(nitro_dist_loop *L) {
  if (!L) return fail(NITRO_E_INVALID_ARG, "bad argument");
  NITRO_CUDA(cudaSetDevice(L->D->device));
  cudaStream_t s = L->A->stream;
  char *xb = (char *)L->xb[L->cur];
  NITRO_TRY(dist_allgather(L->D, xb + L->my_off, xb, (size_t)L->st->B * L->sv, s));
  if (L->D->lb) {
    NITRO_CUDA(cudaStreamSynchronize(s));
    L->D->lb->barrier();
  }
  return NITRO_OK;
}

nitro_status_t nitro_dist_loop_step(nitro_dist_loop *L, int variant, void *d_y_local) {
  if (!L || variant < 0 || variant >= NITRO_NUM_VARIANTS) return fail(NITRO_E_INVALID_ARG, "bad argument");
  nitro_dist *D = L->D;
  DistState *st = L->st;
  NITRO_CUDA(cudaSetDevice(D->device));
  cudaStream_t s = L->A->stream;
  const int P = D->nranks, nxt = L->cur ^ 1;
  const void *x = L->xb[L->cur];
  void *const *dst = L->table.as<void *>() + (size_t)nxt * P;
  char *mine_next = (char *)L->xb[nxt] + L->my_off;
  for (int k = 0; k < 3; ++k) {
    nitro_spmv *Pt = st->part[k];
    if (!Pt) continue;
    Pt->stream = s;
    int ok = 0, v = variant;
    NITRO_TRY(nitro_spmv_allowed(Pt, v, &ok));
    if (!ok) v = NITRO_CSR_VECTOR;  // part-level constraint fallback
    char *y = d_y_local ? (char *)d_y_local + (size_t)st->part_begin[k] * L->sv : nullptr;
    if (fusable(v)) {
      NITRO_TRY(nitro_spmv_prepare(Pt, v));
      PeerOut po;
      po.dst = dst;
      po.n = P;
      po.row_off = st->part_begin[k];
      NITRO_TRY(launch_spmv_fused(Pt, v, x, y, po, s));
    } else {
      char *blk = mine_next + (size_t)st->part_begin[k] * L->sv;
      NITRO_TRY(nitro_spmv_run(Pt, v, x, blk));
      const int64_t n = Pt->N;
      const unsigned g = (unsigned)std::max<int64_t>(1, std::min<int64_t>((n + 255) / 256, (int64_t)num_sms() * 8));
      if (P > 1) {
        if (L->A->fp64) k_push<double><<<g, 256, 0, s>>>((const double *)blk, n, dst, st->part_begin[k], P, D->rank);
        else k_push<float><<<g, 256, 0, s>>>((const float *)blk, n, dst, st->part_begin[k], P, D->rank);
        NITRO_CUDA(cudaGetLastError());
      }
      if (y) NITRO_CUDA(cudaMemcpyAsync(y, blk, (size_t)n * L->sv, cudaMemcpyDeviceToDevice, s));
    }
  }
  NITRO_TRY(loop_barrier(L, s));
  L->cur = nxt;
  return NITRO_OK;
}

}  // extern "C"
