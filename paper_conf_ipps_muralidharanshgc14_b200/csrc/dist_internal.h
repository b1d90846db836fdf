// dist_internal.h — shared by dist.cu and dist_loop.cu (not part of the C ABI).
#pragma once
#include <nccl.h>

#include <condition_variable>
#include <mutex>
#include <string>
#include <vector>

#include "nitro_internal.h"

#define NITRO_NCCL(call)                                                                                         \
  do {                                                                                                           \
    ncclResult_t r_ = (call);                                                                                    \
    if (r_ != ncclSuccess) return nitro::fail(NITRO_E_NCCL, std::string("NCCL: ") + ncclGetErrorString(r_) + " at " #call); \
  } while (0)

namespace nitro {
struct Msg {
  int peer;
  const void *src;  // send: source; recv: unused
  void *dst;        // recv: destination; send: unused
  size_t bytes;
};
}  // namespace nitro

struct nitro_loopback {
  int nranks = 1, device = 0;
  std::mutex mu;
  std::condition_variable cv;
  int arrived = 0;
  uint64_t gen = 0;
  struct Slot {
    const void *send = nullptr;
    void *recv = nullptr;
    size_t bytes = 0;
    cudaEvent_t ready = nullptr, done = nullptr;
    std::vector<nitro::Msg> sends;
    std::vector<unsigned long long> host;
  };
  std::vector<Slot> slot;
  void barrier() {
    std::unique_lock<std::mutex> lk(mu);
    const uint64_t g = gen;
    if (++arrived == nranks) {
      arrived = 0;
      ++gen;
      cv.notify_all();
    } else {
      cv.wait(lk, [&] { return gen != g; });
    }
  }
};

struct nitro_dist {
  ncclComm_t comm = nullptr;
  nitro_loopback *lb = nullptr;  // loopback transport (one process, one GPU)
  int rank = 0, nranks = 1, device = 0;
  cudaStream_t comm_stream = nullptr;
  cudaEvent_t ev_x = nullptr, ev_g = nullptr;
  bool has_transport() const { return comm != nullptr || lb != nullptr; }
};


namespace nitro {
enum { kAllGather = 0, kHalo = 1 };

struct DistState {
  nitro_dist *D = nullptr;
  int64_t global_rows = 0, B = 0, n = 0, row_begin = 0, i0 = 0, i1 = 0;
  int mode = kAllGather;
  std::vector<int64_t> bounds;
  DevBuf colmap, rp_part[3], xbuf, flags;
  // halo mode
  int64_t nh = 0, ns = 0, nb = 0;           // halo entries, send entries, halo entries below lo
  std::vector<int64_t> recv_off, send_off;  // [P+1] offsets into the halo / send lists
  DevBuf halo_cols, send_idx, sendbuf;
  nitro_spmv *part[3] = {nullptr, nullptr, nullptr};
  nitro_spmv *feat = nullptr;  // original global columns, for global features
  int64_t part_begin[3] = {0, 0, 0};
  int64_t layout_len() const { return mode == kHalo ? n + nh : (int64_t)D->nranks * B; }
  int64_t x_offset() const { return mode == kHalo ? nb : (int64_t)D->rank * B; }
  // layout index of halo position k (halo mode)
  int64_t halo_dest(int64_t k) const { return k < nb ? k : n + k; }
};


// transport (dist.cu)
nitro_status_t dist_allgather(nitro_dist *D, const void *send, void *recv, size_t bytes, cudaStream_t s);
}  // namespace nitro
