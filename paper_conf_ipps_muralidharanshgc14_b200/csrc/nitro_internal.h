// nitro_internal.h — internal declarations of libnitro (not part of the ABI).
#pragma once

#include <cuda_runtime.h>
#include <vector>
#include <stdint.h>

#include <string>

#include "../../include/nitro.h"
#include <nvtx3/nvToolsExt.h>   // header-only NVTX v3: ranges cost nothing without an attached tool

namespace nitro {

// NVTX range over one C-ABI call (nsys / ncu --nvtx timelines name the phases:
// features, select, train, conversion, multiply, exchange)
struct NvtxRange {
  explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
  NvtxRange(const NvtxRange &) = delete;
  NvtxRange &operator=(const NvtxRange &) = delete;
};
#define NITRO_NVTX(name) ::nitro::NvtxRange nitro_nvtx_range_(name)

// ------------------------------------------------------------------ errors
void set_error(const std::string &msg);
nitro_status_t fail(nitro_status_t code, const std::string &msg);
nitro_status_t cuda_fail(cudaError_t e, const char *where);

#define NITRO_CUDA(call)                                         \
  do {                                                           \
    cudaError_t e_ = (call);                                     \
    if (e_ != cudaSuccess) return ::nitro::cuda_fail(e_, #call); \
  } while (0)
#define NITRO_TRY(call)                           \
  do {                                            \
    nitro_status_t s_ = (call);                   \
    if (s_ != NITRO_OK) return s_;                \
  } while (0)

// ------------------------------------------------------------------ device buffer
struct DevBuf {
  void *p = nullptr;
  size_t bytes = 0;
  nitro_status_t alloc(size_t n);  // (re)allocates if smaller; contents undefined
  void release();
  template <typename T> T *as() const { return reinterpret_cast<T *>(p); }
  ~DevBuf() { release(); }
  DevBuf() = default;
  DevBuf(const DevBuf &) = delete;
  DevBuf &operator=(const DevBuf &) = delete;
};

// ------------------------------------------------------------------ feature pass
// Device-side accumulators of the K1 pass (exact integers).
struct FeatAcc {
  unsigned long long s1, s2, lmax;
  unsigned int bad;      // bit0 rowptr not monotone / wrong ends, bit1 unsorted/dup col, bit2 col out of range
  unsigned int nlong;    // rows deferred to the long-row pass (k_features_long)
  unsigned long long ndiag;
  unsigned int popc_done;  // k_popc blocks finished (the last one copies the sums to the host)
  unsigned int pad_;
};

// ------------------------------------------------------------------ formats
struct EllFmt {
  bool ready = false;
  int64_t K = 0, ld = 0;
  DevBuf col, val;
};
struct DiaFmt {
  bool ready = false;
  int64_t D = 0, ld = 0;
  int64_t inrange = 0;  // sum over diagonals of in-range slots (compulsory)
  int64_t off_min = 0, off_max = 0;
  DevBuf off, val;
};
struct HybFmt {
  bool ready = false;
  int64_t K = 0, ld = 0, Zt = 0, nchunks = 0, tail_rows = 0;
  int W = 8;  // tail windows per chunk
  DevBuf col, val, trow, tcol, tval, carry_row, carry_val;
  // fixup plan (static per matrix): carry slots grouped by row into segments
  // [fix_seg[s], fix_seg[s+1]); segments longer than 32 slots listed in fix_long
  DevBuf fix_seg, fix_long;
  int64_t fix_S = 0, fix_nlong = 0;
};
struct CsrvFmt {
  bool ready = false;
  int V = 32;
  int64_t n_long = 0;
  DevBuf long_rows;
  // nnz-split stream mode (skewed row lengths, K6s): chunks of
  // 32*EP entries, chunk_row[c] = row holding entry c*32*EP (chunk_row[nch] = N),
  // two carry slots per chunk and the static fixup plan (as HybFmt)
  bool stream = false;
  int EP = 8;
  int64_t nch = 0;
  DevBuf chunk_row, carry_row, carry_val, fix_seg, fix_long;
  int64_t fix_S = 0, fix_nlong = 0;
  // hot-x staging (x-locality, the modern "-Tx"): the nhot most referenced
  // columns (power-law matrices) are copied into shared memory per CTA; hcol
  // = the column ids with a hot column c replaced by ~slot (negative)
  int64_t nhot = 0;
  double hot_share = 0.0;  // fraction of the nonzeros whose column is hot
  DevBuf hot_cols, hcol;
};

}  // namespace nitro

struct nitro_spmv {
  int device = 0;
  cudaStream_t stream = nullptr;
  int64_t N = 0, M = 0, Z = 0;
  int64_t row0 = 0;  // global row of local row 0 (multi-GPU blocks), for diagonal offsets
  const void *rowptr = nullptr;
  bool rp64 = false;
  const int32_t *col = nullptr;
  const void *val = nullptr;
  bool fp64 = false;

  // features
  bool feat_ready = false, feat_pending = false;
  nitro_spmv_feat feat{};
  nitro::DevBuf feat_acc;   // FeatAcc
  nitro::DevBuf bitmap;     // u32 words over offsets [-(N-1) .. M-1] (+row0 shift)
  nitro::DevBuf feat_long;  // int32 row ids of the rows longer than the feature pass's kLong
  nitro::DevBuf offsets;    // int32 [ndiag] ascending
  nitro::DevBuf scratch;    // scan scratch
  nitro::FeatAcc *h_acc = nullptr;  // pinned, mapped: written by k_popc's last block (no D2H copy)
  nitro::FeatAcc *h_acc_dev = nullptr;  // its device address
  cudaEvent_t feat_done = nullptr;

  double budget = -1.0;
  int csr_impl = 0;  // NITRO_CSR_IMPL_*

  nitro::EllFmt ell;
  nitro::DiaFmt dia;
  nitro::HybFmt hyb;
  nitro::CsrvFmt csrv;

  nitro::DevBuf flush;      // L2 flush scratch
  nitro::DevBuf xbuf, ybuf; // run_host staging
  // run_host row-chunk pipeline (H2D of x / multiply / D2H of y on three streams)
  cudaStream_t s_in = nullptr, s_out = nullptr;
  std::vector<cudaEvent_t> ev_pipe;
  bool xhi_ready = false;            // csr_xhi valid (cleared by invalidate)
  std::vector<int64_t> csr_xhi;      // per run_host chunk: 1 + max column of the rows before its end

  // multi-GPU (dist.cu)
  int64_t feat_G = -1;      // bitmap offset shift override (global-offset bitmaps); -1 = row0 + N - 1
  nitro_dist *dist = nullptr;
  void *dist_state = nullptr;
  void (*dist_free)(void *) = nullptr;
};

namespace nitro {

// features.cu
nitro_status_t features_launch(nitro_spmv *A);   // enqueue K1 + compaction, async
nitro_status_t features_finish(nitro_spmv *A);   // wait + host finishing
nitro_status_t row_features(nitro_spmv *A, nitro_spmv_feat *out);  // rowptr-only level, syncs
void finish_features(int64_t N, int64_t M, int64_t Z, uint64_t s1, uint64_t s2, int64_t lmax, int64_t D,
                     nitro_spmv_feat *f);

// convert.cu
nitro_status_t prepare_ell(nitro_spmv *A);
nitro_status_t prepare_dia(nitro_spmv *A);
nitro_status_t prepare_hyb(nitro_spmv *A);
nitro_status_t prepare_csrv(nitro_spmv *A);

// spmv.cu
nitro_status_t launch_spmv(nitro_spmv *A, int variant, const void *x, void *y, cudaStream_t s);
// Fused y -> x epilogue of the solver-loop mode: every
// computed y_i (local row i of this launch) is also stored at element
// row_off + i of each of the n destination arrays dst[q] (device array of
// device pointers: each rank's next-x layout at this rank's block; peer
// memory through NCCL symmetric windows, or loopback buffers).
struct PeerOut {
  void *const *dst = nullptr;
  int n = 0;
  int64_t row_off = 0;
};
// CSR-scalar, ELL and DIA only (NITRO_E_UNSUPPORTED otherwise); y may be NULL
// (peer stores only).
nitro_status_t launch_spmv_fused(nitro_spmv *A, int variant, const void *x, void *y, const PeerOut &po,
                                 cudaStream_t s);
// rows [r0, r1) only (CSR-scalar, ELL, DIA: row-separable launches; r0 a multiple of 32)
nitro_status_t launch_spmv_rows(nitro_spmv *A, int variant, const void *x, void *y, cudaStream_t s, int64_t r0,
                                int64_t r1);
// per-chunk maximum column + 1 of the rows below each chunk end (run_host pipeline)
nitro_status_t csr_chunk_xhi(nitro_spmv *A, const std::vector<int64_t> &ends, std::vector<int64_t> &xhi);
int launches_of(const nitro_spmv *A, int variant);
nitro_status_t launch_flush(nitro_spmv *A, cudaStream_t s);
// spmv_dia_tma.cu: DIA with TMA-streamed diagonal slabs
double compulsory_bytes(const nitro_spmv *A, int variant);

// scan.cu: exclusive scan of int64 counts; out[n] = total.  scratch grows.
nitro_status_t time_variant(nitro_spmv *A, int variant, const void *d_x, void *d_y, int warmup, int reps,
                            int flush_l2, double cutoff_s, double *out_median_s, double *out_all, int *out_reps);
nitro_status_t exclusive_scan_i64(const int64_t *in, int64_t *out, int64_t n, DevBuf &scratch, cudaStream_t s);

inline int64_t round_up(int64_t n, int64_t m) { return (n + m - 1) / m * m; }
constexpr int64_t kCsrvSeg = 256;  // CSR-vector long-row segment (one warp, 8 entries per lane)
// HYB tail chunk = 32 * W entries per warp; W = 8 (fp32) / 4 (fp64: registers),
// NITRO_HYB_W overrides (2/4/8).  Fixed per matrix at prepare time.
int hyb_windows(size_t sv);
// CSR-vector mode: the nnz-split stream kernel (K6s) for skewed row lengths
// (row-length SD above the mean); NITRO_CSRV_STREAM=0/1 forces it off/on.
bool csrv_stream_mode(const nitro_spmv *A);
bool csrv_vec_mode(const nitro_spmv *A);   // K6v (convert.cu)
constexpr bool kCsrvVecDefault = true;      // AUTO picks K6v (B200 A/B)
bool csrv_hot_on();
bool csrv_hot_forced();
int csrv_hot_kb();
// bitmap index of diagonal offset d is d + G; the bitmap spans G + M bits
inline int64_t diag_shift(const nitro_spmv *A) { return A->feat_G >= 0 ? A->feat_G : A->row0 + A->N - 1; }
int num_sms();

}  // namespace nitro
