// scan.cu — device exclusive scan of int64 counts (used by the converters
// and the feature-offset compaction; not on the SpMV hot path).
// Three passes: tile sums -> single-block scan of tile sums -> tile scans.
#include "nitro_internal.h"
#include "util.cuh"

namespace nitro {
namespace {

constexpr int kThreads = 512;
constexpr int kItems = 8;
constexpr int kTile = kThreads * kItems;

__global__ void __launch_bounds__(kThreads) tile_sums(const int64_t *__restrict__ in, int64_t n,
                                                      int64_t *__restrict__ sums) {
  int64_t base = (int64_t)blockIdx.x * kTile;
  int64_t s = 0;
#pragma unroll
  for (int k = 0; k < kItems; ++k) {
    int64_t i = base + (int64_t)k * kThreads + threadIdx.x;
    if (i < n) s += in[i];
  }
  s = block_sum_i64<kThreads>(s);
  if (threadIdx.x == 0) sums[blockIdx.x] = s;
}

// one block: exclusive scan of sums[0..nt) in place; total -> *total
__global__ void __launch_bounds__(1024) scan_sums(int64_t *sums, int64_t nt, int64_t *total) {
  __shared__ int64_t carry_s;
  if (threadIdx.x == 0) carry_s = 0;
  __syncthreads();
  for (int64_t c0 = 0; c0 < nt; c0 += 1024) {
    int64_t i = c0 + threadIdx.x;
    int64_t v = i < nt ? sums[i] : 0;
    int64_t agg;
    int64_t ex = block_exclusive_i64<1024>(v, agg);
    int64_t carry = carry_s;
    if (i < nt) sums[i] = carry + ex;
    __syncthreads();
    if (threadIdx.x == 0) carry_s = carry + agg;
    __syncthreads();
  }
  if (threadIdx.x == 0) *total = carry_s;
}

__global__ void __launch_bounds__(kThreads) tile_scan(const int64_t *__restrict__ in, int64_t n,
                                                      const int64_t *__restrict__ offs, int64_t *__restrict__ out) {
  int64_t base = (int64_t)blockIdx.x * kTile + (int64_t)threadIdx.x * kItems;  // blocked per thread
  int64_t v[kItems];
  int64_t s = 0;
#pragma unroll
  for (int k = 0; k < kItems; ++k) {
    int64_t i = base + k;
    v[k] = i < n ? in[i] : 0;
    s += v[k];
  }
  int64_t agg;
  int64_t ex = block_exclusive_i64<kThreads>(s, agg);
  int64_t run = offs[blockIdx.x] + ex;
#pragma unroll
  for (int k = 0; k < kItems; ++k) {
    int64_t i = base + k;
    if (i < n) out[i] = run;
    run += v[k];
  }
}

}  // namespace

nitro_status_t exclusive_scan_i64(const int64_t *in, int64_t *out, int64_t n, DevBuf &scratch, cudaStream_t s) {
  int64_t nt = (n + kTile - 1) / kTile;
  if (nt < 1) nt = 1;
  NITRO_TRY(scratch.alloc((size_t)(nt + 1) * sizeof(int64_t)));
  int64_t *sums = scratch.as<int64_t>();
  if (n > 0) tile_sums<<<(unsigned)nt, kThreads, 0, s>>>(in, n, sums);
  else NITRO_CUDA(cudaMemsetAsync(sums, 0, sizeof(int64_t), s));
  scan_sums<<<1, 1024, 0, s>>>(sums, nt, out + n);
  if (n > 0) tile_scan<<<(unsigned)nt, kThreads, 0, s>>>(in, n, sums, out);
  NITRO_CUDA(cudaGetLastError());
  return NITRO_OK;
}

}  // namespace nitro
