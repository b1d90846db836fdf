// spmv_dia_tma.cu — K8': DIA SpMV with the diagonal slabs streamed by TMA.
//
// The DIA values are the only large stream (x mostly hits L1/L2).  Instead of
// every thread issuing 16-byte loads, one thread per CTA issues 1D bulk copies
// (cp.async.bulk, SASS UBLKCP) of whole slabs — the tile's 1024-row piece of
// GD diagonals — into a STAGES-deep shared-memory ring tracked by mbarriers,
// so ~48 KB per CTA (x 3 CTAs per SM) of HBM traffic is in flight with almost
// no issue cost.  Threads then read their 4 rows of each slab from shared
// memory (one conflict-free 16-byte LDS per diagonal), gather x through L1,
// and accumulate as the LDG kernel does (fp32 partials per group, fp64 sum).
// Persistent CTAs walk (tile, diagonal-group) pairs round-robin over tiles.
#include "nitro_internal.h"
#include "tma.cuh"
#include "util.cuh"

namespace nitro {
namespace {

constexpr int kThr = 256;
constexpr int kRows = 4 * kThr;  // rows per tile
constexpr int kStages = 4;
constexpr int kStageBytes = 16384;

template <typename VT>
__global__ void __launch_bounds__(kThr) k_dia_tma(const int32_t *__restrict__ offs, const VT *__restrict__ dval,
                                                  const VT *__restrict__ x, VT *__restrict__ y, int64_t N, int64_t M,
                                                  int64_t D, int64_t ld, int64_t row0, int64_t off_min,
                                                  int64_t off_max) {
  constexpr int GD = kStageBytes / (kRows * (int)sizeof(VT));  // diagonals per stage
  extern __shared__ __align__(128) unsigned char smem[];
  VT *ring = reinterpret_cast<VT *>(smem);                     // [kStages][GD][kRows]
  __shared__ __align__(8) uint64_t full[kStages];
  const int tid = threadIdx.x;
  const int64_t ntiles = (ld + kRows - 1) / kRows;
  const int64_t my_tiles = blockIdx.x < ntiles ? (ntiles - 1 - blockIdx.x) / gridDim.x + 1 : 0;
  const int ng = (int)((D + GD - 1) / GD);
  const int64_t Q = my_tiles * ng;
  if (tid == 0) {
    for (int s = 0; s < kStages; ++s) mbar_init(&full[s], 1);
    fence_mbar_init();
  }
  __syncthreads();
  auto issue = [&](int64_t q) {
    const int s = (int)(q % kStages);
    const int64_t tile = blockIdx.x + (q / ng) * gridDim.x;
    const int g = (int)(q % ng);
    const int64_t B0 = tile * kRows;
    const int64_t nrows = ld - B0 < kRows ? ld - B0 : kRows;
    const int nd = (int)(D - (int64_t)g * GD < GD ? D - (int64_t)g * GD : GD);
    const uint32_t bytes = (uint32_t)(nrows * sizeof(VT));
    mbar_arrive_expect_tx(&full[s], bytes * nd);
    for (int j = 0; j < nd; ++j)
      bulk_g2s(ring + ((size_t)s * GD + j) * kRows, dval + ((int64_t)g * GD + j) * ld + B0, bytes, &full[s]);
  };
  if (tid == 0)
    for (int64_t q = 0; q < Q && q < kStages; ++q) issue(q);
  // x values of stage qq for this thread's 4 rows (L1/L2 gathers)
  auto gather = [&](int64_t qq, VT (&xo)[GD][4]) {
    const int64_t tl = blockIdx.x + (qq / ng) * gridDim.x;
    const int gg = (int)(qq % ng);
    const int64_t b0 = tl * kRows, ii = b0 + 4 * tid;
    const int64_t be = (b0 + kRows < ld ? b0 + kRows : ld) - 1;
    const bool inter = row0 + b0 + off_min >= 0 && row0 + be + off_max < M;
    const int ndd = (int)(D - (int64_t)gg * GD < GD ? D - (int64_t)gg * GD : GD);
#pragma unroll
    for (int j = 0; j < GD; ++j) {
      const bool live = j < ndd && ii < ld;
      const int64_t jx = row0 + ii + (live ? __ldg(offs + (int64_t)gg * GD + j) : 0);
#pragma unroll
      for (int t = 0; t < 4; ++t)
        xo[j][t] = (live && (inter || (jx + t >= 0 && jx + t < M))) ? __ldg(x + jx + t) : (VT)0;
    }
  };
  VT xcur[GD][4];
  if (Q > 0) gather(0, xcur);
  double acc[4] = {0.0, 0.0, 0.0, 0.0};
  for (int64_t q = 0; q < Q; ++q) {
    const int s = (int)(q % kStages);
    const int64_t tile = blockIdx.x + (q / ng) * gridDim.x;
    const int g = (int)(q % ng);
    const int64_t B0 = tile * kRows;
    const int64_t i0 = B0 + 4 * tid;
    const int64_t Bend = (B0 + kRows < ld ? B0 + kRows : ld) - 1;
    const bool interior = row0 + B0 + off_min >= 0 && row0 + Bend + off_max < M;
    const int nd = (int)(D - (int64_t)g * GD < GD ? D - (int64_t)g * GD : GD);
    (void)interior;
    // the x gathers do not depend on the TMA data: issue the next stage's now
    VT xnext[GD][4];
    if (q + 1 < Q) gather(q + 1, xnext);
    mbar_wait(&full[s], (uint32_t)((q / kStages) & 1));
    if (i0 < ld) {
      VT v[GD][4];
#pragma unroll
      for (int j = 0; j < GD; ++j) {
        if (j < nd) {
          const VT *sp = ring + ((size_t)s * GD + j) * kRows + 4 * tid;
          if constexpr (sizeof(VT) == 4) {
            const float4 t = *reinterpret_cast<const float4 *>(sp);
            v[j][0] = t.x; v[j][1] = t.y; v[j][2] = t.z; v[j][3] = t.w;
          } else {
            const double2 t0 = reinterpret_cast<const double2 *>(sp)[0];
            const double2 t1 = reinterpret_cast<const double2 *>(sp)[1];
            v[j][0] = t0.x; v[j][1] = t0.y; v[j][2] = t1.x; v[j][3] = t1.y;
          }
        } else {
#pragma unroll
          for (int t = 0; t < 4; ++t) v[j][t] = (VT)0;
        }
      }
      VT part[4] = {0, 0, 0, 0};
#pragma unroll
      for (int j = 0; j < GD; ++j)
#pragma unroll
        for (int t = 0; t < 4; ++t) part[t] = fma(v[j][t], xcur[j][t], part[t]);
#pragma unroll
      for (int t = 0; t < 4; ++t) acc[t] += (double)part[t];
      if (g == ng - 1) {  // tile complete
        if (i0 + 3 < N && ((reinterpret_cast<uintptr_t>(y + i0) & 15) == 0)) {
          if constexpr (sizeof(VT) == 4) {
            *reinterpret_cast<float4 *>(y + i0) =
                make_float4((float)acc[0], (float)acc[1], (float)acc[2], (float)acc[3]);
          } else {
            reinterpret_cast<double2 *>(y + i0)[0] = make_double2(acc[0], acc[1]);
            reinterpret_cast<double2 *>(y + i0)[1] = make_double2(acc[2], acc[3]);
          }
        } else {
          for (int t = 0; t < 4; ++t)
            if (i0 + t < N) y[i0 + t] = (VT)acc[t];
        }
#pragma unroll
        for (int t = 0; t < 4; ++t) acc[t] = 0.0;
      }
    }
    __syncthreads();  // stage s fully consumed
    if (tid == 0 && q + kStages < Q) issue(q + kStages);
#pragma unroll
    for (int j = 0; j < GD; ++j)
#pragma unroll
      for (int t = 0; t < 4; ++t) xcur[j][t] = xnext[j][t];
  }
}

}  // namespace

nitro_status_t launch_dia_tma(nitro_spmv *A, const void *x, void *y, cudaStream_t s) {
  const size_t smem = (size_t)kStages * kStageBytes;
  const int64_t ntiles = (A->dia.ld + kRows - 1) / kRows;
  int64_t grid = (int64_t)num_sms() * 3;
  if (grid > ntiles) grid = ntiles;
  if (grid < 1) grid = 1;
  if (A->fp64) {
    static bool attr = false;
    if (!attr) {
      NITRO_CUDA(cudaFuncSetAttribute(k_dia_tma<double>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
      attr = true;
    }
    k_dia_tma<double><<<(unsigned)grid, kThr, smem, s>>>(A->dia.off.as<int32_t>(), A->dia.val.as<double>(),
                                                        (const double *)x, (double *)y, A->N, A->M, A->dia.D,
                                                        A->dia.ld, A->row0, A->dia.off_min, A->dia.off_max);
  } else {
    static bool attr = false;
    if (!attr) {
      NITRO_CUDA(cudaFuncSetAttribute(k_dia_tma<float>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
      attr = true;
    }
    k_dia_tma<float><<<(unsigned)grid, kThr, smem, s>>>(A->dia.off.as<int32_t>(), A->dia.val.as<float>(),
                                                       (const float *)x, (float *)y, A->N, A->M, A->dia.D, A->dia.ld,
                                                       A->row0, A->dia.off_min, A->dia.off_max);
  }
  NITRO_CUDA(cudaGetLastError());
  return NITRO_OK;
}

}  // namespace nitro
