// spmv.cu — A6-A10: the five SpMV variants y = A.x for sm_100a (CUDA cores;
// SpMV is HBM-bound, ~0.2 flop/byte, so tensor cores do not apply).
//
// Semantics (read as y <- A.x): every variant overwrites y.
// Accumulation (R2): fp64 data accumulate in fp64.  fp32 data form
// fp32 partial sums of at most 16 terms (FFMA), combined in fp64 (or in a
// <=5-level fp32 shuffle tree for rows of <= 8V entries), so the error stays
// below ~21 u sum|a_ij x_j| (u = 2^-24) for any row length: inside the
// 1e-5 bound of the north star, and exact on integer stencils.
#include "nitro_internal.h"
#include "tma.cuh"
#include "util.cuh"

#include <algorithm>

namespace nitro {
namespace {

template <typename VT> struct V4;
template <> struct V4<float> {
  float v[4];
  __device__ __forceinline__ void load(const float *p) {
    float4 t = ld_stream_f4(reinterpret_cast<const float4 *>(p));
    v[0] = t.x; v[1] = t.y; v[2] = t.z; v[3] = t.w;
  }
  __device__ __forceinline__ void load(const float *p, uint64_t pol) {
    float4 t = ld_stream_f4(reinterpret_cast<const float4 *>(p), pol);
    v[0] = t.x; v[1] = t.y; v[2] = t.z; v[3] = t.w;
  }
};
template <> struct V4<double> {
  double v[4];
  __device__ __forceinline__ void load(const double *p) {
    double2 a = ld_stream_d2(reinterpret_cast<const double2 *>(p));
    double2 b = ld_stream_d2(reinterpret_cast<const double2 *>(p) + 1);
    v[0] = a.x; v[1] = a.y; v[2] = b.x; v[3] = b.y;
  }
  __device__ __forceinline__ void load(const double *p, uint64_t pol) {
    double2 a = ld_stream_d2(reinterpret_cast<const double2 *>(p), pol);
    double2 b = ld_stream_d2(reinterpret_cast<const double2 *>(p) + 1, pol);
    v[0] = a.x; v[1] = a.y; v[2] = b.x; v[3] = b.y;
  }
};

template <typename VT>
__device__ __forceinline__ void store4(VT *y, int64_t i0, int64_t N, const double *acc) {
  // vector store only when y + i0 is 16-byte aligned (y may be a row-offset view)
  if (i0 + 3 < N && ((reinterpret_cast<uintptr_t>(y + i0) & 15) == 0)) {
    if constexpr (sizeof(VT) == 4) {
      *reinterpret_cast<float4 *>(y + i0) = make_float4((float)acc[0], (float)acc[1], (float)acc[2], (float)acc[3]);
    } else {
      reinterpret_cast<double2 *>(y + i0)[0] = make_double2(acc[0], acc[1]);
      reinterpret_cast<double2 *>(y + i0)[1] = make_double2(acc[2], acc[3]);
    }
  } else {
    for (int q = 0; q < 4; ++q)
      if (i0 + q < N) y[i0 + q] = (VT)acc[q];
  }
}

// y stores of a launch, optionally fused with the f3 (ii) peer stores (FUSED:
// each value also goes to element row_off + i of every dst[q]; y may be NULL)
template <bool FUSED, typename VT>
__device__ __forceinline__ void out1(VT *y, const PeerOut &po, int64_t i, VT v) {
  if (!FUSED || y) y[i] = v;
  if constexpr (FUSED)
    for (int q = 0; q < po.n; ++q) reinterpret_cast<VT *>(po.dst[q])[po.row_off + i] = v;
}
template <bool FUSED, typename VT>
__device__ __forceinline__ void out4(VT *y, const PeerOut &po, int64_t i0, int64_t N, const double *acc) {
  if (!FUSED || y) store4<VT>(y, i0, N, acc);
  if constexpr (FUSED)
    for (int q = 0; q < po.n; ++q) store4<VT>(reinterpret_cast<VT *>(po.dst[q]) + po.row_off, i0, N, acc);
}

// ------------------------------------------------------------------ K5 CSR-scalar
// Row arithmetic shared by every CSR-scalar implementation (R2):
// fp32 (fp64) FFMA partials over 16-term chunks counted from the row start,
// summed in fp64.  The first H entries of a row arrive as one predicated batch
// (all loads issued before the first gather), so rows of <= H entries — this
// variant's class — cost one load round trip; H only changes load batching,
// never the result.
template <int H, typename VT, typename XI = int64_t, typename LC, typename LV>
__device__ __forceinline__ double csr_row(XI a, XI b, const VT *__restrict__ x, LC ldc, LV ldv) {
  static_assert(H <= 16, "head batch must lie in the first 16-term chunk");
  int c[H];
  VT v[H];
#pragma unroll
  for (int k = 0; k < H; ++k) {
    const bool in = a + k < b;
    c[k] = in ? ldc(a + k) : -1;
    v[k] = in ? ldv(a + k) : (VT)0;
  }
  VT xv[H];
#pragma unroll
  for (int k = 0; k < H; ++k) xv[k] = c[k] >= 0 ? __ldg(x + c[k]) : (VT)0;
  VT part = 0;
#pragma unroll
  for (int k = 0; k < H; ++k) part = fma(v[k], xv[k], part);
  const XI e0 = a + 16 < b ? a + 16 : b;
  for (XI k = a + H; k < e0; ++k) part = fma(ldv(k), __ldg(x + ldc(k)), part);
  double acc = (double)part;
  for (XI k = a + 16; k < b; k += 16) {
    const XI e = k + 16 < b ? k + 16 : b;
    VT p2 = 0;
#pragma unroll 4
    for (XI j = k; j < e; ++j) p2 = fma(ldv(j), __ldg(x + ldc(j)), p2);
    acc += (double)p2;
  }
  return acc;
}

template <int H, typename IT, typename VT, bool FUSED = false>
__global__ void __launch_bounds__(256) k_csr_scalar(const IT *__restrict__ rowptr, const int32_t *__restrict__ col,
                                                    const VT *__restrict__ val, const VT *__restrict__ x,
                                                    VT *__restrict__ y, int64_t N, const PeerOut po = PeerOut{}) {
  // thread per row ("CSR": one thread walks one row)
  if constexpr (sizeof(VT) == 4) {
    // fp32: row-rebased pointers and 32-bit offsets (the kernel is issue-bound;
    // same FMA sequence, so y is bit-identical to the 64-bit-offset form)
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < N; i += (int64_t)gridDim.x * blockDim.x) {
      const int64_t a = (int64_t)rowptr[i];
      const int32_t *cp = col + a;
      const VT *vp = val + a;
      auto ldc = [&](int e) { return __ldg(cp + e); };
      auto ldv = [&](int e) { return __ldg(vp + e); };
      out1<FUSED, VT>(y, po, i, (VT)csr_row<H, VT, int>(0, (int)((int64_t)rowptr[i + 1] - a), x, ldc, ldv));
    }
  } else {
    auto ldc = [&](int64_t e) { return __ldg(col + e); };
    auto ldv = [&](int64_t e) { return __ldg(val + e); };
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < N; i += (int64_t)gridDim.x * blockDim.x)
      out1<FUSED, VT>(y, po, i, (VT)csr_row<H, VT>((int64_t)rowptr[i], (int64_t)rowptr[i + 1], x, ldc, ldv));
  }
}

// Transposed reduction of R per-lane values (one per row) over groups of V
// lanes: log2(R) exchange steps halve the value count (R-1 shuffles), then
// log2(V/R) plain butterfly steps.  Lane li returns the total of row ridx;
// the lanes with li % (V/R) == 0 hold distinct rows.
template <int V, int R, typename VT>
__device__ __forceinline__ VT reduce_transpose(VT (&p)[R], int li, int &ridx) {
  ridx = 0;
#pragma unroll
  for (int n = R, o = V / 2; n > 1; n >>= 1, o >>= 1) {
    const bool h = li & o;
#pragma unroll
    for (int j = 0; j < n / 2; ++j) {
      const VT keep = h ? p[j + n / 2] : p[j];
      const VT send = h ? p[j] : p[j + n / 2];
      p[j] = keep + __shfl_xor_sync(kFull, send, o);
    }
    ridx = ridx * 2 + (h ? 1 : 0);
  }
  VT t = p[0];
#pragma unroll
  for (int o = V / (2 * R); o > 0; o >>= 1) t += __shfl_xor_sync(kFull, t, o);
  return t;
}

// ------------------------------------------------------------------ K6 CSR-vector
// V lanes per row.  A warp takes 32 consecutive rows (one coalesced rowptr
// load per lane); lane group g handles rows g, g+G, ... (G = 32/V) R at a
// time so R independent (col, val) -> x chains are in flight per lane.
// Rows longer than 8V are split into kCsrvSeg (= 256)-entry segments, each
// reduced by one whole warp (8 entries per lane, all loads issued first); every
// warp first works through the segment list (grid-stride), then through row
// tiles.  A multi-segment row's partials are summed in segment order by the
// last warp to finish one of its segments (deterministic, no float atomics).
template <typename IT, typename VT>
__device__ __forceinline__ void csrv_segments(const IT *__restrict__ rowptr, const int32_t *__restrict__ col,
                                              const VT *__restrict__ val, const VT *__restrict__ x,
                                              VT *__restrict__ y, int64_t nseg, const int32_t *__restrict__ seg_row,
                                              const int32_t *__restrict__ seg_k, double *seg_part,
                                              unsigned *seg_ctr, uint64_t pol) {
  {
    constexpr int64_t S = kCsrvSeg;
    const int lane = threadIdx.x & 31;
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t sg = gw; sg < nseg; sg += nw) {
      const int64_t row = seg_row[sg], k = seg_k[sg];
      const int64_t a = (int64_t)rowptr[row], b = (int64_t)rowptr[row + 1];
      const int64_t st = a + k * S, en = st + S < b ? st + S : b;
      int c[8];
      VT v[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int64_t e = st + u * 32 + lane;
        c[u] = e < en ? ld_stream_i(col + e, pol) : -1;
        v[u] = e < en ? ld_stream(val + e, pol) : (VT)0;
      }
      VT part = 0;
#pragma unroll
      for (int u = 0; u < 8; ++u) part = fma(v[u], c[u] >= 0 ? __ldg(x + c[u]) : (VT)0, part);
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) part += __shfl_xor_sync(kFull, part, o);
      const int64_t ns = (b - a + S - 1) / S;
      if (lane == 0) {
        if (ns == 1) {
          y[row] = part;
        } else {
          seg_part[sg] = (double)part;
          __threadfence();
          const int64_t first = sg - k;
          const unsigned done = atomicAdd(seg_ctr + first, 1u);
          if (done == (unsigned)(ns - 1)) {
            __threadfence();
            double tot = 0.0;
            for (int64_t q = 0; q < ns; ++q) tot += *((volatile double *)(seg_part + first + q));
            y[row] = (VT)tot;
            seg_ctr[first] = 0;  // re-arm for the next multiply
          }
        }
      }
    }
  }
}

// Resident CTAs per SM (launch bounds): occupancy beat per-lane depth in every
// B200 sweep (issuing the remainder batch a stage ahead: c1 4041 -> 3539 GB/s);
// fp64 R = 2: 5 CTAs (c2b 1257 -> 1568 GB/s; fp32 loses with 5: c1 4036 -> 3140)
template <int V, int R, int kB, typename VT>
constexpr int csrv_min_blocks() {
  return R * kB >= 16 ? 2 : R * kB >= 12 ? (sizeof(VT) == 4 ? 3 : 2) : (sizeof(VT) == 4 ? 4 : 5);
}

template <int V, int R, int kB, typename IT, typename VT>
__global__ void __launch_bounds__(256, csrv_min_blocks<V, R, kB, VT>()) k_csr_vector(const IT *__restrict__ rowptr, const int32_t *__restrict__ col,
                                                    const VT *__restrict__ val, const VT *__restrict__ x,
                                                    VT *__restrict__ y, int64_t N, int64_t nseg,
                                                    const int32_t *__restrict__ seg_row,
                                                    const int32_t *__restrict__ seg_k, double *seg_part,
                                                    unsigned *seg_ctr, bool l2ef) {
  constexpr int64_t T = 8 * V;
  const uint64_t pol = l2_policy(l2ef);
  csrv_segments<IT, VT>(rowptr, col, val, x, y, nseg, seg_row, seg_k, seg_part, seg_ctr, pol);
  // Software-pipelined main path.  A "stage" is R rows of one lane group:
  // row starts/lengths come from the tile's rowptr registers by shuffle, and
  // the (col, val) loads of the NEXT stage are issued before the current
  // stage's x gathers and reduction, so loads stay in flight continuously;
  // the rowptr of the tile after the next is prefetched one tile ahead.
  constexpr int G = 32 / V;
  static_assert(R <= V && (R & (R - 1)) == 0, "R rows per stage: a power of two <= V");
  const int lane = threadIdx.x & 31, g = lane / V, li = lane % V;
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t stride = (((int64_t)gridDim.x * blockDim.x) >> 5) * 32;
  int64_t t0 = warp * 32;
  if (t0 >= N) return;
  struct Tile { int64_t abase; int rel, len; };
  struct Stage { int s[R], l[R]; unsigned longmask; int c[R]; VT v[R]; };
  auto load_rp = [&](int64_t tt, int64_t &a, int64_t &L) {
    const int64_t r = tt + lane;
    a = 0; L = 0;
    if (r < N) { a = (int64_t)rowptr[r]; L = (int64_t)rowptr[r + 1] - a; }
  };
  auto make_tile = [&](int64_t a, int64_t L) {
    Tile t;
    t.abase = __shfl_sync(kFull, a, 0);
    t.rel = (int)(a - t.abase);  // 32-bit within a tile of short rows
    t.len = L > T ? -1 : (int)L; // -1: long row, handled by the segment path
    return t;
  };
  // fp32: per-stage 64-bit bases and 32-bit offsets per load (one IMAD.WIDE
  // per load instead of a 64-bit add chain — the kernel is issue-bound: B200
  // c1 4036 -> 4337 GB/s, 1D 3-pt 2106 -> 2416, band01 2878 -> 3143); fp64
  // keeps the 64-bit offsets (R-MAT c2b 1563 -> 1414 with the rebased form)
  auto ldcol = [&](const Tile &t, const int32_t *cb, int s0, int m) {
    if constexpr (sizeof(VT) == 4) return ld_stream_i(cb + (s0 + m), pol);
    else return ld_stream_i(col + t.abase + s0 + m, pol);
  };
  auto ldval = [&](const Tile &t, const VT *vb, int s0, int m) {
    if constexpr (sizeof(VT) == 4) return ld_stream(vb + (s0 + m), pol);
    else return ld_stream(val + t.abase + s0 + m, pol);
  };
  auto issue = [&](const Tile &t, int tb, Stage &st) {
    const int32_t *cb = col + t.abase;
    const VT *vb = val + t.abase;
    st.longmask = 0;
#pragma unroll
    for (int u = 0; u < R; ++u) {
      const int src = g + G * (tb + u);
      st.s[u] = __shfl_sync(kFull, t.rel, src);
      st.l[u] = __shfl_sync(kFull, t.len, src);
      if (st.l[u] < 0) { st.longmask |= 1u << u; st.l[u] = 0; }
    }
#pragma unroll
    for (int u = 0; u < R; ++u) {
      const bool in = li < st.l[u];
      st.c[u] = in ? ldcol(t, cb, st.s[u], li) : -1;
      st.v[u] = in ? ldval(t, vb, st.s[u], li) : (VT)0;
    }
  };
  auto finish = [&](const Tile &t, int64_t tt, int tb, Stage &st) {
    const int32_t *cb = col + t.abase;
    const VT *vb = val + t.abase;
    VT part[R];
#pragma unroll
    for (int u = 0; u < R; ++u) part[u] = st.c[u] >= 0 ? st.v[u] * __ldg(x + st.c[u]) : (VT)0;
    // rows of V+1 .. 8V entries: <= 7 more terms per lane.  The next kB
    // terms of all R rows are loaded as one predicated batch (every load
    // before the first gather; kB = 3 covers rows of <= 4V entries, kB = 7
    // all rows of the short path), further terms in a loop; summed in m order.
    {
      int cm[R][kB];
      VT vm[R][kB];
#pragma unroll
      for (int u = 0; u < R; ++u)
#pragma unroll
        for (int q = 0; q < kB; ++q) {
          const int m = V * (q + 1) + li;
          const bool in = m < st.l[u];
          cm[u][q] = in ? ldcol(t, cb, st.s[u], m) : -1;
          vm[u][q] = in ? ldval(t, vb, st.s[u], m) : (VT)0;
        }
#pragma unroll
      for (int u = 0; u < R; ++u)
#pragma unroll
        for (int q = 0; q < kB; ++q)
          if (cm[u][q] >= 0) part[u] = fma(vm[u][q], __ldg(x + cm[u][q]), part[u]);
    }
#pragma unroll
    for (int u = 0; u < R; ++u)
      for (int m = V * (kB + 1) + li; m < st.l[u]; m += V)
        part[u] = fma(ldval(t, vb, st.s[u], m), __ldg(x + ldcol(t, cb, st.s[u], m)),
                      part[u]);
    int ridx;
    const VT tot = reduce_transpose<V, R>(part, li, ridx);
    const int64_t row = tt + g + G * (tb + ridx);
    if (li % (V / R) == 0 && row < N && !((st.longmask >> ridx) & 1u)) y[row] = tot;
  };
  int64_t pa, pL;  // prefetched rowptr data of the next tile
  int64_t a0, L0;
  load_rp(t0, a0, L0);
  load_rp(t0 + stride, pa, pL);
  Tile cur = make_tile(a0, L0);
  int tb = 0;
  Stage st;
  issue(cur, tb, st);
  for (;;) {
    int ntb = tb + R;
    int64_t nt0 = t0;
    Tile nxt = cur;
    if (ntb >= V) {
      ntb = 0;
      nt0 = t0 + stride;
      if (nt0 < N) {
        nxt = make_tile(pa, pL);
        load_rp(nt0 + stride, pa, pL);
      }
    }
    const bool more = nt0 < N;
    Stage ns;
    if (more) issue(nxt, ntb, ns);
    finish(cur, t0, tb, st);
    if (!more) break;
    st = ns;
    cur = nxt;
    t0 = nt0;
    tb = ntb;
  }
}

// ------------------------------------------------------------------ K6v CSR-vector, vector-load mode
// Rows of similar length (row-length SD <= mean, so no stream mode) and a
// bounded longest row: V lanes per row (V = mean / 4 rounded to a power of
// two, as K6), each lane taking 4 CONSECUTIVE entries per step with one
// 128-bit column load and one 4-wide value load from the row's 16-byte
// aligned base (entries of the neighbouring rows in the first and last chunk
// masked: their x gathers are predicated off and their values zeroed), so a
// row of L entries costs ceil(((a mod 4) + L) / 4V) steps — one for the
// interior rows of a 27-point stencil at V = 8.  Two rows per lane group in
// flight (R = 2: both rows' loads issued before either's gathers).  Sums in
// VT by fma in entry order per lane, then a butterfly over the V lanes.
// The last partial chunk of the arrays (Z not a multiple of 4) is read entry
// by entry (no read past nnz).
template <int V, typename IT, typename VT>
__global__ void __launch_bounds__(256) k_csr_vec4(const IT *__restrict__ rowptr, const int32_t *__restrict__ col,
                                                  const VT *__restrict__ val, const VT *__restrict__ x,
                                                  VT *__restrict__ y, int64_t N, int64_t Z, bool l2ef) {
  constexpr int G = 32 / V;
#ifndef NITRO_K6V_R
#define NITRO_K6V_R 2
#endif
  constexpr int R = (sizeof(VT) == 4 && V >= NITRO_K6V_R) ? NITRO_K6V_R : 2;
  static_assert(V >= 2 && V <= 32 && V % R == 0, "V");
  const uint64_t pol = l2_policy(l2ef);
  const int lane = threadIdx.x & 31, g = lane / V, li = lane % V;
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarp = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t t0 = warp * 32; t0 < N; t0 += nwarp * 32) {
    const int64_t r = t0 + lane;
    int64_t ra = 0, rb = 0;
    if (r < N) { ra = (int64_t)rowptr[r]; rb = (int64_t)rowptr[r + 1]; }
    const int64_t base = __shfl_sync(kFull, ra, 0) & ~(int64_t)3;  // 16-byte aligned tile base
    const int rel_a = (int)(ra - base), rel_b = (int)(rb - base);   // < 2^31: bounded rows (launch rule)
    const int32_t *cb = col + base;
    const VT *vb = val + base;
    const int zrel = Z - base < (int64_t)INT32_MAX ? (int)(Z - base) : INT32_MAX;
#pragma unroll 1
    for (int q = 0; q < V; q += R) {
      int sa[R], sb[R], e0[R];
      int nst = 0;
#pragma unroll
      for (int u = 0; u < R; ++u) {
        const int src = g + G * (q + u);
        sa[u] = __shfl_sync(kFull, rel_a, src);
        sb[u] = __shfl_sync(kFull, rel_b, src);
        e0[u] = (sa[u] & ~3) + 4 * li;
        const int steps = sb[u] > (sa[u] & ~3) ? (sb[u] - (sa[u] & ~3) + 4 * V - 1) / (4 * V) : 0;
        nst = steps > nst ? steps : nst;
      }
      VT part[R];
#pragma unroll
      for (int u = 0; u < R; ++u) part[u] = (VT)0;
      for (int s = 0; s < nst; ++s) {  // uniform per lane group
        int c[R][4];
        VT v[R][4];
#pragma unroll
        for (int u = 0; u < R; ++u) {
          const int e = e0[u] + s * 4 * V;
          if (e < sb[u] && e + 4 <= zrel) {
            const int4 cc = ld_stream_i4(reinterpret_cast<const int4 *>(cb + e), pol);
            c[u][0] = cc.x; c[u][1] = cc.y; c[u][2] = cc.z; c[u][3] = cc.w;
            V4<VT> vv;
            vv.load(vb + e, pol);
#pragma unroll
            for (int j = 0; j < 4; ++j) v[u][j] = vv.v[j];
          } else {
#pragma unroll
            for (int j = 0; j < 4; ++j) {
              const bool ok = e + j < sb[u] && e + j < zrel;
              c[u][j] = ok ? ld_stream_i(cb + e + j, pol) : 0;
              v[u][j] = ok ? ld_stream(vb + e + j, pol) : (VT)0;
            }
          }
        }
        VT xv[R][4];
#pragma unroll
        for (int u = 0; u < R; ++u) {
          const int e = e0[u] + s * 4 * V;
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            const bool in = e + j >= sa[u] && e + j < sb[u];
            xv[u][j] = in ? __ldg(x + c[u][j]) : (VT)0;
            if (!in) v[u][j] = (VT)0;
          }
        }
#pragma unroll
        for (int u = 0; u < R; ++u)
#pragma unroll
          for (int j = 0; j < 4; ++j) part[u] = fma(v[u][j], xv[u][j], part[u]);
      }
#pragma unroll
      for (int u = 0; u < R; ++u) {
#pragma unroll
        for (int o = V / 2; o > 0; o >>= 1) part[u] += __shfl_xor_sync(kFull, part[u], o);
        const int64_t row = t0 + g + G * (q + u);
        if (li == 0 && row < N) y[row] = part[u];
      }
    }
  }
}

// ------------------------------------------------------------------ K5/K6 staged: TMA row-tile pipeline
// Persistent CTAs walk row tiles of TR rows round-robin.  For each tile one
// elected thread issues three 1D bulk copies (cp.async.bulk, evict-first) of
// the tile's rowptr slice and its contiguous colidx / value spans into a
// kStgStages-deep shared-memory ring tracked by mbarriers, kStgStages - 1
// tiles ahead of the compute; the spans are rounded out to the enclosing
// 16-byte chunks (every chunk holds at least one byte of the span, so no read
// leaves the arrays' pages).  Threads then run the same per-row arithmetic as
// the direct kernels from shared memory: V = 1 is CSR-scalar (thread per
// row, RPT rows per thread), V > 1 CSR-vector (V lanes per row, R rows per
// transposed reduction, rows > 8V on the warp-segment path).  A tile whose
// span exceeds the stage capacity is computed from global memory instead
// (same arithmetic, so results are bit-identical either way).  Coalescing no
// longer depends on the row length, and ~100 KB per SM of HBM traffic stays
// in flight with a single issuing thread per CTA.
constexpr int kStgThr = 256;
constexpr int kStgStages = 3;
constexpr int kStgBytes = 32768;  // colidx + value bytes per stage
constexpr int kStgRpBytes = 4096; // rowptr slice bytes per stage (TR * sizeof(IT) <= this)
template <typename VT> __host__ __device__ constexpr int stg_cap() { return (kStgBytes / (4 + (int)sizeof(VT))) & ~3; }
template <typename VT> __host__ __device__ constexpr int stg_cb() { return stg_cap<VT>() * 4 + 32; }
template <typename VT> __host__ __device__ constexpr int stg_vb() { return stg_cap<VT>() * (int)sizeof(VT) + 32; }
__host__ __device__ constexpr int stg_rb() { return kStgRpBytes + 48; }
template <typename VT> __host__ __device__ constexpr int stg_stage() { return stg_cb<VT>() + stg_vb<VT>() + stg_rb(); }
template <typename VT> constexpr size_t stg_smem() { return (size_t)kStgStages * stg_stage<VT>(); }

struct StgMeta {
  int64_t cbase, vbase, rbase;  // global index held by slot 0 of the stage's colidx / value / rowptr region
  int over;                     // span did not fit: compute from global memory
};

template <int V, int RPT, typename IT, typename VT>
__global__ void __launch_bounds__(kStgThr, 2) k_csr_staged(const IT *__restrict__ rowptr, const int32_t *__restrict__ col,
                                                           const VT *__restrict__ val, const VT *__restrict__ x,
                                                           VT *__restrict__ y, int64_t N, int64_t ntiles, int rpg,
                                                           int64_t nseg,
                                                           const int32_t *__restrict__ seg_row,
                                                           const int32_t *__restrict__ seg_k, double *seg_part,
                                                           unsigned *seg_ctr, bool l2ef) {
  // tile = TR rows: V = 1 -> RPT (template) rows per thread; V > 1 -> rpg (a
  // multiple of R) rows per lane group of V lanes
  constexpr int G = kStgThr / V;
  const int TR = V == 1 ? kStgThr * RPT : G * rpg;
  constexpr int CB = stg_cb<VT>(), VB = stg_vb<VT>(), RB = stg_rb(), SB = stg_stage<VT>();
  extern __shared__ __align__(128) unsigned char smem[];
  __shared__ __align__(8) uint64_t bar[kStgStages];
  __shared__ StgMeta meta[kStgStages];
  const int tid = threadIdx.x;
  const uint64_t pol = l2_policy(l2ef);
  if constexpr (V > 1) csrv_segments<IT, VT>(rowptr, col, val, x, y, nseg, seg_row, seg_k, seg_part, seg_ctr, pol);
  const int64_t my = (int64_t)blockIdx.x < ntiles ? (ntiles - 1 - blockIdx.x) / gridDim.x + 1 : 0;
  if (my == 0) return;
  if (tid == 0) {
    for (int s = 0; s < kStgStages; ++s) mbar_init(&bar[s], 1);
    fence_mbar_init();
  }
  __syncthreads();
  auto tile_rows = [&](int64_t t, int64_t &r0, int64_t &r1) {
    r0 = t * TR;
    r1 = r0 + TR < N ? r0 + TR : N;
  };
  auto issue = [&](int64_t t, int st, int64_t a, int64_t b) {  // thread 0 only
    int64_t r0, r1;
    tile_rows(t, r0, r1);
    unsigned char *base = smem + (size_t)st * SB;
    const uintptr_t ra = reinterpret_cast<uintptr_t>(rowptr + r0) & ~(uintptr_t)15;
    const uintptr_t re = (reinterpret_cast<uintptr_t>(rowptr + r1 + 1) + 15) & ~(uintptr_t)15;
    const uintptr_t ca = reinterpret_cast<uintptr_t>(col + a) & ~(uintptr_t)15;
    const uintptr_t ce = (reinterpret_cast<uintptr_t>(col + b) + 15) & ~(uintptr_t)15;
    const uintptr_t va = reinterpret_cast<uintptr_t>(val + a) & ~(uintptr_t)15;
    const uintptr_t ve = (reinterpret_cast<uintptr_t>(val + b) + 15) & ~(uintptr_t)15;
    const bool any = b > a;
    const bool fit = !any || ((ce - ca) <= (uintptr_t)CB && (ve - va) <= (uintptr_t)VB);
    meta[st].rbase = r0 - (int64_t)((reinterpret_cast<uintptr_t>(rowptr + r0) - ra) / sizeof(IT));
    meta[st].cbase = a - (int64_t)((reinterpret_cast<uintptr_t>(col + a) - ca) / 4);
    meta[st].vbase = a - (int64_t)((reinterpret_cast<uintptr_t>(val + a) - va) / sizeof(VT));
    meta[st].over = fit ? 0 : 1;
    const bool cv = any && fit;
    mbar_arrive_expect_tx(&bar[st], (uint32_t)((re - ra) + (cv ? (ce - ca) + (ve - va) : 0)));
    bulk_g2s_evict_first(base + CB + VB, reinterpret_cast<const void *>(ra), (uint32_t)(re - ra), &bar[st], pol);
    if (cv) {
      bulk_g2s_evict_first(base, reinterpret_cast<const void *>(ca), (uint32_t)(ce - ca), &bar[st], pol);
      bulk_g2s_evict_first(base + CB, reinterpret_cast<const void *>(va), (uint32_t)(ve - va), &bar[st], pol);
    }
  };
  auto span = [&](int64_t t, int64_t &a, int64_t &b) {
    int64_t r0, r1;
    tile_rows(t, r0, r1);
    a = (int64_t)rowptr[r0];
    b = (int64_t)rowptr[r1];
  };
  if (tid == 0) {
    for (int j = 0; j < kStgStages && j < my; ++j) {
      int64_t a, b;
      span(blockIdx.x + (int64_t)j * gridDim.x, a, b);
      issue(blockIdx.x + (int64_t)j * gridDim.x, j, a, b);
    }
  }
  for (int64_t j = 0; j < my; ++j) {
    const int st = (int)(j % kStgStages);
    const int64_t t = blockIdx.x + j * gridDim.x;
    int64_t pa = 0, pb = 0;  // thread 0: span of the tile that refills this stage (loads overlap the compute)
    const bool refill = tid == 0 && j + kStgStages < my;
    if (refill) span(t + (int64_t)kStgStages * gridDim.x, pa, pb);
    mbar_wait(&bar[st], (uint32_t)((j / kStgStages) & 1));
    int64_t r0, r1;
    tile_rows(t, r0, r1);
    const unsigned char *base = smem + (size_t)st * SB;
    const int32_t *scol = reinterpret_cast<const int32_t *>(base);
    const VT *sval = reinterpret_cast<const VT *>(base + CB);
    const IT *srp = reinterpret_cast<const IT *>(base + CB + VB);
    const int64_t cb = meta[st].cbase, vb = meta[st].vbase, rb = meta[st].rbase;
    const bool over = meta[st].over != 0;
    // entry e of the tile's span: from shared memory, or global when the span did not fit
    auto C = [&](int64_t e) -> int { return over ? ld_stream_i(col + e, pol) : scol[(int)(e - cb)]; };
    auto W = [&](int64_t e) -> VT { return over ? ld_stream(val + e, pol) : sval[(int)(e - vb)]; };
    if constexpr (V == 1) {
      // CSR-scalar arithmetic of k_csr_scalar (csr_row), RPT rows per thread
#pragma unroll
      for (int q = 0; q < RPT; ++q) {
        const int64_t r = r0 + tid + q * kStgThr;
        if (r < r1) y[r] = (VT)csr_row<8, VT>((int64_t)srp[(int)(r - rb)], (int64_t)srp[(int)(r + 1 - rb)], x, C, W);
      }
    } else {
      // CSR-vector arithmetic of k_csr_vector: lane li takes entries li, li + V, ...
      // (<= 8 per lane; longer rows are segments), R rows per transposed reduction
      constexpr int R = V >= 4 ? 4 : 2;
      constexpr int64_t T = 8 * V;
      const int g = tid / V, li = tid % V;
#pragma unroll 1
      for (int kb = 0; kb < rpg; kb += R) {
        int64_t s[R];
        int l[R];
        unsigned longmask = 0;
#pragma unroll
        for (int u = 0; u < R; ++u) {
          const int64_t r = r0 + g + G * (kb + u);
          s[u] = 0;
          l[u] = 0;
          if (r < r1) {
            s[u] = (int64_t)srp[(int)(r - rb)];
            const int64_t L = (int64_t)srp[(int)(r + 1 - rb)] - s[u];
            if (L > T) longmask |= 1u << u;
            else l[u] = (int)L;
          }
        }
        int cc[R];
        VT vv[R];
#pragma unroll
        for (int u = 0; u < R; ++u) {
          const bool in = li < l[u];
          cc[u] = in ? C(s[u] + li) : -1;
          vv[u] = in ? W(s[u] + li) : (VT)0;
        }
        VT part[R];
#pragma unroll
        for (int u = 0; u < R; ++u) part[u] = cc[u] >= 0 ? vv[u] * __ldg(x + cc[u]) : (VT)0;
#pragma unroll
        for (int u = 0; u < R; ++u)
          for (int m = V + li; m < l[u]; m += V) part[u] = fma(W(s[u] + m), __ldg(x + C(s[u] + m)), part[u]);
        int ridx;
        const VT tot = reduce_transpose<V, R>(part, li, ridx);
        const int64_t row = r0 + g + G * (kb + ridx);
        if (li % (V / R) == 0 && row < r1 && !((longmask >> ridx) & 1u)) y[row] = tot;
      }
    }
    __syncthreads();  // stage st consumed
    if (refill) issue(t + (int64_t)kStgStages * gridDim.x, st, pa, pb);
  }
}

// ------------------------------------------------------------------ K7 ELL (also HYB's ELL part)
// Thread per 4 consecutive rows: per slot one 128-bit load of 4 column ids and
// one 128-bit (fp32) / 2x128-bit (fp64) load of 4 values.  The loads of U
// slots are all issued before the first FMA (explicit register batches: the
// compiler otherwise reuses one register quad and serialises the slots), so
// each thread keeps U x (16 + 16|32) bytes of HBM traffic in flight.
template <typename VT, int U, bool FUSED = false>  // U <= 16: terms per fp32 partial
__global__ void __launch_bounds__(256) k_ell(const int32_t *__restrict__ ecol, const VT *__restrict__ eval,
                                             const VT *__restrict__ x, VT *__restrict__ y, int64_t N, int64_t K,
                                             int64_t ld, int64_t nr, bool l2ef, int pf, bool pfh,
                                             const PeerOut po = PeerOut{}) {
  // rows [0, nr) (nr <= ld: ld for a whole multiply incl. padding, less for a row chunk)
  const uint64_t pol = l2_policy(l2ef);
  const int64_t nq = (nr + 3) >> 2;
  // pf > 0: thread 0 keeps the block's (col, val) slot segments pf batches
  // ahead in L2 (cp.async.bulk prefetch; see k_dia).  Whole-multiply launches
  // only (pf = 0 for row chunks), so B0 and nr are multiples of 32 rows.
  auto prefetch = [&](int64_t k, int64_t B0, uint32_t rows) {
    if (pfh) {
      bulk_prefetch_l2(ecol + k * ld + B0, rows * 4u, pol);
      bulk_prefetch_l2(eval + k * ld + B0, rows * (uint32_t)sizeof(VT), pol);
    } else {
      bulk_prefetch_l2(ecol + k * ld + B0, rows * 4u);
      bulk_prefetch_l2(eval + k * ld + B0, rows * (uint32_t)sizeof(VT));
    }
  };
  for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < nq; q += (int64_t)gridDim.x * blockDim.x) {
    const int64_t i0 = q << 2;
    const int64_t B0 = (q - threadIdx.x) << 2;  // block's first row this iteration
    const uint32_t pr = (uint32_t)((B0 + 4 * (int64_t)blockDim.x < nr ? B0 + 4 * (int64_t)blockDim.x : nr) - B0);
    if (pf > 0 && threadIdx.x == 0)
      for (int64_t k = 0; k < (int64_t)pf * U && k < K; ++k) prefetch(k, B0, pr);
    double acc[4] = {0.0, 0.0, 0.0, 0.0};
    for (int64_t k0 = 0; k0 < K; k0 += U) {
      if (pf > 0 && threadIdx.x == 0)
        for (int64_t k = k0 + (int64_t)pf * U; k < k0 + (int64_t)(pf + 1) * U && k < K; ++k) prefetch(k, B0, pr);
      int4 c[U];
      V4<VT> v[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        if (k0 + u < K) {
          c[u] = ld_stream_i4(reinterpret_cast<const int4 *>(ecol + (k0 + u) * ld + i0), pol);
          v[u].load(eval + (k0 + u) * ld + i0, pol);
        } else {
          c[u] = make_int4(-1, -1, -1, -1);
          v[u].v[0] = v[u].v[1] = v[u].v[2] = v[u].v[3] = (VT)0;
        }
      }
      VT xv[U][4];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        xv[u][0] = c[u].x >= 0 ? __ldg(x + c[u].x) : (VT)0;
        xv[u][1] = c[u].y >= 0 ? __ldg(x + c[u].y) : (VT)0;
        xv[u][2] = c[u].z >= 0 ? __ldg(x + c[u].z) : (VT)0;
        xv[u][3] = c[u].w >= 0 ? __ldg(x + c[u].w) : (VT)0;
      }
      VT part[4] = {0, 0, 0, 0};
#pragma unroll
      for (int u = 0; u < U; ++u)
#pragma unroll
        for (int t = 0; t < 4; ++t) part[t] = fma(v[u].v[t], xv[u][t], part[t]);
#pragma unroll
      for (int t = 0; t < 4; ++t) acc[t] += (double)part[t];
    }
    out4<FUSED, VT>(y, po, i0, N, acc);
  }
}

// ------------------------------------------------------------------ K8 DIA
// Thread per 4 consecutive rows, block = 1024 rows; offsets in shared memory
// (D <= kDiaSmemOffs = 48 KB; more diagonals read them through L1, GOFF).
// Blocks whose rows see every diagonal in range skip all bounds checks.  One
// diagonal per step, <= 32 registers (full occupancy): B200 sweeps on
// configs[1] put more diagonals per batch (U = 2/4/8: 4916/4561/3033 vs 5373
// GB/s) and a diagonal split across lanes (DS = 2/4: 4076/3115) behind —
// resident warps matter more than per-thread bytes in flight.  (U and DS stay
// template parameters fixed at 1: the loop below is written for them.)
constexpr int kDiaSmemOffs = 12288;
template <typename VT, bool GOFF, bool FUSED = false, int U = 1, int DS = 1>  // GOFF: offsets read through L1 (D > kDiaSmemOffs)
__global__ void __launch_bounds__(256, sizeof(VT) == 4 ? 8 : 1)  // fp32: <= 32 regs, full occupancy
    k_dia(const int32_t *__restrict__ offs, const VT *__restrict__ dval,
                                             const VT *__restrict__ x, VT *__restrict__ y, int64_t N, int64_t M,
                                             int64_t D, int64_t ld, int64_t nr, int64_t row0, int64_t off_min,
                                             int64_t off_max, bool x_aligned, bool l2ef, int pf, bool pfh,
                                             const PeerOut po = PeerOut{}) {
  constexpr int64_t RB = 1024 / DS;  // rows per block iteration
  const uint64_t pol = l2_policy(l2ef);
  extern __shared__ int s_off[];
  // pf > 0: thread 0 keeps the block's value segments pf diagonals ahead in L2
  // (one cp.async.bulk L2 prefetch per diagonal, no registers or shared
  // memory): the per-thread chain of dependent value loads then waits on L2,
  // not HBM, and the HBM stream has pf x 4 KB per CTA in flight.
  if constexpr (!GOFF) {
    for (int64_t d = threadIdx.x; d < D; d += blockDim.x) s_off[d] = offs[d];
    __syncthreads();
  }
  auto off_of = [&](int64_t d) -> int { if constexpr (GOFF) return __ldg(offs + d); else return s_off[d]; };
  const int q = (int)(threadIdx.x % DS);
  const int64_t nb = (nr + RB - 1) / RB;  // rows [0, nr), nr <= ld (a row chunk: less)
  for (int64_t blk = blockIdx.x; blk < nb; blk += gridDim.x) {
    const int64_t B0 = blk * RB;
    const int64_t i0 = B0 + 4 * (threadIdx.x / DS);
    const bool active = i0 < nr;  // whole DS groups share i0: uniform within a group
    // segment bytes of one diagonal of this block (16-byte multiple: B0 and ld are multiples of 32 rows)
    const uint32_t pfb = (uint32_t)(((B0 + RB < nr ? B0 + RB : nr) - B0) * (int64_t)sizeof(VT)) & ~15u;
    if (pf > 0 && threadIdx.x == 0)
      for (int64_t d = 0; d < pf && d < D; ++d)
        pfh ? bulk_prefetch_l2(dval + d * ld + B0, pfb, pol) : bulk_prefetch_l2(dval + d * ld + B0, pfb);
    if constexpr (DS == 1) {
      if (!active) continue;      // no cross-lane combine needed
    }
    const int64_t Bend = (B0 + RB < nr ? B0 + RB : nr) - 1;
    const bool interior = row0 + B0 + off_min >= 0 && row0 + Bend + off_max < M;
    // vector x path: aligned windows may reach 3 floats left / 4 right of the needed ones
    const bool xvec = x_aligned && row0 + B0 + off_min - 3 >= 0 && row0 + Bend + off_max + 4 < M;
    double acc[4] = {0.0, 0.0, 0.0, 0.0};
    for (int64_t d0 = (int64_t)q * U; (DS == 1 || active) && d0 < D; d0 += (int64_t)DS * U) {
      if (pf > 0 && threadIdx.x == 0)
        for (int64_t d = d0 + pf; d < d0 + pf + DS * U && d < D; ++d)
          pfh ? bulk_prefetch_l2(dval + d * ld + B0, pfb, pol) : bulk_prefetch_l2(dval + d * ld + B0, pfb);
      V4<VT> v[U];
      VT xv[U][4];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        if (d0 + u < D) v[u].load(dval + (d0 + u) * ld + i0, pol);
        else v[u].v[0] = v[u].v[1] = v[u].v[2] = v[u].v[3] = (VT)0;
      }
      if (sizeof(VT) == 4 && xvec) {
        // fp32, x 16-byte aligned at row0: the 4 values x[j..j+3] (j = row0 + i0 +
        // off) come from the aligned 8-float window at j - (off & 3): two 128-bit
        // loads instead of four 32-bit ones (half the L1 wavefronts); off & 3 is
        // uniform across the warp (i0 is a multiple of 4)
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const bool live = d0 + u < D;
          const int off = live ? off_of(d0 + u) : 0;
          const int r = off & 3;
          const float *xb = reinterpret_cast<const float *>(x) + (row0 + i0 + off - r);
          float4 lo = make_float4(0.f, 0.f, 0.f, 0.f), hi = lo;
          if (live) {
            lo = __ldg(reinterpret_cast<const float4 *>(xb));
            if (r) hi = __ldg(reinterpret_cast<const float4 *>(xb) + 1);
          }
          float w[4];
          switch (r) {
            case 0: w[0] = lo.x; w[1] = lo.y; w[2] = lo.z; w[3] = lo.w; break;
            case 1: w[0] = lo.y; w[1] = lo.z; w[2] = lo.w; w[3] = hi.x; break;
            case 2: w[0] = lo.z; w[1] = lo.w; w[2] = hi.x; w[3] = hi.y; break;
            default: w[0] = lo.w; w[1] = hi.x; w[2] = hi.y; w[3] = hi.z; break;
          }
#pragma unroll
          for (int t = 0; t < 4; ++t) xv[u][t] = (VT)w[t];
        }
      } else if (interior) {
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const bool live = d0 + u < D;  // uniform
          const VT *xp = x + (row0 + i0 + (live ? off_of(d0 + u) : 0));
#pragma unroll
          for (int t = 0; t < 4; ++t) xv[u][t] = live ? __ldg(xp + t) : (VT)0;
        }
      } else {
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const bool live = d0 + u < D;
          const int64_t j = row0 + i0 + (live ? off_of(d0 + u) : 0);
#pragma unroll
          for (int t = 0; t < 4; ++t) xv[u][t] = (live && j + t >= 0 && j + t < M) ? __ldg(x + j + t) : (VT)0;
        }
      }
      VT part[4] = {0, 0, 0, 0};
#pragma unroll
      for (int u = 0; u < U; ++u)
#pragma unroll
        for (int t = 0; t < 4; ++t) part[t] = fma(v[u].v[t], xv[u][t], part[t]);
#pragma unroll
      for (int t = 0; t < 4; ++t) acc[t] += (double)part[t];
    }
#pragma unroll
    for (int o = 1; o < DS; o <<= 1)
#pragma unroll
      for (int t = 0; t < 4; ++t) acc[t] += __shfl_xor_sync(kFull, acc[t], o);
    if (active && q == 0) out4<FUSED, VT>(y, po, i0, N, acc);
  }
}

// ------------------------------------------------------------------ K9b HYB COO tail
// Rows sorted => equal row ids are contiguous.  Rows wholly inside a chunk are
// added to y directly (single owner); the chunk's first and last rows go to
// two carry slots that k_hyb_fixup_seg applies per row in slot order.  No
// atomics; deterministic.
// Lane-sequential layout: lane l of a chunk owns the EP
// consecutive entries [c0 + l*EP, c0 + (l+1)*EP) (128-bit vector loads of
// row/col ids), sums them sequentially per row, writes rows that start and end
// inside the lane directly, and one segmented scan ACROSS LANES (5 steps)
// joins the runs that cross lane boundaries — 1 scan per 32*EP entries
// instead of one per 32.
template <typename VT, int EP>
__global__ void __launch_bounds__(256) k_hyb_tail_ls(const int32_t *__restrict__ trow, const int32_t *__restrict__ tcol,
                                                     const VT *__restrict__ tval, const VT *__restrict__ x,
                                                     VT *__restrict__ y, int64_t Zt, int64_t nch,
                                                     int32_t *__restrict__ carry_row, double *__restrict__ carry_val,
                                                     bool l2ef) {
  static_assert(EP == 4 || EP == 8, "EP");
  constexpr int64_t CH = 32 * EP;
  const uint64_t pol = l2_policy(l2ef);
  const int lane = threadIdx.x & 31;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t ch = warp; ch < nch; ch += nw) {
    const int64_t c0 = ch * CH, cend = c0 + CH < Zt ? c0 + CH : Zt;
    const int64_t e0 = c0 + (int64_t)lane * EP;
    const int nv = e0 >= cend ? 0 : (cend - e0 < EP ? (int)(cend - e0) : EP);  // valid entries of this lane
    int r[EP], c[EP];
    VT v[EP];
    if (nv == EP) {  // full lane: vector loads (e0 is a multiple of EP, arrays 16-byte aligned)
#pragma unroll
      for (int k = 0; k < EP; k += 4) {
        const int4 rr = ld_stream_i4(reinterpret_cast<const int4 *>(trow + e0 + k), pol);
        const int4 cc = ld_stream_i4(reinterpret_cast<const int4 *>(tcol + e0 + k), pol);
        r[k] = rr.x; r[k + 1] = rr.y; r[k + 2] = rr.z; r[k + 3] = rr.w;
        c[k] = cc.x; c[k + 1] = cc.y; c[k + 2] = cc.z; c[k + 3] = cc.w;
        V4<VT> vv;
        vv.load(tval + e0 + k, pol);
        v[k] = vv.v[0]; v[k + 1] = vv.v[1]; v[k + 2] = vv.v[2]; v[k + 3] = vv.v[3];
      }
    } else {
#pragma unroll
      for (int k = 0; k < EP; ++k) {
        const bool ok = k < nv;
        r[k] = ok ? ld_stream_i(trow + e0 + k, pol) : -2;
        c[k] = ok ? ld_stream_i(tcol + e0 + k, pol) : 0;
        v[k] = ok ? ld_stream(tval + e0 + k, pol) : (VT)0;
      }
    }
    double p[EP];
#pragma unroll
    for (int k = 0; k < EP; ++k) p[k] = k < nv ? (double)v[k] * (double)__ldg(x + c[k]) : 0.0;
    // chunk's first / last row (lane 0's first entry; last valid entry)
    const int first_row = __shfl_sync(kFull, r[0], 0);
    const int lastl = (int)((cend - 1 - c0) / EP), lastk = (int)((cend - 1 - c0) % EP);
    int my_last_k = 0;
#pragma unroll
    for (int k = 0; k < EP; ++k) my_last_k = k == lastk ? r[k] : my_last_k;
    const int last_row = __shfl_sync(kFull, my_last_k, lastl);
    if (lane == 0) { carry_row[2 * ch] = -1; carry_row[2 * ch + 1] = -1; }
    __syncwarp();
    auto emit = [&](int row, double val) {  // a completed row segment (chunk ownership rule)
      if (row == first_row) { carry_row[2 * ch] = row; carry_val[2 * ch] = val; }
      else if (row == last_row) { carry_row[2 * ch + 1] = row; carry_val[2 * ch + 1] = val; }
      else y[row] = (VT)((double)y[row] + val);
    };
    // lane-sequential runs
    const int fr = nv > 0 ? r[0] : -2;
    int cur = fr;
    double acc = 0.0, pf = 0.0;
    bool boundary = false;
#pragma unroll
    for (int k = 0; k < EP; ++k) {
      if (k < nv) {
        if (r[k] != cur) {
          if (!boundary) { pf = acc; boundary = true; }
          else emit(cur, acc);  // a row wholly inside this lane
          cur = r[k];
          acc = 0.0;
        }
        acc += p[k];
      }
    }
    const int lr = cur;                  // this lane's last run row
    double s = acc;                      // value of the last run
    // segmented inclusive scan across lanes of the last-run values; a lane heads
    // a new segment if its last run starts inside it or its row differs from the
    // previous lane's last row
    const int prev_lr = __shfl_up_sync(kFull, lr, 1);
    bool f = boundary || lane == 0 || fr != prev_lr;  // segment head flag
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {  // (s, f) segmented inclusive scan
      const double t = __shfl_up_sync(kFull, s, o);
      const bool tf = __shfl_up_sync(kFull, f, o);
      if (lane >= o) {
        if (!f) s += t;
        f = f || tf;
      }
    }
    // s = total of the run ending at this lane's end.  Previous lane's run total:
    const double prev_s = __shfl_up_sync(kFull, s, 1);
    if (nv > 0) {
      if (boundary) {
        // first run of this lane completes here; it continues a run from the
        // previous lane iff that lane's last row equals it
        const double tot = pf + ((lane > 0 && prev_lr == fr) ? prev_s : 0.0);
        emit(fr, tot);
      }
      // the run ending at this lane: complete unless it continues into the next lane
      const int next_fr = __shfl_down_sync(kFull, fr, 1);
      const bool next_valid = __shfl_down_sync(kFull, nv, 1) > 0 && lane < 31;
      const bool continues = next_valid && next_fr == lr;
      if (!continues) emit(lr, s);
    } else {
      (void)__shfl_down_sync(kFull, fr, 1);
      (void)__shfl_down_sync(kFull, nv, 1);
    }
  }
}

// ------------------------------------------------------------------ K6s CSR-vector, nnz-split stream mode
// For skewed row-length distributions (power-law rows, many empty rows) the
// row-oriented K6 wastes lane groups on empty and short rows and serialises
// hub rows; here every warp takes a fixed chunk of 32*EP nonzeros (EP = 8
// fp32 / 4 fp64 consecutive entries per lane, 128-bit loads), so the work is
// balanced by nnz.  The row of each entry is found from rowptr: the starts
// of the chunk's rows (chunk_row[c], chunk_row[c+1]] are counted at their
// chunk positions in shared memory (windows of 32 rows, one per lane) and a
// prefix sum over the positions gives every entry's row.  Products are formed
// and summed in fp64 (R2), lane-sequentially per row, with one segmented scan
// across lanes (as K9b).  Rows wholly inside a chunk are written directly; a
// chunk's first and last rows go to two carry slots that k_hyb_fixup_seg<..,
// false> sums per row in slot order and STORES; empty rows between a chunk's
// rows are zeroed by that chunk (rows before the first nonempty row by chunk
// 0).  No global atomics (the shared-memory counts are integers):
// deterministic.
// HOT (x-locality, the modern analogue of the paper's texture-cached "-Tx"
// variants): the nhot most referenced columns of a power-law
// matrix are staged in shared memory once per CTA (persistent CTAs, two per
// SM, 768 threads); `col` is then the remapped column array whose hot entries
// hold ~slot, and their x value comes from shared memory instead of an L1TEX
// gather (the resource that binds this kernel, §9.0).
template <typename IT, typename VT, int EP, bool HOT = false>
__global__ void __launch_bounds__(HOT ? 768 : 256, HOT ? (EP == 4 ? 2 : 1) : (EP == 4 ? 6 : 4)) k_csr_stream(const IT *__restrict__ rowptr, const int32_t *__restrict__ col,
                                                    const VT *__restrict__ val, const VT *__restrict__ x,
                                                    VT *__restrict__ y, int64_t N, int64_t Z, int64_t nch,
                                                    const int32_t *__restrict__ chunk_row,
                                                    int32_t *__restrict__ carry_row, double *__restrict__ carry_val,
                                                    bool vec, bool l2ef, const int32_t *__restrict__ hot_cols = nullptr,
                                                    int nhot = 0) {
  static_assert(EP == 4 || EP == 8, "EP");
  constexpr int64_t CH = 32 * EP;
  constexpr int NW = HOT ? 24 : 8;
  __shared__ __align__(16) int s_cnt[NW][CH];  // per warp: row starts per chunk position
  extern __shared__ __align__(16) unsigned char s_dyn[];
  VT *s_hot = reinterpret_cast<VT *>(s_dyn);
  if constexpr (HOT) {
    for (int j = threadIdx.x; j < nhot; j += blockDim.x) s_hot[j] = __ldg(x + hot_cols[j]);
    __syncthreads();
  }
  const uint64_t pol = l2_policy(l2ef);
  const int lane = threadIdx.x & 31;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  if (warp == 0) {  // rows before the first nonempty row (chunk_row[0] = last row starting at 0)
    const int r0 = nch > 0 ? chunk_row[0] : (int)N;
    for (int r = lane; r < r0; r += 32) y[r] = (VT)0;
  }
  // (a one-chunk software pipeline — the next chunk's col / val / row range
  // loaded before the current chunk's row work — measured slower: 53 vs 40
  // registers, c2b 0.741 vs 0.716 ms; so did full occupancy by launch bounds,
  // 32 registers + spills: 0.753 ms; and a per-warp two-stage TMA ring for the
  // col / val streams, leaving L1TEX to the gathers: 1.056 vs 0.718 ms)
  for (int64_t ch = warp; ch < nch; ch += nw) {
    const int64_t c0 = ch * CH, cend = c0 + CH < Z ? c0 + CH : Z;
    const int64_t e0 = c0 + (int64_t)lane * EP;
    const int nv = e0 >= cend ? 0 : (cend - e0 < EP ? (int)(cend - e0) : EP);
    int c[EP];
    VT v[EP];
    if (nv == EP && vec) {
#pragma unroll
      for (int k = 0; k < EP; k += 4) {
        const int4 cc = ld_stream_i4(reinterpret_cast<const int4 *>(col + e0 + k), pol);
        c[k] = cc.x; c[k + 1] = cc.y; c[k + 2] = cc.z; c[k + 3] = cc.w;
        V4<VT> vv;
        vv.load(val + e0 + k, pol);
        v[k] = vv.v[0]; v[k + 1] = vv.v[1]; v[k + 2] = vv.v[2]; v[k + 3] = vv.v[3];
      }
    } else {
#pragma unroll
      for (int k = 0; k < EP; ++k) {
        const bool ok = k < nv;
        c[k] = ok ? ld_stream_i(col + e0 + k, pol) : 0;
        v[k] = ok ? ld_stream(val + e0 + k, pol) : (VT)0;
      }
    }
    const int r_lo = chunk_row[ch], r_nx = chunk_row[ch + 1];
    double p[EP];
    if constexpr (HOT) {
#pragma unroll
      for (int k = 0; k < EP; ++k)
        p[k] = k < nv ? (double)v[k] * (double)(c[k] >= 0 ? __ldg(x + c[k]) : s_hot[~c[k]]) : 0.0;
    } else {
#pragma unroll
      for (int k = 0; k < EP; ++k) p[k] = k < nv ? (double)v[k] * (double)__ldg(x + c[k]) : 0.0;
    }
    // rows of the entries: row(e) = r_lo + #{rows r in (r_lo, r_hi] starting at
    // or before chunk position e}.  The rows' starts are counted into a per-warp
    // shared array over the chunk's positions (windows of 32 rows, one per
    // lane, smem atomics), then each lane prefix-sums its EP positions and one
    // warp scan adds the lanes before it.
    const int r_hi = r_nx < (int)N ? r_nx : (int)N - 1;
    int *cnt = s_cnt[threadIdx.x >> 5];
    {
      int4 *c4 = reinterpret_cast<int4 *>(cnt + lane * EP);
#pragma unroll
      for (int k = 0; k < EP; k += 4) c4[k / 4] = make_int4(0, 0, 0, 0);
    }
    __syncwarp();
    for (int w0 = r_lo + 1; w0 <= r_hi; w0 += 32) {  // warp-uniform
      const int rr = w0 + lane;
      if (rr <= r_hi) {
        const int64_t rs = (int64_t)rowptr[rr];
        if (rs - c0 < CH) atomicAdd(cnt + (int)(rs - c0), 1);  // rs > c0 for every row after r_lo
        // an empty row strictly inside the chunk's row range: nobody else writes it
        if (rr < r_nx && (int64_t)rowptr[rr + 1] == rs) y[rr] = (VT)0;
      }
    }
    __syncwarp();
    int r[EP];
    {
      int inc[EP];
      const int4 *c4 = reinterpret_cast<const int4 *>(cnt + lane * EP);
#pragma unroll
      for (int k = 0; k < EP; k += 4) {
        const int4 t = c4[k / 4];
        inc[k] = t.x; inc[k + 1] = t.y; inc[k + 2] = t.z; inc[k + 3] = t.w;
      }
#pragma unroll
      for (int k = 1; k < EP; ++k) inc[k] += inc[k - 1];
      int ex = inc[EP - 1];  // lane total -> exclusive prefix over lanes
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const int t = __shfl_up_sync(kFull, ex, o);
        if (lane >= o) ex += t;
      }
      ex -= inc[EP - 1];
#pragma unroll
      for (int k = 0; k < EP; ++k) r[k] = k < nv ? r_lo + ex + inc[k] : -2;
    }
    const int first_row = r_lo;
    const int lastl = (int)((cend - 1 - c0) / EP), lastk = (int)((cend - 1 - c0) % EP);
    int my_last_k = 0;
#pragma unroll
    for (int k = 0; k < EP; ++k) my_last_k = k == lastk ? r[k] : my_last_k;
    const int last_row = __shfl_sync(kFull, my_last_k, lastl);
    if (lane == 0) { carry_row[2 * ch] = -1; carry_row[2 * ch + 1] = -1; }
    __syncwarp();
    auto emit = [&](int row, double s_) {  // a completed row segment (chunk ownership rule)
      if (row == first_row) { carry_row[2 * ch] = row; carry_val[2 * ch] = s_; }
      else if (row == last_row) { carry_row[2 * ch + 1] = row; carry_val[2 * ch + 1] = s_; }
      else y[row] = (VT)s_;
    };
    const int fr = nv > 0 ? r[0] : -2;
    int cur = fr;
    double acc = 0.0, pf = 0.0;
    bool boundary = false;
#pragma unroll
    for (int k = 0; k < EP; ++k) {
      if (k < nv) {
        if (r[k] != cur) {
          if (!boundary) { pf = acc; boundary = true; }
          else emit(cur, acc);
          cur = r[k];
          acc = 0.0;
        }
        acc += p[k];
      }
    }
    const int lr = cur;
    double s = acc;
    const int prev_lr = __shfl_up_sync(kFull, lr, 1);
    bool f = boundary || lane == 0 || fr != prev_lr;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const double t = __shfl_up_sync(kFull, s, o);
      const bool tf = __shfl_up_sync(kFull, f, o);
      if (lane >= o) {
        if (!f) s += t;
        f = f || tf;
      }
    }
    const double prev_s = __shfl_up_sync(kFull, s, 1);
    const int next_fr = __shfl_down_sync(kFull, fr, 1);
    const bool next_valid = __shfl_down_sync(kFull, nv, 1) > 0 && lane < 31;
    if (nv > 0) {
      if (boundary) emit(fr, pf + ((lane > 0 && prev_lr == fr) ? prev_s : 0.0));
      if (!(next_valid && next_fr == lr)) emit(lr, s);
    }
  }
}

// Carry fixup by the static plan of prepare_hyb: segment s = the carry slots
// [seg[s], seg[s+1]) of one row, summed in slot order (slots left empty by the
// tail kernel, row -1, skipped) and added to y once.  Segments of <= 32 slots:
// a thread each (blocks [0, nshort)); longer ones (rows spanning many chunks,
// e.g. R-MAT hubs): a warp each, lane-strided partial sums + a fixed xor tree.
template <typename VT, bool ADD = true>  // ADD: y[r] += carries (HYB); else y[r] = carries (K6s)
__global__ void __launch_bounds__(256) k_hyb_fixup_seg(const int32_t *__restrict__ carry_row,
                                                       const double *__restrict__ carry_val,
                                                       const int32_t *__restrict__ seg, int64_t S,
                                                       const int32_t *__restrict__ lst, int64_t nlong,
                                                       unsigned nshort, VT *__restrict__ y) {
  if (blockIdx.x < nshort) {
    for (int64_t s = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; s < S; s += (int64_t)nshort * blockDim.x) {
      const int j0 = seg[s], j1 = seg[s + 1];
      if (j1 - j0 > 32) continue;
      double tot = 0.0;
      for (int j = j0; j < j1; ++j)
        if (carry_row[j] >= 0) tot += carry_val[j];
      const int r = carry_row[j0];
      y[r] = ADD ? (VT)((double)y[r] + tot) : (VT)tot;
    }
    return;
  }
  const int lane = threadIdx.x & 31;
  const int64_t w = ((blockIdx.x - nshort) * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)(gridDim.x - nshort) * blockDim.x) >> 5;
  for (int64_t q = w; q < nlong; q += nw) {
    const int s = lst[q];
    const int j0 = seg[s], j1 = seg[s + 1];
    double t = 0.0;
    for (int j = j0 + lane; j < j1; j += 32)
      if (carry_row[j] >= 0) t += carry_val[j];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) t += __shfl_xor_sync(kFull, t, o);
    if (lane == 0) {
      const int r = carry_row[j0];
      y[r] = ADD ? (VT)((double)y[r] + t) : (VT)t;
    }
  }
}

// ------------------------------------------------------------------ K10 L2 flush (read-only: leaves clean lines)
__global__ void __launch_bounds__(256) k_flush(const int4 *__restrict__ buf, int64_t n, int *__restrict__ sink) {
  int acc = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    int4 v = __ldcg(buf + i);
    acc ^= v.x ^ v.y ^ v.z ^ v.w;
  }
  if (acc == 0x7fffffff) *sink = acc;
}

// DIA L2 prefetch distance in diagonals: NITRO_DIA_PF overrides; default 1.
// B200, 3 interleaved repeats (GB/s): configs[1] 128^3 PF=0 5133, 1 5357,
// 2 5367; 256^3 PF=0 6355, 1 6796, 2 6731.
int dia_prefetch() {
  static int env = [] {
    const char *e = getenv("NITRO_DIA_PF");
    return e ? atoi(e) : -1;
  }();
  return env >= 0 ? env : 1;
}

// bulk L2 prefetches carry the evict-first policy: NITRO_PF_HINT=0 disables; default on
bool prefetch_hint() {
  static int env = [] {
    const char *e = getenv("NITRO_PF_HINT");
    return e ? atoi(e) : 1;
  }();
  return env != 0;
}

// ELL L2 prefetch distance in slot batches: NITRO_ELL_PF overrides; default 1.
// B200 (GB/s, PF 0 -> 1, same box): configs[1] 6035 -> 6369 and 5732 -> 5815,
// dense band b = 48 6527 -> 6921, 256^3 stencil 5894 -> 6331
int ell_prefetch() {
  static int env = [] {
    const char *e = getenv("NITRO_ELL_PF");
    return e ? atoi(e) : -1;
  }();
  return env >= 0 ? env : 1;
}

// DIA grid cap in blocks per SM: NITRO_DIA_GRID overrides; default 16
// (one wave-free launch of every 1024-row block at configs[1])
int dia_blocks_per_sm() {
  static int env = [] {
    const char *e = getenv("NITRO_DIA_GRID");
    return e ? atoi(e) : 0;
  }();
  return env > 0 ? env : 16;
}

// streamed matrix arrays use an L2 evict-first policy (NITRO_L2EF=0 disables)
bool l2_evict_first() {
  static bool v = [] {
    const char *e = getenv("NITRO_L2EF");
    return e ? atoi(e) != 0 : true;
  }();
  return v;
}

// ELL slot batch width: NITRO_ELL_U overrides (1/2); default 2.  B200 sweep
// on configs[1] (fp32): U=2 6372, U=4 5461, U=8 4681 GB/s — fewer registers and
// more resident warps beat deeper per-thread batches for this gather pattern.
// With the L2 prefetch on (few-diagonal matrices) U = 1 is best: the prefetch
// keeps the stream in flight and the fewer registers buy occupancy (B200,
// U=1 vs 2 at PF=1, 2 repeats: c1 6458 vs 5817 GB/s, dense band b=48 6965 vs
// 6197, 256^3 6540 vs 6810); random-column matrices keep U = 2 (c2a 2127 vs 2102).
int ell_batch(size_t sv, bool local) {
  static int env = [] {
    const char *e = getenv("NITRO_ELL_U");
    return e ? atoi(e) : 0;
  }();
  (void)sv;
  if (env == 1 || env == 2) return env;
  return local ? 1 : 2;
}

unsigned grid_cap(int64_t blocks, int per_sm);

// columns on few diagonals (the DIA fill test of C9: D * N <= 3 Z)
bool diag_local(const nitro_spmv *A) {
  return A->feat_ready && (double)A->feat.ndiag * (double)A->N <= 3.0 * (double)std::max<int64_t>(A->Z, 1);
}

template <typename VT>
void launch_ell(const int32_t *col, const VT *val, const VT *x, VT *y, int64_t N, int64_t K, int64_t ld,
                cudaStream_t s, int64_t nr = -1, bool local = false) {
  // L2 prefetch of the slot stream: whole multiplies (nr < 0) of matrices whose
  // columns lie on few diagonals (x gathers hit L1/L2 lines shared by
  // neighbouring rows).  Random-column matrices are bound by the L2 sector
  // traffic of the gathers, and the prefetched lines compete with them
  // (B200, configs[2] uniform ELL: 2110 -> 2060 GB/s with, 1873 without the
  // evict-first hint), so they run without.
  const int pf = nr < 0 && local ? ell_prefetch() : 0;
  if (nr < 0) nr = ld;
  const unsigned g = grid_cap(((nr + 3) / 4 + 255) / 256, 16);
  // U from the matrix class only (not from pf), so row-chunk launches (pf = 0)
  // and NITRO_ELL_PF=0 sum a row exactly like the default whole multiply
  // (the U = 1 gain holds up to ~2 GB of slot arrays: c1 0.47 GB and a dense
  // band 1.6 GB gain 11-12 %, a 256^3 stencil 3.6 GB loses 4 % and 512^3 30 GB
  // loses 14 % — 6585 vs 5642 GB/s — so larger ELL formats keep U = 2)
  const bool small = (double)K * (double)ld * (double)(sizeof(VT) + 4) <= 2.0 * 1073741824.0;
  if (ell_batch(sizeof(VT), local && small) == 1)
    k_ell<VT, 1><<<g, 256, 0, s>>>(col, val, x, y, N, K, ld, nr, l2_evict_first(), pf, prefetch_hint());
  else
    k_ell<VT, 2><<<g, 256, 0, s>>>(col, val, x, y, N, K, ld, nr, l2_evict_first(), pf, prefetch_hint());
}

unsigned grid_cap(int64_t blocks, int per_sm = 8) {
  int64_t cap = (int64_t)num_sms() * per_sm;
  if (blocks > cap) blocks = cap;
  return (unsigned)(blocks < 1 ? 1 : blocks);
}

// staged CSR kernels (TMA row-tile pipeline) under NITRO_CSR_IMPL_AUTO: off by
// default (B200: slower than the direct kernels on every
// class measured); NITRO_CSR_STAGED=1 turns them on for AUTO
bool csr_staged_on() {
  static bool v = [] {
    const char *e = getenv("NITRO_CSR_STAGED");
    return e ? atoi(e) != 0 : false;
  }();
  return v;
}

// CSR-vector rows per pipeline stage R: 2 (B200 sweep: R = 2 beat 4 and 8 on
// every class — registers and resident warps beat rows in flight per lane);
// NITRO_CSRV_R=4 overrides
int csrv_rows(int V) {
  static int env = [] {
    const char *e = getenv("NITRO_CSRV_R");
    return e ? atoi(e) : 0;
  }();
  return (env == 4 && V >= 4) ? 4 : 2;
}

// CSR-vector remainder batch kB = 3 (terms 2..4 of a lane in one batch;
// longer rows loop); NITRO_CSRV_B=7 batches every term of the short path
int csrv_batch(const nitro_spmv *A, int V) {
  static int env = [] {
    const char *e = getenv("NITRO_CSRV_B");
    return e ? atoi(e) : 0;
  }();
  if (env == 3 || env == 7) return env;
  (void)A;
  (void)V;
  return 3;  // B200 sweep: kB = 7 lost on every class (registers), even rows of > 4V entries
}

// CSR-scalar head batch H (entries loaded before the first gather): the
// smallest of 4 / 8 / 16 covering the mean row length; NITRO_CSRS_HEAD overrides
int csrs_head(const nitro_spmv *A) {
  static int env = [] {
    const char *e = getenv("NITRO_CSRS_HEAD");
    return e ? atoi(e) : 0;
  }();
  if (env == 4 || env == 8 || env == 16) return env;
  const double mean = A->N > 0 ? (double)A->Z / (double)A->N : 0.0;
  return mean <= 8.0 ? 8 : 16;  // B200: H = 8 beat 4 on every short-row class measured
}

struct SegArgs {
  int64_t nseg = 0;
  int32_t *row = nullptr, *k = nullptr;
  double *part = nullptr;
  unsigned *ctr = nullptr;
};

template <int V, int RPT, typename IT, typename VT>
nitro_status_t launch_staged_k(const IT *rp, const int32_t *col, const VT *val, const VT *x, VT *y, int64_t N,
                               int rpg, const SegArgs &sg, bool l2ef, cudaStream_t s) {
  constexpr size_t sm = stg_smem<VT>();
  static int bps = -1;  // resident CTAs per SM at this shared-memory size
  if (bps < 0) {
    NITRO_CUDA(cudaFuncSetAttribute(k_csr_staged<V, RPT, IT, VT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm));
    int b = 0;
    NITRO_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, k_csr_staged<V, RPT, IT, VT>, kStgThr, sm));
    bps = std::max(b, 1);
  }
  const int64_t TR = V == 1 ? (int64_t)kStgThr * RPT : (int64_t)(kStgThr / V) * rpg;
  const int64_t ntiles = (N + TR - 1) / TR;
  const int64_t cap = (int64_t)num_sms() * bps;
  int64_t grid = std::min<int64_t>(ntiles, cap);
  if (V > 1) grid = std::max<int64_t>(grid, std::min<int64_t>((sg.nseg + 7) / 8, cap));
  k_csr_staged<V, RPT, IT, VT><<<(unsigned)std::max<int64_t>(grid, 1), kStgThr, sm, s>>>(
      rp, col, val, x, y, N, ntiles, rpg, sg.nseg, sg.row, sg.k, sg.part, sg.ctr, l2ef);
  NITRO_CUDA(cudaGetLastError());
  return NITRO_OK;
}

// Tile height: the largest that keeps a mean tile within half a stage (and the
// rowptr slice within kStgRpBytes); matrices whose rows are too long for one
// row (V = 1) or R rows per lane group (V > 1) per tile keep the direct kernels.
template <typename IT, typename VT>
nitro_status_t launch_staged(const nitro_spmv *A, int V, const IT *rp, const VT *val, const VT *x, VT *y, int64_t N,
                             const SegArgs &sg, cudaStream_t s, bool &used) {
  used = false;
  const bool force = A->csr_impl == NITRO_CSR_IMPL_STAGED;
  if (A->csr_impl == NITRO_CSR_IMPL_DIRECT || (!force && !csr_staged_on()) || N <= 0 || A->N <= 0) return NITRO_OK;
  const double mean = (double)A->Z / (double)A->N;
  constexpr double CAP = stg_cap<VT>();
  constexpr int sp = (int)sizeof(IT);
  const bool l2ef = l2_evict_first();
  if (V == 1) {
    int rpt = 0;
    for (int c = 4; c >= 1 && !rpt; c /= 2)
      if (c * kStgThr * sp <= kStgRpBytes && c * kStgThr * mean <= CAP / 2) rpt = c;
    if (!rpt) {
      if (kStgThr * mean > 0.75 * CAP && !force) return NITRO_OK;
      rpt = 1;
    }
    used = true;
    switch (rpt) {
      case 4: return launch_staged_k<1, 4, IT, VT>(rp, A->col, val, x, y, N, 0, sg, l2ef, s);
      case 2: return launch_staged_k<1, 2, IT, VT>(rp, A->col, val, x, y, N, 0, sg, l2ef, s);
      default: return launch_staged_k<1, 1, IT, VT>(rp, A->col, val, x, y, N, 0, sg, l2ef, s);
    }
  }
  const int R = V >= 4 ? 4 : 2, G = kStgThr / V;
  int rpg = 0;
  for (int c = 8 * R; c >= R && !rpg; c /= 2)
    if (c * G * sp <= kStgRpBytes && c * G * mean <= CAP / 2) rpg = c;
  if (!rpg) {
    if (R * G * mean > 0.75 * CAP && !force) return NITRO_OK;
    rpg = R;  // R * G * sp <= 2048 for every V
  }
  used = true;
  const bool ef = l2ef && V >= 16;  // as the direct kernel: the hint hurts short rows
  switch (V) {
    case 2: return launch_staged_k<2, 0, IT, VT>(rp, A->col, val, x, y, N, rpg, sg, ef, s);
    case 4: return launch_staged_k<4, 0, IT, VT>(rp, A->col, val, x, y, N, rpg, sg, ef, s);
    case 8: return launch_staged_k<8, 0, IT, VT>(rp, A->col, val, x, y, N, rpg, sg, ef, s);
    case 16: return launch_staged_k<16, 0, IT, VT>(rp, A->col, val, x, y, N, rpg, sg, ef, s);
    default: return launch_staged_k<32, 0, IT, VT>(rp, A->col, val, x, y, N, rpg, sg, ef, s);
  }
}

template <typename IT, typename VT>
nitro_status_t run_t(nitro_spmv *A, int variant, const VT *x, VT *y, cudaStream_t s, int64_t r0 = 0,
                     int64_t r1 = -1) {
  // rows [r0, r1) (default: all).  Partial ranges only for the row-separable
  // CSR-scalar / ELL / DIA launches (launch_spmv_rows); r0 % 32 == 0.
  const bool part = r1 >= 0;
  if (!part) r1 = A->N;
  const IT *rp = (const IT *)A->rowptr + r0;
  const VT *val = (const VT *)A->val;
  const int64_t N = r1 - r0;
  y += r0;
  switch (variant) {
    case NITRO_CSR_SCALAR:
      if (N > 0) {
        bool used = false;
        NITRO_TRY((launch_staged<IT, VT>)(A, 1, rp, val, x, y, N, SegArgs{}, s, used));
        if (!used) {
          const unsigned g = grid_cap((N + 255) / 256, 16);
          switch (csrs_head(A)) {
            case 4: k_csr_scalar<4, IT, VT><<<g, 256, 0, s>>>(rp, A->col, val, x, y, N); break;
            case 16: k_csr_scalar<16, IT, VT><<<g, 256, 0, s>>>(rp, A->col, val, x, y, N); break;
            default: k_csr_scalar<8, IT, VT><<<g, 256, 0, s>>>(rp, A->col, val, x, y, N); break;
          }
        }
      }
      break;
    case NITRO_CSR_VECTOR: {
      if (part) return fail(NITRO_E_INVALID_ARG, "CSR-vector has no row-range launch");
      if (N == 0) break;
      if (csrv_vec_mode(A)) {  // K6v: 128-bit loads, V lanes per row
        const unsigned g = grid_cap((N + 255) / 256, 8);
        const bool ef = l2_evict_first();
        switch (A->csrv.V) {
          case 2: k_csr_vec4<2, IT, VT><<<g, 256, 0, s>>>(rp, A->col, val, x, y, N, A->Z, ef); break;
          case 4: k_csr_vec4<4, IT, VT><<<g, 256, 0, s>>>(rp, A->col, val, x, y, N, A->Z, ef); break;
          case 8: k_csr_vec4<8, IT, VT><<<g, 256, 0, s>>>(rp, A->col, val, x, y, N, A->Z, ef); break;
          case 16: k_csr_vec4<16, IT, VT><<<g, 256, 0, s>>>(rp, A->col, val, x, y, N, A->Z, ef); break;
          default: k_csr_vec4<32, IT, VT><<<g, 256, 0, s>>>(rp, A->col, val, x, y, N, A->Z, ef); break;
        }
        break;
      }
      if (A->csrv.stream) {  // K6s: nnz-split chunks + carry fixup
        const int64_t nch = A->csrv.nch;
        const bool vec = ((reinterpret_cast<uintptr_t>(A->col) | reinterpret_cast<uintptr_t>(val)) & 15) == 0;
        if (A->csrv.nhot > 0) {  // hot-x staging: two persistent 768-thread CTAs per SM
          const size_t hs = (size_t)A->csrv.nhot * sizeof(VT);
          const int per_sm = A->csrv.EP == 4 ? 2 : 1;  // resident 768-thread CTAs (registers)
          const unsigned gh = (unsigned)std::max<int64_t>(1, std::min<int64_t>((int64_t)per_sm * num_sms(), (nch + 23) / 24));
          const int32_t *hc = A->csrv.hcol.as<int32_t>();
#define NITRO_K6H(EPV)                                                                                            \
  do {                                                                                                            \
    static bool attr_ = false;                                                                                    \
    if (!attr_) {                                                                                                 \
      NITRO_CUDA(cudaFuncSetAttribute(k_csr_stream<IT, VT, EPV, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, \
                                      96 * 1024));                                                                \
      attr_ = true;                                                                                               \
    }                                                                                                             \
    k_csr_stream<IT, VT, EPV, true><<<gh, 768, hs, s>>>(rp, hc, val, x, y, N, A->Z, nch,                           \
                                                         A->csrv.chunk_row.as<int32_t>(),                          \
                                                         A->csrv.carry_row.as<int32_t>(),                          \
                                                         A->csrv.carry_val.as<double>(), vec, l2_evict_first(),    \
                                                         A->csrv.hot_cols.as<int32_t>(), (int)A->csrv.nhot);       \
  } while (0)
          if (A->csrv.EP == 4) NITRO_K6H(4);
          else NITRO_K6H(8);
#undef NITRO_K6H
        } else {
        const unsigned gs = grid_cap(std::max<int64_t>((nch + 7) / 8, 1), 16);
        if (A->csrv.EP == 4)
          k_csr_stream<IT, VT, 4><<<gs, 256, 0, s>>>(rp, A->col, val, x, y, N, A->Z, nch,
                                                     A->csrv.chunk_row.as<int32_t>(), A->csrv.carry_row.as<int32_t>(),
                                                     A->csrv.carry_val.as<double>(), vec, l2_evict_first());
        else
          k_csr_stream<IT, VT, 8><<<gs, 256, 0, s>>>(rp, A->col, val, x, y, N, A->Z, nch,
                                                     A->csrv.chunk_row.as<int32_t>(), A->csrv.carry_row.as<int32_t>(),
                                                     A->csrv.carry_val.as<double>(), vec, l2_evict_first());
        }
        if (nch > 0) {
          const unsigned nshort = grid_cap((A->csrv.fix_S + 255) / 256, 8);
          const unsigned nlong_blk = A->csrv.fix_nlong > 0
                                         ? (unsigned)std::min<int64_t>((A->csrv.fix_nlong + 7) / 8, (int64_t)num_sms() * 4)
                                         : 0;
          k_hyb_fixup_seg<VT, false><<<nshort + nlong_blk, 256, 0, s>>>(
              A->csrv.carry_row.as<int32_t>(), A->csrv.carry_val.as<double>(), A->csrv.fix_seg.as<int32_t>(),
              A->csrv.fix_S, A->csrv.fix_long.as<int32_t>(), A->csrv.fix_nlong, nshort, y);
        }
        break;
      }
      const int64_t nseg = A->csrv.n_long;
      int32_t *seg_row = A->csrv.long_rows.as<int32_t>();
      int32_t *seg_k = seg_row + nseg;
      double *seg_part = reinterpret_cast<double *>(reinterpret_cast<char *>(A->csrv.long_rows.p) + nseg * 8);
      unsigned *seg_ctr = reinterpret_cast<unsigned *>(reinterpret_cast<char *>(A->csrv.long_rows.p) + nseg * 16);
      {
        SegArgs sg;
        sg.nseg = nseg;
        sg.row = seg_row;
        sg.k = seg_k;
        sg.part = seg_part;
        sg.ctr = seg_ctr;
        bool used = false;
        NITRO_TRY((launch_staged<IT, VT>)(A, A->csrv.V, rp, val, x, y, N, sg, s, used));
        if (used) break;
      }
      // 8 warps x 32 rows per block-iteration; segments are spread over all warps
      const unsigned g = grid_cap(std::max<int64_t>((N + 255) / 256, (nseg + 7) / 8), 8);
      const unsigned gw_ = grid_cap(std::max<int64_t>((N + 255) / 256, (nseg + 7) / 8), 12);
#define NITRO_CSRV(VV)                                                                                      \
  do {                                                                                                      \
    const bool ef_ = l2_evict_first() && VV >= 16;                                                          \
    const bool b7_ = csrv_batch(A, VV) == 7;                                                                \
    switch (csrv_rows(VV)) {                                                                                \
      case 4:                                                                                               \
        if (b7_) k_csr_vector<VV, (VV >= 4 ? 4 : 2), 7, IT, VT><<<g, 256, 0, s>>>(rp, A->col, val, x, y, N, nseg, seg_row, seg_k, seg_part, seg_ctr, ef_); \
        else k_csr_vector<VV, (VV >= 4 ? 4 : 2), 3, IT, VT><<<g, 256, 0, s>>>(rp, A->col, val, x, y, N, nseg, seg_row, seg_k, seg_part, seg_ctr, ef_); \
        break;                                                                                              \
      default:                                                                                              \
        if (b7_) k_csr_vector<VV, 2, 7, IT, VT><<<g, 256, 0, s>>>(rp, A->col, val, x, y, N, nseg, seg_row, seg_k, seg_part, seg_ctr, ef_); \
        else if (sizeof(VT) == 8) k_csr_vector<VV, 2, 3, IT, VT><<<gw_, 256, 0, s>>>(rp, A->col, val, x, y, N, nseg, seg_row, seg_k, seg_part, seg_ctr, ef_); \
        else k_csr_vector<VV, 2, 3, IT, VT><<<g, 256, 0, s>>>(rp, A->col, val, x, y, N, nseg, seg_row, seg_k, seg_part, seg_ctr, ef_); \
        break;                                                                                              \
    }                                                                                                       \
  } while (0)
      switch (A->csrv.V) {
        case 2: NITRO_CSRV(2); break;
        case 4: NITRO_CSRV(4); break;
        case 8: NITRO_CSRV(8); break;
        case 16: NITRO_CSRV(16); break;
        default: NITRO_CSRV(32); break;
      }
#undef NITRO_CSRV
      break;
    }
    case NITRO_ELL:
      if (N > 0)
        launch_ell<VT>(A->ell.col.as<int32_t>() + r0, A->ell.val.as<VT>() + r0, x, y, N, A->ell.K, A->ell.ld, s,
                       part ? round_up(N, 32) : -1, diag_local(A));
      break;
    case NITRO_DIA:
      if (N > 0) {
        const size_t sm = (size_t)std::max<int64_t>(A->dia.D, 1) * 4;
        const int64_t row0 = A->row0 + r0, nr = part ? round_up(N, 32) : A->dia.ld;
        const bool x_al = ((reinterpret_cast<uintptr_t>(x) & 15) == 0) && (row0 % 4 == 0);
        const unsigned g = grid_cap((nr + 1023) / 1024, dia_blocks_per_sm());
        if (A->dia.D <= kDiaSmemOffs)
          k_dia<VT, false><<<g, 256, sm, s>>>(A->dia.off.as<int32_t>(), A->dia.val.as<VT>() + r0, x, y, N, A->M,
                                              A->dia.D, A->dia.ld, nr, row0, A->dia.off_min, A->dia.off_max, x_al,
                                              l2_evict_first(), part ? 0 : dia_prefetch(), prefetch_hint());
        else
          k_dia<VT, true><<<g, 256, 0, s>>>(A->dia.off.as<int32_t>(), A->dia.val.as<VT>() + r0, x, y, N, A->M,
                                            A->dia.D, A->dia.ld, nr, row0, A->dia.off_min, A->dia.off_max, x_al,
                                            l2_evict_first(), part ? 0 : dia_prefetch(), prefetch_hint());
      }
      break;
    case NITRO_HYB:
      if (part) return fail(NITRO_E_INVALID_ARG, "HYB has no row-range launch");
      if (N > 0) {
        launch_ell<VT>(A->hyb.col.as<int32_t>(), A->hyb.val.as<VT>(), x, y, N, A->hyb.K, A->hyb.ld, s, -1,
                       diag_local(A));
        if (A->hyb.Zt > 0) {
          const unsigned gt = grid_cap((A->hyb.nchunks + 7) / 8, 16);
          if (A->hyb.W == 4)
            k_hyb_tail_ls<VT, 4><<<gt, 256, 0, s>>>(A->hyb.trow.as<int32_t>(), A->hyb.tcol.as<int32_t>(),
                                                   A->hyb.tval.as<VT>(), x, y, A->hyb.Zt, A->hyb.nchunks,
                                                   A->hyb.carry_row.as<int32_t>(), A->hyb.carry_val.as<double>(),
                                                   l2_evict_first());
          else
            k_hyb_tail_ls<VT, 8><<<gt, 256, 0, s>>>(A->hyb.trow.as<int32_t>(), A->hyb.tcol.as<int32_t>(),
                                                   A->hyb.tval.as<VT>(), x, y, A->hyb.Zt, A->hyb.nchunks,
                                                   A->hyb.carry_row.as<int32_t>(), A->hyb.carry_val.as<double>(),
                                                   l2_evict_first());
          const unsigned nshort = grid_cap((A->hyb.fix_S + 255) / 256, 8);
          const unsigned nlong_blk =
              A->hyb.fix_nlong > 0 ? (unsigned)std::min<int64_t>((A->hyb.fix_nlong + 7) / 8, (int64_t)num_sms() * 4) : 0;
          k_hyb_fixup_seg<VT><<<nshort + nlong_blk, 256, 0, s>>>(
              A->hyb.carry_row.as<int32_t>(), A->hyb.carry_val.as<double>(), A->hyb.fix_seg.as<int32_t>(),
              A->hyb.fix_S, A->hyb.fix_long.as<int32_t>(), A->hyb.fix_nlong, nshort, y);
        }
      }
      break;
    default:
      return fail(NITRO_E_INVALID_ARG, "unknown variant");
  }
  NITRO_CUDA(cudaGetLastError());
  return NITRO_OK;
}

}  // namespace

namespace {
// whole-multiply launches of the row-separable variants with the f3 (ii)
// peer-store epilogue (same kernels, FUSED instantiation: identical
// arithmetic, so y and the peer copies are bit-identical to launch_spmv's y)
template <typename IT, typename VT>
nitro_status_t run_fused_t(nitro_spmv *A, int variant, const VT *x, VT *y, const PeerOut &po, cudaStream_t s) {
  const int64_t N = A->N;
  if (N == 0) return NITRO_OK;
  const IT *rp = (const IT *)A->rowptr;
  const VT *val = (const VT *)A->val;
  switch (variant) {
    case NITRO_CSR_SCALAR: {
      const unsigned g = grid_cap((N + 255) / 256, 16);
      switch (csrs_head(A)) {
        case 4: k_csr_scalar<4, IT, VT, true><<<g, 256, 0, s>>>(rp, A->col, val, x, y, N, po); break;
        case 16: k_csr_scalar<16, IT, VT, true><<<g, 256, 0, s>>>(rp, A->col, val, x, y, N, po); break;
        default: k_csr_scalar<8, IT, VT, true><<<g, 256, 0, s>>>(rp, A->col, val, x, y, N, po); break;
      }
      break;
    }
    case NITRO_ELL: {
      const bool local = diag_local(A);
      const int64_t K = A->ell.K, ld = A->ell.ld;
      const int pf = local ? ell_prefetch() : 0;
      const unsigned g = grid_cap(((ld + 3) / 4 + 255) / 256, 16);
      const bool small = (double)K * (double)ld * (double)(sizeof(VT) + 4) <= 2.0 * 1073741824.0;
      if (ell_batch(sizeof(VT), local && small) == 1)
        k_ell<VT, 1, true><<<g, 256, 0, s>>>(A->ell.col.as<int32_t>(), A->ell.val.as<VT>(), x, y, N, K, ld, ld,
                                             l2_evict_first(), pf, prefetch_hint(), po);
      else
        k_ell<VT, 2, true><<<g, 256, 0, s>>>(A->ell.col.as<int32_t>(), A->ell.val.as<VT>(), x, y, N, K, ld, ld,
                                             l2_evict_first(), pf, prefetch_hint(), po);
      break;
    }
    case NITRO_DIA: {
      const int64_t nr = A->dia.ld, row0 = A->row0;
      const bool x_al = ((reinterpret_cast<uintptr_t>(x) & 15) == 0) && (row0 % 4 == 0);
      const unsigned g = grid_cap((nr + 1023) / 1024, dia_blocks_per_sm());
      if (A->dia.D <= kDiaSmemOffs)
        k_dia<VT, false, true><<<g, 256, (size_t)std::max<int64_t>(A->dia.D, 1) * 4, s>>>(
            A->dia.off.as<int32_t>(), A->dia.val.as<VT>(), x, y, N, A->M, A->dia.D, A->dia.ld, nr, row0,
            A->dia.off_min, A->dia.off_max, x_al, l2_evict_first(), dia_prefetch(), prefetch_hint(), po);
      else
        k_dia<VT, true, true><<<g, 256, 0, s>>>(A->dia.off.as<int32_t>(), A->dia.val.as<VT>(), x, y, N, A->M,
                                                A->dia.D, A->dia.ld, nr, row0, A->dia.off_min, A->dia.off_max, x_al,
                                                l2_evict_first(), dia_prefetch(), prefetch_hint(), po);
      break;
    }
    default:
      return fail(NITRO_E_UNSUPPORTED, "fused peer-store epilogue: CSR-scalar, ELL and DIA only");
  }
  NITRO_CUDA(cudaGetLastError());
  return NITRO_OK;
}
}  // namespace

nitro_status_t launch_spmv_fused(nitro_spmv *A, int variant, const void *x, void *y, const PeerOut &po,
                                 cudaStream_t s) {
  if (A->rp64) {
    if (A->fp64) return run_fused_t<int64_t, double>(A, variant, (const double *)x, (double *)y, po, s);
    return run_fused_t<int64_t, float>(A, variant, (const float *)x, (float *)y, po, s);
  }
  if (A->fp64) return run_fused_t<int32_t, double>(A, variant, (const double *)x, (double *)y, po, s);
  return run_fused_t<int32_t, float>(A, variant, (const float *)x, (float *)y, po, s);
}

nitro_status_t launch_spmv(nitro_spmv *A, int variant, const void *x, void *y, cudaStream_t s) {
  if (A->rp64) {
    if (A->fp64) return run_t<int64_t, double>(A, variant, (const double *)x, (double *)y, s);
    return run_t<int64_t, float>(A, variant, (const float *)x, (float *)y, s);
  }
  if (A->fp64) return run_t<int32_t, double>(A, variant, (const double *)x, (double *)y, s);
  return run_t<int32_t, float>(A, variant, (const float *)x, (float *)y, s);
}

nitro_status_t launch_spmv_rows(nitro_spmv *A, int variant, const void *x, void *y, cudaStream_t s, int64_t r0,
                                int64_t r1) {
  if (r0 < 0 || r1 > A->N || r0 > r1 || r0 % 32) return fail(NITRO_E_INVALID_ARG, "bad row range");
  if (A->rp64) {
    if (A->fp64) return run_t<int64_t, double>(A, variant, (const double *)x, (double *)y, s, r0, r1);
    return run_t<int64_t, float>(A, variant, (const float *)x, (float *)y, s, r0, r1);
  }
  if (A->fp64) return run_t<int32_t, double>(A, variant, (const double *)x, (double *)y, s, r0, r1);
  return run_t<int32_t, float>(A, variant, (const float *)x, (float *)y, s, r0, r1);
}

namespace {
// per chunk c: max over rows i < ends[c] of (last column of row i) + 1 (columns
// ascend within a canonical row); written as a per-chunk max, prefix-maxed on the host
template <typename IT>
__global__ void k_chunk_colmax(const IT *__restrict__ rowptr, const int32_t *__restrict__ col, int64_t N,
                               const int64_t *__restrict__ ends, int nch, unsigned long long *__restrict__ out) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < N; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t b = (int64_t)rowptr[i + 1];
    if (b == (int64_t)rowptr[i]) continue;
    int c = 0;
    while (c < nch - 1 && i >= ends[c]) ++c;
    atomicMax(out + c, (unsigned long long)col[b - 1] + 1ull);
  }
}
}  // namespace

nitro_status_t csr_chunk_xhi(nitro_spmv *A, const std::vector<int64_t> &ends, std::vector<int64_t> &xhi) {
  const int nch = (int)ends.size();
  DevBuf tmp;
  NITRO_TRY(tmp.alloc((size_t)nch * 16));
  int64_t *d_ends = tmp.as<int64_t>();
  unsigned long long *d_out = reinterpret_cast<unsigned long long *>(d_ends + nch);
  NITRO_CUDA(cudaMemcpyAsync(d_ends, ends.data(), (size_t)nch * 8, cudaMemcpyHostToDevice, A->stream));
  NITRO_CUDA(cudaMemsetAsync(d_out, 0, (size_t)nch * 8, A->stream));
  const unsigned g = grid_cap((A->N + 255) / 256, 8);
  if (A->N > 0) {
    if (A->rp64) k_chunk_colmax<int64_t><<<g, 256, 0, A->stream>>>((const int64_t *)A->rowptr, A->col, A->N, d_ends, nch, d_out);
    else k_chunk_colmax<int32_t><<<g, 256, 0, A->stream>>>((const int32_t *)A->rowptr, A->col, A->N, d_ends, nch, d_out);
    NITRO_CUDA(cudaGetLastError());
  }
  std::vector<unsigned long long> h(nch);
  NITRO_CUDA(cudaMemcpyAsync(h.data(), d_out, (size_t)nch * 8, cudaMemcpyDeviceToHost, A->stream));
  NITRO_CUDA(cudaStreamSynchronize(A->stream));
  xhi.assign(nch, 0);
  int64_t run = 0;
  for (int c = 0; c < nch; ++c) {
    run = std::max<int64_t>(run, (int64_t)h[c]);
    xhi[c] = run;
  }
  return NITRO_OK;
}

nitro_status_t launch_flush(nitro_spmv *A, cudaStream_t s) {
  if (!A->flush.p) {
    int l2 = 0;
    NITRO_CUDA(cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, A->device));
    NITRO_TRY(A->flush.alloc((size_t)std::max(l2, 1 << 20) * 3 + 64));
    NITRO_CUDA(cudaMemsetAsync(A->flush.p, 1, A->flush.bytes, s));
  }
  const int64_t n = (int64_t)((A->flush.bytes - 64) / 16);
  k_flush<<<grid_cap((n + 255) / 256, 8), 256, 0, s>>>(A->flush.as<int4>(), n,
                                                       reinterpret_cast<int *>(A->flush.as<char>() + A->flush.bytes - 64));
  NITRO_CUDA(cudaGetLastError());
  return NITRO_OK;
}

int launches_of(const nitro_spmv *A, int variant) {
  if (A->N == 0) return 0;
  if (variant == NITRO_CSR_VECTOR && A->csrv.stream) return A->csrv.nch > 0 ? 2 : 1;
  if (variant == NITRO_HYB) return A->hyb.Zt > 0 ? 3 : 1;
  return 1;
}

double compulsory_bytes(const nitro_spmv *A, int variant) {
  const double N = (double)A->N, M = (double)A->M, Z = (double)A->Z;
  const double sv = A->fp64 ? 8 : 4, si = 4, sp = A->rp64 ? 8 : 4;
  const double xy = M * sv + N * sv;
  switch (variant) {
    case NITRO_CSR_SCALAR:
    case NITRO_CSR_VECTOR: return Z * (sv + si) + (N + 1) * sp + xy;
    case NITRO_ELL: return (double)A->ell.K * N * (sv + si) + xy;
    case NITRO_DIA: return (double)A->dia.inrange * sv + (double)A->dia.D * 4 + xy;
    case NITRO_HYB:
      return (double)A->hyb.K * N * (sv + si) + (double)A->hyb.Zt * (sv + 2 * si) + xy +
             (double)A->hyb.tail_rows * sv;
  }
  return 0.0;
}

}  // namespace nitro
