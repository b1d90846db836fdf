// features.cu — K1: the GPU feature pass (one pass over rowptr + colidx).
//
// Features of P:L97-101 (nnz, num_rows) and P:L200/L209 (AvgNZPerRow, RL-SD,
// MaxDeviation, DIA-Fill, ELL-Fillin) reduce to exact integers:
//   S1 = sum L_i, S2 = sum L_i^2, Lmax = max L_i, D = #distinct (col - row),
// plus the canonical-CSR check (R3).  The doubles are finished on
// the host with the fixed expression of DESIGN.md R4, so GPU and oracle agree
// bit for bit.
//
// Layout of the pass: a warp owns 32 consecutive rows (lane j <-> row j, row
// lengths from two coalesced rowptr loads), then streams the rows' colidx
// range [rowptr[r0], rowptr[r0+32]) with coalesced 32-entry windows.  The row
// of each entry is recovered in O(1) per window from a head mask
// (__reduce_or_sync of 1<<(row start - window base)) and a per-warp row slot
// table, so short and long rows cost the same per entry.  Occupied diagonals
// go to a bitmap over the offset range; a per-block direct-mapped cache of
// recently set offsets plus __match_any_sync dedupe keep the atomics off the
// hot words (a 3D stencil hits only 27 offsets with 3.6e9 entries).
#include "nitro_internal.h"
#include "util.cuh"

#include <cmath>

namespace nitro {
namespace {

constexpr int kThreads = 256;
constexpr int kWarps = kThreads / 32;
constexpr int kCache = 1024;            // per-block open-addressing offset set (u32 keys, 4 KB)
constexpr int kProbe = 4;               // linear-probe length
constexpr uint32_t kWin = 1u << 16;     // per-block bitmap of offsets in [-2^15, 2^15) (8 KB)
constexpr uint32_t kEmpty = 0xffffffffu;
constexpr int kStage = 1024;            // per-warp staging buffer (entries) of the short-row path
constexpr int kRowCap = 64;             // rows longer than this use the windowed path

// Offset index idx = col - row + G is < 2^32 (rows, cols < 2^31), so all
// per-entry arithmetic is 32-bit.  Near-diagonal offsets (stencils, banded)
// are recorded in a shared-memory bitmap window (LDS + rare shared atomic per
// entry); the rest go through a small shared-memory set of offsets already in
// the global bitmap and a test-before-set global OR.  Blocks whose set fills
// up (random matrices) stop probing it.
template <typename IT>
__global__ void __launch_bounds__(kThreads) k_features(const IT *__restrict__ rowptr, const int32_t *__restrict__ col,
                                                        int64_t N, int64_t M, int64_t Z, int64_t row0, int64_t G,
                                                        FeatAcc *__restrict__ acc, uint32_t *__restrict__ bitmap) {
  __shared__ int8_t s_slot[kWarps][32];
  __shared__ int s_stage[kWarps][kStage];
  __shared__ uint32_t s_seen[kCache];
  __shared__ uint32_t s_win[kWin / 32];
  __shared__ unsigned long long s_red[3][kWarps];
  __shared__ unsigned s_bad, s_full;
  for (int i = threadIdx.x; i < kCache; i += kThreads) s_seen[i] = kEmpty;
  for (int i = threadIdx.x; i < (int)(kWin / 32); i += kThreads) s_win[i] = 0u;
  if (threadIdx.x == 0) { s_bad = 0; s_full = 0; }
  __syncthreads();

  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const uint32_t G32 = (uint32_t)G, M32 = (uint32_t)M;
  const uint32_t win_lo = G32 - (kWin >> 1);  // idx of offset -kWin/2 (may wrap: rel test below is modular)
  unsigned bad = 0;
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    if ((int64_t)rowptr[0] != 0 || (int64_t)rowptr[N] != Z) bad |= 1;
  }
  unsigned long long s1 = 0, s2 = 0, lmax = 0;
  const int64_t nblk = (N + 31) / 32;
  const int64_t gw = (int64_t)blockIdx.x * kWarps + wib, nw = (int64_t)gridDim.x * kWarps;
  for (int64_t rb = gw; rb < nblk; rb += nw) {
    const int64_t r = rb * 32 + lane;
    int64_t a, b;
    if (r < N) { a = (int64_t)rowptr[r]; b = (int64_t)rowptr[r + 1]; }
    else { a = b = (int64_t)rowptr[N]; }
    const int64_t L = b - a;
    if (L > 0) {
      s1 += (unsigned long long)L;
      s2 += (unsigned long long)L * (unsigned long long)L;
      if ((unsigned long long)L > lmax) lmax = (unsigned long long)L;
    }
    // a block of rows with a broken rowptr is not walked (flagged)
    const bool brk = L < 0 || a < 0 || b > Z;
    if (__any_sync(kFull, brk)) { bad |= brk ? 1u : 0u; continue; }
    const int64_t E0 = __shfl_sync(kFull, a, 0), E1 = __shfl_sync(kFull, b, 31);
    const uint32_t rowbase = (uint32_t)(row0 + rb * 32);  // global row of lane 0's row
    const bool lane_has = L > 0;
    // ---- fast path (short rows, e.g. stencils / banded): stage the block's
    // colidx span in shared memory with coalesced loads, then every lane walks
    // its own row (row id known, ~10 instructions per entry, no shuffles)
    const int Lmax_blk = (int)__reduce_max_sync(kFull, (unsigned)(L > kRowCap ? kRowCap + 1 : L));
    if (E1 - E0 <= kStage && Lmax_blk <= kRowCap) {
      int *buf = s_stage[wib];
      const int span = (int)(E1 - E0);
      // cp.async (LDGSTS): the whole span is in flight at once, no registers,
      // one memory round trip per block of rows
      for (int e = lane; e < span; e += 32)
        asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"((uint32_t)__cvta_generic_to_shared(buf + e)),
                     "l"(col + E0 + e)
                     : "memory");
      asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;" ::: "memory");
      __syncwarp();
      const int rel0 = (int)(a - E0);
      const uint32_t myrow = rowbase + (uint32_t)lane;
      int prev = -1;
      for (int k = 0; k < (int)L; ++k) {
        const int c = buf[rel0 + k];
        if ((uint32_t)c >= M32) { bad |= 4; continue; }
        if (c <= prev) bad |= 2;
        prev = c;
        const uint32_t idx = (uint32_t)c - myrow + G32;
        const uint32_t rel = idx - win_lo;
        if (rel < kWin) {
          const uint32_t bit = 1u << (rel & 31);
          if (!(s_win[rel >> 5] & bit)) atomicOr(&s_win[rel >> 5], bit);
        } else {
          // far from the diagonal: shared offset set, then test-before-set global OR
          bool hit = false;
          int free_slot = -1;
          if (!s_full) {
            const uint32_t h = idx * 0x9E3779B1u >> 22;
            for (int p = 0; p < kProbe; ++p) {
              const int slot = (int)((h + p) & (kCache - 1));
              const uint32_t cur = s_seen[slot];
              if (cur == idx) { hit = true; break; }
              if (cur == kEmpty) { free_slot = slot; break; }
            }
          }
          if (!hit) {
            // fire-and-forget OR (no returned value, so no per-entry dependent
            // L2 round trip in this per-lane sequential loop)
            atomicOr(bitmap + (idx >> 5), 1u << (idx & 31));
            if (free_slot >= 0) atomicCAS(&s_seen[free_slot], kEmpty, idx);
            else if (!s_full) s_full = 1;
          }
        }
      }
      __syncwarp();  // the staging buffer is reused by the next block of rows
      continue;
    }
    int cur_rl = 0, last_c = 0;
    for (int64_t base = E0; base < E1; base += 128) {
      int c[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int64_t e = base + u * 32 + lane;
        c[u] = e < E1 ? ld_stream_i(col + e) : 0;
      }
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int64_t w0 = base + u * 32;
        if (w0 >= E1) break;  // warp-uniform
        const int nvalid = E1 - w0 < 32 ? (int)(E1 - w0) : 32;
        // rows whose first entry falls in this window: head bit at their start
        const int64_t pos = a - w0;
        const bool head = lane_has && pos >= 0 && pos < 32;
        const unsigned mask = __reduce_or_sync(kFull, head ? (1u << (unsigned)pos) : 0u);
        if (head) s_slot[wib][pos] = (int8_t)lane;
        __syncwarp();
        const unsigned hm = mask & (kFull >> (31 - lane));
        const int rl = hm ? (int)s_slot[wib][31 - __clz(hm)] : cur_rl;
        int prevc = __shfl_up_sync(kFull, c[u], 1);
        if (lane == 0) prevc = last_c;
        uint32_t idx = kEmpty;
        if (lane < nvalid) {
          if ((uint32_t)c[u] >= M32) bad |= 4;  // also catches c < 0
          else {
            if (!((mask >> lane) & 1u) && c[u] <= prevc) bad |= 2;
            idx = (uint32_t)c[u] - (rowbase + (uint32_t)rl) + G32;
          }
        }
        bool want = idx != kEmpty;
        if (want) {
          const uint32_t rel = idx - win_lo;
          if (rel < kWin) {
            const uint32_t bit = 1u << (rel & 31);
            if (!(s_win[rel >> 5] & bit)) atomicOr(&s_win[rel >> 5], bit);
            want = false;
          }
        }
        int free_slot = -1;
        if (want && !s_full) {
          const uint32_t h = idx * 0x9E3779B1u >> 22;  // 10-bit hash
#pragma unroll
          for (int p = 0; p < kProbe; ++p) {
            const int slot = (int)((h + p) & (kCache - 1));
            const uint32_t cur = s_seen[slot];
            if (cur == idx) { want = false; break; }
            if (cur == kEmpty) { free_slot = slot; break; }
          }
        }
        const bool saturated = s_full != 0;  // random offsets: dedupe would not pay
        if (saturated) {
          // fire-and-forget OR per entry: no match_any, no dependent L2 read
          if (want) atomicOr(bitmap + (idx >> 5), 1u << (idx & 31));
        } else {
          const unsigned need = __ballot_sync(kFull, want);
          if (want) {
            const unsigned grp = __match_any_sync(need, idx);
            if ((int)(__ffs(grp) - 1) == lane) {
              // test before set: an L2 read is far cheaper than a contended RED
              const uint32_t bit = 1u << (idx & 31);
              if (!(__ldcg(bitmap + (idx >> 5)) & bit)) atomicOr(bitmap + (idx >> 5), bit);
              if (free_slot >= 0) atomicCAS(&s_seen[free_slot], kEmpty, idx);
              else if (!s_full) s_full = 1;  // probe run full: stop using the set
            }
          }
        }
        cur_rl = __shfl_sync(kFull, rl, nvalid - 1);
        last_c = __shfl_sync(kFull, c[u], nvalid - 1);
        __syncwarp();
      }
    }
  }
  // reduce s1, s2 (sum) and lmax (max) over the block
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    s1 += __shfl_xor_sync(kFull, s1, o);
    s2 += __shfl_xor_sync(kFull, s2, o);
    unsigned long long t = __shfl_xor_sync(kFull, lmax, o);
    lmax = t > lmax ? t : lmax;
  }
  bad = __reduce_or_sync(kFull, bad);
  if (lane == 0) {
    s_red[0][wib] = s1; s_red[1][wib] = s2; s_red[2][wib] = lmax;
    if (bad) atomicOr(&s_bad, bad);
  }
  __syncthreads();
  // merge the near-diagonal window into the global bitmap (nonzero words only)
  const int64_t span = G + M;
  for (int i = threadIdx.x; i < (int)(kWin / 32); i += kThreads) {
    uint32_t w = s_win[i];
    while (w) {
      const int bpos = __ffs(w) - 1;
      w &= w - 1;
      const uint32_t gidx = win_lo + (uint32_t)(i * 32 + bpos);
      if ((int64_t)gidx < span) atomicOr(bitmap + (gidx >> 5), 1u << (gidx & 31));
    }
  }
  if (threadIdx.x == 0) {
    unsigned long long a1 = 0, a2 = 0, am = 0;
    for (int w = 0; w < kWarps; ++w) {
      a1 += s_red[0][w]; a2 += s_red[1][w];
      am = s_red[2][w] > am ? s_red[2][w] : am;
    }
    if (a1) atomicAdd(&acc->s1, a1);
    if (a2) atomicAdd(&acc->s2, a2);
    if (am) atomicMax(&acc->lmax, am);
    if (s_bad) atomicOr(&acc->bad, s_bad);
  }
}

__global__ void __launch_bounds__(256) k_popc(const uint32_t *__restrict__ bm, int64_t nwords, FeatAcc *acc) {
  unsigned long long s = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nwords; i += (int64_t)gridDim.x * blockDim.x)
    s += __popc(bm[i]);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(kFull, s, o);
  if ((threadIdx.x & 31) == 0 && s) atomicAdd(&acc->ndiag, s);
}

}  // namespace

void finish_features(int64_t N, int64_t M, int64_t Z, uint64_t s1, uint64_t s2, int64_t lmax, int64_t D,
                     nitro_spmv_feat *f) {
  // DESIGN.md R4 — fixed fp64 expression (compiled with -ffp-contract=off)
  f->rows = N; f->cols = M; f->nnz = Z;
  f->sum_len = s1; f->sum_len2 = s2; f->max_row = lmax; f->ndiag = D;
  f->mean = f->sd = f->max_dev = f->dia_fill = f->ell_fill = 0.0;
  if (N == 0) return;
  const double n = (double)N;
  const __int128 num = (__int128)N * (__int128)s2 - (__int128)s1 * (__int128)s1;
  const double zz = (double)(Z > 1 ? Z : 1);
  f->mean = (double)s1 / n;
  f->sd = std::sqrt((double)num / (n * n));
  f->max_dev = (double)lmax - f->mean;
  f->dia_fill = (double)D * n / zz;
  f->ell_fill = (double)lmax * n / zz;
}

nitro_status_t features_launch(nitro_spmv *A) {
  if (A->feat_ready || A->feat_pending) return NITRO_OK;
  cudaStream_t s = A->stream;
  const int64_t G = diag_shift(A);                 // bitmap index = d + G
  const int64_t span = A->N > 0 ? G + A->M : 0;    // offsets in [-G, M-1]
  const int64_t nwords = (span + 31) / 32;
  NITRO_TRY(A->feat_acc.alloc(sizeof(FeatAcc)));
  NITRO_TRY(A->bitmap.alloc((size_t)(nwords > 0 ? nwords : 1) * 4));
  if (!A->h_acc) NITRO_CUDA(cudaMallocHost(&A->h_acc, sizeof(FeatAcc)));
  if (!A->feat_done) NITRO_CUDA(cudaEventCreateWithFlags(&A->feat_done, cudaEventDisableTiming));
  FeatAcc *acc = A->feat_acc.as<FeatAcc>();
  NITRO_CUDA(cudaMemsetAsync(acc, 0, sizeof(FeatAcc), s));
  if (nwords) NITRO_CUDA(cudaMemsetAsync(A->bitmap.p, 0, (size_t)nwords * 4, s));
  const int64_t nblk = (A->N + 31) / 32;
  int64_t grid = (nblk + kWarps - 1) / kWarps;
  const int64_t cap = (int64_t)num_sms() * 8;
  if (grid > cap) grid = cap;
  if (grid < 1) grid = 1;
  if (A->rp64)
    k_features<int64_t><<<(unsigned)grid, kThreads, 0, s>>>((const int64_t *)A->rowptr, A->col, A->N, A->M, A->Z,
                                                            A->row0, G, acc, A->bitmap.as<uint32_t>());
  else
    k_features<int32_t><<<(unsigned)grid, kThreads, 0, s>>>((const int32_t *)A->rowptr, A->col, A->N, A->M, A->Z,
                                                            A->row0, G, acc, A->bitmap.as<uint32_t>());
  if (nwords) {
    int64_t g2 = (nwords + 255) / 256;
    if (g2 > (int64_t)num_sms() * 8) g2 = (int64_t)num_sms() * 8;
    k_popc<<<(unsigned)g2, 256, 0, s>>>(A->bitmap.as<uint32_t>(), nwords, acc);
  }
  NITRO_CUDA(cudaGetLastError());
  NITRO_CUDA(cudaMemcpyAsync(A->h_acc, acc, sizeof(FeatAcc), cudaMemcpyDeviceToHost, s));
  NITRO_CUDA(cudaEventRecord(A->feat_done, s));
  A->feat_pending = true;
  return NITRO_OK;
}

nitro_status_t features_finish(nitro_spmv *A) {
  if (A->feat_ready) return A->feat.canonical ? NITRO_OK : fail(NITRO_E_BAD_MATRIX, "non-canonical CSR");
  if (!A->feat_pending) NITRO_TRY(features_launch(A));
  NITRO_CUDA(cudaEventSynchronize(A->feat_done));
  A->feat_pending = false;
  const FeatAcc &h = *A->h_acc;
  finish_features(A->N, A->M, A->Z, h.s1, h.s2, (int64_t)h.lmax, (int64_t)h.ndiag, &A->feat);
  A->feat.canonical = h.bad == 0;
  A->feat_ready = true;
  if (!A->feat.canonical) {
    const char *why = (h.bad & 1) ? "rowptr not monotone from 0 to nnz"
                      : (h.bad & 4) ? "column index out of [0, cols)" : "columns not strictly increasing in a row";
    return fail(NITRO_E_BAD_MATRIX, std::string("non-canonical CSR: ") + why);
  }
  return NITRO_OK;
}

}  // namespace nitro
