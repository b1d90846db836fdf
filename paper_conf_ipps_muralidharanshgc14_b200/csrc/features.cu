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
// lengths from two coalesced rowptr loads).  Rows of up to kRowCap entries are
// walked by their own lane (row id known, no shuffles), from a shared-memory
// copy of the rows' colidx span when it fits (cp.async, bank-skewed), else
// straight from global memory in 8-entry batches.  Longer rows are walked by
// the whole warp, 32 coalesced entries at a time; rows longer than kLong are
// deferred to k_features_long, which splits them into kChunk-entry chunks
// spread over every warp of the grid (an R-MAT hub row of 1.5e5 entries would
// otherwise serialise on one warp).  Occupied diagonals go to a bitmap over the
// offset range: near-diagonal offsets through a per-block shared-memory window,
// the rest through a per-block set of offsets already set (until it fills up:
// random matrices) and fire-and-forget global ORs, merged per 32-bit word
// across a warp's window by a segmented OR scan (a dense row then costs one
// OR per word, not per entry).
#include "nitro_internal.h"
#include "util.cuh"

#include <algorithm>
#include <cmath>

namespace nitro {
namespace {

constexpr int kThreads = 256;
constexpr int kWarps = kThreads / 32;
constexpr int kCache = 512;             // per-block open-addressing offset set (u32 keys, 2 KB)
constexpr int kProbe = 4;               // linear-probe length
constexpr uint32_t kWin = 1u << 16;     // per-block bitmap of offsets in [-2^15, 2^15) (8 KB)
constexpr uint32_t kEmpty = 0xffffffffu;
#ifndef NITRO_K1_STAGE
#define NITRO_K1_STAGE 1024
#endif
#ifndef NITRO_K1_MINB
#define NITRO_K1_MINB 4  // 4 resident CTAs per SM: <= 64 registers (at 66 the pass lost 10 %)
#endif
constexpr int kStage = NITRO_K1_STAGE;  // per-warp staging buffer (entries)
constexpr int kRowCap = 64;             // lane-per-row walk only for rows up to this length
constexpr int kQ = 4;                   // 32-row blocks per super-block (one staging round trip for short rows)
constexpr int64_t kLong = 4096;         // rows longer than this go to k_features_long
constexpr int64_t kChunk = 4096;        // entries per task of k_features_long
constexpr int kPatMin = 8;              // shifted-row test for lane-walked blocks with rows of >= this many entries
constexpr int kPatRows = 8;             // ... taken when at most this many of the 32 rows fail the quick test

// staging slot of span entry e (relative to a 16-byte aligned base): four pad
// words per 32 entries, so 16-byte chunks stay aligned (cp.async of 16 bytes)
// and lanes walking rows of 32 entries meet at most 4 to a bank (odd lengths:
// none)
__device__ __forceinline__ int skew(int e) { return e + ((e >> 5) << 2); }

// cp.async of the colidx span [E0, E1) into buf at slots skew(e - E0a), E0a =
// E0 rounded down to a 16-byte boundary of the column array: aligned 16-byte
// chunks, the partial chunks at both ends entry by entry (no read outside
// [E0, E1)).  Returns E0a; the caller waits (cp.async.wait_group 0).
__device__ __forceinline__ int64_t stage_span(int *buf, const int32_t *__restrict__ col, int64_t E0, int64_t E1,
                                              int lane) {
  const int h = (int)((reinterpret_cast<uintptr_t>(col + E0) >> 2) & 3);
  const int64_t E0a = E0 - h;
  const int span = (int)(E1 - E0a);
  const int lo = h ? 4 : 0, hi = span & ~3;
  const uint32_t sb = (uint32_t)__cvta_generic_to_shared(buf);
  const int32_t *g = col + E0a;
  {  // skew(q + 128) = skew(q) + 144: both addresses advance by constants
    const int32_t *gq = g + lo + 4 * lane;
    uint32_t sq = sb + 4u * (uint32_t)skew(lo + 4 * lane);
    for (int q = lo + 4 * lane; q < hi; q += 128, gq += 128, sq += 144u * 4u)
      // .cg: the column stream bypasses L1 (read once; B200 A/B vs .ca: configs[4] 3.42 -> 2.95 ms,
      // configs[1] 0.079 -> 0.073 ms, uniform random rows +3 %)
      asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(sq), "l"(gq) : "memory");
  }
  // head [h, min(lo, span)) and tail [max(hi, lo), span): at most 3 + 3 entries
  const int e = lane < 3 ? h + lane : (hi > lo ? hi : lo) + lane - 3;
  if ((lane < 3 && e < lo && e < span) || (lane >= 3 && lane < 6 && e < span))
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(sb + 4u * (uint32_t)skew(e)), "l"(g + e) : "memory");
  asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;" ::: "memory");
  return E0a;
}

// The offset bits of one 32-entry window held one per lane (key = bitmap word
// or kEmpty, bits = its bit): a segmented inclusive OR scan merges runs of
// equal adjacent keys, and the last lane of each run issues one global OR (a
// dense row costs one OR per word, not per entry).
__device__ __forceinline__ void or_window(uint32_t key, uint32_t bits, int lane, uint32_t *__restrict__ bitmap) {
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t tb = __shfl_up_sync(kFull, bits, o);
    const uint32_t tk = __shfl_up_sync(kFull, key, o);
    if (lane >= o && tk == key) bits |= tb;
  }
  const uint32_t nk = __shfl_down_sync(kFull, key, 1);
  if (key != kEmpty && (lane == 31 || nk != key)) atomicOr(bitmap + key, bits);
}

// Offset index idx of an entry -> near-diagonal window bit (shared) or a
// (key, bits) pair for or_window.
__device__ __forceinline__ void classify(uint32_t idx, uint32_t win_lo, uint32_t *s_win, uint32_t &key,
                                         uint32_t &bits) {
  const uint32_t rel = idx - win_lo;
  if (s_win && rel < kWin) {
    const uint32_t bit = 1u << (rel & 31);
    if (!(s_win[rel >> 5] & bit)) atomicOr(&s_win[rel >> 5], bit);
  } else {
    key = idx >> 5;
    bits = 1u << (idx & 31);
  }
}

// Whole-warp walk of one row's entries [st, en) (row start a, global row grow):
// canonical checks against the previous entry, offsets to the window / bitmap.
__device__ __forceinline__ void walk_row_warp(const int32_t *__restrict__ col, int64_t st, int64_t en, int64_t a,
                                              uint32_t grow, uint32_t G32, uint32_t M32, uint32_t win_lo,
                                              uint32_t *s_win, uint32_t *__restrict__ bitmap, int lane,
                                              unsigned &bad) {
  int last_c = st > a ? __ldg(col + st - 1) : -1;
  for (int64_t base = st; base < en; base += 128) {
    int c[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const int64_t e = base + u * 32 + lane;
      c[u] = e < en ? ld_stream_i(col + e) : 0;
    }
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const int64_t w0 = base + u * 32;
      if (w0 >= en) break;  // warp-uniform
      int prevc = __shfl_up_sync(kFull, c[u], 1);
      if (lane == 0) prevc = last_c;
      uint32_t key = kEmpty, bits = 0;
      if (w0 + lane < en) {
        if ((uint32_t)c[u] >= M32) bad |= 4;  // also catches c < 0
        else {
          if (c[u] <= prevc) bad |= 2;
          classify((uint32_t)c[u] - grow + G32, win_lo, s_win, key, bits);
        }
      }
      or_window(key, bits, lane, bitmap);
      last_c = __shfl_sync(kFull, c[u], 31);
    }
  }
}

// Whole-warp walk of the contiguous entry range [st, en) of the rows
// (lanes) flagged in_run of a 32-row block, entries from the staging buffer
// (SMEM, slots relative to E0) or global memory.  The row of each entry comes
// from the head mask of the window (bit p set <=> a row starts at window entry
// p, __reduce_or_sync) and a per-warp table head position -> lane.
template <bool SMEM>
__device__ __forceinline__ void walk_span_warp(const int32_t *__restrict__ src, int64_t st, int64_t en, int64_t E0,
                                               int64_t a, bool in_run, uint32_t rowbase, uint32_t G32,
                                               uint32_t M32, uint32_t win_lo, uint32_t *s_win, int8_t *slot,
                                               uint32_t *__restrict__ bitmap, int lane, unsigned &bad) {
  int cur_rl = 0, last_c = 0;
  for (int64_t base = st; base < en; base += 128) {
    int c[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const int64_t e = base + u * 32 + lane;
      c[u] = e < en ? (SMEM ? src[skew((int)(e - E0))] : ld_stream_i(src + e)) : 0;
    }
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const int64_t w0 = base + u * 32;
      if (w0 >= en) break;  // warp-uniform
      const int nvalid = en - w0 < 32 ? (int)(en - w0) : 32;
      const int64_t pos = a - w0;
      const bool head = in_run && pos >= 0 && pos < nvalid;
      const unsigned mask = __reduce_or_sync(kFull, head ? (1u << (unsigned)pos) : 0u);
      if (head) slot[pos] = (int8_t)lane;  // in_run excludes empty rows: one head per position
      __syncwarp();
      const unsigned hm = mask & (kFull >> (31 - lane));
      const int rl = hm ? (int)slot[31 - __clz(hm)] : cur_rl;
      int prevc = __shfl_up_sync(kFull, c[u], 1);
      if (lane == 0) prevc = last_c;
      uint32_t key = kEmpty, bits = 0;
      if (lane < nvalid) {
        if ((uint32_t)c[u] >= M32) bad |= 4;
        else {
          if (!((mask >> lane) & 1u) && c[u] <= prevc) bad |= 2;
          classify((uint32_t)c[u] - (rowbase + (uint32_t)rl) + G32, win_lo, s_win, key, bits);
        }
      }
      or_window(key, bits, lane, bitmap);
      cur_rl = __shfl_sync(kFull, rl, nvalid - 1);
      last_c = __shfl_sync(kFull, c[u], nvalid - 1);
      __syncwarp();
    }
  }
}

// merge a block's near-diagonal window into the global bitmap (nonzero words only)
__device__ __forceinline__ void merge_window(const uint32_t *s_win, uint32_t win_lo, int64_t span,
                                             uint32_t *__restrict__ bitmap) {
  for (int i = threadIdx.x; i < (int)(kWin / 32); i += blockDim.x) {
    uint32_t w = s_win[i];
    while (w) {
      const int bpos = __ffs(w) - 1;
      w &= w - 1;
      const uint32_t gidx = win_lo + (uint32_t)(i * 32 + bpos);
      if ((int64_t)gidx < span) atomicOr(bitmap + (gidx >> 5), 1u << (gidx & 31));
    }
  }
}

// Offset index idx = col - row + G is < 2^32 (rows, cols < 2^31), so all
// per-entry arithmetic is 32-bit.
template <typename IT>
__global__ void __launch_bounds__(kThreads, NITRO_K1_MINB) k_features(const IT *__restrict__ rowptr, const int32_t *__restrict__ col,
                                                        int64_t N, int64_t M, int64_t Z, int64_t row0, int64_t G,
                                                        FeatAcc *__restrict__ acc, uint32_t *__restrict__ bitmap,
                                                        int2 *__restrict__ tasks, int64_t cap_tasks) {
  __shared__ __align__(16) int s_stage[kWarps][kStage + 4 + (kStage + 4) / 8];  // skew(kStage + 3) < this
  __shared__ int8_t s_slot[kWarps][32];
  __shared__ uint32_t s_seen[kCache];
  __shared__ uint32_t s_win[kWin / 32];
  __shared__ unsigned long long s_red[3][kWarps];
  __shared__ unsigned s_bad, s_full;
  for (int i = threadIdx.x; i < kCache; i += kThreads) s_seen[i] = kEmpty;
  for (int i = threadIdx.x; i < (int)(kWin / 32); i += kThreads) s_win[i] = 0u;
  if (threadIdx.x == 0) { s_bad = 0; s_full = 0; }
  pdl_trigger();  // k_features_long may be scheduled as CTAs of this grid retire
  pdl_wait();     // the bitmap / FeatAcc zeroing (k_feat_zero) is complete
  __syncthreads();

  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const uint32_t G32 = (uint32_t)G, M32 = (uint32_t)M;
  const uint32_t win_lo = G32 - (kWin >> 1);  // idx of offset -kWin/2 (may wrap: rel test below is modular)
  unsigned bad = 0;
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    if ((int64_t)rowptr[0] != 0 || (int64_t)rowptr[N] != Z) bad |= 1;
  }
  // a far (off-window) offset of a lane-walked row: shared offset set (until it
  // fills: full), then a fire-and-forget global OR (no returned value, so no
  // dependent L2 round trip)
  auto lane_far = [&](uint32_t idx, bool full) {
    // (testing the bit with an L1-cached read before the OR was measured: no
    // gain on configs[2] uniform — 1.529 vs 1.546 ms, the random sector access
    // costs the same as the fire-and-forget OR — and 1.8x slower on short random rows)
    if (full) { atomicOr(bitmap + (idx >> 5), 1u << (idx & 31)); return; }
    bool hit = false;
    int free_slot = -1;
    const uint32_t h = idx * 0x9E3779B1u >> 22;
    for (int p = 0; p < kProbe; ++p) {
      const int slot = (int)((h + p) & (kCache - 1));
      const uint32_t cur = s_seen[slot];
      if (cur == idx) { hit = true; break; }
      if (cur == kEmpty) { free_slot = slot; break; }
    }
    if (!hit) {
      atomicOr(bitmap + (idx >> 5), 1u << (idx & 31));
      if (free_slot >= 0) atomicCAS(&s_seen[free_slot], kEmpty, idx);
      else s_full = 1;
    }
  };

  unsigned long long s1 = 0, s2 = 0, lmax = 0;
  const int64_t nblk = (N + 31) / 32;
  const int64_t gw = (int64_t)blockIdx.x * kWarps + wib, nw = (int64_t)gridDim.x * kWarps;
  // Lane-per-row walk of one row of L entries (staged at buf slots rel0.., or
  // from global memory at entry a).  Per entry: strictly-increasing check
  // (with prev = -1 it also gives c >= 0; c < M then follows from the last
  // entry), and the offset's window bit rel = c - row + kWin/2 tested before
  // it is set.  The bound checks sit outside the loop: the pass is issue-bound
  // on stencils (ncu: SM throughput 74 %, IPC 3.2), so instructions per entry
  // are what the loop is tuned for.
  // (Collecting a row's window bits per 32-bit word in registers and testing /
  // ORing the shared word once per run, through 32-bit shared addresses, was
  // measured slower: configs[1] 0.131 -> 0.140 ms, configs[4] 5.75 -> 6.18 ms.)
  // the window through 32-bit shared addresses computed once (the generic
  // form re-derived the window's shared address on every entry: S2R + 4 ops)
  const uint32_t win_sa = (uint32_t)__cvta_generic_to_shared(s_win);
  auto lane_walk_core = [&](auto ld, int L, uint32_t myrow, bool full) {
    const uint32_t rbase = myrow - (kWin >> 1);
    int prev = -1;
    bool inc = true;
#pragma unroll 4
    for (int k = 0; k < L; ++k) {
      const int c = ld(k);
      inc &= c > prev;
      prev = c;
      const uint32_t rel = (uint32_t)c - rbase;
      if (rel < kWin) {
        const uint32_t bit = 1u << (rel & 31), a = win_sa + ((rel >> 5) << 2);
        uint32_t w;
        asm volatile("ld.shared.u32 %0, [%1];" : "=r"(w) : "r"(a));
        if (!(w & bit)) asm volatile("red.shared.or.b32 [%0], %1;" ::"r"(a), "r"(bit) : "memory");
      } else if ((uint32_t)c < M32) {
        lane_far((uint32_t)c - myrow + G32, full);
      }
    }
    const int first = ld(0);
    if (first < 0 || (uint32_t)prev >= M32) bad |= 4;
    else if (!inc) bad |= 2;
  };
  auto lane_walk_staged = [&](const int *buf, int rel0, int L, uint32_t myrow, bool full) {
    lane_walk_core([&](int k) { return buf[skew(rel0 + k)]; }, L, myrow, full);
  };
  auto lane_walk_global = [&](int64_t a, int L, uint32_t myrow, bool full) {
    lane_walk_core([&](int k) { return __ldg(col + a + k); }, L, myrow, full);
  };
  // Whole-warp walk of one staged row (lane = entry; L <= kRowCap: two steps):
  // canonical checks and the offsets of that row, as lane_walk_core.
  auto row_walk_lanes = [&](auto ld, int L, uint32_t row, bool full) {
    const uint32_t rbase = row - (kWin >> 1);
    int lastc = -1;
    for (int k0 = 0; k0 < L; k0 += 32) {
      const int k = k0 + lane;
      const int c = k < L ? ld(k) : 0;
      int prevc = __shfl_up_sync(kFull, c, 1);
      if (lane == 0) prevc = lastc;
      if (k < L) {
        if ((uint32_t)c >= M32) bad |= 4;  // also catches c < 0
        else {
          if (c <= prevc) bad |= 2;
          const uint32_t rel = (uint32_t)c - rbase;
          if (rel < kWin) {
            const uint32_t bit = 1u << (rel & 31), a = win_sa + ((rel >> 5) << 2);
            uint32_t w;
            asm volatile("ld.shared.u32 %0, [%1];" : "=r"(w) : "r"(a));
            if (!(w & bit)) asm volatile("red.shared.or.b32 [%0], %1;" ::"r"(a), "r"(bit) : "memory");
          } else {
            lane_far((uint32_t)c - row + G32, full);
          }
        }
      }
      lastc = __shfl_sync(kFull, c, 31);
    }
  };
  // Shifted rows (stencils, bands): row j whose entries are row j-1's plus one,
  // entry by entry (same length), has row j-1's offsets c - row, so only the
  // rows that are not such a shift of their predecessor are walked (lane =
  // entry, above); a shifted row adds one check: its last column < M (strictly
  // increasing and >= 0 follow from row j-1).  A first test on the lengths and
  // the first and last entries; when more than kPatRows rows of the 32 fail it
  // (random columns) the warp returns false and walks lane per row instead.
  // Warp-collective; L = this lane's row length, rel0 its staged start.
  auto pattern_walk = [&](const int *buf, int rel0, int L, uint32_t myrow, bool full) -> bool {
    const int relp = __shfl_up_sync(kFull, rel0, 1);
    const int Lp = __shfl_up_sync(kFull, L, 1);
    bool shifted = lane > 0 && L > 1 && L == Lp;
    if (shifted)
      shifted = buf[skew(rel0)] == buf[skew(relp)] + 1 && buf[skew(rel0 + L - 1)] == buf[skew(relp + L - 1)] + 1;
    if (__popc(__ballot_sync(kFull, L > 0 && !shifted)) > kPatRows) return false;
    // entries 1 .. L-2 against the predecessor's through a shuffle (a shifted
    // lane's predecessor has the same length, so it loads the same k)
    const int Lw = __reduce_max_sync(kFull, (unsigned)L);
#pragma unroll 4
    for (int k = 1; k < Lw - 1; ++k) {
      const int c = k < L ? buf[skew(rel0 + k)] : 0;
      const int cp = __shfl_up_sync(kFull, c, 1);
      shifted &= k >= L - 1 || c == cp + 1;
    }
    if (shifted && (uint32_t)buf[skew(rel0 + L - 1)] >= M32) bad |= 4;
    unsigned todo = __ballot_sync(kFull, L > 0 && !shifted);
    while (todo) {
      const int j = __ffs(todo) - 1;
      todo &= todo - 1;
      const int rj = __shfl_sync(kFull, rel0, j);
      row_walk_lanes([&](int k) { return buf[skew(rj + k)]; }, __shfl_sync(kFull, L, j), myrow - lane + j, full);
    }
    return true;
  };

  // A run of consecutive rows j0..j1 of the block all of the maximum length L
  // (interior stencil rows: the whole block; a block holding a grid-line
  // boundary row: all but one or two rows): the shift of each row j0 < j <= j1
  // against row j - 1 is checked position-parallel over the run's staged span
  // — entry e == entry e - L, plus 1 (lane = position: coalesced,
  // conflict-free) — then only row j0 and the rows outside the run are walked
  // (lane = entry).  skew(e + 32) = skew(e) + 36, so both shared addresses
  // advance by a constant (no per-entry skew arithmetic).  False: the rows at
  // the maximum length are not one run, or some row is not a shift
  // (pattern_walk finds which).
  auto run_walk = [&](const int *buf, int rel0, int L, int Lmax, uint32_t rowbase, bool full) -> bool {
    const unsigned m = __ballot_sync(kFull, L == Lmax);
    const int j0 = __ffs(m) - 1, j1 = 31 - __clz(m);
    if (j1 - j0 < 15 || m != ((kFull >> (31 - j1)) & (kFull << j0))) return false;
    const int h = __shfl_sync(kFull, rel0, j0);
    const int span = (j1 - j0 + 1) * Lmax;
    const uint32_t sb = (uint32_t)__cvta_generic_to_shared(buf);
    uint32_t a1 = sb + 4u * (uint32_t)skew(h + Lmax + lane);
    const uint32_t d = a1 - (sb + 4u * (uint32_t)skew(h + lane));
    bool ok = true;
#pragma unroll 4
    for (int e = Lmax + lane; e < span; e += 32, a1 += 36u * 4u) {
      int v1, v0;
      asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v1) : "r"(a1));
      asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v0) : "r"(a1 - d));
      ok &= v1 == v0 + 1;
    }
    if (!__all_sync(kFull, ok)) return false;
    row_walk_lanes([&](int k) { return buf[skew(h + k)]; }, Lmax, rowbase + (uint32_t)j0, full);
    if (lane == 0 && (uint32_t)buf[skew(h + span - 1)] >= M32) bad |= 4;  // row j1's last column
    unsigned todo = __ballot_sync(kFull, L > 0) & ~m;
    while (todo) {
      const int j = __ffs(todo) - 1;
      todo &= todo - 1;
      const int rj = __shfl_sync(kFull, rel0, j);
      row_walk_lanes([&](int k) { return buf[skew(rj + k)]; }, __shfl_sync(kFull, L, j), rowbase + (uint32_t)j, full);
    }
    return true;
  };
  int pat_skip = 0;  // warp-uniform
  // One block of 32 rows (lane j <-> row rb*32 + j) with its row bounds a, b.
  auto process_block = [&](int64_t rb, int64_t a, int64_t b) {
    const int64_t r = rb * 32 + lane;
    const int64_t L = b - a;
    if (L > 0) {
      s1 += (unsigned long long)L;
      s2 += (unsigned long long)L * (unsigned long long)L;
      if ((unsigned long long)L > lmax) lmax = (unsigned long long)L;
    }
    // a block of rows with a broken rowptr is not walked (flagged)
    const bool brk = L < 0 || a < 0 || b > Z;
    if (__any_sync(kFull, brk)) { bad |= brk ? 1u : 0u; return; }
    const int64_t E0 = __shfl_sync(kFull, a, 0), E1 = __shfl_sync(kFull, b, 31);
    const uint32_t rowbase = (uint32_t)(row0 + rb * 32), myrow = rowbase + (uint32_t)lane;
    // long rows: their kChunk-entry chunks become tasks of k_features_long
    const bool is_long = L > kLong;
    if (is_long) {
      const int nc = (int)((L + kChunk - 1) / kChunk);
      const unsigned t0 = atomicAdd(&acc->nlong, (unsigned)nc);
      // a malformed rowptr (rows overlapping, each within [0, Z]) can list more
      // chunks than a monotone one: flag it instead of writing past the list
      if ((int64_t)t0 + nc > cap_tasks) bad |= 1;
      else
        for (int j = 0; j < nc; ++j) tasks[t0 + j] = make_int2((int)r, j);
    }
    const unsigned long_mask = __ballot_sync(kFull, is_long);
    const bool staged = E1 - E0 <= kStage;  // implies no long row
    int *buf = s_stage[wib];
    int64_t E0a = E0;
    if (staged) {
      // cp.async (LDGSTS): the whole span is in flight at once, no registers,
      // one memory round trip per block of rows
      E0a = stage_span(buf, col, E0, E1, lane);
      __syncwarp();
    }
    // lane per row when the rows are short and of similar length (stencils,
    // uniform rows: no divergence), else the whole warp over the entry span
    const int64_t Ln = is_long ? 0 : L;
    const unsigned maxL = __reduce_max_sync(kFull, (unsigned)(Ln > kRowCap ? kRowCap + 1 : Ln));
    const unsigned sumL = __reduce_add_sync(kFull, (unsigned)(Ln > kRowCap ? kRowCap + 1 : Ln));
    if (maxL <= (unsigned)kRowCap && maxL * 32u <= 2u * sumL) {
      const bool full = *(volatile unsigned *)&s_full != 0;
      bool done = false;
      if (staged && maxL >= (unsigned)kPatMin && maxL * 32u <= sumL + 32u) {  // near-equal lengths
        if (pat_skip > 0) --pat_skip;  // the test failed on a recent block of this warp: random rows
        else {
          done = run_walk(buf, (int)(a - E0a), (int)Ln, (int)maxL, rowbase, full);
          if (!done && !(done = pattern_walk(buf, (int)(a - E0a), (int)Ln, myrow, full))) pat_skip = 16;
        }
      }
      if (done) {
      } else if (Ln > 0) {
        if (staged) lane_walk_staged(buf, (int)(a - E0a), (int)Ln, myrow, full);
        else lane_walk_global(a, (int)Ln, myrow, full);
      }
    } else if (staged) {
      walk_span_warp<true>(buf, E0, E1, E0a, a, L > 0, rowbase, G32, M32, win_lo, s_win, s_slot[wib], bitmap, lane,
                           bad);
    } else {
      // runs of consecutive non-long rows between the long ones
      int s = 0;
      while (s < 32) {
        const unsigned rest = long_mask >> s;
        const int l = rest ? s + __ffs(rest) - 1 : 32;  // first long lane at or after s
        if (l > s) {
          const int64_t st = __shfl_sync(kFull, a, s);
          const int64_t en = __shfl_sync(kFull, a, l & 31);
          const int64_t en2 = l < 32 ? en : E1;
          walk_span_warp<false>(col, st, en2, 0, a, lane >= s && lane < l && L > 0, rowbase, G32, M32, win_lo, s_win,
                                s_slot[wib], bitmap, lane, bad);
        }
        s = l + 1;
      }
    }
    __syncwarp();  // the staging buffer is reused by the next block of rows
  };
  // Super-blocks of kQ consecutive 32-row blocks: the rowptr loads of all kQ
  // blocks are issued together, and when every block takes the lane-per-row
  // walk and their joint colidx span fits the staging buffer (short rows:
  // stencils of low order, sparse bands, short random rows) that span is
  // staged by ONE cp.async round trip — the walk of short rows is latency-
  // bound per iteration, so kQ blocks per round trip is up to kQ x faster.
  // Otherwise each block goes through process_block as before.
  const int64_t nsb = (nblk + kQ - 1) / kQ;
  // register array element j < kQ for a runtime j (no local-memory indexing)
  auto pick = [](const int64_t (&v)[kQ], int j) {
    int64_t r = v[0];
#pragma unroll
    for (int t = 1; t < kQ; ++t) r = j == t ? v[t] : r;
    return r;
  };
  for (int64_t sb = gw; sb < nsb; sb += nw) {
    int64_t a[kQ], b[kQ];
#pragma unroll
    for (int j = 0; j < kQ; ++j) {
      const int64_t r = (sb * kQ + j) * 32 + lane;
      if (r < N) { a[j] = (int64_t)rowptr[r]; b[j] = (int64_t)rowptr[r + 1]; }
      else { a[j] = b[j] = -1; }
    }
    const bool full_sb = (sb + 1) * kQ <= nblk;
    // the joint span first (one pair of shuffles): longer rows skip the per-block tests
    bool fast = full_sb && __shfl_sync(kFull, b[kQ - 1], 31) - __shfl_sync(kFull, a[0], 0) <= kStage / 2;
    unsigned mx[kQ];
    if (fast) {
#pragma unroll
      for (int j = 0; j < kQ; ++j) {
        const int64_t L = b[j] - a[j];
        const bool brk = L < 0 || a[j] < 0 || b[j] > Z;
        const unsigned Lc = brk ? (unsigned)(kRowCap + 1) : (unsigned)(L > kRowCap ? kRowCap + 1 : L);
        mx[j] = __reduce_max_sync(kFull, Lc);
        const unsigned sm = __reduce_add_sync(kFull, Lc);
        fast = fast && mx[j] <= (unsigned)kRowCap && mx[j] * 32u <= 2u * sm;
      }
      // contiguous blocks: block j ends where block j + 1 starts (else rowptr is broken)
      if (fast) {
        const int64_t A0 = __shfl_sync(kFull, a[0], 0), B1 = __shfl_sync(kFull, b[kQ - 1], 31);
        bool cont = true;
#pragma unroll
        for (int j = 0; j + 1 < kQ; ++j) cont = cont && __shfl_sync(kFull, b[j], 31) == __shfl_sync(kFull, a[j + 1], 0);
        fast = cont && B1 - A0 <= kStage / 2 && B1 >= A0;  // short rows only (band01-like spans: slower)
      }
    }
    if (!fast) {
#pragma unroll 1
      for (int j = 0; j < kQ; ++j) {
        const int64_t rb = sb * kQ + j;
        if (rb >= nblk) break;
        const int64_t r = rb * 32 + lane;
        // reloaded (L1 hits) rather than kept live across process_block: registers
        const int64_t aa = (int64_t)rowptr[r < N ? r : N], bb = (int64_t)rowptr[r < N ? r + 1 : N];
        process_block(rb, aa, bb);
      }
      continue;
    }
    const int64_t E0 = __shfl_sync(kFull, a[0], 0), E1 = __shfl_sync(kFull, b[kQ - 1], 31);
    int *buf = s_stage[wib];
    const int64_t E0a = stage_span(buf, col, E0, E1, lane);
    __syncwarp();
    const bool full = *(volatile unsigned *)&s_full != 0;
#pragma unroll 1
    for (int j = 0; j < kQ; ++j) {
      const int64_t aj = pick(a, j), L = pick(b, j) - aj;
      if (L > 0) {
        s1 += (unsigned long long)L;
        s2 += (unsigned long long)L * (unsigned long long)L;
        if ((unsigned long long)L > lmax) lmax = (unsigned long long)L;
        const uint32_t myrow = (uint32_t)(row0 + (sb * kQ + j) * 32 + lane);
        lane_walk_staged(buf, (int)(aj - E0a), (int)L, myrow, full);
      }
    }
    __syncwarp();  // the staging buffer is reused by the next iteration
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
  merge_window(s_win, win_lo, G + M, bitmap);
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

// The long rows' chunks (row, j) listed by k_features, one warp per task,
// grid-stride over the task list.
template <typename IT>
__global__ void __launch_bounds__(kThreads) k_features_long(const IT *__restrict__ rowptr,
                                                             const int32_t *__restrict__ col, int64_t M, int64_t row0,
                                                             int64_t G, FeatAcc *__restrict__ acc,
                                                             uint32_t *__restrict__ bitmap,
                                                             const int2 *__restrict__ tasks, int64_t cap_tasks) {
  pdl_trigger();
  pdl_wait();  // k_features has listed every long-row task
  const int64_t n0 = (int64_t)*(volatile unsigned *)&acc->nlong;
  const int64_t n = n0 < cap_tasks ? n0 : cap_tasks;  // more = malformed rowptr (flagged by k_features)
  const int lane = threadIdx.x & 31;
  const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const uint32_t G32 = (uint32_t)G, M32 = (uint32_t)M;
  unsigned bad = 0;
  for (int64_t t = gw; t < n; t += nw) {
    const int2 tk = tasks[t];
    const int64_t a = (int64_t)rowptr[tk.x], b = (int64_t)rowptr[tk.x + 1];
    const int64_t st = a + (int64_t)tk.y * kChunk, en = st + kChunk < b ? st + kChunk : b;
    walk_row_warp(col, st, en, a, (uint32_t)(row0 + tk.x), G32, M32, 0u, nullptr, bitmap, lane, bad);
  }
  bad = __reduce_or_sync(kFull, bad);
  if (lane == 0 && bad) atomicOr(&acc->bad, bad);
}

// Row-length moments only (the cheap feature level): rowptr read once.
template <typename IT>
__global__ void __launch_bounds__(256) k_rowstats(const IT *__restrict__ rowptr, int64_t N, int64_t Z,
                                                  FeatAcc *__restrict__ acc) {
  __shared__ unsigned long long s_red[3][8];
  unsigned long long s1 = 0, s2 = 0, lmax = 0;
  unsigned bad = 0;
  if (blockIdx.x == 0 && threadIdx.x == 0 && ((int64_t)rowptr[0] != 0 || (int64_t)rowptr[N] != Z)) bad |= 1;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < N; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t L = (int64_t)rowptr[i + 1] - (int64_t)rowptr[i];
    if (L < 0) { bad |= 1; continue; }
    s1 += (unsigned long long)L;
    s2 += (unsigned long long)L * (unsigned long long)L;
    lmax = (unsigned long long)L > lmax ? (unsigned long long)L : lmax;
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    s1 += __shfl_xor_sync(kFull, s1, o);
    s2 += __shfl_xor_sync(kFull, s2, o);
    const unsigned long long t = __shfl_xor_sync(kFull, lmax, o);
    lmax = t > lmax ? t : lmax;
  }
  bad = __reduce_or_sync(kFull, bad);
  const int w = threadIdx.x >> 5;
  if ((threadIdx.x & 31) == 0) {
    s_red[0][w] = s1; s_red[1][w] = s2; s_red[2][w] = lmax;
    if (bad) atomicOr(&acc->bad, bad);
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long a1 = 0, a2 = 0, am = 0;
    for (int k = 0; k < 8; ++k) {
      a1 += s_red[0][k]; a2 += s_red[1][k];
      am = s_red[2][k] > am ? s_red[2][k] : am;
    }
    if (a1) atomicAdd(&acc->s1, a1);
    if (a2) atomicAdd(&acc->s2, a2);
    if (am) atomicMax(&acc->lmax, am);
  }
}

// K1s — nnz-split feature pass (the K6s decomposition applied to K1).  Each
// warp walks a contiguous range of 256-entry chunks (8 consecutive entries per
// lane, 128-bit loads); it finds the row of its first entry once (a 32-ary
// cooperative search of rowptr) and then derives every entry's row from the
// row starts falling inside each chunk (counted per chunk position in shared
// memory, prefix-summed), carrying the row and the last column from chunk to
// chunk.  Per entry: the canonical checks (column in [0, cols), strictly above
// the previous entry of the same row) and the occupied-diagonal bit (per-block
// shared window for |offset| < 2^15, else the per-block offset set / global
// OR, as K1).  The row-length moments and the rowptr checks come from
// k_rowstats (one pass over rowptr), launched before it.  The work per warp is
// fixed by nnz, independent of the row-length distribution, and the per-entry
// path has no staging copy.
template <typename IT, int EP>
__global__ void __launch_bounds__(kThreads) k_feat_stream(const IT *__restrict__ rowptr, const int32_t *__restrict__ col,
                                                           int64_t N, int64_t M, int64_t Z, int64_t row0, int64_t G,
                                                           int64_t nch, int64_t q, FeatAcc *__restrict__ acc,
                                                           uint32_t *__restrict__ bitmap) {
  static_assert(EP % 4 == 0 && EP <= 16, "EP");
  constexpr int64_t CH = 32 * EP;
  __shared__ __align__(16) int s_cnt[kWarps][CH];
  __shared__ uint32_t s_seen[kCache];
  __shared__ uint32_t s_win[kWin / 32];
  __shared__ unsigned s_bad, s_full;
  for (int i = threadIdx.x; i < kCache; i += kThreads) s_seen[i] = kEmpty;
  for (int i = threadIdx.x; i < (int)(kWin / 32); i += kThreads) s_win[i] = 0u;
  if (threadIdx.x == 0) { s_bad = 0; s_full = 0; }
  __syncthreads();
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const uint32_t G32 = (uint32_t)G, M32 = (uint32_t)M;
  const uint32_t win_lo = G32 - (kWin >> 1);
  unsigned bad = 0;
  auto far = [&](uint32_t idx) {  // as K1's lane_far
    const bool full = *(volatile unsigned *)&s_full != 0;
    if (full) { atomicOr(bitmap + (idx >> 5), 1u << (idx & 31)); return; }
    bool hit = false;
    int free_slot = -1;
    const uint32_t h = idx * 0x9E3779B1u >> 22;
    for (int p = 0; p < kProbe; ++p) {
      const int slot = (int)((h + p) & (kCache - 1));
      const uint32_t cur = s_seen[slot];
      if (cur == idx) { hit = true; break; }
      if (cur == kEmpty) { free_slot = slot; break; }
    }
    if (!hit) {
      atomicOr(bitmap + (idx >> 5), 1u << (idx & 31));
      if (free_slot >= 0) atomicCAS(&s_seen[free_slot], kEmpty, idx);
      else s_full = 1;
    }
  };
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t ch0 = gw * q, ch1 = ch0 + q < nch ? ch0 + q : nch;
  if (ch0 < ch1) {
    // row of entry ch0 * CH: last r with rowptr[r] <= e (32-ary search)
    const int64_t e = ch0 * CH;
    int64_t lo = 0, hi = N;
    while (hi - lo > 1) {
      const int64_t step = (hi - lo + 31) / 32;
      const int64_t pr = lo + (int64_t)lane * step;
      const int64_t v = pr < hi ? (int64_t)rowptr[pr] : INT64_MAX;
      const unsigned m = __ballot_sync(kFull, v <= e);
      const int j = m ? 31 - __clz(m) : 0;
      lo = lo + (int64_t)j * step;
      hi = lo + step < hi ? lo + step : hi;
    }
    int64_t r_lo = lo;
    int last_c = -1;
    int64_t last_r = -1;
    int *cnt = s_cnt[wib];
    for (int64_t ch = ch0; ch < ch1; ++ch) {
      const int64_t c0 = ch * CH, cend = c0 + CH < Z ? c0 + CH : Z;
      const int64_t e0 = c0 + (int64_t)lane * EP;
      const int nv = e0 >= cend ? 0 : (cend - e0 < EP ? (int)(cend - e0) : EP);
      // the chunk's column loads and its first row-start window are issued together
      int c[EP];
      if (nv == EP && ((reinterpret_cast<uintptr_t>(col + e0) & 15) == 0)) {
#pragma unroll
        for (int k = 0; k < EP; k += 4) {
          const int4 a = ld_stream_i4(reinterpret_cast<const int4 *>(col + e0 + k));
          c[k] = a.x; c[k + 1] = a.y; c[k + 2] = a.z; c[k + 3] = a.w;
        }
      } else {
#pragma unroll
        for (int k = 0; k < EP; ++k) c[k] = k < nv ? ld_stream_i(col + e0 + k) : 0;
      }
      int64_t rs = r_lo + 1 + lane < N ? (int64_t)rowptr[r_lo + 1 + lane] : INT64_MAX;
#pragma unroll
      for (int k = 0; k < EP; k += 4) reinterpret_cast<int4 *>(cnt + lane * EP)[k / 4] = make_int4(0, 0, 0, 0);
      __syncwarp();
      // row starts inside (c0, cend): counted at their chunk position; r_next =
      // the last row starting at or before cend (the next chunk's first row)
      int64_t r_next = r_lo;
      for (int64_t w0 = r_lo + 1; w0 < N; w0 += 32) {
        if (w0 != r_lo + 1) rs = w0 + lane < N ? (int64_t)rowptr[w0 + lane] : INT64_MAX;
        if (rs > c0 && rs < cend) atomicAdd(cnt + (int)(rs - c0), 1);
        const unsigned le = __ballot_sync(kFull, rs <= cend);
        if (le) r_next = w0 + 31 - __clz(le);
        if (le != kFull) break;
      }
      __syncwarp();
      int row[EP];  // relative to r_lo
      {
        int inc[EP];
#pragma unroll
        for (int k = 0; k < EP; k += 4) {
          const int4 a = reinterpret_cast<const int4 *>(cnt + lane * EP)[k / 4];
          inc[k] = a.x; inc[k + 1] = a.y; inc[k + 2] = a.z; inc[k + 3] = a.w;
        }
#pragma unroll
        for (int k = 1; k < EP; ++k) inc[k] += inc[k - 1];
        int ex = inc[EP - 1];
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const int t = __shfl_up_sync(kFull, ex, o);
          if (lane >= o) ex += t;
        }
        ex -= inc[EP - 1];
#pragma unroll
        for (int k = 0; k < EP; ++k) row[k] = ex + inc[k];
      }
      // the previous entry of each lane's first entry: the previous lane's last
      // valid one, or (lane 0) the previous chunk's last entry
      int pc = __shfl_up_sync(kFull, c[EP - 1], 1);
      int64_t pr = r_lo + __shfl_up_sync(kFull, row[EP - 1], 1);
      if (lane == 0) { pc = last_c; pr = last_r; }
      const uint32_t rbase = (uint32_t)(row0 + r_lo);
#pragma unroll
      for (int k = 0; k < EP; ++k) {
        if (k < nv) {
          const int cc = c[k];
          const int64_t rk = r_lo + row[k];
          if ((uint32_t)cc >= M32) {
            bad |= 4;
          } else {
            if (rk == pr && cc <= pc) bad |= 2;
            const uint32_t myrow = rbase + (uint32_t)row[k];
            const uint32_t rel = (uint32_t)cc - myrow + (kWin >> 1);
            if (rel < kWin) {
              const uint32_t bit = 1u << (rel & 31);
              if (!(s_win[rel >> 5] & bit)) atomicOr(&s_win[rel >> 5], bit);
            } else {
              far((uint32_t)cc - myrow + G32);
            }
          }
          pc = cc;
          pr = rk;
        }
      }
      const int lastl = (int)((cend - 1 - c0) / EP);
      last_c = __shfl_sync(kFull, pc, lastl);
      last_r = __shfl_sync(kFull, pr, lastl);
      r_lo = r_next;
    }
  }
  bad = __reduce_or_sync(kFull, bad);
  if (lane == 0 && bad) atomicOr(&s_bad, bad);
  __syncthreads();
  merge_window(s_win, win_lo, G + M, bitmap);
  if (threadIdx.x == 0 && s_bad) atomicOr(&acc->bad, s_bad);
}

__global__ void __launch_bounds__(256) k_feat_zero(FeatAcc *acc, uint32_t *__restrict__ bm, int64_t nwords) {
  const int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, nt = (int64_t)gridDim.x * blockDim.x;
  pdl_trigger();
  if (t == 0) *acc = FeatAcc{};
  const int64_t n4 = (reinterpret_cast<uintptr_t>(bm) & 15) == 0 ? nwords / 4 : 0;
  for (int64_t i = t; i < n4; i += nt) reinterpret_cast<uint4 *>(bm)[i] = make_uint4(0, 0, 0, 0);
  for (int64_t i = n4 * 4 + t; i < nwords; i += nt) bm[i] = 0;
}

// D = popcount of the bitmap; the last block to finish copies the sums into
// the caller's mapped pinned FeatAcc (no separate device-to-host copy).
__global__ void __launch_bounds__(256) k_popc(const uint32_t *__restrict__ bm, int64_t nwords, FeatAcc *acc,
                                              FeatAcc *host_out) {
  pdl_wait();  // every OR of the feature pass has landed
  unsigned long long s = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nwords; i += (int64_t)gridDim.x * blockDim.x)
    s += __popc(bm[i]);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(kFull, s, o);
  if ((threadIdx.x & 31) == 0 && s) atomicAdd(&acc->ndiag, s);
  __syncthreads();
  __shared__ bool last;
  if (threadIdx.x == 0) {
    __threadfence();
    last = atomicAdd(&acc->popc_done, 1u) == gridDim.x - 1;
  }
  __syncthreads();
  if (last && threadIdx.x == 0) {
    __threadfence();
    const volatile FeatAcc *v = acc;
    FeatAcc h;
    h.s1 = v->s1; h.s2 = v->s2; h.lmax = v->lmax; h.bad = v->bad; h.nlong = v->nlong; h.ndiag = v->ndiag;
    h.popc_done = gridDim.x; h.pad_ = 0;
    *host_out = h;
    __threadfence_system();
  }
}

}  // namespace

// K1s (nnz-split feature pass) for matrices whose mean row length exceeds
// kRowCap (K1 walks those rows warp-wide; B200, dense band b = 48, 97 entries
// per row: K1 0.964 ms -> K1s 0.470 ms).  K1 stays for shorter rows: configs[1]
// 0.131 vs 0.175 ms, configs[4] 5.8 vs 12.0 ms, 1D 3-pt 0.118 vs 0.139 ms.  K1s
// is also ahead on skewed rows (configs[2] R-MAT 0.943 -> 0.804 ms) and sparse
// bands (0.275 -> 0.200 ms), but telling those apart needs the row-length SD,
// i.e. a pass before the launch; the rule uses what is known at create time.
bool feat_stream_on(const nitro_spmv *A) { return A->N > 0 && A->Z > (int64_t)kRowCap * A->N; }

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
  if (!A->h_acc) {
    NITRO_CUDA(cudaHostAlloc(&A->h_acc, sizeof(FeatAcc), cudaHostAllocMapped));
    NITRO_CUDA(cudaHostGetDevicePointer(&A->h_acc_dev, A->h_acc, 0));
  }
  if (!A->feat_done) NITRO_CUDA(cudaEventCreateWithFlags(&A->feat_done, cudaEventDisableTiming));
  FeatAcc *acc = A->feat_acc.as<FeatAcc>();
  {  // FeatAcc and the bitmap zeroed by one launch
    int64_t gz = (nwords / 4 + 255) / 256;
    gz = gz < 1 ? 1 : gz > (int64_t)num_sms() * 4 ? (int64_t)num_sms() * 4 : gz;
    k_feat_zero<<<(unsigned)gz, 256, 0, s>>>(acc, A->bitmap.as<uint32_t>(), nwords);
  }

  const int64_t nblk = (A->N + 31) / 32;
  int64_t grid = (nblk + kWarps - 1) / kWarps;
  const int64_t cap = (int64_t)num_sms() * 8;  // (one persistent wave measured: -5 % configs[4], +11 % uniform)
  if (grid > cap) grid = cap;
  if (grid < 1) grid = 1;
  // long-row chunk tasks: at most Z / kChunk + (number of long rows <= Z / kLong) entries
  const int64_t cap_tasks = A->Z / kChunk + A->Z / kLong + 1;
  NITRO_TRY(A->feat_long.alloc((size_t)cap_tasks * sizeof(int2)));
  int2 *tasks = A->feat_long.as<int2>();
  // (one 1024-thread CTA per SM instead: configs[1] -1 %, R-MAT +1 %: kept)
  const unsigned glong = (unsigned)std::max<int64_t>(1, std::min<int64_t>((int64_t)num_sms() * 4,
                                                                           (A->Z / kChunk + kWarps - 1) / kWarps));
  if (feat_stream_on(A)) {  // K1s: rowptr moments (k_rowstats) + the nnz-split pass
    if (A->N > 0) {
      const unsigned gr = (unsigned)std::max<int64_t>(1, std::min<int64_t>((int64_t)num_sms() * 8, (A->N + 255) / 256));
      if (A->rp64) k_rowstats<int64_t><<<gr, 256, 0, s>>>((const int64_t *)A->rowptr, A->N, A->Z, acc);
      else k_rowstats<int32_t><<<gr, 256, 0, s>>>((const int32_t *)A->rowptr, A->N, A->Z, acc);
    }
    constexpr int ep = 8;  // entries per lane (16: configs[1] 0.188 vs 0.175 ms, dense band 0.476 vs 0.470)
    const int64_t nch = (A->Z + 32 * ep - 1) / (32 * ep);
    if (nch > 0) {
      const int64_t gs = std::max<int64_t>(1, std::min<int64_t>((int64_t)num_sms() * 8, (nch + kWarps - 1) / kWarps));
      const int64_t q = (nch + gs * kWarps - 1) / (gs * kWarps);
#define NITRO_K1S(IT, EPV)                                                                                   \
  k_feat_stream<IT, EPV><<<(unsigned)gs, kThreads, 0, s>>>((const IT *)A->rowptr, A->col, A->N, A->M, A->Z, \
                                                           A->row0, G, nch, q, acc, A->bitmap.as<uint32_t>())
      if (A->rp64) NITRO_K1S(int64_t, ep);
      else NITRO_K1S(int32_t, ep);
#undef NITRO_K1S
    }
  } else {
    // the K1 chain zero -> k_features -> k_features_long -> k_popc by
    // programmatic dependent launch: each kernel's launch overlaps the tail of
    // its predecessor and waits (griddepcontrol.wait) before touching its output
#define NITRO_K1(IT)                                                                                               \
  do {                                                                                                             \
    NITRO_CUDA(launch_pdl(k_features<IT>, (unsigned)grid, kThreads, 0, s, (const IT *)A->rowptr, A->col, A->N, A->M,  \
                          A->Z, A->row0, G, acc, A->bitmap.as<uint32_t>(), tasks, cap_tasks));                     \
    if (A->Z > kLong)                                                                                              \
      NITRO_CUDA(launch_pdl(k_features_long<IT>, glong, kThreads, 0, s, (const IT *)A->rowptr, A->col, A->M,       \
                            A->row0, G, acc, A->bitmap.as<uint32_t>(), (const int2 *)tasks, cap_tasks));           \
  } while (0)
    if (A->rp64) NITRO_K1(int64_t);
    else NITRO_K1(int32_t);
#undef NITRO_K1
  }
  {
    int64_t g2 = (nwords + 255) / 256;
    if (g2 > (int64_t)num_sms() * 8) g2 = (int64_t)num_sms() * 8;
    if (g2 < 1) g2 = 1;
    NITRO_CUDA(launch_pdl(k_popc, (unsigned)g2, 256u, 0, s, (const uint32_t *)A->bitmap.as<uint32_t>(), nwords, acc,
                          A->h_acc_dev));
  }
  NITRO_CUDA(cudaGetLastError());
  NITRO_CUDA(cudaEventRecord(A->feat_done, s));
  A->feat_pending = true;
  return NITRO_OK;
}

nitro_status_t row_features(nitro_spmv *A, nitro_spmv_feat *out) {
  cudaStream_t s = A->stream;
  DevBuf acc_buf;
  NITRO_TRY(acc_buf.alloc(sizeof(FeatAcc)));
  FeatAcc *acc = acc_buf.as<FeatAcc>();
  NITRO_CUDA(cudaMemsetAsync(acc, 0, sizeof(FeatAcc), s));
  if (A->N > 0) {
    const unsigned g = (unsigned)std::max<int64_t>(1, std::min<int64_t>((int64_t)num_sms() * 8, (A->N + 255) / 256));
    if (A->rp64) k_rowstats<int64_t><<<g, 256, 0, s>>>((const int64_t *)A->rowptr, A->N, A->Z, acc);
    else k_rowstats<int32_t><<<g, 256, 0, s>>>((const int32_t *)A->rowptr, A->N, A->Z, acc);
    NITRO_CUDA(cudaGetLastError());
  }
  FeatAcc h{};
  NITRO_CUDA(cudaMemcpyAsync(&h, acc, sizeof(FeatAcc), cudaMemcpyDeviceToHost, s));
  NITRO_CUDA(cudaStreamSynchronize(s));
  finish_features(A->N, A->M, A->Z, h.s1, h.s2, (int64_t)h.lmax, 0, out);
  out->ndiag = -1;
  out->dia_fill = -1.0;
  out->canonical = -1;
  if (h.bad) return fail(NITRO_E_BAD_MATRIX, "non-canonical CSR: rowptr not monotone from 0 to nnz");
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
