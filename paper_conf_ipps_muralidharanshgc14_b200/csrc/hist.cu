// hist.cu — the histogram code-variant family (a second
// workload through the same generic Nitro layer; Fig. 4
// "Histogram").
//
// Operation (include/nitro.h §4): h[b] = #{ i : s_i < range, floor(s_i * nbins / range) = b }
// for uint32 samples s, 1 <= nbins <= 65536, 1 <= range <= 2^32 — an even
// binning of [0, range) as in CUB's HistogramEven, which the paper's variants
// come from.  Six variants = three algorithms x two grid mappings
// ("three variants and two grid-mapping strategies"):
//   SORT      — per tile: bin ids sorted in shared memory (bitonic), then run
//               detection; a run [h, t] of bin k adds (t + 1) - h to h[k] as two
//               atomics (+ (t+1) at the run's tail, - h at its head; unsigned
//               wrap-around arithmetic, exact);
//   SHARED    — per CTA a privatised shared-memory histogram (shared atomics),
//               merged into the global one at the end (one atomic per non-zero bin);
//   GLOBAL    — one global atomic per sample;
//   ES        — "even share": CTA c of G owns tiles [c*T/G, (c+1)*T/G);
//   DYNAMIC   — CTAs take tiles from a global atomic queue.
// Features: N, N / #bins, SubSampleSD = population standard
// deviation of the sub-sample s[floor(j*N/k)], j < k, k = min(ceil(N/4), 10000),
// from exact integer moments (bit-exact with the oracle).
#include "nitro_internal.h"

#include <algorithm>
#include <cmath>
#include <new>
#include <vector>

namespace nitro {
namespace {

constexpr int kHThr = 256;
constexpr int kHVec = 4;                           // uint4 loads per thread per tile
constexpr int64_t kHTile = kHThr * kHVec * 4;      // 4096 samples per tile (atomic variants)
constexpr int kSortPer = 8;                        // keys per thread (sort variants)
constexpr int64_t kSortTile = kHThr * kSortPer;    // 2048 samples per tile
constexpr uint32_t kNoBin = 0xffffffffu;
constexpr int kSubMax = 10000;                     // sub-sample cap
constexpr uint32_t kMaxSharedBins = 49152;         // 192 KB of shared counters

// general even binning: floor(s * nbins / range) by an fp64 reciprocal and an
// exact integer correction
struct BinMap {
  uint64_t nbins, range;
  double rinv;  // nbins / range (rounded); corrected below to the exact floor
  __device__ __forceinline__ uint32_t operator()(uint32_t s) const {
    if ((uint64_t)s >= range) return kNoBin;
    const uint64_t a = (uint64_t)s * nbins;  // < 2^48
    uint64_t q = (uint64_t)((double)s * rinv);
    // |q - a/range| <= 1 before correction: make q = floor(a / range) exactly
    if ((q + 1) * range <= a) ++q;
    else if (q * range > a) --q;
    return (uint32_t)q;
  }
};
// range / nbins = 2^sh (equal power-of-two bin widths, e.g. 8/16-bit data):
// the same floor is s >> sh; lim = range - 1 (< 2^32)
struct BinShift {
  uint32_t lim, sh;  // sh <= 32
  __device__ __forceinline__ uint32_t operator()(uint32_t s) const {
    if (s > lim) return kNoBin;
    return sh >= 32 ? 0u : s >> sh;
  }
};

__device__ __forceinline__ void red_shared_inc(uint32_t saddr) {
  asm volatile("red.shared.add.u32 [%0], 1;" ::"r"(saddr) : "memory");
}

// Per-handle control words (no per-call memsets): p[0] = dynamic tile queue,
// p[1] = "output zeroed" flag.  Both only grow: a call with epoch e takes
// tiles as (p[0] value - qbase) and waits for p[1] >= e; the host advances
// qbase by tiles + gridDim after each dynamic call (every CTA makes exactly
// one failing fetch) and e by one per call.  Launched cooperatively, so every
// CTA is resident and the wait on CTA 0's zeroing cannot deadlock.
struct Ctl {
  unsigned long long *p;
  unsigned long long epoch, qbase;
};

__device__ __forceinline__ int64_t next_tile(const Ctl &c, int64_t *s_t) {
  if (threadIdx.x == 0) *s_t = (int64_t)(atomicAdd(c.p, 1ull) - c.qbase);
  __syncthreads();
  const int64_t t = *s_t;
  __syncthreads();
  return t;
}

// CTA 0 zeroes the output and publishes epoch in p[1]
__device__ __forceinline__ void zero_output(uint32_t *__restrict__ hist, uint32_t nb, const Ctl &c) {
  if (blockIdx.x != 0) return;
  for (uint32_t i = threadIdx.x; i < nb; i += blockDim.x) hist[i] = 0;
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    atomicExch(c.p + 1, c.epoch);
  }
}
// every CTA, before its first update of the output
__device__ __forceinline__ void wait_zeroed(const Ctl &c) {
  if (threadIdx.x == 0) {
    while (*((volatile unsigned long long *)(c.p + 1)) < c.epoch) __nanosleep(64);
    __threadfence();
  }
  __syncthreads();
}

// samples of tile t handled by this thread (T threads, T * 16 samples per
// tile): kHVec uint4 (vector path when the array is 16-byte aligned and the
// tile is whole), else scalar
template <int T, typename F>
__device__ __forceinline__ void for_tile_samples(const uint32_t *__restrict__ s, int64_t n, int64_t t, bool vec,
                                                 F f) {
  constexpr int64_t TL = (int64_t)T * kHVec * 4;
  const int64_t base = t * TL;
  if (vec && base + TL <= n) {
#pragma unroll
    for (int k = 0; k < kHVec; ++k) {
      const uint4 q = __ldcs(reinterpret_cast<const uint4 *>(s + base) + k * T + threadIdx.x);
      f(q.x); f(q.y); f(q.z); f(q.w);
    }
  } else {
    for (int64_t i = base + threadIdx.x; i < base + TL && i < n; i += T) f(__ldcs(s + i));
  }
}

// Shared-atomic variants: T threads per CTA (256, or 1024 when the counters
// leave room for one CTA per SM only, so the SM still has 32 warps issuing);
// R copies of the nbins counters (warp w adds to copy w % R) spread the
// same-bin contention of concentrated inputs over R addresses; the copies
// are summed per bin at the end and merged with one global atomic per
// non-zero bin.
template <int T, bool DYN, typename BM>
__global__ void __launch_bounds__(T) k_hist_shared(const uint32_t *__restrict__ s, int64_t n, BM bm, uint32_t nb,
                                                   uint32_t *__restrict__ hist, int64_t tiles, Ctl ctl, bool vec,
                                                   int R) {
  extern __shared__ uint32_t sh[];
  __shared__ int64_t s_t;
  zero_output(hist, nb, ctl);
  for (uint32_t i = threadIdx.x; i < nb * (uint32_t)R; i += T) sh[i] = 0;
  __syncthreads();
  // this warp's counter copy as a 32-bit shared-window address (red.shared per sample)
  const uint32_t mine = (uint32_t)__cvta_generic_to_shared(sh + (uint32_t)((threadIdx.x >> 5) % R) * nb);
  auto add = [&](uint32_t v) {
    const uint32_t b = bm(v);
    if (b != kNoBin) red_shared_inc(mine + 4u * b);
  };
  if (DYN) {
    for (int64_t t = next_tile(ctl, &s_t); t < tiles; t = next_tile(ctl, &s_t))
      for_tile_samples<T>(s, n, t, vec, add);
  } else {
    const int64_t t0 = blockIdx.x * tiles / gridDim.x, t1 = (blockIdx.x + 1) * tiles / gridDim.x;
    for (int64_t t = t0; t < t1; ++t) for_tile_samples<T>(s, n, t, vec, add);
  }
  __syncthreads();
  wait_zeroed(ctl);
  for (uint32_t i = threadIdx.x; i < nb; i += T) {
    uint32_t c = 0;
    for (int r = 0; r < R; ++r) c += sh[(uint32_t)r * nb + i];
    if (c) atomicAdd(hist + i, c);
  }
}

template <bool DYN, typename BM>
__global__ void __launch_bounds__(kHThr) k_hist_global(const uint32_t *__restrict__ s, int64_t n, BM bm,
                                                       uint32_t nb, uint32_t *__restrict__ hist, int64_t tiles,
                                                       Ctl ctl, bool vec) {
  __shared__ int64_t s_t;
  zero_output(hist, nb, ctl);
  wait_zeroed(ctl);
  auto add = [&](uint32_t v) {
    const uint32_t b = bm(v);
    if (b != kNoBin) atomicAdd(hist + b, 1u);
  };
  if (DYN) {
    for (int64_t t = next_tile(ctl, &s_t); t < tiles; t = next_tile(ctl, &s_t))
      for_tile_samples<kHThr>(s, n, t, vec, add);
  } else {
    const int64_t t0 = blockIdx.x * tiles / gridDim.x, t1 = (blockIdx.x + 1) * tiles / gridDim.x;
    for (int64_t t = t0; t < t1; ++t) for_tile_samples<kHThr>(s, n, t, vec, add);
  }
}

// one sort tile: load + bin, bitonic sort of kSortTile keys in shared memory,
// run detection with the (tail + 1) - head atomics
template <typename BM>
__device__ __forceinline__ void sort_tile(const uint32_t *__restrict__ s, int64_t n, const BM &bm,
                                          uint32_t *__restrict__ hist, int64_t t, uint32_t *key) {
  const int64_t base = t * kSortTile;
#pragma unroll
  for (int k = 0; k < kSortPer; ++k) {
    const int64_t i = base + k * kHThr + threadIdx.x;
    key[k * kHThr + threadIdx.x] = i < n ? bm(__ldcs(s + i)) : kNoBin;
  }
  __syncthreads();
  for (int size = 2; size <= (int)kSortTile; size <<= 1) {
    for (int stride = size >> 1; stride > 0; stride >>= 1) {
#pragma unroll
      for (int k = 0; k < kSortPer / 2; ++k) {
        const int p = k * kHThr + threadIdx.x;                   // pair index < kSortTile / 2
        const int lo = 2 * p - (p & (stride - 1)), hi = lo + stride;
        const bool up = (lo & size) == 0;
        const uint32_t a = key[lo], b = key[hi];
        if ((a > b) == up) { key[lo] = b; key[hi] = a; }
      }
      __syncthreads();
    }
  }
#pragma unroll
  for (int k = 0; k < kSortPer; ++k) {
    const int i = k * kHThr + threadIdx.x;
    const uint32_t v = key[i];
    if (v == kNoBin) continue;
    if (i == 0 || key[i - 1] != v) atomicAdd(hist + v, 0u - (uint32_t)i);          // run head
    if (i == (int)kSortTile - 1 || key[i + 1] != v) atomicAdd(hist + v, (uint32_t)i + 1u);  // run tail
  }
  __syncthreads();
}

template <bool DYN, typename BM>
__global__ void __launch_bounds__(kHThr) k_hist_sort(const uint32_t *__restrict__ s, int64_t n, BM bm,
                                                     uint32_t nb, uint32_t *__restrict__ hist, int64_t tiles,
                                                     Ctl ctl) {
  __shared__ uint32_t key[kSortTile];
  __shared__ int64_t s_t;
  zero_output(hist, nb, ctl);
  wait_zeroed(ctl);
  if (DYN) {
    for (int64_t t = next_tile(ctl, &s_t); t < tiles; t = next_tile(ctl, &s_t)) sort_tile(s, n, bm, hist, t, key);
  } else {
    const int64_t t0 = blockIdx.x * tiles / gridDim.x, t1 = (blockIdx.x + 1) * tiles / gridDim.x;
    for (int64_t t = t0; t < t1; ++t) sort_tile(s, n, bm, hist, t, key);
  }
}

// SubSampleSD moments: one CTA; out = {S1, S2 low 64 bits, S2 high 64 bits}
__global__ void __launch_bounds__(kHThr) k_hist_subsample(const uint32_t *__restrict__ s, int64_t n, int64_t k,
                                                          unsigned long long *out) {
  __shared__ unsigned long long s1[kHThr], lo[kHThr], hi[kHThr];
  unsigned long long a = 0;
  unsigned __int128 b = 0;
  for (int64_t j = threadIdx.x; j < k; j += kHThr) {
    const uint64_t v = s[(uint64_t)j * (uint64_t)n / (uint64_t)k];
    a += v;
    b += (unsigned __int128)(v * v);
  }
  s1[threadIdx.x] = a;
  lo[threadIdx.x] = (unsigned long long)b;
  hi[threadIdx.x] = (unsigned long long)(b >> 64);
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long ta = 0;
    unsigned __int128 tb = 0;
    for (int i = 0; i < kHThr; ++i) {
      ta += s1[i];
      tb += ((unsigned __int128)hi[i] << 64) | lo[i];
    }
    out[0] = ta;
    out[1] = (unsigned long long)tb;
    out[2] = (unsigned long long)(tb >> 64);
  }
}

__global__ void k_hist_flush(const int4 *__restrict__ buf, int64_t n, int *__restrict__ sink) {
  int acc = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int4 v = __ldcg(buf + i);
    acc ^= v.x ^ v.y ^ v.z ^ v.w;
  }
  if (acc == 0x7fffffff) *sink = acc;
}

struct DevGuard {
  int prev = -1;
  explicit DevGuard(int dev) {
    if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DevGuard() {
    int cur = -1;
    if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
  }
};

}  // namespace
}  // namespace nitro

struct nitro_hist {
  int device = 0;
  cudaStream_t stream = nullptr;
  int64_t n = 0;
  const uint32_t *s = nullptr;
  uint32_t nbins = 1;
  uint64_t range = 1;
  bool feat_ready = false;
  double feat[3] = {0, 0, 0};
  nitro::DevBuf ctl, moments, flush;  // ctl: 2 x u64 control words (see Ctl)
  unsigned long long epoch = 0, qbase = 0;
};

using namespace nitro;

namespace {

bool hist_valid(int v) { return v >= 0 && v < NITRO_HIST_NUM_VARIANTS; }
bool hist_is_shared(int v) { return v == NITRO_HIST_SHARED_ES || v == NITRO_HIST_SHARED_DYN; }

int blocks_per_sm(const void *fn, size_t smem) {
  int b = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, fn, kHThr, smem) != cudaSuccess || b < 1) b = 1;
  return b;
}

// cooperative launch (all CTAs co-resident: required by the zeroing wait)
template <typename... Args>
nitro_status_t coop(void (*k)(Args...), int64_t g, int threads, size_t smem, cudaStream_t st, Args... args) {
  void *argv[] = {(void *)&args...};
  NITRO_CUDA(cudaLaunchCooperativeKernel((const void *)k, dim3((unsigned)g), dim3((unsigned)threads), argv, smem, st));
  return NITRO_OK;
}

template <typename BM>
nitro_status_t hist_kernels(nitro_hist *H, int v, uint32_t *hist, cudaStream_t st, const BM &bm, bool dyn) {
  const bool vec = (reinterpret_cast<uintptr_t>(H->s) & 15) == 0;
  const int sms = num_sms();
  const uint32_t nb = H->nbins;
  Ctl ctl{H->ctl.as<unsigned long long>(), ++H->epoch, H->qbase};
  int64_t tiles = 0, g = 0;
  if (v == NITRO_HIST_SORT_ES || v == NITRO_HIST_SORT_DYN) {
    tiles = (H->n + kSortTile - 1) / kSortTile;
    auto k = dyn ? k_hist_sort<true, BM> : k_hist_sort<false, BM>;
    g = std::min<int64_t>(tiles, (int64_t)sms * blocks_per_sm((const void *)k, 0));
    NITRO_TRY(coop(k, g, kHThr, 0, st, H->s, H->n, bm, nb, hist, tiles, ctl));
  } else if (hist_is_shared(v)) {
    if (nb > kMaxSharedBins) return fail(NITRO_E_CONSTRAINT, "shared-atomic histogram: nbins > 49152");
    // counter copies: up to 8 while they fit 48 KB (several CTAs per SM)
    int R = 1;
    while (R < 8 && (size_t)(2 * R) * nb * 4 <= 48 * 1024) R *= 2;
    const size_t smem = (size_t)R * nb * 4;
    const bool big = smem > 76 * 1024;  // at most two CTAs per SM: 1024 threads each
    auto k = big ? (dyn ? k_hist_shared<1024, true, BM> : k_hist_shared<1024, false, BM>)
                 : (dyn ? k_hist_shared<256, true, BM> : k_hist_shared<256, false, BM>);
    const int T = big ? 1024 : 256;
    NITRO_CUDA(cudaFuncSetAttribute((const void *)k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int b = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, (const void *)k, T, smem) != cudaSuccess || b < 1) b = 1;
    tiles = (H->n + (int64_t)T * 16 - 1) / ((int64_t)T * 16);
    g = std::min<int64_t>(tiles, (int64_t)sms * b);
    NITRO_TRY(coop(k, g, T, smem, st, H->s, H->n, bm, nb, hist, tiles, ctl, vec, R));
  } else {
    tiles = (H->n + kHTile - 1) / kHTile;
    auto k = dyn ? k_hist_global<true, BM> : k_hist_global<false, BM>;
    g = std::min<int64_t>(tiles, (int64_t)sms * blocks_per_sm((const void *)k, 0));
    NITRO_TRY(coop(k, g, kHThr, 0, st, H->s, H->n, bm, nb, hist, tiles, ctl, vec));
  }
  if (dyn) H->qbase += (unsigned long long)(tiles + g);  // every CTA made exactly one failing fetch
  return NITRO_OK;
}

nitro_status_t hist_launch(nitro_hist *H, int v, uint32_t *hist, cudaStream_t st) {
  if (H->n == 0) {
    NITRO_CUDA(cudaMemsetAsync(hist, 0, (size_t)H->nbins * 4, st));
    return NITRO_OK;
  }
  if (!H->ctl.p) {
    NITRO_TRY(H->ctl.alloc(16));
    NITRO_CUDA(cudaMemsetAsync(H->ctl.p, 0, 16, st));  // once per handle
  }
  const bool dyn = v == NITRO_HIST_SORT_DYN || v == NITRO_HIST_SHARED_DYN || v == NITRO_HIST_GLOBAL_DYN;
  if (H->range % H->nbins == 0) {  // equal integer bins of width w = range / nbins; a power of two -> shift
    const uint64_t w = H->range / H->nbins;
    if ((w & (w - 1)) == 0) {
      uint32_t sh = 0;
      while ((1ull << sh) < w) ++sh;
      return hist_kernels(H, v, hist, st, BinShift{(uint32_t)(H->range - 1), sh}, dyn);
    }
  }
  return hist_kernels(H, v, hist, st, BinMap{H->nbins, H->range, (double)H->nbins / (double)H->range}, dyn);
}

nitro_status_t hist_flush(nitro_hist *H, cudaStream_t st) {
  int dev = 0, l2 = 0;
  NITRO_CUDA(cudaGetDevice(&dev));
  NITRO_CUDA(cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, dev));
  const size_t bytes = (size_t)std::max(l2, 1 << 20) * 3;
  if (H->flush.bytes < bytes) {
    NITRO_TRY(H->flush.alloc(bytes + 64));
    NITRO_CUDA(cudaMemsetAsync(H->flush.p, 0, H->flush.bytes, st));
  }
  k_hist_flush<<<num_sms() * 4, 256, 0, st>>>(H->flush.as<int4>(), (int64_t)(bytes / 16),
                                               reinterpret_cast<int *>(H->flush.as<char>() + bytes));
  NITRO_CUDA(cudaGetLastError());
  return NITRO_OK;
}

nitro_status_t hist_features(nitro_hist *H) {
  if (H->feat_ready) return NITRO_OK;
  const int64_t n = H->n;
  const int64_t k = std::min<int64_t>((n + 3) / 4, kSubMax);
  double sd = 0.0;
  if (k > 0) {
    NITRO_TRY(H->moments.alloc(32));
    k_hist_subsample<<<1, kHThr, 0, H->stream>>>(H->s, n, k, H->moments.as<unsigned long long>());
    NITRO_CUDA(cudaGetLastError());
    unsigned long long m[3] = {0, 0, 0};
    NITRO_CUDA(cudaMemcpyAsync(m, H->moments.p, 24, cudaMemcpyDeviceToHost, H->stream));
    NITRO_CUDA(cudaStreamSynchronize(H->stream));
    const unsigned __int128 s1 = m[0], s2 = ((unsigned __int128)m[2] << 64) | m[1];
    const unsigned __int128 num = (unsigned __int128)k * s2 - s1 * s1;  // k * sum v^2 - (sum v)^2 >= 0
    sd = std::sqrt((double)num / ((double)k * (double)k));
  }
  H->feat[0] = (double)n;
  H->feat[1] = (double)n / (double)H->nbins;
  H->feat[2] = sd;
  H->feat_ready = true;
  return NITRO_OK;
}

#define HIST_GUARD_BEGIN try {
#define HIST_GUARD_END                                               \
  }                                                                  \
  catch (const std::bad_alloc &) {                                   \
    return fail(NITRO_E_OOM, "host allocation failed");             \
  }                                                                  \
  catch (...) {                                                      \
    return fail(NITRO_E_INVALID_ARG, "unexpected exception");       \
  }

}  // namespace

extern "C" {

nitro_status_t nitro_hist_create(int device, void *stream, int64_t n, const uint32_t *d_samples, int32_t nbins,
                                 uint64_t range, nitro_hist **out) {
  HIST_GUARD_BEGIN
  if (!out) return fail(NITRO_E_INVALID_ARG, "out is NULL");
  *out = nullptr;
  if (n < 0 || (n > 0 && !d_samples)) return fail(NITRO_E_INVALID_ARG, "bad samples");
  if (nbins < 1 || nbins > 65536) return fail(NITRO_E_INVALID_ARG, "nbins must be in [1, 65536]");
  if (range < 1 || range > (1ull << 32)) return fail(NITRO_E_INVALID_ARG, "range must be in [1, 2^32]");
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev)
    return fail(NITRO_E_CUDA, "no such CUDA device");
  nitro_hist *H = new nitro_hist();
  H->device = device;
  H->stream = (cudaStream_t)stream;
  H->n = n;
  H->s = d_samples;
  H->nbins = (uint32_t)nbins;
  H->range = range;
  *out = H;
  return NITRO_OK;
  HIST_GUARD_END
}

void nitro_hist_destroy(nitro_hist *H) {
  if (!H) return;
  DevGuard g(H->device);
  delete H;
}

nitro_status_t nitro_hist_features(nitro_hist *H, double *out3) {
  HIST_GUARD_BEGIN
  if (!H || !out3) return fail(NITRO_E_INVALID_ARG, "NULL argument");
  DevGuard g(H->device);
  NITRO_TRY(hist_features(H));
  std::copy(H->feat, H->feat + 3, out3);
  return NITRO_OK;
  HIST_GUARD_END
}

nitro_status_t nitro_hist_allowed(nitro_hist *H, int variant, int *out_allowed) {
  if (!H || !out_allowed || !hist_valid(variant)) return fail(NITRO_E_INVALID_ARG, "bad argument");
  *out_allowed = hist_is_shared(variant) ? (H->nbins <= kMaxSharedBins) : 1;
  return NITRO_OK;
}

nitro_status_t nitro_hist_run(nitro_hist *H, int variant, uint32_t *d_hist) {
  NITRO_NVTX("nitro_hist_run");
  HIST_GUARD_BEGIN
  if (!H || !d_hist || !hist_valid(variant)) return fail(NITRO_E_INVALID_ARG, "bad argument");
  DevGuard g(H->device);
  return hist_launch(H, variant, d_hist, H->stream);
  HIST_GUARD_END
}

nitro_status_t nitro_hist_time(nitro_hist *H, int variant, uint32_t *d_hist, int warmup, int reps, int flush_l2,
                               double *out_median_s) {
  HIST_GUARD_BEGIN
  if (!H || !d_hist || !hist_valid(variant) || reps < 1 || warmup < 0 || !out_median_s)
    return fail(NITRO_E_INVALID_ARG, "bad argument");
  DevGuard g(H->device);
  cudaStream_t s = H->stream;
  for (int w = 0; w < warmup; ++w) NITRO_TRY(hist_launch(H, variant, d_hist, s));
  std::vector<cudaEvent_t> ev(2 * reps, nullptr);
  for (auto &e : ev) NITRO_CUDA(cudaEventCreate(&e));
  nitro_status_t st = NITRO_OK;
  for (int r = 0; r < reps && st == NITRO_OK; ++r) {
    if (flush_l2) st = hist_flush(H, s);
    if (st == NITRO_OK) {
      cudaEventRecord(ev[2 * r], s);
      st = hist_launch(H, variant, d_hist, s);
      cudaEventRecord(ev[2 * r + 1], s);
    }
  }
  std::vector<double> t(reps, 0.0);
  cudaError_t e = cudaStreamSynchronize(s);
  if (st == NITRO_OK && e != cudaSuccess) st = cuda_fail(e, "cudaStreamSynchronize");
  for (int r = 0; r < reps && st == NITRO_OK; ++r) {
    float ms = 0.f;
    cudaEventElapsedTime(&ms, ev[2 * r], ev[2 * r + 1]);
    t[r] = ms * 1e-3;
  }
  for (auto &x : ev) cudaEventDestroy(x);
  if (st != NITRO_OK) return st;
  std::sort(t.begin(), t.end());
  *out_median_s = reps % 2 ? t[reps / 2] : 0.5 * (t[reps / 2 - 1] + t[reps / 2]);
  return NITRO_OK;
  HIST_GUARD_END
}

// ---------------------------------------------------------------- registration
static double hist_variant_fn(void *input, void *user) {
  nitro_hist_input *in = (nitro_hist_input *)input;
  double t = INFINITY;
  if (!in || !in->H || !in->d_hist) return INFINITY;
  if (nitro_hist_time(in->H, (int)(intptr_t)user, in->d_hist, in->warmup, in->reps > 0 ? in->reps : 1, in->flush_l2,
                      &t) != NITRO_OK)
    return INFINITY;
  return t;
}
static int hist_feature_group(const void *input, double *out, int n, void *) {
  const nitro_hist_input *in = (const nitro_hist_input *)input;
  if (!in || !in->H || n != 3) return 1;
  return nitro_hist_features(in->H, out) == NITRO_OK ? 0 : 1;
}
static int hist_constraint(const void *input, void *user) {
  const nitro_hist_input *in = (const nitro_hist_input *)input;
  int ok = 0;
  if (!in || !in->H) return 0;
  if (nitro_hist_allowed(in->H, (int)(intptr_t)user, &ok) != NITRO_OK) return 0;
  return ok;
}

nitro_status_t nitro_hist_register(nitro_cv *cv) {
  HIST_GUARD_BEGIN
  if (!cv) return fail(NITRO_E_INVALID_ARG, "NULL cv");
  int nv = 0, nf = 0;
  NITRO_TRY(nitro_cv_num_variants(cv, &nv));
  NITRO_TRY(nitro_cv_num_features(cv, &nf));
  if (nv != 0 || nf != 0) return fail(NITRO_E_STATE, "register on a fresh code variant");
  static const char *vn[NITRO_HIST_NUM_VARIANTS] = {"sort_es", "sort_dynamic", "shared_atomic_es",
                                                     "shared_atomic_dynamic", "global_atomic_es",
                                                     "global_atomic_dynamic"};
  for (int v = 0; v < NITRO_HIST_NUM_VARIANTS; ++v)
    NITRO_TRY(nitro_cv_add_variant(cv, vn[v], hist_variant_fn, (void *)(intptr_t)v, nullptr));
  static const char *fn[3] = {"n", "n_per_bin", "subsample_sd"};
  NITRO_TRY(nitro_cv_add_feature_group(cv, fn, 3, hist_feature_group, nullptr));
  NITRO_TRY(nitro_cv_add_constraint(cv, NITRO_HIST_SHARED_ES, hist_constraint, (void *)(intptr_t)NITRO_HIST_SHARED_ES));
  NITRO_TRY(nitro_cv_add_constraint(cv, NITRO_HIST_SHARED_DYN, hist_constraint,
                                    (void *)(intptr_t)NITRO_HIST_SHARED_DYN));
  // plain [-1, 1] scaling; log1p + clip is the opt-in extension R11x
  // default: always allowed (the shared variants are not) and robust to skew
  return nitro_cv_set_default(cv, NITRO_HIST_SORT_ES);
  HIST_GUARD_END
}

}  // extern "C"
