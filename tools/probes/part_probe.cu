// part_probe.cu — ways to mark 268 M random diagonal indices (configs[2]
// uniform: 2^23 rows x 32, offsets spread over 2^24 diagonals) in a bitmap,
// each reading the 1.07 GB index stream once:
//   G: fire-and-forget global red.or per entry (what K1 does),
//   B: a plain byte store per entry into a 16 MB byte map,
//   P: partition — P1: a CTA sorts a tile of indices by their high bits
//      (2^16-bit buckets) in shared memory and appends the low 16 bits of each
//      to its bucket in global memory; P2: one CTA per bucket ORs its entries
//      into an 8 KB shared bitmap and stores the words.
// One JSON line per case (median of 9), plus a check that all give one count.
// build: nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -o part_probe part_probe.cu
#include <cuda_runtime.h>
#include <algorithm>
#include <cstdio>
#include <cstdint>
#include <vector>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("{\"error\": \"%s line %d\"}\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

__device__ __forceinline__ uint32_t hash32(uint32_t a) {
  a ^= a >> 16; a *= 0x7feb352dU; a ^= a >> 15; a *= 0x846ca68bU; a ^= a >> 16; return a;
}

__global__ void k_fill(uint32_t *d, int64_t n, uint32_t mask) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    d[i] = hash32((uint32_t)i * 2654435761u + 12345u) & mask;
}

__global__ void k_g(const uint4 *d, int64_t n4, uint32_t *bm) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n4; i += (int64_t)gridDim.x * blockDim.x) {
    uint4 v = __ldcs(d + i);
    atomicOr(bm + (v.x >> 5), 1u << (v.x & 31));
    atomicOr(bm + (v.y >> 5), 1u << (v.y & 31));
    atomicOr(bm + (v.z >> 5), 1u << (v.z & 31));
    atomicOr(bm + (v.w >> 5), 1u << (v.w & 31));
  }
}

__global__ void k_b(const uint4 *d, int64_t n4, uint8_t *bytes) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n4; i += (int64_t)gridDim.x * blockDim.x) {
    uint4 v = __ldcs(d + i);
    bytes[v.x] = 1; bytes[v.y] = 1; bytes[v.z] = 1; bytes[v.w] = 1;
  }
}

__global__ void k_bytes_to_bits(const uint32_t *bytes4, uint32_t *bm, uint32_t nwords) {
  const uint32_t w = blockIdx.x * blockDim.x + threadIdx.x;
  if (w >= nwords) return;
  uint32_t acc = 0;
  for (int k = 0; k < 8; ++k) {
    const uint32_t q = bytes4[w * 8 + k];
    for (int j = 0; j < 4; ++j) acc |= ((q >> (8 * j)) & 1u) << (k * 4 + j);
  }
  bm[w] = acc;
}

constexpr int NT = 256, NB = 256;

// P1: one tile of TILE indices per iteration; bucket = v >> 16
template <int PER>
__global__ void __launch_bounds__(NT) k_p1(const uint32_t *d, int64_t n, uint16_t *bdata, uint32_t *bcnt, uint32_t cap,
                                           uint32_t *bm) {
  constexpr int TILE = NT * PER;
  __shared__ uint32_t hist[NB], base[NB], gbase[NB];
  __shared__ uint16_t keys[TILE];
  __shared__ uint8_t bid[TILE];
  const int t = threadIdx.x;
  for (int64_t t0 = (int64_t)blockIdx.x * TILE; t0 < n; t0 += (int64_t)gridDim.x * TILE) {
    const int cnt = (int)(n - t0 < TILE ? n - t0 : TILE);
    hist[t] = 0;  // NB == NT
    __syncthreads();
    uint32_t v[PER];
    uint32_t r[PER];
#pragma unroll
    for (int k = 0; k < PER; ++k) {
      const int i = k * NT + t;
      v[k] = i < cnt ? __ldcs(d + t0 + i) : 0xffffffffu;
    }
#pragma unroll
    for (int k = 0; k < PER; ++k)
      if (v[k] != 0xffffffffu) r[k] = atomicAdd(&hist[v[k] >> 16], 1u);
    __syncthreads();
    // exclusive scan of hist (NB = 256 = NT): warp scans + one pass over the 8 warp totals
    {
      const uint32_t h = hist[t];
      uint32_t x = h;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
        if ((t & 31) >= o) x += y;
      }
      __shared__ uint32_t wsum[NT / 32];
      if ((t & 31) == 31) wsum[t >> 5] = x;
      __syncthreads();
      uint32_t add = 0;
      for (int w = 0; w < (t >> 5); ++w) add += wsum[w];
      base[t] = x - h + add;
      gbase[t] = h ? atomicAdd(bcnt + t, h) : 0;
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < PER; ++k)
      if (v[k] != 0xffffffffu) {
        const uint32_t p = base[v[k] >> 16] + r[k];
        keys[p] = (uint16_t)v[k];
        bid[p] = (uint8_t)(v[k] >> 16);
      }
    __syncthreads();
    for (int i = t; i < cnt; i += NT) {
      const uint32_t b = bid[i];
      const uint32_t g = gbase[b] + (i - base[b]);
      if (g < cap) bdata[(size_t)b * cap + g] = keys[i];
      else atomicOr(bm + ((b << 16 | keys[i]) >> 5), 1u << (keys[i] & 31));
    }
    __syncthreads();
  }
}

// P2: block per bucket
__global__ void __launch_bounds__(512) k_p2(const uint16_t *bdata, const uint32_t *bcnt, uint32_t cap, uint32_t *bm) {
  __shared__ uint32_t s[2048];
  const uint32_t b = blockIdx.x;
  for (int w = threadIdx.x; w < 2048; w += blockDim.x) s[w] = 0;
  __syncthreads();
  const uint32_t c = min(bcnt[b], cap);
  const uint16_t *p = bdata + (size_t)b * cap;
  const uint32_t c8 = c / 8;
  const uint4 *p4 = reinterpret_cast<const uint4 *>(p);
  for (uint32_t i = threadIdx.x; i < c8; i += blockDim.x) {
    const uint4 q = __ldcs(p4 + i);
    const uint32_t w[4] = {q.x, q.y, q.z, q.w};
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const uint32_t lo = w[j] & 0xffff, hi = w[j] >> 16;
      atomicOr(s + (lo >> 5), 1u << (lo & 31));
      atomicOr(s + (hi >> 5), 1u << (hi & 31));
    }
  }
  for (uint32_t i = c8 * 8 + threadIdx.x; i < c; i += blockDim.x) atomicOr(s + (p[i] >> 5), 1u << (p[i] & 31));
  __syncthreads();
  for (int w = threadIdx.x; w < 2048; w += blockDim.x) {
    const uint32_t q = s[w];
    if (q) atomicOr(bm + b * 2048 + w, q);
  }
}

__global__ void k_popc(const uint32_t *bm, uint32_t nw, unsigned long long *out) {
  uint32_t c = 0;
  for (uint32_t w = blockIdx.x * blockDim.x + threadIdx.x; w < nw; w += gridDim.x * blockDim.x) c += __popc(bm[w]);
  atomicAdd(out, (unsigned long long)c);
}

template <typename F>
float med(F f, int reps = 12) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  std::vector<float> t;
  for (int r = 0; r < reps; ++r) {
    cudaEventRecord(a);
    f();
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    if (r >= 3) t.push_back(ms);
  }
  std::sort(t.begin(), t.end());
  return t[t.size() / 2];
}

int main(int argc, char **argv) {
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  const int64_t n = 268435456;
  const uint32_t nbits = 1u << 24, nw = nbits / 32;
  uint32_t *d, *bm, *bcnt;
  uint8_t *bytes;
  uint16_t *bdata;
  unsigned long long *cnt;
  const uint32_t cap = (uint32_t)(2 * n / NB);
  CK(cudaMalloc(&d, n * 4));
  CK(cudaMalloc(&bm, nbits / 8));
  CK(cudaMalloc(&bytes, nbits));
  CK(cudaMalloc(&bdata, (size_t)cap * NB * 2));
  CK(cudaMalloc(&bcnt, NB * 4));
  CK(cudaMalloc(&cnt, 8));
  k_fill<<<sms * 8, 256>>>(d, n, nbits - 1);
  CK(cudaDeviceSynchronize());
  auto count = [&]() {
    cudaMemset(cnt, 0, 8);
    k_popc<<<sms * 4, 256>>>(bm, nw, cnt);
    unsigned long long h;
    cudaMemcpy(&h, cnt, 8, cudaMemcpyDeviceToHost);
    return h;
  };
  const double clk = 1.965e9;
  auto line = [&](const char *name, float ms, unsigned long long c) {
    printf("{\"case\": \"%s\", \"ms\": %.4f, \"entries_per_sm_clk\": %.3f, \"count\": %llu}\n", name, ms,
           n / (ms * 1e-3) / sms / clk, c);
  };
  float ms = med([&] { cudaMemsetAsync(bm, 0, nbits / 8); k_g<<<sms * 8, 256>>>((const uint4 *)d, n / 4, bm); });
  CK(cudaGetLastError());
  line("G_global_red", ms, count());
  ms = med([&] {
    cudaMemsetAsync(bytes, 0, nbits);
    k_b<<<sms * 8, 256>>>((const uint4 *)d, n / 4, bytes);
    k_bytes_to_bits<<<(nw + 255) / 256, 256>>>((const uint32_t *)bytes, bm, nw);
  });
  CK(cudaGetLastError());
  line("B_byte_store", ms, count());
  auto runp = [&](auto kern, int per, int g) -> int {
    const int grid = sms * g;
    float ms1 = med([&] {
      cudaMemsetAsync(bcnt, 0, NB * 4);
      cudaMemsetAsync(bm, 0, nbits / 8);
      kern<<<grid, NT>>>(d, n, bdata, bcnt, cap, bm);
    });
    CK(cudaGetLastError());
    float ms2 = med([&] { k_p2<<<NB, 512>>>(bdata, bcnt, cap, bm); });
    CK(cudaGetLastError());
    float mst = med([&] {
      cudaMemsetAsync(bcnt, 0, NB * 4);
      cudaMemsetAsync(bm, 0, nbits / 8);
      kern<<<grid, NT>>>(d, n, bdata, bcnt, cap, bm);
      k_p2<<<NB, 512>>>(bdata, bcnt, cap, bm);
    });
    char nm[64];
    snprintf(nm, sizeof nm, "P_partition_per%d_grid%dx", per, g);
    line(nm, mst, count());
    printf("{\"case\": \"%s_parts\", \"p1_ms\": %.4f, \"p2_ms\": %.4f}\n", nm, ms1, ms2);
    return 0;
  };
  for (int g : {2, 3, 4}) runp(k_p1<32>, 32, g);
  for (int g : {4, 6, 8}) runp(k_p1<16>, 16, g);
  for (int g : {6, 8, 12, 16}) runp(k_p1<8>, 8, g);
  return 0;
}
