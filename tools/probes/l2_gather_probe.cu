// l2_gather_probe.cu — the L2 random-gather bound of the random-column SpMV
// classes (configs[2] uniform rows: every nonzero gathers one x value through
// its own 32-byte L2 sector; x = 32 MB fp32 / 64 MB fp64 stays L2-resident).
//
// Measures, with CUDA events (median of 15, after warm-up):
//  A. gathers only: each thread issues U independent loads x[h(i) mod M]
//     (h = a multiplicative hash: no index stream) -> random sectors/s of L2;
//  B. an index stream + gather (the ELL/CSR inner loop without values): int32
//     column ids streamed from HBM (evict-first), x gathered;
//  C. B + a value stream (4 B or 8 B): the full c2a / c2b per-entry traffic.
//  D. plain HBM read stream of the same bytes as C (no gather): the HBM leg.
// Prints one JSON line per case: entries/s, ns/entry, L2 sector GB/s
// (32 B per gather + streamed bytes) and streamed HBM GB/s.
//
// build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o l2_gather_probe l2_gather_probe.cu
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <vector>
#include <algorithm>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

__device__ __forceinline__ uint32_t hash32(uint32_t a) {
  a ^= a >> 16; a *= 0x7feb352dU; a ^= a >> 15; a *= 0x846ca68bU; a ^= a >> 16; return a;
}

template <typename T, int U>
__global__ void __launch_bounds__(256) k_gather_only(const T *__restrict__ x, uint32_t M, int64_t n, T *out) {
  T acc = 0;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x * U;
  for (int64_t b = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) * U; b < n; b += stride) {
    T v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) v[u] = __ldg(x + hash32((uint32_t)(b + u)) % M);
#pragma unroll
    for (int u = 0; u < U; ++u) acc += v[u];
  }
  if (acc == (T)12345.678) out[0] = acc;
}

__device__ __forceinline__ int4 ld_ef(const int4 *p, uint64_t pol) {
  int4 r;
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.s32 {%0,%1,%2,%3}, [%4], %5;"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p), "l"(pol));
  return r;
}

// each thread: 4 consecutive entries per step (int4 column ids, + values), U steps in flight
template <typename T, int U, bool VALS>
__global__ void __launch_bounds__(256) k_stream_gather(const int32_t *__restrict__ col, const T *__restrict__ val,
                                                       const T *__restrict__ x, int64_t n4, T *out) {
  uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  T acc = 0;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x * U;
  for (int64_t b = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x); b < n4; b += stride) {
    int4 c[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t q = b + (int64_t)u * gridDim.x * blockDim.x;
      c[u] = q < n4 ? ld_ef(reinterpret_cast<const int4 *>(col) + q, pol) : make_int4(0, 0, 0, 0);
    }
    T w[U][4];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t q = b + (int64_t)u * gridDim.x * blockDim.x;
      if (VALS && q < n4) {
        if (sizeof(T) == 4) {
          int4 t = ld_ef(reinterpret_cast<const int4 *>(val) + q, pol);
          w[u][0] = __int_as_float(t.x); w[u][1] = __int_as_float(t.y); w[u][2] = __int_as_float(t.z); w[u][3] = __int_as_float(t.w);
        } else {
          int4 t0 = ld_ef(reinterpret_cast<const int4 *>(val) + 2 * q, pol);
          int4 t1 = ld_ef(reinterpret_cast<const int4 *>(val) + 2 * q + 1, pol);
          w[u][0] = __hiloint2double(t0.y, t0.x); w[u][1] = __hiloint2double(t0.w, t0.z);
          w[u][2] = __hiloint2double(t1.y, t1.x); w[u][3] = __hiloint2double(t1.w, t1.z);
        }
      } else {
        w[u][0] = w[u][1] = w[u][2] = w[u][3] = (T)1;
      }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      acc += w[u][0] * __ldg(x + c[u].x) + w[u][1] * __ldg(x + c[u].y) + w[u][2] * __ldg(x + c[u].z) +
             w[u][3] * __ldg(x + c[u].w);
    }
  }
  if (acc == (T)12345.678) out[0] = acc;
}

template <int U>
__global__ void __launch_bounds__(256) k_stream_only(const int4 *__restrict__ a, int64_t n, int *out) {
  uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  int acc = 0;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t b = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; b < n; b += stride * U) {
    int4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) v[u] = b + u * stride < n ? ld_ef(a + b + u * stride, pol) : make_int4(0, 0, 0, 0);
#pragma unroll
    for (int u = 0; u < U; ++u) acc ^= v[u].x ^ v[u].y ^ v[u].z ^ v[u].w;
  }
  if (acc == 0x7fffffff) out[0] = acc;
}

__global__ void k_fill_cols(int32_t *col, int64_t n, uint32_t M) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    col[i] = (int32_t)(hash32((uint32_t)i * 2654435761u + 17u) % M);
}

__global__ void k_flush(const int4 *buf, int64_t n, int *sink) {
  int acc = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    int4 v = __ldcg(buf + i);
    acc ^= v.x ^ v.y ^ v.z ^ v.w;
  }
  if (acc == 0x7fffffff) *sink = acc;
}

template <typename F>
float time_med(F f, int reps, const int4 *fl, int64_t fn, int *sink, int sms, bool flush) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  std::vector<float> t;
  for (int r = 0; r < reps + 3; ++r) {
    if (flush) k_flush<<<sms * 8, 256>>>(fl, fn, sink);
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

int main() {
  int dev = 0, sms = 0, l2 = 0;
  CK(cudaSetDevice(dev));
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
  CK(cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, dev));
  const uint32_t M = 1u << 23;           // configs[2]: 2^23 columns
  const int64_t Z = (int64_t)M * 32;     // c2a: 32 entries per row
  float *xf;
  double *xd;
  int32_t *col;
  float *vf;
  double *vd;
  int *sink;
  int4 *fl;
  const int64_t fn = (int64_t)l2 * 3 / 16;
  CK(cudaMalloc(&xf, M * 4));
  CK(cudaMalloc(&xd, M * 8));
  CK(cudaMalloc(&col, Z * 4));
  CK(cudaMalloc(&vf, Z * 4));
  CK(cudaMalloc(&vd, Z * 8));
  CK(cudaMalloc(&sink, 64));
  CK(cudaMalloc(&fl, fn * 16));
  CK(cudaMemset(xf, 0, M * 4));
  CK(cudaMemset(xd, 0, M * 8));
  CK(cudaMemset(vf, 0, Z * 4));
  CK(cudaMemset(vd, 0, Z * 8));
  CK(cudaMemset(fl, 1, fn * 16));
  k_fill_cols<<<sms * 8, 256>>>(col, Z, M);
  CK(cudaDeviceSynchronize());
  printf("{\"probe\": \"l2_gather\", \"sms\": %d, \"l2_bytes\": %d, \"entries\": %lld}\n", sms, l2, (long long)Z);
  auto report = [&](const char *name, int bpsm, int U, float ms, double streamed, double gathers, int gbytes) {
    const double s = ms * 1e-3;
    printf("{\"case\": \"%s\", \"ctas_per_sm\": %d, \"U\": %d, \"ms\": %.4f, \"ns_per_entry\": %.5f, "
           "\"gathers_per_s\": %.4g, \"l2_sector_gbs\": %.1f, \"stream_gbs\": %.1f}\n",
           name, bpsm, U, ms, s / gathers * 1e9, gathers / s, (gathers * 32 + streamed) / s / 1e9,
           streamed / s / 1e9);
    (void)gbytes;
  };
  // A: gathers only (L2-resident x; no flush between reps so x stays hot)
  for (int bpsm : {4, 8, 16}) {
    float ms;
    ms = time_med([&] { k_gather_only<float, 4><<<sms * bpsm, 256>>>(xf, M, Z, xf); }, 15, fl, fn, sink, sms, false);
    report("A_gather_only_f32", bpsm, 4, ms, 0, (double)Z, 4);
    ms = time_med([&] { k_gather_only<float, 8><<<sms * bpsm, 256>>>(xf, M, Z, xf); }, 15, fl, fn, sink, sms, false);
    report("A_gather_only_f32", bpsm, 8, ms, 0, (double)Z, 4);
    ms = time_med([&] { k_gather_only<double, 4><<<sms * bpsm, 256>>>(xd, M, Z, xd); }, 15, fl, fn, sink, sms, false);
    report("A_gather_only_f64", bpsm, 4, ms, 0, (double)Z, 8);
  }
  // B, C, D: L2 flushed before each rep (matrix streams cold, x re-warms)
  for (int bpsm : {4, 8, 16}) {
    float ms;
    ms = time_med([&] { k_stream_gather<float, 1, false><<<sms * bpsm, 256>>>(col, vf, xf, Z / 4, xf); }, 15, fl, fn, sink, sms, true);
    report("B_colstream_gather_f32", bpsm, 1, ms, Z * 4.0, (double)Z, 4);
    ms = time_med([&] { k_stream_gather<float, 2, false><<<sms * bpsm, 256>>>(col, vf, xf, Z / 4, xf); }, 15, fl, fn, sink, sms, true);
    report("B_colstream_gather_f32", bpsm, 2, ms, Z * 4.0, (double)Z, 4);
    ms = time_med([&] { k_stream_gather<float, 1, true><<<sms * bpsm, 256>>>(col, vf, xf, Z / 4, xf); }, 15, fl, fn, sink, sms, true);
    report("C_full_entry_f32", bpsm, 1, ms, Z * 8.0, (double)Z, 4);
    ms = time_med([&] { k_stream_gather<float, 2, true><<<sms * bpsm, 256>>>(col, vf, xf, Z / 4, xf); }, 15, fl, fn, sink, sms, true);
    report("C_full_entry_f32", bpsm, 2, ms, Z * 8.0, (double)Z, 4);
    ms = time_med([&] { k_stream_gather<double, 1, true><<<sms * bpsm, 256>>>(col, vd, xd, Z / 4, xd); }, 15, fl, fn, sink, sms, true);
    report("C_full_entry_f64", bpsm, 1, ms, Z * 12.0, (double)Z, 8);
    ms = time_med([&] { k_stream_only<2><<<sms * bpsm, 256>>>(reinterpret_cast<const int4 *>(vd), Z * 8 / 16, sink); }, 15, fl, fn, sink, sms, true);
    report("D_stream_only", bpsm, 2, ms, Z * 8.0, 1e-30, 0);
  }
  CK(cudaGetLastError());
  return 0;
}
