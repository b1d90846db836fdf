// dsmem_probe.cu — throughput of random bitmap ORs (the feature pass's
// occupied-diagonal bits on random-column matrices, configs[2] uniform: 268 M
// entries over a 2^24-bit bitmap):
//   G: fire-and-forget global red.or into a 2 MB bitmap (what K1 does),
//   D: red.shared::cluster.or into a cluster-distributed bitmap (16 CTAs x 128 KB
//      = 2^24 bits; non-portable cluster size 16), then
//   L: red.shared.or into the CTA's own 128 KB slice (the local-only bound).
// One JSON line per case: ops/s and ns per op (median of 9).
// build: nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -o dsmem_probe dsmem_probe.cu
#include <cooperative_groups.h>
#include <cuda_runtime.h>
#include <algorithm>
#include <cstdio>
#include <vector>
namespace cg = cooperative_groups;

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("{\"error\": \"%s line %d\"}\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

__device__ __forceinline__ uint32_t hash32(uint32_t a) {
  a ^= a >> 16; a *= 0x7feb352dU; a ^= a >> 15; a *= 0x846ca68bU; a ^= a >> 16; return a;
}

__global__ void k_global(uint32_t *bm, int64_t n_ops, uint32_t nbits) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n_ops; i += stride) {
    const uint32_t b = hash32((uint32_t)i) & (nbits - 1);
    atomicOr(bm + (b >> 5), 1u << (b & 31));
  }
}

template <int CL, bool REMOTE>
__global__ void __cluster_dims__(CL, 1, 1) k_dsm(uint32_t *out, int64_t n_ops_per_cluster, uint32_t slice_words) {
  extern __shared__ uint32_t slice[];
  cg::cluster_group cl = cg::this_cluster();
  for (uint32_t w = threadIdx.x; w < slice_words; w += blockDim.x) slice[w] = 0;
  cl.sync();
  const uint32_t rank = cl.block_rank();
  const int64_t per_cta = n_ops_per_cluster / CL;
  const uint32_t slice_bits = slice_words * 32;
  for (int64_t i = threadIdx.x; i < per_cta; i += blockDim.x) {
    const uint32_t h = hash32((uint32_t)(i * CL + rank + (int64_t)blockIdx.x * 7919));
    const uint32_t target = REMOTE ? (h >> 24) % CL : rank;
    const uint32_t b = h & (slice_bits - 1);
    uint32_t *dst = cl.map_shared_rank(slice, (int)target);
    atomicOr(dst + (b >> 5), 1u << (b & 31));
  }
  cl.sync();
  if (threadIdx.x == 0) out[blockIdx.x] = slice[0];
}

template <typename F>
float med(F f) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  std::vector<float> t;
  for (int r = 0; r < 12; ++r) {
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

template <int CL>
int run_dsm(int sms, int64_t n_ops, uint32_t slice_bytes, const char *name) {
  uint32_t *out;
  CK(cudaMalloc(&out, 4096 * 4));
  CK(cudaFuncSetAttribute(k_dsm<CL, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)slice_bytes));
  CK(cudaFuncSetAttribute(k_dsm<CL, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)slice_bytes));
  if (CL > 8) {
    CK(cudaFuncSetAttribute(k_dsm<CL, true>, cudaFuncAttributeNonPortableClusterSizeAllowed, 1));
    CK(cudaFuncSetAttribute(k_dsm<CL, false>, cudaFuncAttributeNonPortableClusterSizeAllowed, 1));
  }
  cudaLaunchConfig_t cfg = {};
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = CL; attr[0].val.clusterDim.y = 1; attr[0].val.clusterDim.z = 1;
  cfg.blockDim = dim3(1024);
  cfg.dynamicSmemBytes = slice_bytes;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  int ncl = 0;
  cfg.gridDim = dim3(CL);
  CK(cudaOccupancyMaxActiveClusters(&ncl, k_dsm<CL, true>, &cfg));
  if (ncl <= 0) { printf("{\"case\": \"%s\", \"clusters\": 0}\n", name); return 0; }
  cfg.gridDim = dim3(CL * ncl);
  const int64_t per_cluster = n_ops / ncl;
  const uint32_t sw = slice_bytes / 4;
  for (int remote = 1; remote >= 0; --remote) {
    float ms = med([&] {
      if (remote) cudaLaunchKernelEx(&cfg, k_dsm<CL, true>, out, per_cluster, sw);
      else cudaLaunchKernelEx(&cfg, k_dsm<CL, false>, out, per_cluster, sw);
    });
    CK(cudaGetLastError());
    printf("{\"case\": \"%s_%s\", \"cluster\": %d, \"clusters\": %d, \"ctas\": %d, \"ms\": %.4f, \"ops_per_s\": %.4g, "
           "\"ops_per_sm_clk\": %.3f}\n", name, remote ? "remote" : "local", CL, ncl, CL * ncl, ms, n_ops / (ms * 1e-3),
           n_ops / (ms * 1e-3) / (CL * ncl) / 1.965e9);
  }
  return 0;
}

int main() {
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  const int64_t n_ops = 268435456;  // configs[2] uniform: 2^23 rows x 32
  uint32_t *bm;
  CK(cudaMalloc(&bm, (1u << 24) / 8));
  CK(cudaMemset(bm, 0, (1u << 24) / 8));
  float ms = med([&] { k_global<<<sms * 8, 256>>>(bm, n_ops, 1u << 24); });
  CK(cudaGetLastError());
  printf("{\"case\": \"global_red_2MB\", \"ms\": %.4f, \"ops_per_s\": %.4g, \"ops_per_sm_clk\": %.3f}\n", ms,
         n_ops / (ms * 1e-3), n_ops / (ms * 1e-3) / sms / 1.965e9);
  run_dsm<16>(sms, n_ops, 128 * 1024, "dsm16_128KB");
  run_dsm<8>(sms, n_ops, 200 * 1024, "dsm8_200KB");
  run_dsm<4>(sms, n_ops, 200 * 1024, "dsm4_200KB");
  return 0;
}
