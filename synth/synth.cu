// synth/synth.cu — host (OpenMP) and device (CUDA) drivers of gen_core.h.
//
// Input generation only (see gen_core.h header): no SpMV/feature/conversion
// arithmetic lives here.  Both drivers call the same counter-based functions,
// so a matrix generated on the host equals the one generated on the device.
#include <cuda_runtime.h>
#include <omp.h>
#include <stdint.h>
#include <string.h>
#include "gen_core.h"

extern "C" {

/* Mirrors synth.SynthParams (ctypes) field by field. */
typedef struct {
  int32_t cls;       /* 1 stencil, 2 banded, 3 uniform, 4 rmat */
  int32_t kind;      /* stencil kind 1..5 */
  int64_t nx, ny, nz;
  int64_t N, M;      /* banded/uniform dims */
  int32_t band;      /* banded half bandwidth */
  int32_t k;         /* uniform mean row length */
  double density;    /* banded in-band density */
  int32_t variable;  /* uniform: variable lengths */
  int32_t scale;     /* rmat */
  double a, b, c;    /* rmat */
  int32_t permute;   /* rmat */
  int32_t mode;      /* stencil values: 0 Poisson ints, 1 random */
  uint64_t seed;
} synth_params;

}  // extern "C"

namespace {

template <typename T> struct VSel;
template <> struct VSel<float> {
  static SYN_HD float rnd(uint64_t h) { return syn_val32(h); }
  static SYN_HD float st(const synth_params &p, int64_t r, int64_t c) {
    return syn_stencil_value32(p.kind, p.mode, p.seed, r, c);
  }
};
template <> struct VSel<double> {
  static SYN_HD double rnd(uint64_t h) { return syn_val64(h); }
  static SYN_HD double st(const synth_params &p, int64_t r, int64_t c) {
    return syn_stencil_value(p.kind, p.mode, p.seed, r, c);
  }
};

__host__ __device__ inline int row_length(const synth_params &p, int64_t r) {
  switch (p.cls) {
    case 1: return syn_stencil_row(p.kind, p.nx, p.ny, p.nz, r, nullptr);
    case 2: {
      int n = 0;
      int64_t lo = r - p.band < 0 ? 0 : r - p.band, hi = r + p.band >= p.M ? p.M - 1 : r + p.band;
      for (int64_t c = lo; c <= hi; ++c) n += syn_banded_has(p.seed, r, c, p.density);
      return n;
    }
    case 3: return syn_uniform_len(p.seed, r, p.k, p.variable, p.M);
  }
  return 0;
}

template <typename T>
__host__ __device__ inline void row_fill(const synth_params &p, int64_t r, int32_t *col, T *val) {
  int64_t cols[SYN_UNIFORM_KMAX];
  int n = 0;
  switch (p.cls) {
    case 1:
      n = syn_stencil_row(p.kind, p.nx, p.ny, p.nz, r, cols);
      for (int i = 0; i < n; ++i) { col[i] = (int32_t)cols[i]; val[i] = VSel<T>::st(p, r, cols[i]); }
      return;
    case 2: {
      int64_t lo = r - p.band < 0 ? 0 : r - p.band, hi = r + p.band >= p.M ? p.M - 1 : r + p.band;
      for (int64_t c = lo; c <= hi; ++c)
        if (syn_banded_has(p.seed, r, c, p.density)) {
          col[n] = (int32_t)c;
          val[n] = VSel<T>::rnd(syn_h3(p.seed ^ SYN_SALT_VAL, (uint64_t)r, (uint64_t)c));
          ++n;
        }
      return;
    }
    case 3: {
      int L = syn_uniform_len(p.seed, r, p.k, p.variable, p.M);
      n = syn_uniform_row(p.seed, r, L, p.M, cols);
      for (int i = 0; i < n; ++i) {
        col[i] = (int32_t)cols[i];
        val[i] = VSel<T>::rnd(syn_h3(p.seed ^ SYN_SALT_VAL, (uint64_t)r, (uint64_t)cols[i]));
      }
      return;
    }
  }
}

__global__ void k_lengths(synth_params p, int64_t row0, int64_t nrows, int32_t *len) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nrows; i += (int64_t)gridDim.x * blockDim.x)
    len[i] = row_length(p, row0 + i);
}
template <typename T>
__global__ void k_fill(synth_params p, int64_t row0, int64_t nrows, const int64_t *rowptr, int32_t *col, T *val) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nrows; i += (int64_t)gridDim.x * blockDim.x) {
    int64_t o = rowptr[i];
    row_fill<T>(p, row0 + i, col + o, val + o);
  }
}
__global__ void k_rmat(synth_params p, uint64_t e0, uint64_t ne, uint64_t *keys) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < ne; i += (uint64_t)gridDim.x * blockDim.x)
    keys[i] = syn_rmat_key(p.seed, e0 + i, p.scale, p.a, p.b, p.c, p.permute);
}
template <typename T>
__global__ void k_values_rc(uint64_t seed, int64_t n, const int64_t *rows, const int32_t *cols, T *val) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    val[i] = VSel<T>::rnd(syn_h3(seed ^ SYN_SALT_VAL, (uint64_t)rows[i], (uint64_t)cols[i]));
}
template <typename T>
__global__ void k_vector(uint64_t seed, int64_t j0, int64_t n, int mode, T *out) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    if (sizeof(T) == 8) out[i] = (T)syn_x64(seed, j0 + i, mode);
    else out[i] = (T)syn_x32(seed, j0 + i, mode);
  }
}

int grid_for(int64_t n) {
  int64_t g = (n + 255) / 256;
  if (g > 148 * 64) g = 148 * 64;
  if (g < 1) g = 1;
  return (int)g;
}
int finish(cudaStream_t s) {
  cudaError_t e = cudaGetLastError();
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  return e == cudaSuccess ? 0 : (int)e;
}

}  // namespace

extern "C" {

int synth_lengths(int on_device, void *stream, const synth_params *pp, int64_t row0, int64_t nrows, int32_t *len) {
  synth_params p = *pp;
  if (on_device) {
    cudaStream_t s = (cudaStream_t)stream;
    if (nrows > 0) k_lengths<<<grid_for(nrows), 256, 0, s>>>(p, row0, nrows, len);
    return finish(s);
  }
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < nrows; ++i) len[i] = row_length(p, row0 + i);
  return 0;
}

int synth_fill(int on_device, void *stream, const synth_params *pp, int64_t row0, int64_t nrows,
               const int64_t *rowptr, int32_t *col, void *val, int is_fp64) {
  synth_params p = *pp;
  if (on_device) {
    cudaStream_t s = (cudaStream_t)stream;
    if (nrows > 0) {
      if (is_fp64) k_fill<double><<<grid_for(nrows), 256, 0, s>>>(p, row0, nrows, rowptr, col, (double *)val);
      else k_fill<float><<<grid_for(nrows), 256, 0, s>>>(p, row0, nrows, rowptr, col, (float *)val);
    }
    return finish(s);
  }
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t i = 0; i < nrows; ++i) {
    int64_t o = rowptr[i];
    if (is_fp64) row_fill<double>(p, row0 + i, col + o, (double *)val + o);
    else row_fill<float>(p, row0 + i, col + o, (float *)val + o);
  }
  return 0;
}

int synth_rmat_keys(int on_device, void *stream, const synth_params *pp, uint64_t e0, uint64_t ne, uint64_t *keys) {
  synth_params p = *pp;
  if (on_device) {
    cudaStream_t s = (cudaStream_t)stream;
    if (ne > 0) k_rmat<<<grid_for((int64_t)ne), 256, 0, s>>>(p, e0, ne, keys);
    return finish(s);
  }
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < (int64_t)ne; ++i) keys[i] = syn_rmat_key(p.seed, e0 + i, p.scale, p.a, p.b, p.c, p.permute);
  return 0;
}

int synth_values_rc(int on_device, void *stream, uint64_t seed, int64_t n, const int64_t *rows,
                    const int32_t *cols, void *val, int is_fp64) {
  if (on_device) {
    cudaStream_t s = (cudaStream_t)stream;
    if (n > 0) {
      if (is_fp64) k_values_rc<double><<<grid_for(n), 256, 0, s>>>(seed, n, rows, cols, (double *)val);
      else k_values_rc<float><<<grid_for(n), 256, 0, s>>>(seed, n, rows, cols, (float *)val);
    }
    return finish(s);
  }
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) {
    uint64_t h = syn_h3(seed ^ SYN_SALT_VAL, (uint64_t)rows[i], (uint64_t)cols[i]);
    if (is_fp64) ((double *)val)[i] = syn_val64(h);
    else ((float *)val)[i] = syn_val32(h);
  }
  return 0;
}

int synth_vector(int on_device, void *stream, uint64_t seed, int64_t j0, int64_t n, int mode, void *out, int is_fp64) {
  if (on_device) {
    cudaStream_t s = (cudaStream_t)stream;
    if (n > 0) {
      if (is_fp64) k_vector<double><<<grid_for(n), 256, 0, s>>>(seed, j0, n, mode, (double *)out);
      else k_vector<float><<<grid_for(n), 256, 0, s>>>(seed, j0, n, mode, (float *)out);
    }
    return finish(s);
  }
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) {
    if (is_fp64) ((double *)out)[i] = syn_x64(seed, j0 + i, mode);
    else ((float *)out)[i] = syn_x32(seed, j0 + i, mode);
  }
  return 0;
}

int synth_params_size(void) { return (int)sizeof(synth_params); }

}  // extern "C"
