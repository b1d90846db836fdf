/* synth/gen_core.h — counter-based synthetic input generators.
 *
 * This module is the ONE piece shared by the CPU oracle side and the GPU
 * product side (tests and bench feed both from it).  It holds no arithmetic
 * of the method (no SpMV, no features, no conversions): it only decides which
 * (row, col, value) triples exist in a synthetic matrix and what x holds.
 *
 * Every quantity is a pure function of (seed, counters) through splitmix64, so
 * the host (OpenMP) and device (CUDA) builds produce identical matrices
 * without sharing state.  Matrix classes follow the paper's workload mix
 * (§IV: UFL matrices + 13 stencil matrices) as restated in
 * stencils, banded, uniform-random rows, R-MAT power law.
 */
#ifndef SYNTH_GEN_CORE_H
#define SYNTH_GEN_CORE_H

#include <stdint.h>

#if defined(__CUDACC__)
#define SYN_HD __host__ __device__ __forceinline__
#else
#define SYN_HD static inline
#endif

/* splitmix64 finaliser (Steele, Lea, Flood 2014). */
SYN_HD uint64_t syn_mix(uint64_t z) {
  z += 0x9E3779B97F4A7C15ULL;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}
SYN_HD uint64_t syn_h2(uint64_t seed, uint64_t a) { return syn_mix(syn_mix(seed) ^ a); }
SYN_HD uint64_t syn_h3(uint64_t seed, uint64_t a, uint64_t b) {
  return syn_mix(syn_mix(syn_mix(seed) ^ a) ^ (b * 0xD1B54A32D192ED03ULL));
}

/* uniform in (0,1), 53-bit */
SYN_HD double syn_unit(uint64_t h) { return ((double)(h >> 11) + 0.5) * 0x1p-53; }

/* U(-1,1) without 0, exactly representable in the target precision:
 * fp64: odd integer in (-2^52, 2^52) times 2^-52; fp32: odd integer in
 * (-2^23, 2^23) times 2^-23.  Odd => never zero (canonical CSR stores no
 * zeros). */
SYN_HD double syn_val64(uint64_t h) {
  int64_t k = (int64_t)(h >> 12);                     /* < 2^52 */
  return (double)(2 * k + 1 - (1LL << 52)) * 0x1p-52;
}
SYN_HD float syn_val32(uint64_t h) {
  int32_t k = (int32_t)(h >> 41);                     /* < 2^23 */
  return (float)(2 * k + 1 - (1 << 23)) * 0x1p-23f;
}

/* value salt so matrix values and structure draw independent streams */
#define SYN_SALT_VAL 0x5A17A11DULL
#define SYN_SALT_X   0x0C0FFEEULL
#define SYN_SALT_LEN 0x1E6D17ULL

/* ---------------------------------------------------------------- stencils
 * kind: 1 = 1D 3-pt, 2 = 2D 5-pt, 3 = 2D 9-pt, 4 = 3D 7-pt, 5 = 3D 27-pt.
 * Grid nx*ny*nz, row r = x + nx*(y + ny*z).  Neighbours are enumerated in
 * (dz,dy,dx) lexicographic order, which is ascending column order.
 * Value modes: 0 = Poisson-style integers (centre = npts-1, others = -1),
 *              1 = random U(-1,1)\{0} from hash(seed,row,col). */
SYN_HD int syn_stencil_npts(int kind) {
  switch (kind) { case 1: return 3; case 2: return 5; case 3: return 9; case 4: return 7; case 5: return 27; }
  return 0;
}
/* i-th point (0-based, in column order) of stencil `kind`. */
SYN_HD void syn_stencil_point(int kind, int i, int *dz, int *dy, int *dx) {
  *dz = 0; *dy = 0; *dx = 0;
  switch (kind) {
    case 1: *dx = i - 1; break;
    case 2: { const int t[5][2] = {{-1, 0}, {0, -1}, {0, 0}, {0, 1}, {1, 0}}; *dy = t[i][0]; *dx = t[i][1]; } break;
    case 3: *dy = i / 3 - 1; *dx = i % 3 - 1; break;
    case 4: { const int t[7][3] = {{-1,0,0},{0,-1,0},{0,0,-1},{0,0,0},{0,0,1},{0,1,0},{1,0,0}};
              *dz = t[i][0]; *dy = t[i][1]; *dx = t[i][2]; } break;
    case 5: *dz = i / 9 - 1; *dy = (i / 3) % 3 - 1; *dx = i % 3 - 1; break;
  }
}
SYN_HD int syn_stencil_row(int kind, int64_t nx, int64_t ny, int64_t nz, int64_t r,
                           int64_t *cols /* nullable, >= 27 */) {
  int64_t x = r % nx, y = (r / nx) % ny, z = r / (nx * ny);
  int n = 0, np = syn_stencil_npts(kind);
  for (int i = 0; i < np; ++i) {
    int dz, dy, dx; syn_stencil_point(kind, i, &dz, &dy, &dx);
    int64_t X = x + dx, Y = y + dy, Z = z + dz;
    if (X < 0 || X >= nx || Y < 0 || Y >= ny || Z < 0 || Z >= nz) continue;
    if (cols) cols[n] = X + nx * (Y + ny * Z);
    ++n;
  }
  return n;
}
SYN_HD double syn_stencil_value(int kind, int mode, uint64_t seed, int64_t r, int64_t c) {
  if (mode == 0) return (r == c) ? (double)(syn_stencil_npts(kind) - 1) : -1.0;
  return syn_val64(syn_h3(seed ^ SYN_SALT_VAL, (uint64_t)r, (uint64_t)c));
}
SYN_HD float syn_stencil_value32(int kind, int mode, uint64_t seed, int64_t r, int64_t c) {
  if (mode == 0) return (r == c) ? (float)(syn_stencil_npts(kind) - 1) : -1.0f;
  return syn_val32(syn_h3(seed ^ SYN_SALT_VAL, (uint64_t)r, (uint64_t)c));
}

/* ---------------------------------------------------------------- banded
 * Row r holds column c in [r-b, r+b] ∩ [0,M) iff c == r or unit(h) < density. */
SYN_HD int syn_banded_has(uint64_t seed, int64_t r, int64_t c, double density) {
  if (r == c) return 1;
  if (density >= 1.0) return 1;
  return syn_unit(syn_h3(seed, (uint64_t)r, (uint64_t)c)) < density;
}

/* ---------------------------------------------------------------- uniform
 * Row length k (fixed) or U{floor(k/2) .. floor(k/2)+k} (variable); columns drawn
 * uniformly without replacement by rejection, then sorted ascending. */
#define SYN_UNIFORM_KMAX 256
SYN_HD int syn_uniform_len(uint64_t seed, int64_t r, int k, int variable, int64_t M) {
  int L = k;
  if (variable) L = k / 2 + (int)((syn_h2(seed ^ SYN_SALT_LEN, (uint64_t)r) >> 33) % (uint64_t)(k + 1));
  if (L > SYN_UNIFORM_KMAX) L = SYN_UNIFORM_KMAX;
  if ((int64_t)L > M) L = (int)M;
  return L;
}
/* fills cols[0..L) sorted ascending; returns L */
SYN_HD int syn_uniform_row(uint64_t seed, int64_t r, int L, int64_t M, int64_t *cols) {
  int n = 0;
  for (uint64_t t = 0; n < L; ++t) {
    uint64_t h = syn_h3(seed, (uint64_t)r, t);
    int64_t c = (int64_t)(((h >> 32) * (uint64_t)M) >> 32);
    if (M > 0xFFFFFFFFLL) c = (int64_t)(h % (uint64_t)M);
    int dup = 0;
    for (int j = 0; j < n; ++j) dup |= (cols[j] == c);
    if (dup) continue;
    /* insertion into sorted position */
    int j = n++;
    while (j > 0 && cols[j - 1] > c) { cols[j] = cols[j - 1]; --j; }
    cols[j] = c;
  }
  return n;
}

/* ---------------------------------------------------------------- R-MAT
 * Edge e descends `scale` levels of the 2x2 recursive partition with
 * probabilities (a, b, c, 1-a-b-c), then both endpoints are passed through a
 * seeded bijection of [0, 2^scale) (vertex relabelling).  Key = row<<scale|col. */
SYN_HD uint64_t syn_perm(uint64_t v, uint64_t seed, int scale) {
  uint64_t mask = (scale >= 64) ? ~0ULL : ((1ULL << scale) - 1);
  int s = (scale + 1) / 2; if (s < 1) s = 1;
  v = (v * 0x9E3779B97F4A7C15ULL) & mask;
  v ^= v >> s;
  v = (v * 0xBF58476D1CE4E5B9ULL + (syn_mix(seed) & mask)) & mask;
  v ^= v >> s;
  v = (v * 0x94D049BB133111EBULL) & mask;
  return v;
}
SYN_HD uint64_t syn_rmat_key(uint64_t seed, uint64_t e, int scale, double a, double b, double c, int permute) {
  uint64_t row = 0, col = 0;
  for (int l = 0; l < scale; ++l) {
    double u = syn_unit(syn_h3(seed, e, (uint64_t)l));
    int rb = 0, cb = 0;
    if (u < a) { } else if (u < a + b) { cb = 1; } else if (u < a + b + c) { rb = 1; } else { rb = 1; cb = 1; }
    row = (row << 1) | (uint64_t)rb;
    col = (col << 1) | (uint64_t)cb;
  }
  if (permute) { row = syn_perm(row, seed ^ 0x1111ULL, scale); col = syn_perm(col, seed ^ 0x1111ULL, scale); }
  return (row << scale) | col;
}

/* ---------------------------------------------------------------- vectors
 * mode 0: U(-1,1)\{0}; mode 1: integers U{-8..8}; mode 2: all ones. */
SYN_HD double syn_x64(uint64_t seed, int64_t j, int mode) {
  if (mode == 2) return 1.0;
  uint64_t h = syn_h2(seed ^ SYN_SALT_X, (uint64_t)j);
  if (mode == 1) return (double)((int)((h >> 32) % 17u) - 8);
  return syn_val64(h);
}
SYN_HD float syn_x32(uint64_t seed, int64_t j, int mode) {
  if (mode == 2) return 1.0f;
  uint64_t h = syn_h2(seed ^ SYN_SALT_X, (uint64_t)j);
  if (mode == 1) return (float)((int)((h >> 32) % 17u) - 8);
  return syn_val32(h);
}

#endif
