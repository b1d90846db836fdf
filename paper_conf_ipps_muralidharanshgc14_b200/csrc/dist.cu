// dist.cu — multi-GPU row-partitioned SpMV (include/nitro.h §3).
// (Implementation follows in a later commit; entry points exist so the ABI is complete.)
#include "nitro_internal.h"

using namespace nitro;

extern "C" {

nitro_status_t nitro_dist_unique_id(void *) { return fail(NITRO_E_UNSUPPORTED, "multi-GPU path not built yet"); }
nitro_status_t nitro_dist_init(const void *, int, int, int, nitro_dist **) {
  return fail(NITRO_E_UNSUPPORTED, "multi-GPU path not built yet");
}
void nitro_dist_destroy(nitro_dist *) {}
nitro_status_t nitro_dist_partition(int64_t rows, const int64_t *h_rowptr, int nranks, int64_t *bounds) {
  if (rows < 0 || !h_rowptr || nranks < 1 || !bounds) return fail(NITRO_E_INVALID_ARG, "bad argument");
  const int64_t Z = h_rowptr[rows];
  bounds[0] = 0;
  for (int r = 1; r < nranks; ++r) {
    const int64_t target = (r * Z + nranks - 1) / nranks;  // ceil(r Z / P)
    int64_t lo = 0, hi = rows;                              // first i with rowptr[i] >= target
    while (lo < hi) {
      int64_t mid = (lo + hi) / 2;
      if (h_rowptr[mid] < target) lo = mid + 1; else hi = mid;
    }
    bounds[r] = lo;
  }
  bounds[nranks] = rows;
  return NITRO_OK;
}
nitro_status_t nitro_dist_spmv_create(nitro_dist *, int64_t, const int64_t *, int64_t, const void *, int,
                                      const int32_t *, const void *, int, nitro_spmv **) {
  return fail(NITRO_E_UNSUPPORTED, "multi-GPU path not built yet");
}
nitro_status_t nitro_dist_spmv_run(nitro_dist *, nitro_spmv *, int, const void *, void *) {
  return fail(NITRO_E_UNSUPPORTED, "multi-GPU path not built yet");
}
nitro_status_t nitro_dist_features(nitro_dist *, nitro_spmv *, nitro_spmv_feat *) {
  return fail(NITRO_E_UNSUPPORTED, "multi-GPU path not built yet");
}

}  // extern "C"
