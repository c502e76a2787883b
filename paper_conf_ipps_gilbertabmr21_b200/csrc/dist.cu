// dist.cu — coarse-vertex-range construction for the multi-GPU path (§8(e)).
#include "hec_internal.cuh"

using namespace hec;

extern "C" {
HEC_API int hec_build_rows_count(hec_ctx *ctx, const hec_graph *g, const int32_t *M, int64_t n_c,
                                 int64_t a_begin, int64_t a_end, int64_t *counts) {
  (void)ctx; (void)g; (void)M; (void)n_c; (void)a_begin; (void)a_end; (void)counts;
  set_error("hec_build_rows_count: not implemented yet");
  return HEC_EINVAL;
}
HEC_API int hec_build_rows_write(hec_ctx *ctx, const int64_t *offs, int32_t *col_c, int32_t *wgt_c,
                                 int32_t *vwgt_c) {
  (void)ctx; (void)offs; (void)col_c; (void)wgt_c; (void)vwgt_c;
  set_error("hec_build_rows_write: not implemented yet");
  return HEC_EINVAL;
}
}
