// validate.cu — optional device check of the input contract R1 (PAPER.md:L59:
// undirected, no self-loops, no parallel edges, positive weights; CSR stores
// each edge in both rows, L280).  Enabled with hec_ctx_set_validate(ctx, 1).
#include "hec_internal.cuh"

namespace hec {

enum {
  V_ROWPTR = 1,      // row_ptr[0] != 0, row_ptr[n] != nnz or decreasing
  V_RANGE = 2,       // column out of [0, n)
  V_ORDER = 4,       // columns not strictly ascending (duplicate / unsorted)
  V_LOOP = 8,        // self-loop
  V_WEIGHT = 16,     // weight <= 0
  V_ASYM = 32,       // (u,v,w) without (v,u,w)
  V_VWGT = 64        // vertex weight <= 0
};

__global__ void k_validate(int64_t n, int64_t nnz, const int64_t *__restrict__ row_ptr,
                           const int32_t *__restrict__ col, const int32_t *__restrict__ wgt,
                           const int32_t *__restrict__ vwgt, int *__restrict__ flags) {
  const int lane = threadIdx.x & 31;
  const int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  if (w == 0 && lane == 0) {
    if (row_ptr[0] != 0 || row_ptr[n] != nnz) atomicOr(flags, V_ROWPTR);
  }
  for (int64_t u = w; u < n; u += nw) {
    int64_t b = row_ptr[u], e = row_ptr[u + 1];
    if (e < b) { if (lane == 0) atomicOr(flags, V_ROWPTR); continue; }
    if (b < 0 || e > nnz) { if (lane == 0) atomicOr(flags, V_ROWPTR); continue; }
    if (lane == 0 && vwgt && vwgt[u] <= 0) atomicOr(flags, V_VWGT);
    int f = 0;
    for (int64_t i = b + lane; i < e; i += 32) {
      int32_t v = col[i];
      int32_t x = wgt[i];
      if (v < 0 || v >= n) { f |= V_RANGE; continue; }
      if (v == (int32_t)u) f |= V_LOOP;
      if (x <= 0) f |= V_WEIGHT;
      if (i > b && col[i - 1] >= v) f |= V_ORDER;
      // symmetric entry: binary search u in row v
      int64_t lo = row_ptr[v], hi = row_ptr[v + 1] - 1;
      bool found = false;
      while (lo <= hi) {
        int64_t mid = (lo + hi) >> 1;
        int32_t c = col[mid];
        if (c == (int32_t)u) { found = wgt[mid] == x; break; }
        if (c < (int32_t)u) lo = mid + 1;
        else hi = mid - 1;
      }
      if (!found) f |= V_ASYM;
    }
    if (f) atomicOr(flags, f);
  }
}

int validate_graph(hec_ctx *ctx, const hec_graph *g) {
  if (g->n == 0) return HEC_OK;
  int *flags = nullptr;
  HEC_TRY(dev_alloc(ctx, (void **)&flags, 64));
  HEC_CUDA_TRY(cudaMemsetAsync(flags, 0, 64, ctx->stream));
  int64_t blocks = (g->n * 32 + 255) / 256;
  int64_t cap = (int64_t)ctx->num_sms * 16;
  if (blocks > cap) blocks = cap;
  k_validate<<<(unsigned)blocks, 256, 0, ctx->stream>>>(g->n, g->nnz, g->row_ptr, g->col, g->wgt, g->vwgt,
                                                        flags);
  HEC_LAUNCH_CHECK();
  int64_t r[1];
  int rc = read_scalars(ctx, reinterpret_cast<int64_t *>(flags), 1, r);
  dev_free(ctx, flags);
  HEC_TRY(rc);
  int f = (int)(r[0] & 0xffffffff);
  if (f) {
    set_error("input graph violates R1 (flags 0x%x: %s%s%s%s%s%s%s)", f, f & V_ROWPTR ? "row_ptr " : "",
              f & V_RANGE ? "column-range " : "", f & V_ORDER ? "unsorted/duplicate " : "",
              f & V_LOOP ? "self-loop " : "", f & V_WEIGHT ? "weight<=0 " : "",
              f & V_ASYM ? "asymmetric " : "", f & V_VWGT ? "vertex-weight<=0" : "");
    return HEC_EINVAL;
  }
  return HEC_OK;
}

}  // namespace hec
