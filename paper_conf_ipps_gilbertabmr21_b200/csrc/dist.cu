// dist.cu — building blocks of the multi-GPU path: the only
// edge-streaming step of the mapping (heavy neighbours, a1) and the coarse graph
// construction are partitioned across ranks; the caller all-gathers H, M and
// the coarse row counts with NCCL (torch.distributed) between these calls.
//   rank r:  hec_heavy_range(fine slice r)            -> all-gather H
//            hec_mapping_from_heavy(H, fine slice r)   -> all-gather M (+ n_c)
//            hec_balance_rows(M)                       -> identical row ranges
//            hec_build_rows_count(coarse range r)      -> all-gather counts
//            hec_build_rows_write(global offset of r)  -> distributed CSR slice
#include <vector>

#include "hec_internal.cuh"

using namespace hec;

struct DistState {
  CoarseOut slice;
  int64_t a_begin = 0, a_end = 0;
};

static void dist_reset(hec_ctx *ctx) {
  if (!ctx->dist) return;
  dev_free(ctx, ctx->dist->slice.row_ptr);
  dev_free(ctx, ctx->dist->slice.col);
  dev_free(ctx, ctx->dist->slice.wgt);
  dev_free(ctx, ctx->dist->slice.vwgt);
  delete ctx->dist;
  ctx->dist = nullptr;
}

__global__ void k_offset_copy(int64_t n, const int64_t *__restrict__ src, int64_t off, int64_t *__restrict__ dst) {
  int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i < n) dst[i] = src[i] + off;
}

__global__ void k_row_counts(int64_t rows, const int64_t *__restrict__ row_ptr, int64_t *__restrict__ counts) {
  int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i < rows) counts[i] = row_ptr[i + 1] - row_ptr[i];
}

static int dist_begin(hec_ctx *ctx, const hec_graph *g, size_t ws) {
  if (!ctx) { set_error("context is NULL"); return HEC_EINVAL; }
  if (!g || g->n < 0 || g->nnz < 0 || (g->n > 0 && !g->row_ptr)) {
    set_error("invalid graph");
    return HEC_EINVAL;
  }
  HEC_CUDA_TRY(cudaSetDevice(ctx->device));
  HEC_TRY(ws_reserve(ctx, ws));
  ctx->ws.used = 0;
  return HEC_OK;
}

extern "C" {

HEC_API int hec_heavy_range(hec_ctx *ctx, const hec_graph *g, int64_t u_begin, int64_t u_end, int32_t *H) {
  size_t ws = 0;
  ws_bytes_mapping(g ? g->n : 0, g ? g->nnz : 0, &ws);
  HEC_TRY(dist_begin(ctx, g, ws));
  if (u_begin < 0 || u_begin > u_end || u_end > g->n || (u_end > u_begin && !H)) {
    set_error("hec_heavy_range: bad range [%lld, %lld) for n=%lld", (long long)u_begin, (long long)u_end,
              (long long)g->n);
    return HEC_EINVAL;
  }
  HEC_TRY(heavy_range_impl(ctx, g, u_begin, u_end, H));
  HEC_CUDA_TRY(cudaStreamSynchronize(ctx->stream));
  return HEC_OK;
}

HEC_API int hec_mapping_from_heavy(hec_ctx *ctx, const hec_graph *g, const int32_t *H, uint64_t seed, int level,
                                   int64_t u_begin, int64_t u_end, int32_t *M, int64_t *n_c) {
  size_t ws = 0;
  ws_bytes_mapping(g ? g->n : 0, g ? g->nnz : 0, &ws);
  HEC_TRY(dist_begin(ctx, g, ws));
  if (!n_c || (g->n > 0 && (!H || !M)) || u_begin < 0 || u_begin > u_end || u_end > g->n) {
    set_error("hec_mapping_from_heavy: bad arguments");
    return HEC_EINVAL;
  }
  MapResult r;
  HEC_TRY(mapping_from_heavy_impl(ctx, g, H, Prio{nullptr, splitmix64(seed + (uint64_t)level)}, u_begin, u_end,
                                  M, &r));
  *n_c = r.n_c;
  ctx->stats.rounds = r.rounds;
  ctx->stats.n_c = r.n_c;
  return HEC_OK;
}

HEC_API int hec_balance_rows(hec_ctx *ctx, const hec_graph *g, const int32_t *M, int64_t n_c, int parts,
                             int64_t *bounds) {
  HEC_TRY(dist_begin(ctx, g, 0));
  if (parts < 1 || !bounds || n_c < 0 || (g->n > 0 && !M)) {
    set_error("hec_balance_rows: bad arguments");
    return HEC_EINVAL;
  }
  std::vector<int64_t> U((size_t)n_c);
  if (n_c > 0) {
    int64_t *dU = nullptr;
    HEC_TRY(dev_alloc(ctx, (void **)&dU, sizeof(int64_t) * n_c));
    int rc = row_volume_impl(ctx, g, M, n_c, dU);
    if (rc == HEC_OK) {
      cudaError_t e = cudaMemcpyAsync(U.data(), dU, sizeof(int64_t) * n_c, cudaMemcpyDeviceToHost, ctx->stream);
      if (e == cudaSuccess) e = cudaStreamSynchronize(ctx->stream);
      if (e != cudaSuccess) { set_error("hec_balance_rows: %s", cudaGetErrorString(e)); rc = HEC_ECUDA; }
    }
    dev_free(ctx, dU);
    HEC_TRY(rc);
  }
  // bounds[k] = first row whose member-edge prefix reaches k/parts of the total
  int64_t total = 0;
  for (int64_t a = 0; a < n_c; ++a) total += U[a];
  bounds[0] = 0;
  int64_t run = 0, a = 0;
  for (int k = 1; k < parts; ++k) {
    const long double target = (long double)total * k / parts;
    while (a < n_c && (long double)(run + U[a]) <= target) run += U[a++];
    bounds[k] = a > bounds[k - 1] ? a : bounds[k - 1];
  }
  bounds[parts] = n_c;
  return HEC_OK;
}

HEC_API int hec_build_rows_count(hec_ctx *ctx, const hec_graph *g, const int32_t *M, int64_t n_c, int64_t a_begin,
                                 int64_t a_end, int64_t *counts, int64_t *nnz_slice) {
  HEC_TRY(dist_begin(ctx, g, ws_bytes_construct(g ? g->n : 0, g ? g->nnz : 0, n_c)));
  if (!nnz_slice || a_begin < 0 || a_begin > a_end || a_end > n_c) {
    set_error("hec_build_rows_count: bad range [%lld, %lld) for n_c=%lld", (long long)a_begin, (long long)a_end,
              (long long)n_c);
    return HEC_EINVAL;
  }
  dist_reset(ctx);
  DistState *d = new DistState();
  d->a_begin = a_begin;
  d->a_end = a_end;
  int rc = build_coarse_impl(ctx, g, M, n_c, &d->slice, a_begin, a_end);
  ctx->dist = d;
  if (rc != HEC_OK) {
    dist_reset(ctx);
    return rc;
  }
  if (counts && a_end > a_begin) {  // counts[i] = |row a_begin + i|
    k_row_counts<<<(unsigned)((a_end - a_begin + 255) / 256), 256, 0, ctx->stream>>>(a_end - a_begin,
                                                                                   d->slice.row_ptr, counts);
    HEC_LAUNCH_CHECK();
  }
  HEC_CUDA_TRY(cudaStreamSynchronize(ctx->stream));
  *nnz_slice = d->slice.nnz_c;
  return HEC_OK;
}

HEC_API int hec_build_rows_write(hec_ctx *ctx, int64_t offset, int64_t *row_ptr_c, int32_t *col_c, int32_t *wgt_c,
                                 int32_t *vwgt_c) {
  if (!ctx || !ctx->dist) {
    set_error("hec_build_rows_write: no pending hec_build_rows_count on this context");
    return HEC_EINVAL;
  }
  DistState *d = ctx->dist;
  const int64_t rows = d->a_end - d->a_begin, nnz = d->slice.nnz_c;
  if ((!row_ptr_c) || (nnz > 0 && (!col_c || !wgt_c)) || (rows > 0 && !vwgt_c)) {
    set_error("hec_build_rows_write: NULL output");
    return HEC_EINVAL;
  }
  k_offset_copy<<<(unsigned)((rows + 1 + 255) / 256), 256, 0, ctx->stream>>>(rows + 1, d->slice.row_ptr, offset,
                                                                           row_ptr_c);
  HEC_LAUNCH_CHECK();
  if (nnz > 0) {
    HEC_CUDA_TRY(cudaMemcpyAsync(col_c, d->slice.col, sizeof(int32_t) * nnz, cudaMemcpyDeviceToDevice, ctx->stream));
    HEC_CUDA_TRY(cudaMemcpyAsync(wgt_c, d->slice.wgt, sizeof(int32_t) * nnz, cudaMemcpyDeviceToDevice, ctx->stream));
  }
  if (rows > 0)
    HEC_CUDA_TRY(cudaMemcpyAsync(vwgt_c, d->slice.vwgt, sizeof(int32_t) * rows, cudaMemcpyDeviceToDevice,
                                 ctx->stream));
  HEC_CUDA_TRY(cudaStreamSynchronize(ctx->stream));
  dist_reset(ctx);
  return HEC_OK;
}

}  // extern "C"
