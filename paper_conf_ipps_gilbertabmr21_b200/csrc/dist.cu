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

namespace hec {

int balance_rows_impl(hec_ctx *ctx, const hec_graph *g, const int32_t *M, int64_t n_c, int parts, int64_t *bounds) {
  std::vector<int64_t> U((size_t)n_c);
  if (n_c > 0) {
    int64_t *dU = nullptr;
    HEC_TRY(dev_alloc(ctx, (void **)&dU, sizeof(int64_t) * n_c));
    int rc = row_volume_impl(ctx, g, M, n_c, dU);
    if (rc == HEC_OK) {
      cudaError_t e = cudaMemcpyAsync(U.data(), dU, sizeof(int64_t) * n_c, cudaMemcpyDeviceToHost, ctx->stream);
      if (e == cudaSuccess) e = cudaStreamSynchronize(ctx->stream);
      if (e != cudaSuccess) { set_error("balance rows: %s", cudaGetErrorString(e)); rc = HEC_ECUDA; }
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

// [lo, hi) of rank r among world nearly equal contiguous pieces of [0, n)
static void even_range(int64_t n, int world, int r, int64_t *lo, int64_t *hi) {
  const int64_t q = n / world, rem = n % world;
  *lo = (int64_t)r * q + (r < rem ? r : rem);
  *hi = *lo + q + (r < rem ? 1 : 0);
}

// All-gather of uneven pieces: rank r contributes cnt[r] elements of esz
// bytes (its own at src); dst receives them concatenated in rank order.  The
// caller's collective moves equal blocks, so pieces are padded to the largest.
static int allgather_v(hec_ctx *ctx, const hec_comm *comm, const void *src, const std::vector<int64_t> &cnt,
                       size_t esz, void *dst) {
  const int world = comm->world;
  int64_t maxc = 0;
  for (int64_t c : cnt) maxc = c > maxc ? c : maxc;
  if (maxc == 0) return HEC_OK;
  const size_t block = (size_t)maxc * esz;
  const int ph = phase_begin(ctx, "gather", (double)block * world);
  char *sendbuf = nullptr, *recvbuf = nullptr;
  HEC_TRY(dev_alloc(ctx, (void **)&sendbuf, block));
  int rc = dev_alloc(ctx, (void **)&recvbuf, block * world);
  if (rc == HEC_OK && cnt[comm->rank] > 0 &&
      cudaMemcpyAsync(sendbuf, src, (size_t)cnt[comm->rank] * esz, cudaMemcpyDeviceToDevice, ctx->stream) !=
          cudaSuccess)
    rc = HEC_ECUDA;
  if (rc == HEC_OK && comm->allgather(sendbuf, recvbuf, block, (hec_stream_t)ctx->stream, comm->user) != 0) {
    set_error("all-gather callback failed");
    rc = HEC_ECUDA;
  }
  int64_t off = 0;
  for (int r = 0; r < world && rc == HEC_OK; ++r) {
    if (cnt[r] > 0 && cudaMemcpyAsync((char *)dst + (size_t)off * esz, recvbuf + (size_t)r * block,
                                      (size_t)cnt[r] * esz, cudaMemcpyDeviceToDevice, ctx->stream) != cudaSuccess)
      rc = HEC_ECUDA;
    off += cnt[r];
  }
  phase_end(ctx, ph);
  dev_free(ctx, sendbuf);
  dev_free(ctx, recvbuf);
  if (rc == HEC_ECUDA) cudaGetLastError();
  return rc;
}

int find_mapping_dist_impl(hec_ctx *ctx, const hec_graph *g, Prio prio, const hec_comm *comm, int32_t *M,
                           MapResult *res) {
  const int64_t n = g->n;
  res->n_c = 0;
  res->rounds = 0;
  if (n == 0) return HEC_OK;
  std::vector<int64_t> cnt(comm->world);
  int64_t u0 = 0, u1 = 0;
  for (int r = 0; r < comm->world; ++r) {
    int64_t lo, hi;
    even_range(n, comm->world, r, &lo, &hi);
    cnt[r] = hi - lo;
    if (r == comm->rank) { u0 = lo; u1 = hi; }
  }
  int32_t *H = ws_take<int32_t>(ctx, n);
  if (!H) { set_error("workspace under-reserved (dist mapping)"); return HEC_EINVAL; }
  HEC_TRY(heavy_range_impl(ctx, g, u0, u1, H));  // a1 on the rank's fine slice
  HEC_TRY(allgather_v(ctx, comm, H + u0, cnt, sizeof(int32_t), H));
  HEC_TRY(mapping_from_heavy_impl(ctx, g, H, prio, u0, u1, M, res));  // a3-a5 replicated, M of the slice
  return allgather_v(ctx, comm, M + u0, cnt, sizeof(int32_t), M);
}

struct RankOffsets {
  int64_t bound[kMaxWorld + 1];  // row ranges
  int64_t eoff[kMaxWorld + 1];   // entry offsets (eoff[world] = nnz_total)
  int world;
};

// row_ptr[a] (slice-local offsets, concatenated) += entry offset of a's rank; row_ptr[n_c] = total
__global__ void k_stitch_rows(int64_t n_c, RankOffsets ro, int64_t *__restrict__ row_ptr) {
  const int64_t a = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (a > n_c) return;
  if (a == n_c) { row_ptr[a] = ro.eoff[ro.world]; return; }
  int r = 0;
  while (r + 1 < ro.world && ro.bound[r + 1] <= a) ++r;
  row_ptr[a] += ro.eoff[r];
}

int build_coarse_dist_impl(hec_ctx *ctx, const hec_graph *g, const int32_t *M, int64_t n_c, const hec_comm *comm,
                           int gather_full, CoarseOut *out, DistSlice *slice) {
  const int world = comm->world, rank = comm->rank;
  if (world > kMaxWorld) { set_error("at most %d ranks", kMaxWorld); return HEC_EINVAL; }
  std::vector<int64_t> bounds(world + 1);
  HEC_TRY(balance_rows_impl(ctx, g, M, n_c, world, bounds.data()));
  const int64_t a0 = bounds[rank], a1 = bounds[rank + 1];
  CoarseOut sl;
  int rc = build_coarse_impl(ctx, g, M, n_c, &sl, a0, a1);
  if (rc != HEC_OK) { free_coarse(ctx, sl); return rc; }
  // entry counts of all slices -> global offsets (on every rank)
  std::vector<int64_t> nnz(world, 0), ones(world, 1);
  int64_t *dn = nullptr;
  rc = dev_alloc(ctx, (void **)&dn, sizeof(int64_t) * (world + 1));
  if (rc == HEC_OK && cudaMemcpyAsync(dn + world, &sl.nnz_c, sizeof(int64_t), cudaMemcpyHostToDevice, ctx->stream) !=
                          cudaSuccess)
    rc = HEC_ECUDA;
  if (rc == HEC_OK) rc = allgather_v(ctx, comm, dn + world, ones, sizeof(int64_t), dn);
  if (rc == HEC_OK && (cudaMemcpyAsync(nnz.data(), dn, sizeof(int64_t) * world, cudaMemcpyDeviceToHost, ctx->stream) !=
                           cudaSuccess ||
                       cudaStreamSynchronize(ctx->stream) != cudaSuccess))
    rc = HEC_ECUDA;
  dev_free(ctx, dn);
  if (rc != HEC_OK) { free_coarse(ctx, sl); return rc; }
  RankOffsets ro{};
  ro.world = world;
  for (int r = 0; r <= world; ++r) ro.bound[r] = bounds[r];
  for (int r = 0; r < world; ++r) ro.eoff[r + 1] = ro.eoff[r] + nnz[r];
  *slice = DistSlice{a0, a1, ro.eoff[rank], ro.eoff[world]};
  if (!gather_full) {
    *out = sl;
    return HEC_OK;
  }
  // every rank receives the whole G_c: slices all-gathered, row offsets stitched
  std::vector<int64_t> rows(world);
  for (int r = 0; r < world; ++r) rows[r] = bounds[r + 1] - bounds[r];
  const int64_t total = ro.eoff[world];
  out->n_c = n_c;
  out->nnz_c = total;
  rc = dev_alloc(ctx, (void **)&out->row_ptr, sizeof(int64_t) * (n_c + 1));
  if (rc == HEC_OK) rc = dev_alloc(ctx, (void **)&out->col, sizeof(int32_t) * (total > 0 ? total : 1));
  if (rc == HEC_OK) rc = dev_alloc(ctx, (void **)&out->wgt, sizeof(int32_t) * (total > 0 ? total : 1));
  if (rc == HEC_OK) rc = dev_alloc(ctx, (void **)&out->vwgt, sizeof(int32_t) * (n_c > 0 ? n_c : 1));
  if (rc == HEC_OK) rc = allgather_v(ctx, comm, sl.row_ptr, rows, sizeof(int64_t), out->row_ptr);
  if (rc == HEC_OK) rc = allgather_v(ctx, comm, sl.col, nnz, sizeof(int32_t), out->col);
  if (rc == HEC_OK) rc = allgather_v(ctx, comm, sl.wgt, nnz, sizeof(int32_t), out->wgt);
  if (rc == HEC_OK) rc = allgather_v(ctx, comm, sl.vwgt, rows, sizeof(int32_t), out->vwgt);
  if (rc == HEC_OK) {
    k_stitch_rows<<<(unsigned)((n_c + 1 + 255) / 256), 256, 0, ctx->stream>>>(n_c, ro, out->row_ptr);
    ctx->launches++;
    if (cudaGetLastError() != cudaSuccess) rc = HEC_ECUDA;
  }
  free_coarse(ctx, sl);
  if (rc == HEC_OK) *slice = DistSlice{0, n_c, 0, total};
  return rc;
}

}  // namespace hec

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
  return balance_rows_impl(ctx, g, M, n_c, parts, bounds);
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
