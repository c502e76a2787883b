// construct_oneend.cu — the construction variants of the C-ABI (SURVEY §8(f)
// f1; Alg 6).  Every variant yields the same canonical
// coarse CSR (rows ascending, weights summed), so they differ only in speed:
//
//   HEC_BUILD_HASH     the default pipeline: per-row hash merge + order-
//                      preserving bucket rank (DEDUPWITHWTS' hashing, L319-324)
//   HEC_BUILD_SORT     the sort-based DEDUPWITHWTS: register bitonic pieces and
//                      shared-memory bucket sort for every row (L319-324)
//   HEC_BUILD_ONE_END  the paper's skewed-degree optimisation: C'[a] = number
//                      of fine entries of coarse row a that are not self loops
//                      (l.1-5); an entry is stored only at its end with the
//                      smaller C' (ties: smaller coarse id, reading Z7; l.9,
//                      l.17), deduplicated there (l.20-21), and
//                      GraphConsWithTrans (l.22) adds every kept (a, b, w) as
//                      (b, a, w): the union of a row's own and transposed
//                      entries is duplicate-free; its unordered rows are put in
//                      order by the default pipeline under the identity map.
//   HEC_BUILD_AUTO     ONE_END when max degree / average degree > 10 (the
//                      skew estimate of L324; threshold: reading Z15), else HASH
#include "construct_common.cuh"

namespace hec {

// C'[M[u]] += #{v in N(u) : M[v] != M[u]}   (Alg 6 l.2-5; a warp per fine vertex)
__global__ void k_cprime(int64_t n, const int64_t *__restrict__ rp, const int32_t *__restrict__ col,
                         const int32_t *__restrict__ M, unsigned long long *__restrict__ Cp) {
  const int lane = threadIdx.x & 31;
  const int64_t w0 = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t u = w0; u < n; u += nw) {
    const int32_t a = M[u];
    unsigned c = 0;
    for (int64_t e = rp[u] + lane; e < rp[u + 1]; e += 32) c += __ldg(M + __ldg(col + e)) != a;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
    if (lane == 0 && c) atomicAdd(Cp + a, (unsigned long long)c);
  }
}

// in-degree of every coarse row in the one-end graph D (its transposed entries)
__global__ void k_oe_indeg(int64_t nnz, const int32_t *__restrict__ col, unsigned *__restrict__ indeg) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < nnz; e += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(indeg + col[e], 1u);
}
struct FDegIn {
  const int64_t *rp;
  const unsigned *indeg;
  __device__ __forceinline__ int64_t operator()(int64_t a) const { return rp[a + 1] - rp[a] + indeg[a]; }
};
struct FPtrOut {
  int64_t *p;
  __device__ __forceinline__ void operator()(int64_t a, int64_t pre) const { p[a] = pre; }
};
// row a of F: D(a) (kept order) then the transposed entries from the rows b with a in D(b)
__global__ void k_oe_fill(int64_t n_c, const int64_t *__restrict__ rp, const int32_t *__restrict__ col,
                          const int32_t *__restrict__ wgt, const int64_t *__restrict__ rpF, unsigned *__restrict__ cursor,
                          int32_t *__restrict__ colF, int32_t *__restrict__ wgtF) {
  const int lane = threadIdx.x & 31;
  const int64_t w0 = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t a = w0; a < n_c; a += nw) {
    const int64_t e0 = rp[a], len = rp[a + 1] - e0, f0 = rpF[a];
    for (int64_t i = lane; i < len; i += 32) {
      const int32_t b = col[e0 + i], w = wgt[e0 + i];
      colF[f0 + i] = b;
      wgtF[f0 + i] = w;
      const int64_t q = rpF[b] + (rp[b + 1] - rp[b]) + atomicAdd(cursor + b, 1u);
      colF[q] = (int32_t)a;
      wgtF[q] = w;
    }
  }
}
__global__ void k_iota(int64_t n, int32_t *__restrict__ M) {
  const int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (u < n) M[u] = (int32_t)u;
}
__global__ void k_max_degree(int64_t n, const int64_t *__restrict__ rp, unsigned long long *__restrict__ mx) {
  const int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (u < n) atomicMax(mx, (unsigned long long)(rp[u + 1] - rp[u]));
}

static int one_end_impl(hec_ctx *ctx, const hec_graph *g, const int32_t *M, int64_t n_c, CoarseOut *out) {
  cudaStream_t s = ctx->stream;
  unsigned long long *Cp = nullptr;
  unsigned *indeg = nullptr;
  int64_t *rpF = nullptr;
  int32_t *colF = nullptr, *wgtF = nullptr, *Mid = nullptr;
  uint64_t *desc = nullptr;
  unsigned *ticket = nullptr;
  CoarseOut D;
  int rc = dev_alloc(ctx, (void **)&Cp, sizeof(unsigned long long) * (n_c + 1));
  if (rc == HEC_OK && cudaMemsetAsync(Cp, 0, sizeof(unsigned long long) * (n_c + 1), s) != cudaSuccess) rc = HEC_ECUDA;
  const int ph = phase_begin(ctx, "one_end", 4.0 * (double)g->nnz);
  if (rc == HEC_OK && g->n > 0) {
    k_cprime<<<ctx->num_sms * 8, 256, 0, s>>>(g->n, g->row_ptr, g->col, M, Cp);
    ctx->launches++;
    if (cudaGetLastError() != cudaSuccess) rc = HEC_ECUDA;
  }
  phase_end(ctx, ph);
  BuildOpts o;
  o.one_end_cp = Cp;
  const size_t ws_used = ctx->ws.used;
  if (rc == HEC_OK) rc = build_coarse_impl(ctx, g, M, n_c, &D, 0, -1, &o);  // D: every coarse edge once
  const int64_t nnzD = D.nnz_c, nnzF = 2 * nnzD;
  const int ph2 = phase_begin(ctx, "transpose", 24.0 * (double)nnzD + 16.0 * (double)n_c);
  if (rc == HEC_OK) rc = dev_alloc(ctx, (void **)&indeg, sizeof(unsigned) * (n_c + 1));
  if (rc == HEC_OK) rc = dev_alloc(ctx, (void **)&rpF, sizeof(int64_t) * (n_c + 1));
  if (rc == HEC_OK) rc = dev_alloc(ctx, (void **)&colF, sizeof(int32_t) * (nnzF > 0 ? nnzF : 1));
  if (rc == HEC_OK) rc = dev_alloc(ctx, (void **)&wgtF, sizeof(int32_t) * (nnzF > 0 ? nnzF : 1));
  if (rc == HEC_OK) rc = dev_alloc(ctx, (void **)&Mid, sizeof(int32_t) * (n_c > 0 ? n_c : 1));
  if (rc == HEC_OK) rc = dev_alloc(ctx, (void **)&desc, sizeof(uint64_t) * scan_tiles(n_c));
  if (rc == HEC_OK) rc = dev_alloc(ctx, (void **)&ticket, sizeof(unsigned));
  if (rc == HEC_OK && cudaMemsetAsync(indeg, 0, sizeof(unsigned) * (n_c + 1), s) != cudaSuccess) rc = HEC_ECUDA;
  if (rc == HEC_OK && nnzD > 0) {
    k_oe_indeg<<<ctx->num_sms * 8, 256, 0, s>>>(nnzD, D.col, indeg);
    ctx->launches++;
  }
  if (rc == HEC_OK) rc = chained_scan(ctx, n_c, FDegIn{D.row_ptr, indeg}, FPtrOut{rpF}, ScanTiles{desc, ticket}, rpF + n_c);
  if (rc == HEC_OK && cudaMemsetAsync(indeg, 0, sizeof(unsigned) * (n_c + 1), s) != cudaSuccess) rc = HEC_ECUDA;
  if (rc == HEC_OK && n_c > 0) {
    k_oe_fill<<<ctx->num_sms * 8, 256, 0, s>>>(n_c, D.row_ptr, D.col, D.wgt, rpF, indeg, colF, wgtF);
    k_iota<<<(unsigned)((n_c + 255) / 256), 256, 0, s>>>(n_c, Mid);
    ctx->launches += 2;
    if (cudaGetLastError() != cudaSuccess) rc = HEC_ECUDA;
  }
  phase_end(ctx, ph2);
  // F's rows in order (identity map: nothing merges, every row is sorted)
  if (rc == HEC_OK) {
    const hec_graph F{n_c, nnzF, rpF, colF, wgtF, D.vwgt};
    ctx->ws.used = ws_used;
    rc = build_coarse_impl(ctx, &F, Mid, n_c, out);
  }
  free_coarse(ctx, D);
  dev_free(ctx, Cp);
  dev_free(ctx, indeg);
  dev_free(ctx, rpF);
  dev_free(ctx, colF);
  dev_free(ctx, wgtF);
  dev_free(ctx, Mid);
  dev_free(ctx, desc);
  dev_free(ctx, ticket);
  return rc;
}

int build_coarse_method_impl(hec_ctx *ctx, const hec_graph *g, const int32_t *M, int64_t n_c, int method,
                             CoarseOut *out) {
  if (method == HEC_BUILD_AUTO) {
    // skew = max degree / average degree (L324)
    unsigned long long *mx = nullptr;
    HEC_TRY(dev_alloc(ctx, (void **)&mx, sizeof(unsigned long long)));
    unsigned long long h = 0;
    int rc = cudaMemsetAsync(mx, 0, sizeof h, ctx->stream) == cudaSuccess ? HEC_OK : HEC_ECUDA;
    if (rc == HEC_OK && g->n > 0) {
      k_max_degree<<<(unsigned)((g->n + 255) / 256), 256, 0, ctx->stream>>>(g->n, g->row_ptr, mx);
      ctx->launches++;
    }
    if (rc == HEC_OK && (cudaMemcpyAsync(&h, mx, sizeof h, cudaMemcpyDeviceToHost, ctx->stream) != cudaSuccess ||
                         cudaStreamSynchronize(ctx->stream) != cudaSuccess))
      rc = HEC_ECUDA;
    dev_free(ctx, mx);
    HEC_TRY(rc);
    const double avg = g->n > 0 ? (double)g->nnz / (double)g->n : 0.0;
    method = avg > 0.0 && (double)h / avg > 10.0 ? HEC_BUILD_ONE_END : HEC_BUILD_HASH;
  }
  switch (method) {
    case HEC_BUILD_HASH:
      return build_coarse_impl(ctx, g, M, n_c, out);
    case HEC_BUILD_SORT: {
      BuildOpts o;
      o.sort_dedup = true;
      return build_coarse_impl(ctx, g, M, n_c, out, 0, -1, &o);
    }
    case HEC_BUILD_ONE_END:
      return one_end_impl(ctx, g, M, n_c, out);
    default:
      set_error("unknown construction method %d", method);
      return HEC_EINVAL;
  }
}

}  // namespace hec
