// spectral.cu — multilevel spectral bisection on the HEC hierarchy (SURVEY
// §8(f) f3; §III-C, stopping rule L367).  The consumer of the
// hierarchy: power iteration for the Fiedler vector of each level's Laplacian,
// coarsest level first, interpolated through the mapping vectors, then a
// balanced split.  fp64 throughout.
//
//   per level:  d[u] = sum_v w(u,v),  sigma = 2 max d (>= lambda_max(L))
//   iterate:    y = (sigma I - L) x = (sigma - d) x + A x     (k_lap_spmv: vector CSR)
//               y <- y - mean(y), y <- y / ||y||, delta = ||y - x||
//               stop when delta < tol (L367: 1e-10) or after max_iter
//   down:       x_fine[u] = x_coarse[M[u]]                    (L330 interpolation)
//   split:      part 0 = the n/2 smallest (x, id): radix select over the
//               order-preserving 64-bit image of x, ids ranked by a scan
//
// Reductions are deterministic: per-block partials in a fixed order, summed
// by every consumer in the same order (no floating-point atomics).  The
// iteration loop runs on the device: each kernel reads a `done` flag set by
// the finalising kernel, so launched iterations after convergence do nothing
// and the host only polls the flag every kPoll iterations.
#include "hec_internal.cuh"

namespace hec {

constexpr int kSpT = 256;       // threads per CTA
constexpr int kSpBlocks = 592;  // reduction CTAs (4 per SM)
constexpr int kPoll = 32;

struct SpState {
  double sigma;
  double mean, norm, delta;
  int64_t it;
  int32_t done, parity;
};

__device__ __forceinline__ double block_sum_d(double v, double *sh) {
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  if (lane == 0) sh[wid] = v;
  __syncthreads();
  double s = 0.0;
  if (threadIdx.x == 0)
    for (int w = 0; w < kSpT / 32; ++w) s += sh[w];
  __syncthreads();
  return s;  // valid in thread 0
}

// the total of the kSpBlocks partials, computed by warp 0 of the CTA (lane-strided, fixed xor
// tree: identical in every CTA) and broadcast through shared memory
__device__ __forceinline__ double block_total(const double *part, double *sh_one) {
  if (threadIdx.x < 32) {
    double s = 0.0;
    for (int b = threadIdx.x; b < kSpBlocks; b += 32) s += part[b];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if (threadIdx.x == 0) *sh_one = s;
  }
  __syncthreads();
  return *sh_one;
}

__global__ void k_sp_degree(int64_t n, const int64_t *__restrict__ rp, const int32_t *__restrict__ wgt,
                            double *__restrict__ d, unsigned long long *__restrict__ dmax) {
  const int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (u >= n) return;
  int64_t s = 0;
  for (int64_t e = rp[u]; e < rp[u + 1]; ++e) s += wgt[e];
  d[u] = (double)s;
  atomicMax(dmax, (unsigned long long)s);
}

__global__ void k_sp_start(int64_t n, uint64_t seed, double *__restrict__ x) {
  const int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (u < n) x[u] = (double)(splitmix64(seed ^ (uint64_t)u) >> 11) * (1.0 / 9007199254740992.0) - 0.5;
}

__global__ void k_sp_interp(int64_t n, const int32_t *__restrict__ M, const double *__restrict__ xc,
                            double *__restrict__ x) {
  const int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (u < n) x[u] = xc[M[u]];
}

// y = (sigma - d) x + A x over buf[parity] -> buf[parity ^ 1]; partial sums of y.
// Vector CSR: a group of G lanes per row (G matched to the average degree, so
// short mesh rows do not leave most of a warp idle), lane-strided entries,
// shuffle reduction inside the group.
template <int G>
__global__ void __launch_bounds__(kSpT) k_lap_spmv(int64_t n, const int64_t *__restrict__ rp,
                                                   const int32_t *__restrict__ col, const int32_t *__restrict__ wgt,
                                                   const double *__restrict__ d, double *buf0, double *buf1,
                                                   const SpState *__restrict__ st, double *__restrict__ part) {
  __shared__ double sh[kSpT / 32];
  if (st->done) return;
  const double *x = st->parity ? buf1 : buf0;
  double *y = st->parity ? buf0 : buf1;
  const double sigma = st->sigma;
  const int gl = threadIdx.x & (G - 1);
  const int64_t g0 = (blockIdx.x * (int64_t)kSpT + threadIdx.x) / G, ng = ((int64_t)gridDim.x * kSpT) / G;
  double acc = 0.0;  // group leaders: this group's rows
  const int64_t rows = (n + ng - 1) / ng * ng;  // every lane runs the same trip count (shuffles)
  for (int64_t u = g0; u < rows; u += ng) {
    double sum = 0.0;
    if (u < n) {
      const int64_t e1 = rp[u + 1];
      for (int64_t e = rp[u] + gl; e < e1; e += G) sum += (double)__ldg(wgt + e) * x[__ldg(col + e)];
    }
#pragma unroll
    for (int o = G / 2; o > 0; o >>= 1) sum += __shfl_xor_sync(0xffffffffu, sum, o);
    if (gl == 0 && u < n) {
      const double v = (sigma - d[u]) * x[u] + sum;
      y[u] = v;
      acc += v;
    }
  }
  const double b = block_sum_d(gl == 0 ? acc : 0.0, sh);
  if (threadIdx.x == 0) part[blockIdx.x] = b;
}

// in = buf[sel]: mode 0: in -= mean(in), partials of in^2
__global__ void __launch_bounds__(kSpT) k_sp_center(int64_t n, double *buf0, double *buf1, SpState *st, int which,
                                                    const double *__restrict__ part_in, double *__restrict__ part) {
  __shared__ double sh[kSpT / 32], tot;
  if (st->done) return;
  double *v = (which ^ st->parity) ? buf1 : buf0;
  const double mean = n > 0 ? block_total(part_in, &tot) / (double)n : 0.0;
  double acc = 0.0;
  for (int64_t u = blockIdx.x * (int64_t)kSpT + threadIdx.x; u < n; u += (int64_t)gridDim.x * kSpT) {
    const double t = v[u] - mean;
    v[u] = t;
    acc += t * t;
  }
  const double b = block_sum_d(acc, sh);
  if (threadIdx.x == 0) part[blockIdx.x] = b;
}

// y /= ||y||; partials of (y - x)^2
__global__ void __launch_bounds__(kSpT) k_sp_normalize(int64_t n, double *buf0, double *buf1, SpState *st, int which,
                                                       const double *__restrict__ part_in, double *__restrict__ part) {
  __shared__ double sh[kSpT / 32], tot;
  if (st->done) return;
  double *y = (which ^ st->parity) ? buf1 : buf0;
  const double *x = (which ^ st->parity) ? buf0 : buf1;
  const double nrm = sqrt(block_total(part_in, &tot));
  const double inv = nrm > 0.0 ? 1.0 / nrm : 1.0;
  double acc = 0.0;
  for (int64_t u = blockIdx.x * (int64_t)kSpT + threadIdx.x; u < n; u += (int64_t)gridDim.x * kSpT) {
    const double t = y[u] * inv;
    y[u] = t;
    const double dd = t - x[u];
    acc += dd * dd;
  }
  const double b = block_sum_d(acc, sh);
  if (threadIdx.x == 0) part[blockIdx.x] = b;
}

__global__ void __launch_bounds__(kSpT) k_sp_sum(int64_t n, const double *__restrict__ x, double *__restrict__ part) {
  __shared__ double sh[kSpT / 32];
  double acc = 0.0;
  for (int64_t u = blockIdx.x * (int64_t)kSpT + threadIdx.x; u < n; u += (int64_t)gridDim.x * kSpT) acc += x[u];
  const double b = block_sum_d(acc, sh);
  if (threadIdx.x == 0) part[blockIdx.x] = b;
}
__global__ void __launch_bounds__(kSpT) k_sp_scale(int64_t n, double *__restrict__ x, const double *__restrict__ part) {
  __shared__ double tot;
  const double nrm = sqrt(block_total(part, &tot));
  const double inv = nrm > 0.0 ? 1.0 / nrm : 1.0;
  for (int64_t u = blockIdx.x * (int64_t)kSpT + threadIdx.x; u < n; u += (int64_t)gridDim.x * kSpT) x[u] *= inv;
}

// one CTA: delta, iteration count, convergence, swap
__global__ void k_sp_finish(SpState *st, const double *__restrict__ part, double tol, int64_t max_iter) {
  __shared__ double tot;
  if (st->done) return;
  const double delta = sqrt(block_total(part, &tot));
  if (threadIdx.x) return;
  st->delta = delta;
  st->it += 1;
  st->parity ^= 1;
  if (delta < tol || st->it >= max_iter) st->done = 1;
}

// ---- balanced split: radix select of the n/2-th smallest (key(x), id)
__device__ __forceinline__ uint64_t order_key(double v) {
  const uint64_t b = (uint64_t)__double_as_longlong(v);
  return (b >> 63) ? ~b : (b | 0x8000000000000000ull);
}
__global__ void k_sp_hist(int64_t n, const double *__restrict__ x, uint64_t prefix, int shift,
                          unsigned long long *__restrict__ hist) {
  __shared__ unsigned h[256];
  for (int i = threadIdx.x; i < 256; i += blockDim.x) h[i] = 0;
  __syncthreads();
  const uint64_t hi_mask = shift >= 56 ? 0ull : (~0ull << (shift + 8));
  for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < n; u += (int64_t)gridDim.x * blockDim.x) {
    const uint64_t k = order_key(x[u]);
    if ((k & hi_mask) == (prefix & hi_mask)) atomicAdd(&h[(k >> shift) & 255], 1u);
  }
  __syncthreads();
  for (int i = threadIdx.x; i < 256; i += blockDim.x)
    if (h[i]) atomicAdd(hist + i, (unsigned long long)h[i]);
}
struct TieIn {
  const double *x;
  uint64_t T;
  __device__ __forceinline__ int64_t operator()(int64_t u) const { return order_key(x[u]) == T; }
};
struct TieOut {
  const double *x;
  uint64_t T;
  int64_t take;  // vertices with key == T that go to part 0 (the smallest ids)
  uint8_t *part;
  __device__ __forceinline__ void operator()(int64_t u, int64_t prefix) const {
    const uint64_t k = order_key(x[u]);
    part[u] = (k < T || (k == T && prefix < take)) ? 0 : 1;
  }
};
__global__ void k_sp_cut(int64_t n, const int64_t *__restrict__ rp, const int32_t *__restrict__ col,
                         const int32_t *__restrict__ wgt, const uint8_t *__restrict__ part,
                         unsigned long long *__restrict__ cut) {
  const int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (u >= n) return;
  unsigned long long s = 0;
  for (int64_t e = rp[u]; e < rp[u + 1]; ++e)
    if (part[col[e]] != part[u]) s += (unsigned long long)wgt[e];
  if (s) atomicAdd(cut, s);
}

}  // namespace hec

using namespace hec;

extern "C" HEC_API int hec_spectral_bisection(hec_ctx *ctx, const hec_graph *g0, const hec_hierarchy *h,
                                              const hec_spectral_opts *opts, uint8_t *part, double *x_out,
                                              int64_t *cut, int64_t *iters) {
  if (!ctx || !g0 || !h || !part || !cut) { set_error("NULL argument"); return HEC_EINVAL; }
  HEC_CUDA_TRY(cudaSetDevice(ctx->device));
  const int64_t max_iter = opts && opts->max_iter > 0 ? opts->max_iter : 1000;
  const double tol = opts && opts->tol >= 0 ? opts->tol : 1e-10;
  const uint64_t seed = opts ? opts->seed : 0x5EED;
  const int L = (int)h->levels.size();
  cudaStream_t s = ctx->stream;
  // graphs[0] = G0, graphs[i] = G_i
  std::vector<hec_graph> graphs(L + 1);
  graphs[0] = *g0;
  int64_t nmax = g0->n;
  for (int i = 1; i <= L; ++i) {
    const CoarseOut &c = h->levels[i - 1].g;
    graphs[i] = hec_graph{c.n_c, c.nnz_c, c.row_ptr, c.col, c.wgt, c.vwgt};
    nmax = c.n_c > nmax ? c.n_c : nmax;
  }
  double *buf[2] = {nullptr, nullptr}, *xc = nullptr, *d = nullptr, *partials = nullptr;
  SpState *st = nullptr;
  unsigned long long *scr = nullptr;  // [0] dmax [1..256] histogram [257] cut
  int rc = HEC_OK;
  auto alloc = [&](void **p, size_t b) { if (rc == HEC_OK) rc = dev_alloc(ctx, p, b); };
  alloc((void **)&buf[0], sizeof(double) * (nmax + 1));
  alloc((void **)&buf[1], sizeof(double) * (nmax + 1));
  alloc((void **)&xc, sizeof(double) * (nmax + 1));
  alloc((void **)&d, sizeof(double) * (nmax + 1));
  alloc((void **)&partials, sizeof(double) * 3 * kSpBlocks);
  alloc((void **)&st, sizeof(SpState));
  alloc((void **)&scr, sizeof(unsigned long long) * 264);
  SpState hs{};
  int64_t total_it = 0;
  const int ph = phase_begin(ctx, "spectral", 0.0);
  for (int lvl = L; lvl >= 0 && rc == HEC_OK; --lvl) {
    const hec_graph &G = graphs[lvl];
    const int64_t n = G.n;
    const unsigned b = (unsigned)((n + 255) / 256);
    if (n == 0) continue;
    // x: the start vector (coarsest) or the interpolation of the coarser level's x
    if (lvl == L) k_sp_start<<<b, 256, 0, s>>>(n, seed, buf[0]);
    else k_sp_interp<<<b, 256, 0, s>>>(n, h->levels[lvl].M, xc, buf[0]);
    ctx->launches++;
    // sigma = 2 max weighted degree (exact: integer weights)
    if (cudaMemsetAsync(scr, 0, sizeof(unsigned long long) * 264, s) != cudaSuccess) { rc = HEC_ECUDA; break; }
    k_sp_degree<<<b, 256, 0, s>>>(n, G.row_ptr, G.wgt, d, scr);
    ctx->launches++;
    unsigned long long dmax = 0;
    if (cudaMemcpyAsync(&dmax, scr, sizeof dmax, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
        cudaStreamSynchronize(s) != cudaSuccess) { rc = HEC_ECUDA; break; }
    hs = SpState{};
    hs.sigma = 2.0 * (double)dmax;
    if (cudaMemcpyAsync(st, &hs, sizeof hs, cudaMemcpyHostToDevice, s) != cudaSuccess) { rc = HEC_ECUDA; break; }
    // initial projection: x -= mean(x), x /= ||x||
    double *p0 = partials, *p1 = partials + kSpBlocks, *p2 = partials + 2 * kSpBlocks;
    k_sp_sum<<<kSpBlocks, kSpT, 0, s>>>(n, buf[0], p1);
    k_sp_center<<<kSpBlocks, kSpT, 0, s>>>(n, buf[0], buf[1], st, 0, p1, p0);
    k_sp_scale<<<kSpBlocks, kSpT, 0, s>>>(n, buf[0], p0);
    ctx->launches += 3;
    if (max_iter > 0) {
      const int64_t cap = max_iter;
      for (int64_t it = 0; it < cap && rc == HEC_OK; ++it) {
        const int64_t avg = G.nnz / n;
        if (avg <= 6) k_lap_spmv<4><<<kSpBlocks, kSpT, 0, s>>>(n, G.row_ptr, G.col, G.wgt, d, buf[0], buf[1], st, p0);
        else if (avg <= 12) k_lap_spmv<8><<<kSpBlocks, kSpT, 0, s>>>(n, G.row_ptr, G.col, G.wgt, d, buf[0], buf[1], st, p0);
        else if (avg <= 24) k_lap_spmv<16><<<kSpBlocks, kSpT, 0, s>>>(n, G.row_ptr, G.col, G.wgt, d, buf[0], buf[1], st, p0);
        else k_lap_spmv<32><<<kSpBlocks, kSpT, 0, s>>>(n, G.row_ptr, G.col, G.wgt, d, buf[0], buf[1], st, p0);
        k_sp_center<<<kSpBlocks, kSpT, 0, s>>>(n, buf[0], buf[1], st, 1, p0, p1);
        k_sp_normalize<<<kSpBlocks, kSpT, 0, s>>>(n, buf[0], buf[1], st, 1, p1, p2);
        k_sp_finish<<<1, 32, 0, s>>>(st, p2, tol, cap);
        ctx->launches += 4;
        if (cudaGetLastError() != cudaSuccess) { rc = HEC_ECUDA; break; }
        if ((it + 1) % kPoll == 0 || it + 1 == cap) {
          if (cudaMemcpyAsync(&hs, st, sizeof hs, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
              cudaStreamSynchronize(s) != cudaSuccess) { rc = HEC_ECUDA; break; }
          if (hs.done) break;
        }
      }
      if (rc != HEC_OK) break;
      if (cudaMemcpyAsync(&hs, st, sizeof hs, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
          cudaStreamSynchronize(s) != cudaSuccess) { rc = HEC_ECUDA; break; }
    } else {
      hs.it = 0;
      hs.parity = 0;
    }
    if (iters) iters[L - lvl] = hs.it;
    total_it += hs.it;
    // the level's x -> xc (interpolated by the next finer level)
    const double *xf = hs.parity ? buf[1] : buf[0];
    if (cudaMemcpyAsync(xc, xf, sizeof(double) * n, cudaMemcpyDeviceToDevice, s) != cudaSuccess) rc = HEC_ECUDA;
  }
  // balanced split of G0 by (x, id)
  if (rc == HEC_OK && g0->n > 0) {
    const int64_t n = g0->n, k = n / 2;
    uint64_t prefix = 0;
    int64_t less = 0;  // vertices with key below the prefix's range
    for (int shift = 56; shift >= 0 && rc == HEC_OK; shift -= 8) {
      unsigned long long hist[256];
      if (cudaMemsetAsync(scr + 1, 0, sizeof(unsigned long long) * 256, s) != cudaSuccess) { rc = HEC_ECUDA; break; }
      k_sp_hist<<<kSpBlocks, 256, 0, s>>>(n, xc, prefix, shift, scr + 1);
      ctx->launches++;
      if (cudaMemcpyAsync(hist, scr + 1, sizeof hist, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
          cudaStreamSynchronize(s) != cudaSuccess) { rc = HEC_ECUDA; break; }
      int dgt = 0;
      while (dgt < 255 && less + (int64_t)hist[dgt] <= k) less += (int64_t)hist[dgt++];
      prefix |= (uint64_t)dgt << shift;
    }
    // prefix = T, the key of the k-th smallest; less = #keys < T
    if (rc == HEC_OK) {
      ScanTiles stt{};
      uint64_t *desc = nullptr;
      unsigned *ticket = nullptr;
      int64_t *tot = nullptr;
      alloc((void **)&desc, sizeof(uint64_t) * scan_tiles(n));
      alloc((void **)&ticket, sizeof(unsigned));
      alloc((void **)&tot, sizeof(int64_t));
      stt.desc = desc;
      stt.ticket = ticket;
      if (rc == HEC_OK) rc = chained_scan(ctx, n, TieIn{xc, prefix}, TieOut{xc, prefix, k - less, part}, stt, tot);
      dev_free(ctx, desc);
      dev_free(ctx, ticket);
      dev_free(ctx, tot);
    }
    if (rc == HEC_OK) {
      k_sp_cut<<<(unsigned)((n + 255) / 256), 256, 0, s>>>(n, g0->row_ptr, g0->col, g0->wgt, part, scr + 257);
      ctx->launches++;
      unsigned long long c2 = 0;
      if (cudaMemcpyAsync(&c2, scr + 257, sizeof c2, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
          cudaStreamSynchronize(s) != cudaSuccess) rc = HEC_ECUDA;
      *cut = (int64_t)(c2 / 2);
    }
    if (rc == HEC_OK && x_out)
      if (cudaMemcpyAsync(x_out, xc, sizeof(double) * n, cudaMemcpyDeviceToDevice, s) != cudaSuccess) rc = HEC_ECUDA;
  }
  phase_end(ctx, ph);
  if (rc == HEC_OK) cudaStreamSynchronize(s);
  dev_free(ctx, buf[0]);
  dev_free(ctx, buf[1]);
  dev_free(ctx, xc);
  dev_free(ctx, d);
  dev_free(ctx, partials);
  dev_free(ctx, st);
  dev_free(ctx, scr);
  if (rc == HEC_ECUDA) set_error("hec_spectral_bisection: CUDA failure");
  (void)total_it;
  return rc;
}
