// api.cu — the C-ABI of libhec (include/hec.h): context, allocation, errors,
// the three north-star entry points and the Alg 1 hierarchy driver.
#include <stdarg.h>
#include <string.h>

#include <new>
#include <vector>

#include "hec_internal.cuh"

namespace hec {

static thread_local char g_err[512] = "";

void set_error(const char *fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(g_err, sizeof g_err, fmt, ap);
  va_end(ap);
}

int dev_alloc(hec_ctx *ctx, void **p, size_t bytes) {
  if (bytes == 0) bytes = 16;
  *p = nullptr;
  if (ctx->alloc) {
    *p = ctx->alloc(bytes, (hec_stream_t)ctx->stream, ctx->user);
    if (!*p) {
      set_error("allocator callback failed for %zu bytes", bytes);
      return HEC_ENOMEM;
    }
    return HEC_OK;
  }
  cudaError_t e = cudaMallocFromPoolAsync(p, bytes, ctx->pool, ctx->stream);
  if (e != cudaSuccess) {
    cudaGetLastError();
    set_error("cudaMallocFromPoolAsync(%zu): %s", bytes, cudaGetErrorString(e));
    *p = nullptr;
    return e == cudaErrorMemoryAllocation ? HEC_ENOMEM : HEC_ECUDA;
  }
  return HEC_OK;
}

void dev_free(hec_ctx *ctx, void *p) {
  if (!p) return;
  if (ctx->free) ctx->free(p, (hec_stream_t)ctx->stream, ctx->user);
  else cudaFreeAsync(p, ctx->stream);
}

int out_alloc(hec_ctx *ctx, void **p, size_t bytes) {
  Slab *sl = ctx->slab;
  if (!sl || bytes >= kSlabDirect) return dev_alloc(ctx, p, bytes);
  bytes = (bytes + 255) & ~(size_t)255;
  if (sl->chunks.empty() || sl->chunks.back().used + bytes > sl->chunks.back().cap) {
    void *c = nullptr;
    HEC_TRY(dev_alloc(ctx, &c, kSlabChunk));
    sl->chunks.push_back({(char *)c, kSlabChunk, 0});
  }
  auto &c = sl->chunks.back();
  *p = c.base + c.used;
  c.used += bytes;
  return HEC_OK;
}

void out_free(hec_ctx *ctx, void *p) {
  if (!p || (ctx->slab && ctx->slab->owns(p))) return;
  dev_free(ctx, p);
}

int arena_reserve(hec_ctx *ctx, Arena *a, size_t bytes) {
  if (bytes <= a->cap) return HEC_OK;
  size_t want = bytes + bytes / 8;  // headroom for the next level / call
  if (a->base) {
    dev_free(ctx, a->base);
    a->base = nullptr;
    a->cap = 0;
  }
  void *p = nullptr;
  HEC_TRY(dev_alloc(ctx, &p, want));
  a->base = (char *)p;
  a->cap = want;
  a->used = 0;
  return HEC_OK;
}

// blockIdx.y = region; 4-byte words (all regions are 4-byte multiples except
// byte flag arrays, whose tail bytes are cleared one by one)
__global__ void k_zero_regions(ZeroList z) {
  const int r = blockIdx.y;
  char *p = reinterpret_cast<char *>(z.p[r]);
  const int64_t b = z.bytes[r];
  const int64_t words = ((uintptr_t)p & 3) == 0 ? b >> 2 : 0;
  uint32_t *w = reinterpret_cast<uint32_t *>(p);
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < words; i += (int64_t)gridDim.x * blockDim.x)
    w[i] = 0u;
  for (int64_t i = 4 * words + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < b;
       i += (int64_t)gridDim.x * blockDim.x)
    p[i] = 0;
}

int zero_regions(hec_ctx *ctx, const ZeroList &z) {
  if (z.n == 0) return HEC_OK;
  int64_t mx = 0;
  for (int i = 0; i < z.n; ++i) mx = z.bytes[i] > mx ? z.bytes[i] : mx;
  int64_t gx = (mx / 4 + 255) / 256;
  if (gx > 4 * (int64_t)ctx->num_sms) gx = 4 * (int64_t)ctx->num_sms;
  if (gx < 1) gx = 1;
  k_zero_regions<<<dim3((unsigned)gx, (unsigned)z.n), 256, 0, ctx->stream>>>(z);
  HEC_LAUNCH_CHECK();
  return HEC_OK;
}

int read_scalars(hec_ctx *ctx, const int64_t *dev, int count, int64_t *host_out) {
  HEC_CUDA_TRY(cudaMemcpyAsync(ctx->h_pinned, dev, sizeof(int64_t) * count, cudaMemcpyDeviceToHost,
                               ctx->stream));
  HEC_CUDA_TRY(cudaStreamSynchronize(ctx->stream));
  memcpy(host_out, ctx->h_pinned, sizeof(int64_t) * count);
  return HEC_OK;
}

static cudaEvent_t take_event(hec_ctx *ctx) {
  if (!ctx->prof_pool.empty()) {
    cudaEvent_t e = ctx->prof_pool.back();
    ctx->prof_pool.pop_back();
    return e;
  }
  cudaEvent_t e = nullptr;
  cudaEventCreate(&e);
  return e;
}

int phase_begin(hec_ctx *ctx, const char *name, double bytes) {
  if (!ctx->prof_on) return -1;
  hec_ctx::PhaseRec r{name, take_event(ctx), take_event(ctx), bytes, ctx->prof_level};
  cudaEventRecord(r.a, ctx->stream);
  ctx->prof_pending.push_back(r);
  return (int)ctx->prof_pending.size() - 1;
}

void phase_end(hec_ctx *ctx, int handle) {
  if (handle < 0 || handle >= (int)ctx->prof_pending.size()) return;
  cudaEventRecord(ctx->prof_pending[handle].b, ctx->stream);
}

void phase_set_bytes(hec_ctx *ctx, int handle, double bytes) {
  if (handle < 0 || handle >= (int)ctx->prof_pending.size()) return;
  ctx->prof_pending[handle].bytes = bytes;
}

static void resolve_profile(hec_ctx *ctx) {
  for (auto &r : ctx->prof_pending) {
    float ms = 0;
    cudaEventSynchronize(r.b);
    cudaEventElapsedTime(&ms, r.a, r.b);
    hec_ctx::PhaseAcc *acc = nullptr;
    for (auto &x : ctx->prof_acc)
      if (x.name == r.name && x.level == r.level) acc = &x;
    if (!acc) {
      ctx->prof_acc.push_back(hec_ctx::PhaseAcc{});
      acc = &ctx->prof_acc.back();
      acc->name = r.name;
      acc->level = r.level;
    }
    acc->ms += ms;
    acc->bytes += r.bytes;
    acc->calls += 1;
    ctx->prof_pool.push_back(r.a);
    ctx->prof_pool.push_back(r.b);
  }
  ctx->prof_pending.clear();
}

static int check_graph(const hec_graph *g) {
  if (!g) { set_error("graph is NULL"); return HEC_EINVAL; }
  if (g->n < 0 || g->n >= (int64_t)INT32_MAX || g->nnz < 0) {
    set_error("graph sizes out of range (n=%lld, nnz=%lld)", (long long)g->n, (long long)g->nnz);
    return HEC_EINVAL;
  }
  if (g->n > 0 && !g->row_ptr) { set_error("row_ptr is NULL"); return HEC_EINVAL; }
  if (g->nnz > 0 && (!g->col || !g->wgt)) { set_error("col/wgt is NULL"); return HEC_EINVAL; }
  return HEC_OK;
}

static int begin_call(hec_ctx *ctx, size_t ws) {
  if (!ctx) { set_error("context is NULL"); return HEC_EINVAL; }
  HEC_CUDA_TRY(cudaSetDevice(ctx->device));
  HEC_TRY(ws_reserve(ctx, ws));
  ctx->ws.used = 0;
  return HEC_OK;
}

}  // namespace hec

using namespace hec;

namespace hec {
void free_coarse(hec_ctx *ctx, CoarseOut &c) {
  out_free(ctx, c.row_ptr);
  out_free(ctx, c.col);
  out_free(ctx, c.wgt);
  out_free(ctx, c.vwgt);
  c = CoarseOut{};
}
}  // namespace hec

extern "C" {

HEC_API const char *hec_last_error(void) { return g_err; }

HEC_API int hec_ctx_create(hec_stream_t stream, hec_alloc_fn alloc, hec_free_fn free, void *user,
                           hec_ctx **out) {
  if (!out) { set_error("out is NULL"); return HEC_EINVAL; }
  *out = nullptr;
  if ((alloc == nullptr) != (free == nullptr)) {
    set_error("alloc and free callbacks must be given together");
    return HEC_EINVAL;
  }
  hec_ctx *c = new (std::nothrow) hec_ctx();
  if (!c) { set_error("out of host memory"); return HEC_ENOMEM; }
  c->stream = (cudaStream_t)stream;
  c->alloc = alloc;
  c->free = free;
  c->user = user;
  cudaError_t e = cudaGetDevice(&c->device);
  if (e == cudaSuccess) e = cudaDeviceGetAttribute(&c->num_sms, cudaDevAttrMultiProcessorCount, c->device);
  int smem = 0;
  if (e == cudaSuccess) e = cudaDeviceGetAttribute(&smem, cudaDevAttrMaxSharedMemoryPerBlockOptin, c->device);
  c->smem_optin = (size_t)smem;
  int major = 0, minor = 0;
  if (e == cudaSuccess) e = cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, c->device);
  if (e == cudaSuccess) e = cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, c->device);
  if (e == cudaSuccess) e = cudaMallocHost((void **)&c->h_pinned, 64 * sizeof(int64_t));
  if (e == cudaSuccess && !alloc) {
    // no allocator callback: an own stream-ordered pool that keeps its memory
    // (the device default pool returns freed memory at every synchronisation,
    // so each call would pay for fresh allocations)
    cudaMemPoolProps props{};
    props.allocType = cudaMemAllocationTypePinned;
    props.location.type = cudaMemLocationTypeDevice;
    props.location.id = c->device;
    e = cudaMemPoolCreate(&c->pool, &props);
    uint64_t keep = UINT64_MAX;
    if (e == cudaSuccess) e = cudaMemPoolSetAttribute(c->pool, cudaMemPoolAttrReleaseThreshold, &keep);
  }
  if (e != cudaSuccess) {
    set_error("CUDA init failed: %s", cudaGetErrorString(e));
    cudaGetLastError();
    if (c->pool) cudaMemPoolDestroy(c->pool);
    if (c->h_pinned) cudaFreeHost(c->h_pinned);
    delete c;
    return HEC_ECUDA;
  }
  if (major != 10 || minor != 0) {
    set_error("libhec is built for sm_100a (B200); device is sm_%d%d", major, minor);
    cudaFreeHost(c->h_pinned);
    if (c->pool) cudaMemPoolDestroy(c->pool);
    delete c;
    return HEC_ECUDA;
  }
  *out = c;
  return HEC_OK;
}

HEC_API void hec_ctx_destroy(hec_ctx *ctx) {
  if (!ctx) return;
  cudaStreamSynchronize(ctx->stream);
  dev_free(ctx, ctx->ws.base);
  dev_free(ctx, ctx->ws2.base);
  cudaStreamSynchronize(ctx->stream);
  if (ctx->h_pinned) cudaFreeHost(ctx->h_pinned);
  // memory still held by live results is released once they are freed
  if (ctx->pool) cudaMemPoolDestroy(ctx->pool);
  resolve_profile(ctx);
  for (auto e : ctx->prof_pool) cudaEventDestroy(e);
  delete ctx;
}

HEC_API int hec_ctx_set_validate(hec_ctx *ctx, int validate) {
  if (!ctx) { set_error("context is NULL"); return HEC_EINVAL; }
  ctx->validate = validate ? 1 : 0;
  return HEC_OK;
}

HEC_API int hec_ctx_set_stream(hec_ctx *ctx, hec_stream_t stream) {
  if (!ctx) { set_error("context is NULL"); return HEC_EINVAL; }
  ctx->stream = (cudaStream_t)stream;
  return HEC_OK;
}

HEC_API int hec_ctx_set_profiling(hec_ctx *ctx, int on) {
  if (!ctx) { set_error("context is NULL"); return HEC_EINVAL; }
  ctx->prof_on = on ? 1 : 0;
  return HEC_OK;
}

HEC_API int hec_ctx_profile_reset(hec_ctx *ctx) {
  if (!ctx) { set_error("context is NULL"); return HEC_EINVAL; }
  HEC_CUDA_TRY(cudaStreamSynchronize(ctx->stream));
  resolve_profile(ctx);
  ctx->prof_acc.clear();
  ctx->launches = 0;
  return HEC_OK;
}

HEC_API int hec_ctx_profile(hec_ctx *ctx, hec_phase_time *out, int max, int *count) {
  if (!ctx || !count) { set_error("NULL argument"); return HEC_EINVAL; }
  HEC_CUDA_TRY(cudaStreamSynchronize(ctx->stream));
  resolve_profile(ctx);
  int k = 0;
  for (auto &x : ctx->prof_acc) {
    if (out && k < max) {
      memset(out[k].name, 0, sizeof out[k].name);
      strncpy(out[k].name, x.name.c_str(), sizeof out[k].name - 1);
      out[k].ms = x.ms;
      out[k].calls = x.calls;
      out[k].bytes = x.bytes;
      out[k].level = x.level;
    }
    ++k;
  }
  *count = k;
  return HEC_OK;
}

HEC_API int64_t hec_ctx_launches(const hec_ctx *ctx) { return ctx ? ctx->launches : 0; }

HEC_API int hec_ctx_last_stats(const hec_ctx *ctx, hec_stats *out) {
  if (!ctx || !out) { set_error("NULL argument"); return HEC_EINVAL; }
  *out = ctx->stats;
  return HEC_OK;
}

HEC_API uint64_t hec_prio(uint64_t seed, int level, int64_t u) {
  return prio_of(splitmix64(seed + (uint64_t)level), (uint32_t)u);
}

static int mapping_common(hec_ctx *ctx, const hec_graph *g, Prio prio, int32_t *M, int64_t *n_c,
                          uint8_t *root, int32_t *H) {
  HEC_TRY(check_graph(g));
  if ((g->n > 0 && !M) || !n_c) { set_error("M / n_c is NULL"); return HEC_EINVAL; }
  size_t ws = 0;
  ws_bytes_mapping(g->n, g->nnz, &ws);
  HEC_TRY(begin_call(ctx, ws));
  if (ctx->validate) HEC_TRY(validate_graph(ctx, g));
  MapResult r;
  HEC_TRY(find_mapping_impl(ctx, g, prio, M, root, H, &r));
  *n_c = r.n_c;
  ctx->stats.rounds = r.rounds;
  ctx->stats.n_c = r.n_c;
  return HEC_OK;
}

HEC_API int hec_find_mapping(hec_ctx *ctx, const hec_graph *g, uint64_t seed, int level, int32_t *M,
                             int64_t *n_c) {
  Prio p{nullptr, splitmix64(seed + (uint64_t)level)};
  return mapping_common(ctx, g, p, M, n_c, nullptr, nullptr);
}

HEC_API int hec_find_mapping_prio(hec_ctx *ctx, const hec_graph *g, const uint64_t *prio, int32_t *M,
                                  int64_t *n_c) {
  if (!prio && g && g->n > 0) { set_error("prio is NULL"); return HEC_EINVAL; }
  Prio p{prio, 0};
  return mapping_common(ctx, g, p, M, n_c, nullptr, nullptr);
}

HEC_API int hec_debug_heavy(hec_ctx *ctx, const hec_graph *g, int32_t *H) {
  HEC_TRY(check_graph(g));
  if (g->n > 0 && !H) { set_error("H is NULL"); return HEC_EINVAL; }
  size_t ws = 0;
  ws_bytes_mapping(g->n, g->nnz, &ws);
  HEC_TRY(begin_call(ctx, ws));
  HEC_TRY(heavy_only_impl(ctx, g, H));
  HEC_CUDA_TRY(cudaStreamSynchronize(ctx->stream));
  return HEC_OK;
}

HEC_API int hec_debug_roots(hec_ctx *ctx, const hec_graph *g, const uint64_t *prio, uint64_t seed, int level,
                            uint8_t *root, int *rounds) {
  HEC_TRY(check_graph(g));
  if (g->n > 0 && !root) { set_error("root is NULL"); return HEC_EINVAL; }
  int32_t *M = nullptr;
  if (g->n > 0) HEC_TRY(dev_alloc(ctx, (void **)&M, sizeof(int32_t) * g->n));
  Prio p{prio, prio ? 0 : splitmix64(seed + (uint64_t)level)};
  int64_t nc = 0;
  int rc = mapping_common(ctx, g, p, M, &nc, root, nullptr);
  dev_free(ctx, M);
  if (rc == HEC_OK && rounds) *rounds = ctx->stats.rounds;
  return rc;
}

HEC_API int build_coarse_graph(hec_ctx *ctx, const hec_graph *g, const int32_t *M, int64_t n_c,
                               hec_csr_owned **out) {
  return build_coarse_graph_ex(ctx, g, M, n_c, HEC_BUILD_HASH, out);
}

HEC_API int build_coarse_graph_ex(hec_ctx *ctx, const hec_graph *g, const int32_t *M, int64_t n_c, int method,
                                  hec_csr_owned **out) {
  if (!out) { set_error("out is NULL"); return HEC_EINVAL; }
  *out = nullptr;
  HEC_TRY(check_graph(g));
  if (g->n > 0 && !M) { set_error("M is NULL"); return HEC_EINVAL; }
  HEC_TRY(begin_call(ctx, ws_bytes_construct(g->n, g->nnz, n_c)));
  if (ctx->validate) HEC_TRY(validate_graph(ctx, g));
  hec_csr_owned *o = new (std::nothrow) hec_csr_owned();
  if (!o) { set_error("out of host memory"); return HEC_ENOMEM; }
  o->ctx = ctx;
  int rc = build_coarse_method_impl(ctx, g, M, n_c, method, &o->c);
  o->slice = DistSlice{0, n_c, 0, o->c.nnz_c};
  if (rc != HEC_OK) {
    free_coarse(ctx, o->c);
    delete o;
    return rc;
  }
  *out = o;
  return HEC_OK;
}

HEC_API int hec_csr_dist_slice(const hec_csr_owned *csr, int64_t *row_begin, int64_t *row_end, int64_t *entry_offset,
                               int64_t *nnz_total) {
  if (!csr) { set_error("NULL argument"); return HEC_EINVAL; }
  if (row_begin) *row_begin = csr->slice.row_begin;
  if (row_end) *row_end = csr->slice.row_end;
  if (entry_offset) *entry_offset = csr->slice.entry_offset;
  if (nnz_total) *nnz_total = csr->slice.nnz_total;
  return HEC_OK;
}

HEC_API int build_coarse_graph_dist(hec_ctx *ctx, const hec_graph *g, const int32_t *M, int64_t n_c,
                                    const hec_comm *comm, int gather_full, hec_csr_owned **out) {
  if (!out) { set_error("out is NULL"); return HEC_EINVAL; }
  *out = nullptr;
  HEC_TRY(check_graph(g));
  if (g->n > 0 && !M) { set_error("M is NULL"); return HEC_EINVAL; }
  if (!comm || comm->world < 1 || comm->rank < 0 || comm->rank >= comm->world || !comm->allgather) {
    set_error("build_coarse_graph_dist: invalid comm");
    return HEC_EINVAL;
  }
  HEC_TRY(begin_call(ctx, ws_bytes_construct(g->n, g->nnz, n_c)));
  if (ctx->validate) HEC_TRY(validate_graph(ctx, g));
  hec_csr_owned *o = new (std::nothrow) hec_csr_owned();
  if (!o) { set_error("out of host memory"); return HEC_ENOMEM; }
  o->ctx = ctx;
  int rc = build_coarse_dist_impl(ctx, g, M, n_c, comm, gather_full, &o->c, &o->slice);
  if (rc != HEC_OK) {
    free_coarse(ctx, o->c);
    delete o;
    return rc;
  }
  *out = o;
  return HEC_OK;
}

HEC_API int hec_find_mapping_dist(hec_ctx *ctx, const hec_graph *g, uint64_t seed, int level, const hec_comm *comm,
                                  int32_t *M, int64_t *n_c) {
  HEC_TRY(check_graph(g));
  if ((g->n > 0 && !M) || !n_c) { set_error("M / n_c is NULL"); return HEC_EINVAL; }
  if (!comm || comm->world < 1 || comm->rank < 0 || comm->rank >= comm->world || !comm->allgather) {
    set_error("hec_find_mapping_dist: invalid comm");
    return HEC_EINVAL;
  }
  size_t ws = 0;
  ws_bytes_mapping(g->n, g->nnz, &ws);
  HEC_TRY(begin_call(ctx, ws));
  if (ctx->validate) HEC_TRY(validate_graph(ctx, g));
  MapResult r;
  HEC_TRY(find_mapping_dist_impl(ctx, g, Prio{nullptr, splitmix64(seed + (uint64_t)level)}, comm, M, &r));
  *n_c = r.n_c;
  ctx->stats.rounds = r.rounds;
  ctx->stats.n_c = r.n_c;
  return HEC_OK;
}

HEC_API int hec_csr_view(const hec_csr_owned *csr, hec_graph *view) {
  if (!csr || !view) { set_error("NULL argument"); return HEC_EINVAL; }
  view->n = csr->c.n_c;
  view->nnz = csr->c.nnz_c;
  view->row_ptr = csr->c.row_ptr;
  view->col = csr->c.col;
  view->wgt = csr->c.wgt;
  view->vwgt = csr->c.vwgt;
  return HEC_OK;
}

HEC_API void hec_csr_free(hec_csr_owned *csr) {
  if (!csr) return;
  free_coarse(csr->ctx, csr->c);
  delete csr;
}

static int hierarchy_impl(hec_ctx *ctx, const hec_graph *g0, int64_t cutoff, uint64_t seed, int64_t discard_below,
                          int max_levels, const hec_comm *comm, int64_t min_nnz, int method, int build,
                          hec_hierarchy **out);

HEC_API int coarsen_hierarchy(hec_ctx *ctx, const hec_graph *g0, int64_t cutoff, uint64_t seed,
                              int64_t discard_below, int max_levels, hec_hierarchy **out) {
  return hierarchy_impl(ctx, g0, cutoff, seed, discard_below, max_levels, nullptr, 0, HEC_MAP_HEC, HEC_BUILD_HASH,
                        out);
}

HEC_API int coarsen_hierarchy_ex(hec_ctx *ctx, const hec_graph *g0, int64_t cutoff, uint64_t seed,
                                 int64_t discard_below, int max_levels, int map_method, int build_method,
                                 hec_hierarchy **out) {
  if (map_method != HEC_MAP_HEC && map_method != HEC_MAP_HEC3 && map_method != HEC_MAP_HEM) {
    set_error("unknown mapping method %d", map_method);
    return HEC_EINVAL;
  }
  if (build_method < HEC_BUILD_HASH || build_method > HEC_BUILD_AUTO) {
    set_error("unknown construction method %d", build_method);
    return HEC_EINVAL;
  }
  return hierarchy_impl(ctx, g0, cutoff, seed, discard_below, max_levels, nullptr, 0, map_method, build_method,
                        out);
}

static int method_common(hec_ctx *ctx, const hec_graph *g, int method, Prio prio, int32_t *M, int64_t *n_c) {
  HEC_TRY(check_graph(g));
  if ((g->n > 0 && !M) || !n_c) { set_error("M / n_c is NULL"); return HEC_EINVAL; }
  size_t ws = 0;
  ws_bytes_mapping_variant(g->n, g->nnz, &ws);
  HEC_TRY(begin_call(ctx, ws));
  if (ctx->validate) HEC_TRY(validate_graph(ctx, g));
  MapResult r;
  HEC_TRY(find_mapping_method_impl(ctx, g, method, prio, M, &r));
  *n_c = r.n_c;
  ctx->stats.rounds = r.rounds;
  ctx->stats.n_c = r.n_c;
  return HEC_OK;
}

HEC_API int hec_find_mapping_method(hec_ctx *ctx, const hec_graph *g, int method, uint64_t seed, int level,
                                    int32_t *M, int64_t *n_c) {
  return method_common(ctx, g, method, Prio{nullptr, splitmix64(seed + (uint64_t)level)}, M, n_c);
}

HEC_API int hec_find_mapping_method_prio(hec_ctx *ctx, const hec_graph *g, int method, const uint64_t *prio,
                                         int32_t *M, int64_t *n_c) {
  if (!prio && g && g->n > 0) { set_error("prio is NULL"); return HEC_EINVAL; }
  return method_common(ctx, g, method, Prio{prio, 0}, M, n_c);
}

HEC_API int coarsen_hierarchy_dist(hec_ctx *ctx, const hec_graph *g0, int64_t cutoff, uint64_t seed,
                                   int64_t discard_below, int max_levels, const hec_comm *comm,
                                   int64_t partition_min_nnz, hec_hierarchy **out) {
  if (!comm || comm->world < 1 || comm->rank < 0 || comm->rank >= comm->world || !comm->allgather) {
    set_error("coarsen_hierarchy_dist: invalid comm");
    return HEC_EINVAL;
  }
  return hierarchy_impl(ctx, g0, cutoff, seed, discard_below, max_levels, comm, partition_min_nnz, HEC_MAP_HEC,
                        HEC_BUILD_HASH, out);
}

constexpr int64_t kFuseHeavyAvgU = 256;
static int hierarchy_impl(hec_ctx *ctx, const hec_graph *g0, int64_t cutoff, uint64_t seed, int64_t discard_below,
                          int max_levels, const hec_comm *comm, int64_t min_nnz, int method, int build,
                          hec_hierarchy **out) {
  if (!out) { set_error("out is NULL"); return HEC_EINVAL; }
  *out = nullptr;
  HEC_TRY(check_graph(g0));
  if (!ctx) { set_error("context is NULL"); return HEC_EINVAL; }
  if (discard_below <= 0) discard_below = 10;
  if (max_levels <= 0) max_levels = 200;
  hec_hierarchy *h = new (std::nothrow) hec_hierarchy();
  if (!h) { set_error("out of host memory"); return HEC_ENOMEM; }
  h->ctx = ctx;
  Slab *prev_slab = ctx->slab;
  ctx->slab = &h->slab;
  // reserve level-0 sized workspace once; later levels are smaller
  size_t wsm = 0;
  ws_bytes_mapping_variant(g0->n, g0->nnz, &wsm);
  size_t wsc = ws_bytes_construct(g0->n, g0->nnz, g0->n / 2 + 1);
  int rc = begin_call(ctx, wsm > wsc ? wsm : wsc);
  if (rc == HEC_OK && ctx->validate) rc = validate_graph(ctx, g0);
  hec_graph cur = *g0;
  int level = 0;
  while (rc == HEC_OK) {
    if (cur.n <= cutoff) { h->stop_reason = HEC_STOP_CUTOFF; break; }
    if (level >= max_levels) { h->stop_reason = HEC_STOP_MAX_LEVELS; break; }
    int32_t *M = nullptr;
    rc = out_alloc(ctx, (void **)&M, sizeof(int32_t) * cur.n);
    if (rc != HEC_OK) break;
    // one "level" phase per level: mapping + construction (SURVEY §8(d) B_l);
    // a discarded level is its mapping only (B = 8 nnz + 12 n)
    ctx->prof_level = level;
    const int ph_level = phase_begin(ctx, "level", 8.0 * (double)cur.nnz + 12.0 * (double)cur.n);
    size_t ws = 0;
    if (method == HEC_MAP_HEC) ws_bytes_mapping(cur.n, cur.nnz, &ws);
    else ws_bytes_mapping_variant(cur.n, cur.nnz, &ws);
    rc = ws_reserve(ctx, ws);
    ctx->ws.used = 0;
    MapResult r;
    // multi-GPU: only levels with at least min_nnz fine entries are partitioned
    const bool part = comm && comm->world > 1 && cur.nnz >= min_nnz;
    const Prio prio{nullptr, splitmix64(seed + (uint64_t)level)};
    if (rc == HEC_OK)
      rc = part ? find_mapping_dist_impl(ctx, &cur, prio, comm, M, &r)
                : find_mapping_method_impl(ctx, &cur, method, prio, M, &r);
    if (ctx->hk_map) {  // this level's heavy keys (fused into the previous placement) are used
      dev_free(ctx, ctx->hk_map);
      ctx->hk_map = nullptr;
      ctx->hk_map_col = nullptr;
    }
    if (rc != HEC_OK) { out_free(ctx, M); break; }
    ctx->stats.rounds = r.rounds;
    ctx->stats.n_c = r.n_c;
    phase_end(ctx, ph_level);  // (extended below when the level is built)
    if (r.n_c < discard_below) {
      h->stop_reason = HEC_STOP_DISCARD;
      h->discarded_n_c = r.n_c;
      out_free(ctx, M);
      break;
    }
    if (r.n_c == cur.n) {
      h->stop_reason = HEC_STOP_STALL;
      out_free(ctx, M);
      break;
    }
    rc = ws_reserve(ctx, ws_bytes_construct(cur.n, cur.nnz, r.n_c));
    ctx->ws.used = 0;
    hec_hierarchy::Level L;
    L.M = M;
    L.n_fine = cur.n;
    L.rounds = r.rounds;
    if (rc == HEC_OK) {
      if (part) {
        DistSlice sl;
        rc = build_coarse_dist_impl(ctx, &cur, M, r.n_c, comm, 1, &L.g, &sl);
      } else {
        // G_{l+1}'s heavy-neighbour keys computed by its placement (k_place),
        // so the next level's mapping skips its a1 pass over G_{l+1}
        unsigned long long *hk = nullptr;
        // (only when rows average >= kFuseHeavyAvgU entries: otherwise most entries sit in
        // multi-row piece blocks, whose per-entry row search costs more than the a1 pass)
        // (HEC_FUSE_HEAVY_ALL: test hook, every level regardless of the row volume)
        const bool fuse = method == HEC_MAP_HEC && build == HEC_BUILD_HASH &&
                          (cur.nnz >= kFuseHeavyAvgU * r.n_c || getenv("HEC_FUSE_HEAVY_ALL") != nullptr);
        if (fuse &&
            dev_alloc(ctx, (void **)&hk, sizeof(unsigned long long) * (r.n_c > 0 ? r.n_c : 1)) != HEC_OK)
          hk = nullptr;  // (optional: the mapping then runs its own a1 pass)
        ctx->hk_build = hk;
        ctx->hk_built = false;
        ctx->build_unit_wgt = r.unit_weights ? cur.wgt : nullptr;  // the expansion need not read them
        rc = build_coarse_method_impl(ctx, &cur, M, r.n_c, build, &L.g);
        ctx->build_unit_wgt = nullptr;
        ctx->hk_build = nullptr;
        if (hk && rc == HEC_OK && ctx->hk_built) {
          ctx->hk_map = hk;
          ctx->hk_map_col = L.g.col;
          ctx->hk_map_n = L.g.n_c;
        } else if (hk) {
          dev_free(ctx, hk);
        }
      }
    }
    if (rc != HEC_OK) {
      free_coarse(ctx, L.g);
      out_free(ctx, M);
      break;
    }
    phase_end(ctx, ph_level);
    phase_set_bytes(ctx, ph_level, 16.0 * (double)cur.nnz + 8.0 * (double)L.g.nnz_c + 28.0 * (double)cur.n +
                                       12.0 * (double)L.g.n_c);
    h->levels.push_back(L);
    cur.n = L.g.n_c;
    cur.nnz = L.g.nnz_c;
    cur.row_ptr = L.g.row_ptr;
    cur.col = L.g.col;
    cur.wgt = L.g.wgt;
    cur.vwgt = L.g.vwgt;
    ++level;
  }
  ctx->prof_level = -1;
  ctx->slab = prev_slab;
  if (ctx->hk_map) {  // keys of a level the loop did not map (cutoff / cap)
    dev_free(ctx, ctx->hk_map);
    ctx->hk_map = nullptr;
    ctx->hk_map_col = nullptr;
  }
  if (rc != HEC_OK) {
    hec_hierarchy_free(h);
    return rc;
  }
  *out = h;
  return HEC_OK;
}

HEC_API int hec_hierarchy_levels(const hec_hierarchy *h) { return h ? (int)h->levels.size() : 0; }

HEC_API int hec_hierarchy_level(const hec_hierarchy *h, int i, hec_graph *g_i, const int32_t **M_i,
                                int64_t *n_fine) {
  if (!h || i < 1 || i > (int)h->levels.size()) { set_error("level index out of range"); return HEC_EINVAL; }
  const auto &L = h->levels[i - 1];
  if (g_i) {
    g_i->n = L.g.n_c;
    g_i->nnz = L.g.nnz_c;
    g_i->row_ptr = L.g.row_ptr;
    g_i->col = L.g.col;
    g_i->wgt = L.g.wgt;
    g_i->vwgt = L.g.vwgt;
  }
  if (M_i) *M_i = L.M;
  if (n_fine) *n_fine = L.n_fine;
  return HEC_OK;
}

HEC_API int hec_hierarchy_stop_reason(const hec_hierarchy *h) { return h ? h->stop_reason : -1; }
HEC_API int64_t hec_hierarchy_discarded_n_c(const hec_hierarchy *h) { return h ? h->discarded_n_c : -1; }
HEC_API int hec_hierarchy_rounds(const hec_hierarchy *h, int i) {
  if (!h || i < 1 || i > (int)h->levels.size()) return -1;
  return h->levels[i - 1].rounds;
}

HEC_API void hec_hierarchy_free(hec_hierarchy *h) {
  if (!h) return;
  hec_ctx *ctx = h->ctx;
  Slab *prev = ctx->slab;
  ctx->slab = &h->slab;
  for (auto &L : h->levels) {
    free_coarse(ctx, L.g);
    out_free(ctx, L.M);
  }
  ctx->slab = prev;
  for (auto &c : h->slab.chunks) dev_free(ctx, c.base);
  delete h;
}

}  // extern "C"
