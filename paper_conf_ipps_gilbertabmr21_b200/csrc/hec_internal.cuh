// hec_internal.cuh — shared device/host plumbing of libhec (sm_100a only).
// Context + grow-only workspace arena, error reporting, the splitmix64 visit
// order, a CUB-free single-pass decoupled-look-back scan, and
// a software grid barrier for cooperative (co-resident) launches.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>

#include <string>
#include <vector>

#include "hec.h"

#if defined(__CUDA_ARCH__) && (__CUDA_ARCH__ != 1000)
#error "libhec is written for sm_100a only"
#endif

namespace hec {

// ------------------------------------------------------------------ errors
void set_error(const char *fmt, ...);
struct Status {
  int code = HEC_OK;
};

#define HEC_CUDA_TRY(expr)                                                        \
  do {                                                                            \
    cudaError_t _e = (expr);                                                      \
    if (_e != cudaSuccess) {                                                      \
      ::hec::set_error("%s:%d %s: %s", __FILE__, __LINE__, #expr,                 \
                       cudaGetErrorString(_e));                                   \
      return _e == cudaErrorMemoryAllocation ? HEC_ENOMEM : HEC_ECUDA;            \
    }                                                                             \
  } while (0)

#define HEC_TRY(expr)            \
  do {                           \
    int _rc = (expr);            \
    if (_rc != HEC_OK) return _rc; \
  } while (0)

// Every kernel launch site is followed by HEC_LAUNCH_CHECK(): counts the launch
// on the context in scope (`ctx`) and surfaces launch errors.
#define HEC_LAUNCH_CHECK()           \
  do {                               \
    ctx->launches++;                 \
    HEC_CUDA_TRY(cudaGetLastError()); \
  } while (0)

// ---------------------------------------------------------- visit order R3
__host__ __device__ __forceinline__ uint64_t splitmix64(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ULL;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}
// s_l = splitmix64(seed + level);  prio(u) = (splitmix64(s_l ^ u) >> 32) << 32 | u
__host__ __device__ __forceinline__ uint64_t prio_of(uint64_t s_l, uint32_t u) {
  return ((splitmix64(s_l ^ (uint64_t)u) >> 32) << 32) | (uint64_t)u;
}

// Either an explicit device priority array (test hook) or the R3 hash.
struct Prio {
  const uint64_t *arr;  // nullable
  uint64_t s_l;
  __device__ __forceinline__ uint64_t operator()(uint32_t u) const {
    return arr ? __ldg(arr + u) : prio_of(s_l, u);
  }
};

// --------------------------------------------------------------- context
struct Arena {
  char *base = nullptr;
  size_t cap = 0, used = 0;
};

// Output slab of one hierarchy: output buffers below kSlabDirect bytes (M,
// row_ptr, vwgt, col, wgt of the small levels) are bump-allocated from shared
// chunks, so a hierarchy of many small levels makes a few allocator calls
// instead of five per level.  Freed with the hierarchy.
struct Slab {
  struct Chunk {
    char *base;
    size_t cap, used;
  };
  std::vector<Chunk> chunks;
  bool owns(const void *p) const {
    for (const auto &c : chunks)
      if ((const char *)p >= c.base && (const char *)p < c.base + c.cap) return true;
    return false;
  }
};
constexpr size_t kSlabDirect = (size_t)16 << 20;
constexpr size_t kSlabChunk = (size_t)64 << 20;

}  // namespace hec

struct hec_ctx {
  cudaStream_t stream = nullptr;
  hec_alloc_fn alloc = nullptr;
  hec_free_fn free = nullptr;
  void *user = nullptr;
  int validate = 0;
  int device = 0;
  int num_sms = 148;
  size_t smem_optin = 0;
  hec::Arena ws;   // per-call workspace (reserved up front)
  hec::Arena ws2;  // construction skew-path workspace (sized after classification)
  hec::Slab *slab = nullptr;      // output slab of the hierarchy being built (out_alloc)
  cudaMemPool_t pool = nullptr;   // own memory pool when no allocator callback is given
  int64_t *h_pinned = nullptr;  // pinned host scalars for D2H reads
  hec_stats stats{};
  // state carried between hec_build_rows_count and hec_build_rows_write
  struct DistState *dist = nullptr;
  // heavy-neighbour keys fused into the placement of G_{l+1} (hierarchy only):
  // hk_build: target of the build in progress (k_place), hk_built: it was filled;
  // hk_map / hk_map_col / hk_map_n: keys of the graph whose col array is hk_map_col,
  // used by the next mapping instead of its a1 pass
  // weight array of the graph being built whose weights are all 1 (the a1 pass's
  // flag; hierarchy only; nested builds on other graphs read their weights)
  const int32_t *build_unit_wgt = nullptr;
  bool unit_flag_armed = false;  // the a1 span pass of the current mapping sets h_pinned[63]
  unsigned long long *hk_build = nullptr;
  bool hk_built = false;
  unsigned long long *hk_map = nullptr;
  const int32_t *hk_map_col = nullptr;
  int64_t hk_map_n = 0;
  // profiling (hec_ctx_set_profiling)
  int64_t launches = 0;
  int prof_on = 0;
  int prof_level = -1;  // hierarchy level of the phases being recorded (-1: single calls)
  struct PhaseRec {
    const char *name;
    cudaEvent_t a, b;
    double bytes;
    int level;
  };
  std::vector<PhaseRec> prof_pending;
  std::vector<cudaEvent_t> prof_pool;
  struct PhaseAcc {
    std::string name;
    int level = -1;
    double ms = 0, bytes = 0;
    int64_t calls = 0;
  };
  std::vector<PhaseAcc> prof_acc;
  // launch setup per kernel (hec::kernel_occupancy): a context is bound to one
  // device, so the cache is per device by construction
  std::vector<std::pair<const void *, int>> kcache;
};

namespace hec {

// Device memory owned by outputs goes through ctx->alloc (or cudaMallocAsync).
int dev_alloc(hec_ctx *ctx, void **p, size_t bytes);
void dev_free(hec_ctx *ctx, void *p);
// output buffers: from ctx->slab when one is set and the buffer is small, else dev_alloc
int out_alloc(hec_ctx *ctx, void **p, size_t bytes);
void out_free(hec_ctx *ctx, void *p);  // no-op for slab memory (freed with its hierarchy)

// Workspace: reserve(total) once per call (grow-only), then bump-allocate.
int arena_reserve(hec_ctx *ctx, Arena *a, size_t bytes);
inline int ws_reserve(hec_ctx *ctx, size_t bytes) { return arena_reserve(ctx, &ctx->ws, bytes); }
inline size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }
template <typename T>
T *arena_take(Arena &ar, size_t count) {
  size_t off = align_up(ar.used, 256);
  size_t bytes = align_up(count * sizeof(T), 256);
  if (off + bytes > ar.cap) return nullptr;  // caller reserved too little: bug
  ar.used = off + bytes;
  return reinterpret_cast<T *>(ar.base + off);
}
template <typename T>
T *ws_take(hec_ctx *ctx, size_t count) { return arena_take<T>(ctx->ws, count); }
inline size_t ws_bytes(size_t count, size_t elem) { return align_up(count * elem, 256) + 256; }

int read_scalars(hec_ctx *ctx, const int64_t *dev, int count, int64_t *host_out);

// Launch setup of a kernel on the context's device, cached in the context:
// the dynamic shared-memory opt-in (when smem > 48 KB) and the resident CTAs
// per SM for (threads, smem).  Each kernel is always launched with the same
// (threads, smem) at its call site.
template <typename K>
int kernel_occupancy(hec_ctx *ctx, K kernel, int threads, size_t smem, int *occ) {
  const void *key = reinterpret_cast<const void *>(kernel);
  for (const auto &e : ctx->kcache)
    if (e.first == key) {
      *occ = e.second;
      return HEC_OK;
    }
  if (smem > 48 * 1024)
    HEC_CUDA_TRY(cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int o = 0;
  HEC_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, kernel, threads, smem));
  if (o < 1) o = 1;
  ctx->kcache.emplace_back(key, o);
  *occ = o;
  return HEC_OK;
}

// Phase timing: returns a handle for phase_end (-1 when profiling is off).
int phase_begin(hec_ctx *ctx, const char *name, double bytes);
void phase_end(hec_ctx *ctx, int handle);
void phase_set_bytes(hec_ctx *ctx, int handle, double bytes);

// ------------------------------------------------------ memory ordering
__device__ __forceinline__ uint64_t ld_acquire(const uint64_t *p) {
  uint64_t v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release(uint64_t *p, uint64_t v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned ld_acquire_u32(const unsigned *p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

// ----------------------------------------------------------- grid barrier
// For kernels launched with cudaLaunchCooperativeKernel (all CTAs resident).
struct GridBarrier {
  unsigned *count;  // zero-initialised
  unsigned *gen;
  __device__ __forceinline__ void sync(unsigned nblocks) const {
    __syncthreads();
    if (threadIdx.x == 0) {
      unsigned g = ld_acquire_u32(gen);
      __threadfence();
      if (atomicAdd(count, 1u) == nblocks - 1) {
        atomicExch(count, 0u);
        __threadfence();
        atomicAdd(gen, 1u);
      } else {
        while (ld_acquire_u32(gen) == g) __nanosleep(20);
      }
      __threadfence();
    }
    __syncthreads();
  }
};

// ------------------------------------------------ decoupled look-back scan
// Single-pass exclusive scan (Merrill & Garland's chained scan with decoupled
// look-back).  Tile descriptors pack a 2-bit status above a 62-bit value.
constexpr uint64_t kFlagA = 1ull << 62;  // aggregate available
constexpr uint64_t kFlagP = 2ull << 62;  // inclusive prefix available
constexpr uint64_t kValMask = (1ull << 62) - 1;

struct ScanTiles {
  uint64_t *desc;     // [num_tiles], zeroed before the scan
  unsigned *ticket;   // [1], zeroed
};

template <int BLOCK>
__device__ __forceinline__ int64_t block_exclusive_sum(int64_t v, int64_t *total, int64_t *s_warp) {
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  int64_t x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    int64_t y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) s_warp[wid] = x;
  __syncthreads();
  if (wid == 0) {
    int64_t w = lane < BLOCK / 32 ? s_warp[lane] : 0;
    int64_t ws = w;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      int64_t y = __shfl_up_sync(0xffffffffu, ws, o);
      if (lane >= o) ws += y;
    }
    if (lane < BLOCK / 32) s_warp[lane] = ws - w;  // exclusive warp offsets
    if (lane == BLOCK / 32 - 1) s_warp[32] = ws;
  }
  __syncthreads();
  int64_t r = s_warp[wid] + x - v;
  *total = s_warp[32];
  __syncthreads();
  return r;
}

// Publish the aggregate of `tile` (tile 0 publishes its inclusive prefix).
__device__ __forceinline__ void lookback_publish(uint64_t *desc, int tile, int64_t agg) {
  st_release(desc + tile, (tile == 0 ? kFlagP : kFlagA) | (uint64_t)agg);
}

// Warp 0 resolves the exclusive prefix of `tile` whose aggregate `agg` was
// already published, then publishes the inclusive prefix.
__device__ __forceinline__ int64_t lookback_resolve(uint64_t *desc, int tile, int64_t agg) {
  const int lane = threadIdx.x & 31;
  if (tile == 0) return 0;
  // Windows of 32 x kLB predecessors per round: with hundreds of blocks in
  // flight the nearest inclusive prefix is typically ~that far back, so a wide
  // window resolves in one or two L2 round trips.  Predecessor at distance
  // lane + 32*i (i < kLB) is examined by `lane`.
  constexpr int kLB = 8;
  int64_t prefix = 0;
  int base = tile - 1;
  while (true) {
    uint64_t d[kLB];
#pragma unroll
    for (int i = 0; i < kLB; ++i) {
      const int j = base - lane - 32 * i;
      d[i] = j >= 0 ? ld_acquire(desc + j) : kFlagP;  // virtual prefix 0 before tile 0
    }
#pragma unroll
    for (int i = 0; i < kLB; ++i) {
      const int j = base - lane - 32 * i;
      // poll with backoff: hundreds of CTAs spinning on L2 would otherwise steal
      // request bandwidth from the predecessors they wait for
      unsigned ns = 32;
      while ((d[i] >> 62) == 0) {
        __nanosleep(ns);
        ns = ns < 1024 ? ns * 2 : ns;
        d[i] = ld_acquire(desc + j);
      }
    }
    // nearest predecessor holding an inclusive prefix: smallest distance
    int near = 32 * kLB;
#pragma unroll
    for (int i = kLB - 1; i >= 0; --i)
      if ((d[i] >> 62) == 2) near = lane + 32 * i;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) near = min(near, __shfl_xor_sync(0xffffffffu, near, o));
    int64_t v = 0;
#pragma unroll
    for (int i = 0; i < kLB; ++i)
      if (lane + 32 * i <= near) v += (int64_t)(d[i] & kValMask);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    prefix += v;
    if (near < 32 * kLB) break;
    base -= 32 * kLB;
  }
  if (lane == 0) st_release(desc + tile, kFlagP | (uint64_t)(prefix + agg));
  return prefix;
}

// Warp 0: publish the aggregate and resolve the exclusive prefix.
__device__ __forceinline__ int64_t lookback(uint64_t *desc, int tile, int64_t agg) {
  if ((threadIdx.x & 31) == 0) lookback_publish(desc, tile, agg);
  __syncwarp();
  return lookback_resolve(desc, tile, agg);
}

// Exclusive scan over i in [0, N): out(i, prefix_i) with in(i) >= 0.
// ITEMS consecutive elements per thread; total written to *total and *total2
// (each if non-null; total2: a copy for a batched host read).
template <int BLOCK, int ITEMS, typename In, typename Out>
__global__ void __launch_bounds__(BLOCK) k_chained_scan(int64_t N, In in, Out out, ScanTiles st,
                                                       int64_t *total, int64_t *total2) {
  __shared__ int s_tile;
  __shared__ int64_t s_warp[33];
  __shared__ int64_t s_prefix;
  if (threadIdx.x == 0) s_tile = (int)atomicAdd(st.ticket, 1u);
  __syncthreads();
  const int tile = s_tile;
  const int64_t base = (int64_t)tile * BLOCK * ITEMS + (int64_t)threadIdx.x * ITEMS;
  int64_t v[ITEMS];
  int64_t sum = 0;
#pragma unroll
  for (int i = 0; i < ITEMS; ++i) {
    int64_t idx = base + i;
    v[i] = idx < N ? in(idx) : 0;
    sum += v[i];
  }
  int64_t agg;
  int64_t excl = block_exclusive_sum<BLOCK>(sum, &agg, s_warp);
  if (threadIdx.x < 32) {
    int64_t p = lookback(st.desc, tile, agg);
    if (threadIdx.x == 0) s_prefix = p;
  }
  __syncthreads();
  int64_t run = s_prefix + excl;
#pragma unroll
  for (int i = 0; i < ITEMS; ++i) {
    int64_t idx = base + i;
    if (idx < N) out(idx, run);
    run += v[i];
  }
  // the thread holding element N-1 writes the grand total
  if (N > 0 && base <= N - 1 && N - 1 < base + ITEMS) {
    if (total) *total = run;
    if (total2) *total2 = run;
  }
}

constexpr int kScanBlock = 256, kScanItems = 8;
inline int64_t scan_tiles(int64_t N) {
  int64_t per = (int64_t)kScanBlock * kScanItems;
  return N <= 0 ? 1 : (N + per - 1) / per;
}
// Launch helper: `st` must point to scan_tiles(N) descriptors + ticket (workspace).
template <typename In, typename Out>
int chained_scan(hec_ctx *ctx, int64_t N, In in, Out out, ScanTiles st, int64_t *total, bool zeroed = false,
                 int64_t *total2 = nullptr) {
  int64_t tiles = scan_tiles(N);
  if (!zeroed) {  // (zeroed: the caller cleared desc / ticket, e.g. in one ZeroList launch)
    HEC_CUDA_TRY(cudaMemsetAsync(st.desc, 0, sizeof(uint64_t) * tiles, ctx->stream));
    HEC_CUDA_TRY(cudaMemsetAsync(st.ticket, 0, sizeof(unsigned), ctx->stream));
  }
  if (N == 0) {
    if (total) HEC_CUDA_TRY(cudaMemsetAsync(total, 0, sizeof(int64_t), ctx->stream));
    if (total2) HEC_CUDA_TRY(cudaMemsetAsync(total2, 0, sizeof(int64_t), ctx->stream));
    return HEC_OK;
  }
  k_chained_scan<kScanBlock, kScanItems><<<(unsigned)tiles, kScanBlock, 0, ctx->stream>>>(
      N, in, out, st, total, total2);
  HEC_LAUNCH_CHECK();
  return HEC_OK;
}
// Several workspace regions cleared by one launch instead of one memset each
// (small levels are bound by the number of stream operations).
struct ZeroList {
  static constexpr int kMax = 20;
  void *p[kMax];
  int64_t bytes[kMax];
  int n = 0;
  void add(void *ptr, int64_t b) {
    if (b > 0) { p[n] = ptr; bytes[n] = b; ++n; }
  }
  void add(ScanTiles st, int64_t N);  // a scan's tile descriptors and ticket
};
int zero_regions(hec_ctx *ctx, const ZeroList &z);

inline ScanTiles take_scan_tiles(Arena &ar, int64_t N) {
  ScanTiles st;
  st.desc = arena_take<uint64_t>(ar, (size_t)scan_tiles(N));
  st.ticket = arena_take<unsigned>(ar, 1);
  return st;
}
inline ScanTiles take_scan_tiles(hec_ctx *ctx, int64_t N) { return take_scan_tiles(ctx->ws, N); }
inline void ZeroList::add(ScanTiles st, int64_t N) {
  add(st.desc, (int64_t)sizeof(uint64_t) * scan_tiles(N));
  add(st.ticket, (int64_t)sizeof(unsigned));
}
inline size_t scan_ws_bytes(int64_t N) {
  return ws_bytes((size_t)scan_tiles(N), 8) + ws_bytes(1, 4);
}

// ----------------------------------------------------- internal entry points
struct MapResult {
  int64_t n_c = 0;
  int rounds = 0;
  bool unit_weights = false;  // the a1 span pass saw only weights of 1
};
int ws_bytes_mapping(int64_t n, int64_t nnz, size_t *bytes);
// M (device) and optional root (device u8) outputs; uses workspace already reserved.
int find_mapping_impl(hec_ctx *ctx, const hec_graph *g, Prio prio, int32_t *M, uint8_t *root_out,
                      int32_t *H_out, MapResult *res);
int heavy_only_impl(hec_ctx *ctx, const hec_graph *g, int32_t *H);
// HEC / HEC3 / HEM (HEC_MAP_*) of one level (mapping_variants.cu).
int ws_bytes_mapping_variant(int64_t n, int64_t nnz, size_t *bytes);
int find_mapping_method_impl(hec_ctx *ctx, const hec_graph *g, int method, Prio prio, int32_t *M, MapResult *res);

struct CoarseOut {
  int64_t n_c = 0, nnz_c = 0;
  int64_t *row_ptr = nullptr;
  int32_t *col = nullptr, *wgt = nullptr, *vwgt = nullptr;
};
size_t ws_bytes_construct(int64_t n, int64_t nnz, int64_t n_c);
void free_coarse(hec_ctx *ctx, CoarseOut &c);
// Construction variants: sort_dedup = the sort / bucket path for all rows
// instead of the hash rank (HEC_BUILD_SORT); one_end_cp = C' of Alg 6 (one-end
// storage of every coarse edge, HEC_BUILD_ONE_END's first pass).
struct BuildOpts {
  bool sort_dedup = false;
  const unsigned long long *one_end_cp = nullptr;
};
// Coarse rows [a_lo, a_hi) only (a_hi < 0: all rows); out->n_c = a_hi - a_lo and
// row_ptr/vwgt are indexed from a_lo, row_ptr[0] = 0 (range partition, §8(e)).
int build_coarse_impl(hec_ctx *ctx, const hec_graph *g, const int32_t *M, int64_t n_c,
                      CoarseOut *out, int64_t a_lo = 0, int64_t a_hi = -1, const BuildOpts *opt = nullptr);
// HEC_BUILD_* dispatch (construct_oneend.cu).
int build_coarse_method_impl(hec_ctx *ctx, const hec_graph *g, const int32_t *M, int64_t n_c, int method,
                             CoarseOut *out);
// Heavy neighbours of fine rows [u0, u1) only (H indexed globally).
int heavy_range_impl(hec_ctx *ctx, const hec_graph *g, int64_t u0, int64_t u1, int32_t *H);
// Resolution rounds + relabel from a full heavy array H; M written for [u0, u1).
int mapping_from_heavy_impl(hec_ctx *ctx, const hec_graph *g, const int32_t *H, Prio prio, int64_t u0,
                            int64_t u1, int32_t *M, MapResult *res);
// Member-edge volume U(a) of every coarse row (int64, device) for range balancing.
int row_volume_impl(hec_ctx *ctx, const hec_graph *g, const int32_t *M, int64_t n_c, int64_t *U);
int validate_graph(hec_ctx *ctx, const hec_graph *g);
// Coarse rows split into `parts` ranges of about equal member-edge volume (host bounds[parts+1]).
int balance_rows_impl(hec_ctx *ctx, const hec_graph *g, const int32_t *M, int64_t n_c, int parts, int64_t *bounds);
// Multi-GPU (dist.cu): mapping with H / M all-gathered; construction by coarse-row range.
int find_mapping_dist_impl(hec_ctx *ctx, const hec_graph *g, Prio prio, const hec_comm *comm, int32_t *M,
                           MapResult *res);
constexpr int kMaxWorld = 64;  // ranks of the multi-GPU calls
struct DistSlice {
  int64_t row_begin = 0, row_end = 0, entry_offset = 0, nnz_total = 0;
};
int build_coarse_dist_impl(hec_ctx *ctx, const hec_graph *g, const int32_t *M, int64_t n_c, const hec_comm *comm,
                           int gather_full, CoarseOut *out, DistSlice *slice);

}  // namespace hec

// Owned results (opaque in hec.h).
struct hec_csr_owned {
  hec_ctx *ctx;
  hec::CoarseOut c;
  hec::DistSlice slice;  // rows / entries this result holds (the whole graph unless a dist slice)
};

struct hec_hierarchy {
  hec_ctx *ctx;
  struct Level {
    hec::CoarseOut g;
    int32_t *M;
    int64_t n_fine;
    int rounds;
  };
  std::vector<Level> levels;
  hec::Slab slab;
  int stop_reason = HEC_STOP_CUTOFF;
  int64_t discarded_n_c = -1;
};
