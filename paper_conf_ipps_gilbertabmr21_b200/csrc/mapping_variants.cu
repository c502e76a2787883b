// mapping_variants.cu — the paper's other FINDCOARSEMAPPING methods on sm_100a
// (SURVEY §8(f) f2, f4), behind the same C-ABI and construction as HEC.
//
//  HEC3 (Alg 5): the order-free second phase of HEC.  With
//     H from the same segmented heavy-neighbour stream (a1), five vertex
//     passes: mutual heavy neighbours collapse onto the smaller id (l.5-8),
//     every heavy neighbour not yet mapped becomes its own root (l.9-12,
//     idempotent stores replace the paper's AtomicCAS -- all writers store the
//     same value), the in-degree-0 vertices inherit (l.13-16), pointer jumping
//     to the root (l.17-21), FINDUNIQANDRELABEL by ascending root id (l.22,
//     reading Z3) with the decoupled-look-back scan.  P is the identity
//     (reading Z17: Alg 5's O only renames vertices).
//
//  HEM (Alg 2): greedy heavy-edge matching in the R3 visit
//     order, reproduced exactly by rounds: an undecided u is
//     decided once no undecided lower-priority vertex is adjacent to u (then
//     every vertex visited before u has already acted) nor to u's heaviest
//     undecided neighbour x (then nothing visited before u can take x first);
//     it pairs with x, or stays single.  Decisions of one round never
//     conflict (a vertex taken by u has u as its lowest-priority undecided
//     neighbour), so each round reads a snapshot of the previous one.  One
//     cooperative kernel runs all rounds; rows are scanned by a warp each.
#include "hec_internal.cuh"

namespace hec {

static inline unsigned nblk_v(int64_t n, int b) { return (unsigned)((n + b - 1) / b); }

// ------------------------------------------------------------------ HEC3
__global__ void k_hec3_mutual(int64_t n, const int32_t *__restrict__ H, int32_t *__restrict__ M) {
  const int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (u >= n) return;
  const int32_t v = H[u];
  int32_t m = -1;
  if (v == (int32_t)u) m = (int32_t)u;                    // isolated: singleton (reading Z6)
  else if (H[v] == (int32_t)u) m = v < (int32_t)u ? v : (int32_t)u;  // l.5-8
  M[u] = m;
}
__global__ void k_hec3_claim(int64_t n, const int32_t *__restrict__ H, int32_t *__restrict__ M) {
  const int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (u >= n) return;
  const int32_t v = H[u];
  if (v != (int32_t)u && M[v] == -1) M[v] = v;  // l.9-12 (every writer stores v)
}
__global__ void k_hec3_inherit(int64_t n, const int32_t *__restrict__ H, int32_t *__restrict__ M) {
  const int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (u >= n) return;
  if (M[u] == -1) M[u] = M[H[u]];  // l.13-16: H[u] has in-degree >= 1, so M[H[u]] is set
}
__global__ void k_hec3_jump(int64_t n, const int32_t *__restrict__ M, int32_t *__restrict__ R) {
  const int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (u >= n) return;
  int32_t p = M[u];  // l.17-21 (into R: M stays the snapshot the chains are read from)
  while (M[p] != p) p = M[M[p]];
  R[u] = p;
}
struct SelfRootIn {
  const int32_t *R;
  __device__ __forceinline__ int64_t operator()(int64_t u) const { return R[u] == (int32_t)u; }
};
struct SelfRootOut {
  const int32_t *R;
  int32_t *lab;
  __device__ __forceinline__ void operator()(int64_t u, int64_t prefix) const {
    if (R[u] == (int32_t)u) lab[u] = (int32_t)prefix;
  }
};
__global__ void k_label_of_root(int64_t n, const int32_t *__restrict__ R, const int32_t *__restrict__ lab,
                                int32_t *__restrict__ M) {
  const int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (u < n) M[u] = lab[R[u]];
}

// R: roots (R[u] = root vertex of u's aggregate) -> M = coarse ids by ascending root id, *n_c.
static int relabel_roots(hec_ctx *ctx, int64_t n, const int32_t *R, int32_t *lab, int32_t *M, int64_t *n_c) {
  int64_t *total = ws_take<int64_t>(ctx, 1);
  ScanTiles st = take_scan_tiles(ctx, n);
  if (!total || !st.desc) { set_error("workspace under-reserved (relabel)"); return HEC_EINVAL; }
  HEC_TRY(chained_scan(ctx, n, SelfRootIn{R}, SelfRootOut{R, lab}, st, total));
  k_label_of_root<<<nblk_v(n, 256), 256, 0, ctx->stream>>>(n, R, lab, M);
  HEC_LAUNCH_CHECK();
  return read_scalars(ctx, total, 1, n_c);
}

static int hec3_impl(hec_ctx *ctx, const hec_graph *g, int32_t *M, MapResult *res) {
  const int64_t n = g->n;
  int32_t *H = ws_take<int32_t>(ctx, n);
  int32_t *R = ws_take<int32_t>(ctx, n);
  int32_t *lab = ws_take<int32_t>(ctx, n);
  if (!H || !R || !lab) { set_error("workspace under-reserved (hec3)"); return HEC_EINVAL; }
  int ph = phase_begin(ctx, "heavy", 8.0 * (double)g->nnz + 12.0 * (double)n);
  HEC_TRY(heavy_only_impl(ctx, g, H));
  phase_end(ctx, ph);
  ph = phase_begin(ctx, "rounds", 24.0 * (double)n);
  const unsigned b = nblk_v(n, 256);
  k_hec3_mutual<<<b, 256, 0, ctx->stream>>>(n, H, M);
  HEC_LAUNCH_CHECK();
  k_hec3_claim<<<b, 256, 0, ctx->stream>>>(n, H, M);
  HEC_LAUNCH_CHECK();
  k_hec3_inherit<<<b, 256, 0, ctx->stream>>>(n, H, M);
  HEC_LAUNCH_CHECK();
  k_hec3_jump<<<b, 256, 0, ctx->stream>>>(n, M, R);
  HEC_LAUNCH_CHECK();
  phase_end(ctx, ph);
  ph = phase_begin(ctx, "relabel", 12.0 * (double)n);
  HEC_TRY(relabel_roots(ctx, n, R, lab, M, &res->n_c));
  phase_end(ctx, ph);
  res->rounds = 0;
  return HEC_OK;
}

// ------------------------------------------------------------------- HEM
struct HemArgs {
  int64_t n;
  const int64_t *row_ptr;
  const int32_t *col, *wgt;
  Prio prio;
  int32_t *Mprev, *Mnext;   // -1 undecided, else the root (deciding vertex) of the pair / singleton
  uint64_t *minp;           // lowest priority among a vertex's undecided neighbours (~0: none)
  int32_t *wl[2];
  unsigned *cnt;            // [3] rotating list counters (zeroed)
  int32_t *rounds_out;
  GridBarrier bar;
};

__device__ __forceinline__ uint64_t warp_min_u64(uint64_t v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const uint64_t y = __shfl_xor_sync(0xffffffffu, v, o);
    v = y < v ? y : v;
  }
  return v;
}
__device__ __forceinline__ uint64_t warp_max_u64(uint64_t v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const uint64_t y = __shfl_xor_sync(0xffffffffu, v, o);
    v = y > v ? y : v;
  }
  return v;
}

constexpr int kHemBlock = 256;

__global__ void __launch_bounds__(kHemBlock) k_hem_rounds(HemArgs A) {
  const unsigned nb = gridDim.x;
  const int lane = threadIdx.x & 31;
  const int64_t gwarp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)nb * blockDim.x) >> 5;
  const int64_t gtid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  const int64_t gstride = (int64_t)nb * blockDim.x;
  __shared__ unsigned s_len;
  int64_t len = A.n;
  int cur = 0, r = 1;
  while (len > 0) {
    const int32_t *list = A.wl[cur];
    // ---- 1. minp over the undecided neighbours (snapshot Mprev); one warp per vertex
    for (int64_t i = gwarp; i < len; i += nwarps) {
      const int32_t u = r == 1 ? (int32_t)i : list[i];
      uint64_t m = ~0ull;
      for (int64_t e = A.row_ptr[u] + lane; e < A.row_ptr[u + 1]; e += 32) {
        const int32_t v = __ldg(A.col + e);
        if (A.Mprev[v] == -1) {
          const uint64_t p = A.prio((uint32_t)v);
          m = p < m ? p : m;
        }
      }
      m = warp_min_u64(m);
      if (lane == 0) A.minp[u] = m;
    }
    A.bar.sync(nb);
    // ---- 2. decide: heaviest undecided neighbour x (packed key w << 32 | ~v:
    // the first maximum in column order), conditions on u and on x
    for (int64_t i = gwarp; i < len; i += nwarps) {
      const int32_t u = r == 1 ? (int32_t)i : list[i];
      const uint64_t pu = A.prio((uint32_t)u);
      if (A.minp[u] < pu) continue;  // an undecided lower-priority neighbour acts first
      uint64_t best = 0;
      for (int64_t e = A.row_ptr[u] + lane; e < A.row_ptr[u + 1]; e += 32) {
        const int32_t v = __ldg(A.col + e);
        if (A.Mprev[v] == -1) {
          const uint64_t k = ((uint64_t)(uint32_t)__ldg(A.wgt + e) << 32) | (uint64_t)(~(uint32_t)v);
          best = k > best ? k : best;
        }
      }
      best = warp_max_u64(best);
      if (lane != 0) continue;
      if (best == 0) {  // no undecided neighbour: single (Alg 2 l.13 with w = 0)
        A.Mnext[u] = u;
        continue;
      }
      const int32_t x = (int32_t)(~(uint32_t)best);
      if (A.minp[x] < pu) continue;  // an earlier vertex may take x first
      A.Mnext[u] = u;                // l.11-13: pair (u, x), root u
      A.Mnext[x] = u;
    }
    A.bar.sync(nb);
    // ---- 3. snapshot the decisions, compact the undecided
    unsigned *next_cnt = A.cnt + r % 3;
    if (gtid == 0) A.cnt[(r + 1) % 3] = 0u;
    const int64_t lim = (len + 31) & ~(int64_t)31;
    for (int64_t i = gtid; i < lim; i += gstride) {
      bool keep = false;
      int32_t u = 0;
      if (i < len) {
        u = r == 1 ? (int32_t)i : list[i];
        const int32_t m = A.Mnext[u];
        A.Mprev[u] = m;
        keep = m == -1;
      }
      const unsigned bal = __ballot_sync(0xffffffffu, keep);
      if (bal) {
        const int leader = __ffs(bal) - 1;
        unsigned base = 0;
        if (lane == leader) base = atomicAdd(next_cnt, (unsigned)__popc(bal));
        base = __shfl_sync(0xffffffffu, base, leader);
        if (keep) A.wl[cur ^ 1][base + __popc(bal & ((1u << lane) - 1))] = u;
      }
    }
    A.bar.sync(nb);
    if (threadIdx.x == 0) s_len = ld_acquire_u32(next_cnt);
    __syncthreads();
    len = s_len;
    cur ^= 1;
    ++r;
  }
  if (gtid == 0) *A.rounds_out = r - 1;
}

static int hem_impl(hec_ctx *ctx, const hec_graph *g, Prio prio, int32_t *M, MapResult *res) {
  const int64_t n = g->n;
  int32_t *Mprev = ws_take<int32_t>(ctx, n);
  int32_t *R = ws_take<int32_t>(ctx, n);
  int32_t *lab = ws_take<int32_t>(ctx, n);
  uint64_t *minp = ws_take<uint64_t>(ctx, n);
  int32_t *wl0 = ws_take<int32_t>(ctx, n);
  int32_t *wl1 = ws_take<int32_t>(ctx, n);
  unsigned *cnt = ws_take<unsigned>(ctx, 4);
  unsigned *bar = ws_take<unsigned>(ctx, 4);
  int64_t *scal = ws_take<int64_t>(ctx, 2);
  if (!Mprev || !R || !lab || !minp || !wl0 || !wl1 || !cnt || !bar || !scal) {
    set_error("workspace under-reserved (hem)");
    return HEC_EINVAL;
  }
  cudaStream_t s = ctx->stream;
  int ph = phase_begin(ctx, "rounds", 16.0 * (double)g->nnz + 24.0 * (double)n);
  HEC_CUDA_TRY(cudaMemsetAsync(Mprev, 0xff, sizeof(int32_t) * n, s));
  HEC_CUDA_TRY(cudaMemsetAsync(R, 0xff, sizeof(int32_t) * n, s));
  HEC_CUDA_TRY(cudaMemsetAsync(cnt, 0, sizeof(unsigned) * 4, s));
  HEC_CUDA_TRY(cudaMemsetAsync(bar, 0, sizeof(unsigned) * 4, s));
  HEC_CUDA_TRY(cudaMemsetAsync(scal, 0, sizeof(int64_t) * 2, s));
  HemArgs A{n, g->row_ptr, g->col, g->wgt, prio, Mprev, R, minp, {wl0, wl1}, cnt,
            reinterpret_cast<int32_t *>(scal + 1), GridBarrier{bar, bar + 1}};
  int occ = 1;
  HEC_TRY(kernel_occupancy(ctx, k_hem_rounds, kHemBlock, 0, &occ));
  int64_t grid = (int64_t)ctx->num_sms * occ;
  const int64_t want = (n * 32 + kHemBlock - 1) / kHemBlock;
  if (want < grid) grid = want < 1 ? 1 : want;
  void *args[] = {&A};
  HEC_CUDA_TRY(cudaLaunchCooperativeKernel((const void *)k_hem_rounds, dim3((unsigned)grid), dim3(kHemBlock), args,
                                           0, s));
  ctx->launches++;
  phase_end(ctx, ph);
  ph = phase_begin(ctx, "relabel", 12.0 * (double)n);
  HEC_TRY(relabel_roots(ctx, n, R, lab, M, &res->n_c));  // R: the final state (root of every vertex)
  phase_end(ctx, ph);
  int64_t rr = 0;
  HEC_TRY(read_scalars(ctx, scal + 1, 1, &rr));
  res->rounds = (int)(int32_t)(rr & 0xffffffff);
  return HEC_OK;
}

int ws_bytes_mapping_variant(int64_t n, int64_t nnz, size_t *bytes) {
  size_t b = 0;
  ws_bytes_mapping(n, nnz, &b);  // the heavy-neighbour stream's own workspace and more
  b += 6 * ws_bytes(n, 4) + ws_bytes(n, 8) + 4 * ws_bytes(4, 8) + scan_ws_bytes(n);
  *bytes = b;
  return HEC_OK;
}

int find_mapping_method_impl(hec_ctx *ctx, const hec_graph *g, int method, Prio prio, int32_t *M,
                             MapResult *res) {
  res->n_c = 0;
  res->rounds = 0;
  if (g->n == 0) return HEC_OK;
  switch (method) {
    case HEC_MAP_HEC:
      return find_mapping_impl(ctx, g, prio, M, nullptr, nullptr, res);
    case HEC_MAP_HEC3:
      return hec3_impl(ctx, g, M, res);
    case HEC_MAP_HEM:
      return hem_impl(ctx, g, prio, M, res);
    default:
      set_error("unknown mapping method %d", method);
      return HEC_EINVAL;
  }
}

}  // namespace hec
