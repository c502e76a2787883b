// mapping.cu — FINDCOARSEMAPPING for HEC on sm_100a.
//
//  a1 heavy neighbour  H[u] = argmax_{v in N(u)} W(u,v), ties -> smallest v,
//     isolated -> u.  PAPER.md Alg 4 l.2-8 (L177-187) / Alg 3 l.6-10 (L109-119).
//     Merge-path tiles over (row ends + entries): every tile covers a fixed
//     number of items regardless of the degree skew, the tile's col/wgt are
//     staged into shared memory with one cp.async.bulk (TMA) copy each, and the
//     per-row argmax runs on the packed key (w << 32) | ~v.
//  a3 resolution rounds replacing Alg 4's CAS passes (L189-224): a vertex is
//     ROOT iff a lower child (H[y]=u, prio(y)<prio(u)) is ACTIVE, ACTIVE iff no
//     lower child is still undecided.  Deterministic: only idempotent flag
//     stores; result == sequential Alg 3 (derived).  One
//     persistent cooperative kernel runs all rounds with a compacted worklist.
//  a4 relabel  coarse id = exclusive scan of root flags (FINDUNIQANDRELABEL,
//     L273) with the decoupled-look-back scan.
//  a5 inherit  M[u] = M[first root on the H-path from u] (Alg 3 l.14 L128,
//     pointer chase as in Alg 5 l.17-21 L264-271).
#include "hec_internal.cuh"

namespace hec {

// ---------------------------------------------------------------- a1 heavy
// 2048-item tiles keep a CTA's shared memory at ~37 KB, so six CTAs share an SM
// and one CTA's TMA load overlaps the others' walks (HBM needs ~35 KB in flight
// per SM); 4096-item tiles (82 KB, two per SM) left the stream latency-bound.
constexpr int kHvBlock = 256;
constexpr int kHvItems = 8;
constexpr int kHvTile = kHvBlock * kHvItems;  // merge items (row ends + entries) per tile

// Merge-path split of diagonal d between the row-end list row_ptr[1..n] and the
// entry indices 0..nnz-1: returns x = row ends consumed (entries = d - x).
__device__ __forceinline__ int64_t merge_path_x(int64_t d, const int64_t *__restrict__ row_ptr,
                                                int64_t n, int64_t nnz, int64_t ebase) {
  int64_t lo = d - nnz > 0 ? d - nnz : 0;
  int64_t hi = d < n ? d : n;
  while (lo < hi) {
    int64_t mid = (lo + hi) >> 1;
    if (__ldg(row_ptr + mid + 1) - ebase <= d - mid - 1) lo = mid + 1;
    else hi = mid;
  }
  return lo;
}

// Rows [vbase, vbase + n) of a CSR whose entries of those rows start at ebase:
// row_ptr arguments point at row vbase, values are absolute (minus ebase here).
__global__ void k_tile_coords(int64_t n, int64_t nnz, const int64_t *__restrict__ row_ptr, int64_t ebase,
                              int64_t ntiles, int64_t *__restrict__ cx) {
  int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (t > ntiles) return;
  int64_t d = t * kHvTile;
  if (d > n + nnz) d = n + nnz;
  cx[t] = merge_path_x(d, row_ptr, n, nnz, ebase);
}

__device__ __forceinline__ uint64_t pack_key(int32_t w, int32_t v) {
  return ((uint64_t)(uint32_t)w << 32) | (uint64_t)(~(uint32_t)v);
}
__device__ __forceinline__ int32_t key_vertex(uint64_t k) { return (int32_t)(~(uint32_t)k); }

__device__ __forceinline__ void mbar_init(uint64_t *bar, unsigned count) {
  unsigned a = (unsigned)__cvta_generic_to_shared(bar);
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(a), "r"(count) : "memory");
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, unsigned bytes) {
  unsigned a = (unsigned)__cvta_generic_to_shared(bar);
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(a), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void tma_bulk_g2s(void *dst, const void *src, unsigned bytes,
                                             uint64_t *bar) {
  unsigned d = (unsigned)__cvta_generic_to_shared(dst);
  unsigned b = (unsigned)__cvta_generic_to_shared(bar);
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(d),
      "l"(src), "r"(bytes), "r"(b)
      : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, unsigned phase) {
  unsigned a = (unsigned)__cvta_generic_to_shared(bar);
  unsigned done = 0;
  while (!done) {
    asm volatile(
        "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
        : "=r"(done)
        : "r"(a), "r"(phase)
        : "memory");
  }
}

static_assert(kHvTile + 2 < 32767, "rb[] holds int16 offsets");
struct HeavySmem {
  alignas(16) int32_t col[kHvTile + 8];
  alignas(16) int32_t wgt[kHvTile + 8];
  int16_t rb[kHvTile + 2];        // row begin offsets relative to the tile's first entry
  uint64_t key[kHvTile + 2];      // per-row partial argmax keys (rows split across threads)
  uint64_t bar;
};

// One tile = kHvTile merge items.  head_key[t]: partial of the tile's first row
// when that row started in an earlier tile and ends here; mid_key[t]: partial of
// the unfinished row at the tile's end (row x1 < n).
__global__ void __launch_bounds__(kHvBlock) k_heavy(int64_t n, int64_t nnz,
                                                   const int64_t *__restrict__ row_ptr, int64_t ebase,
                                                   int64_t vbase, int64_t esh,
                                                   const int32_t *__restrict__ col,
                                                   const int32_t *__restrict__ wgt,
                                                   const int64_t *__restrict__ cx,
                                                   int32_t *__restrict__ H,
                                                   uint64_t *__restrict__ head_key,
                                                   uint64_t *__restrict__ mid_key) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  HeavySmem &S = *reinterpret_cast<HeavySmem *>(smem_raw);
  const int64_t t = blockIdx.x;
  const int64_t total = n + nnz;
  const int64_t d0 = t * kHvTile;
  const int64_t d1 = (d0 + kHvTile < total) ? d0 + kHvTile : total;
  const int64_t x0 = cx[t], x1 = cx[t + 1];
  const int64_t y0 = d0 - x0, y1 = d1 - x1;
  // col/wgt point 16-byte aligned at entry ebase - esh: local entry y is element
  // y + esh there, so TMA sources stay 16-byte aligned for any range start
  const int64_t y0a = y0 + esh, y1a = y1 + esh;
  const int64_t ybase = y0a & ~(int64_t)3;
  const int64_t ya = (y0a + 3) & ~(int64_t)3, yb = y1a & ~(int64_t)3;
  const bool bulk = yb > ya;

  if (threadIdx.x == 0) {
    mbar_init(&S.bar, 1);
    if (bulk) {
      unsigned bytes = (unsigned)((yb - ya) * 4);
      mbar_expect_tx(&S.bar, 2 * bytes);
      tma_bulk_g2s(S.col + (ya - ybase), col + ya, bytes, &S.bar);
      tma_bulk_g2s(S.wgt + (ya - ybase), wgt + ya, bytes, &S.bar);
    }
  }
  // head / tail entries outside the 16-byte aligned interior
  {
    int64_t hend = bulk ? ya : y1a;
    for (int64_t y = y0a + threadIdx.x; y < hend; y += kHvBlock) {
      S.col[y - ybase] = __ldg(col + y);
      S.wgt[y - ybase] = __ldg(wgt + y);
    }
    if (bulk) {
      for (int64_t y = yb + threadIdx.x; y < y1a; y += kHvBlock) {
        S.col[y - ybase] = __ldg(col + y);
        S.wgt[y - ybase] = __ldg(wgt + y);
      }
    }
  }
  // row begins rows x0..x1+1 (clamped), and zeroed partial keys
  const int nrows = (int)(x1 - x0);  // rows whose end item lies in this tile
  for (int k = threadIdx.x; k <= nrows + 1; k += kHvBlock) {
    int64_t r = x0 + k;
    int64_t b = r <= n ? __ldg(row_ptr + r) - ebase : nnz;
    int64_t rel = b - y0;
    S.rb[k] = (int16_t)(rel < -1 ? -1 : (rel > kHvTile + 1 ? kHvTile + 1 : rel));
    S.key[k] = 0;
  }
  __syncthreads();
  if (bulk) mbar_wait(&S.bar, 0);

  // ---- per-thread merge-path walk over kHvItems items
  const int64_t tile_items = d1 - d0;
  const int64_t ld = (int64_t)threadIdx.x * kHvItems;
  if (ld < tile_items) {
    const int64_t ents = y1 - y0;
    // local search: a[k] = row end of row x0+k = rb[k+1]; b[j] = j
    int64_t lo = ld - ents > 0 ? ld - ents : 0;
    int64_t hi = ld < nrows ? ld : nrows;
    while (lo < hi) {
      int64_t mid = (lo + hi) >> 1;
      if (S.rb[mid + 1] <= ld - mid - 1) lo = mid + 1;
      else hi = mid;
    }
    int k = (int)lo;            // local row
    int y = (int)(ld - lo);     // local entry
    const int ystart = y;
    int items = (int)((tile_items - ld) < kHvItems ? (tile_items - ld) : kHvItems);
    uint64_t key = 0;
    for (int i = 0; i < items; ++i) {
      if (k < nrows && y >= S.rb[k + 1]) {
        // end item of row x0+k
        if (S.rb[k] >= ystart) {
          H[vbase + x0 + k] = key ? key_vertex(key) : (int32_t)(vbase + x0 + k);
        } else if (key) {
          atomicMax((unsigned long long *)&S.key[k], (unsigned long long)key);
        }
        ++k;
        key = 0;
      } else {
        int idx = (int)(y0a - ybase) + y;
        uint64_t kk = pack_key(S.wgt[idx], S.col[idx]);
        key = kk > key ? kk : key;
        ++y;
      }
    }
    if (key) atomicMax((unsigned long long *)&S.key[k], (unsigned long long)key);
  }
  __syncthreads();
  // ---- rows split across threads / tiles
  for (int k = threadIdx.x; k <= nrows; k += kHvBlock) {
    uint64_t key = S.key[k];
    if (k < nrows) {
      if (k == 0 && S.rb[0] < 0) {
        head_key[t] = key;                 // tail piece of a row begun in an earlier tile
      } else if (key) {
        H[vbase + x0 + k] = key_vertex(key);
      }
    } else if (x1 < n) {
      mid_key[t] = key;                    // unfinished row at the tile end
    }
  }
}

// Rows spanning tile boundaries: the tile holding the row's end item combines
// its head piece with the mid pieces of the preceding tiles of the same row.
__global__ void k_heavy_fixup(int64_t n, int64_t nnz, const int64_t *__restrict__ row_ptr, int64_t ebase,
                              int64_t vbase, int64_t ntiles, const int64_t *__restrict__ cx,
                              const uint64_t *__restrict__ head_key,
                              const uint64_t *__restrict__ mid_key, int32_t *__restrict__ H) {
  int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (t >= ntiles) return;
  int64_t x0 = cx[t], x1 = cx[t + 1];
  int64_t y0 = t * kHvTile - x0;
  if (!(x0 < x1 && x0 < n && __ldg(row_ptr + x0) - ebase < y0)) return;
  int64_t x = x0;
  uint64_t key = head_key[t];
  const int64_t rb = __ldg(row_ptr + x) - ebase;
  for (int64_t s = t - 1; s >= 0; --s) {
    if (cx[s + 1] != x) break;
    uint64_t m = mid_key[s];
    key = m > key ? m : key;
    int64_t ys = s * kHvTile - cx[s];
    if (rb >= ys) break;  // row begins in tile s
  }
  H[vbase + x] = key ? key_vertex(key) : (int32_t)(vbase + x);
}

__global__ void k_fill_identity(int64_t n, int64_t vbase, int32_t *__restrict__ H) {
  int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (u < n) H[vbase + u] = (int32_t)(vbase + u);
}

static inline unsigned nblk(int64_t n, int b) { return (unsigned)((n + b - 1) / b); }

// ------------------------------------------------- a1 heavy, segmented streaming
// Entries are streamed in warp spans of kSpan = 512 (16-byte vector loads of col
// and wgt, all issued up front).  Each warp marks the row starts / row ends that
// fall in its span in warp-private shared bitmaps, then runs a segmented max of
// the packed key (w << 32 | ~v) over the span.
// A row ending in the span is final there if it also starts in the span;
// otherwise the span's "head" value is combined by k_heavy_seg_fixup with the
// "mid" values of the spans the row covers.  No CTA barriers: warps are
// independent, so the stream never waits on a barrier.
constexpr int kSpan = 512;
constexpr int kSegWarps = 8;
struct SegWarpSmem {
  uint32_t head[kSpan / 32];
  uint32_t end[kSpan / 32];
  int32_t endrow[kSpan];
};

// x0: aligned index of span 0 (aligned index = entry + off; col/wgt - off are
// 16-byte aligned); entries [ebase, ebase + nnz) belong to rows [0, n) of rp.
// (also clears the spans' head values: one launch instead of a memset)
__global__ void k_span_coords(int64_t n, int64_t nnz, const int64_t *__restrict__ rp, int64_t ebase,
                              int64_t x0, int64_t off, int64_t nspans, int32_t *__restrict__ cx,
                              uint64_t *__restrict__ head) {
  const int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (k > nspans) return;
  if (k < nspans) head[k] = 0ull;
  if (k == nspans) { cx[k] = (int32_t)(n - 1); return; }
  if (k == 0) { cx[k] = 0; return; }  // leading empty rows belong to span 0
  int64_t e = x0 + k * kSpan - off;
  if (e < ebase) e = ebase;
  if (e > ebase + nnz - 1) e = ebase + nnz - 1;
  int64_t lo = 0, hi = n - 1;  // largest r with rp[r] <= e
  while (lo < hi) {
    const int64_t mid = (lo + hi + 1) >> 1;
    if (__ldg(rp + mid) <= e) lo = mid;
    else hi = mid - 1;
  }
  cx[k] = (int32_t)lo;
}

// Lane l of the warp owns the 16 consecutive entries [16 l, 16 l + 16) of the
// span: a sequential segmented max over them (resets at row starts, final H for
// rows that start and end inside the lane), ONE warp scan of the lane
// aggregates per span, then the lane's first row end (which may continue a row
// from earlier lanes or spans) is resolved with the scanned prefix.
// kVec: col/wgt share a 16-byte phase (int4 loads); else scalar loads.
struct SegArgs {
  int64_t n, nnz;
  const int64_t *rp;
  int64_t ebase, vbase, x0, off, nspans;
  const int32_t *colA, *wgtA;
  const int32_t *cx;
  int32_t *H;
  uint64_t *head_key, *mid_key;
  volatile int *nonunit;  // pinned host flag: set when a weight other than 1 is seen (or nullptr)
};

// lane's 16 consecutive entries of span k (4 x 16 B of col and of wgt, or scalars)
template <bool kVec>
__device__ __forceinline__ void seg_load(const SegArgs &A, int64_t k, int (&cc)[16], int (&ww)[16]) {
  const int lane = threadIdx.x & 31;
  const int64_t xs = A.x0 + k * kSpan, es = xs - A.off;
  const int64_t elo = A.ebase, ehi = A.ebase + A.nnz;
  const bool interior = es >= elo && es + kSpan <= ehi;
  if (kVec) {
    const int4 *c4 = reinterpret_cast<const int4 *>(A.colA + xs) + 4 * lane;
    const int4 *w4 = reinterpret_cast<const int4 *>(A.wgtA + xs) + 4 * lane;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int64_t e0 = es + 16 * lane + 4 * j;
      int4 c = make_int4(0, 0, 0, 0), w = make_int4(0, 0, 0, 0);
      if (interior || (e0 >= elo && e0 + 3 < ehi)) {
        c = __ldcs(c4 + j);
        w = __ldcs(w4 + j);
      } else if (e0 + 3 >= elo && e0 < ehi) {  // a group cut by the range: only its in-range entries
        const int32_t *cs = reinterpret_cast<const int32_t *>(c4 + j), *ws = reinterpret_cast<const int32_t *>(w4 + j);
        if (e0 >= elo && e0 < ehi) { c.x = __ldcs(cs); w.x = __ldcs(ws); }
        if (e0 + 1 >= elo && e0 + 1 < ehi) { c.y = __ldcs(cs + 1); w.y = __ldcs(ws + 1); }
        if (e0 + 2 >= elo && e0 + 2 < ehi) { c.z = __ldcs(cs + 2); w.z = __ldcs(ws + 2); }
        if (e0 + 3 >= elo && e0 + 3 < ehi) { c.w = __ldcs(cs + 3); w.w = __ldcs(ws + 3); }
      }
      cc[4 * j] = c.x; cc[4 * j + 1] = c.y; cc[4 * j + 2] = c.z; cc[4 * j + 3] = c.w;
      ww[4 * j] = w.x; ww[4 * j + 1] = w.y; ww[4 * j + 2] = w.z; ww[4 * j + 3] = w.w;
    }
  } else {
#pragma unroll
    for (int q = 0; q < 16; ++q) {
      const int64_t e = es + 16 * lane + q;
      cc[q] = 0;
      ww[q] = 0;
      if (interior || (e >= elo && e < ehi)) { cc[q] = __ldcs(A.colA + e); ww[q] = __ldcs(A.wgtA + e); }
    }
  }
}

// Span k with its entries in cc/ww: row starts/ends of the span as warp-private
// bitmaps, lane-sequential segmented max, ONE warp scan of the lane aggregates,
// then the lane's first row end (which may continue a row from earlier lanes or
// spans) resolved with the scanned prefix.
__device__ __forceinline__ void seg_process(const SegArgs &A, int64_t k, SegWarpSmem &W, const int (&cc)[16],
                                            int (&ww)[16]) {
  const int lane = threadIdx.x & 31;
  const int64_t xs = A.x0 + k * kSpan, es = xs - A.off;
  const int64_t elo = A.ebase, ehi = A.ebase + A.nnz;
  const bool interior = es >= elo && es + kSpan <= ehi;
  if (lane < kSpan / 32) { W.head[lane] = 0u; W.end[lane] = 0u; }
  __syncwarp();
  const int64_t r0 = A.cx[k], r1 = A.cx[k + 1];
  for (int64_t r = r0 + lane; r <= r1; r += 32) {
    const int64_t s = __ldg(A.rp + r), e = __ldg(A.rp + r + 1);
    if (s == e) {
      A.H[A.vbase + r] = (int32_t)(A.vbase + r);  // isolated (idempotent)
      continue;
    }
    const int64_t ps = s - es, pe = e - 1 - es;
    if (ps >= 0 && ps < kSpan) atomicOr(&W.head[ps >> 5], 1u << (ps & 31));
    if (pe >= 0 && pe < kSpan) {
      atomicOr(&W.end[pe >> 5], 1u << (pe & 31));
      W.endrow[pe] = (int32_t)r;
    }
  }
  __syncwarp();
  const unsigned hb = (W.head[lane >> 1] >> (16 * (lane & 1))) & 0xffffu;
  const unsigned eb = (W.end[lane >> 1] >> (16 * (lane & 1))) & 0xffffu;
  if (!interior) {
#pragma unroll
    for (int q = 0; q < 16; ++q) {
      const int64_t e = es + 16 * lane + q;
      if (e < elo || e >= ehi) ww[q] = 0;  // key 0: never a maximum
    }
  }
  uint64_t run = 0, pend = 0;
  int pend_q = -1;  // the lane's first row end before any row start in the lane
#pragma unroll
  for (int q = 0; q < 16; ++q) {
    const uint64_t key = ww[q] ? pack_key(ww[q], cc[q]) : 0ull;
    if ((hb >> q) & 1u) run = key;
    else run = key > run ? key : run;
    if ((eb >> q) & 1u) {
      if (hb & ((2u << q) - 1u)) A.H[A.vbase + W.endrow[16 * lane + q]] = key_vertex(run);
      else if (pend_q < 0) { pend = run; pend_q = q; }
    }
  }
  bool stop = hb != 0u || lane == 0;
  uint64_t incl = run;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint64_t y = __shfl_up_sync(0xffffffffu, incl, o);
    const bool ys = __shfl_up_sync(0xffffffffu, stop, o);
    if (lane >= o && !stop) {
      incl = y > incl ? y : incl;
      stop = ys;
    }
  }
  uint64_t pre = __shfl_up_sync(0xffffffffu, incl, 1);  // running value before the lane
  if (lane == 0) pre = 0;
  const unsigned hm = __ballot_sync(0xffffffffu, hb != 0u);
  if (pend_q >= 0) {
    const uint64_t v = pre > pend ? pre : pend;
    if (hm & ((1u << lane) - 1u)) A.H[A.vbase + W.endrow[16 * lane + pend_q]] = key_vertex(v);
    else A.head_key[k] = v;  // the row began in an earlier span
  }
  if (lane == 31) {
    const uint64_t last = hb ? run : (pre > run ? pre : run);
    A.mid_key[k] = (eb >> 15) & 1u ? 0ull : last;
  }
  __syncwarp();
}

// Persistent warps stride over the spans; the next span's 8 x 16 B per lane are
// loaded before the current span is processed, so every warp keeps a span of
// loads in flight while it computes.
template <bool kVec>
__global__ void __launch_bounds__(32 * kSegWarps, 2) k_heavy_seg(SegArgs A) {
  __shared__ SegWarpSmem smem[kSegWarps];
  const int wid = threadIdx.x >> 5;
  SegWarpSmem &W = smem[wid];
  const int64_t nw = (int64_t)gridDim.x * kSegWarps;
  int64_t k = blockIdx.x * (int64_t)kSegWarps + wid;
  if (k >= A.nspans) return;
  int cc[16], ww[16];
  seg_load<kVec>(A, k, cc, ww);
  bool nu = false;
  while (true) {
    const int64_t kn = k + nw;
    int nc[16], nw_[16];
    if (kn < A.nspans) seg_load<kVec>(A, kn, nc, nw_);
    seg_process(A, k, W, cc, ww);
#pragma unroll
    for (int q = 0; q < 16; ++q) nu |= (unsigned)ww[q] > 1u;  // (entries outside the range read 0)
    if (kn >= A.nspans) break;
    k = kn;
#pragma unroll
    for (int q = 0; q < 16; ++q) { cc[q] = nc[q]; ww[q] = nw_[q]; }
  }
  if (A.nonunit && __any_sync(0xffffffffu, nu) && (threadIdx.x & 31) == 0) *A.nonunit = 1;
}

// Rows that end in span k but began in an earlier span s0: max of span k's head
// value and the mid values of spans s0 .. k-1.  One thread per span (a row
// longer than a few spans is rare; its thread loops over independent loads).
__global__ void k_heavy_seg_fixup(const int64_t *__restrict__ rp, int64_t vbase, int64_t x0, int64_t off,
                                  int64_t nspans, const int32_t *__restrict__ cx,
                                  const uint64_t *__restrict__ head_key, const uint64_t *__restrict__ mid_key,
                                  int32_t *__restrict__ H) {
  const int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (k >= nspans) return;
  uint64_t m = head_key[k];
  if (m == 0ull) return;
  const int32_t x = cx[k];
  const int64_t s0 = (__ldg(rp + x) + off - x0) / kSpan;
#pragma unroll 4
  for (int64_t s = s0; s < k; ++s) {
    const uint64_t y = mid_key[s];
    m = y > m ? y : m;
  }
  H[vbase + x] = key_vertex(m);
}

static size_t heavy_ws(int64_t n, int64_t nnz) {
  int64_t ntiles = (n + nnz + kHvTile - 1) / kHvTile;
  int64_t nspans = nnz / kSpan + 2;
  size_t a = ws_bytes(ntiles + 1, 8) + 2 * ws_bytes(ntiles + 1, 8);
  size_t b = ws_bytes(nspans + 1, 4) + 2 * ws_bytes(nspans + 1, 8);
  return a > b ? a : b;
}

// Heavy neighbours of rows [u0, u1): ebase = row_ptr[u0] and nnz of the range are
// read from the device when the range is partial (one small synchronous read).
// Small graphs (nnz <= kHeavyRowsMax): one warp per row, lanes stride the row's
// entries, warp max of the packed key -- one launch instead of the span
// coordinates + segmented pass + fixup (small levels are launch-bound).
constexpr int64_t kHeavyRowsMax = 1 << 18;
__global__ void k_heavy_rows(int64_t n, const int64_t *__restrict__ rp, int64_t vbase,
                             const int32_t *__restrict__ col, const int32_t *__restrict__ wgt,
                             int32_t *__restrict__ H) {
  const int lane = threadIdx.x & 31;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t r = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; r < n; r += nw) {
    const int64_t s = rp[r], e = rp[r + 1];
    uint64_t best = 0;
    for (int64_t i = s + lane; i < e; i += 32) {
      const int32_t w = __ldg(wgt + i);
      const uint64_t k = w ? pack_key(w, __ldg(col + i)) : 0ull;  // weight 0 never wins (strict >, L116)
      best = k > best ? k : best;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      const uint64_t y = __shfl_xor_sync(0xffffffffu, best, o);
      best = y > best ? y : best;
    }
    if (lane == 0) H[vbase + r] = best ? key_vertex(best) : (int32_t)(vbase + r);  // isolated -> itself
  }
}

static int run_heavy(hec_ctx *ctx, const hec_graph *g, int32_t *H, int64_t u0 = 0, int64_t u1 = -1) {
  if (u1 < 0) u1 = g->n;
  const int64_t n = u1 - u0;
  int64_t nnz = g->nnz, ebase = 0;
  if (n <= 0) return HEC_OK;
  if (u0 != 0 || u1 != g->n) {
    HEC_CUDA_TRY(cudaMemcpyAsync(ctx->h_pinned, g->row_ptr + u0, sizeof(int64_t), cudaMemcpyDeviceToHost,
                                 ctx->stream));
    HEC_CUDA_TRY(cudaMemcpyAsync(ctx->h_pinned + 1, g->row_ptr + u1, sizeof(int64_t), cudaMemcpyDeviceToHost,
                                 ctx->stream));
    HEC_CUDA_TRY(cudaStreamSynchronize(ctx->stream));
    ebase = ctx->h_pinned[0];
    nnz = ctx->h_pinned[1] - ebase;
  }
  const int64_t *rp = g->row_ptr + u0;
  if (nnz == 0) {
    k_fill_identity<<<nblk(n, 256), 256, 0, ctx->stream>>>(n, u0, H);
    HEC_LAUNCH_CHECK();
    return HEC_OK;
  }
  // (HEC_HEAVY_SEG / HEC_HEAVY_TILES: test hooks that keep small graphs on the span / tile kernels)
  if (nnz <= kHeavyRowsMax && getenv("HEC_HEAVY_SEG") == nullptr && getenv("HEC_HEAVY_TILES") == nullptr) {
    const int64_t want = (n + 7) / 8;  // 8 warps per CTA, a row per warp
    const int64_t grid = want < (int64_t)ctx->num_sms * 8 ? want : (int64_t)ctx->num_sms * 8;
    k_heavy_rows<<<(unsigned)grid, 256, 0, ctx->stream>>>(n, rp, u0, g->col, g->wgt, H);
    HEC_LAUNCH_CHECK();
    return HEC_OK;
  }
  const uintptr_t ca = (uintptr_t)g->col, wa = (uintptr_t)g->wgt;
  const bool aligned16 = (ca & 15) == 0 && (wa & 15) == 0;
  if (n < INT32_MAX && !(aligned16 && getenv("HEC_HEAVY_TILES") != nullptr)) {
    // segmented streaming path; int4 loads when col/wgt share their 16-byte phase
    const bool vec = (ca & 3) == 0 && (ca & 15) == (wa & 15);
    const int64_t off = vec ? (int64_t)((ca & 15) >> 2) : 0;
    const int64_t x0 = (ebase + off) & ~(int64_t)3;
    const int64_t nspans = (ebase + off + nnz - x0 + kSpan - 1) / kSpan;
    int32_t *cx = ws_take<int32_t>(ctx, nspans + 1);
    uint64_t *head = ws_take<uint64_t>(ctx, nspans + 1);
    uint64_t *mid = ws_take<uint64_t>(ctx, nspans + 1);
    if (!cx || !head || !mid) { set_error("workspace under-reserved (heavy)"); return HEC_EINVAL; }
    k_span_coords<<<nblk(nspans + 1, 256), 256, 0, ctx->stream>>>(n, nnz, rp, ebase, x0, off, nspans, cx, head);
    HEC_LAUNCH_CHECK();
    // unit-weight flag (pinned host word, written by the kernel, read after the
    // mapping's host read): only for whole graphs
    volatile int *flag = (u0 == 0 && u1 == g->n) ? reinterpret_cast<volatile int *>(ctx->h_pinned + 63) : nullptr;
    if (flag) *flag = 0;
    ctx->unit_flag_armed = flag != nullptr;
    SegArgs SA{n, nnz, rp, ebase, u0, x0, off, nspans, g->col - off, g->wgt - off, cx, H, head, mid, flag};
    int occ[2] = {1, 1};
    if (vec) HEC_TRY(kernel_occupancy(ctx, k_heavy_seg<true>, 32 * kSegWarps, 0, &occ[1]));
    else HEC_TRY(kernel_occupancy(ctx, k_heavy_seg<false>, 32 * kSegWarps, 0, &occ[0]));
    int64_t grid = (int64_t)ctx->num_sms * occ[vec];
    const int64_t want = (nspans + kSegWarps - 1) / kSegWarps;
    if (want < grid) grid = want;
    if (vec) k_heavy_seg<true><<<(unsigned)grid, 32 * kSegWarps, 0, ctx->stream>>>(SA);
    else k_heavy_seg<false><<<(unsigned)grid, 32 * kSegWarps, 0, ctx->stream>>>(SA);
    HEC_LAUNCH_CHECK();
    k_heavy_seg_fixup<<<nblk(nspans, 256), 256, 0, ctx->stream>>>(rp, u0, x0, off, nspans, cx, head, mid, H);
    HEC_LAUNCH_CHECK();
    return HEC_OK;
  }
  int64_t ntiles = (n + nnz + kHvTile - 1) / kHvTile;
  int64_t *cx = ws_take<int64_t>(ctx, ntiles + 1);
  uint64_t *head = ws_take<uint64_t>(ctx, ntiles + 1);
  uint64_t *mid = ws_take<uint64_t>(ctx, ntiles + 1);
  if (!cx || !head || !mid) { set_error("workspace under-reserved (heavy)"); return HEC_EINVAL; }
  k_tile_coords<<<nblk(ntiles + 1, 256), 256, 0, ctx->stream>>>(n, nnz, rp, ebase, ntiles, cx);
  HEC_LAUNCH_CHECK();
  int occ_tiles = 1;
  HEC_TRY(kernel_occupancy(ctx, k_heavy, kHvBlock, sizeof(HeavySmem), &occ_tiles));
  k_heavy<<<(unsigned)ntiles, kHvBlock, sizeof(HeavySmem), ctx->stream>>>(
      n, nnz, rp, ebase, u0, ebase & 3, g->col + (ebase & ~(int64_t)3), g->wgt + (ebase & ~(int64_t)3), cx, H,
      head, mid);
  HEC_LAUNCH_CHECK();
  k_heavy_fixup<<<nblk(ntiles, 256), 256, 0, ctx->stream>>>(n, nnz, rp, ebase, u0, ntiles, cx, head,
                                                            mid, H);
  HEC_LAUNCH_CHECK();
  return HEC_OK;
}

// --------------------------------------------------------- a3 resolution rounds
enum : uint8_t { UNDEC = 0, ACTIVE = 2, ROOT = 3 };

// status, lower-child "blocked" stamps for round 1.
__global__ void k_round_init(int64_t n, const int32_t *__restrict__ H, Prio prio,
                             uint8_t *__restrict__ status, int32_t *__restrict__ blocked) {
  int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (u >= n) return;
  int32_t x = H[u];
  status[u] = (x == (int32_t)u) ? ROOT : UNDEC;
  if (x != (int32_t)u && prio((uint32_t)u) < prio((uint32_t)x)) blocked[x] = 1;
}

struct RoundArgs {
  int64_t n;
  const int32_t *H;
  Prio prio;
  uint8_t *status;
  uint8_t *rootflag;
  int32_t *blocked;
  int32_t *wl[2];
  unsigned *cnt;      // [3] next-list sizes, rotating by round (zeroed)
  int32_t *rounds_out;
  GridBarrier bar;
  // residual compression (adversarial visit orders): per-vertex scratch
  int32_t *child;     // an undecided lower child
  uint8_t *kind;      // K_ROOT / K_ACT / K_UNARY / K_BRANCH
  uint32_t *jmp[2];   // (target << 0) | parity << 31, double-buffered pointer jumping
};
constexpr int kSoloThreshold = 8192;  // finish small residuals in one CTA
constexpr int kRoundBlock = 512;

constexpr int kComprEvery = 32;  // rounds between residual compressions

// Round r appends its next worklist to cnt[r % 3] and zeroes cnt[(r + 1) % 3]
// before its barrier.  That counter was last appended in round r - 2 and read
// right after barrier r - 2, i.e. by every CTA before it arrived at barrier
// r - 1; its next appends (round r + 1) follow barrier r, which orders the
// zeroing store before them.  (A single reused counter reset after the barrier
// would race with the next round's appends.)
__device__ __forceinline__ unsigned *round_counter(const RoundArgs &A, int r) { return A.cnt + r % 3; }

// decide(r) for u, then scatter(r+1); returns true if u stays undecided.
__device__ __forceinline__ bool round_step(const RoundArgs &A, uint32_t u, int r) {
  uint8_t s;
  if (A.rootflag[u]) s = ROOT;
  else if (A.blocked[u] < r) s = ACTIVE;
  else s = UNDEC;
  int32_t x = A.H[u];
  if (s != UNDEC) A.status[u] = s;
  if (s != ROOT && x != (int32_t)u && A.prio(u) < A.prio((uint32_t)x)) {
    if (s == ACTIVE) A.rootflag[x] = 1;      // an active lower child makes x a root
    else A.blocked[x] = r + 1;               // x must wait for u
  }
  return s == UNDEC;
}

__device__ __forceinline__ void append(int32_t *list, unsigned *count, bool keep, uint32_t u) {
  unsigned m = __ballot_sync(0xffffffffu, keep);
  if (!m) return;
  int lane = threadIdx.x & 31;
  int leader = __ffs(m) - 1;
  unsigned base = 0;
  if (lane == leader) base = atomicAdd(count, (unsigned)__popc(m));
  base = __shfl_sync(0xffffffffu, base, leader);
  if (keep) list[base + __popc(m & ((1u << lane) - 1))] = (int32_t)u;
}

// ---- residual compression (SURVEY §8(c) "adversarial inputs")
// After round r the undecided vertices U form a forest under y -> H[y] (y a
// lower child of H[y], both undecided), and every decided child of an
// undecided x is ROOT unless it already flagged x (rootflag: an ACTIVE lower
// child makes x a ROOT).  Alg 3's outcome on U is the NOR evaluation
//   ACTIVE(x) = !rootflag[x] && no undecided lower child c of x is ACTIVE,
// so a vertex with exactly one undecided lower child c is NOT(c): unary chains
// -- the shape of adversarial orders (a path visited against its H direction
// needs n/2 rounds) -- are resolved by pointer jumping with parity in
// O(log |U|) passes; branching vertices are left to the following rounds.
enum : uint8_t { K_ROOT = 1, K_ACT = 2, K_UNARY = 3, K_BRANCH = 4 };

__device__ __forceinline__ bool is_lower(const RoundArgs &A, uint32_t y, int32_t x) {
  return x != (int32_t)y && A.prio(y) < A.prio((uint32_t)x);
}

struct GridSync {
  GridBarrier bar;
  unsigned nb;
  __device__ __forceinline__ void operator()() const { bar.sync(nb); }
};
struct BlockSync {
  __device__ __forceinline__ void operator()() const {
    __threadfence_block();
    __syncthreads();
  }
};

// Compress the residual list (len vertices in `list`, undecided); the new
// residual goes to `out` (its size counted in *out_cnt, zeroed by the caller),
// stamped for round r_next.  Returns the new length.
template <typename Sync>
__device__ int64_t compress_residual(const RoundArgs &A, const int32_t *list, int64_t len, int32_t *out,
                                     unsigned *out_cnt, int r_next, int64_t tid, int64_t stride, Sync sync,
                                     unsigned *s_len) {
  int32_t *ucnt = A.blocked;  // blocked stamps are rebuilt at the end
  for (int64_t i = tid; i < len; i += stride) ucnt[list[i]] = 0;
  sync();
  for (int64_t i = tid; i < len; i += stride) {
    const uint32_t y = (uint32_t)list[i];
    const int32_t x = A.H[y];
    if (is_lower(A, y, x) && A.status[x] == UNDEC) {
      atomicAdd(ucnt + x, 1);
      A.child[x] = (int32_t)y;
    }
  }
  sync();
  for (int64_t i = tid; i < len; i += stride) {
    const int32_t x = list[i];
    uint8_t k;
    if (A.rootflag[x]) k = K_ROOT;
    else if (ucnt[x] == 0) k = K_ACT;
    else if (ucnt[x] == 1) k = K_UNARY;
    else k = K_BRANCH;
    A.kind[x] = k;
    if (k == K_UNARY) A.jmp[0][x] = (uint32_t)A.child[x] | 0x80000000u;  // one NOT step
  }
  sync();
  int passes = 1;
  for (int64_t l = 1; l < len; l <<= 1) ++passes;
  for (int p = 0; p < passes; ++p) {
    const uint32_t *src = A.jmp[p & 1];
    uint32_t *dst = A.jmp[(p & 1) ^ 1];
    for (int64_t i = tid; i < len; i += stride) {
      const int32_t x = list[i];
      if (A.kind[x] != K_UNARY) continue;
      const uint32_t e = src[x];
      const int32_t y = (int32_t)(e & 0x7fffffffu);
      if (A.kind[y] == K_UNARY) {
        const uint32_t f = src[y];
        dst[x] = (f & 0x7fffffffu) | ((e ^ f) & 0x80000000u);
      } else {
        dst[x] = e;
      }
    }
    sync();
  }
  const uint32_t *fin = A.jmp[passes & 1];
  for (int64_t i = tid; i < len; i += stride) {
    const int32_t x = list[i];
    const uint8_t k = A.kind[x];
    int v = -1;  // 1 ACTIVE, 0 ROOT, -1 undecided
    if (k == K_ROOT) v = 0;
    else if (k == K_ACT) v = 1;
    else if (k == K_UNARY) {
      const uint32_t e = fin[x];
      const uint8_t ky = A.kind[e & 0x7fffffffu];
      if (ky == K_ROOT || ky == K_ACT) v = (ky == K_ACT) ^ (int)(e >> 31);
    }
    if (v >= 0) {
      A.status[x] = v ? ACTIVE : ROOT;
      if (v && is_lower(A, (uint32_t)x, A.H[x])) A.rootflag[A.H[x]] = 1;
    }
  }
  sync();
  const int64_t lim = (len + 31) & ~(int64_t)31;
  for (int64_t i = tid; i < lim; i += stride) {
    const int32_t u = i < len ? list[i] : 0;
    const bool keep = i < len && A.status[u] == UNDEC;
    append(out, out_cnt, keep, (uint32_t)u);
  }
  sync();
  if (threadIdx.x == 0) *s_len = *(volatile unsigned *)out_cnt;
  __syncthreads();
  const int64_t nlen = *s_len;
  for (int64_t i = tid; i < nlen; i += stride) A.blocked[out[i]] = 0;
  sync();
  for (int64_t i = tid; i < nlen; i += stride) {
    const uint32_t y = (uint32_t)out[i];
    const int32_t x = A.H[y];
    if (is_lower(A, y, x)) A.blocked[x] = r_next;
  }
  sync();
  return nlen;
}

__global__ void __launch_bounds__(kRoundBlock) k_rounds(RoundArgs A) {
  const unsigned nb = gridDim.x;
  const int64_t gtid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  const int64_t gstride = (int64_t)nb * blockDim.x;
  int r = 1;
  int64_t len = A.n;  // round 1 walks all vertices
  int cur = 0;
  __shared__ unsigned s_len;
  // ---- grid-wide rounds
  while (true) {
    unsigned *next_cnt = round_counter(A, r);
    if (gtid == 0) *round_counter(A, r + 1) = 0u;
    int32_t *next = A.wl[cur ^ 1];
    int64_t lim = (len + 31) & ~(int64_t)31;
    for (int64_t i = gtid; i < lim; i += gstride) {
      bool keep = false;
      uint32_t u = 0;
      if (i < len) {
        u = (r == 1) ? (uint32_t)i : (uint32_t)A.wl[cur][i];
        if (r > 1 || A.status[u] == UNDEC) keep = round_step(A, u, r);
      }
      append(next, next_cnt, keep, u);
    }
    A.bar.sync(nb);
    if (threadIdx.x == 0) s_len = ld_acquire_u32(next_cnt);
    __syncthreads();
    len = s_len;
    cur ^= 1;
    ++r;
    if (len == 0) {
      if (gtid == 0) *A.rounds_out = r - 1;
      return;
    }
    if (r % kComprEvery == 0) {  // long decision chains: compress the residual (counts as one round)
      unsigned *cnt_c = round_counter(A, r);
      if (gtid == 0) *round_counter(A, r + 1) = 0u;
      len = compress_residual(A, A.wl[cur], len, A.wl[cur ^ 1], cnt_c, r + 1, gtid, gstride, GridSync{A.bar, nb},
                              &s_len);
      cur ^= 1;
      ++r;
      if (len == 0) {
        if (gtid == 0) *A.rounds_out = r - 1;
        return;
      }
    }
    if (len <= kSoloThreshold) break;
  }
  // ---- small residual: CTA 0 alone, block barriers only (same counter rotation)
  if (blockIdx.x != 0) return;
  while (true) {
    unsigned *next_cnt = round_counter(A, r);
    if (threadIdx.x == 0) *round_counter(A, r + 1) = 0u;
    int32_t *next = A.wl[cur ^ 1];
    int64_t lim = (len + 31) & ~(int64_t)31;
    for (int64_t i = threadIdx.x; i < lim; i += blockDim.x) {
      bool keep = false;
      uint32_t u = 0;
      if (i < len) {
        u = (uint32_t)A.wl[cur][i];
        keep = round_step(A, u, r);
      }
      append(next, next_cnt, keep, u);
    }
    __threadfence_block();
    __syncthreads();
    if (threadIdx.x == 0) s_len = *(volatile unsigned *)next_cnt;
    __syncthreads();
    len = s_len;
    cur ^= 1;
    ++r;
    if (len == 0) break;
    if (r % kComprEvery == 0) {
      unsigned *cnt_c = round_counter(A, r);
      if (threadIdx.x == 0) *round_counter(A, r + 1) = 0u;
      __syncthreads();
      len = compress_residual(A, A.wl[cur], len, A.wl[cur ^ 1], cnt_c, r + 1, threadIdx.x, blockDim.x, BlockSync{},
                              &s_len);
      cur ^= 1;
      ++r;
      if (len == 0) break;
    }
  }
  if (threadIdx.x == 0) *A.rounds_out = r - 1;
}

// ------------------------------------------------------- a4 / a5 relabel + M
struct RootFlagIn {
  const uint8_t *status;
  __device__ __forceinline__ int64_t operator()(int64_t u) const { return status[u] == ROOT; }
};
struct RootLabelOut {
  const uint8_t *status;
  int32_t *lab;       // coarse id of each root (M itself when M covers all vertices)
  uint8_t *root_out;  // nullable
  __device__ __forceinline__ void operator()(int64_t u, int64_t prefix) const {
    bool r = status[u] == ROOT;
    if (r) lab[u] = (int32_t)prefix;
    if (root_out) root_out[u] = r;
  }
};

// M[u] for u in [u0, u1): the label of the first root on u's H-path (Alg 3
// l.14 inherit, Alg 5 l.17-21 pointer jumping).
// Active chains strictly decrease in priority, so with R3's hashed priorities
// they are a few steps long; a walk is cut after kAssignWalk steps and the
// vertex is left to the pointer-jumping passes below (adversarial explicit
// priorities, e.g. a path visited in id order: one chain of length n).
constexpr int kAssignWalk = 64;
__global__ void k_assign(int64_t u0, int64_t u1, const int32_t *__restrict__ H,
                         const uint8_t *__restrict__ status, const int32_t *__restrict__ lab,
                         int32_t *__restrict__ M, int32_t *__restrict__ jump, int *__restrict__ long_chain) {
  int64_t u = u0 + blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (u >= u1) return;
  if (status[u] == ROOT) {
    if (lab != M) M[u] = lab[u];
    return;
  }
  int32_t x = H[u];
  for (int s = 0; s < kAssignWalk; ++s) {
    if (status[x] == ROOT) {
      M[u] = lab[x];
      return;
    }
    x = H[x];
  }
  jump[u] = x;  // resumed by k_jump
  *long_chain = 1;
}

// Pointer jumping over all vertices: jump[u] = first root on u's H-path for
// roots' predecessors.  Init: jump[u] = u (root) or H[u]; each pass replaces
// jump[u] by jump[jump[u]] (concurrent updates only move further along the
// same path, so every interleaving converges), ceil(log2 n) passes suffice.
__global__ void k_jump_init(int64_t n, const int32_t *__restrict__ H, const uint8_t *__restrict__ status,
                            int32_t *__restrict__ jump) {
  int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (u < n) jump[u] = status[u] == ROOT ? (int32_t)u : H[u];
}
__global__ void k_jump(int64_t n, const uint8_t *__restrict__ status, int32_t *__restrict__ jump) {
  int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (u >= n) return;
  const int32_t x = jump[u];
  if (status[x] != ROOT) jump[u] = jump[x];
}
__global__ void k_assign_jumped(int64_t u0, int64_t u1, const uint8_t *__restrict__ status,
                                const int32_t *__restrict__ jump, const int32_t *__restrict__ lab,
                                int32_t *__restrict__ M) {
  int64_t u = u0 + blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (u >= u1 || status[u] == ROOT) return;
  M[u] = lab[jump[u]];
}

int ws_bytes_mapping(int64_t n, int64_t nnz, size_t *bytes) {
  size_t b = 0;
  b += ws_bytes(n, 4);          // H
  b += ws_bytes(n, 1) * 2;      // status, rootflag
  b += ws_bytes(n, 4);          // blocked
  b += 2 * ws_bytes(n, 4);      // worklists
  b += 3 * ws_bytes(n, 4) + ws_bytes(n, 1);  // residual compression: child, jmp[2], kind
  b += ws_bytes(4, 4) + ws_bytes(4, 4) + ws_bytes(4, 8);
  b += heavy_ws(n, nnz);
  b += scan_ws_bytes(n);
  b += ws_bytes(n, 4);          // labels (partial-range mapping)
  *bytes = b;
  return HEC_OK;
}

int heavy_only_impl(hec_ctx *ctx, const hec_graph *g, int32_t *H) { return run_heavy(ctx, g, H); }

// a3-a5 from a full heavy-neighbour array H; M written for [u0, u1).
static int resolve_impl(hec_ctx *ctx, const hec_graph *g, const int32_t *H, Prio prio, int64_t u0, int64_t u1,
                        int32_t *M, uint8_t *root_out, MapResult *res) {
  const int64_t n = g->n;
  cudaStream_t s = ctx->stream;
  uint8_t *status = ws_take<uint8_t>(ctx, n);
  uint8_t *rootflag = ws_take<uint8_t>(ctx, n);
  int32_t *blocked = ws_take<int32_t>(ctx, n);
  int32_t *wl0 = ws_take<int32_t>(ctx, n);
  int32_t *wl1 = ws_take<int32_t>(ctx, n);
  int32_t *child = ws_take<int32_t>(ctx, n);
  uint32_t *jmp0 = ws_take<uint32_t>(ctx, n);
  uint32_t *jmp1 = ws_take<uint32_t>(ctx, n);
  uint8_t *kind = ws_take<uint8_t>(ctx, n);
  unsigned *cnt = ws_take<unsigned>(ctx, 4);
  unsigned *bar = ws_take<unsigned>(ctx, 4);
  int64_t *scal = ws_take<int64_t>(ctx, 4);  // [0] n_c, [1] rounds (int32 in low word), [2] long chain
  const bool full = u0 == 0 && u1 == n;
  int32_t *lab = full ? M : ws_take<int32_t>(ctx, n);
  if (!status || !rootflag || !blocked || !wl0 || !wl1 || !cnt || !bar || !scal || !lab || !child || !jmp0 || !jmp1 ||
      !kind) {
    set_error("workspace under-reserved (mapping)");
    return HEC_EINVAL;
  }
  const double dn = (double)n;
  int ph = phase_begin(ctx, "rounds", 5.0 * dn);
  ScanTiles st = take_scan_tiles(ctx, n);  // (relabel scan below)
  if (!st.desc || !st.ticket) { set_error("workspace under-reserved (scan)"); return HEC_EINVAL; }
  {
    ZeroList z;
    z.add(rootflag, n);
    z.add(blocked, (int64_t)sizeof(int32_t) * n);
    z.add(cnt, (int64_t)sizeof(unsigned) * 4);
    z.add(bar, (int64_t)sizeof(unsigned) * 4);
    z.add(scal, (int64_t)sizeof(int64_t) * 4);
    z.add(st, n);
    HEC_TRY(zero_regions(ctx, z));
  }
  k_round_init<<<nblk(n, 256), 256, 0, s>>>(n, H, prio, status, blocked);
  HEC_LAUNCH_CHECK();

  RoundArgs A;
  A.n = n; A.H = H; A.prio = prio; A.status = status; A.rootflag = rootflag; A.blocked = blocked;
  A.wl[0] = wl0; A.wl[1] = wl1; A.cnt = cnt; A.rounds_out = reinterpret_cast<int32_t *>(scal + 1);
  A.bar.count = bar; A.bar.gen = bar + 1;
  A.child = child; A.kind = kind; A.jmp[0] = jmp0; A.jmp[1] = jmp1;
  int occ = 1;
  HEC_TRY(kernel_occupancy(ctx, k_rounds, kRoundBlock, 0, &occ));
  int64_t want = (n + kRoundBlock - 1) / kRoundBlock;
  int64_t grid = (int64_t)ctx->num_sms * occ;
  if (want < grid) grid = want < 1 ? 1 : want;
  void *args[] = {&A};
  HEC_CUDA_TRY(cudaLaunchCooperativeKernel((const void *)k_rounds, dim3((unsigned)grid),
                                           dim3(kRoundBlock), args, 0, s));
  ctx->launches++;
  phase_end(ctx, ph);
  ph = phase_begin(ctx, "relabel", 9.0 * dn);
  // a4: labels by ascending root id; a5: inherit along H
  HEC_TRY(chained_scan(ctx, n, RootFlagIn{status}, RootLabelOut{status, lab, root_out}, st, scal, true));
  int *long_chain = reinterpret_cast<int *>(scal + 2);
  if (u1 > u0) {  // wl0 is free after the rounds: jump targets of cut walks
    k_assign<<<nblk(u1 - u0, 256), 256, 0, s>>>(u0, u1, H, status, lab, M, wl0, long_chain);
    HEC_LAUNCH_CHECK();
  }
  int64_t h[3];
  HEC_TRY(read_scalars(ctx, scal, 3, h));
  if ((int32_t)(h[2] & 0xffffffff)) {  // some H-chain is longer than kAssignWalk
    k_jump_init<<<nblk(n, 256), 256, 0, s>>>(n, H, status, wl0);
    HEC_LAUNCH_CHECK();
    for (int64_t reach = 1; reach < n; reach *= 2) {
      k_jump<<<nblk(n, 256), 256, 0, s>>>(n, status, wl0);
      HEC_LAUNCH_CHECK();
    }
    k_assign_jumped<<<nblk(u1 - u0, 256), 256, 0, s>>>(u0, u1, status, wl0, lab, M);
    HEC_LAUNCH_CHECK();
  }
  phase_end(ctx, ph);
  res->n_c = h[0];
  res->rounds = (int)(int32_t)(h[1] & 0xffffffff);
  return HEC_OK;
}

// H from the heavy keys the previous level's placement left (k_place): the
// row maximum of w << 32 | ~v, 0 for an empty row (-> itself)
__global__ void k_hkey_to_H(int64_t n, const unsigned long long *__restrict__ hk, int32_t *__restrict__ H) {
  const int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (u >= n) return;
  const unsigned long long k = hk[u];
  H[u] = k ? key_vertex(k) : (int32_t)u;
}

int find_mapping_impl(hec_ctx *ctx, const hec_graph *g, Prio prio, int32_t *M, uint8_t *root_out,
                      int32_t *H_out, MapResult *res) {
  const int64_t n = g->n;
  res->n_c = 0;
  res->rounds = 0;
  if (n == 0) return HEC_OK;
  int32_t *H = H_out ? H_out : ws_take<int32_t>(ctx, n);
  if (!H) { set_error("workspace under-reserved (mapping)"); return HEC_EINVAL; }
  const double dn = (double)n, dnnz = (double)g->nnz;
  if (ctx->hk_map && ctx->hk_map_col == g->col && ctx->hk_map_n == n) {
    int ph = phase_begin(ctx, "heavy", 20.0 * dn);  // keys (8 B) in, H out; computed with the placement of g
    k_hkey_to_H<<<nblk(n, 256), 256, 0, ctx->stream>>>(n, ctx->hk_map, H);
    HEC_LAUNCH_CHECK();
    phase_end(ctx, ph);
  } else {
    int ph = phase_begin(ctx, "heavy", 8.0 * dnnz + 8.0 * (dn + 1) + 4.0 * dn);
    ctx->unit_flag_armed = false;
    HEC_TRY(run_heavy(ctx, g, H));
    phase_end(ctx, ph);
  }
  const bool armed = ctx->unit_flag_armed;
  ctx->unit_flag_armed = false;
  HEC_TRY(resolve_impl(ctx, g, H, prio, 0, n, M, root_out, res));
  // (resolve_impl's host read synchronised the stream: the span kernel's flag is final)
  res->unit_weights = armed && *reinterpret_cast<volatile int *>(ctx->h_pinned + 63) == 0;
  return HEC_OK;
}

int heavy_range_impl(hec_ctx *ctx, const hec_graph *g, int64_t u0, int64_t u1, int32_t *H) {
  int ph = phase_begin(ctx, "heavy", 0);
  int rc = run_heavy(ctx, g, H, u0, u1);
  phase_end(ctx, ph);
  return rc;
}

int mapping_from_heavy_impl(hec_ctx *ctx, const hec_graph *g, const int32_t *H, Prio prio, int64_t u0,
                            int64_t u1, int32_t *M, MapResult *res) {
  res->n_c = 0;
  res->rounds = 0;
  if (g->n == 0) return HEC_OK;
  return resolve_impl(ctx, g, H, prio, u0, u1, M, nullptr, res);
}

}  // namespace hec
