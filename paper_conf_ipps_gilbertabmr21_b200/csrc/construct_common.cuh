// construct_common.cuh — shared pieces of CONSTRUCTCOARSEGRAPH (construct*.cu):
// sizes, the member-edge layout, the warp-level expansion of fine entries into
// (b = M[v], w) register tuples, block descriptors and kernel arguments.
#pragma once
#include "hec_internal.cuh"

namespace hec {

constexpr int kT = 512;            // threads per CTA of the row kernels
constexpr int kIt = 8;             // entries held per thread (registers)
constexpr int kCap = kT * kIt;     // entries per work block (4096)
constexpr int kHash = kCap + kCap / 2 + 8;  // hash slots per work block (regions of 1.5 U + 1)
constexpr int kWin = 2048;         // window weight; a block's weight is < 2*kWin
constexpr int kRowW = 8;           // per-row weight: bounds rows per block
constexpr int kMaxRows = 2 * kWin / kRowW;  // 512
constexpr int kSmallMax = kWin - kRowW;     // rows with U <= 2040 are small
constexpr int kMC = 1024;          // member-table chunk
constexpr int kBucketAvg = 32;     // target entries per key-range bin of a skewed row
constexpr int kGroupWin = 128;     // bins are grouped into pieces by windows of this weight
constexpr int kPieceWin = 64;      // piece window weight (piece weight < 2*kPieceWin; 128 measured
                                   // 2% slower on C2: the 256-slot networks cost more per entry)
constexpr int kPieceMax = kPieceWin - 4;  // rows with U <= kPieceMax (60) go to warp pieces
constexpr int kPieceRowW = 4;      // per-row piece weight
constexpr int kPieceRows = kPieceWin / kPieceRowW;  // rows per piece (all start in one window)
constexpr int kPieceCap = 256;     // entries per warp piece
constexpr int kDenseMax = 32768;   // n_c bound of the DENSE skew path
constexpr int32_t kEmpty = -1;
// Bitmap-rank items (construct_rbm.cu), used in BUCKET mode when n_c <= kRbmRange:
// rows with kPieceMax < U <= kRbmRow are single-row items; larger rows are
// partitioned into bins of ~kRbmBinAvg entries, each bin an item.
constexpr int64_t kRbmRange = 917504;  // keys covered by the shared-memory bitmap
constexpr int kRbmRow = 4096;
constexpr int kRbmBinAvg = 1024;
constexpr int kRbmCap = 4096;          // distinct keys per rank window

enum : int32_t { B_SMALL = 0, B_BUCKET = 1, B_DENSE = 2, B_PIECE = 3, B_RBM = 4 };
__host__ __device__ __forceinline__ bool rows_kind(int32_t k) { return k == B_SMALL || k == B_PIECE; }
enum : int { ERR_LABEL = 1, ERR_OVERFLOW = 2, ERR_WIDE = 4, ERR_INTERNAL = 8 };

inline unsigned nblk(int64_t n, int b) { return (unsigned)((n + b - 1) / b); }

// largest i in [lo, hi) with a[i] <= x (a non-decreasing, a[lo] <= x)
template <typename T>
__device__ __forceinline__ int64_t last_le(const T *a, int64_t lo, int64_t hi, int64_t x) {
  hi -= 1;
  while (lo < hi) {
    int64_t mid = (lo + hi + 1) >> 1;
    if ((int64_t)a[mid] <= x) lo = mid;
    else hi = mid - 1;
  }
  return lo;
}

// In-place exclusive scan of n <= kCap+1 int32 values in shared memory by a CTA
// of kT threads; returns the total.  `tmp` holds >= 33 ints.
__device__ __forceinline__ int smem_exclusive_scan(int32_t *a, int n, int32_t *tmp) {
  const int t = threadIdx.x, lane = t & 31, wid = t >> 5;
  const int chunk = (n + kT - 1) / kT;
  const int beg = t * chunk;
  int local = 0;
  for (int i = 0; i < chunk && beg + i < n; ++i) local += a[beg + i];
  int x = local;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    int y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) tmp[wid] = x;
  __syncthreads();
  if (wid == 0) {
    int w = lane < kT / 32 ? tmp[lane] : 0;
    int ws = w;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      int y = __shfl_up_sync(0xffffffffu, ws, o);
      if (lane >= o) ws += y;
    }
    if (lane < kT / 32) tmp[lane] = ws - w;
    if (lane == kT / 32 - 1) tmp[32] = ws;
  }
  __syncthreads();
  int run = tmp[wid] + x - local;
  for (int i = 0; i < chunk && beg + i < n; ++i) {
    int v = a[beg + i];
    a[beg + i] = run;
    run += v;
  }
  int total = tmp[32];
  __syncthreads();
  return total;
}

// CTA-wide sum of a 64-bit value; `tmp` holds >= kT/32 long longs.
__device__ __forceinline__ long long block_sum64(long long v, long long *tmp) {
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  if (lane == 0) tmp[wid] = v;
  __syncthreads();
  long long s = 0;
  for (int w = 0; w < kT / 32; ++w) s += tmp[w];
  __syncthreads();
  return s;
}

struct Layout {
  int64_t n_c;
  const int64_t *member_ptr;  // [n_c+1]
  const int32_t *members;     // [n]
  const int64_t *mpre;        // [n+1] member-edge prefix
  const int64_t *row_ptr;
  const int32_t *col;
  const int32_t *wgt;
  const int32_t *M;
  int64_t a_lo, a_hi;  // coarse rows produced by this call (range partition, §8(e))
  int64_t bin_avg;     // target entries per key-range bin of a skewed row (rank items)
  bool unit_w = false;  // every weight of the fine graph is 1 (a1's flag): weights not read
  __device__ __forceinline__ bool active(int64_t a) const { return a >= a_lo && a < a_hi; }
  __device__ __forceinline__ int64_t upos(int64_t a) const { return mpre[member_ptr[a]]; }
  __device__ __forceinline__ int64_t U(int64_t a) const { return upos(a + 1) - upos(a); }
};

// Largest member i in [lo, hi) with mpre[i] <= P (mpre[lo] <= P), by a warp:
// 32-ary search, one coalesced probe per round.
__device__ __forceinline__ int64_t warp_find_member(const Layout &L, int64_t lo, int64_t hi, int64_t P) {
  const int lane = threadIdx.x & 31;
  while (hi - lo > 32) {
    const int64_t step = (hi - lo + 31) / 32;
    const int64_t idx = lo + lane * step;
    const bool le = idx < hi && L.mpre[idx] <= P;
    const int k = __popc(__ballot_sync(0xffffffffu, le)) - 1;
    const int64_t nlo = lo + k * step;
    hi = nlo + step < hi ? nlo + step : hi;
    lo = nlo;
  }
  const int64_t idx = lo + lane;
  const bool le = idx < hi && L.mpre[idx] <= P;
  return lo + __popc(__ballot_sync(0xffffffffu, le)) - 1;
}

// ------------------------------------------------------- member walk
constexpr int kXBig = 64;

// Walk the member-edge positions [P, Pend) (all inside members [.., m_hi)):
// sink(e[4], p[4], ok) receives, per step, up to four positions per lane (e:
// source entry in col/wgt, p: position); a sink with kRows also receives the
// coarse row M[member] of each position (sink(e, p, ok, row)).  Members whose coarse row a has
// U(a) > skip_thr (and skip[a] >= 0 when skip != nullptr) are passed over: rows
// that their own kernels walk (rank items, DENSE accumulation, unit partition).
template <int kLong, typename Sink, int kShort = 4, typename IdxT = int64_t>
__device__ __forceinline__ void x2_walk(const Layout &L, const int64_t *__restrict__ mstart, int64_t m_lo,
                                        int64_t m_hi, int64_t P, int64_t Pend, const int32_t *__restrict__ skip,
                                        Sink &sink, int64_t skip_thr = INT64_MAX) {
  const int lane = threadIdx.x & 31;
  int64_t i = warp_find_member(L, m_lo, m_hi, P);
  while (true) {
    const int64_t j = i + lane;
    int64_t mp0 = L.mpre[m_hi], mp1 = mp0, rs = 0;
    bool skipped = false;
    int32_t ra = 0;  // the member's coarse row (kRows sinks)
    if (j < m_hi) {
      mp0 = L.mpre[j];
      mp1 = L.mpre[j + 1];
      rs = mstart[j];
      if constexpr (Sink::kRows) ra = L.M[L.members[j]];
      if (skip_thr != INT64_MAX) {
        const int32_t a = L.M[L.members[j]];
        skipped = L.U(a) > skip_thr && (!skip || skip[a] >= 0);
      }
    }
    const int64_t ps = mp0 > P ? mp0 : P;
    const int64_t pe = mp1 < Pend ? mp1 : Pend;
    const int d = (pe > ps && !skipped) ? (int)(pe - ps) : 0;
    rs += ps - mp0;  // source entry of position ps
    const bool big = d > kXBig;
    // ---- packed short members
    const int ds = big ? 0 : d;
    int incl = ds;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int y = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= o) incl += y;
    }
    const int excl = incl - ds;
    const int T = __shfl_sync(0xffffffffu, incl, 31);
    for (int base = 0; base < T; base += 32 * kShort) {
      IdxT e[kShort], p[kShort];
      int32_t rw[kShort];
      unsigned ok = 0;
#pragma unroll
      for (int u = 0; u < kShort; ++u) {
        const int t = base + lane + 32 * u;
        int lo = 0;  // largest lane with excl <= t
#pragma unroll
        for (int st = 16; st > 0; st >>= 1) {
          const int c = lo + st;
          const int v = __shfl_sync(0xffffffffu, excl, c & 31);
          if (c < 32 && v <= t) lo = c;
        }
        const int64_t ors = __shfl_sync(0xffffffffu, rs, lo);
        const int64_t ops = __shfl_sync(0xffffffffu, ps, lo);
        const int oex = __shfl_sync(0xffffffffu, excl, lo);
        e[u] = (IdxT)(ors + (t - oex));
        p[u] = (IdxT)(ops + (t - oex));
        if constexpr (Sink::kRows) rw[u] = __shfl_sync(0xffffffffu, ra, lo);
        if (t < T) ok |= 1u << u;
      }
      if constexpr (Sink::kRows) sink(e, p, ok, rw);
      else sink(e, p, ok);
    }
    // ---- long members, one at a time
    unsigned bm = __ballot_sync(0xffffffffu, big);
    while (bm) {
      const int src = __ffs(bm) - 1;
      bm &= bm - 1;
      const int bd = __shfl_sync(0xffffffffu, d, src);
      const int64_t brs = __shfl_sync(0xffffffffu, rs, src);
      const int64_t bps = __shfl_sync(0xffffffffu, ps, src);
      const int32_t bra = __shfl_sync(0xffffffffu, ra, src);
      for (int base = 0; base < bd; base += 32 * kLong) {  // kLong positions per lane in flight
        IdxT e[kLong], p[kLong];
        int32_t rw[kLong];
        unsigned ok = 0;
#pragma unroll
        for (int u = 0; u < kLong; ++u) {
          const int t = base + lane + 32 * u;
          e[u] = (IdxT)(brs + t);
          p[u] = (IdxT)(bps + t);
          rw[u] = bra;
          if (t < bd) ok |= 1u << u;
        }
        if constexpr (Sink::kRows) sink(e, p, ok, rw);
        else sink(e, p, ok);
      }
    }
    // the window reaches the chunk end (or the last member): done
    if (__any_sync(0xffffffffu, mp1 >= Pend)) break;
    i += 32;
  }
}


// A warp-tier work item, self-contained so a warp goes straight to its data:
// entries [base, base + n) of the staging (PIECE: sc_col/sc_wgt) or of the
// partitioned pairs (bin group: pb_g/pw_g); R > 0 rows starting at row0.
struct WorkItem {
  int64_t base;
  int32_t bi;  // block index (count, flags)
  int32_t n;
  int32_t row0;
  int32_t R;
};

// Size classes of the rank items (k_tiers): n <= 1024, <= 2048, <= 4096 go to
// k_hrank<128/256/512> (construct_hrank.cu), larger ones to k_rbm.
constexpr int kHrMaxT = 128, kHrMaxS = 512, kHrMax0 = 1024, kHrMax1 = 2048, kHrMax2 = 4096;
constexpr int kDirectR = 4096;  // bins with a key range this small: direct-indexed counters (k_drank)

// A bitmap-rank item (construct_rbm.cu), self-contained so a CTA prefetches it:
// entries [src, src + n) of sc_col/sc_wgt (B_RBM whole row) or pb_g/pw_g (bin),
// keys in [lo, hi); row = the coarse row (its self entries are dropped).
// Chunk c of nchunk of a split direct-indexed bin (k_drank) reuses the fields
// k_drank does not read: bk = -2 - s (s: the split bin's index; its counters
// accumulate at gacc[s kDirectR ...), its completion ticket is done[s]) and
// hi = c << 16 | nchunk.
struct RbmItem {
  int64_t src;
  int32_t n, row, lo, hi, bi, bk;  // bk: bin index (-1 for a whole row, <= -2 for a drank chunk)
};

// smallest b in [0, n_c] whose partition bin floor(b * nb / n_c) (float, clamped
// to nb - 1 -- the exact function k_part_* use) is >= k
__device__ __forceinline__ int64_t bin_lower(int64_t k, int64_t nb, int64_t n_c) {
  if (k <= 0) return 0;
  if (k >= nb) return n_c;
  const float scale = (float)nb / (float)n_c;
  int64_t lo = 0, hi = n_c;
  while (lo < hi) {
    const int64_t mid = (lo + hi) >> 1;
    int bk = (int)__fmul_rz((float)mid, scale);
    bk = bk < nb - 1 ? bk : (int)(nb - 1);
    if (bk >= k) hi = mid;
    else lo = mid + 1;
  }
  return lo;
}

__device__ __forceinline__ RbmItem rbm_at(const RbmItem *items, int dir, int64_t cap, int64_t i) {
  return items[dir > 0 ? i : cap - 1 - i];
}

struct BlockDesc {
  int32_t kind;
  int32_t row0;  // first row (SMALL) / the row (BUCKET, DENSE)
  int32_t row1;  // one past the last row (SMALL)
  int32_t sub;   // bucket index within the row / dense key chunk
};

// Arguments of the work-block kernels (construct_rows.cu).  Each block leaves
// its sorted distinct (b, w) in a staging place that depends on its kind:
//   SMALL   sc_col/sc_wgt at the block's first member-edge position
//   BUCKET  in place over its partitioned pairs pb_g/pw_g
//   DENSE   interleaved (b, w) int32 pairs over its chunk of the dense row
//   fallback buckets: fb_b/fb_w (written by k_bucket_fallback)
// and its count in blk_cnt; row_ptr_c holds row offsets relative to the block.
// An exclusive scan of blk_cnt then gives every block's output offset and
// k_place copies the staged entries into the final CSR (coalesced).
struct RowsArgs {
  Layout L;
  const BlockDesc *blk;
  int64_t nblocks;
  unsigned *ticket;
  int32_t *blk_cnt;                 // [nblocks] distinct entries per block
  int32_t *need_wide;               // [nblocks] 1: redo with 64-bit sums (zeroed)
  const int64_t *blk_off;           // [nblocks+1] exclusive scan of blk_cnt (k_place)
  const unsigned long long *vw64;
  const int32_t *big_idx;
  int32_t *sc_col, *sc_wgt;         // SMALL staging, member-edge space [nnz]
  // BUCKET mode
  const int64_t *bkt_ptr;           // [nbig+1] first bucket of big row h
  const int64_t *bkt_off;           // [nbkt+1] pair offsets (bin start in pb_g/pw_g)
  const unsigned *bkt_n;            // [nbkt] pairs per bin (a row's bins are contiguous)
  const int64_t *grp_end;           // [nblocks] BUCKET group: one past its last bin (k_tiers)
  int32_t *pb_g, *pw_g;             // partitioned pairs (sorted uniques written back in place)
  const int32_t *fb_cnt;            // fallback unique count per bucket (-1: not overflowed)
  const int64_t *fb_off;            // fallback scratch offset per bucket
  const int32_t *fb_b, *fb_w;
  // bitmap-rank items with several rank windows stage to the fallback scratch
  unsigned long long *fb_total;
  int64_t *fb_off_w;
  int32_t *fb_cnt_w, *fb_b_w, *fb_w_w;
  // DENSE mode
  unsigned long long *dense;        // [nbig][n_c] sums, then staged pairs
  // outputs (row-indexed outputs start at row L.a_lo)
  int64_t *row_ptr_c;
  int32_t *col_c, *wgt_c, *vwgt_c;
  int *err;
  const int64_t *mstart;  // row_ptr[members[i]]: rank items walk their member rows (x2_walk)
  bool idx32;             // entry / position indices of the walks fit 32 bits (nnz < 2^32)
  const int32_t *list;    // blocks of this launch (a tier list)
  const WorkItem *items;  // warp tier: the same, as work items
  const RbmItem *ritems;  // bitmap-rank / hash-rank tier (one size class per launch)
  int32_t rdir;           // +1: items ritems[0 .. n); -1: ritems[rcap - 1], ritems[rcap - 2], ...
  int64_t rcap;
  const unsigned *nlist;  // device count of `list` / `items`
  // k_place only: max packed key (w << 32 | ~b) per coarse row a at hkey[a - a_lo]
  // (zeroed; the next level's heavy neighbours, Alg 3 l.6-10), or nullptr
  unsigned long long *hkey;
};

// Work-block kernel and placement launchers (construct_rows.cu).
// Work-block kernels take their blocks from A.list / *A.nlist (device count).
int launch_rows(hec_ctx *ctx, const RowsArgs &A, bool wide);
int launch_pieces(hec_ctx *ctx, const RowsArgs &A, unsigned *ticket);  // construct_pieces.cu
int launch_place(hec_ctx *ctx, const RowsArgs &A, bool *hkey_done = nullptr);
int launch_rbm(hec_ctx *ctx, const RowsArgs &A);  // construct_rbm.cu
int launch_hrank(hec_ctx *ctx, const RowsArgs &A, int cls);  // construct_hrank.cu (cls -2..2: n <= 128/512/1024/2048/4096)
int launch_hrank_big(hec_ctx *ctx, const RowsArgs &A, RbmItem *redo, unsigned *nredo);  // n > 4096

// bins with hi - lo <= kDirectR; bins above kDrSplit entries are cut into chunks
// (list dc, global accumulators gacc / tickets done, sized by drank_split_bound)
constexpr int kDrSplit = 16384;
inline int64_t drank_split_bound(int64_t entries) { return entries / kDrSplit + 1; }  // split bins
int launch_drank(hec_ctx *ctx, const RowsArgs &A, RbmItem *dc, unsigned *ndc, uint32_t *gacc, unsigned *done,
                 unsigned *nsplit);

}  // namespace hec
