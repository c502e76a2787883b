// construct_hrank.cu — ordered duplicate merge by shared-memory hash + key-range
// bucket rank, several CTAs per SM (PAPER.md:L319-324
// DEDUPWITHWTS: "deduplicate ... and sum the weights", L280: self loops omitted).
//
// Consumes the same items as k_rbm (construct_rbm.cu): one coarse row with
// kPieceMax < U <= kRbmRow read from the expansion staging, or one key-range
// bin of a partitioned row; keys lie in [lo, hi).  For an item of n <= NT*8
// entries (all held in registers) the CTA
//   1. merges duplicates in a shared-memory hash table (CAS on the key, add on
//      the weight; the inserting entry "owns" the distinct key) -- the hash
//      half of the paper's hash-vs-sort dedup, on B200's fast smem atomics;
//   2. counts the distinct keys per order-preserving key-range bucket
//      (bucket = floor((b - lo) * NB / (hi - lo)), NB >= n buckets, so a bucket
//      holds ~1 key) and scans the counts; owners place key and sum in bucket
//      order;
//   3. thread t takes bucket-order positions t, t + NT, ...: the key's rank is
//      its bucket offset plus the keys of its bucket below it (neighbouring
//      lanes share buckets), i.e. its position in the sorted row, so no sorting
//      pass runs; (b, sum) is written at the rank, in place over the item's own
//      input range.
// Work is O(n) per item with four CTA barriers; several CTAs per SM overlap
// them.  Items with n > NT*8 entries are left to k_hrank_big / k_rbm.
#include "construct_common.cuh"

namespace hec {

// bucket counters / offsets are indexed through hr_p: one pad word per 32 so
// that the scan's per-thread runs (stride 1, 2, 4 or 8 words) are bank-conflict
// free
__device__ __forceinline__ int hr_p(int j) { return j + (j >> 5); }

template <int NT, int PER = 8>
struct HrSmem {
  static constexpr int kCapE = NT * PER;     // entries per item
  static constexpr int kSlots = 2 * kCapE;   // hash slots (load <= 1/2)
  static constexpr int kNB = kCapE;          // buckets at most
  static constexpr int kCntN = kNB + kNB / 32 + 2;
  int32_t key[kSlots];
  uint32_t val[kSlots];
  int32_t cnt[kCntN];                        // bucket counts (zeroed by the scan), hr_p-indexed
  uint16_t offs[kCntN + 2];                  // bucket offsets (<= kCapE), hr_p-indexed
  int32_t scr[kCapE];                        // distinct keys in bucket order
  int32_t wsum[NT / 32 + 1];
  int32_t nd;                                // distinct keys of the item
};

__device__ __forceinline__ uint32_t hr_hash(int32_t b) { return (uint32_t)b * 0x9E3779B1u; }

// Block exclusive scan of c[0..nb) into o[0..nb] (nb <= NT * 8), zeroing c;
// returns the total.
template <int NT, int PER = 8>
__device__ __forceinline__ int hr_scan(int32_t *c, uint16_t *o, int nb, int32_t *wsum) {
  const int t = threadIdx.x, lane = t & 31, wid = t >> 5;
  const int per = (nb + NT - 1) / NT;
  const int beg = t * per;
  int v[PER];
  int local = 0;
#pragma unroll
  for (int i = 0; i < PER; ++i) {
    v[i] = 0;
    if (i < per && beg + i < nb) { v[i] = c[hr_p(beg + i)]; c[hr_p(beg + i)] = 0; }
    local += v[i];
  }
  int x = local;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) wsum[wid] = x;
  __syncthreads();
  int before = 0, total = 0;
#pragma unroll
  for (int w = 0; w < NT / 32; ++w) {
    const int s = wsum[w];
    before += w < wid ? s : 0;
    total += s;
  }
  int run = before + x - local;
#pragma unroll
  for (int i = 0; i < PER; ++i) {
    if (i < per && beg + i < nb) o[hr_p(beg + i)] = (uint16_t)run;
    run += v[i];
  }
  if (t == NT - 1) o[hr_p(nb)] = (uint16_t)total;
  return total;
}

template <int NT, int PER = 8>
__global__ void __launch_bounds__(NT, PER == 8 ? (NT == 128 ? 9 : 1024 / NT) : (NT == 32 ? 32 : 4)) k_hrank(RowsArgs A) {
  constexpr int kCapE = HrSmem<NT, PER>::kCapE;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  HrSmem<NT, PER> &S = *reinterpret_cast<HrSmem<NT, PER> *>(smem_raw);
  const int t = threadIdx.x;
  const int64_t nitems = *A.nlist;
  // kernel-argument pointers held in registers (not re-read per slot)
  int32_t *const scb = A.sc_col, *const scw = A.sc_wgt, *const pbg = A.pb_g, *const pwg = A.pw_g;
  int *const err = A.err;
  for (int i = t; i < HrSmem<NT, PER>::kSlots; i += NT) { S.key[i] = kEmpty; S.val[i] = 0u; }
  for (int i = t; i < HrSmem<NT, PER>::kCntN; i += NT) S.cnt[i] = 0;
  if (t == 0) S.nd = 0;
  __syncthreads();
  RbmItem nx{};
  if (blockIdx.x < nitems) nx = rbm_at(A.ritems, A.rdir, A.rcap, blockIdx.x);
  for (int64_t ii = blockIdx.x; ii < nitems; ii += gridDim.x) {
    const RbmItem it = nx;  // descriptor prefetched one item ahead
    if (ii + gridDim.x < nitems) nx = rbm_at(A.ritems, A.rdir, A.rcap, ii + gridDim.x);
    const int n = it.n;
    const int32_t a = it.row, lo = it.lo;
    int32_t *const src_b = (it.bk < 0 ? scb : pbg) + it.src;
    int32_t *const src_w = (it.bk < 0 ? scw : pwg) + it.src;
    // table geometry: NB buckets (power of two >= n), 2 NB hash slots
    const int lg = (n <= 1 ? 0 : 32 - __clz(n - 1));
    const int NB = 1 << lg;
    const uint32_t hmask = 2u * NB - 1u;
    const int hshift = 31 - lg;  // top lg + 1 bits of the hash
    // any positive scale keeps the buckets monotone in b (approximate division)
    const float scale = __fdividef((float)NB, (float)(it.hi - lo));
    int32_t kb[PER], kw[PER];
#pragma unroll
    for (int k = 0; k < PER; ++k) {
      const int i = t + NT * k;
      kb[k] = -1;
      kw[k] = 0;
      if (i < n) { kb[k] = __ldcs(src_b + i); kw[k] = __ldcs(src_w + i); }
    }
    // ---- 1. hash merge; owners count their bucket (keys lie in [lo, hi) by
    // construction of the items: whole rows span [0, n_c), bins their range)
    bool wrap = false;
    int slot[PER], bpos[PER];
    unsigned own = 0;
#pragma unroll
    for (int k = 0; k < PER; ++k) {
      if (kb[k] == a) kb[k] = -1;  // self entry (L280)
      if (kb[k] < 0) continue;
      uint32_t h = (hr_hash(kb[k]) >> hshift) & hmask;
      while (true) {
        const int32_t old = atomicCAS(&S.key[h], kEmpty, kb[k]);
        if (old == kEmpty) { own |= 1u << k; break; }
        if (old == kb[k]) break;
        h = (h + 1) & hmask;
      }
      slot[k] = (int)h;
      const uint32_t o = atomicAdd(&S.val[h], (uint32_t)kw[k]);
      wrap |= o + (uint32_t)kw[k] < o;
      if (own & (1u << k)) {
        int bk = (int)__fmul_rz((float)(kb[k] - lo), scale);
        bk = bk < NB - 1 ? bk : NB - 1;
        bpos[k] = atomicAdd(&S.cnt[hr_p(bk)], 1);
        slot[k] |= bk << 16;  // slot < 2^14, bucket < 2^13
      }
    }
    if (wrap) atomicOr(err, ERR_OVERFLOW);
    __syncthreads();
    // ---- 2. bucket offsets; owners place their key in bucket order
    const int D = hr_scan<NT, PER>(S.cnt, S.offs, NB, S.wsum);
    __syncthreads();
    // owners place their key in bucket order (scr) and its sum at the same
    // position of the (zeroed) counter array, and free their slot
#pragma unroll
    for (int k = 0; k < PER; ++k) {
      if (!(own & (1u << k))) continue;
      const int h = slot[k] & 0xffff;
      const int pos = S.offs[hr_p(slot[k] >> 16)] + bpos[k];
      S.scr[pos] = kb[k];
      S.cnt[hr_p(pos)] = (int32_t)S.val[h];
      S.key[h] = kEmpty;
      S.val[h] = 0u;
    }
    __syncthreads();
    // ---- 3. thread t ranks the keys at bucket-order positions t, t + NT, ...:
    // rank = bucket offset + keys of the bucket below it (neighbouring lanes
    // share buckets: broadcast reads), written at the rank (near-coalesced);
    // the sums are taken from the counter array, which is zeroed again
    const float bscale = scale;
    bool over = false;
    for (int i = t; i < D; i += NT) {
      const int32_t key = S.scr[i];
      const uint32_t sum = (uint32_t)S.cnt[hr_p(i)];
      S.cnt[hr_p(i)] = 0;
      int bk = (int)__fmul_rz((float)(key - lo), bscale);
      bk = bk < NB - 1 ? bk : NB - 1;
      const int o0 = S.offs[hr_p(bk)], o1 = S.offs[hr_p(bk + 1)];
      int r = o0;
      for (int j = o0; j < o1; ++j) r += S.scr[j] < key;
      over |= sum > 0x7fffffffu;
      src_b[r] = key;
      src_w[r] = (int32_t)sum;
    }
    if (over) atomicOr(err, ERR_OVERFLOW);
    if (t == 0) A.blk_cnt[it.bi] = D;
    __syncthreads();
  }
}

// Items above NT*8 entries (rank class 3): the entries are merged into the hash
// table round by round (NT*8 per round); the distinct keys are then taken from
// the table itself (sweep: bucket counts, scan, placement in bucket order,
// rank).  An item whose distinct keys would push the table past 3/8 load is
// abandoned (its slots cleared) and appended to the redo list for k_rbm.
template <int NT>
__global__ void __launch_bounds__(NT, 1024 / NT) k_hrank_big(RowsArgs A, RbmItem *__restrict__ redo,
                                                          unsigned *__restrict__ nredo) {
  constexpr int kCapE = HrSmem<NT>::kCapE;
  constexpr int kSlots = HrSmem<NT>::kSlots;
  constexpr int kMaxD = (3 * kSlots) / 8;  // abandon threshold (in-flight inserts stay below kSlots)
  static_assert(kMaxD + kCapE < kSlots, "probe loops must terminate");
  extern __shared__ __align__(16) unsigned char smem_raw[];
  HrSmem<NT> &S = *reinterpret_cast<HrSmem<NT> *>(smem_raw);
  const int t = threadIdx.x;
  const int64_t nitems = *A.nlist;
  for (int i = t; i < kSlots; i += NT) { S.key[i] = kEmpty; S.val[i] = 0u; }
  for (int i = t; i < HrSmem<NT>::kCntN; i += NT) S.cnt[i] = 0;
  if (t == 0) S.nd = 0;
  __syncthreads();
  for (int64_t ii = blockIdx.x; ii < nitems; ii += gridDim.x) {
    const RbmItem it = rbm_at(A.ritems, A.rdir, A.rcap, ii);
    const int32_t a = it.row, lo = it.lo;
    int32_t *src_b = (it.bk < 0 ? A.sc_col : A.pb_g) + it.src;
    int32_t *src_w = (it.bk < 0 ? A.sc_wgt : A.pw_g) + it.src;
    const uint32_t hmask = kSlots - 1u;
    constexpr int kLg = 31 - __builtin_ctz(kSlots);  // hash shift: top log2(kSlots) bits
    bool bad = false, wrap = false, full = false;
    for (int64_t r0 = 0; r0 < it.n && !full; r0 += kCapE) {
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        const int64_t i = r0 + t + NT * k;
        int32_t b = -1, w = 0;
        if (i < it.n) { b = __ldcs(src_b + i); w = __ldcs(src_w + i); }
        if (b == a) b = -1;  // self entry (L280)
        if (b < 0) continue;
        if (b < lo || b >= it.hi) { bad = true; continue; }
        uint32_t h = (hr_hash(b) >> kLg) & hmask;
        bool placed = true;
        while (true) {
          const int32_t old = S.key[h];
          if (old == b) break;
          if (old == kEmpty) {
            if (*(volatile int32_t *)&S.nd >= kMaxD) { placed = false; break; }
            const int32_t o2 = atomicCAS(&S.key[h], kEmpty, b);
            if (o2 == kEmpty) { atomicAdd(&S.nd, 1); break; }
            if (o2 == b) break;
          }
          h = (h + 1) & hmask;
        }
        if (!placed) continue;
        const uint32_t o = atomicAdd(&S.val[h], (uint32_t)w);
        wrap |= o + (uint32_t)w < o;
      }
      __syncthreads();
      full = S.nd >= kMaxD;
      __syncthreads();
    }
    if (bad) atomicOr(A.err, ERR_INTERNAL);
    if (full) {  // too many distinct keys: clear, hand the item to k_rbm
      for (int i = t; i < kSlots; i += NT) { S.key[i] = kEmpty; S.val[i] = 0u; }
      if (t == 0) {
        redo[atomicAdd(nredo, 1u)] = it;
        S.nd = 0;
      }
      __syncthreads();
      continue;
    }
    if (wrap) atomicOr(A.err, ERR_OVERFLOW);
    // ---- distinct keys from the table: bucket counts
    const int D = S.nd;
    int lgb = D <= 1 ? 0 : 32 - __clz(D - 1);
    const int NB = 1 << lgb;  // <= kCapE
    const float scale = (float)NB / (float)(it.hi - lo);
    for (int sl = t; sl < kSlots; sl += NT) {
      const int32_t b = S.key[sl];
      if (b == kEmpty) continue;
      int bk = (int)__fmul_rz((float)(b - lo), scale);
      bk = bk < NB - 1 ? bk : NB - 1;
      atomicAdd(&S.cnt[hr_p(bk)], 1);
    }
    __syncthreads();
    hr_scan<NT>(S.cnt, S.offs, NB, S.wsum);  // counts zeroed, offsets in offs
    __syncthreads();
    for (int sl = t; sl < kSlots; sl += NT) {  // place keys in bucket order (cnt reused as cursors)
      const int32_t b = S.key[sl];
      if (b == kEmpty) continue;
      int bk = (int)__fmul_rz((float)(b - lo), scale);
      bk = bk < NB - 1 ? bk : NB - 1;
      S.scr[S.offs[hr_p(bk)] + atomicAdd(&S.cnt[hr_p(bk)], 1)] = b;
    }
    __syncthreads();
    for (int sl = t; sl < kSlots; sl += NT) {
      const int32_t b = S.key[sl];
      if (b == kEmpty) continue;
      int bk = (int)__fmul_rz((float)(b - lo), scale);
      bk = bk < NB - 1 ? bk : NB - 1;
      int r = S.offs[hr_p(bk)];
      for (int j = S.offs[hr_p(bk)]; j < S.offs[hr_p(bk + 1)]; ++j) r += S.scr[j] < b;
      const uint32_t sum = S.val[sl];
      if (sum > 0x7fffffffu) atomicOr(A.err, ERR_OVERFLOW);
      src_b[r] = b;
      src_w[r] = (int32_t)sum;
    }
    __syncthreads();
    for (int sl = t; sl < kSlots; sl += NT) { S.key[sl] = kEmpty; S.val[sl] = 0u; }
    for (int i = t; i < NB; i += NT) S.cnt[hr_p(i)] = 0;
    if (t == 0) {
      A.blk_cnt[it.bi] = D;
      S.nd = 0;
    }
    __syncthreads();
  }
}

int launch_hrank_big(hec_ctx *ctx, const RowsArgs &A, RbmItem *redo, unsigned *nredo) {
  constexpr int NT = 512;
  const size_t smem = sizeof(HrSmem<NT>);
  int occ = 1;
  HEC_TRY(kernel_occupancy(ctx, k_hrank_big<NT>, NT, smem, &occ));
  int64_t grid = (int64_t)ctx->num_sms * 2;
  if (A.nblocks < grid) grid = A.nblocks;
  if (grid < 1) return HEC_OK;
  k_hrank_big<NT><<<(unsigned)grid, NT, smem, ctx->stream>>>(A, redo, nredo);
  HEC_LAUNCH_CHECK();
  return HEC_OK;
}

// Bins whose key range is at most kDirectR keys (bins of the largest skewed
// rows): the range itself is the table.  Every entry adds its weight at
// b - lo (one shared-memory atomic, no probing); a scan over the range's
// non-zero counters then gives every distinct key its rank, and each thread
// writes its slice of keys in order -- already sorted, no hashing, no ranking
// pass.
// Bins above kDrSplit entries (the hub aggregates' bins: on C5 level 1 a few
// of them held most entries, and one CTA per bin left 79% of the SMs idle at
// the tail) are cut into chunks of kDrSplit entries: each chunk accumulates in
// shared memory, adds its non-zero counters to the bin's global accumulator,
// and the chunk that takes the bin's last completion ticket (after a fence)
// sweeps the accumulator and writes the bin -- so no CTA holds more than one
// chunk of work.
constexpr int kDrT = 256;
static_assert(kDirectR == kDrT * 16, "16 counters per thread");

// Ordered sweep of the direct counters c[0 .. R) (shared or global memory):
// warp w takes the 32-counter rows [w Q, (w + 1) Q) (lane = counter within a
// row: conflict-free / coalesced reads), counts the non-zero counters with
// ballots, one CTA scan of the warp counts, then writes (lo + i, c[i]) for the
// non-zero counters in order (contiguous positions per row: coalesced), and
// zeroes them when `clear`.  Returns the number written (D); `wsum` holds
// kDrT / 32 ints; the caller's next barrier protects it.
constexpr int kDrRowSweep = 1024;  // bins with a key range up to this: dr_sweep (cost ~ range)
template <bool kClear>
__device__ __forceinline__ int dr_sweep(uint32_t *c, int R, int32_t lo, int32_t *__restrict__ dst_b,
                                        int32_t *__restrict__ dst_w, int32_t *wsum, bool &over) {
  constexpr int NW = kDrT / 32;
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int rows = (R + 31) >> 5, per = (rows + NW - 1) / NW;
  const int q0 = wid * per, q1 = min(q0 + per, rows);
  int cnt = 0;
  for (int q = q0; q < q1; ++q) {
    const int i = 32 * q + lane;
    const uint32_t v = i < R ? (kClear ? c[i] : __ldcg(c + i)) : 0u;
    cnt += __popc(__ballot_sync(0xffffffffu, v != 0u));
  }
  if (lane == 0) wsum[wid] = cnt;
  __syncthreads();
  int base = 0, D = 0;
#pragma unroll
  for (int w = 0; w < NW; ++w) {
    const int sw = wsum[w];
    base += w < wid ? sw : 0;
    D += sw;
  }
  for (int q = q0; q < q1; ++q) {
    const int i = 32 * q + lane;
    const uint32_t v = i < R ? (kClear ? c[i] : __ldcg(c + i)) : 0u;
    const unsigned m = __ballot_sync(0xffffffffu, v != 0u);
    if (v) {
      const int p = base + __popc(m & ((1u << lane) - 1u));
      over |= v > 0x7fffffffu;
      dst_b[p] = lo + i;
      dst_w[p] = (int32_t)v;
      if (kClear) c[i] = 0u;
    }
    base += __popc(m);
  }
  return D;
}

// chunk items of the split bins (list_d items with n > kDrSplit)
__global__ void k_drank_split(const RbmItem *__restrict__ items, const unsigned *__restrict__ nitems,
                              RbmItem *__restrict__ dc, unsigned *__restrict__ ndc, unsigned *__restrict__ nsplit) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= *nitems) return;
  const RbmItem it = items[i];
  if (it.n <= kDrSplit) return;
  const int nch = (it.n + kDrSplit - 1) / kDrSplit;
  const unsigned base = atomicAdd(ndc, (unsigned)nch);
  const int32_t sidx = (int32_t)atomicAdd(nsplit, 1u);
  for (int c = 0; c < nch; ++c) {
    RbmItem ch = it;
    ch.src = it.src + (int64_t)c * kDrSplit;
    ch.n = min(kDrSplit, it.n - c * kDrSplit);
    ch.hi = c << 16 | nch;
    ch.bk = -2 - sidx;
    dc[base + c] = ch;
  }
}

// p[0 .. *count * scale) = 0
__global__ void k_zero_u32(uint32_t *__restrict__ p, const unsigned *__restrict__ count, int scale) {
  const int64_t n = (int64_t)*count * scale;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    p[i] = 0u;
}

__global__ void __launch_bounds__(kDrT) k_drank(RowsArgs A) {
  __shared__ uint32_t val[kDirectR];
  __shared__ int32_t wsum[kDrT / 32];
  const int t = threadIdx.x, lane = t & 31, wid = t >> 5;
  const int64_t nitems = *A.nlist;
  int32_t *const pbg = A.pb_g, *const pwg = A.pw_g;
  for (int i = t; i < kDirectR; i += kDrT) val[i] = 0u;
  __syncthreads();
  for (int64_t ii = blockIdx.x; ii < nitems; ii += gridDim.x) {
    const RbmItem it = rbm_at(A.ritems, A.rdir, A.rcap, ii);
    if (it.n > kDrSplit) continue;  // split into chunks: k_drank_chunks
    const int32_t a = it.row, lo = it.lo;
    int32_t *const src_b = pbg + it.src;  // bins only (it.bk >= 0)
    int32_t *const src_w = pwg + it.src;
    bool wrap = false;
    for (int64_t r0 = 0; r0 < it.n; r0 += 8 * kDrT) {
      int32_t kb[8], kw[8];
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        const int64_t i = r0 + t + kDrT * k;
        kb[k] = -1;
        kw[k] = 0;
        if (i < it.n) { kb[k] = __ldcs(src_b + i); kw[k] = __ldcs(src_w + i); }
      }
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        if (kb[k] < 0 || kb[k] == a) continue;  // self entry (L280)
        const uint32_t o = atomicAdd(&val[kb[k] - lo], (uint32_t)kw[k]);
        wrap |= o + (uint32_t)kw[k] < o;
      }
    }
    if (wrap) atomicOr(A.err, ERR_OVERFLOW);
    __syncthreads();
    bool over = false;
    int D;
    if (it.hi - lo <= kDrRowSweep) {
      D = dr_sweep<true>(val, it.hi - lo, lo, src_b, src_w, wsum, over);
    } else {  // wide bins: thread t owns counters [16 t, 16 t + 16) (fewer instructions)
      const int R = it.hi - lo;
      uint32_t v[16];
      int c = 0;
      if (16 * t < R) {  // (counters at or past R are never touched: zero)
#pragma unroll
        for (int q = 0; q < 16; ++q) {
          v[q] = val[16 * t + q];
          c += v[q] != 0u;
        }
      } else {
#pragma unroll
        for (int q = 0; q < 16; ++q) v[q] = 0u;
      }
      int x = c;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const int y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
      }
      if (lane == 31) wsum[wid] = x;
      __syncthreads();
      int before = 0;
      D = 0;
#pragma unroll
      for (int w = 0; w < kDrT / 32; ++w) {
        const int sw = wsum[w];
        before += w < wid ? sw : 0;
        D += sw;
      }
      int pos = before + x - c;
#pragma unroll
      for (int q = 0; q < 16; ++q) {
        if (v[q] != 0u) {
          over |= v[q] > 0x7fffffffu;
          src_b[pos] = lo + 16 * t + q;
          src_w[pos] = (int32_t)v[q];
          ++pos;
          val[16 * t + q] = 0u;
        }
      }
    }
    if (over) atomicOr(A.err, ERR_OVERFLOW);
    if (t == 0) A.blk_cnt[it.bi] = D;
    __syncthreads();
  }
}

// Chunks of the split bins (dc): accumulate, add to the bin's accumulator,
// the chunk that takes the bin's last ticket sweeps it and writes the bin.
__global__ void __launch_bounds__(kDrT) k_drank_chunks(RowsArgs A, const RbmItem *__restrict__ dc,
                                                       const unsigned *__restrict__ ndc, uint32_t *__restrict__ gacc,
                                                       unsigned *__restrict__ done) {
  __shared__ uint32_t val[kDirectR];
  __shared__ int32_t wsum[kDrT / 32];
  __shared__ int s_last;
  const int t = threadIdx.x, lane = t & 31, wid = t >> 5;
  const int64_t nitems = *ndc;
  int32_t *const pbg = A.pb_g, *const pwg = A.pw_g;
  for (int i = t; i < kDirectR; i += kDrT) val[i] = 0u;
  __syncthreads();
  for (int64_t ii = blockIdx.x; ii < nitems; ii += gridDim.x) {
    const RbmItem it = dc[ii];
    const int32_t a = it.row, lo = it.lo;
    const int sidx = -2 - it.bk, chunk = it.hi >> 16, nchunk = it.hi & 0xffff;
    const int32_t *const src_b = pbg + it.src, *const src_w = pwg + it.src;
    bool wrap = false;
    for (int64_t r0 = 0; r0 < it.n; r0 += 8 * kDrT) {
      int32_t kb[8], kw[8];
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        const int64_t i = r0 + t + kDrT * k;
        kb[k] = -1;
        kw[k] = 0;
        if (i < it.n) { kb[k] = __ldcs(src_b + i); kw[k] = __ldcs(src_w + i); }
      }
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        if (kb[k] < 0 || kb[k] == a) continue;  // self entry (L280)
        const uint32_t o = atomicAdd(&val[kb[k] - lo], (uint32_t)kw[k]);
        wrap |= o + (uint32_t)kw[k] < o;
      }
    }
    __syncthreads();
    uint32_t *const g = gacc + (int64_t)sidx * kDirectR;
#pragma unroll
    for (int q = 0; q < 16; ++q) {  // counter q kDrT + t: conflict-free, coalesced
      const int i = q * kDrT + t;
      const uint32_t x = val[i];
      if (x) {
        const uint32_t o = atomicAdd(g + i, x);
        wrap |= o + x < o;
        val[i] = 0u;
      }
    }
    if (wrap) atomicOr(A.err, ERR_OVERFLOW);
    __threadfence();
    __syncthreads();
    if (t == 0) s_last = atomicAdd(done + sidx, 1u) == (unsigned)(nchunk - 1);
    __syncthreads();
    if (!s_last) continue;
    __threadfence();
    bool over = false;
    const int64_t out = it.src - (int64_t)chunk * kDrSplit;  // the bin's entries start here
    const int D = dr_sweep<false>(g, kDirectR, lo, pbg + out, pwg + out, wsum, over);
    if (over) atomicOr(A.err, ERR_OVERFLOW);
    if (t == 0) A.blk_cnt[it.bi] = D;
    __syncthreads();
  }
}

int launch_drank(hec_ctx *ctx, const RowsArgs &A, RbmItem *dc, unsigned *ndc, uint32_t *gacc, unsigned *done,
                 unsigned *nsplit) {
  if (A.nblocks < 1) return HEC_OK;
  k_drank_split<<<nblk(A.nblocks + 1, 256), 256, 0, ctx->stream>>>(A.ritems, A.nlist, dc, ndc, nsplit);
  HEC_LAUNCH_CHECK();
  k_zero_u32<<<ctx->num_sms * 4, 256, 0, ctx->stream>>>(gacc, nsplit, kDirectR);
  HEC_LAUNCH_CHECK();
  k_zero_u32<<<ctx->num_sms, 256, 0, ctx->stream>>>(done, nsplit, 1);
  HEC_LAUNCH_CHECK();
  int occ = 1;
  HEC_TRY(kernel_occupancy(ctx, k_drank, kDrT, 0, &occ));
  int64_t grid = (int64_t)ctx->num_sms * occ;
  if (A.nblocks < grid) grid = A.nblocks;
  k_drank<<<(unsigned)grid, kDrT, 0, ctx->stream>>>(A);
  HEC_LAUNCH_CHECK();
  HEC_TRY(kernel_occupancy(ctx, k_drank_chunks, kDrT, 0, &occ));
  grid = (int64_t)ctx->num_sms * occ;
  k_drank_chunks<<<(unsigned)grid, kDrT, 0, ctx->stream>>>(A, dc, ndc, gacc, done);
  HEC_LAUNCH_CHECK();
  return HEC_OK;
}

template <int NT, int PER = 8>
static int launch_hrank_t(hec_ctx *ctx, const RowsArgs &A) {
  const size_t smem = sizeof(HrSmem<NT, PER>);
  int occ = 1;
  HEC_TRY(kernel_occupancy(ctx, k_hrank<NT, PER>, NT, smem, &occ));
  int64_t grid = (int64_t)ctx->num_sms * occ;
  if (A.nblocks < grid) grid = A.nblocks;
  if (grid < 1) return HEC_OK;
  k_hrank<NT, PER><<<(unsigned)grid, NT, smem, ctx->stream>>>(A);
  HEC_LAUNCH_CHECK();
  return HEC_OK;
}

// One size class of items (the list in A.ritems / A.nlist): cls -2, -1, 0, 1, 2 =
// n <= 128, 512, 1024, 2048, 4096 on 32-, 64-, 128-, 256-, 512-thread CTAs.
int launch_hrank(hec_ctx *ctx, const RowsArgs &A, int cls) {
  static_assert(HrSmem<32, 4>::kCapE == kHrMaxT && HrSmem<64>::kCapE == kHrMaxS && HrSmem<128>::kCapE == kHrMax0 && HrSmem<256>::kCapE == kHrMax1 &&
                    HrSmem<512>::kCapE == kHrMax2,
                "size classes");
  if (cls < -1) return launch_hrank_t<32, 4>(ctx, A);  // one warp per item (rows of <= 128 entries)
  if (cls < 0) return launch_hrank_t<64>(ctx, A);  // two warps per item: barriers among 64 threads
  if (cls == 0) return launch_hrank_t<128>(ctx, A);
  if (cls == 1) return launch_hrank_t<256>(ctx, A);  // (<128, 16>: 1.6x slower, measured)
  return launch_hrank_t<512>(ctx, A);
}

}  // namespace hec
