// construct_pieces.cu — warp-level work pieces of CONSTRUCTCOARSEGRAPH
// (SURVEY §8 rows a8, a9).  A piece is either a window of consecutive small
// coarse rows (member-edge volume U <= kPieceMax each, < 256 entries in total)
// or one key-range bucket of a partitioned row with <= 256 entries.  One warp
// owns a piece and never waits for other warps:
//
//  1. entries (b, w) — expanded by k_expand / partitioned by k_part_write —
//     are loaded into registers (striped, coalesced); self entries are dropped;
//  2. the packed keys (local row, b) are sorted with a register bitonic network
//     over 64, 128 or 256 slots (shuffles across lanes, register swaps inside a
//     lane) — the sort-based DEDUPWITHWTS that PAPER.md:L324 and Table II find
//     fastest on GPUs, at warp scale and oblivious to the key distribution;
//  3. equal adjacent keys are merged: inclusive prefix sums of w give each run's
//     total (exact: the piece's total weight is checked to fit int32 first);
//  4. the sorted distinct entries are staged in place over the piece's input and
//     its count goes to blk_cnt (k_place moves them to the final CSR later).
// A piece whose total weight exceeds int32 is flagged for the 64-bit CTA pass.
#include <stdlib.h>

#include "construct_common.cuh"

namespace hec {

constexpr int kPW = 8;  // warps per CTA

struct PieceTab {
  uint64_t ukey[kPieceCap];        // key of distinct entry u
  int32_t upre[kPieceCap];         // inclusive weight prefix at the end of run u
  int32_t rstart[kPieceRows + 1];  // row start positions, then first distinct index per row
};

template <typename K>
struct KeyTraits;
template <>
struct KeyTraits<uint32_t> {  // row pieces: (row << 26) | b with b < 2^26; buckets: b
  static constexpr int kShift = 26;
  static constexpr uint32_t kPad = 0xffffffffu;
};
template <>
struct KeyTraits<uint64_t> {  // row pieces: (row << 32) | b
  static constexpr int kShift = 32;
  static constexpr uint64_t kPad = ~0ull;
};

__device__ __forceinline__ uint32_t shfl_xor_k(uint32_t v, int m) { return __shfl_xor_sync(0xffffffffu, v, m); }
__device__ __forceinline__ uint64_t shfl_xor_k(uint64_t v, int m) { return __shfl_xor_sync(0xffffffffu, v, m); }
__device__ __forceinline__ uint32_t shfl_up_k(uint32_t v, int d) { return __shfl_up_sync(0xffffffffu, v, d); }
__device__ __forceinline__ uint64_t shfl_up_k(uint64_t v, int d) { return __shfl_up_sync(0xffffffffu, v, d); }
__device__ __forceinline__ uint32_t shfl_down_k(uint32_t v, int d) { return __shfl_down_sync(0xffffffffu, v, d); }
__device__ __forceinline__ uint64_t shfl_down_k(uint64_t v, int d) { return __shfl_down_sync(0xffffffffu, v, d); }

// Exchange step between lanes (partner lane ^ lm, same register): keep the min
// (keep_min) or the max.  The key is a min/max (one IMNMX for 32-bit keys); the
// value follows when the kept key is the partner's.  Equal keys keep their own
// values on both lanes, so the multiset of (key, value) pairs is preserved.
// (The earlier complement-and-compare form spent 7 ALU operations per
// exchange on the ALU pipe that bounds this kernel; this one spends 3.)
template <int J, typename K>
__device__ __forceinline__ void bitonic_lanes(K (&key)[J], int32_t (&val)[J], int lm, bool keep_min) {
#pragma unroll
  for (int k = 0; k < J; ++k) {
    const K pk = shfl_xor_k(key[k], lm);
    const int32_t pv = __shfl_xor_sync(0xffffffffu, val[k], lm);
    const K nk = keep_min ? (pk < key[k] ? pk : key[k]) : (pk > key[k] ? pk : key[k]);
    if (nk != key[k]) val[k] = pv;
    key[k] = nk;
  }
}

// Exchange step inside a lane: registers k, k | STRIDE; `asc_of(k)` gives the direction.
template <int J, int STRIDE, typename K, typename AscFn>
__device__ __forceinline__ void bitonic_regs(K (&key)[J], int32_t (&val)[J], AscFn asc_of) {
#pragma unroll
  for (int k = 0; k < J; ++k) {
    if (k & STRIDE) continue;
    const int k2 = k | STRIDE;
    const K a = key[k], b = key[k2];
    const K lo = a < b ? a : b, hi = a < b ? b : a;
    const bool asc = asc_of(k);
    const K na = asc ? lo : hi;
    const bool sw = na != a;
    const int32_t va = val[k], vb = val[k2];
    key[k] = na;
    key[k2] = asc ? hi : lo;
    val[k] = sw ? vb : va;
    val[k2] = sw ? va : vb;
  }
}

// All in-lane strides J/2 .. 1 of a merge step whose direction is uniform per lane.
template <int J, typename K>
__device__ __forceinline__ void bitonic_regs_all(K (&key)[J], int32_t (&val)[J], bool asc) {
  auto f = [asc](int) { return asc; };
  if (J >= 16) bitonic_regs<J, (J >= 16 ? 8 : 1)>(key, val, f);
  if (J >= 8) bitonic_regs<J, (J >= 8 ? 4 : 1)>(key, val, f);
  if (J >= 4) bitonic_regs<J, (J >= 4 ? 2 : 1)>(key, val, f);
  bitonic_regs<J, 1>(key, val, f);
}

// Ascending bitonic sort of the 32*J (key, val) pairs of a warp; element
// i = lane*J + k on return (blocked).  Input order is arbitrary.  Sizes up to J
// are unrolled (in-lane); larger sizes run as a compact runtime loop so the
// three piece sizes share little code (the unrolled network overflowed the
// instruction cache).
template <int J, typename K>
__device__ __forceinline__ void warp_bitonic(K (&key)[J], int32_t (&val)[J]) {
  const int lane = threadIdx.x & 31;
  // sizes 2 .. J/2: inside each lane; direction from bit `size` of k
#pragma unroll
  for (int size = 2; size < J; size <<= 1) {
    auto asc_of = [size](int k) { return (k & size) == 0; };
    if (size >= 16) bitonic_regs<J, (J >= 16 ? 8 : 1)>(key, val, asc_of);
    if (size >= 8) bitonic_regs<J, (J >= 8 ? 4 : 1)>(key, val, asc_of);
    if (size >= 4) bitonic_regs<J, (J >= 4 ? 2 : 1)>(key, val, asc_of);
    bitonic_regs<J, 1>(key, val, asc_of);
  }
  // sizes J .. 32J: strides >= J across lanes, then the in-lane strides; the
  // direction (bit `size` of i = lane*J + k) comes from the lane
#pragma unroll 1
  for (int sz = 1; sz <= 32; sz <<= 1) {  // size = sz * J
    const bool asc = (lane & sz) == 0;
#pragma unroll 1
    for (int lm = sz >> 1; lm > 0; lm >>= 1) bitonic_lanes<J, K>(key, val, lm, ((lane & lm) != 0) != asc);
    bitonic_regs_all<J, K>(key, val, asc);
  }
}

// Sort, merge and stage one piece held in registers (padding slots carry kPad).
// R > 0: row piece of R rows (keys carry the local row); R == 0: one bucket.
// Returns the distinct count; row_ptr_rel[r] = first distinct index of row r.
template <int J, typename K>
__device__ __forceinline__ int piece_sort_merge(K (&key)[J], int32_t (&val)[J], PieceTab &S,
                                                int32_t *__restrict__ dst_b, int32_t *__restrict__ dst_w,
                                                int64_t base, int R, int64_t *__restrict__ row_ptr_rel) {
  using KT = KeyTraits<K>;
  const int lane = threadIdx.x & 31;
  warp_bitonic<J, K>(key, val);
  // key before slot 0 (previous lane's last; none for lane 0), key after slot J-1
  K prevk = shfl_up_k(key[J - 1], 1);
  if (lane == 0) prevk = KT::kPad;
  K nextk = shfl_down_k(key[0], 1);
  if (lane == 31) nextk = KT::kPad;
  // inclusive weight prefix and run heads (padding has weight 0 and sorts last)
  int32_t pre[J];
  int run = 0, nh = 0;
#pragma unroll
  for (int k = 0; k < J; ++k) {
    run += val[k];
    pre[k] = run;
    const K pk = k ? key[k - 1] : prevk;
    nh += (key[k] != KT::kPad && pk != key[k]) ? 1 : 0;
  }
  int xs = run, xh = nh;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int ys = __shfl_up_sync(0xffffffffu, xs, o), yh = __shfl_up_sync(0xffffffffu, xh, o);
    if (lane >= o) { xs += ys; xh += yh; }
  }
  const int T = __shfl_sync(0xffffffffu, xh, 31);
  int u = xh - nh;              // distinct entries before this lane's first slot
  const int woff = xs - run;    // weight before this lane's first slot
  if (lane < R) S.rstart[lane] = T;  // rows without distinct entries: fixed below
  __syncwarp();
#pragma unroll
  for (int k = 0; k < J; ++k) {
    if (key[k] == KT::kPad) break;
    const K pk = k ? key[k - 1] : prevk;
    if (pk != key[k]) {  // head of run u
      if (R > 0 && (pk >> KT::kShift) != (key[k] >> KT::kShift)) S.rstart[(int)(key[k] >> KT::kShift)] = u;
      ++u;
    }
    const K nk = k + 1 < J ? key[k + 1] : nextk;
    if (nk != key[k]) {  // tail of run u - 1
      S.ukey[u - 1] = (uint64_t)key[k];
      S.upre[u - 1] = woff + pre[k];
    }
  }
  __syncwarp();
  const uint64_t mask = R > 0 ? (1ull << KT::kShift) - 1 : 0xffffffffull;
  for (int q = lane; q < T; q += 32) {
    dst_b[base + q] = (int32_t)(S.ukey[q] & mask);
    dst_w[base + q] = S.upre[q] - (q ? S.upre[q - 1] : 0);
  }
  if (R > 0) {  // rows without entries start where the next non-empty row starts
    int v = lane < R ? S.rstart[lane] : T;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int y = __shfl_down_sync(0xffffffffu, v, o);
      if (lane + o < 32) v = min(v, y);
    }
    if (lane < R) row_ptr_rel[lane] = v;
  }
  __syncwarp();
  return T;
}

// Load a piece (striped) into J slots per lane, check the int32 bound, sort/merge.
// Returns the distinct count, or -1 when the piece needs 64-bit sums.
template <int J, typename K>
__device__ __forceinline__ int piece_run(int32_t row0, PieceTab &S, int R, int n, int32_t *__restrict__ src_b,
                                         int32_t *__restrict__ src_w, int64_t base, int64_t *row_ptr_rel) {
  using KT = KeyTraits<K>;
  const int lane = threadIdx.x & 31;
  K key[J];
  int32_t val[J];
#pragma unroll
  for (int k = 0; k < J; ++k) {
    const int s = lane + 32 * k;
    key[k] = KT::kPad;
    val[k] = 0;
    if (s < n) {
      const int32_t b = __ldcs(src_b + base + s);
      const int32_t w = __ldcs(src_w + base + s);
      if (R > 0) {
        const int r = (int)last_le(S.rstart, 0, R, s);
        if (b != row0 + r) {  // self entries are dropped (L280)
          key[k] = ((K)r << KT::kShift) | (K)(uint32_t)b;
          val[k] = w;
        }
      } else {
        key[k] = (K)(uint32_t)b;
        val[k] = w;
      }
    }
  }
  __syncwarp();  // rstart is rewritten by piece_sort_merge
  long long wsum = 0;
#pragma unroll
  for (int k = 0; k < J; ++k) wsum += val[k];
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) wsum += __shfl_xor_sync(0xffffffffu, wsum, o);
  if (wsum > 0x7fffffffLL) return -1;
  return piece_sort_merge<J, K>(key, val, S, src_b, src_w, base, R, row_ptr_rel);
}

// ---------------------------------------------------------------------------
// Bin groups with a narrow key range: ordered dedup by bitmap rank, no sort.
// All keys of a group lie in [lo, lo + kGrpBits); a warp-private bitmap marks
// the distinct keys, so the rank of a key in the sorted output is the number of
// set bits before it (per-lane 32-word block totals -> warp scan, per-word
// prefixes inside a block).  Each entry then adds its weight at its rank: the
// duplicate merge of DEDUPWITHWTS with O(entries) work
// instead of a sorting network.  Bitmap words are XOR-swizzled inside their
// 32-word block so the per-lane block walks are bank-conflict free.
// 16K-key bitmaps keep the warp tables at 5 KB, so 4 CTAs of 8 warps fit an SM
// (with the 64-register bound below); 32K-key bitmaps allowed 3 (C2: -0.1 ms)
constexpr int kGrpBits = 16384;
constexpr int kGrpWords = kGrpBits / 32;

struct GroupTab {
  uint32_t bm[kGrpWords];
  uint16_t pref[kGrpWords];   // set bits before the word inside its 32-word block
  int32_t key[kPieceCap];
  int32_t val[kPieceCap];
};
union WarpTab {
  PieceTab p;
  GroupTab g;
};

__device__ __forceinline__ int grp_swz(int wd) { return wd ^ ((wd >> 5) & 31); }

// Entries b[k] >= 0 (padding: -1) with total weight <= INT32_MAX; keys in
// [lo, lo + 32 * nwords).  Writes the sorted distinct (key, summed weight) to
// dst_b/dst_w[base ...] and returns their number.
template <int J>
__device__ __forceinline__ int group_bitmap(const int32_t (&b)[J], const int32_t (&w)[J], int32_t lo, int nwords,
                                            GroupTab &G, int32_t *__restrict__ dst_b, int32_t *__restrict__ dst_w,
                                            int64_t base) {
  const int lane = threadIdx.x & 31;
  const int nblk = (nwords + 31) >> 5;
  for (int i = lane; i < nblk * 32; i += 32) G.bm[i] = 0;
  for (int i = lane; i < kPieceCap; i += 32) G.val[i] = 0;
  __syncwarp();
#pragma unroll
  for (int k = 0; k < J; ++k)
    if (b[k] >= 0) {
      const int o = b[k] - lo;
      atomicOr(&G.bm[grp_swz(o >> 5)], 1u << (o & 31));
    }
  __syncwarp();
  int cnt = 0;
  if (lane < nblk) {
#pragma unroll 8
    for (int i = 0; i < 32; ++i) {
      const int ph = lane * 32 + (i ^ lane);  // grp_swz(lane * 32 + i)
      G.pref[ph] = (uint16_t)cnt;
      cnt += __popc(G.bm[ph]);
    }
  }
  int incl = cnt;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int y = __shfl_up_sync(0xffffffffu, incl, o);
    if (lane >= o) incl += y;
  }
  const int excl = incl - cnt;
  const int T = __shfl_sync(0xffffffffu, incl, 31);
  __syncwarp();
#pragma unroll
  for (int k = 0; k < J; ++k) {
    const bool v = b[k] >= 0;
    const int o = v ? b[k] - lo : 0;
    const int wd = o >> 5;
    const int bb = __shfl_sync(0xffffffffu, excl, wd >> 5);
    if (v) {
      const int ph = grp_swz(wd);
      const int r = bb + G.pref[ph] + __popc(G.bm[ph] & ((1u << (o & 31)) - 1u));
      atomicAdd(&G.val[r], w[k]);
      G.key[r] = b[k];  // every duplicate stores the same key
    }
  }
  __syncwarp();
  for (int q = lane; q < T; q += 32) {
    dst_b[base + q] = G.key[q];
    dst_w[base + q] = G.val[q];
  }
  __syncwarp();
  return T;
}

// Small bin groups (n <= 32 J entries, J <= 2): rank by bit-serial ballots.
// For each own key, eq[s] / less[s] are the lanes whose slot-s key equals /
// is below it on the bits seen so far (most significant first, only the bits
// where the group's keys differ).  Equal keys share a rank among the distinct
// keys, so duplicates merge with one shared-memory atomicAdd at that rank and
// the first copy (lowest slot, then lane) writes (key, sum) -- no sorting
// network.  (A labelled-partition __reduce_add_sync was measured to serialise
// per distinct mask.)
template <int J>
__device__ __forceinline__ int group_ballot(const int32_t (&b)[J], const int32_t (&w)[J], int32_t mn, int32_t mx,
                                            int32_t *__restrict__ val, int32_t *__restrict__ dst_b,
                                            int32_t *__restrict__ dst_w, int64_t base) {
  const int lane = threadIdx.x & 31;
  const unsigned lt = (1u << lane) - 1u;
  unsigned vm[J];
#pragma unroll
  for (int s = 0; s < J; ++s) {
    vm[s] = __ballot_sync(0xffffffffu, b[s] >= 0);
    val[lane + 32 * s] = 0;
  }
  unsigned eq[J][J], less[J][J];
#pragma unroll
  for (int t = 0; t < J; ++t)
#pragma unroll
    for (int s = 0; s < J; ++s) { eq[t][s] = vm[s]; less[t][s] = 0u; }
  const int nbits = 32 - __clz((unsigned)(mx ^ mn));
  for (int i = nbits - 1; i >= 0; --i) {
    unsigned ones[J];
#pragma unroll
    for (int s = 0; s < J; ++s) ones[s] = __ballot_sync(0xffffffffu, (b[s] >> i) & 1);
#pragma unroll
    for (int t = 0; t < J; ++t) {
      const unsigned bt = 0u - (((unsigned)b[t] >> i) & 1u);  // all ones when the bit is set
#pragma unroll
      for (int s = 0; s < J; ++s) {
        less[t][s] |= bt & eq[t][s] & ~ones[s];
        eq[t][s] &= ~(bt ^ ones[s]);
      }
    }
  }
  // first copy of each key: no equal key in a lower slot, none on a lower lane of its slot
  bool lead[J];
  unsigned lm[J];
#pragma unroll
  for (int t = 0; t < J; ++t) {
    bool l = b[t] >= 0 && (eq[t][t] & lt) == 0u;
#pragma unroll
    for (int s = 0; s < t; ++s) l = l && eq[t][s] == 0u;
    lead[t] = l;
  }
#pragma unroll
  for (int s = 0; s < J; ++s) lm[s] = __ballot_sync(0xffffffffu, lead[s]);
  int T = 0, rank[J];
#pragma unroll
  for (int s = 0; s < J; ++s) T += __popc(lm[s]);
  __syncwarp();
#pragma unroll
  for (int t = 0; t < J; ++t) {
    rank[t] = 0;
#pragma unroll
    for (int s = 0; s < J; ++s) rank[t] += __popc(less[t][s] & lm[s]);
    if (b[t] >= 0) atomicAdd(&val[rank[t]], w[t]);
  }
  __syncwarp();
#pragma unroll
  for (int t = 0; t < J; ++t)
    if (lead[t]) {
      dst_b[base + rank[t]] = b[t];
      dst_w[base + rank[t]] = val[rank[t]];
    }
  __syncwarp();
  return T;
}

// A bin group (R == 0): bitmap rank when its key range is narrow, else the
// sorting network.  Returns the distinct count or -1 (needs 64-bit sums).
template <int J>
__device__ __forceinline__ int group_run(WarpTab &S, int n, int32_t *__restrict__ src_b, int32_t *__restrict__ src_w,
                                         int64_t base) {
  const int lane = threadIdx.x & 31;
  int32_t b[J], w[J];
  long long wsum = 0;
  int mn = INT32_MAX, mx = -1;
#pragma unroll
  for (int k = 0; k < J; ++k) {
    const int s = lane + 32 * k;
    b[k] = -1;
    w[k] = 0;
    if (s < n) {
      b[k] = __ldcs(src_b + base + s);
      w[k] = __ldcs(src_w + base + s);
      wsum += w[k];
      mn = min(mn, b[k]);
      mx = max(mx, b[k]);
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    wsum += __shfl_xor_sync(0xffffffffu, wsum, o);
    mn = min(mn, __shfl_xor_sync(0xffffffffu, mn, o));
    mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
  }
  if (wsum > 0x7fffffffLL) return -1;
  if (mx < 0) return 0;
  if constexpr (J <= 2) {
    return group_ballot<J>(b, w, mn, mx, S.g.val, src_b, src_w, base);
  } else if ((int64_t)mx - mn < kGrpBits) {
    return group_bitmap<J>(b, w, mn, ((mx - mn) >> 5) + 1, S.g, src_b, src_w, base);
  }
  uint32_t key[J];
#pragma unroll
  for (int k = 0; k < J; ++k) key[k] = (uint32_t)b[k];  // padding -1 == kPad
  return piece_sort_merge<J, uint32_t>(key, w, S.p, src_b, src_w, base, 0, nullptr);
}

template <int J, bool WIDE_KEYS>
__device__ __forceinline__ int piece_dispatch(int32_t row0, PieceTab &S, int R, int n, int32_t *src_b,
                                              int32_t *src_w, int64_t base, int64_t *rp) {
  if (WIDE_KEYS && R > 0) return piece_run<J, uint64_t>(row0, S, R, n, src_b, src_w, base, rp);
  return piece_run<J, uint32_t>(row0, S, R, n, src_b, src_w, base, rp);
}

template <bool WIDE_KEYS>
__global__ void __launch_bounds__(kPW * 32, 4) k_pieces(RowsArgs A, unsigned *__restrict__ ticket) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  WarpTab &W = reinterpret_cast<WarpTab *>(smem_raw)[wid];
  PieceTab &S = W.p;
  const Layout &L = A.L;
  const int64_t P_lo = L.upos(L.a_lo);
  const int64_t nlist = *A.nlist;
  // items per ticket: 4 (one global atomic per 4 pieces), 1 when the list is
  // short next to the grid (small levels: spread the pieces over all warps)
  const int kBatch = nlist >= 4ll * gridDim.x * kPW ? 4 : 1;
  int64_t item = 0, item_end = 0;
  while (true) {
    if (item == item_end) {
      int64_t t = 0;
      if (lane == 0) t = (int64_t)atomicAdd(ticket, (unsigned)kBatch);
      item = __shfl_sync(0xffffffffu, t, 0) ;
      item_end = item + kBatch < nlist ? item + kBatch : nlist;
      if (item >= nlist) return;
    }
    const WorkItem wi = A.items[item++];
    const int64_t bi = wi.bi;
    const int R = wi.R, n = wi.n;
    const int64_t base = wi.base;  // where the piece's entries are read and its result is staged
    int32_t *src_b, *src_w;
    int64_t *rp = nullptr;
    if (R > 0) {  // PIECE: rows row0 .. row0 + R
      const int64_t P0 = L.upos(wi.row0);
      for (int r = lane; r <= R; r += 32) S.rstart[r] = (int32_t)(L.upos(wi.row0 + r) - P0);
      __syncwarp();
      src_b = A.sc_col;
      src_w = A.sc_wgt;
      rp = A.row_ptr_c + (wi.row0 - L.a_lo);
    } else {  // bin group with <= kPieceCap entries (self entries already dropped)
      src_b = A.pb_g;
      src_w = A.pw_g;
    }
    int T;
    if (R == 0) {
      if (n <= 32) T = group_run<1>(W, n, src_b, src_w, base);
      else if (n <= 64) T = group_run<2>(W, n, src_b, src_w, base);
      else if (n <= 128) T = group_run<4>(W, n, src_b, src_w, base);
      else T = group_run<8>(W, n, src_b, src_w, base);
    } else if (n <= 64) T = piece_dispatch<2, WIDE_KEYS>(wi.row0, S, R, n, src_b, src_w, base, rp);
    else if (n <= 128) T = piece_dispatch<4, WIDE_KEYS>(wi.row0, S, R, n, src_b, src_w, base, rp);
    else T = piece_dispatch<8, WIDE_KEYS>(wi.row0, S, R, n, src_b, src_w, base, rp);
    if (T < 0) {
      if (lane == 0) {
        A.need_wide[bi] = 1;
        atomicOr(A.err, ERR_WIDE);
      }
      continue;
    }
    if (R > 0) {
      for (int r = lane; r < R; r += 32) {
        const int32_t a = wi.row0 + r;
        const unsigned long long s = A.vw64[a];
        if (s > 0x7fffffffull) atomicOr(A.err, ERR_OVERFLOW);
        A.vwgt_c[a - L.a_lo] = (int32_t)s;
      }
    }  // (vertex weights of skewed rows: k_place)
    if (lane == 0) A.blk_cnt[bi] = T;
  }
}

// Persistent: one grid of resident CTAs; the list length is read on the device.
// Keys of row pieces pack (row, b) into 32 bits while n_c <= 2^26.
int launch_pieces(hec_ctx *ctx, const RowsArgs &A, unsigned *ticket) {
  constexpr size_t smem = sizeof(WarpTab) * kPW;
  int occ[2] = {1, 1};
  HEC_TRY(kernel_occupancy(ctx, k_pieces<false>, kPW * 32, smem, &occ[0]));
  HEC_TRY(kernel_occupancy(ctx, k_pieces<true>, kPW * 32, smem, &occ[1]));
  // (HEC_FORCE_WIDE_KEYS: test hook that exercises the 64-bit key path on small graphs)
  const bool wide_keys = A.L.n_c > (1ll << KeyTraits<uint32_t>::kShift) || getenv("HEC_FORCE_WIDE_KEYS") != nullptr;
  int64_t grid = (int64_t)ctx->num_sms * occ[wide_keys ? 1 : 0];
  if (A.nblocks < grid * kPW) grid = (A.nblocks + kPW - 1) / kPW;
  if (grid < 1) return HEC_OK;
  if (wide_keys) k_pieces<true><<<(unsigned)grid, kPW * 32, smem, ctx->stream>>>(A, ticket);
  else k_pieces<false><<<(unsigned)grid, kPW * 32, smem, ctx->stream>>>(A, ticket);
  HEC_LAUNCH_CHECK();
  return HEC_OK;
}

}  // namespace hec
