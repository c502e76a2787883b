// construct_rows.cu — the ordered work-block kernel of CONSTRUCTCOARSEGRAPH
// (SURVEY §8 rows a8, a9 output, a10).
//
// Persistent CTAs take work blocks through a ticket (dynamic balancing):
//  1. entries (b = M[v], w) of the block's rows arrive in registers (expansion of
//     the member rows, or a partitioned bucket of a skewed row);
//  2. per-row shared-memory hash tables (regions of 1.5*U slots) merge duplicate
//     keys — DEDUPWITHWTS's hash variant.  The thread whose CAS
//     created a key owns it from then on;
//  3. owned keys are bucket-sorted per row in shared memory (one bucket per
//     distinct key of the row on average, bucket = scaled key within the row's
//     key range, rank from one smem atomic, insertion sort inside buckets);
//  4. the sorted distinct entries are staged (see RowsArgs), the block's count
//     goes to blk_cnt; after an exclusive scan of the counts, k_place copies
//     every block to its final CSR position (no CTA ever waits for another).
// Sums are exact: int32 accumulators are used only when the block's total
// weight fits in int32; otherwise the block is flagged and the host reruns the
// flagged blocks with the 64-bit (WIDE) instantiation.
#include <type_traits>

#include <stdlib.h>

#include "construct_common.cuh"

namespace hec {

template <bool WIDE>
struct RowsSmemT {
  // phase-aliased areas: [expansion: member table] -> [hash keys] -> [bucket histogram]
  union {
    int32_t hkey[kHash];
    int32_t hist[kCap + 1];
  } a;
  // [hash values] -> [sorted pairs]
  union {
    typename std::conditional<WIDE, unsigned long long, unsigned>::type hval[kHash];
    struct {
      int32_t pb[kCap];
      int32_t pw[kCap];
    } p;
  } v;
  int64_t mptr[kMaxRows + 1];
  int32_t kmin[kMaxRows];
  int32_t kmax[kMaxRows];
  int32_t hbase[kMaxRows + 1];  // hash region offsets
  int32_t ucnt[kMaxRows + 1];   // distinct keys per row -> exclusive offsets
  float bscale[kMaxRows];
  int32_t tmp[40];
  unsigned long long wtot;
  int32_t blk;
};

__device__ __forceinline__ int warp_min(int v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = min(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}
__device__ __forceinline__ int warp_max(int v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = max(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}

// min/max of key over lanes with row r >= 0; one atomic per warp when uniform.
__device__ __forceinline__ void range_update(int32_t *kmin, int32_t *kmax, int r, int32_t key) {
  const int r0 = __shfl_sync(0xffffffffu, r, 0);
  if (__all_sync(0xffffffffu, r == r0)) {
    if (r0 >= 0) {
      int mn = warp_min(key), mx = warp_max(key);
      if ((threadIdx.x & 31) == 0) { atomicMin(kmin + r0, mn); atomicMax(kmax + r0, mx); }
    }
  } else if (r >= 0) {
    atomicMin(kmin + r, key);
    atomicMax(kmax + r, key);
  }
}

// count of lanes with `flag` per row r; one atomic per warp when uniform.
__device__ __forceinline__ void count_update(int32_t *cnt, int r, bool flag) {
  const unsigned m = __ballot_sync(0xffffffffu, flag);
  if (!m) return;
  const int leader = __ffs(m) - 1;
  const int r0 = __shfl_sync(0xffffffffu, r, leader);
  if (__all_sync(0xffffffffu, !flag || r == r0)) {
    if ((int)(threadIdx.x & 31) == leader) atomicAdd(cnt + r0, __popc(m));
  } else if (flag) {
    atomicAdd(cnt + r, 1);
  }
}

template <bool WIDE>
__global__ void __launch_bounds__(kT, 2) k_rows(RowsArgs A) {
  using V = typename std::conditional<WIDE, unsigned long long, unsigned>::type;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  RowsSmemT<WIDE> &S = *reinterpret_cast<RowsSmemT<WIDE> *>(smem_raw);
  int32_t *pb = S.v.p.pb;
  int32_t *pw = S.v.p.pw;
  const int t = threadIdx.x;
  const Layout &L = A.L;
  while (true) {
    if (t == 0) {
      const unsigned it = atomicAdd(A.ticket, 1u);
      S.blk = it < *A.nlist ? A.list[it] : -1;
    }
    __syncthreads();
    const int64_t bi = S.blk;
    if (bi < 0) return;
    const BlockDesc d = A.blk[bi];
    int T = 0, R = 1;
    if (d.kind == B_DENSE) {
      // key chunk [k0, k0 + kCap) of a dense row, already in key order
      const int32_t h = A.big_idx[d.row0];
      const int64_t k0 = (int64_t)d.sub * kCap;
      const unsigned long long *row = A.dense + (int64_t)h * L.n_c;
      unsigned long long v[kIt];
      int c = 0;
#pragma unroll
      for (int k = 0; k < kIt; ++k) {  // blocked: thread t owns keys k0 + t*kIt + k
        const int64_t key = k0 + (int64_t)t * kIt + k;
        v[k] = key < L.n_c ? row[key] : 0ull;
        c += v[k] != 0;
      }
      S.a.hist[t] = c;
      __syncthreads();
      T = smem_exclusive_scan(S.a.hist, kT, S.tmp);
      int pos = S.a.hist[t];
#pragma unroll
      for (int k = 0; k < kIt; ++k) {
        if (v[k] != 0) {
          if (v[k] > 0x7fffffffull) atomicOr(A.err, ERR_OVERFLOW);
          pb[pos] = (int32_t)(k0 + (int64_t)t * kIt + k);
          pw[pos] = (int32_t)v[k];
          ++pos;
        }
      }
    } else {  // (fallback buckets are in no list: their counts come from k_tiers)
      // ---- 1. entries into registers
      int32_t kb[kIt], kw[kIt], kr[kIt];
      if (rows_kind(d.kind)) {
        R = d.row1 - d.row0;
        for (int r = t; r <= R; r += kT) S.mptr[r] = L.upos(d.row0 + r);  // member-edge start of each row
        if (t == 0) S.wtot = 0;
        __syncthreads();
        for (int r = t; r < R; r += kT) {
          S.kmin[r] = INT32_MAX;
          S.kmax[r] = -1;
          S.ucnt[r] = 0;
          const int32_t U = (int32_t)(S.mptr[r + 1] - S.mptr[r]);
          S.hbase[r] = U + (U >> 1) + 1;
        }
        // entries of the block's rows, expanded by k_expand (coalesced)
        const int64_t P0 = S.mptr[0];
        const int nP = (int)(S.mptr[R] - P0);
        const int64_t P_lo = L.upos(L.a_lo);
#pragma unroll
        for (int k = 0; k < kIt; ++k) {
          const int s = t + kT * k;
          kb[k] = -1;
          kw[k] = 0;
          kr[k] = 0;
          if (s < nP) {
            const int32_t b = A.sc_col[P0 + s - P_lo];
            const int r = (int)last_le(S.mptr, 0, R, P0 + s);
            kr[k] = r;
            if (b != d.row0 + r) {  // self entries are dropped (L280)
              kb[k] = b;
              kw[k] = A.sc_wgt[P0 + s - P_lo];
            }
          }
        }
      } else {  // B_BUCKET: partitioned pairs of one skewed row (self entries already dropped)
        const int64_t bk = A.bkt_ptr[A.big_idx[d.row0]] + d.sub;
        const int64_t ge = A.grp_end[bi] - 1;
        const int64_t q0 = A.bkt_off[bk], cnt = A.bkt_off[ge] + A.bkt_n[ge] - q0;  // the bin group
#pragma unroll
        for (int k = 0; k < kIt; ++k) {
          const int s = t + kT * k;
          kb[k] = -1;
          kw[k] = 0;
          kr[k] = 0;
          if (s < cnt) { kb[k] = A.pb_g[q0 + s]; kw[k] = A.pw_g[q0 + s]; }
        }
        if (t == 0) {
          S.kmin[0] = INT32_MAX;
          S.kmax[0] = -1;
          S.ucnt[0] = 0;
          S.hbase[0] = (int32_t)(cnt + (cnt >> 1) + 1);
          S.wtot = 0;
        }
        __syncthreads();
      }
      // ---- 2. per-row hash regions; the creating thread owns each key
      const int Hs = smem_exclusive_scan(S.hbase, R, S.tmp);
      if (t == 0) S.hbase[R] = Hs;
      for (int i = t; i < Hs; i += kT) { S.a.hkey[i] = kEmpty; S.v.hval[i] = 0; }
      {
        long long ws = 0;
#pragma unroll
        for (int k = 0; k < kIt; ++k) ws += kb[k] >= 0 ? kw[k] : 0;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) ws += __shfl_xor_sync(0xffffffffu, ws, o);
        if ((t & 31) == 0 && ws) atomicAdd(&S.wtot, (unsigned long long)ws);
      }
      __syncthreads();
      if (!WIDE && S.wtot > 0x7fffffffull) {
        // a merged weight could exceed int32: leave the inputs untouched and let
        // the 64-bit pass redo this block
        if (t == 0) {
          A.need_wide[bi] = 1;
          atomicOr(A.err, ERR_WIDE);
        }
        __syncthreads();
        continue;
      }
      int32_t ks[kIt];  // owned slot or -1
#pragma unroll
      for (int k = 0; k < kIt; ++k) {
        bool fresh = false;
        ks[k] = -1;
        const int r = kr[k];
        if (kb[k] >= 0) {
          const int32_t b = kb[k];
          const int hb = S.hbase[r], hs = S.hbase[r + 1] - hb;
          int s = hb + (int)(((uint64_t)((uint32_t)b * 0x9E3779B1u) * (uint32_t)hs) >> 32);
          while (true) {
            int32_t cur = ((volatile int32_t *)S.a.hkey)[s];
            if (cur == b) break;
            if (cur == kEmpty) {
              int32_t old = atomicCAS(S.a.hkey + s, kEmpty, b);
              if (old == kEmpty) { fresh = true; break; }
              if (old == b) break;
            }
            if (++s == hb + hs) s = hb;
          }
          atomicAdd(S.v.hval + s, (V)kw[k]);
          if (fresh) ks[k] = s;
        }
        count_update(S.ucnt, r, fresh);
        if (!fresh) kb[k] = -1;  // not an owner
      }
      __syncthreads();
      T = smem_exclusive_scan(S.ucnt, R, S.tmp);
      if (t == 0) S.ucnt[R] = T;
      // ---- 3. owned keys: key range per row, buckets, ranks
#pragma unroll
      for (int k = 0; k < kIt; ++k) range_update(S.kmin, S.kmax, kb[k] >= 0 ? kr[k] : -1, kb[k]);
      __syncthreads();
      for (int r = t; r < R; r += kT) {
        const int lo = S.kmin[r], hi = S.kmax[r];
        const int cnt = S.ucnt[r + 1] - S.ucnt[r];
        S.bscale[r] = hi >= lo ? (float)cnt / (float)((int64_t)hi - lo + 1) : 0.f;
      }
      for (int i = t; i <= T; i += kT) S.a.hist[i] = 0;  // hash keys are dead
      __syncthreads();
#pragma unroll
      for (int k = 0; k < kIt; ++k) {
        if (kb[k] >= 0) {
          const int r = kr[k];
          const int nb = S.ucnt[r + 1] - S.ucnt[r];  // one bucket per distinct key
          int off = (int)((float)(kb[k] - S.kmin[r]) * S.bscale[r]);
          off = off < nb - 1 ? off : nb - 1;
          const int bin = S.ucnt[r] + off;
          kr[k] = (bin << 12) | atomicAdd(&S.a.hist[bin], 1);
          const V wv = S.v.hval[ks[k]];
          if (WIDE && (unsigned long long)wv > 0x7fffffffull) atomicOr(A.err, ERR_OVERFLOW);
          kw[k] = (int32_t)wv;  // final sum, read before the pairs overwrite the values
        }
      }
      __syncthreads();
      smem_exclusive_scan(S.a.hist, T + 1, S.tmp);
#pragma unroll
      for (int k = 0; k < kIt; ++k) {
        if (kb[k] >= 0) {
          const int q = S.a.hist[kr[k] >> 12] + (kr[k] & 4095);
          pb[q] = kb[k];
          pw[q] = kw[k];
        }
      }
      __syncthreads();
      // insertion sort inside each bucket (distinct keys, ~1 per bucket)
      for (int bin = t; bin < T; bin += kT) {
        const int lo = S.a.hist[bin], hi = S.a.hist[bin + 1];
        for (int i = lo + 1; i < hi; ++i) {
          const int32_t kk = pb[i], ww = pw[i];
          int j = i - 1;
          while (j >= lo && pb[j] > kk) {
            pb[j + 1] = pb[j];
            pw[j + 1] = pw[j];
            --j;
          }
          pb[j + 1] = kk;
          pw[j + 1] = ww;
        }
      }
    }
    __syncthreads();
    // ---- 4. stage the block's sorted distinct entries; k_place moves them
    if (rows_kind(d.kind)) {
      const int64_t P0 = S.mptr[0] - L.upos(L.a_lo);  // staging covers the active rows only
      for (int q = t; q < T; q += kT) {
        A.sc_col[P0 + q] = pb[q];
        A.sc_wgt[P0 + q] = pw[q];
      }
      for (int r = t; r < R; r += kT) {
        const int32_t a = d.row0 + r;
        A.row_ptr_c[a - L.a_lo] = S.ucnt[r];  // relative to the block's output offset
        const unsigned long long s = A.vw64[a];
        if (s > 0x7fffffffull) atomicOr(A.err, ERR_OVERFLOW);
        A.vwgt_c[a - L.a_lo] = (int32_t)s;
      }
    } else {
      if (d.kind == B_BUCKET) {
        const int64_t q0 = A.bkt_off[A.bkt_ptr[A.big_idx[d.row0]] + d.sub];
        for (int q = t; q < T; q += kT) {  // in place over the bucket's own pairs
          A.pb_g[q0 + q] = pb[q];
          A.pw_g[q0 + q] = pw[q];
        }
      } else if (d.kind == B_DENSE) {
        int32_t *st = reinterpret_cast<int32_t *>(A.dense + (int64_t)A.big_idx[d.row0] * L.n_c +
                                                  (int64_t)d.sub * kCap);
        for (int q = t; q < T; q += kT) {
          st[2 * q] = pb[q];
          st[2 * q + 1] = pw[q];
        }
      }
    }
    if (t == 0) A.blk_cnt[bi] = T;
    __syncthreads();
  }
}

// Placement: each warp owns 32 consecutive blocks (one per lane).  The
// blocks' outputs are contiguous in the final CSR, so the warp copies the
// whole range flattened: output element j finds its block by a 5-step shuffle
// search over the lanes' output offsets and reads from that block's staging
// (4 elements per lane in flight; per-block serial copies were latency-bound).
// Row offsets and vertex weights are then fixed per block.
constexpr int kPlaceT = 256;
enum : int { SRC_SC = 0, SRC_PB = 1, SRC_FB = 2, SRC_DENSE = 3 };

constexpr int kPlaceBig = 96;

// Heavy-neighbour keys of the graph being placed (fused: the next level's a1
// pass over G_{l+1} is not run).  key = w << 32 | ~b, the row's maximum = its
// heaviest neighbour, ties to the smallest id (Alg 3 l.6-10, reading Z1).
__device__ __forceinline__ unsigned long long place_key(int32_t w, int32_t b) {
  return ((unsigned long long)(uint32_t)w << 32) | (unsigned long long)(~(uint32_t)b);
}
// Row of block-relative entry r: the block's row unless it is a rows block
// holding several rows (row_ptr_c still block-relative: k_place fixes it after
// its copies, in the same warp).
__device__ __forceinline__ int32_t place_row(const RowsArgs &A, int kind, int32_t row0, int32_t row1, int64_t r) {
  if (!rows_kind(kind) || row1 - row0 <= 1) return row0;
  int32_t lo = row0, hi = row1 - 1;  // last row starting at or before r
  while (lo < hi) {
    const int32_t mid = (lo + hi + 1) >> 1;
    if (A.row_ptr_c[mid - A.L.a_lo] <= r) lo = mid;
    else hi = mid - 1;
  }
  return lo;
}
// The warp's 32 entries at consecutive output positions (rows non-decreasing
// over the valid lanes): segmented max per row, one atomicMax per row segment.
__device__ __forceinline__ void place_key_flush(const RowsArgs &A, bool valid, int32_t row, unsigned long long key) {
  const int lane = threadIdx.x & 31;
  unsigned long long v = valid ? key : 0ull;
  int32_t rw = valid ? row : -1;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const unsigned long long y = __shfl_up_sync(0xffffffffu, v, o);
    const int32_t ry = __shfl_up_sync(0xffffffffu, rw, o);
    if (lane >= o && ry == rw && y > v) v = y;
  }
  const int32_t rn = __shfl_down_sync(0xffffffffu, rw, 1);
  if (valid && (lane == 31 || rn != rw) && v) atomicMax(A.hkey + (rw - A.L.a_lo), v);
}

__global__ void __launch_bounds__(kPlaceT) k_place(RowsArgs A) {
  const int lane = threadIdx.x & 31;
  const int64_t b0 = ((int64_t)blockIdx.x * (kPlaceT / 32) + (threadIdx.x >> 5)) * 32;
  if (b0 >= A.nblocks) return;
  const Layout &L = A.L;
  const int64_t mine = b0 + lane;
  BlockDesc dm{-1, 0, 0, 0};
  int64_t Om = A.blk_off[A.nblocks - 1] + A.blk_cnt[A.nblocks - 1];  // past the end: empty
  int Tm = 0, src = SRC_SC;
  int64_t soff = 0;
  if (mine < A.nblocks) {
    dm = A.blk[mine];
    Om = A.blk_off[mine];
    Tm = A.blk_cnt[mine];
    if (rows_kind(dm.kind) || dm.kind == B_RBM) {  // staged over the expansion staging
      soff = L.upos(dm.row0) - L.upos(L.a_lo);
    } else if (dm.kind == B_DENSE) {
      src = SRC_DENSE;
      soff = 2 * ((int64_t)A.big_idx[dm.row0] * L.n_c + (int64_t)dm.sub * kCap);
    } else if (Tm > 0) {
      const int64_t bk = A.bkt_ptr[A.big_idx[dm.row0]] + dm.sub;
      if (A.fb_cnt[bk] >= 0) { src = SRC_FB; soff = A.fb_off[bk]; }
      else { src = SRC_PB; soff = A.bkt_off[bk]; }
    }
  }
  // blockIdx.y: slice of the copies (small levels: several warps per 32 blocks)
  const int S = gridDim.y, sl = blockIdx.y;
  if (sl == 0 && mine == A.nblocks - 1) A.row_ptr_c[L.a_hi - L.a_lo] = Om + Tm;
  const int64_t O0 = __shfl_sync(0xffffffffu, Om, 0);
  const int64_t total = __shfl_sync(0xffffffffu, Om + Tm, 31) - O0;
  const int32_t *dn = reinterpret_cast<const int32_t *>(A.dense);
  // blocks with >= kPlaceBig entries: copied one at a time by the whole warp
  // (8 entries per lane in flight); the others packed, entry -> block by a
  // 5-step shuffle search over the lanes' block offsets
  const bool bigb = Tm >= kPlaceBig;
  const int64_t Ps = bigb ? 0 : Tm;  // packed sizes
  int64_t pincl = Ps;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int64_t y = __shfl_up_sync(0xffffffffu, pincl, o);
    if (lane >= o) pincl += y;
  }
  const int64_t pex = pincl - Ps;
  const int64_t ptot = __shfl_sync(0xffffffffu, pincl, 31);
  for (int64_t j0 = (int64_t)sl * 128; j0 < ptot; j0 += (int64_t)S * 128) {
    int32_t c[4], w[4];
    int64_t dst[4];
#pragma unroll
    int32_t prow[4];
    for (int t = 0; t < 4; ++t) {
      const int64_t j = j0 + lane + 32 * t;
      int k = 0;  // last lane whose packed range starts at or before j
#pragma unroll
      for (int step = 16; step > 0; step >>= 1) {
        const int64_t Pc = __shfl_sync(0xffffffffu, pex, k + step);
        if (Pc <= j) k += step;
      }
      const int sk = __shfl_sync(0xffffffffu, src, k);
      const int64_t sb = __shfl_sync(0xffffffffu, soff, k);
      const int64_t r = j - __shfl_sync(0xffffffffu, pex, k);  // index inside the block
      dst[t] = __shfl_sync(0xffffffffu, Om, k) + r;
      if (A.hkey) {
        const int kk = __shfl_sync(0xffffffffu, dm.kind, k);
        const int32_t r0 = __shfl_sync(0xffffffffu, dm.row0, k), r1 = __shfl_sync(0xffffffffu, dm.row1, k);
        prow[t] = j < ptot ? place_row(A, kk, r0, r1, r) : -1;
      }
      if (j < ptot) {
        if (sk == SRC_SC) { c[t] = __ldcs(A.sc_col + sb + r); w[t] = __ldcs(A.sc_wgt + sb + r); }
        else if (sk == SRC_PB) { c[t] = __ldcs(A.pb_g + sb + r); w[t] = __ldcs(A.pw_g + sb + r); }
        else if (sk == SRC_FB) { c[t] = __ldcs(A.fb_b + sb + r); w[t] = __ldcs(A.fb_w + sb + r); }
        else { c[t] = dn[sb + 2 * r]; w[t] = dn[sb + 2 * r + 1]; }  // interleaved (b, w) pairs
      }
    }
    if (A.hkey) {
#pragma unroll
      for (int t = 0; t < 4; ++t) {
        const bool ok = j0 + lane + 32 * t < ptot;
        place_key_flush(A, ok, prow[t], ok ? place_key(w[t], c[t]) : 0ull);
      }
    }
#pragma unroll
    for (int t = 0; t < 4; ++t) {
      const int64_t j = j0 + lane + 32 * t;
      if (j < ptot) {
        __stcs(A.col_c + dst[t], c[t]);
        __stcs(A.wgt_c + dst[t], w[t]);
      }
    }
  }
  unsigned bmask = __ballot_sync(0xffffffffu, bigb);
  while (bmask) {
    const int jl = __ffs(bmask) - 1;
    bmask &= bmask - 1;
    const int sk = __shfl_sync(0xffffffffu, src, jl);
    const int64_t sb = __shfl_sync(0xffffffffu, soff, jl);
    const int64_t O = __shfl_sync(0xffffffffu, Om, jl);
    const int T = __shfl_sync(0xffffffffu, Tm, jl);
    const int32_t *sc, *sw;
    int stride = 1;
    if (sk == SRC_SC) { sc = A.sc_col + sb; sw = A.sc_wgt + sb; }
    else if (sk == SRC_PB) { sc = A.pb_g + sb; sw = A.pw_g + sb; }
    else if (sk == SRC_FB) { sc = A.fb_b + sb; sw = A.fb_w + sb; }
    else { sc = dn + sb; sw = dn + sb + 1; stride = 2; }
    const int bkind = __shfl_sync(0xffffffffu, dm.kind, jl);
    const int32_t brow0 = __shfl_sync(0xffffffffu, dm.row0, jl), brow1 = __shfl_sync(0xffffffffu, dm.row1, jl);
    const bool one_row = !rows_kind(bkind) || brow1 - brow0 <= 1;
    for (int r0 = sl * 256; r0 < T; r0 += S * 256) {
      int32_t c[8], w[8];
#pragma unroll
      for (int t = 0; t < 8; ++t) {
        const int r = r0 + lane + 32 * t;
        if (r < T) { c[t] = __ldcs(sc + (int64_t)stride * r); w[t] = __ldcs(sw + (int64_t)stride * r); }
      }
#pragma unroll
      for (int t = 0; t < 8; ++t) {
        const int r = r0 + lane + 32 * t;
        if (r < T) { __stcs(A.col_c + O + r, c[t]); __stcs(A.wgt_c + O + r, w[t]); }
      }
      if (A.hkey) {
        if (one_row) {  // one row: lane maxima, warp maximum, one atomic per 256 entries
          unsigned long long m = 0ull;
#pragma unroll
          for (int t = 0; t < 8; ++t)
            if (r0 + lane + 32 * t < T) {
              const unsigned long long key = place_key(w[t], c[t]);
              m = key > m ? key : m;
            }
#pragma unroll
          for (int o = 16; o > 0; o >>= 1) {
            const unsigned long long y = __shfl_xor_sync(0xffffffffu, m, o);
            m = y > m ? y : m;
          }
          if (lane == 0 && m) atomicMax(A.hkey + (brow0 - L.a_lo), m);
        } else {
#pragma unroll
          for (int t = 0; t < 8; ++t) {
            const int r = r0 + lane + 32 * t;
            const bool ok = r < T;
            place_key_flush(A, ok, ok ? place_row(A, bkind, brow0, brow1, r) : -1,
                            ok ? place_key(w[t], c[t]) : 0ull);
          }
        }
      }
    }
  }
  // per-block metadata: row offsets (rows blocks) / row start + vertex weight (skewed rows)
  // (block lane j is fixed up by slice j % S)
  unsigned m = __ballot_sync(0xffffffffu, mine < A.nblocks && (rows_kind(dm.kind) || dm.sub == 0) && lane % S == sl);
  while (m) {
    const int jl = __ffs(m) - 1;
    m &= m - 1;
    const int kind = __shfl_sync(0xffffffffu, dm.kind, jl);
    const int32_t row0 = __shfl_sync(0xffffffffu, dm.row0, jl);
    const int32_t row1 = __shfl_sync(0xffffffffu, dm.row1, jl);
    const int64_t O = __shfl_sync(0xffffffffu, Om, jl);
    if (rows_kind(kind)) {
      for (int a = row0 + lane; a < row1; a += 32) A.row_ptr_c[a - L.a_lo] += O;
    } else if (lane == 0) {  // the row's first block: row start and vertex weight
      A.row_ptr_c[row0 - L.a_lo] = O;
      A.vwgt_c[row0 - L.a_lo] = (int32_t)A.vw64[row0];  // bound checked by k_tiers
    }
  }
}

int launch_place(hec_ctx *ctx, const RowsArgs &A, bool *hkey_done) {
  if (hkey_done) *hkey_done = false;
  if (A.nblocks <= 0) return HEC_OK;
  // slices per 32-block group: enough warps for ~16 per SM on small levels
  const int64_t groups = (A.nblocks + 31) / 32;
  int64_t S = (int64_t)ctx->num_sms * 16 / groups;
  S = S < 1 ? 1 : S > 32 ? 32 : S;
  if (getenv("HEC_PLACE_ONE_SLICE") != nullptr) S = 1;  // test hook: fused heavy keys on small levels
  // heavy keys only with one slice per group: a rows block's offsets are then
  // read (row search) and fixed up by the same warp
  RowsArgs B = A;
  if (S != 1) B.hkey = nullptr;
  if (hkey_done) *hkey_done = B.hkey != nullptr;
  k_place<<<dim3((unsigned)nblk(groups, kPlaceT / 32), (unsigned)S), kPlaceT, 0, ctx->stream>>>(B);
  HEC_LAUNCH_CHECK();
  return HEC_OK;
}

int launch_rows(hec_ctx *ctx, const RowsArgs &A, bool wide) {
  int occ[2] = {1, 1};
  HEC_TRY(kernel_occupancy(ctx, k_rows<false>, kT, sizeof(RowsSmemT<false>), &occ[0]));
  HEC_TRY(kernel_occupancy(ctx, k_rows<true>, kT, sizeof(RowsSmemT<true>), &occ[1]));
  // persistent; the list length is read on the device
  int64_t grid = (int64_t)ctx->num_sms * occ[wide ? 1 : 0];
  if (A.nblocks < grid) grid = A.nblocks;
  if (grid < 1) return HEC_OK;
  if (wide) k_rows<true><<<(unsigned)grid, kT, sizeof(RowsSmemT<true>), ctx->stream>>>(A);
  else k_rows<false><<<(unsigned)grid, kT, sizeof(RowsSmemT<false>), ctx->stream>>>(A);
  HEC_LAUNCH_CHECK();
  return HEC_OK;
}

}  // namespace hec
