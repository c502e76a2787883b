// construct_rbm.cu — ordered duplicate merge by bitmap rank, one CTA per item
// (PAPER.md:L319-324 DEDUPWITHWTS, L280 self loops).
//
// An item is a set of entries (b, w) of ONE coarse row whose keys lie in a key
// range [lo, hi) of at most kRbmRange keys:
//   B_RBM     a whole row with kPieceMax < U <= kRbmRow, read from the
//             expansion staging (self entries b == row are dropped here), range
//             [0, n_c);
//   B_BUCKET  one key-range bin of a partitioned row (U > kRbmRow), read from
//             the partitioned pairs, range = the bin's key interval.
// The CTA marks every key in a shared-memory bitmap over the range (a summary
// bitmap records which words were touched), turns the touched words into
// prefix counts, and so knows the rank of every key among the item's distinct
// keys -- its position in the sorted output.  Each entry then adds its weight
// at its rank (64-bit sums, exact), and the distinct keys come out sorted with
// no sorting pass.  Work is O(entries + touched words); the bitmap is cleaned
// incrementally through the summary.  Items with more distinct keys than
// kRbmCap run in several rank windows and stage to the fallback scratch.
#include "construct_common.cuh"

namespace hec {

constexpr int kRbmT = 1024;                 // threads per CTA (one CTA per SM)
constexpr int kRbmIt = 4;                   // entries per thread per round
constexpr int kRbmRound = kRbmT * kRbmIt;   // 4096 entries per round
constexpr int kRbmWords = (int)(kRbmRange / 32);
constexpr int kRbmSumm = kRbmWords / 32;    // summary words (<= kRbmT)
static_assert(kRbmSumm <= kRbmT, "one summary word per thread");

struct RbmSmem {
  uint32_t bm[kRbmWords];
  uint16_t pref[kRbmWords];  // set bits before the word inside its 32-word summary group
  uint32_t sm[kRbmSumm];     // bit j of sm[s]: word 32 s + j was touched
  int32_t sbase[kRbmSumm];   // set bits before summary group s
  int32_t key[kRbmCap];
  unsigned long long val[kRbmCap];
  int32_t wtot[kRbmT / 32];  // set bits per warp's summary groups
  int64_t out;               // multi-window items: fallback scratch offset
};

__device__ __forceinline__ int rbm_rank(const RbmSmem &S, int o) {
  const int wd = o >> 5;
  return S.sbase[wd >> 5] + S.pref[wd] + __popc(S.bm[wd] & ((1u << (o & 31)) - 1u));
}

__device__ __forceinline__ RbmItem rbm_item(const RowsArgs &A, int64_t i, int64_t nitems) {
  RbmItem it{};
  it.n = -1;
  if (i < nitems) it = rbm_at(A.ritems, A.rdir, A.rcap, i);
  return it;
}

// round r0 of an item's entries: slot k of thread t is entry r0 + t + kRbmT k
__device__ __forceinline__ void rbm_load(const RowsArgs &A, const RbmItem &it, int64_t r0, int32_t (&kb)[kRbmIt],
                                         int32_t (&kw)[kRbmIt]) {
  const int32_t *sb = it.bk < 0 ? A.sc_col : A.pb_g;
  const int32_t *sw = it.bk < 0 ? A.sc_wgt : A.pw_g;
#pragma unroll
  for (int k = 0; k < kRbmIt; ++k) {
    const int64_t i = r0 + threadIdx.x + (int64_t)kRbmT * k;
    kb[k] = -1;
    kw[k] = 0;
    if (i < it.n) {
      kb[k] = __ldcs(sb + it.src + i);
      kw[k] = __ldcs(sw + it.src + i);
    }
  }
}

// Persistent: CTA c takes items c, c + G, c + 2G, ... (items are prefetched one
// ahead: the next item's descriptor and first 4096 entries are in flight while
// the current one is processed; a dynamic ticket would add an L2 round trip
// per item on the critical path).  Five CTA barriers per item.
__global__ void __launch_bounds__(kRbmT, 1) k_rbm(RowsArgs A) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  RbmSmem &S = *reinterpret_cast<RbmSmem *>(smem_raw);
  const int t = threadIdx.x, lane = t & 31, wid = t >> 5;
  const int64_t nitems = *A.nlist, G = gridDim.x;
  for (int i = t; i < kRbmWords; i += kRbmT) S.bm[i] = 0;
  for (int i = t; i < kRbmSumm; i += kRbmT) S.sm[i] = 0;
  for (int i = t; i < kRbmCap; i += kRbmT) S.val[i] = 0ull;
  int64_t ii = blockIdx.x;
  RbmItem cur = rbm_item(A, ii, nitems);
  RbmItem nxt = rbm_item(A, ii + G, nitems);
  int32_t kb[kRbmIt], kw[kRbmIt];
  rbm_load(A, cur, 0, kb, kw);
  __syncthreads();
  while (cur.n >= 0) {
    // prefetch: the next item's first round, the descriptor after it
    int32_t nb_[kRbmIt], nw_[kRbmIt];
    rbm_load(A, nxt, 0, nb_, nw_);
    const RbmItem nn = rbm_item(A, ii + 2 * G, nitems);
    const int32_t a = cur.row;
    const int64_t n = cur.n;
    const int lo = cur.lo;
    const int nw = (cur.hi - lo + 31) >> 5;
    const int ns = (nw + 31) >> 5;
    const bool one_round = n <= kRbmRound;
    const int32_t *src_b = (cur.bk < 0 ? A.sc_col : A.pb_g) + cur.src;
    const int32_t *src_w = (cur.bk < 0 ? A.sc_wgt : A.pw_g) + cur.src;
    // ---- 1. mark keys (first toucher of a word sets its summary bit)
    bool bad = false;
    for (int64_t r0 = 0; r0 < n; r0 += kRbmRound) {
      if (r0 > 0) rbm_load(A, cur, r0, kb, kw);
#pragma unroll
      for (int k = 0; k < kRbmIt; ++k) {
        if (kb[k] == a) kb[k] = -1;  // self entry (L280)
        if (kb[k] < 0) continue;
        if (kb[k] < lo || kb[k] >= cur.hi) { bad = true; kb[k] = -1; continue; }
        const int o = kb[k] - lo;
        const uint32_t old = atomicOr(&S.bm[o >> 5], 1u << (o & 31));
        if (old == 0u) atomicOr(&S.sm[o >> 10], 1u << ((o >> 5) & 31));
      }
    }
    if (bad) atomicOr(A.err, ERR_INTERNAL);
    __syncthreads();
    // ---- 2. prefix counts over the touched words, CTA scan of the group totals
    int cnt = 0;
    if (t < ns) {
      uint32_t bits = S.sm[t];
      while (bits) {
        const int j = __ffs(bits) - 1;
        bits &= bits - 1;
        const int wd = 32 * t + j;
        S.pref[wd] = (uint16_t)cnt;
        cnt += __popc(S.bm[wd]);
      }
    }
    int x = cnt;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int y = __shfl_up_sync(0xffffffffu, x, o);
      if (lane >= o) x += y;
    }
    if (lane == 31) S.wtot[wid] = x;
    __syncthreads();
    int before = 0, T = 0;
#pragma unroll 8
    for (int w = 0; w < kRbmT / 32; ++w) {
      const int v = S.wtot[w];
      before += w < wid ? v : 0;
      T += v;
    }
    if (t < ns) S.sbase[t] = before + x - cnt;
    const int passes = (T + kRbmCap - 1) / kRbmCap;
    if (passes > 1 && t == 0) {  // several rank windows: stage to the fallback scratch
      S.out = (int64_t)atomicAdd(A.fb_total, (unsigned long long)T);
      A.fb_off_w[cur.bk] = S.out;
      A.fb_cnt_w[cur.bk] = T;
    }
    if (t == 0) A.blk_cnt[cur.bi] = T;
    __syncthreads();
    int32_t *dst_b = const_cast<int32_t *>(src_b), *dst_w = const_cast<int32_t *>(src_w);
    if (passes > 1) {
      dst_b = A.fb_b_w + S.out;
      dst_w = A.fb_w_w + S.out;
    }
    // ---- 3. weights added at their rank, one rank window at a time
    for (int p = 0; p < passes; ++p) {
      const int r_lo = p * kRbmCap, r_hi = min(T, r_lo + kRbmCap);
      for (int64_t r0 = 0; r0 < n; r0 += kRbmRound) {
        if (!one_round) {
          rbm_load(A, cur, r0, kb, kw);
#pragma unroll
          for (int k = 0; k < kRbmIt; ++k)
            if (kb[k] == a || kb[k] < lo || kb[k] >= cur.hi) kb[k] = -1;
        }
#pragma unroll
        for (int k = 0; k < kRbmIt; ++k) {
          if (kb[k] < 0) continue;
          const int r = rbm_rank(S, kb[k] - lo);
          if (r >= r_lo && r < r_hi) {
            atomicAdd(&S.val[r - r_lo], (unsigned long long)(uint32_t)kw[k]);
            S.key[r - r_lo] = kb[k];
          }
        }
      }
      __syncthreads();
      for (int i = t; i < r_hi - r_lo; i += kRbmT) {
        const unsigned long long v = S.val[i];
        if (v > 0x7fffffffull) atomicOr(A.err, ERR_OVERFLOW);
        dst_b[r_lo + i] = S.key[i];
        dst_w[r_lo + i] = (int32_t)v;
        S.val[i] = 0ull;
      }
      if (p + 1 < passes) __syncthreads();
    }
    // ---- 4. clean the touched words for the next item
    if (t < ns) {
      uint32_t bits = S.sm[t];
      while (bits) {
        const int j = __ffs(bits) - 1;
        bits &= bits - 1;
        S.bm[32 * t + j] = 0u;
      }
      S.sm[t] = 0u;
    }
    __syncthreads();
    cur = nxt;
    nxt = nn;
    ii += G;
#pragma unroll
    for (int k = 0; k < kRbmIt; ++k) { kb[k] = nb_[k]; kw[k] = nw_[k]; }
  }
}

int launch_rbm(hec_ctx *ctx, const RowsArgs &A) {
  int occ = 1;
  HEC_TRY(kernel_occupancy(ctx, k_rbm, kRbmT, sizeof(RbmSmem), &occ));
  int64_t grid = ctx->num_sms;  // one CTA per SM (shared-memory bound); items read from *A.nlist
  if (A.nblocks < grid) grid = A.nblocks;
  if (grid < 1) return HEC_OK;
  k_rbm<<<(unsigned)grid, kRbmT, sizeof(RbmSmem), ctx->stream>>>(A);
  HEC_LAUNCH_CHECK();
  return HEC_OK;
}

}  // namespace hec
