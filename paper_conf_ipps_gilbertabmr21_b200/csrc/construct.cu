// construct.cu — CONSTRUCTCOARSEGRAPH on sm_100a.
//
// Result: W_c(a,b) = sum over fine entries (u,v) with
// M[u]=a, M[v]=b, a != b of W(u,v); rows ascending in b; vwgt_c(a) = sum vwgt.
//
// Coarse-row-centric pipeline (replaces Alg 6's edge-parallel atomic count/fill,
// L287-316, and the per-vertex DEDUPWITHWTS, L319-324):
//  a7  bucketing: counting sort of the fine vertices by M (member_ptr, members)
//      and the "member-edge space": fine entries regrouped by coarse row; row a
//      owns positions [upos(a), upos(a+1)), U(a) = their number (bound on |row|).
//  a8  rows with U <= 2040 ("small") are packed into work blocks of < 4096
//      entries.  One CTA per block: edge-balanced expansion of (b = M[v], w) into
//      registers through shared-memory member tables, key-range bucket sort in
//      shared memory (one smem atomic per entry gives each entry its slot), then
//      per-bucket insertion sort and duplicate merge with exact int64 sums (the
//      paper's sort-based DEDUPWITHWTS, fastest on GPUs per Table II).
//  a9  skewed rows (U > 2040):
//        BUCKET  (n_c > 32768): the row's pairs are partitioned by key range into
//                buckets of ~1024 entries in global memory (two passes), each
//                bucket then is one work block of the a8 kind (the paper's
//                segmented global sort alternative, L324); buckets that overflow
//                a CTA go through an exact hash-based fallback.
//        DENSE   (n_c <= 32768): persistent CTAs accumulate the row into a
//                shared-memory dense array, merged into a dense int64 row; the
//                row is read back in key order (no sort).
//  a10 output placement fused into the same kernel: work blocks are taken in
//      order and each obtains its output offset with a decoupled look-back over
//      block totals, then writes col_c/wgt_c/row_ptr_c/vwgt_c in place (no
//      scratch + compaction pass).
#include "hec_internal.cuh"

namespace hec {

constexpr int kT = 512;            // threads per CTA of the row kernels
constexpr int kIt = 8;             // entries held per thread (registers)
constexpr int kCap = kT * kIt;     // entries per work block (4096)
constexpr int kWin = 2048;         // window weight; a block's weight is < 2*kWin
constexpr int kRowW = 8;           // per-row weight: bounds rows per block
constexpr int kMaxRows = 2 * kWin / kRowW;   // 512
constexpr int kSmallMax = kWin - kRowW;      // rows with U <= 2040 are small
constexpr int kMC = 1024;          // member-table chunk
constexpr int kBucketAvg = 1024;   // target entries per BUCKET
constexpr int kDenseMax = 32768;   // n_c bound of the DENSE skew path
constexpr int kFbTab = 16384;      // fallback hash slots (int64 values)
constexpr int kFbCap = 8192;       // fallback distinct keys per sub-range pass
constexpr int32_t kEmpty = -1;

enum : int32_t { B_SMALL = 0, B_BUCKET = 1, B_DENSE = 2 };

static inline unsigned nblk(int64_t n, int b) { return (unsigned)((n + b - 1) / b); }

// ----------------------------------------------------------------- helpers
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
__device__ int smem_exclusive_scan(int32_t *a, int n, int32_t *tmp) {
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

__device__ __forceinline__ int block_sum(int v, int32_t *tmp) {
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  if (lane == 0) tmp[wid] = v;
  __syncthreads();
  int s = 0;
  for (int w = 0; w < kT / 32; ++w) s += tmp[w];
  __syncthreads();
  return s;
}

__device__ __forceinline__ unsigned hslot(int32_t b, unsigned mask) {
  return ((uint32_t)b * 0x9E3779B1u) >> 7 & mask;
}

// ------------------------------------------------------------ a7 bucketing
__global__ void k_member_count(int64_t n, const int32_t *__restrict__ M, int64_t n_c,
                               const int32_t *__restrict__ vwgt, unsigned *__restrict__ mcount,
                               unsigned long long *__restrict__ vw64, int *__restrict__ err) {
  int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (u >= n) return;
  int32_t a = M[u];
  if (a < 0 || a >= n_c) { atomicOr(err, 1); return; }
  atomicAdd(mcount + a, 1u);
  atomicAdd(vw64 + a, (unsigned long long)(vwgt ? vwgt[u] : 1));
}

__global__ void k_member_fill(int64_t n, int64_t n_c, const int32_t *__restrict__ M,
                              const int64_t *__restrict__ member_ptr, unsigned *__restrict__ mcount,
                              int32_t *__restrict__ members) {
  int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (u >= n) return;
  int32_t a = M[u];
  if (a < 0 || a >= n_c) return;  // reported through err by k_member_count
  unsigned k = atomicSub(mcount + a, 1u) - 1u;
  members[member_ptr[a] + k] = (int32_t)u;
}

struct CountIn {
  const unsigned *c;
  __device__ __forceinline__ int64_t operator()(int64_t i) const { return c[i]; }
};
struct PtrOut {
  int64_t *p;
  __device__ __forceinline__ void operator()(int64_t i, int64_t pre) const { p[i] = pre; }
};
struct DegIn {
  const int32_t *members;
  const int64_t *row_ptr;
  const int64_t *valid;  // number of bucketed members (< n only for invalid M)
  __device__ __forceinline__ int64_t operator()(int64_t i) const {
    if (i >= *valid) return 0;
    int32_t u = members[i];
    return row_ptr[u + 1] - row_ptr[u];
  }
};

struct Layout {
  int64_t n_c;
  const int64_t *member_ptr;  // [n_c+1]
  const int32_t *members;     // [n]
  const int64_t *mpre;        // [n+1] member-edge prefix
  const int64_t *row_ptr;
  const int32_t *col;
  const int32_t *wgt;
  const int32_t *M;
  __device__ __forceinline__ int64_t upos(int64_t a) const { return mpre[member_ptr[a]]; }
  __device__ __forceinline__ int64_t U(int64_t a) const { return upos(a + 1) - upos(a); }
};

// window weight of small rows (U + kRowW), 0 for big rows
struct RowWeightIn {
  Layout L;
  __device__ __forceinline__ int64_t operator()(int64_t a) const {
    int64_t U = L.U(a);
    return U <= kSmallMax ? U + kRowW : 0;
  }
};

// big rows: list (unordered) + row -> list index; member-edge volume per class
__global__ void k_big_rows(Layout L, int32_t *__restrict__ big_list, int32_t *__restrict__ big_idx,
                           unsigned *__restrict__ nbig, unsigned long long *__restrict__ vol) {
  int64_t a = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  bool in = a < L.n_c;
  int64_t U = in ? L.U(a) : 0;
  bool big = in && U > kSmallMax;
  unsigned m = __ballot_sync(0xffffffffu, big);
  int lane = threadIdx.x & 31;
  unsigned base = 0;
  if (m) {
    int leader = __ffs(m) - 1;
    if (lane == leader) base = atomicAdd(nbig, (unsigned)__popc(m));
    base = __shfl_sync(0xffffffffu, base, leader);
  }
  if (big) {
    unsigned pos = base + __popc(m & ((1u << lane) - 1));
    big_list[pos] = (int32_t)a;
    big_idx[a] = (int32_t)pos;
  } else if (in) {
    big_idx[a] = -1;
  }
  unsigned long long vs = big ? 0 : U, vb = big ? U : 0;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    vs += __shfl_xor_sync(0xffffffffu, vs, o);
    vb += __shfl_xor_sync(0xffffffffu, vb, o);
  }
  if (lane == 0) {
    if (vs) atomicAdd(vol + 0, vs);
    if (vb) atomicAdd(vol + 1, vb);
  }
}

__host__ __device__ __forceinline__ int64_t row_buckets(int64_t U, int64_t n_c) {
  int64_t nb = (U + kBucketAvg - 1) / kBucketAvg;
  if (nb > n_c) nb = n_c;
  return nb < 1 ? 1 : nb;
}
__host__ __device__ __forceinline__ int64_t dense_chunks(int64_t n_c) { return (n_c + kCap - 1) / kCap; }

// number of work blocks starting at row a
struct BlockCountIn {
  Layout L;
  const int64_t *S;  // exclusive scan of RowWeightIn
  bool dense;
  __device__ __forceinline__ int64_t operator()(int64_t a) const {
    int64_t U = L.U(a);
    if (U > kSmallMax) return dense ? dense_chunks(L.n_c) : row_buckets(U, L.n_c);
    if (a == 0) return 1;
    if (L.U(a - 1) > kSmallMax) return 1;
    return (S[a] / kWin) != (S[a - 1] / kWin) ? 1 : 0;
  }
};

struct BlockDesc {
  int32_t kind;
  int32_t row0;  // first row (SMALL) / the row (BUCKET, DENSE)
  int32_t row1;  // one past the last row (SMALL)
  int32_t sub;   // bucket index within the row / dense key chunk
};

__global__ void k_block_desc(Layout L, const int64_t *__restrict__ blk_ptr, const int32_t *__restrict__ big_idx,
                             bool dense, BlockDesc *__restrict__ blk) {
  int64_t a = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (a >= L.n_c) return;
  int64_t b0 = blk_ptr[a], b1 = blk_ptr[a + 1];
  if (b1 == b0) return;
  if (big_idx[a] >= 0) {
    for (int64_t k = b0; k < b1; ++k)
      blk[k] = BlockDesc{dense ? B_DENSE : B_BUCKET, (int32_t)a, (int32_t)a + 1, (int32_t)(k - b0)};
  } else {
    blk[b0] = BlockDesc{B_SMALL, (int32_t)a, -1, 0};
  }
}
// row1 of SMALL blocks = first row of the next block (or n_c)
__global__ void k_block_ends(int64_t nblocks, int64_t n_c, BlockDesc *__restrict__ blk) {
  int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (k >= nblocks) return;
  if (blk[k].kind == B_SMALL) blk[k].row1 = (k + 1 < nblocks) ? blk[k + 1].row0 : (int32_t)n_c;
}

// ------------------------------------------------------------- expansion
struct MemberTab {
  int64_t mstart[kMC];     // row_ptr[u] of the member
  int32_t moff[kMC + 1];   // member's first position relative to the window start
  int32_t mrow[kMC];       // local row of the member
};

// Expand the member-edge window [P0, P0+nP) (nP <= kCap), whose members are
// [m0, m1), into registers: slot s = tid + kT*k holds (b = M[v], w, local row).
// Slots without an entry keep kb = -1.  s_mptr[0..R]: member_ptr slice of the
// rows (nullptr => one row, index 0).
__device__ __forceinline__ void expand_window(const Layout &L, MemberTab &T, int64_t P0, int nP, int64_t m0,
                                              int64_t m1, const int64_t *s_mptr, int R, int32_t (&kb)[kIt],
                                              int32_t (&kw)[kIt], int32_t (&kr)[kIt]) {
  const int t = threadIdx.x;
#pragma unroll
  for (int k = 0; k < kIt; ++k) { kb[k] = -1; kw[k] = 0; kr[k] = 0; }
  for (int64_t cm = m0; cm < m1; cm += kMC) {
    const int nm = (int)((m1 - cm) < kMC ? (m1 - cm) : kMC);
    for (int i = t; i < nm; i += kT) {
      int32_t u = L.members[cm + i];
      T.mstart[i] = L.row_ptr[u];
      T.moff[i] = (int32_t)(L.mpre[cm + i] - P0);
      T.mrow[i] = s_mptr ? (int32_t)last_le(s_mptr, 0, R, cm + i) : 0;
    }
    if (t == 0) {
      int64_t e = L.mpre[cm + nm] - P0;
      T.moff[nm] = (int32_t)(e > (int64_t)kCap + 1 ? kCap + 1 : e);
    }
    __syncthreads();
    const int lo = T.moff[0] > 0 ? T.moff[0] : 0;
    const int hi = T.moff[nm] < nP ? T.moff[nm] : nP;
    unsigned fresh = 0;
    int64_t ev[kIt];
#pragma unroll
    for (int k = 0; k < kIt; ++k) {
      const int s = t + kT * k;
      ev[k] = 0;
      if (s >= lo && s < hi) {
        int i = (int)last_le(T.moff, 0, nm, s);
        ev[k] = T.mstart[i] + (s - T.moff[i]);
        kr[k] = T.mrow[i];
        fresh |= 1u << k;
      }
    }
#pragma unroll
    for (int k = 0; k < kIt; ++k)
      if (fresh & (1u << k)) { kb[k] = __ldg(L.col + ev[k]); kw[k] = __ldg(L.wgt + ev[k]); }
#pragma unroll
    for (int k = 0; k < kIt; ++k)
      if (fresh & (1u << k)) kb[k] = __ldg(L.M + kb[k]);
    __syncthreads();
  }
}

// Members of a big row covering the window [P0, P0+nP): [m0, m1).
__device__ __forceinline__ void window_members(const Layout &L, int32_t a, int64_t P0, int nP, int64_t *m0,
                                               int64_t *m1) {
  const int64_t m0r = L.member_ptr[a], m1r = L.member_ptr[a + 1];
  *m0 = last_le(L.mpre, m0r, m1r, P0);
  int64_t lo = *m0, hi = m1r - 1;  // last member i with mpre[i] < P0 + nP
  while (lo < hi) {
    int64_t mid = (lo + hi + 1) >> 1;
    if (L.mpre[mid] < P0 + nP) lo = mid;
    else hi = mid - 1;
  }
  *m1 = lo + 1;
}

// ---------------------------------------------------- bucket sort + dedup
struct RowsSmem {
  MemberTab T;
  int64_t mptr[kMaxRows + 1];
  int32_t row_id[kMaxRows];
  int32_t kmin[kMaxRows];
  int32_t kmax[kMaxRows];
  int32_t bbase[kMaxRows + 1];
  float bscale[kMaxRows];
  int32_t hist[kCap + 1];  // bucket histogram -> bucket offsets
  int32_t ucnt[kCap + 1];  // unique count per bucket -> output offsets
  int32_t pb[kCap];        // pairs in bucket order
  int32_t pw[kCap];
  int32_t tmp[40];
  int64_t prefix;
  int32_t blk;
  int32_t nbins;
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

// Key range per local row over the valid register entries.
__device__ __forceinline__ void row_key_range(RowsSmem &S, const int32_t (&kb)[kIt], const int32_t (&kr)[kIt]) {
#pragma unroll
  for (int k = 0; k < kIt; ++k) {
    const bool valid = kb[k] >= 0;
    const int r = valid ? kr[k] : -1;
    const int r0 = __shfl_sync(0xffffffffu, r, 0);
    if (__all_sync(0xffffffffu, r == r0)) {
      if (r0 >= 0) {
        int mn = warp_min(kb[k]), mx = warp_max(kb[k]);
        if ((threadIdx.x & 31) == 0) { atomicMin(&S.kmin[r0], mn); atomicMax(&S.kmax[r0], mx); }
      }
    } else if (valid) {
      atomicMin(&S.kmin[r], kb[k]);
      atomicMax(&S.kmax[r], kb[k]);
    }
  }
}

// Bucket-sort the register entries of rows 0..R-1 (key ranges in kmin/kmax,
// entry bounds rowU) and merge duplicates.  Leaves S.hist = bucket offsets into
// pb/pw, S.ucnt = exclusive offsets of the unique entries per bucket (S.ucnt[nbins]
// = total), returns the number of unique entries.  A merged weight above
// INT32_MAX sets err bit 2 (exact: sums are int64).
__device__ int sort_dedup(RowsSmem &S, int R, const int64_t *rowU, int32_t (&kb)[kIt], int32_t (&kw)[kIt],
                          int32_t (&kr)[kIt], int *err) {
  const int t = threadIdx.x;
  for (int r = t; r < R; r += kT) {
    int lo = S.kmin[r], hi = S.kmax[r];
    int nb = 0;
    if (hi >= lo) {
      int64_t span = (int64_t)hi - lo + 1;
      int64_t lim = rowU[r] < span ? rowU[r] : span;
      nb = 1;
      while ((int64_t)nb * 2 <= lim && nb * 2 <= kCap) nb *= 2;
      S.bscale[r] = (float)nb / (float)span;
    } else {
      S.bscale[r] = 0.f;
    }
    S.bbase[r] = nb;
  }
  __syncthreads();
  const int nbins = smem_exclusive_scan(S.bbase, R, S.tmp);
  if (t == 0) S.bbase[R] = nbins;
  for (int i = t; i <= nbins; i += kT) S.hist[i] = 0;
  __syncthreads();
  // bucket (monotone in the key within a row) and rank inside the bucket
#pragma unroll
  for (int k = 0; k < kIt; ++k) {
    if (kb[k] >= 0) {
      const int r = kr[k];
      const int nb = S.bbase[r + 1] - S.bbase[r];
      int off = (int)((float)(kb[k] - S.kmin[r]) * S.bscale[r]);
      off = off < nb - 1 ? off : nb - 1;
      const int bin = S.bbase[r] + off;
      const int rank = atomicAdd(&S.hist[bin], 1);
      kr[k] = (bin << 12) | rank;
    }
  }
  __syncthreads();
  smem_exclusive_scan(S.hist, nbins + 1, S.tmp);
#pragma unroll
  for (int k = 0; k < kIt; ++k) {
    if (kb[k] >= 0) {
      const int q = S.hist[kr[k] >> 12] + (kr[k] & 4095);
      S.pb[q] = kb[k];
      S.pw[q] = kw[k];
    }
  }
  __syncthreads();
  for (int bin = t; bin < nbins; bin += kT) {
    const int lo = S.hist[bin], hi = S.hist[bin + 1];
    for (int i = lo + 1; i < hi; ++i) {
      int kk = S.pb[i], ww = S.pw[i];
      int j = i - 1;
      while (j >= lo && S.pb[j] > kk) {
        S.pb[j + 1] = S.pb[j];
        S.pw[j + 1] = S.pw[j];
        --j;
      }
      S.pb[j + 1] = kk;
      S.pw[j + 1] = ww;
    }
    int out = lo;
    int i = lo;
    while (i < hi) {
      int kk = S.pb[i];
      long long acc = 0;
      while (i < hi && S.pb[i] == kk) acc += S.pw[i++];
      if (acc > 0x7fffffffLL) atomicOr(err, 2);
      S.pb[out] = kk;
      S.pw[out] = (int32_t)acc;
      ++out;
    }
    S.ucnt[bin] = out - lo;
  }
  __syncthreads();
  const int T = smem_exclusive_scan(S.ucnt, nbins, S.tmp);
  if (t == 0) { S.ucnt[nbins] = T; S.nbins = nbins; }
  __syncthreads();
  return T;
}

// unique entry q of the block -> (b, w); the largest bucket whose unique offset
// is <= q is never empty, so it holds q.
__device__ __forceinline__ void emit(const RowsSmem &S, int nbins, int T, int64_t O, int32_t *__restrict__ col_c,
                                     int32_t *__restrict__ wgt_c) {
  for (int q = threadIdx.x; q < T; q += kT) {
    int bin = (int)last_le(S.ucnt, 0, nbins, q);
    int src = S.hist[bin] + (q - S.ucnt[bin]);
    col_c[O + q] = S.pb[src];
    wgt_c[O + q] = S.pw[src];
  }
}

struct RowsArgs {
  Layout L;
  const BlockDesc *blk;
  int64_t nblocks;
  unsigned *ticket;
  uint64_t *desc;  // look-back descriptors [nblocks]
  const unsigned long long *vw64;
  const int32_t *big_idx;
  // BUCKET mode
  const int64_t *bkt_ptr;      // [nbig+1] first bucket of big row h
  const int64_t *bkt_off;      // [nbkt+1] pair offsets
  const int32_t *pb_g, *pw_g;  // partitioned pairs
  const int32_t *fb_cnt;       // fallback unique count per bucket (-1: not overflowed)
  const int64_t *fb_off;       // fallback scratch offset per bucket
  const int32_t *fb_b, *fb_w;
  // DENSE mode
  const unsigned long long *dense;  // [nbig][n_c]
  // outputs
  int64_t *row_ptr_c;
  int32_t *col_c, *wgt_c, *vwgt_c;
  int *err;
};

__device__ __forceinline__ void write_vwgt(const RowsArgs &A, int32_t a) {
  unsigned long long s = A.vw64[a];
  if (s > 0x7fffffffull) atomicOr(A.err, 2);
  A.vwgt_c[a] = (int32_t)s;
}

// keys b with floor(b * nb / n_c) == k: [ceil(k n_c / nb), ceil((k+1) n_c / nb))
__device__ __forceinline__ void bucket_range(int64_t k, int64_t nb, int64_t n_c, int32_t *lo, int32_t *hi) {
  *lo = (int32_t)((k * n_c + nb - 1) / nb);
  int64_t h = ((k + 1) * n_c + nb - 1) / nb;
  *hi = (int32_t)(h < n_c ? h : n_c);
}

__global__ void __launch_bounds__(kT, 2) k_rows(RowsArgs A) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  RowsSmem &S = *reinterpret_cast<RowsSmem *>(smem_raw);
  const int t = threadIdx.x;
  const Layout &L = A.L;
  int64_t *rowU = reinterpret_cast<int64_t *>(S.T.mstart);  // member table is free after expansion
  while (true) {
    if (t == 0) S.blk = (int32_t)atomicAdd(A.ticket, 1u);
    __syncthreads();
    const int64_t bi = S.blk;
    if (bi >= A.nblocks) return;
    const BlockDesc d = A.blk[bi];
    int32_t kb[kIt], kw[kIt], kr[kIt];
    int T = 0, nbins = 0, R = 1;
    bool direct = false;  // DENSE / fallback: uniques already in key order
    if (d.kind == B_SMALL) {
      R = d.row1 - d.row0;
      for (int r = t; r <= R; r += kT) {
        S.mptr[r] = L.member_ptr[d.row0 + r];
        if (r < R) { S.row_id[r] = d.row0 + r; S.kmin[r] = INT32_MAX; S.kmax[r] = -1; }
      }
      __syncthreads();
      const int64_t m0 = S.mptr[0], m1 = S.mptr[R];
      const int64_t P0 = L.mpre[m0];
      const int nP = (int)(L.mpre[m1] - P0);
      expand_window(L, S.T, P0, nP, m0, m1, S.mptr, R, kb, kw, kr);
#pragma unroll
      for (int k = 0; k < kIt; ++k)
        if (kb[k] >= 0 && kb[k] == S.row_id[kr[k]]) kb[k] = -1;  // self entries are dropped (L280)
      row_key_range(S, kb, kr);
      for (int r = t; r < R; r += kT) rowU[r] = L.mpre[S.mptr[r + 1]] - L.mpre[S.mptr[r]];
      __syncthreads();
      T = sort_dedup(S, R, rowU, kb, kw, kr, A.err);
      nbins = S.nbins;
    } else if (d.kind == B_BUCKET) {
      const int32_t h = A.big_idx[d.row0];
      const int64_t bk = A.bkt_ptr[h] + d.sub;
      const int64_t q0 = A.bkt_off[bk], cnt = A.bkt_off[bk + 1] - q0;
      if (A.fb_cnt[bk] >= 0) {
        T = A.fb_cnt[bk];
        direct = true;
      } else {
        const int64_t nb = A.bkt_ptr[h + 1] - A.bkt_ptr[h];
        int32_t lo, hi;
        bucket_range(d.sub, nb, L.n_c, &lo, &hi);
#pragma unroll
        for (int k = 0; k < kIt; ++k) {
          const int s = t + kT * k;
          kb[k] = -1;
          kr[k] = 0;
          kw[k] = 0;
          if (s < cnt) { kb[k] = A.pb_g[q0 + s]; kw[k] = A.pw_g[q0 + s]; }
        }
        if (t == 0) { S.kmin[0] = lo; S.kmax[0] = hi - 1; rowU[0] = cnt; }
        __syncthreads();
        T = sort_dedup(S, 1, rowU, kb, kw, kr, A.err);
        nbins = S.nbins;
      }
    } else {  // B_DENSE: key chunk [k0, k0 + kCap) of a dense row, in key order
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
      S.ucnt[t] = c;
      __syncthreads();
      T = smem_exclusive_scan(S.ucnt, kT, S.tmp);
      int pos = S.ucnt[t];
#pragma unroll
      for (int k = 0; k < kIt; ++k) {
        if (v[k] != 0) {
          if (v[k] > 0x7fffffffull) atomicOr(A.err, 2);
          S.pb[pos] = (int32_t)(k0 + (int64_t)t * kIt + k);
          S.pw[pos] = (int32_t)v[k];
          ++pos;
        }
      }
      __syncthreads();
      direct = true;
    }
    // ---- a10: decoupled look-back over block totals, then write in place
    if (t < 32) {
      int64_t p = lookback(A.desc, (int)bi, T);
      if (t == 0) S.prefix = p;
    }
    __syncthreads();
    const int64_t O = S.prefix;
    if (!direct) {
      emit(S, nbins, T, O, A.col_c, A.wgt_c);
    } else if (d.kind == B_BUCKET) {
      const int64_t bk = A.bkt_ptr[A.big_idx[d.row0]] + d.sub;
      const int64_t f0 = A.fb_off[bk];
      for (int q = t; q < T; q += kT) {
        A.col_c[O + q] = A.fb_b[f0 + q];
        A.wgt_c[O + q] = A.fb_w[f0 + q];
      }
    } else {
      for (int q = t; q < T; q += kT) {
        A.col_c[O + q] = S.pb[q];
        A.wgt_c[O + q] = S.pw[q];
      }
    }
    if (d.kind == B_SMALL) {
      for (int r = t; r < R; r += kT) {
        A.row_ptr_c[S.row_id[r]] = O + S.ucnt[S.bbase[r]];
        write_vwgt(A, S.row_id[r]);
      }
    } else if (d.sub == 0 && t == 0) {
      A.row_ptr_c[d.row0] = O;
      write_vwgt(A, d.row0);
    }
    if (bi == A.nblocks - 1 && t == 0) A.row_ptr_c[L.n_c] = O + T;
    __syncthreads();
  }
}

// ------------------------------------------------------- a9 BUCKET partition
// Work units: big row h (list index) split into ceil(U/kCap) windows of kCap
// member-edge positions; unit_ptr = exclusive scan over big rows.
struct UnitsIn {
  Layout L;
  const int32_t *big_list;
  __device__ __forceinline__ int64_t operator()(int64_t h) const {
    return (L.U(big_list[h]) + kCap - 1) / kCap;
  }
};
struct BucketsIn {
  Layout L;
  const int32_t *big_list;
  __device__ __forceinline__ int64_t operator()(int64_t h) const { return row_buckets(L.U(big_list[h]), L.n_c); }
};

struct PartSmem {
  MemberTab T;
  int32_t hist[8192];
  int64_t base[8192];
};

// Expand unit `unit` into registers; kr = bucket of each entry (self dropped).
__device__ __forceinline__ void unit_expand(const Layout &L, PartSmem &S, const int32_t *big_list, int64_t nbig,
                                            const int64_t *unit_ptr, const int64_t *bkt_ptr, int64_t unit,
                                            int64_t *h_out, int64_t *nb_out, int32_t (&kb)[kIt],
                                            int32_t (&kw)[kIt], int32_t (&kr)[kIt]) {
  const int64_t h = last_le(unit_ptr, 0, nbig, unit);
  const int32_t a = big_list[h];
  const int64_t P0 = L.upos(a) + (unit - unit_ptr[h]) * kCap;
  const int64_t Pend = L.upos(a + 1);
  const int nP = (int)((Pend - P0) < kCap ? (Pend - P0) : kCap);
  int64_t m0, m1;
  window_members(L, a, P0, nP, &m0, &m1);
  expand_window(L, S.T, P0, nP, m0, m1, nullptr, 1, kb, kw, kr);
  const int64_t nb = bkt_ptr[h + 1] - bkt_ptr[h];
#pragma unroll
  for (int k = 0; k < kIt; ++k) {
    if (kb[k] == a) kb[k] = -1;
    kr[k] = kb[k] >= 0 ? (int32_t)(((int64_t)kb[k] * nb) / L.n_c) : 0;
  }
  *h_out = h;
  *nb_out = nb;
}

__global__ void __launch_bounds__(kT) k_part_count(Layout L, const int32_t *__restrict__ big_list, int64_t nbig,
                                                   const int64_t *__restrict__ unit_ptr,
                                                   const int64_t *__restrict__ bkt_ptr,
                                                   unsigned *__restrict__ bkt_cnt) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  PartSmem &S = *reinterpret_cast<PartSmem *>(smem_raw);
  int32_t kb[kIt], kw[kIt], kr[kIt];
  int64_t h, nb;
  unit_expand(L, S, big_list, nbig, unit_ptr, bkt_ptr, blockIdx.x, &h, &nb, kb, kw, kr);
  const bool sh = nb <= 8192;
  if (sh)
    for (int i = threadIdx.x; i < nb; i += kT) S.hist[i] = 0;
  __syncthreads();
#pragma unroll
  for (int k = 0; k < kIt; ++k)
    if (kb[k] >= 0) {
      if (sh) atomicAdd(&S.hist[kr[k]], 1);
      else atomicAdd(bkt_cnt + bkt_ptr[h] + kr[k], 1u);
    }
  __syncthreads();
  if (sh)
    for (int i = threadIdx.x; i < nb; i += kT)
      if (S.hist[i]) atomicAdd(bkt_cnt + bkt_ptr[h] + i, (unsigned)S.hist[i]);
}

__global__ void __launch_bounds__(kT) k_part_write(Layout L, const int32_t *__restrict__ big_list, int64_t nbig,
                                                   const int64_t *__restrict__ unit_ptr,
                                                   const int64_t *__restrict__ bkt_ptr,
                                                   const int64_t *__restrict__ bkt_off, unsigned *__restrict__ bkt_cur,
                                                   int32_t *__restrict__ pb, int32_t *__restrict__ pw) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  PartSmem &S = *reinterpret_cast<PartSmem *>(smem_raw);
  int32_t kb[kIt], kw[kIt], kr[kIt];
  int64_t h, nb;
  unit_expand(L, S, big_list, nbig, unit_ptr, bkt_ptr, blockIdx.x, &h, &nb, kb, kw, kr);
  const int64_t b0 = bkt_ptr[h];
  if (nb <= 8192) {
    for (int i = threadIdx.x; i < nb; i += kT) S.hist[i] = 0;
    __syncthreads();
    int rank[kIt];
#pragma unroll
    for (int k = 0; k < kIt; ++k) rank[k] = kb[k] >= 0 ? atomicAdd(&S.hist[kr[k]], 1) : 0;
    __syncthreads();
    for (int i = threadIdx.x; i < nb; i += kT) {
      int c = S.hist[i];
      S.base[i] = c ? bkt_off[b0 + i] + atomicAdd(bkt_cur + b0 + i, (unsigned)c) : 0;
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < kIt; ++k)
      if (kb[k] >= 0) {
        int64_t q = S.base[kr[k]] + rank[k];
        pb[q] = kb[k];
        pw[q] = kw[k];
      }
  } else {
#pragma unroll
    for (int k = 0; k < kIt; ++k)
      if (kb[k] >= 0) {
        int64_t q = bkt_off[b0 + kr[k]] + atomicAdd(bkt_cur + b0 + kr[k], 1u);
        pb[q] = kb[k];
        pw[q] = kw[k];
      }
  }
}

// Buckets with more than kCap entries: exact hash with int64 sums over adaptive
// key sub-ranges, bitonic sort per sub-range, sorted uniques into scratch.
struct FbSmem {
  int32_t key[kFbTab];
  unsigned long long val[kFbTab];
  unsigned nkeys, nout;
  int64_t job;
};

template <typename V>
__device__ void block_bitonic(int32_t *key, V *val, int N) {
  for (int size = 2; size <= N; size <<= 1) {
    for (int stride = size >> 1; stride > 0; stride >>= 1) {
      for (int i = threadIdx.x; i < (N >> 1); i += blockDim.x) {
        int lo = 2 * i - (i & (stride - 1));
        int hi = lo + stride;
        bool asc = (lo & size) == 0;
        int32_t kl = key[lo], kh = key[hi];
        if ((kl > kh) == asc) {
          key[lo] = kh;
          key[hi] = kl;
          V tv = val[lo];
          val[lo] = val[hi];
          val[hi] = tv;
        }
      }
      __syncthreads();
    }
  }
}

__global__ void __launch_bounds__(kT) k_bucket_fallback(int64_t n_c, const int64_t *__restrict__ jobs, int64_t njobs,
                                                        const int32_t *__restrict__ job_rn,  // (sub, nb) per job
                                                        const int64_t *__restrict__ bkt_off,
                                                        const int32_t *__restrict__ pb, const int32_t *__restrict__ pw,
                                                        const int64_t *__restrict__ fb_off, int32_t *__restrict__ fb_cnt,
                                                        int32_t *__restrict__ fb_b, int32_t *__restrict__ fb_w,
                                                        unsigned *__restrict__ ticket, int *__restrict__ err) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  FbSmem &S = *reinterpret_cast<FbSmem *>(smem_raw);
  while (true) {
    if (threadIdx.x == 0) S.job = (int64_t)atomicAdd(ticket, 1u);
    __syncthreads();
    const int64_t j = S.job;
    if (j >= njobs) return;
    const int64_t bk = jobs[j];
    const int64_t q0 = bkt_off[bk], q1 = bkt_off[bk + 1];
    int32_t lo, hi;
    bucket_range(job_rn[2 * j], job_rn[2 * j + 1], n_c, &lo, &hi);
    const int64_t out = fb_off[bk];
    int64_t written = 0;
    int nsub = 1, sub = 0;
    while (sub < nsub) {
      const int64_t slo = lo + ((int64_t)hi - lo) * sub / nsub, shi = lo + ((int64_t)hi - lo) * (sub + 1) / nsub;
      for (int s = threadIdx.x; s < kFbTab; s += kT) { S.key[s] = kEmpty; S.val[s] = 0; }
      if (threadIdx.x == 0) S.nkeys = 0;
      __syncthreads();
      for (int64_t q = q0 + threadIdx.x; q < q1; q += kT) {
        int32_t b = pb[q];
        if (b < slo || b >= shi) continue;
        if (((volatile unsigned *)&S.nkeys)[0] > kFbCap) break;
        unsigned s = hslot(b, kFbTab - 1);
        while (true) {
          int32_t k = ((volatile int32_t *)S.key)[s];
          if (k == b) { atomicAdd(S.val + s, (unsigned long long)pw[q]); break; }
          if (k == kEmpty) {
            int32_t old = atomicCAS(S.key + s, kEmpty, b);
            if (old == kEmpty) atomicAdd(&S.nkeys, 1u);
            if (old == kEmpty || old == b) { atomicAdd(S.val + s, (unsigned long long)pw[q]); break; }
          }
          s = (s + 1) & (kFbTab - 1);
        }
      }
      __syncthreads();
      if (S.nkeys > kFbCap) {  // too many distinct keys: restart with twice the sub-ranges
        nsub *= 2;
        sub = 0;
        written = 0;
        __syncthreads();
        continue;
      }
      if (threadIdx.x == 0) S.nout = 0;
      __syncthreads();
      for (int s = threadIdx.x; s < kFbTab; s += kT) {
        int32_t kk = S.key[s];
        if (kk != kEmpty) {
          unsigned long long v = S.val[s];
          if (v > 0x7fffffffull) atomicOr(err, 2);
          unsigned pos = atomicAdd(&S.nout, 1u);
          fb_b[out + written + pos] = kk;
          fb_w[out + written + pos] = (int32_t)v;
        }
      }
      __syncthreads();
      const int n_here = (int)S.nout;
      int N = 1;
      while (N < n_here) N <<= 1;
      int32_t *tk = S.key;
      int32_t *tv = reinterpret_cast<int32_t *>(S.val);
      for (int i = threadIdx.x; i < N; i += kT) {
        tk[i] = i < n_here ? fb_b[out + written + i] : INT32_MAX;
        tv[i] = i < n_here ? fb_w[out + written + i] : 0;
      }
      __syncthreads();
      block_bitonic<int32_t>(tk, tv, N);
      for (int i = threadIdx.x; i < n_here; i += kT) {
        fb_b[out + written + i] = tk[i];
        fb_w[out + written + i] = tv[i];
      }
      written += n_here;
      ++sub;
      __syncthreads();
    }
    if (threadIdx.x == 0) fb_cnt[bk] = (int32_t)written;
    __syncthreads();
  }
}

// fallback jobs: buckets with more than kCap entries
__global__ void k_fb_jobs(int64_t nbig, const int64_t *__restrict__ bkt_ptr, const int64_t *__restrict__ bkt_off,
                          int64_t *__restrict__ jobs, int32_t *__restrict__ job_rn, unsigned *__restrict__ njobs,
                          int32_t *__restrict__ fb_cnt, int64_t *__restrict__ fb_off,
                          unsigned long long *__restrict__ fb_total) {
  int64_t h = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (h >= nbig) return;
  const int64_t b0 = bkt_ptr[h], b1 = bkt_ptr[h + 1];
  for (int64_t k = b0; k < b1; ++k) {
    int64_t c = bkt_off[k + 1] - bkt_off[k];
    if (c > kCap) {
      unsigned j = atomicAdd(njobs, 1u);
      jobs[j] = k;
      job_rn[2 * j] = (int32_t)(k - b0);
      job_rn[2 * j + 1] = (int32_t)(b1 - b0);
      fb_off[k] = (int64_t)atomicAdd(fb_total, (unsigned long long)c);
      fb_cnt[k] = 0;
    } else {
      fb_cnt[k] = -1;
    }
  }
}

// ------------------------------------------------------------ a9 DENSE path
// Persistent CTAs take units in order; the shared-memory int32 accumulator of
// the current row is merged into dense[h] (int64) when the row changes or the
// running weight could exceed int32 (exact).
struct DenseArgs {
  Layout L;
  const int32_t *big_list;
  int64_t nbig;
  const int64_t *unit_ptr;
  int64_t nunits;
  unsigned *ticket;
  unsigned long long *dense;  // [nbig][n_c] (zeroed)
};

__global__ void __launch_bounds__(kT) k_dense_accum(DenseArgs A) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  MemberTab &T = *reinterpret_cast<MemberTab *>(smem_raw);
  int32_t *acc = reinterpret_cast<int32_t *>(smem_raw + sizeof(MemberTab));
  __shared__ int64_t s_unit;
  const Layout &L = A.L;
  const int nc = (int)L.n_c;
  for (int b = threadIdx.x; b < nc; b += kT) acc[b] = 0;
  int64_t cur_h = -1;
  long long running = 0;  // weight accumulated since the last merge
  while (true) {
    if (threadIdx.x == 0) s_unit = (int64_t)atomicAdd(A.ticket, 1u);
    __syncthreads();
    const int64_t unit = s_unit;
    const int64_t h = unit < A.nunits ? last_le(A.unit_ptr, 0, A.nbig, unit) : -1;
    int32_t kb[kIt], kw[kIt], kr[kIt];
    int a = -1;
    if (h >= 0) {
      a = A.big_list[h];
      const int64_t P0 = L.upos(a) + (unit - A.unit_ptr[h]) * kCap;
      const int64_t Pend = L.upos(a + 1);
      const int nP = (int)((Pend - P0) < kCap ? (Pend - P0) : kCap);
      int64_t m0, m1;
      window_members(L, a, P0, nP, &m0, &m1);
      expand_window(L, T, P0, nP, m0, m1, nullptr, 1, kb, kw, kr);
    }
    long long usum = 0;  // exact weight of this unit
    if (h >= 0) {
#pragma unroll
      for (int k = 0; k < kIt; ++k)
        if (kb[k] >= 0 && kb[k] != a) usum += kw[k];
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) usum += __shfl_xor_sync(0xffffffffu, usum, o);
    __shared__ long long s_w[kT / 32];
    if ((threadIdx.x & 31) == 0) s_w[threadIdx.x >> 5] = usum;
    __syncthreads();
    long long unit_w = 0;
    for (int w = 0; w < kT / 32; ++w) unit_w += s_w[w];
    __syncthreads();
    if (cur_h >= 0 && (h != cur_h || running + unit_w > 0x7fffffffLL)) {  // merge the accumulator
      unsigned long long *dst = A.dense + cur_h * (int64_t)nc;
      for (int b = threadIdx.x; b < nc; b += kT) {
        int32_t v = acc[b];
        if (v) { atomicAdd(dst + b, (unsigned long long)(uint32_t)v); acc[b] = 0; }
      }
      running = 0;
      __syncthreads();
    }
    if (h < 0) return;
    cur_h = h;
    running += unit_w;
#pragma unroll
    for (int k = 0; k < kIt; ++k)
      if (kb[k] >= 0 && kb[k] != a) atomicAdd(acc + kb[k], kw[k]);
    __syncthreads();
  }
}

// ---------------------------------------------------------------- driver
size_t ws_bytes_construct(int64_t n, int64_t nnz, int64_t n_c) {
  (void)nnz;
  size_t b = 0;
  b += ws_bytes(n_c + 1, 4);      // mcount
  b += ws_bytes(n_c + 1, 8);      // vw64
  b += ws_bytes(n_c + 1, 8);      // member_ptr
  b += ws_bytes(n + 1, 4);        // members
  b += ws_bytes(n + 1, 8);        // mpre
  b += ws_bytes(n_c + 1, 8);      // window scan
  b += ws_bytes(n_c + 1, 8);      // blk_ptr
  b += 2 * ws_bytes(n_c + 1, 4);  // big_list, big_idx
  b += 2 * ws_bytes(n_c + 1, 8);  // unit_ptr, bkt_ptr
  b += ws_bytes(64, 4) + ws_bytes(32, 8);
  b += 6 * scan_ws_bytes(n > n_c ? n : n_c);
  return b;
}

int build_coarse_impl(hec_ctx *ctx, const hec_graph *g, const int32_t *M, int64_t n_c, CoarseOut *out) {
  cudaStream_t s = ctx->stream;
  const int64_t n = g->n;
  out->n_c = n_c;
  out->nnz_c = 0;
  if (n_c <= 0 || n_c > n) {
    if (n == 0 && n_c == 0) {
      HEC_TRY(dev_alloc(ctx, (void **)&out->row_ptr, sizeof(int64_t)));
      HEC_CUDA_TRY(cudaMemsetAsync(out->row_ptr, 0, sizeof(int64_t), s));
      return HEC_OK;
    }
    set_error("build_coarse_graph: n_c=%lld out of range for n=%lld", (long long)n_c, (long long)n);
    return HEC_EINVAL;
  }
  unsigned *mcount = ws_take<unsigned>(ctx, n_c + 1);
  unsigned long long *vw64 = ws_take<unsigned long long>(ctx, n_c + 1);
  int64_t *member_ptr = ws_take<int64_t>(ctx, n_c + 1);
  int32_t *members = ws_take<int32_t>(ctx, n + 1);
  int64_t *mpre = ws_take<int64_t>(ctx, n + 1);
  int64_t *Sw = ws_take<int64_t>(ctx, n_c + 1);
  int64_t *blk_ptr = ws_take<int64_t>(ctx, n_c + 1);
  int32_t *big_list = ws_take<int32_t>(ctx, n_c + 1);
  int32_t *big_idx = ws_take<int32_t>(ctx, n_c + 1);
  int64_t *unit_ptr = ws_take<int64_t>(ctx, n_c + 1);
  int64_t *bkt_ptr = ws_take<int64_t>(ctx, n_c + 1);
  // counts: [0] nbig [1] rows ticket [2] dense ticket [3] fallback ticket [4] fallback jobs
  unsigned *counts = ws_take<unsigned>(ctx, 64);
  // scal: [0] err bits [1] small volume [2] big volume [4] nbig [5] nunits [6] nbkt [7] nblocks
  //       [9] fallback jobs [10] fallback total
  int64_t *scal = ws_take<int64_t>(ctx, 32);
  ScanTiles st[6];
  for (auto &x : st) x = take_scan_tiles(ctx, n > n_c ? n : n_c);
  if (!mcount || !vw64 || !member_ptr || !members || !mpre || !Sw || !blk_ptr || !big_list || !big_idx ||
      !unit_ptr || !bkt_ptr || !counts || !scal || !st[5].desc) {
    set_error("workspace under-reserved (construct)");
    return HEC_EINVAL;
  }
  int *err = reinterpret_cast<int *>(scal);
  HEC_CUDA_TRY(cudaMemsetAsync(mcount, 0, sizeof(unsigned) * (n_c + 1), s));
  HEC_CUDA_TRY(cudaMemsetAsync(vw64, 0, sizeof(unsigned long long) * (n_c + 1), s));
  HEC_CUDA_TRY(cudaMemsetAsync(counts, 0, sizeof(unsigned) * 64, s));
  HEC_CUDA_TRY(cudaMemsetAsync(scal, 0, sizeof(int64_t) * 32, s));
  const double dn = (double)n, dnc = (double)n_c;
  // ---- a7
  int ph = phase_begin(ctx, "bucket", 16.0 * dn + 4.0 * dnc);
  if (n > 0) {
    k_member_count<<<nblk(n, 256), 256, 0, s>>>(n, M, n_c, g->vwgt, mcount, vw64, err);
    HEC_LAUNCH_CHECK();
  }
  HEC_TRY(chained_scan(ctx, n_c, CountIn{mcount}, PtrOut{member_ptr}, st[0], member_ptr + n_c));
  if (n > 0) {
    k_member_fill<<<nblk(n, 256), 256, 0, s>>>(n, n_c, M, member_ptr, mcount, members);
    HEC_LAUNCH_CHECK();
  }
  HEC_TRY(chained_scan(ctx, n, DegIn{members, g->row_ptr, member_ptr + n_c}, PtrOut{mpre}, st[1], mpre + n));
  Layout L{n_c, member_ptr, members, mpre, g->row_ptr, g->col, g->wgt, M};
  k_big_rows<<<nblk(n_c, 256), 256, 0, s>>>(L, big_list, big_idx, counts + 0,
                                            reinterpret_cast<unsigned long long *>(scal + 1));
  HEC_LAUNCH_CHECK();
  HEC_TRY(chained_scan(ctx, n_c, RowWeightIn{L}, PtrOut{Sw}, st[2], Sw + n_c));
  const bool dense = n_c <= kDenseMax;
  HEC_TRY(chained_scan(ctx, n_c, BlockCountIn{L, Sw, dense}, PtrOut{blk_ptr}, st[3], blk_ptr + n_c));
  HEC_CUDA_TRY(cudaMemcpyAsync(scal + 4, counts + 0, sizeof(unsigned), cudaMemcpyDeviceToDevice, s));
  phase_end(ctx, ph);
  int64_t r0[5];
  HEC_TRY(read_scalars(ctx, scal, 5, r0));
  if ((int)(r0[0] & 0xffffffff) & 1) {
    set_error("build_coarse_graph: M has values outside [0, n_c)");
    return HEC_EINVAL;
  }
  const int64_t small_vol = r0[1], big_vol = r0[2];
  const int64_t nbig = r0[4] & 0xffffffffLL;
  if (nbig > 0) {
    HEC_TRY(chained_scan(ctx, nbig, UnitsIn{L, big_list}, PtrOut{unit_ptr}, st[4], unit_ptr + nbig));
    if (!dense) HEC_TRY(chained_scan(ctx, nbig, BucketsIn{L, big_list}, PtrOut{bkt_ptr}, st[5], bkt_ptr + nbig));
    HEC_CUDA_TRY(cudaMemcpyAsync(scal + 5, unit_ptr + nbig, sizeof(int64_t), cudaMemcpyDeviceToDevice, s));
    if (!dense) HEC_CUDA_TRY(cudaMemcpyAsync(scal + 6, bkt_ptr + nbig, sizeof(int64_t), cudaMemcpyDeviceToDevice, s));
  }
  HEC_CUDA_TRY(cudaMemcpyAsync(scal + 7, blk_ptr + n_c, sizeof(int64_t), cudaMemcpyDeviceToDevice, s));
  int64_t r1[3];
  HEC_TRY(read_scalars(ctx, scal + 5, 3, r1));
  const int64_t nunits = r1[0], nbkt = r1[1], nblocks = r1[2];
  ctx->stats.huge_rows = nbig;
  ctx->stats.dense_rows = dense ? nbig : 0;

  // ---- second arena: block list, look-back descriptors, skew-path buffers
  {
    size_t b2 = ws_bytes(nblocks + 1, sizeof(BlockDesc)) + ws_bytes(nblocks + 1, 8);
    if (nbig > 0 && dense) b2 += ws_bytes((size_t)nbig * n_c, 8);
    if (nbig > 0 && !dense) {
      b2 += 2 * ws_bytes(nbkt + 1, 4) + 2 * ws_bytes(nbkt + 1, 8) + ws_bytes(nbkt + 1, 4);
      b2 += 4 * ws_bytes((size_t)big_vol + 1, 4) + scan_ws_bytes(nbkt);
      b2 += ws_bytes(nbkt + 1, 8) + ws_bytes(2 * nbkt + 2, 4);
    }
    HEC_TRY(arena_reserve(ctx, &ctx->ws2, b2));
    ctx->ws2.used = 0;
  }
  Arena &W2 = ctx->ws2;
  BlockDesc *blk = arena_take<BlockDesc>(W2, nblocks + 1);
  uint64_t *desc = arena_take<uint64_t>(W2, nblocks + 1);
  HEC_CUDA_TRY(cudaMemsetAsync(desc, 0, sizeof(uint64_t) * (nblocks + 1), s));
  k_block_desc<<<nblk(n_c, 256), 256, 0, s>>>(L, blk_ptr, big_idx, dense, blk);
  HEC_LAUNCH_CHECK();
  k_block_ends<<<nblk(nblocks, 256), 256, 0, s>>>(nblocks, n_c, blk);
  HEC_LAUNCH_CHECK();

  RowsArgs A{};
  A.L = L;
  A.blk = blk;
  A.nblocks = nblocks;
  A.ticket = counts + 1;
  A.desc = desc;
  A.vw64 = vw64;
  A.big_idx = big_idx;
  A.bkt_ptr = bkt_ptr;
  A.err = err;

  static bool attr = false;
  if (!attr) {
    HEC_CUDA_TRY(cudaFuncSetAttribute(k_rows, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(RowsSmem)));
    HEC_CUDA_TRY(cudaFuncSetAttribute(k_part_count, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                      (int)sizeof(PartSmem)));
    HEC_CUDA_TRY(cudaFuncSetAttribute(k_part_write, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                      (int)sizeof(PartSmem)));
    HEC_CUDA_TRY(cudaFuncSetAttribute(k_bucket_fallback, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                      (int)sizeof(FbSmem)));
    HEC_CUDA_TRY(cudaFuncSetAttribute(k_dense_accum, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                      (int)(sizeof(MemberTab) + 4 * kDenseMax)));
    attr = true;
  }

  // ---- a9 skewed rows
  const int ph_skew = phase_begin(ctx, "rows_skew", 8.0 * (double)big_vol);
  if (nbig > 0 && dense) {
    unsigned long long *dn_arr = arena_take<unsigned long long>(W2, (size_t)nbig * n_c);
    HEC_CUDA_TRY(cudaMemsetAsync(dn_arr, 0, sizeof(unsigned long long) * nbig * n_c, s));
    DenseArgs D{L, big_list, nbig, unit_ptr, nunits, counts + 2, dn_arr};
    k_dense_accum<<<ctx->num_sms, kT, sizeof(MemberTab) + 4 * (size_t)n_c, s>>>(D);
    HEC_LAUNCH_CHECK();
    A.dense = dn_arr;
  } else if (nbig > 0) {
    unsigned *bkt_cnt = arena_take<unsigned>(W2, nbkt + 1);
    unsigned *bkt_cur = arena_take<unsigned>(W2, nbkt + 1);
    int64_t *bkt_off = arena_take<int64_t>(W2, nbkt + 1);
    int64_t *fb_off = arena_take<int64_t>(W2, nbkt + 1);
    int32_t *fb_cnt = arena_take<int32_t>(W2, nbkt + 1);
    int32_t *pb = arena_take<int32_t>(W2, (size_t)big_vol + 1);
    int32_t *pw = arena_take<int32_t>(W2, (size_t)big_vol + 1);
    ScanTiles stb = take_scan_tiles(W2, nbkt);
    int64_t *jobs = arena_take<int64_t>(W2, nbkt + 1);
    int32_t *job_rn = arena_take<int32_t>(W2, 2 * nbkt + 2);
    int32_t *fb_b = arena_take<int32_t>(W2, (size_t)big_vol + 1);
    int32_t *fb_w = arena_take<int32_t>(W2, (size_t)big_vol + 1);
    if (!fb_w) { set_error("workspace under-reserved (buckets)"); return HEC_EINVAL; }
    HEC_CUDA_TRY(cudaMemsetAsync(bkt_cnt, 0, sizeof(unsigned) * (nbkt + 1), s));
    HEC_CUDA_TRY(cudaMemsetAsync(bkt_cur, 0, sizeof(unsigned) * (nbkt + 1), s));
    k_part_count<<<(unsigned)nunits, kT, sizeof(PartSmem), s>>>(L, big_list, nbig, unit_ptr, bkt_ptr, bkt_cnt);
    HEC_LAUNCH_CHECK();
    HEC_TRY(chained_scan(ctx, nbkt, CountIn{bkt_cnt}, PtrOut{bkt_off}, stb, bkt_off + nbkt));
    k_part_write<<<(unsigned)nunits, kT, sizeof(PartSmem), s>>>(L, big_list, nbig, unit_ptr, bkt_ptr, bkt_off,
                                                                bkt_cur, pb, pw);
    HEC_LAUNCH_CHECK();
    k_fb_jobs<<<nblk(nbig, 256), 256, 0, s>>>(nbig, bkt_ptr, bkt_off, jobs, job_rn, counts + 4, fb_cnt, fb_off,
                                             reinterpret_cast<unsigned long long *>(scal + 10));
    HEC_LAUNCH_CHECK();
    HEC_CUDA_TRY(cudaMemcpyAsync(scal + 9, counts + 4, sizeof(unsigned), cudaMemcpyDeviceToDevice, s));
    int64_t rj[1];
    HEC_TRY(read_scalars(ctx, scal + 9, 1, rj));
    const int64_t njobs = rj[0] & 0xffffffffLL;
    if (njobs > 0) {
      k_bucket_fallback<<<ctx->num_sms, kT, sizeof(FbSmem), s>>>(n_c, jobs, njobs, job_rn, bkt_off, pb, pw, fb_off,
                                                                fb_cnt, fb_b, fb_w, counts + 3, err);
      HEC_LAUNCH_CHECK();
    }
    A.bkt_off = bkt_off;
    A.pb_g = pb;
    A.pw_g = pw;
    A.fb_cnt = fb_cnt;
    A.fb_off = fb_off;
    A.fb_b = fb_b;
    A.fb_w = fb_w;
  }
  phase_end(ctx, ph_skew);

  // ---- outputs: nnz_c is known only after the ordered pass; allocate the upper
  // bound sum(U) <= nnz (the tail beyond nnz_c is never read).
  const int64_t cap_out = small_vol + big_vol;
  HEC_TRY(dev_alloc(ctx, (void **)&out->row_ptr, sizeof(int64_t) * (n_c + 1)));
  HEC_TRY(dev_alloc(ctx, (void **)&out->col, sizeof(int32_t) * (cap_out > 0 ? cap_out : 1)));
  HEC_TRY(dev_alloc(ctx, (void **)&out->wgt, sizeof(int32_t) * (cap_out > 0 ? cap_out : 1)));
  HEC_TRY(dev_alloc(ctx, (void **)&out->vwgt, sizeof(int32_t) * n_c));
  A.row_ptr_c = out->row_ptr;
  A.col_c = out->col;
  A.wgt_c = out->wgt;
  A.vwgt_c = out->vwgt;
  const int ph_rows = phase_begin(ctx, "rows", 8.0 * (double)small_vol);
  {
    int grid = ctx->num_sms * 2;
    if (nblocks < grid) grid = (int)(nblocks > 0 ? nblocks : 1);
    k_rows<<<grid, kT, sizeof(RowsSmem), s>>>(A);
    HEC_LAUNCH_CHECK();
  }
  phase_end(ctx, ph_rows);
  HEC_CUDA_TRY(cudaMemcpyAsync(scal + 12, out->row_ptr + n_c, sizeof(int64_t), cudaMemcpyDeviceToDevice, s));
  int64_t r2[13];
  HEC_TRY(read_scalars(ctx, scal, 13, r2));
  out->nnz_c = r2[12];
  phase_set_bytes(ctx, ph_rows, 8.0 * (double)small_vol + 8.0 * (double)out->nnz_c + 12.0 * dnc);
  if ((int)(r2[0] & 0xffffffff) & 2) {
    set_error("build_coarse_graph: a coarse weight exceeds INT32_MAX");
    return HEC_EOVERFLOW;
  }
  ctx->stats.nnz_c = out->nnz_c;
  return HEC_OK;
}

}  // namespace hec
