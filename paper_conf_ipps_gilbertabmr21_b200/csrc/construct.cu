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
//  a8  expansion (k_expand2): every entry's (b = M[v], w) staged once at its
//      member-edge position (coalesced runs per coarse row); rows with U <= 60
//      -> warp pieces (construct_pieces.cu: register bitonic sort + merge), rows
//      with U <= 4096 -> rank items (construct_hrank.cu: smem hash merge +
//      order-preserving bucket rank; the sort path HEC_BUILD_SORT uses the
//      bucket-sort blocks of construct_rows.cu instead).
//  a9  skewed rows (U > 4096):
//        BUCKET  (n_c > 32768): the row's staged pairs are partitioned by key
//                range into bins of ~1024 entries (k_part_count / k_part_write,
//                the paper's segmented global sort alternative, L324); each bin
//                is a rank item, direct-indexed (k_drank) when its key range is
//                at most 4096 keys.
//        DENSE   (n_c <= 32768): persistent CTAs walk the row's members and
//                accumulate into a shared-memory dense array (k_dense_accum2),
//                merged into a dense row read back in key order (no sort).
//  a10 output placement: every work block stages its sorted distinct entries
//      (in place over its input) and counts them; an exclusive scan of the
//      block counts gives each block its output offset, and k_place copies the
//      staged entries into the final CSR (construct_rows.cu).
#include <stdlib.h>

#include "construct_common.cuh"

namespace hec {

constexpr int kFbTab = 16384;      // fallback hash slots (int64 values)
constexpr int kFbCap = 8192;       // fallback distinct keys per sub-range pass

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
                              int32_t *__restrict__ members, const int64_t *__restrict__ row_ptr,
                              int64_t *__restrict__ mstart) {
  int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (u >= n) return;
  int32_t a = M[u];
  if (a < 0 || a >= n_c) return;  // reported through err by k_member_count
  unsigned k = atomicSub(mcount + a, 1u) - 1u;
  members[member_ptr[a] + k] = (int32_t)u;
  mstart[member_ptr[a] + k] = row_ptr[u];
}

struct BlkCntIn {
  const int32_t *c;
  __device__ __forceinline__ int64_t operator()(int64_t i) const { return c[i]; }
};
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

// Row classes by member-edge volume U (bound on the row's length):
//   U <= kPieceMax                  warp pieces (windows of kPieceWin, weight U + kPieceRowW)
//   kPieceMax < U <= big_thr        CTA work blocks (windows of kWin, weight U + kRowW)
//   U > big_thr                     skewed: key-range buckets (BUCKET mode, big_thr =
//                                   kPieceMax) or dense accumulation (DENSE mode)
static int64_t big_threshold_host(bool dense) { return dense ? kSmallMax : kPieceMax; }

struct RowWeightIn {
  Layout L;
  int64_t big_thr;
  __device__ __forceinline__ int64_t operator()(int64_t a) const {
    if (!L.active(a)) return 0;
    int64_t U = L.U(a);
    if (U <= kPieceMax) return U + kPieceRowW;
    return U <= big_thr ? U + kRowW : 0;
  }
};

// big rows: list (unordered) + row -> list index; member-edge volume per class
__global__ void k_big_rows(Layout L, int64_t big_thr, int32_t *__restrict__ big_list, int32_t *__restrict__ big_idx,
                           unsigned *__restrict__ nbig, unsigned long long *__restrict__ vol) {
  int64_t a = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  bool in = a < L.n_c;
  const bool act = in && L.active(a);
  int64_t U = act ? L.U(a) : 0;
  bool big = act && U > big_thr;
  unsigned m = __ballot_sync(0xffffffffu, big);
  int lane = threadIdx.x & 31;
  unsigned base = 0;
  if (m) {
    int leader = __ffs(m) - 1;
    if (lane == leader) {
      base = atomicAdd(nbig, (unsigned)__popc(m));
      atomicAdd(vol + 3, (unsigned long long)__popc(m));  // the host's copy (scal[4])
    }
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
  unsigned long long mx = act ? (unsigned long long)U : 0ull;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const unsigned long long y = __shfl_xor_sync(0xffffffffu, mx, o);
    mx = y > mx ? y : mx;
  }
  if (lane == 0) {
    if (vs) atomicAdd(vol + 0, vs);
    if (vb) atomicAdd(vol + 1, vb);
    if (mx) atomicMax(vol + 2, mx);  // scal[3]: the largest U (host skips empty rank classes)
  }
}

constexpr int kPartHist = 8192;  // buckets per skewed row (bounds the partition's smem tables)
constexpr int kUnit = 32768;     // member-edge positions per partition CTA

__host__ __device__ __forceinline__ int64_t row_buckets(int64_t U, int64_t n_c, bool rbm, int64_t bin_avg) {
  const int64_t avg = rbm ? bin_avg : kBucketAvg;
  int64_t nb = (U + avg - 1) / avg;
  // rows holding >= 1/16 of the key range in entries: bins no wider than
  // kDirectR keys (>= 256 entries each on average) for the direct-indexed kernel
  if (rbm && U >= n_c / 16 && nb < (n_c + kDirectR - 1) / kDirectR) nb = (n_c + kDirectR - 1) / kDirectR;
  // k_rbm (items with too many distinct keys) needs bins no wider than kRbmRange keys
  if (rbm && nb < (n_c + kRbmRange - 1) / kRbmRange) nb = (n_c + kRbmRange - 1) / kRbmRange;
  if (nb > kPartHist) nb = kPartHist;
  if (nb > n_c) nb = n_c;
  return nb < 1 ? 1 : nb;
}
__host__ __device__ __forceinline__ int64_t dense_chunks(int64_t n_c) { return (n_c + kCap - 1) / kCap; }

// number of work blocks starting at row a
struct BlockCountIn {
  Layout L;
  const int64_t *S;  // exclusive scan of RowWeightIn
  bool dense;
  int64_t big_thr;
  bool rbm;  // class-1 rows are single-row bitmap-rank items
  __device__ __forceinline__ int cls(int64_t U) const {
    return U <= kPieceMax ? 0 : (U <= big_thr ? 1 : 2);
  }
  __device__ __forceinline__ int64_t operator()(int64_t a) const {
    if (!L.active(a)) return 0;
    const int64_t U = L.U(a);
    const int c = cls(U);
    if (c == 2) return dense ? dense_chunks(L.n_c) : row_buckets(U, L.n_c, rbm, L.bin_avg);
    if (c == 1 && rbm) return 1;
    if (a == L.a_lo || cls(L.U(a - 1)) != c) return 1;
    const int64_t win = c == 0 ? kPieceWin : kWin;  // rows of one class are contiguous in S
    return (S[a] / win) != (S[a - 1] / win) ? 1 : 0;
  }
};

// descriptors of PIECE / SMALL blocks and DENSE chunks (BUCKET blocks: k_bucket_blocks)
__global__ void k_block_desc(Layout L, const int64_t *__restrict__ blk_ptr, const int32_t *__restrict__ big_idx,
                             bool dense, bool rbm, BlockDesc *__restrict__ blk) {
  int64_t a = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (a >= L.n_c) return;
  int64_t b0 = blk_ptr[a], b1 = blk_ptr[a + 1];
  if (b1 == b0) return;
  if (big_idx[a] >= 0) {
    // BUCKET bins are (re)written by k_bucket_blocks after the partition; their
    // kind is set here already so that work split by kind before then is exact
    const int32_t kind = dense ? B_DENSE : B_BUCKET;
    for (int64_t k = b0; k < b1; ++k) blk[k] = BlockDesc{kind, (int32_t)a, (int32_t)a + 1, (int32_t)(k - b0)};
  } else {
    const int64_t U = L.U(a);
    if (U <= kPieceMax) blk[b0] = BlockDesc{B_PIECE, (int32_t)a, -1, 0};
    else if (rbm) blk[b0] = BlockDesc{B_RBM, (int32_t)a, (int32_t)a + 1, 0};
    else blk[b0] = BlockDesc{B_SMALL, (int32_t)a, -1, 0};
  }
}
// row1 of PIECE / SMALL blocks = first row of the next block (or the end of the range)
__global__ void k_block_ends(int64_t nblocks, int64_t a_hi, BlockDesc *__restrict__ blk) {
  int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (k >= nblocks) return;
  if (rows_kind(blk[k].kind)) blk[k].row1 = (k + 1 < nblocks) ? blk[k + 1].row0 : (int32_t)a_hi;
}

// ------------------------------------------------------- a9 BUCKET partition
// Work units: big row h (list index) split into ceil(U/unit) windows of `unit`
// member-edge positions (kUnit: partition, kCap: dense accumulation);
// unit_ptr = exclusive scan over big rows.
// Rows with U <= min_u get no units (BUCKET mode: partitioned by one warp).
// UnitsIn / BucketsIn run over the n_c upper bound of the big-row count (read
// on the device) so that their totals come back in the same host read as the
// volumes: entries h >= nbig contribute 0.
struct UnitsIn {
  Layout L;
  const int32_t *big_list;
  const unsigned *nbig;
  int64_t unit;
  int64_t min_u;
  __device__ __forceinline__ int64_t operator()(int64_t h) const {
    if (h >= (int64_t)*nbig) return 0;
    const int64_t U = L.U(big_list[h]);
    return U <= min_u ? 0 : (U + unit - 1) / unit;
  }
};
// Member-edge volume of big row h: prow = its exclusive scan places every
// skewed row's partitioned pairs at [prow[h], prow[h] + U) (self entries leave
// a gap at the end), so a row's bin offsets need no global scan.
struct RowUIn {
  Layout L;
  const int32_t *big_list;
  __device__ __forceinline__ int64_t operator()(int64_t h) const { return L.U(big_list[h]); }
};
constexpr int64_t kWarpRowMax = 4096;  // skewed rows up to this volume: one warp partitions the row
constexpr int kWarpBins = (int)((kWarpRowMax + 31) / 32);  // row_buckets(kWarpRowMax) with kBucketAvg 32
struct BucketsIn {
  Layout L;
  const int32_t *big_list;
  const unsigned *nbig;
  bool rbm;
  __device__ __forceinline__ int64_t operator()(int64_t h) const {
    if (h >= (int64_t)*nbig) return 0;
    return row_buckets(L.U(big_list[h]), L.n_c, rbm, L.bin_avg);
  }
};

// Segment -> owner table: out[k] = h for k in [ptr[h], ptr[h+1]) (a warp per
// segment), replacing per-thread binary searches over the segment offsets.
__global__ void k_seg_fill(int64_t nseg, const int64_t *__restrict__ ptr, int32_t *__restrict__ out) {
  const int64_t h = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  if (h >= nseg) return;
  const int lane = threadIdx.x & 31;
  for (int64_t k = ptr[h] + lane; k < ptr[h + 1]; k += 32) out[k] = (int32_t)h;
}

// ------------------------------------------------------------ expansion
// Every member-edge position p in [P_lo, P_hi) (the active rows) gets its
// fine entry's (b = M[v], w): Sb/Sw[p - P_lo].  One streaming pass with warp-level
// member walks (no CTA barriers); all later construction kernels read these
// arrays with coalesced loads.  Self entries are kept (b == own row): the
// consumers know their row and drop them.
constexpr int kXT = 256;       // threads per CTA
constexpr int kXChunk = 4096;  // positions per warp task (most; small volumes use less, >= kXChunkMin)
constexpr int kXChunkMin = 256;

// Expansion (k_expand2): every entry of the rows not walked by the DENSE
// accumulation is staged once, as (b = M[v], w), in member-edge space by
// x2_walk (construct_common.cuh): the partition, rank and piece kernels then
// read coalesced runs.  (Walking the member rows inside those kernels instead
// was measured 1.4x slower on C4: the walk's M[v] gathers need this kernel's
// occupancy to hide their latency.)
// sink of the expansion: (M[v], w) to the staging at position - P_lo
// One-end storage (Alg 6 l.9 / l.17): the entry
// (a, b) stays in row a only at the end with the smaller degree estimate C',
// ties to the smaller coarse id (reading Z7); the other end's copy becomes a
// self entry and is dropped (its weight arrives by the transpose).
__device__ __forceinline__ bool one_end_keeps(const unsigned long long *__restrict__ Cp, int32_t a, int32_t b) {
  const unsigned long long ca = __ldg(Cp + a), cb = __ldg(Cp + b);
  return ca < cb || (ca == cb && a < b);
}

template <bool kOneEnd = false>
struct StageSink {
  static constexpr bool kRows = kOneEnd;
  const Layout &L;
  int32_t *__restrict__ Sb, *__restrict__ Sw;
  int64_t P_lo;
  const unsigned long long *Cp;  // C' (one-end mode)
  template <int N, typename IdxT>
  __device__ __forceinline__ void store(int32_t (&b)[N], int32_t (&w)[N], const IdxT (&p)[N], unsigned ok) {
#pragma unroll
    for (int u = 0; u < N; ++u)
      if (ok & (1u << u)) { __stcs(Sb + ((int64_t)p[u] - P_lo), b[u]); __stcs(Sw + ((int64_t)p[u] - P_lo), w[u]); }
  }
  template <int N, typename IdxT>
  __device__ __forceinline__ void load(int32_t (&b)[N], int32_t (&w)[N], const IdxT (&e)[N], unsigned ok) {
#pragma unroll
    for (int u = 0; u < N; ++u)
      if (ok & (1u << u)) { b[u] = __ldcs(L.col + e[u]); w[u] = L.unit_w ? 1 : __ldcs(L.wgt + e[u]); }
#pragma unroll
    for (int u = 0; u < N; ++u)
      if (ok & (1u << u)) b[u] = __ldg(L.M + b[u]);
  }
  template <int N, typename IdxT>
  __device__ __forceinline__ void operator()(const IdxT (&e)[N], const IdxT (&p)[N], unsigned ok) {
    int32_t b[N], w[N];
    load(b, w, e, ok);
    store(b, w, p, ok);
  }
  template <int N, typename IdxT>
  __device__ __forceinline__ void operator()(const IdxT (&e)[N], const IdxT (&p)[N], unsigned ok,
                                             const int32_t (&row)[N]) {
    int32_t b[N], w[N];
    load(b, w, e, ok);
#pragma unroll
    for (int u = 0; u < N; ++u)
      if ((ok & (1u << u)) && b[u] != row[u] && !one_end_keeps(Cp, row[u], b[u])) b[u] = row[u];
    store(b, w, p, ok);
  }
};

// skip: big_idx in DENSE mode (those rows are expanded by k_dense_accum2), else nullptr
template <typename IdxT, int kPer, bool kOneEnd = false>
__global__ void __launch_bounds__(kXT) k_expand2(Layout L, const int64_t *__restrict__ mstart,
                                               int32_t *__restrict__ Sb, int32_t *__restrict__ Sw,
                                               const int32_t *__restrict__ skip, int64_t skip_thr,
                                               const unsigned long long *__restrict__ Cp, int64_t chunk) {
  const int64_t m_lo = L.member_ptr[L.a_lo], m_hi = L.member_ptr[L.a_hi];
  const int64_t P_lo = L.mpre[m_lo], P_hi = L.mpre[m_hi];
  const int64_t gw = ((int64_t)blockIdx.x * kXT + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * kXT) >> 5;
  StageSink<kOneEnd> sink{L, Sb, Sw, P_lo, Cp};
  for (int64_t P = P_lo + gw * chunk; P < P_hi; P += nw * chunk) {
    const int64_t Pend = P + chunk < P_hi ? P + chunk : P_hi;
    x2_walk<kPer, StageSink<kOneEnd>, kPer, IdxT>(L, mstart, m_lo, m_hi, P, Pend, skip, sink, skip_thr);
  }
}

// ------------------------------------------------------- a9 BUCKET partition
// One CTA per unit (<= kUnit positions of one skewed row): a shared-memory
// histogram over the row's key-range buckets (bucket = floor(b * nb / n_c)),
// flushed once per unit; the write pass reserves each bucket's slice of the unit
// with one global atomic and scatters with shared-memory cursors, so a bucket
// receives a contiguous run from every unit.  Offsets inside a row fit int32.
struct PartSmem {
  int32_t hist[kPartHist];
  int32_t base[kPartHist];  // slot cursor relative to the row's first bucket
};

struct PartArgs {
  Layout L;
  const int32_t *big_list;
  int64_t nbig;
  const int64_t *unit_ptr;  // units of kUnit positions
  const int32_t *unit_row;  // unit -> big row index
  const int64_t *bkt_ptr;
  const int32_t *Sb, *Sw;   // expanded entries, indexed from upos(a_lo)
};

struct UnitInfo {
  int64_t p0, p1;  // staging index range of the unit
  int64_t b0;      // first bucket of the row
  int32_t a;       // the row
  int32_t nb;      // buckets of the row
  float scale;     // nb / n_c
};

__device__ __forceinline__ UnitInfo unit_info(const PartArgs &A, int64_t unit) {
  const Layout &L = A.L;
  const int64_t h = A.unit_row[unit];
  UnitInfo u;
  u.a = A.big_list[h];
  const int64_t P_lo = L.upos(L.a_lo);
  const int64_t P0 = L.upos(u.a) + (unit - A.unit_ptr[h]) * kUnit;
  const int64_t Pe = L.upos(u.a + 1);
  u.p0 = P0 - P_lo;
  u.p1 = (P0 + kUnit < Pe ? P0 + kUnit : Pe) - P_lo;
  u.b0 = A.bkt_ptr[h];
  u.nb = (int32_t)(A.bkt_ptr[h + 1] - u.b0);
  u.scale = (float)u.nb / (float)L.n_c;
  return u;
}

// bucket of key b: floor(b * nb / n_c) in float arithmetic, clamped.  Any
// function works as long as it is monotone in b (buckets are key ranges, so the
// concatenation of sorted buckets is the sorted row) and identical in both passes.
__device__ __forceinline__ int part_bucket(const UnitInfo &u, int32_t b) {
  const int k = (int)__fmul_rz((float)b, u.scale);
  return k < u.nb - 1 ? k : u.nb - 1;
}

constexpr int kPartU = 16;  // loads in flight per thread in the partition passes

// Bucket of the entry, or -1 for a self entry (dropped, L280) / past the unit.
__device__ __forceinline__ int entry_bucket(const UnitInfo &u, int32_t b) {
  return b == u.a ? -1 : part_bucket(u, b);
}

// Slot of the entry in its bucket (shared-memory cursor), or -1.  (A
// __match_any_sync warp aggregation of equal buckets was measured slower: the
// passes are bound by per-unit latency, not by same-address replays.)
__device__ __forceinline__ int agg_add(int32_t *ctr, int bk) { return bk < 0 ? -1 : atomicAdd(ctr + bk, 1); }

// histogram of the unit's entries (self entries dropped) into S.hist
__device__ __forceinline__ void unit_hist(const PartArgs &A, const UnitInfo &u, PartSmem &S) {
  for (int i = threadIdx.x; i < u.nb; i += kT) S.hist[i] = 0;
  __syncthreads();
  const int32_t *Sb = A.Sb + u.p0;
  const int cnt = (int)(u.p1 - u.p0);  // <= kUnit
  // warp-uniform trip count: agg_add's __match_any_sync needs every lane
  for (int p = threadIdx.x; p - (int)(threadIdx.x & 31) < cnt; p += kPartU * kT) {
    int32_t b[kPartU];
#pragma unroll
    for (int j = 0; j < kPartU; ++j) b[j] = p + j * kT < cnt ? __ldcs(Sb + p + j * kT) : u.a;
#pragma unroll
    for (int j = 0; j < kPartU; ++j) agg_add(S.hist, entry_bucket(u, b[j]));
  }
  __syncthreads();
}

// The unit's slice of each bin is reserved here: the returned running count
// is the unit's offset inside the bin (ubase), so the write pass needs no
// second histogram.
__global__ void __launch_bounds__(kT) k_part_count(PartArgs A, unsigned *__restrict__ bkt_cnt,
                                                   int32_t *__restrict__ ubase) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  PartSmem &S = *reinterpret_cast<PartSmem *>(smem_raw);
  const UnitInfo u = unit_info(A, blockIdx.x);
  unit_hist(A, u, S);
  int32_t *ub = ubase + (int64_t)blockIdx.x * kPartHist;
  for (int i = threadIdx.x; i < u.nb; i += kT)
    if (S.hist[i]) ub[i] = (int32_t)atomicAdd(bkt_cnt + u.b0 + i, (unsigned)S.hist[i]);
}

__global__ void __launch_bounds__(kT) k_part_write(PartArgs A, const int64_t *__restrict__ bkt_off,
                                                   const int32_t *__restrict__ ubase, int32_t *__restrict__ pb,
                                                   int32_t *__restrict__ pw) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  PartSmem &S = *reinterpret_cast<PartSmem *>(smem_raw);
  const UnitInfo u = unit_info(A, blockIdx.x);
  const int64_t off0 = bkt_off[u.b0];
  const int32_t *ub = ubase + (int64_t)blockIdx.x * kPartHist;
  for (int i = threadIdx.x; i < u.nb; i += kT)  // (slots of bins the unit never hits stay unused)
    S.base[i] = (int32_t)(bkt_off[u.b0 + i] - off0) + ub[i];
  __syncthreads();
  const int32_t *Sb = A.Sb + u.p0, *Sw = A.Sw + u.p0;
  int32_t *pbr = pb + off0, *pwr = pw + off0;
  const int cnt = (int)(u.p1 - u.p0);
  for (int p = threadIdx.x; p - (int)(threadIdx.x & 31) < cnt; p += kPartU * kT) {
    int32_t b[kPartU], w[kPartU];
#pragma unroll
    for (int j = 0; j < kPartU; ++j) {
      const bool in = p + j * kT < cnt;
      b[j] = in ? __ldcs(Sb + p + j * kT) : u.a;
      w[j] = in ? __ldcs(Sw + p + j * kT) : 0;
    }
#pragma unroll
    for (int j = 0; j < kPartU; ++j) {
      const int q = agg_add(S.base, entry_bucket(u, b[j]));
      if (q >= 0) {
        pbr[q] = b[j];
        pwr[q] = w[j];
      }
    }
  }
}

// Skewed rows with U <= kWarpRowMax (<= kWarpBins bins): one warp counts the
// row's entries per bin in shared memory, scans the counts into the row's bin
// offsets (bkt_off = prow[h] + prefix, bkt_n = count) and scatters the pairs --
// count, offsets and scatter without a CTA barrier or a global scan.
constexpr int kPWT = 256;
__global__ void __launch_bounds__(kPWT) k_part_warp(PartArgs A, const int64_t *__restrict__ prow,
                                                    int64_t *__restrict__ bkt_off, unsigned *__restrict__ bkt_n,
                                                    int32_t *__restrict__ pb, int32_t *__restrict__ pw) {
  __shared__ int32_t hist[kPWT / 32][kWarpBins];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int64_t h = (blockIdx.x * (int64_t)kPWT + threadIdx.x) >> 5;
  if (h >= A.nbig) return;
  const Layout &L = A.L;
  UnitInfo u;
  u.a = A.big_list[h];
  const int64_t P_lo = L.upos(L.a_lo);
  const int64_t P0 = L.upos(u.a), U = L.upos(u.a + 1) - P0;
  if (U > kWarpRowMax) return;
  u.b0 = A.bkt_ptr[h];
  u.nb = (int32_t)(A.bkt_ptr[h + 1] - u.b0);
  u.scale = (float)u.nb / (float)L.n_c;
  int32_t *H = hist[wid];
  for (int i = lane; i < u.nb; i += 32) H[i] = 0;
  __syncwarp();
  const int32_t *Sb = A.Sb + (P0 - P_lo), *Sw = A.Sw + (P0 - P_lo);
  const int n = (int)U;
  for (int p = lane; p < n; p += 32) {
    const int32_t b = __ldg(Sb + p);
    if (b != u.a) atomicAdd(&H[part_bucket(u, b)], 1);
  }
  __syncwarp();
  // exclusive scan of the <= 128 bin counts (4 consecutive per lane)
  int c[4], tot = 0;
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    const int i = 4 * lane + j;
    c[j] = i < u.nb ? H[i] : 0;
    tot += c[j];
  }
  int x = tot;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  int run = x - tot;
  const int64_t base = prow[h];
  __syncwarp();
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    const int i = 4 * lane + j;
    if (i < u.nb) {
      H[i] = run;
      bkt_off[u.b0 + i] = base + run;
      bkt_n[u.b0 + i] = (unsigned)c[j];
    }
    run += c[j];
  }
  __syncwarp();
  for (int p = lane; p < n; p += 32) {
    const int32_t b = __ldg(Sb + p);
    if (b != u.a) {
      const int64_t q = base + atomicAdd(&H[part_bucket(u, b)], 1);
      pb[q] = b;
      pw[q] = __ldg(Sw + p);
    }
  }
}

// Bin offsets of the CTA-partitioned rows (U > kWarpRowMax): a warp scans the
// row's bin counts (from k_part_count) into bkt_off = prow[h] + prefix.
__global__ void k_row_bins(PartArgs A, const int64_t *__restrict__ prow, const unsigned *__restrict__ bkt_n,
                           int64_t *__restrict__ bkt_off) {
  const int lane = threadIdx.x & 31;
  const int64_t h = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  if (h >= A.nbig) return;
  const Layout &L = A.L;
  const int32_t a = A.big_list[h];
  if (L.U(a) <= kWarpRowMax) return;
  const int64_t b0 = A.bkt_ptr[h], b1 = A.bkt_ptr[h + 1];
  int64_t run = prow[h];
  for (int64_t k0 = b0; k0 < b1; k0 += 32) {
    const int64_t k = k0 + lane;
    const int64_t c = k < b1 ? (int64_t)bkt_n[k] : 0;
    int64_t x = c;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int64_t y = __shfl_up_sync(0xffffffffu, x, o);
      if (lane >= o) x += y;
    }
    if (k < b1) bkt_off[k] = run + x - c;
    run += __shfl_sync(0xffffffffu, x, 31);
  }
}

// Buckets with more than kCap entries: exact hash with int64 sums over adaptive
// key sub-ranges, bitonic sort per sub-range, sorted uniques into scratch.
struct FbSmem {
  int32_t key[kFbTab];
  unsigned long long val[kFbTab];
  unsigned nkeys, nout;
  int32_t kmin, kmax;
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

__global__ void __launch_bounds__(kT) k_bucket_fallback(const int64_t *__restrict__ jobs, int64_t njobs,
                                                        const int64_t *__restrict__ bkt_off,
                                                        const unsigned *__restrict__ bkt_n,
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
    const int64_t q0 = bkt_off[bk], q1 = q0 + bkt_n[bk];
    // key range of the bucket's entries (sub-ranges split it when a pass overflows)
    if (threadIdx.x == 0) { S.kmin = INT32_MAX; S.kmax = -1; }
    __syncthreads();
    {
      int32_t mn = INT32_MAX, mx = -1;
      for (int64_t q = q0 + threadIdx.x; q < q1; q += kT) {
        const int32_t b = pb[q];
        mn = min(mn, b);
        mx = max(mx, b);
      }
      atomicMin(&S.kmin, mn);
      atomicMax(&S.kmax, mx);
    }
    __syncthreads();
    const int32_t lo = S.kmin, hi = S.kmax + 1;
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

// Per bucket k (of big row h): its block descriptor, and a fallback job when it
// holds more than kCap entries.
__global__ void k_bucket_blocks(int64_t nbig, int64_t nbkt, const int32_t *__restrict__ big_list,
                                const int64_t *__restrict__ bkt_ptr, const int32_t *__restrict__ bin_row,
                                const unsigned *__restrict__ bkt_n,
                                const int64_t *__restrict__ blk_ptr, BlockDesc *__restrict__ blk,
                                int64_t *__restrict__ jobs, unsigned *__restrict__ njobs,
                                int32_t *__restrict__ fb_cnt, int64_t *__restrict__ fb_off,
                                unsigned long long *__restrict__ fb_total, int64_t fb_thr) {
  int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (k >= nbkt) return;
  const int64_t h = bin_row[k];
  const int64_t b0 = bkt_ptr[h];
  const int32_t a = big_list[h];
  blk[blk_ptr[a] + (k - b0)] = BlockDesc{B_BUCKET, a, a + 1, (int32_t)(k - b0)};
  const int64_t c = bkt_n[k];
  if (c > fb_thr) {
    unsigned j = atomicAdd(njobs, 1u);
    jobs[j] = k;
    fb_off[k] = (int64_t)atomicAdd(fb_total, (unsigned long long)c);
    fb_cnt[k] = 0;
  } else {
    fb_cnt[k] = -1;
  }
}

// Bin groups: consecutive bins of a skewed row form one piece while they start
// inside one window of kGroupWin entries (so a group of bins <= kGroupWin each
// holds < 2 kGroupWin entries); a bin above kGroupWin stands alone.  The group's
// first bin carries its block (count, staging at its first pair); the other
// bins' blocks are empty.
// Groups also break where the bins' key ranges cross a kGroupRange window, so a
// group of a dense enough row spans < 2 kGroupRange keys and takes the
// bitmap-rank path of k_pieces (bin k covers keys ~[k n_c / nb, (k+1) n_c / nb)).
constexpr int64_t kGroupRange = 16384;
__device__ __forceinline__ bool group_start(const int64_t *__restrict__ bkt_off, const unsigned *__restrict__ bkt_n,
                                            int64_t b0, int64_t b1, int64_t n_c, int64_t k) {
  if (k == b0) return true;
  const int64_t ck = bkt_n[k], cp = bkt_n[k - 1];
  if (ck > kGroupWin || cp > kGroupWin) return true;
  const int64_t nb = b1 - b0;
  if (((k - b0) * n_c / nb) / kGroupRange != ((k - 1 - b0) * n_c / nb) / kGroupRange) return true;
  return (bkt_off[k] - bkt_off[b0]) / kGroupWin != (bkt_off[k - 1] - bkt_off[b0]) / kGroupWin;
}

// Tier lists: warp pieces (PIECE blocks, bin groups of <= kPieceCap entries) and
// CTA blocks (SMALL, DENSE, larger bins).  Fallback bins are complete: their
// count is final here.  list_n: [0] warp list, [1] CTA list.
__global__ void k_tiers(Layout L, int64_t nblocks, const BlockDesc *__restrict__ blk, const int32_t *__restrict__ big_idx,
                        const int64_t *__restrict__ bkt_ptr, const int64_t *__restrict__ bkt_off,
                        const unsigned *__restrict__ bkt_n,
                        const int32_t *__restrict__ fb_cnt, int32_t *__restrict__ blk_cnt,
                        int64_t *__restrict__ grp_end,
                        WorkItem *__restrict__ list_w, int32_t *__restrict__ list_c, RbmItem *__restrict__ list_r,
                        RbmItem *__restrict__ list_r2, RbmItem *__restrict__ list_d, RbmItem *__restrict__ list_r3,
                        RbmItem *__restrict__ list_r4,
                        unsigned *__restrict__ list_n,
                        bool rbm, bool direct, int mode,
                        const unsigned long long *__restrict__ vw64, int *__restrict__ err) {
  const int64_t bi = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  int tier = -1;  // 0 warp, 1 CTA, 2 bitmap-rank CTA
  WorkItem it{0, (int32_t)bi, 0, 0, 0};
  RbmItem ri{};
  // mode 0: every block; 1: all but key-range bins; 2: bins only (split launch)
  const bool take = bi < nblocks && (mode == 0 || ((blk[bi].kind == B_BUCKET) == (mode == 2)));
  if (take) {
    const BlockDesc d = blk[bi];
    it.row0 = d.row0;
    // vertex weight of a skewed row (written by k_place): int32 bound
    if (!rows_kind(d.kind) && d.sub == 0 && vw64[d.row0] > 0x7fffffffull) atomicOr(err, ERR_OVERFLOW);
    if (d.kind == B_PIECE) {
      tier = 0;
      const int64_t p0 = L.upos(d.row0);
      it.base = p0 - L.upos(L.a_lo);
      it.n = (int32_t)(L.upos(d.row1) - p0);
      it.R = d.row1 - d.row0;
    } else if (d.kind == B_RBM || (rbm && d.kind == B_BUCKET)) {
      tier = 2;
      ri.bi = (int32_t)bi;
      ri.row = d.row0;
      if (d.kind == B_RBM) {
        const int64_t p0 = L.upos(d.row0);
        ri.src = p0 - L.upos(L.a_lo);
        ri.n = (int32_t)(L.upos(d.row0 + 1) - p0);
        ri.lo = 0;
        ri.hi = (int32_t)L.n_c;
        ri.bk = -1;
      } else {
        const int64_t h = big_idx[d.row0];
        const int64_t b0 = bkt_ptr[h], nb = bkt_ptr[h + 1] - b0, bk = b0 + d.sub;
        ri.src = bkt_off[bk];
        ri.n = (int32_t)bkt_n[bk];
        ri.lo = (int32_t)bin_lower(d.sub, nb, L.n_c);
        ri.hi = (int32_t)bin_lower(d.sub + 1, nb, L.n_c);
        ri.bk = (int32_t)bk;
      }
      // size class (k_tiers lists: list_r front/back, list_r2 front/back)
      tier = ri.n <= kHrMaxT ? 8 : ri.n <= kHrMaxS ? 7 : ri.n <= kHrMax0 ? 2 : ri.n <= kHrMax1 ? 3 : ri.n <= kHrMax2 ? 4 : 5;
      if (direct && ri.bk >= 0 && ri.hi - ri.lo <= kDirectR) tier = 6;  // direct-indexed bin
    } else if (d.kind != B_BUCKET) tier = 1;
    else {
      const int64_t h = big_idx[d.row0];
      const int64_t b0 = bkt_ptr[h], b1 = bkt_ptr[h + 1], bk = b0 + d.sub;
      if (fb_cnt[bk] >= 0) {
        blk_cnt[bi] = fb_cnt[bk];
      } else if (!group_start(bkt_off, bkt_n, b0, b1, L.n_c, bk)) {
        blk_cnt[bi] = 0;
      } else {
        int64_t e = bk + 1;
        while (e < b1 && !group_start(bkt_off, bkt_n, b0, b1, L.n_c, e)) ++e;
        grp_end[bi] = e;
        it.base = bkt_off[bk];
        it.n = (int32_t)(bkt_off[e - 1] + bkt_n[e - 1] - bkt_off[bk]);
        tier = it.n <= kPieceCap ? 0 : 1;
      }
    }
  }
  const int lane = threadIdx.x & 31;
  // list_n: [0] warp [1] CTA [2] list_r front [4] list_r back [5] list_r2 front [6] list_r2 back
  //         [8] list_d [3] list_r3 (n <= kHrMaxS) [12] list_r4 (n <= kHrMaxT)
#pragma unroll
  for (int q = 0; q < 9; ++q) {
    const unsigned m = __ballot_sync(0xffffffffu, tier == q);
    if (!m) continue;
    const int leader = __ffs(m) - 1;
    const int slot = q < 3 ? q : q < 6 ? q + 1 : q == 6 ? 8 : q == 7 ? 3 : 12;
    unsigned base = 0;
    if (lane == leader) base = atomicAdd(list_n + slot, (unsigned)__popc(m));
    base = __shfl_sync(0xffffffffu, base, leader);
    if (tier == q) {
      const int64_t pos = base + __popc(m & ((1u << lane) - 1));
      if (q == 2) list_r[pos] = ri;
      else if (q == 3) list_r[nblocks - pos] = ri;  // lists hold nblocks + 1 items
      else if (q == 4) list_r2[pos] = ri;
      else if (q == 5) list_r2[nblocks - pos] = ri;
      else if (q == 6) list_d[pos] = ri;
      else if (q == 7) list_r3[pos] = ri;
      else if (q == 8) list_r4[pos] = ri;
      else if (q) list_c[pos] = (int32_t)bi;
      else list_w[pos] = it;
    }
  }
}

// blocks flagged for the 64-bit pass
__global__ void k_wide_list(int64_t nblocks, const int32_t *__restrict__ need_wide, int32_t *__restrict__ list,
                            unsigned *__restrict__ n) {
  const int64_t bi = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (bi < nblocks && need_wide[bi]) list[atomicAdd(n, 1u)] = (int32_t)bi;
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
  const int32_t *unit_row;
  int64_t nunits;
  unsigned *ticket;
  unsigned long long *dense;  // [nbig][n_c] (zeroed)
  const unsigned long long *Cp;  // C' (one-end mode) or nullptr
};

constexpr int kDenseUnit2 = 32768;  // DENSE units: 2048 positions per warp, one barrier per unit

// DENSE rows fused with their expansion: a persistent CTA takes units of
// kDenseUnit2 member-edge positions of one big row; each warp walks its
// kDenseUnit2/16 positions of the row's member rows (x2_walk), gathers M[v] and
// adds w into the shared-memory accumulator of the row (uint32: a partial sum
// above INT32_MAX or a wrap means the coarse weight overflows -- ERR_OVERFLOW
// here or in k_rows); the accumulator is merged into dense[h] when the CTA
// moves to another row.  The staging is never written for these rows.
struct AccSink {
  static constexpr bool kRows = false;
  const Layout &L;
  uint32_t *acc;
  int32_t a;
  bool wrap;
  const unsigned long long *Cp;  // C' (one-end mode) or nullptr
  template <int N, typename IdxT>
  __device__ __forceinline__ void operator()(const IdxT (&e)[N], const IdxT (&p)[N], unsigned ok) {
    (void)p;
    int32_t b[N], w[N];
#pragma unroll
    for (int u = 0; u < N; ++u)
      if (ok & (1u << u)) { b[u] = __ldcs(L.col + e[u]); w[u] = L.unit_w ? 1 : __ldcs(L.wgt + e[u]); }
#pragma unroll
    for (int u = 0; u < N; ++u)
      if (ok & (1u << u)) b[u] = __ldg(L.M + b[u]);
#pragma unroll
    for (int u = 0; u < N; ++u)
      if ((ok & (1u << u)) && b[u] != a && (!Cp || one_end_keeps(Cp, a, b[u]))) {  // self entries dropped (L280)
        const uint32_t o = atomicAdd(acc + b[u], (uint32_t)w[u]);
        wrap |= o + (uint32_t)w[u] < o;
      }
  }
};

__global__ void __launch_bounds__(kT) k_dense_accum2(DenseArgs A, const int64_t *__restrict__ mstart,
                                                    int *__restrict__ err) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  uint32_t *acc = reinterpret_cast<uint32_t *>(smem_raw);
  __shared__ int64_t s_unit;
  const Layout &L = A.L;
  const int nc = (int)L.n_c;
  const int wid = threadIdx.x >> 5;
  constexpr int kSlice = kDenseUnit2 / (kT / 32);
  for (int b = threadIdx.x; b < nc; b += kT) acc[b] = 0u;
  int64_t cur_h = -1;
  bool wrap = false;
  while (true) {
    if (threadIdx.x == 0) s_unit = (int64_t)atomicAdd(A.ticket, 1u);
    __syncthreads();
    const int64_t unit = s_unit;
    const int64_t h = unit < A.nunits ? A.unit_row[unit] : -1;
    if (cur_h >= 0 && h != cur_h) {  // merge the accumulator of the previous row
      unsigned long long *dst = A.dense + cur_h * (int64_t)nc;
      for (int b = threadIdx.x; b < nc; b += kT) {
        const uint32_t v = acc[b];
        if (v) {
          if (v > 0x7fffffffu) wrap = true;
          atomicAdd(dst + b, (unsigned long long)v);
          acc[b] = 0u;
        }
      }
      __syncthreads();
    }
    if (h < 0) break;
    cur_h = h;
    const int32_t a = A.big_list[h];
    const int64_t P0 = L.upos(a) + (unit - A.unit_ptr[h]) * kDenseUnit2;
    const int64_t Pe = min(P0 + (int64_t)kDenseUnit2, L.upos(a + 1));
    const int64_t Pw = P0 + (int64_t)wid * kSlice;
    const int64_t Pwe = min(Pw + (int64_t)kSlice, Pe);
    AccSink sink{L, acc, a, false, A.Cp};
    if (Pw < Pwe) x2_walk<8>(L, mstart, L.member_ptr[a], L.member_ptr[a + 1], Pw, Pwe, nullptr, sink);
    wrap |= sink.wrap;
    __syncthreads();
  }
  if (wrap) atomicOr(err, ERR_OVERFLOW);
}

// ---------------------------------------------------------------- driver
size_t ws_bytes_construct(int64_t n, int64_t nnz, int64_t n_c) {
  (void)nnz;
  size_t b = 0;
  b += ws_bytes(n_c + 1, 4);      // mcount
  b += ws_bytes(n_c + 1, 8);      // vw64
  b += ws_bytes(n_c + 1, 8);      // member_ptr
  b += ws_bytes(n + 1, 4);        // members
  b += ws_bytes(n + 1, 8);        // mstart
  b += ws_bytes(n + 1, 8);        // mpre
  b += ws_bytes(n_c + 1, 8);      // window scan
  b += ws_bytes(n_c + 1, 8);      // blk_ptr
  b += 2 * ws_bytes(n_c + 1, 4);  // big_list, big_idx
  b += 2 * ws_bytes(n_c + 1, 8);  // unit_ptr, bkt_ptr
  b += ws_bytes(64, 4) + ws_bytes(32, 8);
  b += 6 * scan_ws_bytes(n > n_c ? n : n_c);
  return b;
}

int build_coarse_impl(hec_ctx *ctx, const hec_graph *g, const int32_t *M, int64_t n_c, CoarseOut *out,
                      int64_t a_lo, int64_t a_hi, const BuildOpts *opt) {
  const unsigned long long *Cp = opt ? opt->one_end_cp : nullptr;
  if (a_hi < 0) a_hi = n_c;
  cudaStream_t s = ctx->stream;
  const int64_t n = g->n;
  out->n_c = n_c;
  out->nnz_c = 0;
  if (n_c <= 0 || n_c > n) {
    if (n == 0 && n_c == 0) {
      HEC_TRY(out_alloc(ctx, (void **)&out->row_ptr, sizeof(int64_t)));
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
  int64_t *mstart = ws_take<int64_t>(ctx, n + 1);
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
  if (!mcount || !vw64 || !member_ptr || !members || !mstart || !mpre || !Sw || !blk_ptr || !big_list || !big_idx ||
      !unit_ptr || !bkt_ptr || !counts || !scal || !st[5].desc) {
    set_error("workspace under-reserved (construct)");
    return HEC_EINVAL;
  }
  int *err = reinterpret_cast<int *>(scal);
  {
    ZeroList z;
    z.add(mcount, (int64_t)sizeof(unsigned) * (n_c + 1));
    z.add(vw64, (int64_t)sizeof(unsigned long long) * (n_c + 1));
    z.add(counts, (int64_t)sizeof(unsigned) * 64);
    z.add(scal, (int64_t)sizeof(int64_t) * 32);
    for (auto &x : st) z.add(x, n > n_c ? n : n_c);
    HEC_TRY(zero_regions(ctx, z));
  }
  const double dn = (double)n, dnc = (double)n_c;
  // ---- a7
  int ph = phase_begin(ctx, "bucket", 16.0 * dn + 4.0 * dnc);
  if (n > 0) {
    k_member_count<<<nblk(n, 256), 256, 0, s>>>(n, M, n_c, g->vwgt, mcount, vw64, err);
    HEC_LAUNCH_CHECK();
  }
  HEC_TRY(chained_scan(ctx, n_c, CountIn{mcount}, PtrOut{member_ptr}, st[0], member_ptr + n_c, true));
  if (n > 0) {
    k_member_fill<<<nblk(n, 256), 256, 0, s>>>(n, n_c, M, member_ptr, mcount, members, g->row_ptr, mstart);
    HEC_LAUNCH_CHECK();
  }
  HEC_TRY(chained_scan(ctx, n, DegIn{members, g->row_ptr, member_ptr + n_c}, PtrOut{mpre}, st[1], mpre + n, true));
  if (a_lo < 0 || a_lo > a_hi || a_hi > n_c) {
    set_error("coarse row range [%lld, %lld) outside [0, %lld)", (long long)a_lo, (long long)a_hi, (long long)n_c);
    return HEC_EINVAL;
  }
  const int64_t n_out = a_hi - a_lo;  // rows produced by this call
  // 32-bit entry / position indices in the member walks when nnz < 2^32
  // (HEC_FORCE_WIDE_INDEX: test hook for the 64-bit instantiation)
  const bool idx32 = g->nnz < ((int64_t)1 << 32) && getenv("HEC_FORCE_WIDE_INDEX") == nullptr;
  Layout L{n_c, member_ptr, members, mpre, g->row_ptr, g->col, g->wgt, M, a_lo, a_hi, kRbmBinAvg,
           ctx->build_unit_wgt != nullptr && ctx->build_unit_wgt == g->wgt};
  const bool dense = n_c <= kDenseMax;
  // bitmap-rank items replace the bin pieces when the key range fits the
  // shared-memory bitmap (BuildOpts::sort_dedup, HEC_BUILD_SORT: the bin-piece / bucket-sort path)
  // rank items for every level (DENSE levels: the small rows); bins are kept
  // <= kRbmRange keys wide (row_buckets) for the bitmap-rank fallback
  const bool rbm = !(opt && opt->sort_dedup);
  const int64_t big_thr = rbm ? (int64_t)kRbmRow : big_threshold_host(dense);
  k_big_rows<<<nblk(n_c, 256), 256, 0, s>>>(L, big_thr, big_list, big_idx, counts + 0,
                                            reinterpret_cast<unsigned long long *>(scal + 1));
  HEC_LAUNCH_CHECK();
  HEC_TRY(chained_scan(ctx, n_c, RowWeightIn{L, big_thr}, PtrOut{Sw}, st[2], Sw + n_c, true));
  HEC_TRY(chained_scan(ctx, n_c, BlockCountIn{L, Sw, dense, big_thr, rbm}, PtrOut{blk_ptr}, st[3], blk_ptr + n_c, true, scal + 7));
  HEC_TRY(chained_scan(ctx, n_c, UnitsIn{L, big_list, counts + 0, dense ? (int64_t)kDenseUnit2 : (int64_t)kUnit,
                                          dense ? (int64_t)0 : kWarpRowMax}, PtrOut{unit_ptr},
                       st[4], unit_ptr + n_c, true, scal + 5));
  if (!dense) HEC_TRY(chained_scan(ctx, n_c, BucketsIn{L, big_list, counts + 0, rbm}, PtrOut{bkt_ptr}, st[5], bkt_ptr + n_c, true, scal + 6));
  phase_end(ctx, ph);
  int64_t r0[8];
  HEC_TRY(read_scalars(ctx, scal, 8, r0));
  if ((int)(r0[0] & 0xffffffff) & 1) {
    set_error("build_coarse_graph: M has values outside [0, n_c)");
    return HEC_EINVAL;
  }
  const int64_t small_vol = r0[1], big_vol = r0[2];
  const int64_t nbig = r0[4] & 0xffffffffLL;
  const int64_t nunits = r0[5], nbkt = r0[6], nblocks = r0[7];
  const int64_t maxU = r0[3];
  ctx->stats.huge_rows = nbig;
  ctx->stats.dense_rows = dense ? nbig : 0;

  // ---- second arena: block list, block counts/offsets, staging, skew-path buffers
  {
    size_t b2 = ws_bytes(nblocks + 1, sizeof(BlockDesc)) + 4 * ws_bytes(nblocks + 1, 4) + ws_bytes(nblocks + 1, 8) +
                8 * ws_bytes(nblocks + 1, sizeof(RbmItem)) +
                ws_bytes(2 * drank_split_bound(big_vol) + 1, sizeof(RbmItem)) +
                ws_bytes((size_t)drank_split_bound(big_vol) * kDirectR, 4) + ws_bytes(drank_split_bound(big_vol), 4) +
                ws_bytes(nblocks + 1, sizeof(WorkItem)) +
                ws_bytes(nblocks + 1, 8) + scan_ws_bytes(nblocks) +
                2 * ws_bytes((size_t)(small_vol + big_vol) + 1, 4);
    if (nbig > 0) b2 += ws_bytes(nunits + 1, 4);  // unit_row
    if (nbig > 0 && dense) b2 += ws_bytes((size_t)nbig * n_c, 8);
    if (nbig > 0 && !dense) {
      b2 += 2 * ws_bytes(nbkt + 1, 4) + 2 * ws_bytes(nbkt + 1, 8) + ws_bytes(nbkt + 1, 4);
      b2 += ws_bytes((size_t)nunits * kPartHist + 1, 4);  // ubase
      b2 += 4 * ws_bytes((size_t)big_vol + 1, 4) + scan_ws_bytes(nbkt);
      b2 += ws_bytes(nbkt + 1, 8) + ws_bytes(2 * nbkt + 2, 4);
      b2 += ws_bytes(nbkt + 1, 4);  // bin_row
      b2 += ws_bytes(nbig + 1, 8);  // prow
    }
    HEC_TRY(arena_reserve(ctx, &ctx->ws2, b2));
    ctx->ws2.used = 0;
  }
  Arena &W2 = ctx->ws2;
  BlockDesc *blk = arena_take<BlockDesc>(W2, nblocks + 1);
  int32_t *blk_cnt = arena_take<int32_t>(W2, nblocks + 1);
  int32_t *need_wide = arena_take<int32_t>(W2, nblocks + 1);
  WorkItem *list_w = arena_take<WorkItem>(W2, nblocks + 1);   // warp-tier work items
  int32_t *list_c = arena_take<int32_t>(W2, nblocks + 1);     // CTA-tier blocks
  int32_t *list_wide = arena_take<int32_t>(W2, nblocks + 1);  // blocks flagged for 64-bit sums
  RbmItem *list_r = arena_take<RbmItem>(W2, nblocks + 1);     // rank items n <= 2048 (front / back)
  RbmItem *list_r2 = arena_take<RbmItem>(W2, nblocks + 1);    // rank items n > 2048 (front / back)
  RbmItem *list_redo = arena_take<RbmItem>(W2, nblocks + 1);  // n > 4096 items left to k_rbm
  RbmItem *list_d = arena_take<RbmItem>(W2, nblocks + 1);     // direct-indexed bins (k_drank)
  // chunks of the direct-indexed bins above kDrSplit entries, their accumulators and tickets
  const int64_t nsplit_max = drank_split_bound(big_vol);
  RbmItem *list_dc = arena_take<RbmItem>(W2, 2 * nsplit_max + 1);
  uint32_t *drank_acc = arena_take<uint32_t>(W2, (size_t)nsplit_max * kDirectR);
  unsigned *drank_done = arena_take<unsigned>(W2, nsplit_max);
  RbmItem *list_r3 = arena_take<RbmItem>(W2, nblocks + 1);    // rank items n <= kHrMaxS
  RbmItem *list_r4 = arena_take<RbmItem>(W2, nblocks + 1);    // rank items n <= kHrMaxT
  int64_t *grp_end = arena_take<int64_t>(W2, nblocks + 1);    // BUCKET groups: end bin
  int64_t *blk_off = arena_take<int64_t>(W2, nblocks + 1);
  ScanTiles st_blk = take_scan_tiles(W2, nblocks);
  // expanded (b, w) of every active member-edge position; SMALL blocks stage
  // their sorted rows in place over their own entries
  int32_t *sc_col = arena_take<int32_t>(W2, (size_t)(small_vol + big_vol) + 1);
  int32_t *sc_wgt = arena_take<int32_t>(W2, (size_t)(small_vol + big_vol) + 1);
  if (!sc_wgt) { set_error("workspace under-reserved (blocks)"); return HEC_EINVAL; }
  {
    const int phx = phase_begin(ctx, "expand", 12.0 * (double)(small_vol + big_vol) + 16.0 * dn);
    // chunk: kXChunk positions per warp task, less when that would leave
    // fewer than 8 tasks per warp slot of the capped grid (small levels)
    const int64_t cap = (int64_t)ctx->num_sms * 8;
    const int64_t vol = small_vol + big_vol;
    int64_t chunk = (vol + cap * (kXT / 32) * 8 - 1) / (cap * (kXT / 32) * 8);
    chunk = (chunk + 127) / 128 * 128;
    chunk = chunk < kXChunkMin ? kXChunkMin : chunk > kXChunk ? kXChunk : chunk;
    const int64_t warps = (vol + chunk - 1) / chunk;
    int64_t grid = (warps + kXT / 32 - 1) / (kXT / 32);
    if (grid > cap) grid = cap;
    // DENSE rows are walked by their accumulation kernel (k_dense_accum2);
    // everything else is staged once here
    const int32_t *skip = dense ? big_idx : nullptr;
    const int64_t skip_thr = dense ? 0 : INT64_MAX;
    if (grid > 0) {
      if (Cp && idx32)
        k_expand2<uint32_t, 4, true><<<(unsigned)grid, kXT, 0, s>>>(L, mstart, sc_col, sc_wgt, skip, skip_thr, Cp, chunk);
      else if (Cp)
        k_expand2<int64_t, 4, true><<<(unsigned)grid, kXT, 0, s>>>(L, mstart, sc_col, sc_wgt, skip, skip_thr, Cp, chunk);
      else if (idx32)
        k_expand2<uint32_t, 4><<<(unsigned)grid, kXT, 0, s>>>(L, mstart, sc_col, sc_wgt, skip, skip_thr, nullptr, chunk);
      else
        k_expand2<int64_t, 4><<<(unsigned)grid, kXT, 0, s>>>(L, mstart, sc_col, sc_wgt, skip, skip_thr, nullptr, chunk);
      HEC_LAUNCH_CHECK();
    }
    phase_end(ctx, phx);
  }
  {
    ZeroList z;
    z.add(need_wide, (int64_t)sizeof(int32_t) * (nblocks + 1));
    z.add(st_blk, nblocks);
    HEC_TRY(zero_regions(ctx, z));
  }
  k_block_desc<<<nblk(n_c, 256), 256, 0, s>>>(L, blk_ptr, big_idx, dense, rbm, blk);
  HEC_LAUNCH_CHECK();

  RowsArgs A{};
  A.L = L;
  A.blk = blk;
  A.nblocks = nblocks;
  A.ticket = counts + 1;
  A.blk_cnt = blk_cnt;
  A.need_wide = need_wide;
  A.blk_off = blk_off;
  A.sc_col = sc_col;
  A.sc_wgt = sc_wgt;
  A.vw64 = vw64;
  A.big_idx = big_idx;
  A.bkt_ptr = bkt_ptr;
  A.grp_end = grp_end;
  A.err = err;
  A.mstart = mstart;
  A.idx32 = idx32;

  int occ_unused = 0;  // dynamic shared-memory opt-ins (cached per context)
  HEC_TRY(kernel_occupancy(ctx, k_part_count, kT, sizeof(PartSmem), &occ_unused));
  HEC_TRY(kernel_occupancy(ctx, k_part_write, kT, sizeof(PartSmem), &occ_unused));
  HEC_TRY(kernel_occupancy(ctx, k_bucket_fallback, kT, sizeof(FbSmem), &occ_unused));
  HEC_TRY(kernel_occupancy(ctx, k_dense_accum2, kT, 4 * (size_t)kDenseMax, &occ_unused));

  const bool direct = getenv("HEC_NO_DRANK") == nullptr;  // test hook: bins through the hash-rank kernels
  int ph_rows = -1;

  // ---- a9 skewed rows
  const int ph_skew = phase_begin(ctx, "rows_skew", 8.0 * (double)big_vol);
  int32_t *unit_row = nullptr;
  if (nbig > 0) {
    unit_row = arena_take<int32_t>(W2, nunits + 1);
    if (!unit_row) { set_error("workspace under-reserved (units)"); return HEC_EINVAL; }
    k_seg_fill<<<nblk(nbig * 32, 256), 256, 0, s>>>(nbig, unit_ptr, unit_row);
    HEC_LAUNCH_CHECK();
  }
  if (nbig > 0 && dense) {
    unsigned long long *dn_arr = arena_take<unsigned long long>(W2, (size_t)nbig * n_c);
    HEC_CUDA_TRY(cudaMemsetAsync(dn_arr, 0, sizeof(unsigned long long) * nbig * n_c, s));
    DenseArgs D{L, big_list, nbig, unit_ptr, unit_row, nunits, counts + 2, dn_arr, Cp};
    int occ = 1;
    HEC_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_dense_accum2, kT, 4 * (size_t)n_c));
    if (occ < 1) occ = 1;
    k_dense_accum2<<<ctx->num_sms * occ, kT, 4 * (size_t)n_c, s>>>(D, mstart, err);
    HEC_LAUNCH_CHECK();
    A.dense = dn_arr;
  } else if (nbig > 0) {
    unsigned *bkt_cnt = arena_take<unsigned>(W2, nbkt + 1);
    int32_t *ubase = arena_take<int32_t>(W2, (size_t)nunits * kPartHist + 1);  // unit offsets inside bins
    int64_t *bkt_off = arena_take<int64_t>(W2, nbkt + 1);
    int64_t *fb_off = arena_take<int64_t>(W2, nbkt + 1);
    int32_t *fb_cnt = arena_take<int32_t>(W2, nbkt + 1);
    int32_t *pb = arena_take<int32_t>(W2, (size_t)big_vol + 1);
    int32_t *pw = arena_take<int32_t>(W2, (size_t)big_vol + 1);
    ScanTiles stb = take_scan_tiles(W2, nbkt);
    int64_t *jobs = arena_take<int64_t>(W2, nbkt + 1);
    int32_t *fb_b = arena_take<int32_t>(W2, (size_t)big_vol + 1);
    int32_t *fb_w = arena_take<int32_t>(W2, (size_t)big_vol + 1);
    if (!fb_w) { set_error("workspace under-reserved (buckets)"); return HEC_EINVAL; }
    int64_t *prow = arena_take<int64_t>(W2, nbig + 1);
    if (!prow) { set_error("workspace under-reserved (prow)"); return HEC_EINVAL; }
    {
      ZeroList z;
      z.add(bkt_cnt, (int64_t)sizeof(unsigned) * (nbkt + 1));
      z.add(stb, nbig);
      HEC_TRY(zero_regions(ctx, z));
    }
    HEC_TRY(chained_scan(ctx, nbig, RowUIn{L, big_list}, PtrOut{prow}, stb, prow + nbig, true));
    PartArgs PA{L, big_list, nbig, unit_ptr, unit_row, bkt_ptr, sc_col, sc_wgt};
    if (nunits > 0) {  // rows above kWarpRowMax: CTA units count, per-row scan, scatter
      k_part_count<<<(unsigned)nunits, kT, sizeof(PartSmem), s>>>(PA, bkt_cnt, ubase);
      HEC_LAUNCH_CHECK();
      k_row_bins<<<nblk(nbig * 32, 256), 256, 0, s>>>(PA, prow, bkt_cnt, bkt_off);
      HEC_LAUNCH_CHECK();
      k_part_write<<<(unsigned)nunits, kT, sizeof(PartSmem), s>>>(PA, bkt_off, ubase, pb, pw);
      HEC_LAUNCH_CHECK();
    }
    k_part_warp<<<nblk(nbig * 32, kPWT), kPWT, 0, s>>>(PA, prow, bkt_off, bkt_cnt, pb, pw);
    HEC_LAUNCH_CHECK();
    int32_t *bin_row = arena_take<int32_t>(W2, nbkt + 1);
    if (!bin_row) { set_error("workspace under-reserved (bins)"); return HEC_EINVAL; }
    k_seg_fill<<<nblk(nbig * 32, 256), 256, 0, s>>>(nbig, bkt_ptr, bin_row);
    HEC_LAUNCH_CHECK();
    k_bucket_blocks<<<nblk(nbkt, 256), 256, 0, s>>>(nbig, nbkt, big_list, bkt_ptr, bin_row, bkt_cnt, blk_ptr, blk, jobs,
                                                   counts + 4, fb_cnt, fb_off,
                                                   reinterpret_cast<unsigned long long *>(scal + 10),
                                                   rbm ? INT64_MAX : (int64_t)kCap);
    HEC_LAUNCH_CHECK();
    int64_t rj[1];  // counts[4] (low word; counts is 8-byte aligned)
    HEC_TRY(read_scalars(ctx, reinterpret_cast<const int64_t *>(counts + 4), 1, rj));
    const int64_t njobs = rj[0] & 0xffffffffLL;
    if (njobs > 0) {
      k_bucket_fallback<<<ctx->num_sms, kT, sizeof(FbSmem), s>>>(jobs, njobs, bkt_off, bkt_cnt, pb, pw, fb_off,
                                                                fb_cnt, fb_b, fb_w, counts + 3, err);
      HEC_LAUNCH_CHECK();
    }
    A.bkt_off = bkt_off;
    A.bkt_n = bkt_cnt;
    A.pb_g = pb;
    A.pw_g = pw;
    A.fb_cnt = fb_cnt;
    A.fb_off = fb_off;
    A.fb_b = fb_b;
    A.fb_w = fb_w;
    A.fb_total = reinterpret_cast<unsigned long long *>(scal + 10);
    A.fb_off_w = fb_off;
    A.fb_cnt_w = fb_cnt;
    A.fb_b_w = fb_b;
    A.fb_w_w = fb_w;
  }
  if (ph_skew >= 0) phase_end(ctx, ph_skew);
  // counts: [5] pieces ticket [8] wide list [10] warp list [11] CTA list [12] bitmap-rank list
  //         [13] bitmap-rank ticket
  if (nblocks > 0) {
    k_block_ends<<<nblk(nblocks, 256), 256, 0, s>>>(nblocks, a_hi, blk);
    HEC_LAUNCH_CHECK();
    k_tiers<<<nblk(nblocks, 256), 256, 0, s>>>(L, nblocks, blk, big_idx, bkt_ptr, A.bkt_off, A.bkt_n, A.fb_cnt, blk_cnt, grp_end, list_w,
                                              list_c, list_r, list_r2, list_d, list_r3, list_r4, counts + 10, rbm, direct, 0, vw64, err);
    HEC_LAUNCH_CHECK();
  }

  // ---- work blocks (a8/a9 output), then placement (a10)
  HEC_TRY(out_alloc(ctx, (void **)&out->row_ptr, sizeof(int64_t) * (n_out + 1)));
  HEC_TRY(out_alloc(ctx, (void **)&out->vwgt, sizeof(int32_t) * (n_out > 0 ? n_out : 1)));
  out->n_c = n_out;
  A.row_ptr_c = out->row_ptr;
  A.vwgt_c = out->vwgt;
  ph_rows = phase_begin(ctx, "rows", 8.0 * (double)small_vol);
  A.items = list_w;
  A.nlist = counts + 10;
  HEC_TRY(launch_pieces(ctx, A, counts + 5));
  A.list = list_c;
  A.nlist = counts + 11;
  // (rank-item levels without skewed rows have only PIECE / RBM blocks: no CTA list)
  if (!(rbm && nbig == 0)) HEC_TRY(launch_rows(ctx, A, false));
  if (rbm) {
    A.ticket = counts + 30;  // (unused by the rank kernels)
    A.rcap = nblocks + 1;
    // hash-rank size classes, then the multi-round hash rank above kHrMax2
    // entries (items with too many distinct keys -> the bitmap rank k_rbm)
    struct RankList { RbmItem *items; unsigned *n; int dir; };
    const RankList cls[6] = {{list_r4, counts + 22, 1}, {list_r3, counts + 13, 1},
        {list_r, counts + 12, 1}, {list_r, counts + 14, -1}, {list_r2, counts + 15, 1}, {list_r2, counts + 16, -1}};
    // Without skewed rows every rank item is a whole row (kPieceMax < U <= maxU):
    // classes above maxU, the multi-round class and the direct-indexed bins are
    // empty and not launched (small levels are bound by launches); DENSE levels
    // have no bins and no whole-row item above kHrMax2 either.
    const bool no_bins = nbig == 0 || dense;
    const int64_t cls_lo[6] = {kPieceMax, kHrMaxT, kHrMaxS, kHrMax0, kHrMax1, kHrMax2};
    for (int c = -2; c < 4; ++c) {
      if (nbig == 0 && maxU <= cls_lo[c + 2]) continue;
      if (c == 3 && no_bins) continue;
      const RankList &C = cls[c + 2];
      A.ritems = C.items;
      A.nlist = C.n;
      A.rdir = C.dir;
      if (c < 3) {
        HEC_TRY(launch_hrank(ctx, A, c));
      } else {
        HEC_TRY(launch_hrank_big(ctx, A, list_redo, counts + 17));
        A.ritems = list_redo;
        A.nlist = counts + 17;
        A.rdir = 1;
        HEC_TRY(launch_rbm(ctx, A));
      }
    }
    A.ritems = list_d;
    A.nlist = counts + 18;
    A.rdir = 1;
    if (!no_bins) HEC_TRY(launch_drank(ctx, A, list_dc, counts + 19, drank_acc, drank_done, counts + 21));
    A.ticket = counts + 1;
  }
  phase_end(ctx, ph_rows);
  HEC_TRY(chained_scan(ctx, nblocks, BlkCntIn{blk_cnt}, PtrOut{blk_off}, st_blk, blk_off + nblocks, true, scal + 12));
  int64_t r2[13];
  HEC_TRY(read_scalars(ctx, scal, 13, r2));
  if ((int)(r2[0] & 0xffffffff) & ERR_WIDE) {
    // some block's total weight exceeds int32: those blocks (flagged, inputs left
    // untouched) are redone with int64 sums
    HEC_CUDA_TRY(cudaMemsetAsync(counts + 1, 0, sizeof(unsigned), s));
    HEC_CUDA_TRY(cudaMemsetAsync(err, 0, sizeof(int), s));
    k_wide_list<<<nblk(nblocks, 256), 256, 0, s>>>(nblocks, need_wide, list_wide, counts + 8);
    HEC_LAUNCH_CHECK();
    A.list = list_wide;
    A.nlist = counts + 8;
    HEC_TRY(launch_rows(ctx, A, true));
    HEC_TRY(chained_scan(ctx, nblocks, BlkCntIn{blk_cnt}, PtrOut{blk_off}, st_blk, blk_off + nblocks));
    HEC_CUDA_TRY(cudaMemcpyAsync(scal + 12, blk_off + nblocks, sizeof(int64_t), cudaMemcpyDeviceToDevice, s));
    HEC_TRY(read_scalars(ctx, scal, 13, r2));
  }
  out->nnz_c = r2[12];
  if ((int)(r2[0] & 0xffffffff) & ERR_INTERNAL) {
    set_error("build_coarse_graph: internal error (bitmap-rank key outside its bin)");
    return HEC_ECUDA;
  }
  if ((int)(r2[0] & 0xffffffff) & ERR_OVERFLOW) {
    set_error("build_coarse_graph: a coarse weight exceeds INT32_MAX");
    return HEC_EOVERFLOW;
  }
  const int64_t nnz_c = out->nnz_c;
  HEC_TRY(out_alloc(ctx, (void **)&out->col, sizeof(int32_t) * (nnz_c > 0 ? nnz_c : 1)));
  HEC_TRY(out_alloc(ctx, (void **)&out->wgt, sizeof(int32_t) * (nnz_c > 0 ? nnz_c : 1)));
  A.col_c = out->col;
  A.wgt_c = out->wgt;
  const int ph_place = phase_begin(ctx, "place", 16.0 * (double)nnz_c + 16.0 * dnc);
  // heavy keys of G_{l+1} fused into the placement (hierarchy, hash construction
  // of the whole row range only)
  bool hk_done = false;
  if (ctx->hk_build && rbm && !Cp && a_lo == 0 && a_hi == n_c) {
    HEC_CUDA_TRY(cudaMemsetAsync(ctx->hk_build, 0, sizeof(unsigned long long) * n_c, s));
    A.hkey = ctx->hk_build;
  }
  HEC_TRY(launch_place(ctx, A, &hk_done));
  ctx->hk_built = hk_done;
  phase_end(ctx, ph_place);
  // rows phase: staged / partitioned entries read (8 B each; DENSE rows were
  // accumulated in rows_skew), distinct entries staged (8 B), row_ptr_c + vwgt_c
  phase_set_bytes(ctx, ph_rows, 8.0 * (double)(small_vol + (dense ? 0 : big_vol)) + 8.0 * (double)nnz_c + 12.0 * dnc);
  if (nblocks == 0) HEC_CUDA_TRY(cudaMemsetAsync(out->row_ptr, 0, sizeof(int64_t) * (n_out + 1), s));
  ctx->stats.nnz_c = out->nnz_c;
  return HEC_OK;
}

}  // namespace hec

namespace hec {

__global__ void k_row_volume(int64_t n, const int32_t *__restrict__ M, int64_t n_c,
                             const int64_t *__restrict__ row_ptr, unsigned long long *__restrict__ U,
                             int *__restrict__ err) {
  int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (u >= n) return;
  int32_t a = M[u];
  if (a < 0 || a >= n_c) { atomicOr(err, ERR_LABEL); return; }
  atomicAdd(U + a, (unsigned long long)(row_ptr[u + 1] - row_ptr[u]));
}

int row_volume_impl(hec_ctx *ctx, const hec_graph *g, const int32_t *M, int64_t n_c, int64_t *U) {
  int *err = nullptr;
  HEC_TRY(dev_alloc(ctx, (void **)&err, 64));
  HEC_CUDA_TRY(cudaMemsetAsync(err, 0, 64, ctx->stream));
  HEC_CUDA_TRY(cudaMemsetAsync(U, 0, sizeof(int64_t) * n_c, ctx->stream));
  if (g->n > 0) {
    k_row_volume<<<nblk(g->n, 256), 256, 0, ctx->stream>>>(g->n, M, n_c, g->row_ptr,
                                                          reinterpret_cast<unsigned long long *>(U), err);
    HEC_LAUNCH_CHECK();
  }
  int64_t r[1];
  int rc = read_scalars(ctx, reinterpret_cast<int64_t *>(err), 1, r);
  dev_free(ctx, err);
  HEC_TRY(rc);
  if ((int)(r[0] & 0xffffffff) & ERR_LABEL) {
    set_error("M has values outside [0, n_c)");
    return HEC_EINVAL;
  }
  return HEC_OK;
}

}  // namespace hec
