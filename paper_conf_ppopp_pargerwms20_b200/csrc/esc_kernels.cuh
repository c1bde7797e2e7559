// esc_kernels.cuh — rows accumulated by a counting sort on monotone column buckets in shared
// memory ("expand, bucket, sort, compress"), the B200 alternative to the hash map for rows whose
// products are mostly distinct columns.
//
// The paper accumulates every row in a scratchpad hash map and sorts it afterwards (P:972-994,
// P:1130-1143).  On inputs whose rows have almost no repeated columns (C5: 1.1e10 products give
// 1.099e10 entries) the hash map does a find-or-claim probe per product and a run-ranking
// write-out per slot; ncu put that at ~22 warp instructions per product (profiles/r02b_*).  This
// path instead:
//   H  expands the row's products once and counts them per bucket, bucket(col) =
//      (col - colmin) * NB / (colmax - colmin + 1) (monotone in the column, ~4 products each);
//   S  scans the counts into bucket offsets and expands the products again, appending each
//      (col, a·b) to its bucket with one shared-memory atomic (no probing, no CAS);
//   W  ranks every entry inside its bucket (the buckets are in column order, so bucket start +
//      rank is the sorted position) and writes C — or, symbolic, counts the first occurrences.
// Equal columns always share a bucket, so duplicates are found by the rank loop: the first
// occurrence sums the values of its equals and the others are dropped (numeric rows with
// products > nnz(C_i) take a second ranking pass over the surviving entries).  Shared memory
// holds exactly the row's products (4 + sizeof(V) bytes each, plus 4 bytes per bucket), i.e.
// 100% load instead of the hash map's 40-50%.
//
// Products are enumerated by expand_esc: the referenced B rows of a batch of 32 NZ of A are
// compacted to the low lanes (no empty rows), and the owner of product pp of a 32-product chunk
// is found from one warp-wide OR of the row starts falling into the chunk (REDUX) and a popcount
// — ~4 instructions per product instead of the 5-step shuffle binary search of expand_row.
#pragma once

#include <type_traits>

#include "speck_internal.cuh"

namespace speck {

#ifndef SPECK_ESC_LAMBDA
#define SPECK_ESC_LAMBDA 2
#endif
constexpr int kEscLambda = SPECK_ESC_LAMBDA;   // target products per bucket
#ifndef SPECK_ESC_RATIO_PCT
#define SPECK_ESC_RATIO_PCT 200
#endif
// numeric rows take the counting sort when products <= this % of their entries (repeated
// columns cost the rank passes a second round)
constexpr int kEscRatioPct = SPECK_ESC_RATIO_PCT;
#ifndef SPECK_ESC_MAX_CFG
#define SPECK_ESC_MAX_CFG 4   // block configurations that may take the counting sort (experiments)
#endif
#ifndef SPECK_ESC_TABLE
#define SPECK_ESC_TABLE 1
#endif
constexpr bool kEscTable = SPECK_ESC_TABLE != 0;   // block rows: reference table in shared memory
#ifndef SPECK_ESC_STAGED
#define SPECK_ESC_STAGED 1
#endif
constexpr bool kEscStaged = SPECK_ESC_STAGED != 0;   // numeric rows: one expansion (esc_row_staged)
// a row whose largest bucket exceeds this goes back to the hash map: clustered columns (stencil
// rows: many products on few columns) would make the in-bucket ranking quadratic
constexpr int kEscMaxBucket = 8 * kEscLambda + 16;
constexpr uint32_t kEscDropBit = 0x80000000u;   // marks a non-first duplicate (columns are < 2^31)

template <typename V>
__host__ __device__ constexpr int esc_entry_bytes(int pass) { return pass == 0 ? 4 : 4 + (int)sizeof(V); }
// products a region of `bytes` can hold (keys [+ values] + two bucket arrays of NB ~ n/4 ints)
template <typename V>
__host__ __device__ inline int64_t esc_capacity(int pass, int64_t bytes) {
  return (bytes - 320) * kEscLambda / ((int64_t)esc_entry_bytes<V>(pass) * kEscLambda + 8);
}
// rank of k among keys[s, en) (keys < k).  The trip count is the warp's largest bucket (a
// warp-uniform loop: no divergent exits, no reconvergence barriers), 4 keys per iteration;
// lanes past their bucket's end read nothing.  Inactive lanes pass s == en.
__device__ __forceinline__ int esc_rank(const uint32_t* keys, int s, int en, uint32_t k) {
  const int len = en - s;
  const int mx = (int)__reduce_max_sync(0xffffffffu, (unsigned)len);
  int r = 0;
  for (int d = 0; d < mx; d += 4) {
#pragma unroll
    for (int u = 0; u < 4; ++u)
      if (d + u < len) r += keys[s + d + u] < k;
  }
  return r;
}

template <int NW>
__device__ __forceinline__ void esc_sync() {
  if (NW == 1) __syncwarp(); else __syncthreads();
}

// Products of A_i (NZ [a0, a0 + alen)) for warp wi of nw (a power of two): chunks of 32 products
// rotate over the warps across batches.  f(col, a*b, active) is called by all 32 lanes.
// `pre` (optional): the row's first batch, loaded ahead by the caller (lane f: B row start /
// length and a of the row's f-th NZ).
template <typename V>
struct PreBatch {
  int64_t bst = 0;
  int blen = 0;
  V a = V(0);
  bool valid = false;
};

// The chunks of one batch whose references are compacted to lanes [0, nn) (lane o: its
// products [excl_o, excl_o + len) start at B entry boff_o + excl_o; own_any = len > 0): chunk c of
// 32 products goes to warp (c + rot) mod nw; the owner of product pp of a chunk is found from one
// warp-wide OR of the row starts falling into the chunk and a popcount.
template <int PASS, typename V, int U, typename F>
__device__ __forceinline__ void esc_batch_chunks(const SpgemmArgs<V>& p, int excl, bool own_any, int64_t boff, V a,
                                                 int Pb, int pb0, int wi, int nw, int& rot, F& f) {
  const int lane = lane_id();
  const int nch = (Pb + 31) >> 5;
  int c = (wi - rot) & (nw - 1);
  rot = (rot + nch) & (nw - 1);
  for (; c < nch; c += U * nw) {
    uint32_t col[U];
    V bv[U], av[U];
    bool act[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int q0 = (c + u * nw) * 32;
      col[u] = 0x80000000u | (uint32_t)lane;
      bv[u] = V(0);
      av[u] = V(0);
      act[u] = false;
      if (q0 >= Pb) continue;                                   // warp-uniform
      const uint32_t d = (uint32_t)(excl - q0);
      const uint32_t bits = __reduce_or_sync(0xffffffffu, (own_any && d < 32u) ? (1u << d) : 0u);
      const int base = __popc(__ballot_sync(0xffffffffu, own_any && excl < q0));
      const int own = base + __popc(bits & (0xffffffffu >> (31 - lane))) - 1;
      const int pp = q0 + lane;
      const int64_t idx = __shfl_sync(0xffffffffu, boff, own) + pp;
      if (PASS == 1) av[u] = __shfl_sync(0xffffffffu, a, own);
      act[u] = pp < Pb;
      if (act[u]) {
        col[u] = (uint32_t)p.B_col[idx];
        if (PASS == 1) bv[u] = __ldg(p.B_val + idx);
      }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      if ((c + u * nw) * 32 >= Pb) continue;                   // warp-uniform
      if constexpr (std::is_invocable_v<F, uint32_t, V, bool, int>)
        f(col[u], av[u] * bv[u], act[u], pb0 + (c + u * nw) * 32 + lane);
      else
        f(col[u], av[u] * bv[u], act[u]);
    }
  }
}

// One batch of 32 NZ of A_i (NZ [a0 + b0, a0 + b0 + 32) of the row's alen): lane f loads its
// reference (B row start, length, a), the non-empty references are compacted to the low lanes
// and scanned.  Returns Pb (products of the batch); excl/boff/a/own_any as esc_batch_chunks wants.
// first entry >= x of the sorted columns col[l, h)
__device__ __forceinline__ int64_t esc_lower_bound(const int32_t* __restrict__ col, int64_t l, int64_t h, uint32_t x) {
  while (l < h) {
    const int64_t m = (l + h) >> 1;
    if ((uint32_t)col[m] < x) l = m + 1;
    else h = m;
  }
  return l;
}

template <int PASS, typename V>
__device__ __forceinline__ int esc_batch_setup(const SpgemmArgs<V>& p, int64_t a0, int alen, int b0,
                                               const PreBatch<V>* pre, int& excl, bool& own_any, int64_t& boff,
                                               V& a, bool clip = false, uint32_t clo = 0, uint32_t chi = 0) {
  const int lane = lane_id();
  const int fi = b0 + lane;
  int64_t bst = 0;
  int blen = 0;
  a = V(0);
  if (pre && b0 == 0 && pre->valid) {
    bst = pre->bst;
    blen = pre->blen;
    a = pre->a;
  } else if (fi < alen) {
    const int32_t kc = p.A_col[a0 + fi];
    if (PASS == 1) a = __ldg(p.A_val + a0 + fi);
    bst = p.B_rp[kc];
    blen = (int)(p.B_rp[kc + 1] - bst);
    if (clip && blen > 0) {
      // column segment [clo, chi) of a long row: only the part of B_k inside it
      const int64_t s0 = esc_lower_bound(p.B_col, bst, bst + blen, clo);
      const int64_t e0 = esc_lower_bound(p.B_col, s0, bst + blen, chi);
      bst = s0;
      blen = (int)(e0 - s0);
    }
  }
  const uint32_t ne = __ballot_sync(0xffffffffu, blen > 0);
  if (!ne) {
    excl = 0;
    own_any = false;
    boff = 0;
    return 0;
  }
  const int nn = __popc(ne);
  if (ne != (0xffffffffu >> (32 - nn))) {
    // compact the non-empty references to lanes [0, nn): lane j takes the (j+1)-th set bit
    int src = 0;
#pragma unroll
    for (int step = 16; step > 0; step >>= 1)
      if (__popc(ne & ((2u << (src + step - 1)) - 1u)) <= lane) src += step;
    src = min(src, 31);
    bst = __shfl_sync(0xffffffffu, bst, src);
    blen = __shfl_sync(0xffffffffu, blen, src);
    if (PASS == 1) a = __shfl_sync(0xffffffffu, a, src);
    if (lane >= nn) blen = 0;
  }
  const int incl = warp_incl_scan(blen);
  excl = incl - blen;
  own_any = blen > 0;
  boff = bst - excl;          // product pp of owner o is B entry boff_o + pp
  return __shfl_sync(0xffffffffu, incl, 31);
}

// Products of A_i (NZ [a0, a0 + alen)) for warp wi of nw (a power of two): every warp sets up
// every batch of 32 NZ, chunks of 32 products rotate over the warps across batches.
// f(col, a*b, active[, product index]) is called by all 32 lanes.  `pre` (optional): the row's
// first batch, loaded ahead by the caller (lane f: B row start / length and a of the row's f-th NZ).
template <int PASS, typename V, int U, typename F>
__device__ __forceinline__ void expand_esc(const SpgemmArgs<V>& p, int64_t a0, int alen, int wi, int nw, F&& f,
                                           const PreBatch<V>* pre = nullptr) {
  int rot = 0;
  int pbase = 0;   // products of the earlier batches (the row's product index of q0 = pbase + q0)
  for (int b0 = 0; b0 < alen; b0 += 32) {
    int excl;
    bool own_any;
    int64_t boff;
    V a;
    const int Pb = esc_batch_setup<PASS, V>(p, a0, alen, b0, pre, excl, own_any, boff, a);
    if (!Pb) continue;
    esc_batch_chunks<PASS, V, U>(p, excl, own_any, boff, a, Pb, pbase, wi, nw, rot, f);
    pbase += Pb;
  }
}

// Shared-memory reference table of a row (block rows): bytes for nb = ceil(alen / 32) batches.
template <typename V>
__host__ __device__ inline int64_t esc_tbl_bytes(int alen) {
  const int64_t nb = (alen + 31) / 32;
  return nb * 32 * (8 + 4 + (int64_t)sizeof(V)) + ((nb * 4 + 15) & ~(int64_t)15);
}
// As expand_esc for the NW warps of a block, but every batch is set up once: warp w sets up
// batches w, w + NW, ... into the table `tbl` (esc_tbl_bytes, 16-byte aligned) in parallel, then
// all warps stream the chunks from it (one dependent A -> B-row-bounds round trip per row instead
// of one per batch per warp).  Barrier inside.
template <typename V>
struct EscTbl {
  int64_t* boff;
  int* excl;
  V* a;
  int* pb;
  __device__ __forceinline__ EscTbl(unsigned char* tbl, int alen) {
    const int nb = (alen + 31) >> 5;
    boff = reinterpret_cast<int64_t*>(tbl);
    excl = reinterpret_cast<int*>(boff + nb * 32);
    a = reinterpret_cast<V*>(excl + nb * 32);
    pb = reinterpret_cast<int*>(a + nb * 32);
  }
};
// Reference table of a row: warp w sets up batches w, w + NW, ... (clip: only B entries with
// columns in [clo, chi)).  Barrier at the end.
template <int PASS, typename V, int NW>
__device__ __forceinline__ void esc_tbl_build(const SpgemmArgs<V>& p, int64_t a0, int alen, int wi, unsigned char* tbl,
                                              bool clip = false, uint32_t clo = 0, uint32_t chi = 0) {
  const int lane = lane_id();
  const int nb = (alen + 31) >> 5;
  EscTbl<V> t(tbl, alen);
  for (int j = wi; j < nb; j += NW) {
    int excl;
    bool own_any;
    int64_t boff;
    V a;
    const int Pb = esc_batch_setup<PASS, V>(p, a0, alen, j * 32, nullptr, excl, own_any, boff, a, clip, clo, chi);
    t.boff[j * 32 + lane] = boff;
    t.excl[j * 32 + lane] = own_any ? excl : 0x7fffffff;
    if (PASS == 1) t.a[j * 32 + lane] = a;
    if (lane == 0) t.pb[j] = Pb;
  }
  __syncthreads();
}
// Chunks of every batch of a built table, rotated over the NW warps.
template <int PASS, typename V, int NW, int U, typename F>
__device__ __forceinline__ void esc_tbl_gather(const SpgemmArgs<V>& p, int alen, int wi, const unsigned char* tbl, F&& f) {
  const int lane = lane_id();
  const int nb = (alen + 31) >> 5;
  EscTbl<V> t(const_cast<unsigned char*>(tbl), alen);
  int rot = 0, pbase = 0;
  for (int j = 0; j < nb; ++j) {
    const int Pb = t.pb[j];
    if (!Pb) continue;
    const int ex = t.excl[j * 32 + lane];
    const V a = PASS == 1 ? t.a[j * 32 + lane] : V(0);
    esc_batch_chunks<PASS, V, U>(p, ex, ex != 0x7fffffff, t.boff[j * 32 + lane], a, Pb, pbase, wi, NW, rot, f);
    pbase += Pb;
  }
}
template <int PASS, typename V, int NW, int U, typename F>
__device__ __forceinline__ void expand_tbl(const SpgemmArgs<V>& p, int64_t a0, int alen, int wi, unsigned char* tbl,
                                           F&& f) {
  esc_tbl_build<PASS, V, NW>(p, a0, alen, wi, tbl);
  esc_tbl_gather<PASS, V, NW, U>(p, alen, wi, tbl, f);
}

// In-place exclusive scan of bc[0, NB) by the NW warps of the row (each thread a contiguous run
// of ceil(NB / (32 NW)) entries); returns the largest count.  `red` = >= 2 * NW + 2 ints of
// scratch (block-level only).  Barriers inside.
template <int NW>
__device__ __forceinline__ int esc_scan(int* bc, int NB, int wi, int* red) {
  const int lane = lane_id();
  const int t = wi * 32 + lane;
  const int per = (NB + 32 * NW - 1) / (32 * NW);
  const int b0 = min(NB, t * per), b1 = min(NB, b0 + per);
  int sum = 0, mx = 0;
  for (int b = b0; b < b1; ++b) {
    const int x = bc[b];
    sum += x;
    mx = max(mx, x);
  }
  const int incl = warp_incl_scan(sum);
  mx = __reduce_max_sync(0xffffffffu, (unsigned)mx);
  int off = incl - sum;
  if (NW > 1) {
    if (lane == 31) { red[wi] = incl; red[NW + wi] = mx; }
    __syncthreads();
    int wbase = 0, m2 = 0;
    if (NW >= 8) {
      // lane w reads warp w's total: one warp scan instead of 2 NW shared loads per thread
      const int rv = lane < NW ? red[lane] : 0;
      const int inc = warp_incl_scan(rv);
      wbase = __shfl_sync(0xffffffffu, inc - rv, wi);
      m2 = (int)__reduce_max_sync(0xffffffffu, (unsigned)(lane < NW ? red[NW + lane] : 0));
    } else {
      for (int w = 0; w < NW; ++w) {
        if (w < wi) wbase += red[w];
        m2 = max(m2, red[NW + w]);
      }
    }
    off += wbase;
    mx = m2;
  }
  for (int b = b0; b < b1; ++b) {
    const int x = bc[b];
    bc[b] = off;
    off += x;
  }
  esc_sync<NW>();
  return mx;
}

// One row by the NW warps (warp wi) that share `region` (region_bytes, 16-byte aligned).
//   PASS 0: returns the number of distinct columns (every thread), or -1 if the row's buckets are
//           too uneven (the caller then runs the hash map on the same region).
//   PASS 1: writes the row sorted at C[cbase, cbase + cnt); returns cnt, or -1 (fallback).
// chist (symbolic, may be null): distinct columns per 2^chunk_shift-column chunk (long rows).
template <int NW, int PASS, typename V>
__device__ __forceinline__ int esc_row(const SpgemmArgs<V>& p, unsigned char* region, uint32_t region_bytes, int wi, int64_t a0,
                       int alen, int n, int cnt, int32_t cmin, int32_t cmax, int64_t cbase, int* red, int* chist,
                       int chunk_shift) {
  const int lane = lane_id();
  const int t = wi * 32 + lane;
  constexpr int T = NW * 32;
  int NB = (n + kEscLambda - 1) / kEscLambda;
  NB = (NB + 31) & ~31;
  int* bc = reinterpret_cast<int*>(region);
  int* dc = bc + NB;
  uint32_t* keys = reinterpret_cast<uint32_t*>(region + (((size_t)NB * 8 + 15) & ~(size_t)15));
  V* vals = reinterpret_cast<V*>(reinterpret_cast<unsigned char*>(keys) + (((size_t)n * 4 + 15) & ~(size_t)15));
  (void)region_bytes;
  const uint32_t lo = (uint32_t)cmin;
  const uint32_t range = (uint32_t)(cmax - cmin + 1);
  const uint64_t mult = range ? ((uint64_t)NB << 32) / range : 0;   // floor: bucket <= (range-1) NB / range < NB
  const uint32_t mlo = (uint32_t)mult, mhi = (uint32_t)(mult >> 32);
  auto home = [&](uint32_t col) {
    const uint32_t x = col - lo;
    return __umulhi(x, mlo) + x * mhi;
  };

  for (int b = t; b < NB; b += T) bc[b] = 0;
  esc_sync<NW>();
  // ---- H: bucket counts -------------------------------------------------------------------
  expand_esc<0, V, 4>(p, a0, alen, wi, NW, [&](uint32_t col, V, bool act) {
    if (act) atomicAdd(&bc[home(col)], 1);
  });
  esc_sync<NW>();
  const int mx = esc_scan<NW>(bc, NB, wi, red);
  if (mx > kEscMaxBucket) {
    if (t == 0) count_path(p.paths, SPECK_PATH_ESC_FALLBACK);
    return -1;
  }
  if (t == 0) count_path(p.paths, PASS == 0 ? SPECK_PATH_SYM_ESC : n == cnt ? SPECK_PATH_NUM_ESC : SPECK_PATH_NUM_ESC_DUP);
  // ---- S: append (col, a*b) to its bucket -----------------------------------------------------
  expand_esc<PASS, V, 2>(p, a0, alen, wi, NW, [&](uint32_t col, V v, bool act) {
    if (act) {
      const int pos = atomicAdd(&bc[home(col)], 1);
      keys[pos] = col;
      if (PASS == 1) vals[pos] = v;
    }
  });
  esc_sync<NW>();
  // now bc[b] = end of bucket b, start = bc[b - 1] (0 for b = 0)
  if (PASS == 0) {
    // distinct columns = first occurrences (no equal key earlier in the bucket)
    int d = 0;
    for (int e = t; e < n; e += T) {
      const uint32_t k = keys[e];
      const uint32_t b = home(k);
      const int s = b ? bc[b - 1] : 0;
      bool first = true;
      for (int j = s; j < e; ++j) first &= keys[j] != k;
      d += first;
      if (first && chist) atomicAdd(&chist[k >> chunk_shift], 1);
    }
    d = warp_sum(d);
    if (NW == 1) return d;
    if (lane == 0) red[2 * NW] = 0;
    __syncthreads();
    if (lane == 0) atomicAdd(&red[2 * NW], d);
    __syncthreads();
    const int total = red[2 * NW];
    __syncthreads();
    return total;
  }
  if (n == cnt) {
    // no repeated column in the row: sorted position = bucket start + rank in the bucket
    for (int e0 = wi * 32; e0 < n; e0 += T) {          // warp-uniform: every lane calls esc_rank
      const int e = e0 + lane;
      const bool act = e < n;
      const uint32_t k = act ? keys[e] : 0u;
      const uint32_t b = act ? home(k) : 0u;
      const int s = act ? (b ? bc[b - 1] : 0) : 0, en = act ? bc[b] : 0;
      const int r = esc_rank(keys, s, en, k);
      if (act) {
        p.C_col[cbase + s + r] = (int32_t)k;
        p.C_val[cbase + s + r] = vals[e];
      }
    }
    esc_sync<NW>();
    return cnt;
  }
  // ---- repeated columns: W1 the first occurrence of a column sums its equals; the others are
  // marked dropped (after a barrier: the marks must not disturb the comparisons) ----------------
  for (int b = t; b < NB; b += T) dc[b] = 0;
  uint32_t drop = 0;   // bit i: entry t + i*T is a non-first duplicate (n <= 32 T, see esc_capacity users)
  int i = 0;
  for (int e = t; e < n; e += T, ++i) {
    const uint32_t k = keys[e];
    const uint32_t b = home(k);
    const int s = b ? bc[b - 1] : 0, en = bc[b];
    bool first = true;
    for (int j = s; j < e; ++j) first &= keys[j] != k;
    if (first) {
      V sum = vals[e];
      for (int j = e + 1; j < en; ++j)
        if (keys[j] == k) sum += vals[j];
      vals[e] = sum;                     // only this lane reads vals[e] as a first occurrence
    } else {
      drop |= 1u << i;
    }
  }
  esc_sync<NW>();
  i = 0;
  for (int e = t; e < n; e += T, ++i) {
    if ((drop >> i) & 1u) keys[e] |= kEscDropBit;
    else atomicAdd(&dc[home(keys[e])], 1);
  }
  esc_sync<NW>();
  esc_scan<NW>(dc, NB, wi, red);      // dc[b] = first distinct position of bucket b
  // ---- W2: rank the surviving entries among the surviving entries of their bucket ------------
  for (int e0 = wi * 32; e0 < n; e0 += T) {
    const int e = e0 + lane;
    const uint32_t kk = e < n ? keys[e] : kEscDropBit;
    const bool act = !(kk & kEscDropBit);
    const uint32_t b = act ? home(kk) : 0u;
    const int s = act ? (b ? bc[b - 1] : 0) : 0, en = act ? bc[b] : 0;
    const int r = esc_rank(keys, s, en, kk);          // dropped keys have the top bit set: never smaller
    if (act) {
      const int64_t o = cbase + dc[b] + r;
      p.C_col[o] = (int32_t)kk;
      p.C_val[o] = vals[e];
    }
  }
  esc_sync<NW>();
  return cnt;
}

// ---------------------------------------------------------------------------------------------
// Numeric rows with ONE expansion ("staged"): the products are gathered once, in product order,
// into shared memory (column, a*b, arrival index inside the column bucket), the bucket counts are
// scanned, and a shared-memory-only pass files every product's index under its bucket slot.  The
// rank/write-out then reads the bucket members through that index.  esc_row's S pass re-expands
// the row from global memory (A -> B row bounds -> B columns and values again: ~35% of the
// numeric ESC instructions and a second dependent load chain, ncu profiles/r02/r02u_*); here the
// second pass touches shared memory only.  Shared memory per product: 4 (column) + sizeof(V) +
// 2 (slot -> product) + 1 (arrival index) + 8/lambda (bucket starts, distinct starts).
// ---------------------------------------------------------------------------------------------
template <typename V>
__host__ __device__ inline int64_t esc_staged_capacity(int pass, int64_t bytes) {
  const int64_t per = pass == 0 ? 7 : 7 + (int64_t)sizeof(V);   // bytes per product besides the buckets
  const int64_t c = (bytes - 320) * kEscLambda / (per * kEscLambda + 8);
  return c < 65535 ? c : 65535;     // slot -> product indices are 16-bit
}

// exact shared-memory bytes of esc_row_staged's arrays for n products (without a reference table)
template <typename V>
__host__ __device__ inline int64_t esc_staged_bytes(int pass, int64_t n) {
  int64_t NB = (n + kEscLambda - 1) / kEscLambda;
  NB = (NB + 31) & ~(int64_t)31;
  auto p16 = [](int64_t b) { return (b + 15) & ~(int64_t)15; };
  return NB * 8 + p16(n * 4) + (pass == 1 ? p16(n * (int64_t)sizeof(V)) : 0) + p16(n * 2) + p16(n);
}

// rank of k among keys[idx[s .. en)] (keys < k); warp-uniform trip count as esc_rank
__device__ __forceinline__ int esc_rank_ind(const uint32_t* keys, const uint16_t* idx, int s, int en, uint32_t k) {
  const int len = en - s;
  const int mx = (int)__reduce_max_sync(0xffffffffu, (unsigned)len);
  int r = 0;
  for (int d = 0; d < mx; d += 4) {
#pragma unroll
    for (int u = 0; u < 4; ++u)
      if (d + u < len) r += keys[idx[s + d + u]] < k;
  }
  return r;
}

// One row by NW warps (warp wi) in `region`; n = products (<= esc_staged_capacity of the region).
//   PASS 0: returns the number of distinct columns (every thread).
//   PASS 1: cnt = exact entries; writes the row sorted at C[cbase, cbase + cnt) and returns cnt.
// -1: the buckets are too uneven (the caller then takes the hash map on the same region).
template <int NW, int PASS, typename V>
__device__ __forceinline__ int esc_row_staged(const SpgemmArgs<V>& p, unsigned char* region, uint32_t region_bytes,
                                              int wi, int64_t a0, int alen, int n, int cnt, int32_t cmin,
                                              int32_t cmax, int64_t cbase, int* red, const PreBatch<V>* pre = nullptr,
                                              const unsigned char* ptbl = nullptr) {
  const int lane = lane_id();
  const int t = wi * 32 + lane;
  constexpr int T = NW * 32;
  int NB = (n + kEscLambda - 1) / kEscLambda;
  NB = (NB + 31) & ~31;
  auto pad16 = [](size_t b) { return (b + 15) & ~(size_t)15; };
  int* bc = reinterpret_cast<int*>(region);
  int* dc = bc + NB;
  uint32_t* keys = reinterpret_cast<uint32_t*>(region + (size_t)NB * 8);
  V* vals = reinterpret_cast<V*>(reinterpret_cast<unsigned char*>(keys) + pad16((size_t)n * 4));
  uint16_t* sidx = reinterpret_cast<uint16_t*>(reinterpret_cast<unsigned char*>(vals) +
                                               (PASS == 1 ? pad16((size_t)n * sizeof(V)) : 0));
  uint8_t* jb = reinterpret_cast<uint8_t*>(sidx) + pad16((size_t)n * 2);
  const uint32_t lo = (uint32_t)cmin;
  const uint32_t range = (uint32_t)(cmax - cmin + 1);
  const uint64_t mult = range ? ((uint64_t)NB << 32) / range : 0;
  // bucket = floor((col - lo) * mult / 2^32), written out as high(x * mult_lo) + x * mult_hi
  const uint32_t mlo = (uint32_t)mult, mhi = (uint32_t)(mult >> 32);
  auto home = [&](uint32_t col) {
    const uint32_t x = col - lo;
    return __umulhi(x, mlo) + x * mhi;
  };
  const bool dups = PASS == 1 && n != cnt;

  for (int b = t; b < NB; b += T) {
    bc[b] = 0;
    if (dups) dc[b] = 0;
  }
  unsigned char* tbl = jb + pad16((size_t)n);
  const bool use_tbl = !ptbl && NW > 1 && kEscTable && (size_t)(tbl - region) + (size_t)esc_tbl_bytes<V>(alen) <= region_bytes;
  if (!use_tbl) esc_sync<NW>();     // (expand_tbl's barrier after the table build orders the clearing)
  // ---- G: gather (column, a*b) in product order; count the buckets --------------------------
  auto gather = [&](uint32_t col, V v, bool act, int pi) {
    if (act) {
      const int j = atomicAdd(&bc[home(col)], 1);
      keys[pi] = col;
      if (PASS == 1) vals[pi] = v;
      jb[pi] = (uint8_t)(j < 255 ? j : 255);
    }
  };
  if (ptbl)
    esc_tbl_gather<PASS, V, NW, PASS == 0 ? 4 : 2>(p, alen, wi, ptbl, gather);   // table built by the caller
  else if (use_tbl)
    expand_tbl<PASS, V, NW, PASS == 0 ? 4 : 2>(p, a0, alen, wi, tbl, gather);   // batches set up once per row
  else
    expand_esc<PASS, V, PASS == 0 ? 4 : 2>(p, a0, alen, wi, NW, gather, pre);
  esc_sync<NW>();
  const int mx = esc_scan<NW>(bc, NB, wi, red);      // bc[b] = first slot of bucket b
  if (mx > kEscMaxBucket) {
    if (t == 0) count_path(p.paths, SPECK_PATH_ESC_FALLBACK);
    return -1;
  }
  if (t == 0) count_path(p.paths, PASS == 0 ? SPECK_PATH_SYM_ESC : dups ? SPECK_PATH_NUM_ESC_DUP : SPECK_PATH_NUM_ESC);
  // ---- F: file every product under its bucket slot (shared memory only) ----------------------
  for (int e = t; e < n; e += T) sidx[bc[home(keys[e])] + jb[e]] = (uint16_t)e;
  esc_sync<NW>();
  auto bend = [&](uint32_t b) { return b + 1 < (uint32_t)NB ? bc[b + 1] : n; };
  if (PASS == 0) {
    // distinct columns = entries without an equal key in an earlier slot of their bucket
    int d = 0;
    for (int q0 = wi * 32; q0 < n; q0 += T) {
      const int q = q0 + lane;
      const bool act = q < n;
      const uint32_t k = act ? keys[sidx[q]] : 0u;
      const uint32_t b = act ? home(k) : 0u;
      const int s = act ? bc[b] : 0, len = act ? q - s : 0;
      const int mxl = (int)__reduce_max_sync(0xffffffffu, (unsigned)len);
      bool first = act;
      for (int j = 0; j < mxl; ++j)
        if (j < len) first &= keys[sidx[s + j]] != k;
      d += first;
    }
    d = warp_sum(d);
    if (NW == 1) return d;
    if (lane == 0) red[2 * NW] = 0;
    __syncthreads();
    if (lane == 0) atomicAdd(&red[2 * NW], d);
    __syncthreads();
    const int total = red[2 * NW];
    __syncthreads();
    return total;
  }
  if (!dups) {
    // sorted position = bucket start + rank in the bucket; slots in bucket order keep the
    // warp's stores to C nearly contiguous
    for (int q0 = wi * 32; q0 < n; q0 += T) {        // warp-uniform: every lane calls esc_rank_ind
      const int q = q0 + lane;
      const bool act = q < n;
      const int e = act ? sidx[q] : 0;
      const uint32_t k = act ? keys[e] : 0u;
      const uint32_t b = act ? home(k) : 0u;
      const int s = act ? bc[b] : 0, en = act ? bend(b) : 0;
      const int r = esc_rank_ind(keys, sidx, s, en, k);
      if (act) {
        p.C_col[cbase + s + r] = (int32_t)k;
        p.C_val[cbase + s + r] = vals[e];
      }
    }
    if (NW == 1) esc_sync<NW>();   // block rows: the caller's barrier follows
    return cnt;
  }
  // ---- repeated columns (rare: C5 has ~1 per 1000 products, but most large rows have one) ----
  // R1: one pass over each entry's bucket gives its rank among ALL keys of the bucket (lt), whether
  // an equal key sits in an earlier slot (then it is a dropped duplicate), and, for the first
  // occurrence, the sum of its equals; first occurrences count one distinct entry for their
  // bucket, and a bucket holding any equal pair is flagged (bit 30 of its start).
  // R2: distinct starts by a scan; an entry of an unflagged bucket is written at distinct start +
  // lt, only flagged buckets rank again among their first occurrences.
  constexpr int kDupF = 0x40000000, kBcMask = 0x3fffffff;
  auto bend2 = [&](uint32_t b) { return b + 1 < (uint32_t)NB ? (bc[b + 1] & kBcMask) : n; };
  for (int q0 = wi * 32; q0 < n; q0 += T) {           // warp-uniform trip counts inside
    const int q = q0 + lane;
    const bool act = q < n;
    const int e = act ? sidx[q] : 0;
    const uint32_t k = act ? keys[e] : 0u;
    const uint32_t b = act ? home(k) : 0u;
    const int s = act ? (bc[b] & kBcMask) : 0, len = act ? bend2(b) - s : 0;
    const int mxl = (int)__reduce_max_sync(0xffffffffu, (unsigned)len);
    int lt = 0;
    bool earlier = false, eq = false;
    V sum = V(0);
    for (int d = 0; d < mxl; ++d) {
      if (d < len && s + d != q) {
        const int f = sidx[s + d];
        const uint32_t kd = keys[f];
        lt += kd < k;
        if (kd == k) {
          eq = true;
          if (s + d < q) earlier = true;
          else sum += vals[f];
        }
      }
    }
    if (act) {
      if (!earlier) {
        if (eq) vals[e] += sum;          // the later equals' values are only read here
        atomicAdd(&dc[b], 1);
      }
      if (eq) atomicOr(&bc[b], kDupF);
      jb[e] = (uint8_t)(lt | (earlier ? 0x80 : 0));
    }
  }
  esc_sync<NW>();
  esc_scan<NW>(dc, NB, wi, red);      // dc[b] = first distinct position of bucket b
  for (int q0 = wi * 32; q0 < n; q0 += T) {
    const int q = q0 + lane;
    const int e = q < n ? sidx[q] : 0;
    const int j = q < n ? jb[e] : 0x80;
    const bool act = !(j & 0x80);
    const uint32_t k = act ? keys[e] : 0u;
    const uint32_t b = act ? home(k) : 0u;
    const int fl = act ? bc[b] : 0;
    int r = j & 0x7f;
    const bool flagged = act && (fl & kDupF);
    if (__any_sync(0xffffffffu, flagged)) {
      const int s = flagged ? (fl & kBcMask) : 0, len = flagged ? bend2(b) - s : 0;
      const int mxl = (int)__reduce_max_sync(0xffffffffu, (unsigned)len);
      int r2 = 0;
      for (int d = 0; d < mxl; ++d) {
        if (d < len) {
          const int f = sidx[s + d];
          r2 += keys[f] < k && !(jb[f] & 0x80);
        }
      }
      if (flagged) r = r2;
    }
    if (act) {
      const int64_t o = cbase + dc[b] + r;
      p.C_col[o] = (int32_t)k;
      p.C_val[o] = vals[e];
    }
  }
  if (NW == 1) esc_sync<NW>();     // block rows: the caller's barrier follows
  return cnt;
}

}  // namespace speck
