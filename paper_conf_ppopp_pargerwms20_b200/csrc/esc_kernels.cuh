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

#include "speck_internal.cuh"

namespace speck {

#ifndef SPECK_ESC_LAMBDA
#define SPECK_ESC_LAMBDA 2
#endif
constexpr int kEscLambda = SPECK_ESC_LAMBDA;   // target products per bucket
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

template <int PASS, typename V, int U, typename F>
__device__ __forceinline__ void expand_esc(const SpgemmArgs<V>& p, int64_t a0, int alen, int wi, int nw, F&& f,
                                           const PreBatch<V>* pre = nullptr) {
  const int lane = lane_id();
  int rot = 0;
  for (int b0 = 0; b0 < alen; b0 += 32) {
    const int fi = b0 + lane;
    int64_t bst = 0;
    int blen = 0;
    V a = V(0);
    if (pre && b0 == 0 && pre->valid) {
      bst = pre->bst;
      blen = pre->blen;
      a = pre->a;
    } else if (fi < alen) {
      const int32_t kc = p.A_col[a0 + fi];
      if (PASS == 1) a = __ldg(p.A_val + a0 + fi);
      bst = p.B_rp[kc];
      blen = (int)(p.B_rp[kc + 1] - bst);
    }
    const uint32_t ne = __ballot_sync(0xffffffffu, blen > 0);
    if (!ne) continue;
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
    const int excl = incl - blen;
    const int Pb = __shfl_sync(0xffffffffu, incl, 31);
    const int64_t boff = bst - excl;          // product pp of owner o is B entry boff_o + pp
    const bool own_any = blen > 0;
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
        f(col[u], av[u] * bv[u], act[u]);
      }
    }
  }
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
    for (int w = 0; w < NW; ++w) {
      if (w < wi) wbase += red[w];
      m2 = max(m2, red[NW + w]);
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
  auto home = [&](uint32_t col) { return (uint32_t)(((uint64_t)(col - lo) * mult) >> 32); };

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
      const uint32_t b = home(k);
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

}  // namespace speck
