// plan_kernels.cuh — row analysis (Alg. 1), classification/binning (global load balancer)
// and the single-pass decoupled look-back scan.  Included by speck_api.cu.
#pragma once

#include <climits>

#include "speck_internal.cuh"

namespace speck {

// ------------------------------------------------------------------------------------
// Row analysis (§4.1, Algorithm 1).  Parallel over the NZ of A:
// GA lanes cooperate on one row, each lane streams a strided part of the row's NZ and
// gathers len(B_k) from B.row_ptr and the first/last column of B_k; a GA-wide shuffle
// reduction produces prods_r, prods_r,max, colmin, colmax.  Global Σprods / max prods and
// the #single-NZ / #empty rows go to the stats block with one atomic per CTA.
// ------------------------------------------------------------------------------------
constexpr int kAnaU = 4;   // NZ per lane per iteration of the analysis

// Per row of B: {length, first column, last column, 0} (first = INT_MAX, last = -1 if empty),
// one 16-byte record, so the analysis makes one random access per NZ of A instead of three
// (the B.row_ptr pair and two B.col gathers).  Built when rows of B are referenced several times.
__global__ void __launch_bounds__(256) k_brow_info(const int64_t* __restrict__ B_rp, const int32_t* __restrict__ B_col,
                                                   int64_t k, int4* __restrict__ info) {
  for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < k; r += (int64_t)gridDim.x * blockDim.x) {
    const int64_t b0 = B_rp[r], b1 = B_rp[r + 1];
    int4 v;
    v.x = (int)(b1 - b0);
    v.y = b1 > b0 ? B_col[b0] : INT_MAX;
    v.z = b1 > b0 ? B_col[b1 - 1] : -1;
    v.w = 0;
    info[r] = v;
  }
}

template <int GA>
__global__ void __launch_bounds__(256) k_analysis(const int64_t* __restrict__ A_rp, const int32_t* __restrict__ A_col,
                                                  const int64_t* __restrict__ B_rp, const int32_t* __restrict__ B_col,
                                                  int64_t m, int64_t* __restrict__ prods, int32_t* __restrict__ maxlen,
                                                  int32_t* __restrict__ colmin, int32_t* __restrict__ colmax,
                                                  AnalysisStats* st, int32_t* __restrict__ long_rows,
                                                  unsigned int* n_long, const int4* __restrict__ binfo) {
  const int sub = threadIdx.x % GA;
  constexpr int RPW = 32 / GA;  // rows per warp and iteration
  const int64_t gwarp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t wstride = ((int64_t)gridDim.x * blockDim.x >> 5) * RPW;
  unsigned long long t_sum = 0, t_max = 0, t_direct = 0, t_empty = 0, t_maxa = 0;
  // warp-uniform loop so the GA-wide shuffles always see the whole warp
  for (int64_t wrow0 = gwarp * RPW; wrow0 < m; wrow0 += wstride) {
    const int64_t row = wrow0 + lane_id() / GA;
    bool valid = row < m;
    int64_t a0 = valid ? A_rp[row] : 0, a1 = valid ? A_rp[row + 1] : 0;
    if (long_rows && a1 - a0 > kAnaLong) {
      // very long rows of A (e.g. C4's 200k-NZ rows) go to k_analysis_long: one CTA each
      if (sub == 0) long_rows[atomicAdd(n_long, 1u)] = (int32_t)row;
      valid = false;
      a1 = a0;
    }
    int64_t p = 0;
    int32_t ml = 0, cmin = INT_MAX, cmax = -1;
    // kAnaU NZ per lane per iteration, each stage's loads issued together (the A col ->
    // B row_ptr -> B col chain is three dependent round trips; unrolling overlaps them)
    for (int64_t q = a0 + sub; q < a1; q += GA * kAnaU) {
      int32_t k[kAnaU];
      int64_t b0[kAnaU], b1[kAnaU];
#pragma unroll
      for (int u = 0; u < kAnaU; ++u) k[u] = q + u * GA < a1 ? A_col[q + u * GA] : -1;
      if (binfo) {
        int4 r[kAnaU];
#pragma unroll
        for (int u = 0; u < kAnaU; ++u) r[u] = k[u] >= 0 ? __ldg(binfo + k[u]) : make_int4(0, INT_MAX, -1, 0);
#pragma unroll
        for (int u = 0; u < kAnaU; ++u) {
          p += r[u].x;
          ml = max(ml, r[u].x);
          cmin = min(cmin, r[u].y);
          cmax = max(cmax, r[u].z);
        }
        continue;
      }
#pragma unroll
      for (int u = 0; u < kAnaU; ++u) {
        b0[u] = k[u] >= 0 ? B_rp[k[u]] : 0;
        b1[u] = k[u] >= 0 ? B_rp[k[u] + 1] : 0;
      }
#pragma unroll
      for (int u = 0; u < kAnaU; ++u) {
        const int64_t len = b1[u] - b0[u];
        p += len;
        ml = max(ml, (int32_t)len);
        if (len > 0) {
          cmin = min(cmin, B_col[b0[u]]);
          cmax = max(cmax, B_col[b1[u] - 1]);
        }
      }
    }
#pragma unroll
    for (int o = GA / 2; o > 0; o >>= 1) {
      p += __shfl_xor_sync(0xffffffffu, p, o, GA);
      ml = max(ml, __shfl_xor_sync(0xffffffffu, ml, o, GA));
      cmin = min(cmin, __shfl_xor_sync(0xffffffffu, cmin, o, GA));
      cmax = max(cmax, __shfl_xor_sync(0xffffffffu, cmax, o, GA));
    }
    if (valid && sub == 0) {
      prods[row] = p;
      if (maxlen) maxlen[row] = ml;
      if (colmin) colmin[row] = cmin;
      if (colmax) colmax[row] = cmax;
      t_sum += (unsigned long long)p;
      t_max = max(t_max, (unsigned long long)p);
      t_direct += (a1 - a0 == 1 && p > 0);
      t_empty += (p == 0);
      t_maxa = max(t_maxa, (unsigned long long)(a1 - a0));
    }
  }
  if (st == nullptr) return;
  // CTA reduction -> one atomic per statistic per CTA
  __shared__ unsigned long long red[5][8];
  t_sum = warp_sum(t_sum);
  t_direct = warp_sum(t_direct);
  t_empty = warp_sum(t_empty);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    t_max = max(t_max, __shfl_xor_sync(0xffffffffu, t_max, o));
    t_maxa = max(t_maxa, __shfl_xor_sync(0xffffffffu, t_maxa, o));
  }
  if (lane_id() == 0) {
    red[0][warp_id()] = t_sum; red[1][warp_id()] = t_max; red[2][warp_id()] = t_direct;
    red[3][warp_id()] = t_empty; red[4][warp_id()] = t_maxa;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long s = 0, mx = 0, d = 0, e = 0, ma = 0;
    for (int w = 0; w < (int)(blockDim.x / 32); ++w) {
      s += red[0][w]; mx = max(mx, red[1][w]); d += red[2][w]; e += red[3][w]; ma = max(ma, red[4][w]);
    }
    atomicAdd(&st->sum_prods, s);
    atomicMax(&st->max_prods, mx);
    atomicAdd(&st->n_direct, d);
    atomicAdd(&st->n_empty, e);
    atomicMax(&st->max_nnza, ma);
  }
}

// Rows of A with more than kAnaLong NZ: one CTA per row, block-wide reduction.
__global__ void __launch_bounds__(256) k_analysis_long(const int64_t* __restrict__ A_rp, const int32_t* __restrict__ A_col,
                                                       const int64_t* __restrict__ B_rp, const int32_t* __restrict__ B_col,
                                                       int64_t* __restrict__ prods, int32_t* __restrict__ maxlen,
                                                       int32_t* __restrict__ colmin, int32_t* __restrict__ colmax,
                                                       AnalysisStats* st, const int32_t* __restrict__ long_rows,
                                                       const unsigned int* n_long) {
  __shared__ int64_t sp[8];
  __shared__ int32_t sml[8], smn[8], smx[8];
  const unsigned n = *n_long;
  for (unsigned i = blockIdx.x; i < n; i += gridDim.x) {
    const int32_t row = long_rows[i];
    const int64_t a0 = A_rp[row], a1 = A_rp[row + 1];
    int64_t p = 0;
    int32_t ml = 0, cmin = INT_MAX, cmax = -1;
    for (int64_t q = a0 + threadIdx.x; q < a1; q += blockDim.x) {
      const int32_t k = A_col[q];
      const int64_t b0 = B_rp[k], b1 = B_rp[k + 1];
      const int64_t len = b1 - b0;
      p += len;
      ml = max(ml, (int32_t)len);
      if (len > 0) {
        cmin = min(cmin, B_col[b0]);
        cmax = max(cmax, B_col[b1 - 1]);
      }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      p += __shfl_xor_sync(0xffffffffu, p, o);
      ml = max(ml, __shfl_xor_sync(0xffffffffu, ml, o));
      cmin = min(cmin, __shfl_xor_sync(0xffffffffu, cmin, o));
      cmax = max(cmax, __shfl_xor_sync(0xffffffffu, cmax, o));
    }
    if (lane_id() == 0) { sp[warp_id()] = p; sml[warp_id()] = ml; smn[warp_id()] = cmin; smx[warp_id()] = cmax; }
    __syncthreads();
    if (threadIdx.x == 0) {
      for (int w = 1; w < (int)(blockDim.x / 32); ++w) {
        p += sp[w]; ml = max(ml, sml[w]); cmin = min(cmin, smn[w]); cmax = max(cmax, smx[w]);
      }
      prods[row] = p;
      if (maxlen) maxlen[row] = ml;
      if (colmin) colmin[row] = cmin;
      if (colmax) colmax[row] = cmax;
      if (st) {
        atomicAdd(&st->sum_prods, (unsigned long long)p);
        atomicMax(&st->max_prods, (unsigned long long)p);
        if (p == 0) atomicAdd(&st->n_empty, 1ull);
        atomicMax(&st->max_nnza, (unsigned long long)(a1 - a0));
      }
    }
    __syncthreads();
  }
}

// ------------------------------------------------------------------------------------
// Global load balancer, step 1: classify every row into a bin and count the
// rows of each bin per tile of kBinTile rows: hist[cat * n_tiles + tile].
// The numeric pass classifies by the exact row size from the symbolic step
// and also records the largest row size (max_cnt) for the no-balancing decision.
// ------------------------------------------------------------------------------------
__global__ void __launch_bounds__(kBinTile) k_classify(const int64_t* __restrict__ A_rp, const int64_t* __restrict__ prods,
                                                       const int64_t* __restrict__ C_rp, int64_t m, BinParams bp,
                                                       int64_t* __restrict__ hist, int64_t n_tiles,
                                                       unsigned long long* __restrict__ bin_sums) {
  // per category: rows (histogram) and, for the statistics / per-kernel byte model, the sums
  // of nnz(A_i), products and (numeric) nnz(C_i) — bin_sums[cat * 3 + {0, 1, 2}]
  __shared__ int cnt[CAT_COUNT];
  __shared__ unsigned long long sums[CAT_COUNT][3];
  if (threadIdx.x < CAT_COUNT) cnt[threadIdx.x] = 0;
  if (threadIdx.x < CAT_COUNT * 3) sums[threadIdx.x / 3][threadIdx.x % 3] = 0ull;
  __syncthreads();
  const int64_t row = (int64_t)blockIdx.x * kBinTile + threadIdx.x;
  if (row < m) {
    const int64_t nnza = A_rp[row + 1] - A_rp[row];
    const int64_t c = bp.pass ? C_rp[row + 1] - C_rp[row] : 0;
    const int64_t p = prods[row];
    const int cat = classify_row(nnza, p, c, bp);
    // warp-aggregated increment
    const uint32_t peers = __match_any_sync(__activemask(), cat);
    if (lane_id() == __ffs(peers) - 1) atomicAdd(&cnt[cat], __popc(peers));
    if (bin_sums) {
      // warp-aggregated: sum over the lanes of the same category in 16-bit halves (rows < 2^40)
      auto wsum = [&](unsigned long long x) {
        const unsigned lo = __reduce_add_sync(peers, (unsigned)(x & 0xffffu));
        const unsigned hi = __reduce_add_sync(peers, (unsigned)(x >> 16));
        return (unsigned long long)lo + ((unsigned long long)hi << 16);
      };
      const unsigned long long s0 = wsum((unsigned long long)nnza), s1 = wsum((unsigned long long)p),
                               s2 = bp.pass ? wsum((unsigned long long)c) : 0ull;
      if (lane_id() == __ffs(peers) - 1) {
        atomicAdd(&sums[cat][0], s0);
        atomicAdd(&sums[cat][1], s1);
        if (bp.pass) atomicAdd(&sums[cat][2], s2);
      }
    }
  }
  __syncthreads();
  if (threadIdx.x < CAT_COUNT) hist[(int64_t)threadIdx.x * n_tiles + blockIdx.x] = cnt[threadIdx.x];
  if (bin_sums && threadIdx.x < CAT_COUNT * 3) {
    const unsigned long long v = sums[threadIdx.x / 3][threadIdx.x % 3];
    if (v) atomicAdd(&bin_sums[threadIdx.x], v);
  }
}

// ------------------------------------------------------------------------------------
// Global load balancer, step 2 (after scanning hist): every tile writes its rows into the
// bins in CSR order — a block-local prefix sum per bin and one write position per bin per
// tile ("we perform binning locally in each block first and append them globally in a
// single transaction ... to ensure the ordering is kept").  Rows whose C size
// is already known from the analysis (empty, direct) get cnt written here (symbolic).
// ------------------------------------------------------------------------------------
__global__ void __launch_bounds__(kBinTile) k_bin_scatter(const int64_t* __restrict__ A_rp, const int64_t* __restrict__ prods,
                                                          const int64_t* __restrict__ C_rp, int64_t m, BinParams bp,
                                                          const int64_t* __restrict__ offs, int64_t n_tiles,
                                                          int32_t* __restrict__ bins, int64_t* __restrict__ cnt_out) {
  __shared__ int wcnt[CAT_COUNT][kBinTile / 32];
  const int64_t row = (int64_t)blockIdx.x * kBinTile + threadIdx.x;
  int cat = -1;
  if (row < m) {
    const int64_t nnza = A_rp[row + 1] - A_rp[row];
    const int64_t p = prods[row];
    const int64_t c = bp.pass ? C_rp[row + 1] - C_rp[row] : 0;
    cat = classify_row(nnza, p, c, bp);
    if (bp.pass == 0 && cnt_out && (cat == CAT_EMPTY || cat == CAT_DIRECT)) cnt_out[row] = p;
  }
  // per-warp ballots per category, then a prefix over warps
  int my_rank = 0;
#pragma unroll
  for (int c = 0; c < CAT_COUNT; ++c) {
    const uint32_t b = __ballot_sync(0xffffffffu, cat == c);
    if (cat == c) my_rank = __popc(b & ((1u << lane_id()) - 1u));
    if (lane_id() == 0) wcnt[c][warp_id()] = __popc(b);
  }
  __syncthreads();
  if (threadIdx.x < CAT_COUNT * 32) {
    // warp w of the first CAT_COUNT warps scans category w over the 32 warps
    const int c = warp_id();
    const int v = wcnt[c][lane_id()];
    const int inc = warp_incl_scan(v);
    wcnt[c][lane_id()] = inc - v;
  }
  __syncthreads();
  if (cat >= 0) {
    const int64_t pos = offs[(int64_t)cat * n_tiles + blockIdx.x] + wcnt[cat][warp_id()] + my_rank;
    bins[pos] = (int32_t)row;
  }
}

// ------------------------------------------------------------------------------------
// Row-range numeric (speck_spgemm_rows): the bins keep CSR order, so the rows of [r0, r1) form
// one contiguous sub-range of every category's bin.  Thread c finds category c's sub-range by
// binary search; out[2c], out[2c+1] = begin / end positions in `bins`; out[2 CAT_COUNT],
// out[2 CAT_COUNT + 1] = C_rp[r0], C_rp[r1] (the chunk's entries).
// ------------------------------------------------------------------------------------
struct CatStarts { int64_t s[CAT_COUNT + 1]; };
__global__ void k_bin_range(const int32_t* __restrict__ bins, CatStarts cs, int64_t r0, int64_t r1,
                            const int64_t* __restrict__ C_rp, int64_t* __restrict__ out) {
  const int c = threadIdx.x;
  if (c < CAT_COUNT) {
    auto lb = [&](int64_t x) {
      int64_t l = cs.s[c], h = cs.s[c + 1];
      while (l < h) {
        const int64_t mid = (l + h) >> 1;
        if ((int64_t)bins[mid] < x) l = mid + 1; else h = mid;
      }
      return l;
    };
    out[2 * c] = lb(r0);
    out[2 * c + 1] = lb(r1);
  }
  if (c == 0) { out[2 * CAT_COUNT] = C_rp[r0]; out[2 * CAT_COUNT + 1] = C_rp[r1]; }
}

// Memory-bounded chunks (speck_row_chunks): bound_j = first row whose C offset is >= j * step,
// j = 1 .. parts-1 (step = max_nnz - longest row), so every chunk holds < max_nnz entries.
__global__ void k_chunk_bounds(const int64_t* __restrict__ C_rp, int64_t m, int64_t step, int64_t parts,
                               int64_t* __restrict__ out) {
  const int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (j > parts) return;
  if (j == 0) { out[0] = 0; return; }
  if (j == parts) { out[parts] = m; return; }
  const int64_t x = j * step;
  int64_t l = 0, h = m;
  while (l < h) {
    const int64_t mid = (l + h) >> 1;
    if (C_rp[mid] < x) l = mid + 1; else h = mid;
  }
  out[j] = l;
}

// ------------------------------------------------------------------------------------
// Single-pass exclusive scan of int64 (decoupled look-back), used for the C row offsets
// and for the bin offsets.  out[0..n] with out[n] = total.  Each CTA takes
// a dynamic tile id so predecessors are always scheduled before successors.
// status[t]: bits 62..63 = flag (0 none, 1 aggregate, 2 inclusive prefix), bits 0..61 value.
// Also reports max(in) through *max_out if non-null.
// ------------------------------------------------------------------------------------
constexpr int kScanThreads = 256;
constexpr int kScanItems = 8;
constexpr int kScanTile = kScanThreads * kScanItems;
constexpr unsigned long long kFlagAgg = 1ull << 62;
constexpr unsigned long long kFlagInc = 2ull << 62;
constexpr unsigned long long kValMask = (1ull << 62) - 1;

__global__ void __launch_bounds__(kScanThreads) k_scan(const int64_t* __restrict__ in, int64_t n, int64_t* __restrict__ out,
                                                       unsigned long long* status, unsigned int* tile_counter,
                                                       unsigned long long* max_out) {
  __shared__ int64_t part[kScanThreads / 32 + 1];
  __shared__ unsigned int s_tile;
  __shared__ int64_t s_prefix;
  if (threadIdx.x == 0) s_tile = atomicAdd(tile_counter, 1u);
  __syncthreads();
  const int64_t tile = s_tile;
  const int64_t base = tile * kScanTile + (int64_t)threadIdx.x * kScanItems;
  int64_t v[kScanItems];
  int64_t local = 0, lmax = 0;
#pragma unroll
  for (int i = 0; i < kScanItems; ++i) {
    v[i] = base + i < n ? in[base + i] : 0;
    local += v[i];
    lmax = max(lmax, v[i]);
  }
  int64_t total;
  int64_t excl = block_excl_scan<kScanThreads>(local, part, &total);
  if (threadIdx.x == 0) {
    if (tile == 0) {
      atomicExch(&status[0], kFlagInc | (unsigned long long)total);
      s_prefix = 0;
    } else {
      atomicExch(&status[tile], kFlagAgg | (unsigned long long)total);
      int64_t prefix = 0;
      int64_t t = tile - 1;
      while (true) {
        unsigned long long s = atomicAdd(&status[t], 0ull);   // L2-coherent read
        if ((s >> 62) == 0) continue;                          // predecessor not ready: spin
        prefix += (int64_t)(s & kValMask);
        if ((s >> 62) == 2) break;
        --t;
      }
      atomicExch(&status[tile], kFlagInc | (unsigned long long)(prefix + total));
      s_prefix = prefix;
    }
  }
  if (max_out) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) lmax = max(lmax, __shfl_xor_sync(0xffffffffu, lmax, o));
    if (lane_id() == 0) atomicMax(max_out, (unsigned long long)lmax);
  }
  __syncthreads();
  int64_t run = s_prefix + excl;
  // launched with n / kScanTile + 1 tiles, so exactly one thread covers position n
#pragma unroll
  for (int i = 0; i < kScanItems; ++i) {
    if (base + i <= n) out[base + i] = run;   // position n receives the total
    run += v[i];
  }
}

// ------------------------------------------------------------------------------------
// Input validation (SPECK_OPT_VALIDATE): columns strictly ascending and in range.
// ------------------------------------------------------------------------------------
__global__ void k_validate(const int64_t* __restrict__ rp, const int32_t* __restrict__ col, int64_t rows, int64_t ncols,
                           int* bad) {
  for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < rows; r += (int64_t)gridDim.x * blockDim.x) {
    const int64_t a = rp[r], b = rp[r + 1];
    if (b < a) { atomicOr(bad, 1); continue; }
    for (int64_t q = a; q < b; ++q) {
      const int32_t c = col[q];
      if (c < 0 || c >= ncols || (q > a && c <= col[q - 1])) { atomicOr(bad, 1); break; }
    }
  }
}

}  // namespace speck
