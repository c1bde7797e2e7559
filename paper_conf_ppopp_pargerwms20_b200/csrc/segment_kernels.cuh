// segment_kernels.cuh — numeric long rows (beyond the largest hash map).
//
// The paper processes a row that needs the largest kernel with windowed dense accumulation,
// one window after the other inside one block.  B200 keeps that
// for rows whose window overhead is small ("windows" jobs: one CTA of configuration kSegCfg,
// dense windows of that configuration's shared memory, each referenced B row located in the
// window by binary search), and splits the others into *column segments*: consecutive
// 2^s-column chunks grouped so that each segment's exact size (from the per-chunk counts the
// symbolic pass recorded) fits the kSegCfg hash map at the ordered fill (ordered hash, sorted
// write-out), or a single chunk that is accumulated densely.  kSegCfg = 3 (512 threads,
// 2 CTAs/SM) so two jobs share an SM and one job's barriers hide behind the other's work.  Segments of one row are independent CTAs writing disjoint, known
// ranges of the row, so a long, wide, sparse row (C5) or one of a few giant rows (C4) is
// spread over many SMs.
#pragma once

#include "spgemm_kernels.cuh"

namespace speck {

enum SegMode : int { SEG_HASH = 0, SEG_DENSE = 1, SEG_WINDOWS = 2 };

// Greedy grouping of a row's chunks [c0, c1] (counts cc) into segments; calls emit(lo_chunk,
// hi_chunk_exclusive, cnt, out_offset_in_row, dense).  `limit` = max entries of a hashed
// segment; a chunk above it is a dense segment of its own.
template <typename F>
__device__ void plan_row_segments(const int32_t* cc, int c0, int c1, int64_t limit, F&& emit) {
  int cs = c0;
  int64_t sum = 0, done = 0;
  for (int c = c0; c <= c1; ++c) {
    const int64_t x = cc[c];
    if (x > limit) {
      if (sum > 0) emit(cs, c, sum, done, false);
      done += sum;
      emit(c, c + 1, x, done, true);
      done += x;
      sum = 0;
      cs = c + 1;
    } else if (sum + x > limit) {
      emit(cs, c, sum, done, false);
      done += sum;
      sum = x;
      cs = c;
    } else {
      sum += x;
    }
  }
  if (sum > 0) emit(cs, c1 + 1, sum, done, false);
}

struct SegPlanArgs {
  const int32_t* cand;     // long-row candidates (the symbolic cfg4 bin)
  int64_t ncand;
  const int64_t* C_rp;
  const int64_t* A_rp;
  const int64_t* prods;
  const int32_t* colmin;
  const int32_t* colmax;
  const int32_t* chunk_cnt;
  int nchunks;
  int shift;
  int64_t limit;           // numeric long-row threshold (entries of the largest map)
  int64_t seg_limit;       // max entries of a hashed segment (map of kSegCfg)
  int64_t dense_window;    // columns of one dense window of the largest configuration
  int64_t map_slots;       // slots of the largest numeric hash map
  int prefer_parallel;     // few long rows: always split (parallelism across SMs)
  int64_t bitmap_cols;     // >0: rows whose column range fits are done by k_long_bitmap (no segments)
  const uint32_t* bm_pool; // bitmaps kept by the symbolic step (SpgemmArgs::bm_pool), or null
  const int64_t* bm_off;   // per candidate: word offset in bm_pool, -1 = rebuild
  int split_max;           // >1: CTAs per candidate; rows with a kept bitmap split their A entries
                           //     over up to this many CTAs (C.val zeroed beforehand by the host)
};
#ifndef SPECK_SPLIT_LOG2
#define SPECK_SPLIT_LOG2 18     // C4 long_bitmap 2.95 -> 2.68 ms (profiles/r02/r02aq_*)
#endif
#ifndef SPECK_SPLIT_MAX_CAND
#define SPECK_SPLIT_MAX_CAND 4096
#endif
constexpr int64_t kSplitProducts = (int64_t)1 << SPECK_SPLIT_LOG2;   // products per CTA of a split long row
constexpr int kSplitPieces = 8;               // CTAs per candidate when splitting
constexpr int64_t kSplitMaxCand = SPECK_SPLIT_MAX_CAND;   // split only with few candidates (grid = candidates x pieces)

// Long rows whose column range fits the shared-memory bitmap of k_long_bitmap.
__device__ __forceinline__ bool bitmap_row(const SegPlanArgs& a, int32_t row) {
  if (a.bitmap_cols <= 0) return false;
  return (int64_t)a.colmax[row] + 1 - (a.colmin[row] & ~31) <= a.bitmap_cols;
}

// One "windows" job or column segments for a long row: estimated per-row overheads (the
// products themselves cost the same either way).  Windows: per window, clear + scan the dense
// array and revisit every referenced B row (resume position + one binary search).  Segments:
// per segment, two binary searches per referenced B row and a map clear.  With few long rows
// the row is always split so its work spreads over the SMs.
__device__ __forceinline__ bool use_windows(const SegPlanArgs& a, int32_t row, int64_t cnt, int64_t map_slots) {
  if (a.prefer_parallel) return false;
  const int64_t range = (int64_t)a.colmax[row] - a.colmin[row] + 1;
  const int64_t nwin = (range + a.dense_window - 1) / a.dense_window;
  const int64_t dA = a.A_rp[row + 1] - a.A_rp[row];
  const int64_t avg = dA > 0 ? a.prods[row] / dA + 1 : 1;
  int64_t lg = 1;
  while ((int64_t)1 << lg < avg) ++lg;
  const int64_t nseg = cnt / a.seg_limit + 1;
  const int64_t win_cost = nwin * (a.dense_window / 8 + dA * (1 + lg));
  const int64_t seg_cost = nseg * (dA * 2 * lg + map_slots / 4);
  return win_cost <= seg_cost;
}

// Pass 1: number of jobs of every long-row candidate (one thread per candidate).
__global__ void k_seg_count(SegPlanArgs a, int64_t* __restrict__ nseg) {
  const int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (e >= a.ncand) return;
  const int32_t row = a.cand[e];
  const int64_t cnt = a.C_rp[row + 1] - a.C_rp[row];
  int64_t n = 0;
  if (cnt > a.limit && !bitmap_row(a, row)) {
    if (use_windows(a, row, cnt, a.map_slots)) {
      n = 1;
    } else {
      plan_row_segments(a.chunk_cnt + e * a.nchunks, a.colmin[row] >> a.shift, a.colmax[row] >> a.shift, a.seg_limit,
                        [&](int, int, int64_t, int64_t, bool) { ++n; });
    }
  }
  nseg[e] = n;
}

// Pass 2: write the job descriptors at the scanned offsets.
__global__ void k_seg_emit(SegPlanArgs a, const int64_t* __restrict__ seg_off, Seg* __restrict__ segs) {
  const int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (e >= a.ncand) return;
  const int32_t row = a.cand[e];
  const int64_t c0 = a.C_rp[row];
  const int64_t cnt = a.C_rp[row + 1] - c0;
  if (cnt <= a.limit || bitmap_row(a, row)) return;
  const int32_t lo = a.colmin[row], hi = a.colmax[row];
  int64_t o = seg_off[e];
  if (use_windows(a, row, cnt, a.map_slots)) {
    Seg s;
    s.row = row; s.col_lo = lo; s.col_hi = hi + 1; s.cnt = (int32_t)(cnt < 0x7fffffff ? cnt : 0x7fffffff); s.out = c0;
    s.dense = SEG_WINDOWS; s.pad = 0;
    segs[o] = s;
    return;
  }
  const int shift = a.shift;
  plan_row_segments(a.chunk_cnt + e * a.nchunks, lo >> shift, hi >> shift, a.seg_limit,
                    [&](int ca, int cb, int64_t n, int64_t done, bool dense) {
                      Seg s;
                      s.row = row;
                      s.col_lo = max(lo, ca << shift);
                      s.col_hi = (int32_t)min((int64_t)hi + 1, (int64_t)cb << shift);
                      s.cnt = (int32_t)n;
                      s.out = c0 + done;
                      const int64_t range = (int64_t)s.col_hi - s.col_lo;
                      // dense when forced by size, or when the segment is dense enough to skip
                      // hashing and sorting altogether (18% rule)
                      s.dense = (dense || (range <= a.dense_window && n * 100 > (int64_t)kDensePct * range)) ? SEG_DENSE
                                                                                                               : SEG_HASH;
                      s.pad = 0;
                      segs[o++] = s;
                    });
}

// Dense window [wlo, whi) of a row -> flags/values in shared memory -> compacted, sorted
// output at `out`; returns the entries written.  Block-wide (barriers inside).
template <typename V, int T, typename Rng>
__device__ int64_t dense_window_pass(const SpgemmArgs<V>& p, int64_t a0, int alen, uint32_t* bits, V* dvals,
                                     uint32_t wlo, uint32_t whi, int64_t out, int64_t* part, Rng rng) {
  constexpr int NW = T / 32;
  const int tid = threadIdx.x;
  const uint32_t range = whi - wlo;
  const int nwords = (int)((range + 31) / 32);
  for (int i = tid; i < nwords; i += T) bits[i] = 0u;
  for (uint32_t i = tid; i < range; i += T) dvals[i] = V(0);
  __syncthreads();
  expand_row<1, V>(p, a0, alen, warp_id(), NW,
                   [&](uint32_t col, V v, bool act) { dense_insert<1, V>(bits, dvals, wlo, col, v, act); }, rng);
  __syncthreads();
  return dense_emit<T, V>(bits, dvals, nwords, wlo, out, p.C_col, p.C_val, part);
}

// One CTA of configuration kSegCfg (2 CTAs/SM) per job.
template <typename V>
__global__ void __launch_bounds__(kCfgThreads[kSegCfg], 1024 / kCfgThreads[kSegCfg])
    k_segments(const __grid_constant__ SpgemmArgs<V> p, const Seg* __restrict__ segs) {
  constexpr int CFG = kSegCfg;
  constexpr int T = kCfgThreads[CFG];
  constexpr int NW = T / 32;
  extern __shared__ __align__(16) unsigned char smem[];
  __shared__ int64_t part[33];
  __shared__ int s_wrap;
  const int tid = threadIdx.x;
  const Seg sg = segs[blockIdx.x];
  if (sg.row < p.row_lo || sg.row >= p.row_hi) return;    // row-range numeric: another chunk's row
  const int64_t a0 = p.A_rp[sg.row];
  const int alen = (int)(p.A_rp[sg.row + 1] - a0);
  const uint32_t lo = (uint32_t)sg.col_lo, hi = (uint32_t)sg.col_hi, range = hi - lo;
  if (tid == 0)
    count_path(p.paths, sg.dense == SEG_HASH ? SPECK_PATH_SEG_HASH : sg.dense == SEG_DENSE ? SPECK_PATH_SEG_DENSE
                                                                                         : SPECK_PATH_SEG_WINDOWS);

  if (sg.dense == SEG_HASH && kEscStaged && p.esc >= 1) {
    // counting sort of the segment (esc_row_staged): the clipped reference table goes to the
    // end of the region, the products of the segment are counted from it; segments that do not
    // fit (or have uneven buckets) take the ordered hash map below
    constexpr uint32_t R = (uint32_t)kCfgMapBytes[CFG];
    const int64_t tb = esc_tbl_bytes<V>(alen);
    if (tb + 4096 <= (int64_t)R) {
      const uint32_t toff = (uint32_t)(((int64_t)R - tb) & ~(int64_t)15);
      unsigned char* tbl = smem + toff;
      esc_tbl_build<1, V, NW>(p, a0, alen, warp_id(), tbl, true, lo, hi);
      const int* tpb = EscTbl<V>(tbl, alen).pb;
      int64_t n = 0;
      for (int j = 0; j < (alen + 31) >> 5; ++j) n += tpb[j];
      if (n > 0 && n <= 65535 && esc_staged_bytes<V>(1, n) <= (int64_t)toff) {
        const int c = esc_row_staged<NW, 1, V>(p, smem, toff, warp_id(), a0, alen, (int)n, sg.cnt, (int32_t)lo,
                                               (int32_t)(hi - 1), sg.out, reinterpret_cast<int*>(part), nullptr, tbl);
        if (c >= 0) return;
      }
      __syncthreads();   // the hash map below reuses the region
    }
  }
  if (sg.dense == SEG_HASH) {
    uint32_t* keys = reinterpret_cast<uint32_t*>(smem);
    V* vals = reinterpret_cast<V*>(smem + num_val_offset<V>(CFG));
    const uint32_t S = num_map_cap<V>(CFG);
    const uint64_t mmult = bkt_mult(range, S);
    for (uint32_t i = tid; i < S; i += T) { keys[i] = kEmptyKey; vals[i] = V(0); }
    if (tid == 0) s_wrap = 0;
    __syncthreads();
    int wrapped = 0;
    expand_row<1, V>(
        p, a0, alen, warp_id(), NW,
        [&](uint32_t col, V v, bool act) {
          uint32_t s = 0;
          if (act) s = probe_insert_bkt(keys, S >> 3, bkt_home(col, lo, mmult), col, &wrapped);
          bool leader;
          const V sum = warp_key_sum(col, v, leader);
          if (act && leader) atomicAdd(&vals[s], sum);
        },
        SegRange{p.B_col, lo, hi});
    if (wrapped) s_wrap = 1;
    __syncthreads();
    if (!s_wrap) {
      block_write_ordered<T, V>(keys, vals, S, sg.out, p.C_col, p.C_val, part);
    } else {
      // compaction + bitonic sort (a probing run wrapped around)
      int64_t running = 0;
      for (uint32_t base = 0; base < S; base += T) {
        const uint32_t s = base + tid;
        uint32_t kk = kEmptyKey;
        V vv = V(0);
        if (s < S) { kk = keys[s]; vv = vals[s]; }
        const int64_t fl = kk != kEmptyKey;
        int64_t tot;
        const int64_t pos = block_excl_scan<T>(fl, part, &tot);
        if (fl) { keys[running + pos] = kk; vals[running + pos] = vv; }
        running += tot;
        __syncthreads();
      }
      smem_bitonic_sort<T, V>(keys, vals, (int)running);
      for (int i = tid; i < (int)running; i += T) {
        p.C_col[sg.out + i] = (int32_t)keys[i];
        p.C_val[sg.out + i] = vals[i];
      }
    }
  } else {
    const int64_t W = num_dense_window<V>(CFG);
    uint32_t* bits = reinterpret_cast<uint32_t*>(smem);
    V* dvals = reinterpret_cast<V*>(smem + ((((W + 31) / 32) * 4 + 15) / 16) * 16);
    if (sg.dense == SEG_DENSE) {
      dense_window_pass<V, T>(p, a0, alen, bits, dvals, lo, hi, sg.out, part, SegRange{p.B_col, lo, hi});
    } else {
      // whole row, dense windows in ascending column order; each referenced B
      // row is located in the window by binary search (two CTAs share an SM, so the per-SM
      // resume slots of the largest configuration are not used here)
      int64_t out = sg.out;
      for (uint32_t wlo = lo; wlo < hi; wlo = (uint32_t)min((int64_t)hi, (int64_t)wlo + W)) {
        const uint32_t whi = (uint32_t)min((int64_t)hi, (int64_t)wlo + W);
        out += dense_window_pass<V, T>(p, a0, alen, bits, dvals, wlo, whi, out, part, SegRange{p.B_col, wlo, whi});
      }
    }
  }
}


// ------------------------------------------------------------------------------------
// Long rows by bitmap + rank (B200 design for rows beyond the largest hash map whose column
// range fits a shared-memory bitmap; C3's ~175k long rows): one CTA of 1024 threads per row.
//   1. structure: every product sets its column's bit (the symbolic pass's dense bitmap,
//      P:1064-1084) — or, when the symbolic step kept this row's bitmap in the pool
//      (SPECK_OPT_BITMAP_REUSE), the bitmap is loaded from there and no product is expanded;
//   2. one block scan gives every 32-bit word its exclusive prefix = the output position of
//      its first entry; C.col is written in order from the bitmap (sorted by construction)
//      and the row's C.val range is zeroed;
//   3. values: every product's position is prefix[word] + popc(lower bits of its word), and
//      a·b is added there with a global atomic (the row's C range stays in L2).
// No column segments, no binary searches in B rows, no hash probing and no sort.  Hub rows of
// B (>= kLongB entries) referenced by the row are streamed by all 32 warps from a shared list,
// the other batches go round-robin over the warps, so no warp is left with a hub row alone.  Columns are
// relative to lo = colmin & ~31; smem: bits (4 B/word) + per-word prefix within its 32-word
// group (uint16) + per-group prefix (int32).
// ------------------------------------------------------------------------------------
constexpr int kBitmapThreads = 1024;
// 196 B of shared memory per 32-word group (128 bits + 4 prefix + 64 word prefixes)
constexpr int64_t kBitmapMaxCols = (int64_t)(kCfgMapBytes[kNumCfg - 1] / 196) * 1024;

// Split long rows (SegPlanArgs::split_max > 1) add their values with global atomics from several
// CTAs: zero exactly those rows' C.val ranges first (one CTA per candidate; the rows that will
// not be split zero their own range inside k_long_bitmap).
template <typename V>
__global__ void __launch_bounds__(256) k_zero_split_rows(const __grid_constant__ SpgemmArgs<V> p,
                                                         const __grid_constant__ SegPlanArgs a) {
  const int32_t row = a.cand[blockIdx.x];
  if (row < p.row_lo || row >= p.row_hi) return;
  const int64_t ob = a.C_rp[row], cnt = a.C_rp[row + 1] - ob;
  if (cnt <= a.limit || !bitmap_row(a, row)) return;
  if (a.bm_off[blockIdx.x] < 0 || p.prods[row] / kSplitProducts < 2) return;   // one piece: zeroed in place
  for (int64_t i = threadIdx.x; i < cnt; i += blockDim.x) p.C_val[ob + i] = V(0);
}

template <typename V>
__global__ void __launch_bounds__(kBitmapThreads, 1) k_long_bitmap(const __grid_constant__ SpgemmArgs<V> p, const __grid_constant__ SegPlanArgs a) {
  constexpr int T = kBitmapThreads, NW = T / 32;
  extern __shared__ __align__(16) unsigned char smem[];
  __shared__ int64_t part[NW + 1];
  __shared__ LongList<V> longs;
  const int ci = blockIdx.x / a.split_max, piece = blockIdx.x % a.split_max;
  const int32_t row = a.cand[ci];
  if (row < p.row_lo || row >= p.row_hi) return;           // row-range numeric: another chunk's row
  const int64_t ob = a.C_rp[row], cnt = a.C_rp[row + 1] - ob;
  if (cnt <= a.limit || !bitmap_row(a, row)) return;
  const long long bmo = a.bm_pool ? a.bm_off[ci] : -1ll;
  // giant rows whose bitmap was kept (the structure needs no cross-CTA merge): the row's A
  // entries are split over `pieces` CTAs, each adding its products' values (C4: 64 rows of 4M
  // products were the numeric step's critical path on 64 SMs)
  int pieces = 1;
  if (bmo >= 0 && a.split_max > 1) {
    const int64_t want = p.prods[row] / kSplitProducts;
    pieces = want < 1 ? 1 : (want > a.split_max ? a.split_max : (int)want);
  }
  if (piece >= pieces) return;
  const int tid = threadIdx.x, lane = lane_id(), wp = warp_id();
  if (tid == 0) count_path(p.paths, pieces == 1 ? SPECK_PATH_LONG_BITMAP : SPECK_PATH_LONG_BITMAP_SPLIT);
  const uint32_t lo = (uint32_t)a.colmin[row] & ~31u;
  const int W = (int)(((int64_t)a.colmax[row] + 1 - lo + 31) / 32);
  const int G = (W + 31) / 32;                                   // 32-word groups
  uint32_t* bits = reinterpret_cast<uint32_t*>(smem);
  int32_t* gpre = reinterpret_cast<int32_t*>(smem + (size_t)G * 128);       // after 32*G words
  uint16_t* wpre = reinterpret_cast<uint16_t*>(smem + (size_t)G * 128 + (size_t)G * 4);
  const int64_t ar0 = p.A_rp[row];
  const int arlen = (int)(p.A_rp[row + 1] - ar0);
  const int64_t a0 = ar0 + (int64_t)arlen * piece / pieces;             // this CTA's slice of A_i
  const int alen = (int)(ar0 + (int64_t)arlen * (piece + 1) / pieces - a0);
  if (bmo >= 0) {
    // the symbolic step kept this row's bitmap: load it instead of rebuilding it (pass 1)
    const uint32_t* src = a.bm_pool + bmo;
    for (int i = tid; i < G * 32; i += T) bits[i] = i < W ? __ldcs(src + i) : 0u;
  } else {
    for (int i = tid; i < G * 32; i += T) bits[i] = 0u;
  }
  // Rows whose referenced B rows are long on average (C3: ~800) rotate every chunk over all
  // warps, each warp reading every batch (ALL mode; the redundant batch loads are cheap next to
  // the products).  Rows of A with many short references (C4: 200k NZ, ~20 products each) would
  // pay 32x their A traffic that way: there hub rows of B (>= kLongB entries) go to a shared
  // list streamed by all warps and the other batches go round-robin over the warps.
  bool listed = false;
  if (p.prods[row] < (int64_t)kAllAvgLen * arlen) listed = collect_long_rows<1, V>(p, a0, alen, longs);
  else __syncthreads();
  // 1. structure
  auto set_bit = [&](uint32_t col, V, bool act) {
    if (act) {
      const uint32_t c = col - lo;
      atomicOr(&bits[c >> 5], 1u << (c & 31));
    }
  };
  if (bmo >= 0) {
  } else if (listed) {
    expand_long_list<0, V>(p, longs, wp, NW, set_bit);
    expand_row<0, V, true, false>(p, a0, alen, wp, NW, set_bit, FullRange(), nullptr, kLongB);
  } else {
    expand_row<0, V, true, true>(p, a0, alen, wp, NW, set_bit);
  }
  __syncthreads();
  // 2. prefixes: warp w owns groups [w*GW, (w+1)*GW); lane i holds word i of a group
  const int GW = (G + NW - 1) / NW;
  const int g0 = min(G, wp * GW), g1 = min(G, g0 + GW);
  int wc = 0;
  for (int g = g0; g < g1; ++g) wc += __popc(bits[g * 32 + lane]);
  wc = warp_sum(wc);
  if (lane == 0) part[wp] = wc;
  __syncthreads();
  int run = 0;
  for (int w = 0; w < wp; ++w) run += (int)part[w];
  for (int g = g0; g < g1; ++g) {
    const uint32_t word = bits[g * 32 + lane];
    const int pc = __popc(word);
    const int incl = warp_incl_scan(pc);
    const int excl = incl - pc;
    wpre[g * 32 + lane] = (uint16_t)excl;
    if (lane == 0) gpre[g] = run;
    // C.col of the group: sparse groups per lane (a lane's entries are consecutive and the
    // group's entries span few sectors), dense groups one word at a time across the warp
    const int mx = __reduce_max_sync(0xffffffffu, (unsigned)pc);
    const uint32_t cbase = lo + (uint32_t)g * 1024u;
    if (piece > 0) {
      // another piece of a split row writes C.col
    } else if (mx <= 8) {
      uint32_t wv = word;
      int o = run + excl;
      while (wv) {
        const int b = __ffs(wv) - 1;
        wv &= wv - 1;
        p.C_col[ob + o++] = (int32_t)(cbase + (uint32_t)lane * 32u + (uint32_t)b);
      }
    } else {
      for (int j = 0; j < 32; ++j) {
        const uint32_t wj = __shfl_sync(0xffffffffu, word, j);
        if (!wj) continue;
        const int oj = __shfl_sync(0xffffffffu, excl, j);
        if ((wj >> lane) & 1u)
          p.C_col[ob + run + oj + __popc(wj & ((1u << lane) - 1u))] = (int32_t)(cbase + (uint32_t)j * 32u + (uint32_t)lane);
      }
    }
    run += __shfl_sync(0xffffffffu, incl, 31);
  }
  // zero the row's values (coalesced), then make the zeros visible to the block's atomics
  // (split rows: C.val was zeroed before the launch)
  if (pieces == 1)
    for (int64_t i = tid; i < cnt; i += T) p.C_val[ob + i] = V(0);
  __syncthreads();
  // 3. values
  V* cv = p.C_val + ob;
  auto add_val = [&](uint32_t col, V v, bool act) {
    if (act) {
      const uint32_t c = col - lo, w = c >> 5;
      const int r = gpre[w >> 5] + (int)wpre[w] + __popc(bits[w] & ((1u << (c & 31)) - 1u));
      atomicAdd(cv + r, v);
    }
  };
  if (listed) {
    expand_long_list<1, V>(p, longs, wp, NW, add_val);
    expand_row<1, V, true, false>(p, a0, alen, wp, NW, add_val, FullRange(), nullptr, kLongB);
  } else {
    expand_row<1, V, true, true>(p, a0, alen, wp, NW, add_val);
  }
}

}  // namespace speck
