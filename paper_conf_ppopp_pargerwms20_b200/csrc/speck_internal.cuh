// speck_internal.cuh — shared device/host definitions of the B200 spECK kernels.
//
// Paper: Parger et al., "spECK", PPoPP'20 (P:a-b = PAPER.md lines).  The B200 design
// (configuration ladder, accumulator tiers, data layout) is documented in DESIGN.md.
#pragma once

#include <cstdint>
#include <cuda_runtime.h>

#include "../../include/speck.h"

namespace speck {

// ----------------------------------------------------------------------------------
// Kernel configuration ladder: each successive configuration halves the
// threads and the scratchpad.  B200: 228 KB smem per SM, up to 227 KB per CTA; kernels
// run at <= 64 registers/thread -> 1024 resident threads/SM, so the ladder keeps
// ~220 B of scratchpad per thread and every configuration fills one SM's smem:
//   cfg0   64 thr  x16 CTA/SM      cfg3  512 thr  x2 CTA/SM
//   cfg1  128 thr  x8  CTA/SM      cfg4 1024 thr  x1 CTA/SM (largest map; long rows)
//   cfg2  256 thr  x4  CTA/SM
// ----------------------------------------------------------------------------------
constexpr int kNumCfg = 5;
constexpr int kCfgThreads[kNumCfg] = {64, 128, 256, 512, 1024};
// accumulator (hash map / dense window) bytes per configuration
constexpr int kCfgMapBytes[kNumCfg] = {11264, 25856, 54272, 111616, 225280};
__host__ __device__ constexpr int cfg_map_bytes(int c) {
  return c == 0 ? 11264 : c == 1 ? 25856 : c == 2 ? 54272 : c == 3 ? 111616 : 225280;
}
// B200: 228 KB shared memory per SM (233472 B), 1 KB reserved per resident CTA, <= 227 KB per CTA
constexpr int kSmemPerSM = 233472;
constexpr int kSmemPerCtaMax = 232448;
static_assert(cfg_map_bytes(4) == kCfgMapBytes[4] && cfg_map_bytes(0) == kCfgMapBytes[0], "ladder");
constexpr int kMaxGroupRows = 32;     // rows per block (5-bit local row id)
constexpr int kBinTile = 1024;        // rows per binning tile
constexpr int kMaxStreams = 8;
constexpr int64_t kAnaLong = 4096;    // rows of A longer than this get a whole CTA in the analysis

// categories (bins) of a row for one pass
enum Cat : int {
  CAT_EMPTY = 0,  // no products: row of C is empty
  CAT_DIRECT = 1, // single NZ in the row of A
  CAT_CFG0 = 2,   // CAT_CFG0 + j = configuration j (cfg0 bin = merged small rows)
  CAT_LONG = CAT_CFG0 + kNumCfg,  // numeric rows beyond the largest map: split into column segments
  CAT_TINY = CAT_LONG + 1,        // numeric rows of the smallest bin with <= kTinyCnt entries (rank-counted)
  CAT_COUNT = CAT_TINY + 1
};
// numeric rows with at most this many entries keep a scrambled hash and rank counting
// (P:1130-1133); larger ones use the order-preserving map.  They get separate warp-row
// kernels so each stays compact in the instruction cache.
constexpr int kTinyCnt = 64;

// Long rows (numeric nnz beyond the largest hash map) are split into column segments whose
// exact sizes come from per-chunk counts recorded by the symbolic pass: chunks of 2^s
// columns (2^s <= one dense window of the largest configuration: s = 15 fp32, 14 fp64), at
// most kMaxChunks per row.
constexpr int kMaxChunks = 1024;
// Long-row jobs run in configuration 3 (512 threads, 2 CTAs per SM), so one CTA's barriers
// overlap with the other's work; segments hold up to that map's fill.
constexpr int kSegCfg = kNumCfg - 2;
// rows of A longer than this make column segments expensive (see seg_plan_args)
constexpr int64_t kSegMaxNnzA = 16384;
struct Seg {
  int32_t row;
  int32_t col_lo;   // first column of the segment
  int32_t col_hi;   // one past the last column
  int32_t cnt;      // exact entries of C in [col_lo, col_hi)
  int64_t out;      // position of the segment's first entry in C
  int32_t dense;    // 1: dense window accumulator, 0: ordered hash map
  int32_t pad;
};

constexpr uint32_t kEmptyKey = 0xFFFFFFFFu;

// Fill rule for the numeric hash maps: final occupancy <= 66%.
#ifndef SPECK_SYM_FILL
#define SPECK_SYM_FILL 66
#endif
constexpr int kFillNum = SPECK_SYM_FILL;
#ifndef SPECK_SYM_WARP_U
#define SPECK_SYM_WARP_U 4   // product chunks in flight per symbolic warp row
#endif
#ifndef SPECK_SYM_REGION_X2
#define SPECK_SYM_REGION_X2 8     // symbolic single-row regions: need * this / 2 slots (4x products: C5 symbolic 99 -> 91 ms)
#endif
// Numeric maps: the order-preserving hash (spgemm_kernels.cuh) walks its probing runs in the
// write-out, and runs grow like 1/(1-load)^2; homes cover 7/8 of a map, so a 50% fill keeps
// the effective load near 57% (runs ~5) instead of 75% (runs ~16) at the paper's 66%.
constexpr int kFillOrdered = 50;
// Dense-accumulator rule (reading R13): dense if <= 3 windows and density > 18%.
constexpr int kDenseMaxWindows = 3;
constexpr int kDensePct = 18;

template <typename V>
__host__ __device__ constexpr int num_slot_bytes() { return 4 + (int)sizeof(V); }

// capacity (slots) of a configuration's hash map
__host__ __device__ inline uint32_t sym_map_cap(int cfg) { return (uint32_t)(cfg_map_bytes(cfg) / 4); }
// Symbolic rows are binned by products, an upper bound of their distinct columns.
// The paper relies on the average compaction of ~7 to keep the map sparse; for
// inputs without compaction (R-MAT C5: ~1.05) the bound is tight, so B200 bins against 66% of
// the slots as in the numeric step — linear probing stays short either way.
__host__ __device__ inline uint32_t sym_map_fill(int cfg) { return (uint32_t)((uint64_t)sym_map_cap(cfg) * kFillNum / 100); }
template <typename V>
__host__ __device__ inline uint32_t num_map_cap(int cfg) { return (uint32_t)((cfg_map_bytes(cfg) - 16) / num_slot_bytes<V>()); }
// byte offset of the value array of a numeric hash map (keys first, 16-B aligned values)
template <typename V>
__host__ __device__ inline uint32_t num_val_offset(int cfg) { return (num_map_cap<V>(cfg) * 4u + 15u) & ~15u; }
// max entries (66% fill) a numeric map of configuration cfg accepts
template <typename V>
__host__ __device__ inline uint32_t num_map_fill(int cfg) { return (uint32_t)((uint64_t)num_map_cap<V>(cfg) * kFillOrdered / 100); }
// dense windows (columns) of a configuration: symbolic = bitmap, numeric = values + flag bits
__host__ __device__ inline int64_t sym_dense_window(int cfg) { return (int64_t)cfg_map_bytes(cfg) * 8; }
template <typename V>
__host__ __device__ inline int64_t num_dense_window(int cfg) {
  return ((int64_t)(cfg_map_bytes(cfg) - 16) * 8 / (8 * (int64_t)sizeof(V) + 1)) & ~int64_t(31);
}

// Small rows: one warp per row in a private region (k_warp_rows).  8 warps x 7 KB per CTA and
// 4 CTAs per SM = 1024 resident threads and the whole 228 KB; a row belongs here when its need
// fits the region at the pass's fill.
constexpr int kWarpRowThreads = 256;
constexpr int kWarpRegionBytes = 7168;
constexpr int kWarpRowCtasPerSM = 4;
// symbolic (keys only, <= 40 registers): 6 CTAs x 8 warps x 4.5 KB per SM — 48 warps hide more
// of the gather latency (C2 symbolic A*P 1.85 -> 1.62 ms measured with this geometry)
constexpr int kWarpRegionBytesSym = 4608;
constexpr int kWarpRowCtasPerSMSym = 6;
static_assert((kWarpRegionBytesSym * (kWarpRowThreads / 32) + 1024) * kWarpRowCtasPerSMSym <= kSmemPerSM, "warp-row CTAs");
// numeric tiny rows (<= kTinyCnt entries, MODE 1): 2 KB regions hold 2.5x 64 entries, so the
// smem no longer caps the CTAs; 5 CTAs (40 warps, 48 registers) measured best (C2 numeric A*P
// 2.64 -> 2.56 ms; 6 CTAs at 40 registers spill and lose: 2.61 ms; ty_* runs, round 1), and
// 2 products per lane per chunk instead of 4 at the same geometry: 2.56 -> 2.35 ms
constexpr int kWarpRegionBytesTiny = 2048;
constexpr int kWarpRowCtasPerSMTiny = 5;
static_assert((kWarpRegionBytesTiny * (kWarpRowThreads / 32) + 1024) * kWarpRowCtasPerSMTiny <= kSmemPerSM, "warp-row CTAs");
__host__ __device__ constexpr int wr_region_bytes(int pass, int mode = 0) {
  return pass == 0 ? kWarpRegionBytesSym : mode == 1 ? kWarpRegionBytesTiny : kWarpRegionBytes;
}
__host__ __device__ constexpr int wr_ctas_per_sm(int pass, int mode = 0) {
  return pass == 0 ? kWarpRowCtasPerSMSym : mode == 1 ? kWarpRowCtasPerSMTiny : kWarpRowCtasPerSM;
}
constexpr int kWarpRowChunk = 8;     // rows a warp claims per counter increment
static_assert((kWarpRegionBytes * (kWarpRowThreads / 32) + 1024) * kWarpRowCtasPerSM <= kSmemPerSM, "warp-row CTAs");
__host__ __device__ inline uint32_t wr_sym_cap() { return (uint32_t)(kWarpRegionBytesSym / 4); }
__host__ __device__ inline uint32_t wr_sym_fill() { return (uint32_t)((uint64_t)wr_sym_cap() * kFillNum / 100); }
template <typename V>
__host__ __device__ constexpr uint32_t wr_num_cap(int bytes = kWarpRegionBytes) { return (uint32_t)((bytes - 16) / num_slot_bytes<V>()); }
template <typename V>
__host__ __device__ constexpr uint32_t wr_num_val_offset(int bytes = kWarpRegionBytes) { return (wr_num_cap<V>(bytes) * 4u + 15u) & ~15u; }
static_assert(wr_num_cap<double>(kWarpRegionBytesTiny) >= (uint32_t)(kTinyCnt * 5 / 2), "tiny region holds 2.5x kTinyCnt");
template <typename V>
__host__ __device__ inline uint32_t wr_num_fill() { return (uint32_t)((uint64_t)wr_num_cap<V>() * kFillOrdered / 100); }

// ----------------------------------------------------------------------------------
// Analysis statistics block written by the analysis kernel (read back once, sync #1).
// ----------------------------------------------------------------------------------
struct AnalysisStats {
  unsigned long long sum_prods;
  unsigned long long max_prods;
  unsigned long long n_direct;
  unsigned long long n_empty;
  unsigned long long max_nnza;     // max nnz of a row of A
  unsigned long long max_nnza_long;// max nnz of a row of A in the largest symbolic bin
  unsigned long long pad[2];
};

// ----------------------------------------------------------------------------------
// Per-pass plan parameters shared by classification and binning kernels.
// ----------------------------------------------------------------------------------
struct BinParams {
  int pass;                 // 0 symbolic, 1 numeric
  int use_direct;           // route single-NZ rows to the direct path
  int64_t cap[kNumCfg];     // need thresholds: row goes to the smallest cfg with need <= cap[cfg]
  int64_t long_thr;         // numeric: rows with cnt > long_thr are split into segments
  int64_t tiny_cap;         // numeric: smallest-bin rows with cnt <= tiny_cap go to CAT_TINY (-1: off)
};

__host__ __device__ inline int classify_row(int64_t nnza, int64_t prods, int64_t cnt, const BinParams& bp) {
  if (prods == 0) return CAT_EMPTY;
  if (bp.use_direct && nnza == 1) return CAT_DIRECT;
  if (bp.pass == 1 && cnt > bp.long_thr) return CAT_LONG;
  int64_t need = bp.pass == 0 ? prods : cnt;
  if (bp.pass == 1 && need <= bp.tiny_cap && need <= bp.cap[0]) return CAT_TINY;
#pragma unroll
  for (int c = 0; c < kNumCfg - 1; ++c)
    if (need <= bp.cap[c]) return CAT_CFG0 + c;
  return CAT_CFG0 + kNumCfg - 1;
}

// ----------------------------------------------------------------------------------
// Device helpers
// ----------------------------------------------------------------------------------
__device__ __forceinline__ uint32_t hash_slot(uint32_t key, uint32_t cap) {
  // multiplicative hash ("multiplies the element index with a prime") mapped to
  // [0, cap) by a 32x32->64 multiply-high instead of a modulo (reading R12)
  uint32_t h = key * 2654435761u;
  return (uint32_t)(((uint64_t)h * cap) >> 32);
}

__device__ __forceinline__ int lane_id() { return threadIdx.x & 31; }
__device__ __forceinline__ int warp_id() { return threadIdx.x >> 5; }

template <typename T>
__device__ __forceinline__ T warp_incl_scan(T v) {
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    T n = __shfl_up_sync(0xffffffffu, v, o);
    if (lane_id() >= o) v += n;
  }
  return v;
}

template <typename T>
__device__ __forceinline__ T warp_sum(T v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

// Block-wide exclusive scan for NT threads; `part` = smem scratch of NT/32 + 1 elements.
// Returns the exclusive prefix of v; *total gets the block total.  Contains barriers.
template <int NT, typename T>
__device__ __forceinline__ T block_excl_scan(T v, T* part, T* total) {
  constexpr int NW = NT / 32;
  T inc = warp_incl_scan(v);
  if (lane_id() == 31) part[warp_id()] = inc;
  __syncthreads();
  if (warp_id() == 0) {
    T p = lane_id() < NW ? part[lane_id()] : T(0);
    T pi = warp_incl_scan(p);
    if (lane_id() < NW) part[lane_id()] = pi - p;
    if (lane_id() == NW - 1) part[NW] = pi;
  }
  __syncthreads();
  T res = inc - v + part[warp_id()];
  *total = part[NW];
  __syncthreads();
  return res;
}

// Round to the closest power of two in linear distance, ties upward.
__host__ __device__ inline int64_t closest_pow2(double x) {
  if (x <= 1.0) return 1;
  int64_t p = 1;
  while ((double)(p * 2) <= x) p *= 2;      // p <= x < 2p
  return (x - (double)p >= (double)(2 * p) - x) ? 2 * p : p;
}

// Local load balancer, reading R9 of DESIGN.md.
__host__ __device__ inline int32_t local_group_size(int32_t T, int64_t nnzA, int64_t prods, int64_t maxlen) {
  if (nnzA <= 0 || prods <= 0) return T;
  double g = (double)closest_pow2((double)prods / (double)nnzA);   // average referenced row length
  if (g > (double)T) g = (double)T;
  double k = (double)T / g;
  double iter_max = ceil((double)maxlen / g);
  double n_rows = (double)nnzA / k;
  if (iter_max > 2.0 * n_rows) g = g * sqrt(iter_max / (2.0 * n_rows));
  else if (n_rows > 2.0 * iter_max) g = g * sqrt(iter_max / n_rows);
  int64_t gi = closest_pow2(g);
  if (gi > T) gi = T;
  if (gi < 1) gi = 1;
  if ((int64_t)T / gi > nnzA) {        // more groups than B rows: k <- largest pow2 <= nnzA
    int64_t p = 1;
    while (p * 2 <= nnzA) p *= 2;
    gi = T / p;
    if (gi < 1) gi = 1;
  }
  return (int32_t)gi;
}

// Block merge (Alg. 2; Fig. 3), reading R10, over one aligned group of <= 32
// entries held one per lane by a full warp.  `need` of lanes >= n is ignored.  Returns
// a warp-uniform bit mask with bit i set where a block starts.
__device__ __forceinline__ uint32_t warp_block_merge(int64_t need, int n, int64_t cap) {
  const int lane = lane_id();
  uint32_t valid = n >= 32 ? 0xffffffffu : ((1u << n) - 1u);
  uint32_t starts = valid;
  int64_t sum = lane < n ? need : 0;     // valid at block-start lanes
#pragma unroll
  for (int s = 0; s < 5; ++s) {
    const int half = 1 << s;
    const int gbase = lane & ~((2 << s) - 1);
    const int mid = gbase + half;
    // the left half's last block start (every lane of the group computes it)
    uint32_t lowmask = (mid >= 32 ? 0xffffffffu : ((1u << mid) - 1u)) & ~((1u << gbase) - 1u);
    uint32_t lm = starts & lowmask;
    int left = lm ? 31 - __clz(lm) : gbase;
    int64_t sum_left = __shfl_sync(0xffffffffu, sum, left);
    int64_t sum_mid = __shfl_sync(0xffffffffu, sum, mid & 31);
    bool can = (mid < n) && (sum_left + sum_mid < cap);
    uint32_t merged_mid = __ballot_sync(0xffffffffu, can && lane == mid);
    if (can && lane == left) sum = sum_left + sum_mid;
    starts &= ~merged_mid;
  }
  return starts;
}

// SPECK_OPT_PATH_COUNTERS: one thread per row (segment, CTA) counts the path it took.
__device__ __forceinline__ void count_path(unsigned long long* paths, int path) {
  if (paths) atomicAdd(paths + path, 1ull);
}

// ----------------------------------------------------------------------------------
// Problem description handed to the SpGEMM kernels (device pointers).
// ----------------------------------------------------------------------------------
template <typename V>
struct SpgemmArgs {
  const int64_t* A_rp;
  const int32_t* A_col;
  const V* A_val;
  const int64_t* B_rp;
  const int32_t* B_col;
  const V* B_val;
  int64_t m;                 // rows of A
  int64_t n;                 // cols of B
  // analysis record (SoA, Alg. 1)
  const int64_t* prods;
  const int32_t* maxlen;
  const int32_t* colmin;
  const int32_t* colmax;
  // row list of this launch (nullptr -> identity: entry e is row e)
  const int32_t* rows;
  int64_t n_entries;
  int group_rows;            // entries per CTA group
  int merge;                 // 1: block-merge the group (Alg. 2) with merge_cap
  int64_t merge_cap;
  int col_bits;              // column bits of the compound key (row << col_bits | col)
  int force_acc;             // 0 auto, 1 hash, 2 dense
  int64_t dense_window_cap;  // >0: cap dense window (test knob)
  int fixed_g;               // >0: fixed group size
  int esc;                   // bucket counting-sort rows (esc_kernels.cuh): 0 off, 1 numeric, 2 + symbolic
  unsigned long long* paths; // SPECK_OPT_PATH_COUNTERS: rows per speck_path_t (nullptr: off)
  int64_t row_lo, row_hi;    // row-range numeric (speck_spgemm_rows): long-row jobs outside [row_lo, row_hi) exit
  // symbolic out
  int64_t* cnt;
  // numeric in/out
  const int64_t* C_rp;
  int32_t* C_col;
  V* C_val;
  // resume-position scratch for multi-window dense rows: [num_sms][resume_stride]
  int32_t* resume;
  int64_t resume_stride;
  int64_t resume_slots;      // slots in `resume` (%nsmid of the device)
  // counters
  unsigned long long* n_dense_rows;
  // symbolic, largest configuration: per-chunk counts of long-row candidates
  int32_t* chunk_cnt;        // [bin entries][nchunks] or nullptr
  int nchunks;
  int chunk_shift;           // chunk = col >> chunk_shift
  int64_t long_thr;          // rows with prods > long_thr record chunk counts
  // symbolic, largest configuration: the dense bitmap of a row that will be a numeric long row
  // is kept in a pool for k_long_bitmap (bm_off[entry] = word offset, -1 if not kept)
  uint32_t* bm_pool;
  unsigned long long bm_pool_words;
  unsigned long long* bm_ctr;
  int64_t* bm_off;
};

}  // namespace speck
