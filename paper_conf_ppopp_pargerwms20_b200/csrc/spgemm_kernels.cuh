// spgemm_kernels.cuh — symbolic and numeric SpGEMM kernels (§4.3).
//
// One kernel template per configuration of the ladder (speck_internal.cuh) and pass.  A CTA
// takes a group of <= 32 consecutive entries of its bin (or of the identity row list when
// the global load balancer is off), splits the group into blocks with the
// block merge of Alg. 2 (merged small-row bin only), and for each block:
//   1. picks the accumulator: hash map, dense array; direct
//      rows have their own kernel below;
//   2. enumerates the products with the expand-balanced local load balancer (expand_row:
//      the B200 form of P:867-970 — every lane gets the same number of products);
//   3. symbolic: counts the distinct columns per row;
//      numeric: accumulates values and writes each row SORTED at its C row offset
//      (P:1121-1148).
//
// B200 differences from the paper's Titan V design:
//   * merged rows use per-row regions of the map instead of a 5-bit row + 27-bit column
//     compound key, so blocks of up to 32 rows work for any column count;
//   * multi-row blocks run one warp per row (no block barriers, warp-aggregated updates);
//   * rows > 64 entries use an order-preserving hash: runs are insertion-sorted in place and
//     the write-out is a compaction; short rows use rank counting; no global sort pass;
//   * dense windows of rows needing several windows keep resume positions per referenced
//     B row in a per-SM global scratch slot.
#pragma once

#include "speck_internal.cuh"
#include "esc_kernels.cuh"

namespace speck {

#ifndef SPECK_WARP_U
#define SPECK_WARP_U 1      // product chunks in flight per numeric warp-row expansion step (C2: 1 beats 2)
#endif
constexpr int kSmallSeg = kTinyCnt;   // rows with <= this many C entries are ranked, not sorted
constexpr int kPPL = 4;         // products per lane per chunk in the warp-per-row path
constexpr int kAllAvgLen = 256;  // expand_row ALL mode for rows whose references average >= this many products
constexpr int kStreamLen = 64;  // referenced B rows at least this long are streamed, not balanced

struct BlockMeta {
  int32_t row[kMaxGroupRows];
  int64_t astart[kMaxGroupRows];
  int64_t aoff[kMaxGroupRows + 1];   // prefix of nnz(A_r) over the block
  int64_t cbase[kMaxGroupRows];      // numeric: C_rp[row]
  int32_t cseg[kMaxGroupRows + 1];   // numeric: prefix of cnt_r over the block
  uint32_t rbase[kMaxGroupRows + 1]; // hash region start of each row
  int32_t rcnt[kMaxGroupRows];       // symbolic: distinct columns per row
  int32_t rlo[kMaxGroupRows];        // colmin / colmax per row (order-preserving hash)
  int32_t rhi[kMaxGroupRows];
  int32_t rwrap[kMaxGroupRows];      // block path: a probing run of the row wrapped around
  uint32_t starts;
  int nr, g, dense, ordered, esc;
  int64_t nnzA, prods, maxlen, cnt;
  int32_t colmin, colmax;
  int64_t scan_part[33];
  int64_t total;
};

// every configuration must keep 1024 threads resident per SM: (map + meta + 1 KB) x CTAs/SM
template <int C>
constexpr bool cfg_fits() {
  return (kCfgMapBytes[C] + (int)sizeof(BlockMeta) + 1024) * (1024 / kCfgThreads[C]) <= kSmemPerSM &&
         kCfgMapBytes[C] + (int)sizeof(BlockMeta) <= kSmemPerCtaMax;
}
static_assert(cfg_fits<0>() && cfg_fits<1>() && cfg_fits<2>() && cfg_fits<3>() && cfg_fits<4>(),
              "a ladder configuration no longer fits 1024 resident threads per SM");

template <typename V>
__device__ __forceinline__ V ldv(const V* p) { return __ldg(p); }
// a + b rounded once, never contracted with the product that produced b (in-order, per-product
// rounded sums: the warp-per-row paths give the sequential sum of reading R15 bit for bit)
__device__ __forceinline__ float add_rn(float a, float b) { return __fadd_rn(a, b); }
__device__ __forceinline__ double add_rn(double a, double b) { return __dadd_rn(a, b); }

// Order-preserving numeric maps: 8-slot buckets, the home bucket monotone in the column over
// the row's [colmin, colmax] and covering the first 7/8 of the buckets (the rest absorbs
// overflow).  A key takes the first empty slot of its home bucket, or of the next non-full
// bucket; occupied slots of a bucket are always a prefix of it.  Hence every key sits in the
// probing run (maximal occupied range) that contains its home, runs appear in column order, and
// an entry's position in the sorted row is (#occupied slots before its run) + (rank of its key
// in the run); a run that ends in a non-full bucket and starts after one is just that bucket
// (warp_write_ordered's fast path ranks it with 7 shuffles).
// home = floor((col - lo) * mult / 2^32) with mult = floor(nh * 2^32 / range), nh = 7/8 of the
// S/8 buckets: monotone in col, < nh, a multiply per product instead of a 64-bit division.
__device__ __forceinline__ uint64_t bkt_mult(uint32_t range, uint32_t S) {
  const uint64_t nb = S >> 3, nh = nb - (nb >> 3);
  return range ? (nh << 32) / range : 0;
}
__device__ __forceinline__ uint32_t bkt_home(uint32_t col, uint32_t lo, uint64_t mult) {
  // floor((col - lo) * mult / 2^32) as high(x * mult_lo) + x * mult_hi: nvcc 12.9 folded the
  // 64-bit product-and-shift form wrongly inside one loop of esc_row_staged (illegal shared
  // addresses on every run; the explicit form compiles to IMAD.HI + IMAD)
  const uint32_t x = col - lo;
  return __umulhi(x, (uint32_t)mult) + x * (uint32_t)(mult >> 32);
}

// Insert into the bucketed ordered map (keys 16-byte aligned, NB = S/8 buckets): two 16-byte
// shared loads examine a bucket; a wrap-around past the last bucket (breaks the run order) is
// reported.  Returns the key's slot.
__device__ __forceinline__ uint32_t probe_insert_bkt(uint32_t* keys, uint32_t NB, uint32_t b, uint32_t key, int* wrapped) {
  while (true) {
    uint32_t k[8];
    const uint32_t a = (uint32_t)__cvta_generic_to_shared(keys + 8 * b);
    asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(k[0]), "=r"(k[1]), "=r"(k[2]), "=r"(k[3]) : "r"(a));
    asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(k[4]), "=r"(k[5]), "=r"(k[6]), "=r"(k[7]) : "r"(a + 16));
    uint32_t hit = 0, emp = 0;
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      hit |= (uint32_t)(k[i] == key) << i;
      emp |= (uint32_t)(k[i] == kEmptyKey) << i;
    }
    if (hit) return 8 * b + __ffs(hit) - 1;
    if (emp) {
      const uint32_t s = 8 * b + __ffs(emp) - 1;
      const uint32_t old = atomicCAS(&keys[s], kEmptyKey, key);
      if (old == kEmptyKey || old == key) return s;
      continue;   // the slot was taken by another key: re-read the bucket
    }
    if (++b == NB) { b = 0; *wrapped = 1; }
  }
}

// Linear probing from slot s (Fig. 4): find `key` or claim the first empty slot
// with a CAS, moving to the next slot (mod S) while the slot holds another key; reports a
// wrap-around past the last slot (which breaks the cluster order of monotone homes).  The
// numeric maps of scrambled rows use it (home = hash_slot), and speck_hash_probe runs it with
// injected homes for the Fig. 4 example.
__device__ __forceinline__ uint32_t probe_insert_mono(uint32_t* keys, uint32_t S, uint32_t s, uint32_t key, int* wrapped) {
  while (true) {
    const uint32_t k = keys[s];
    if (k == key) return s;
    if (k == kEmptyKey) {
      const uint32_t old = atomicCAS(&keys[s], kEmptyKey, key);
      if (old == kEmptyKey || old == key) return s;
    }
    if (s + 1 == S) { s = 0; *wrapped = 1; } else ++s;
  }
}

// Sorted write-out of the slots [w0, w1) of an ordered map region rk/rv[0, S) by one warp,
// without moving anything in shared memory.  With monotone homes and no wrap-around, every
// occupied slot s lies in a probing run [rs, re) (maximal occupied range) that holds exactly
// the keys homed inside it, and runs appear in column order; so the sorted position of slot s
// is (#occupied before rs) + #{j in [rs, re) : key_j < key_s}, where
// #occupied before rs = #occupied before s - (s - rs).  Run bounds come from the window's
// occupancy ballot (a short walk only for runs crossing a window edge); the rank loop is as
// long as the window's longest run.  `before` = #occupied slots of the region before w0.
// Returns the number of entries written.
template <typename V>
__device__ __forceinline__ int warp_write_ordered(const uint32_t* rk, const V* rv, uint32_t S, uint32_t w0, uint32_t w1,
                                                  int64_t ob, int before, int32_t* __restrict__ C_col,
                                                  V* __restrict__ C_val) {
  const int lane = lane_id();
  const uint32_t lt = (1u << lane) - 1u;
  const uint32_t gt = ~(lt | (1u << lane));
  // occupied slots immediately before the window (a run entering it from the left)
  uint32_t carry = 0;
  if (w0 > 0 && w0 < w1 && rk[w0] != kEmptyKey)
    while (carry < w0 && rk[w0 - 1 - carry] != kEmptyKey) ++carry;
  int written = 0;
  for (uint32_t c0 = w0; c0 < w1; c0 += 32) {
    const uint32_t s = c0 + lane;
    const uint32_t k = s < S ? rk[s] : kEmptyKey;        // slots past w1 only bound runs
    const uint32_t occ = __ballot_sync(0xffffffffu, k != kEmptyKey);
    const uint32_t mine = occ & (w1 - c0 >= 32 ? 0xffffffffu : ((1u << (w1 - c0)) - 1u));
    // fast path (warp-uniform): no full bucket in the window and no run entering it, so every
    // run is its bucket: rank among the bucket's 8 keys by shuffles, no divergent walk
    const uint32_t fullb = __vcmpeq4(occ, 0xffffffffu);   // 0xff in every byte (bucket) that is full
    if (!fullb && carry == 0) {
      // rank among the bucket's 8 keys: two 16-byte loads shared by the bucket's 8 lanes
      uint32_t q[8];
      const uint32_t a = (uint32_t)__cvta_generic_to_shared(rk + c0 + (lane & ~7));
      asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(q[0]), "=r"(q[1]), "=r"(q[2]), "=r"(q[3]) : "r"(a));
      asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(q[4]), "=r"(q[5]), "=r"(q[6]), "=r"(q[7]) : "r"(a + 16));
      int rank = 0;
#pragma unroll
      for (int d = 0; d < 8; ++d) rank += q[d] < k;
      if ((mine >> lane) & 1u) {
        const int64_t o = ob + before + written + __popc(occ & ((1u << (lane & ~7)) - 1u)) + rank;
        C_col[o] = (int32_t)k;
        C_val[o] = rv[s];
      }
      written += __popc(mine);
      carry = __clz(~occ);
      continue;
    }
    if ((mine >> lane) & 1u) {
      const uint32_t zb = ~occ & lt;
      const uint32_t rs = zb ? c0 + 32 - __clz(zb) : c0 - carry;
      const uint32_t za = ~occ & gt;
      uint32_t re;
      if (za) {
        re = c0 + __ffs(za) - 1;
      } else {
        re = c0 + 32;
        while (re < S && rk[re] != kEmptyKey) ++re;
      }
      int rank = 0;
      uint32_t j = rs;
      for (; j + 4 <= re; j += 4) rank += (rk[j] < k) + (rk[j + 1] < k) + (rk[j + 2] < k) + (rk[j + 3] < k);
      for (; j < re; ++j) rank += rk[j] < k;
      const int64_t o = ob + before + written + __popc(occ & lt) - (int)(s - rs) + rank;
      C_col[o] = (int32_t)k;
      C_val[o] = rv[s];
    }
    written += __popc(mine);
    carry = occ == 0xffffffffu ? carry + 32 : __clz(~occ);
  }
  return written;
}

// Linear probing over 4-slot groups for the unordered maps (symbolic keys, numeric rows of
// <= kSmallSeg entries): one 16-byte shared load examines a whole group, a key takes the
// first empty slot of the first group with room, groups are visited in order from the home
// group (so the probe sequence of a key is fixed and, slots only ever going EMPTY -> key,
// a key is never inserted twice).  At C5's ~67% symbolic load the scalar probe loop was half
// of the symbolic kernel's instructions; groups cut the iterations ~4x.  keys must be 16-byte
// aligned; only the first S & ~3 slots are used.
__device__ __forceinline__ uint32_t probe_insert_grp(uint32_t* keys, uint32_t S, uint32_t key, bool* is_new) {
  const uint32_t S4 = S & ~3u;
  uint32_t g = hash_slot(key, S4) & ~3u;
  while (true) {
    uint4 q;
    asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(q.x), "=r"(q.y), "=r"(q.z), "=r"(q.w)
                 : "r"((uint32_t)__cvta_generic_to_shared(keys + g)));
    if (q.x == key) { *is_new = false; return g; }
    if (q.y == key) { *is_new = false; return g + 1; }
    if (q.z == key) { *is_new = false; return g + 2; }
    if (q.w == key) { *is_new = false; return g + 3; }
    const int e = q.x == kEmptyKey ? 0 : q.y == kEmptyKey ? 1 : q.z == kEmptyKey ? 2 : q.w == kEmptyKey ? 3 : -1;
    if (e >= 0) {
      const uint32_t old = atomicCAS(&keys[g + e], kEmptyKey, key);
      if (old == kEmptyKey) { *is_new = true; return g + e; }
      if (old == key) { *is_new = false; return g + e; }
      continue;   // another key took the slot: re-read the group
    }
    g += 4;
    if (g >= S4) g = 0;
  }
}

// symbolic insert: true if the key was new.  Same probe sequence as probe_insert_grp, with the
// group's matches and empty slots as 4-bit masks (two branches per group instead of eight;
// C5 symbolic 91 -> 84 ms, profiles/r02/r02ag_*).
__device__ __forceinline__ bool hash_insert_key(uint32_t* keys, uint32_t S, uint32_t col) {
  const uint32_t S4 = S & ~3u;
  uint32_t g = hash_slot(col, S4) & ~3u;
  const uint32_t sb = (uint32_t)__cvta_generic_to_shared(keys);
  while (true) {
    uint32_t x, y, z, w;
    asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(x), "=r"(y), "=r"(z), "=r"(w) : "r"(sb + 4u * g));
    if ((x == col) | (y == col) | (z == col) | (w == col)) return false;
    const uint32_t em = (x == kEmptyKey ? 1u : 0u) | (y == kEmptyKey ? 2u : 0u) | (z == kEmptyKey ? 4u : 0u) |
                        (w == kEmptyKey ? 8u : 0u);
    if (em) {
      const uint32_t old = atomicCAS(&keys[g + __ffs(em) - 1], kEmptyKey, col);
      if (old == kEmptyKey) return true;
      if (old == col) return false;
      continue;   // another key took the slot: re-read the group
    }
    g += 4;
    if (g >= S4) g = 0;
  }
}

// Bitonic sort of (keys, vals)[0, n) ascending in shared memory, any n: the "flip"
// formulation keeps all sub-sorts ascending, so comparisons with a partner index >= n
// (a virtual +inf) are no-ops and can be skipped.
// WARP = true: one warp sorts (lanes 0..31, __syncwarp between stages).
template <int T, typename V, bool WARP = false>
__device__ __noinline__ void smem_bitonic_sort(uint32_t* keys, V* vals, int n) {
  if (n <= 1) return;
  const int t0 = WARP ? (int)(threadIdx.x & 31) : (int)threadIdx.x;
  int P = 1;
  while (P < n) P <<= 1;
  for (int k = 2; k <= P; k <<= 1) {
    const int lhk = __ffs(k) - 2;   // log2(k/2)
    for (int t = t0; t < P / 2; t += T) {
      const int blk = t >> lhk, off = t & ((1 << lhk) - 1);
      const int i = blk * k + off, j = blk * k + k - 1 - off;
      if (j < n) {
        const uint32_t a = keys[i], b = keys[j];
        if (a > b) {
          keys[i] = b; keys[j] = a;
          const V va = vals[i]; vals[i] = vals[j]; vals[j] = va;
        }
      }
    }
    if (WARP) __syncwarp(); else __syncthreads();
    for (int d = k >> 2; d >= 1; d >>= 1) {
      const int ld = __ffs(d) - 1;
      for (int t = t0; t < P / 2; t += T) {
        const int blk = t >> ld, off = t & (d - 1);
        const int i = (blk << (ld + 1)) + off, j = i + d;
        if (j < n) {
          const uint32_t a = keys[i], b = keys[j];
          if (a > b) {
            keys[i] = b; keys[j] = a;
            const V va = vals[i]; vals[i] = vals[j]; vals[j] = va;
          }
        }
      }
      if (WARP) __syncwarp(); else __syncthreads();
    }
  }
}

// Block-wide write-out of one ordered map region [0, S): warp-contiguous slot ranges, one
// block-level prefix of the per-warp occupancy, then warp_write_ordered per range (runs may
// cross range edges; slots are only read).  Barriers inside; `part` = >= 32 int64 scratch.
template <int T, typename V>
__device__ void block_write_ordered(const uint32_t* rk, const V* rv, uint32_t S, int64_t ob, int32_t* __restrict__ C_col,
                                    V* __restrict__ C_val, int64_t* part) {
  constexpr int NW = T / 32;
  const int lane = lane_id(), wp = warp_id();
  const uint32_t SW = ((S + NW - 1) / NW + 31u) & ~31u;
  const uint32_t w0 = min(S, wp * SW), w1 = min(S, w0 + SW);
  // occupancy of the warp's range: 4 slots per lane per 16-byte load
  int cw = 0;
  for (uint32_t c = w0 + 4 * lane; c < w1; c += 128) {
    if (c + 4 <= w1) {
      uint32_t q0, q1, q2, q3;
      asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(q0), "=r"(q1), "=r"(q2), "=r"(q3)
                   : "r"((uint32_t)__cvta_generic_to_shared(rk + c)));
      cw += (q0 != kEmptyKey) + (q1 != kEmptyKey) + (q2 != kEmptyKey) + (q3 != kEmptyKey);
    } else {
      for (uint32_t t = c; t < w1; ++t) cw += rk[t] != kEmptyKey;
    }
  }
  cw = warp_sum(cw);
  if (lane == 0) part[wp] = cw;
  __syncthreads();
  int before = 0;
  for (int w = 0; w < wp; ++w) before += (int)part[w];
  warp_write_ordered<V>(rk, rv, S, w0, w1, ob, before, C_col, C_val);
  __syncthreads();
}

// Sum of v over the lanes of the warp holding the same key (all 32 lanes call it; keys of
// inactive lanes must be unique).  `leader` = lowest lane of its key group, which receives
// the sum — so one update per distinct key per warp step instead of one atomic per product.
template <typename V>
__device__ __forceinline__ V warp_key_sum(uint32_t key, V v, bool& leader) {
  const int lane = lane_id();
  const uint32_t peers = __match_any_sync(0xffffffffu, key);
  leader = lane == __ffs(peers) - 1;
  const int maxg = (int)__reduce_max_sync(0xffffffffu, (unsigned)__popc(peers));
  V sum = v;
  if (maxg > 1) {
    uint32_t others = leader ? (peers & ~(1u << lane)) : 0u;
    for (int t = 1; t < maxg; ++t) {
      int src = lane;
      if (others) { src = __ffs(others) - 1; others &= others - 1; }
      const V x = __shfl_sync(0xffffffffu, v, src);
      if (src != lane) sum += x;
    }
  }
  return sum;
}

// Expand-balanced local load balancing (B200 form of the paper's local load balancer,
// P:867-970, which calls exact per-entry balancing ideal but too costly).
// Products of a row of A are enumerated in batches of 32 referenced B rows (one per lane:
// A col -> B row start/length), a warp scan of the lengths, then every lane takes products
// lane, lane+32, ... located by a 5-step shuffle binary search, kPPL per lane per chunk with
// independent loads (memory-level parallelism).  `nw` warps (index wi) share a row: a single
// batch splits its product chunks across the warps, several batches go round-robin.
// ins(col, val, active) is called by all 32 lanes (inactive lanes get a unique non-column key).
// Variant with a per-referenced-row sub-range: rng(f, j0, j1, s, e) narrows B row [j0, j1)
// of the f-th NZ of the row of A to [s, e) (column windows / segments); called once per f.
struct FullRange {
  __device__ __forceinline__ void operator()(int, int64_t j0, int64_t j1, int64_t& s, int64_t& e) const { s = j0; e = j1; }
};

// (PreBatch, the first batch of a row loaded ahead by k_warp_rows, is defined in esc_kernels.cuh)

//
// ALL = true (single-row blocks): every warp reads every batch (its 32 A entries and B row
// bounds, L1-resident after the first warp) and the batch's product chunks go round-robin over
// all nw warps, continuing the rotation across batches and streamed rows, so every warp ends
// within one chunk of the others — no warp waits at the block barrier for a batch holding a
// hub row of B (ncu, C5: 22-50% of the stall samples of the single-row kernels were that
// barrier with batches assigned round-robin).  Rng must then be pure (evaluated by every warp)
// or write the same value from every warp.
template <int PASS, typename V, bool STREAM = (PASS == 0), bool ALL = false, int PPL = kPPL, typename Ins,
          typename Rng = FullRange>
__device__ __forceinline__ void expand_row(const SpgemmArgs<V>& p, int64_t a0, int alen, int wi, int nw, Ins&& ins,
                                           Rng rng = Rng(), const PreBatch<V>* pre = nullptr, int skip_len = 0) {
  const int lane = lane_id();
  const int nb = (alen + 31) >> 5;
  constexpr int CH = 32 * PPL;
  // fewer batches than warps: G = nw/nb warps per batch, splitting its product chunks;
  // otherwise batches go round-robin and a warp takes all chunks of its batch
  const int G = ALL ? nw : (nb >= nw ? 1 : nw / nb);
  const bool share = G > 1;
  const int b_first = ALL ? 0 : (share ? wi / G : wi), b_step = ALL ? 1 : (share ? nb : nw);
  int c_first = ALL ? 0 : (share ? wi % G : 0);
  const int c_step = share ? G : 1;
  int rot = 0;   // ALL: warp taking the next chunk (warp-uniform, identical in every warp)
  auto my_first = [&](int nsub) {   // ALL: first chunk of this warp among nsub, then advance the rotation
    const int j0 = (wi - rot) & (nw - 1);   // nw is a power of two (warps per CTA)
    rot = (rot + nsub) & (nw - 1);
    return j0;
  };
  for (int b = b_first; b < nb; b += b_step) {
    const int f = b * 32 + lane;
    int64_t bst = 0;
    int blen = 0;
    V a = V(0);
    if (pre && b == 0 && pre->valid) {
      bst = pre->bst;
      blen = pre->blen;
      a = pre->a;
    } else if (f < alen) {
      const int32_t kc = p.A_col[a0 + f];
      if (PASS == 1) a = ldv(p.A_val + a0 + f);
      int64_t s, e;
      rng(f, p.B_rp[kc], p.B_rp[kc + 1], s, e);
      bst = s;
      blen = (int)(e - s);
      if (skip_len > 0 && blen >= skip_len) blen = 0;   // taken from the caller's shared list
    }
    // STREAM (symbolic, long-row bitmap kernel): long referenced B rows (>= kStreamLen
    // products) are streamed by the warp directly — contiguous, coalesced loads, no owner
    // search; the balanced expansion below takes the short ones (C3 symbolic 130 -> 83 ms).
    // The hash-map numeric kernels keep the balanced expansion for every row: a second
    // inlined copy of their larger insert code cost more in instruction-cache misses than the
    // search it saves (C5 numeric 429 -> 490 ms).
    if (STREAM) {
      const uint32_t lm = __ballot_sync(0xffffffffu, blen >= kStreamLen);
      for (uint32_t rem = lm; rem; rem &= rem - 1) {
        const int o = __ffs(rem) - 1;
        const int64_t s0 = __shfl_sync(0xffffffffu, bst, o);
        const int L = __shfl_sync(0xffffffffu, blen, o);
        const V ao = PASS == 1 ? __shfl_sync(0xffffffffu, a, o) : V(0);
        if (ALL) c_first = my_first((L + CH - 1) / CH);
        for (int q0 = c_first * CH; q0 < L; q0 += c_step * CH) {
          uint32_t c[PPL];
          V bv[PPL];
#pragma unroll
          for (int i = 0; i < PPL; ++i) {
            const int q = q0 + 32 * i + lane;
            c[i] = q < L ? (uint32_t)p.B_col[s0 + q] : (0x80000000u | (uint32_t)lane);
            bv[i] = (PASS == 1 && q < L) ? ldv(p.B_val + s0 + q) : V(0);
          }
#pragma unroll
          for (int i = 0; i < PPL; ++i) {
            if (q0 + 32 * i >= L) continue;   // warp-uniform
            ins(c[i], ao * bv[i], q0 + 32 * i + lane < L);
          }
        }
      }
      if (blen >= kStreamLen) blen = 0;
    }
    const int incl = warp_incl_scan(blen);
    const int excl = incl - blen;
    const int Pb = __shfl_sync(0xffffffffu, incl, 31);
    const int64_t boff = bst - excl;   // product pp of owner o is B entry boff_o + pp
    // locate the products of chunk q0 and issue their loads (not consumed here)
    auto gather = [&](int q0, uint32_t (&c)[PPL], V (&bv)[PPL], int (&ow)[PPL]) {
#pragma unroll
      for (int i = 0; i < PPL; ++i) {
        c[i] = 0x80000000u | (uint32_t)lane;   // inactive lanes keep a key that is never a real column
        bv[i] = V(0);
        ow[i] = 0;
        if (q0 + 32 * i >= Pb) continue;       // warp-uniform: the whole sub-chunk is past the row
        const int pp = q0 + lane + 32 * i;
        int lo = 0;                            // owner lane: smallest o with incl_o > pp
#pragma unroll
        for (int step = 16; step > 0; step >>= 1) {
          const int probe = __shfl_sync(0xffffffffu, incl, lo + step - 1);
          if (probe <= pp) lo += step;
        }
        const int o = lo > 31 ? 31 : lo;
        const int64_t idx = __shfl_sync(0xffffffffu, boff, o) + pp;
        ow[i] = o;
        if (pp < Pb) {
          c[i] = (uint32_t)p.B_col[idx];
          if (PASS == 1) bv[i] = ldv(p.B_val + idx);
        }
      }
    };
    // gather a chunk (PPL independent loads per lane), then insert it
    uint32_t ca[PPL];
    V va[PPL];
    int oa[PPL];
    if (ALL) c_first = my_first((Pb + CH - 1) / CH);
    for (int p0 = c_first * CH; p0 < Pb; p0 += c_step * CH) {
      gather(p0, ca, va, oa);
#pragma unroll
      for (int i = 0; i < PPL; ++i) {
        if (p0 + 32 * i >= Pb) continue;   // uniform skip of empty sub-chunks
        const V ao = PASS == 1 ? __shfl_sync(0xffffffffu, a, oa[i]) : V(0);
        ins(ca[i], ao * va[i], p0 + lane + 32 * i < Pb);
      }
    }
  }
}

// The paper's local load balancer: groups of g threads (g a power of two, 1..32*nw)
// are assigned round-robin to the referenced B rows of the row of A; the g threads of a group
// stride over their B row.  g = SPECK_OPT_FIXED_GROUP_SIZE, or the dynamic group
// size of P:940-970 (local_group_size, reading R9) when the option is -1.  Kept for the Fig. 13
// ablation and as an option; the default is the expand-balanced enumeration (expand_esc /
// expand_row), which gives every lane the same number of products.  f(col, a*b, active) is
// called by all 32 lanes of the warp in step.
template <int PASS, typename V, typename F>
__device__ __forceinline__ void expand_grouped(const SpgemmArgs<V>& p, int64_t a0, int alen, int wi, int nw, int g,
                                               F&& f) {
  const int lane = lane_id();
  const int T = 32 * nw;
  g = g < 1 ? 1 : (g > T ? T : g);
  const int k = T / g;                                  // groups
  const int tid = wi * 32 + lane;
  const int q = tid / g, t = tid % g;                   // group, thread within the group
  for (int r0 = 0; r0 < alen; r0 += k) {
    const int fi = r0 + q;                              // this group's referenced row in the round
    int64_t bst = 0;
    int len = 0;
    V a = V(0);
    if (fi < alen) {
      const int32_t kc = p.A_col[a0 + fi];
      if (PASS == 1) a = __ldg(p.A_val + a0 + fi);
      bst = p.B_rp[kc];
      len = (int)(p.B_rp[kc + 1] - bst);
    }
    const int iters = (int)__reduce_max_sync(0xffffffffu, (unsigned)((len - t + g - 1) > 0 ? (len - t + g - 1) / g : 0));
    for (int it = 0; it < iters; ++it) {
      const int j = t + it * g;
      const bool act = j < len;
      uint32_t col = 0x80000000u | (uint32_t)lane;
      V bv = V(0);
      if (act) {
        col = (uint32_t)p.B_col[bst + j];
        if (PASS == 1) bv = __ldg(p.B_val + bst + j);
      }
      f(col, a * bv, act);
    }
  }
}

// Referenced B rows of at least kLongB entries collected into a shared list (collect_long_rows)
// and streamed by all nw warps, product chunks rotated over the warps (no redundant batch
// loads, unlike expand_row's ALL mode, which re-reads every batch in every warp: for C4's
// 200k-NZ rows of A that was 32x the A traffic).
constexpr int kLongB = 1024;
constexpr int kLongListCap = 128;
template <typename V>
struct LongList {
  int64_t bst[kLongListCap];
  int32_t len[kLongListCap];
  V a[kLongListCap];
  int n;
};
// All threads of the block; barriers inside.  Returns true if every long row fit the list.
template <int PASS, typename V>
__device__ bool collect_long_rows(const SpgemmArgs<V>& p, int64_t a0, int alen, LongList<V>& L) {
  if (threadIdx.x == 0) L.n = 0;
  __syncthreads();
  for (int f = threadIdx.x; f < alen; f += blockDim.x) {
    const int32_t kc = p.A_col[a0 + f];
    const int64_t b0 = p.B_rp[kc];
    const int len = (int)(p.B_rp[kc + 1] - b0);
    if (len >= kLongB) {
      const int i = atomicAdd(&L.n, 1);
      if (i < kLongListCap) {
        L.bst[i] = b0;
        L.len[i] = len;
        L.a[i] = PASS == 1 ? ldv(p.A_val + a0 + f) : V(0);
      }
    }
  }
  __syncthreads();
  return L.n <= kLongListCap;
}
template <int PASS, typename V, typename Ins>
__device__ __forceinline__ void expand_long_list(const SpgemmArgs<V>& p, const LongList<V>& L, int wi, int nw, Ins&& ins) {
  constexpr int CH = 32 * kPPL;
  const int lane = lane_id();
  int rot = 0;
  for (int r = 0; r < L.n; ++r) {
    const int len = L.len[r];
    const int64_t s0 = L.bst[r];
    const V ao = L.a[r];
    const int nsub = (len + CH - 1) / CH;
    const int j0 = (wi - rot) & (nw - 1);   // nw is a power of two (warps per CTA)
    rot = (rot + nsub) & (nw - 1);
    for (int q0 = j0 * CH; q0 < len; q0 += nw * CH) {
      uint32_t c[kPPL];
      V bv[kPPL];
#pragma unroll
      for (int i = 0; i < kPPL; ++i) {
        const int q = q0 + 32 * i + lane;
        c[i] = q < len ? (uint32_t)p.B_col[s0 + q] : (0x80000000u | (uint32_t)lane);
        bv[i] = (PASS == 1 && q < len) ? ldv(p.B_val + s0 + q) : V(0);
      }
#pragma unroll
      for (int i = 0; i < kPPL; ++i) {
        if (q0 + 32 * i >= len) continue;   // warp-uniform
        ins(c[i], ao * bv[i], q0 + 32 * i + lane < len);
      }
    }
  }
}

// first index in [l, h) with col >= x (rows of B are sorted)
__device__ __forceinline__ int64_t lower_bound_col(const int32_t* __restrict__ col, int64_t l, int64_t h, uint32_t x) {
  while (l < h) {
    const int64_t mid = (l + h) >> 1;
    if ((uint32_t)col[mid] < x) l = mid + 1; else h = mid;
  }
  return l;
}

// Column windows processed in ascending order: each referenced B row resumes where the
// previous window stopped and ends at the first column >= whi.  The resume
// offsets are double-buffered (read cur, write next; the caller swaps after the window's
// barrier), because warps sharing one batch of a row all evaluate the same f.
struct WindowRange {
  const int32_t* cur;        // resume offsets per NZ of the row of A (relative to the B row start)
  int32_t* next;
  const int32_t* bcol;
  uint32_t whi;
  __device__ __forceinline__ void operator()(int f, int64_t j0, int64_t j1, int64_t& s, int64_t& e) const {
    s = j0 + cur[f];
    e = lower_bound_col(bcol, s, j1, whi);
    next[f] = (int32_t)(e - j0);
  }
};

// Per referenced B row, [j0 + cur[f], j0 + next[f]) precomputed by the caller (pure: every warp
// may evaluate it).
struct KnownRange {
  const int32_t* cur;
  const int32_t* next;
  __device__ __forceinline__ void operator()(int f, int64_t j0, int64_t, int64_t& s, int64_t& e) const {
    s = j0 + cur[f];
    e = j0 + next[f];
  }
};

// An independent column range [lo, hi) of every referenced B row (long-row segments).
struct SegRange {
  const int32_t* bcol;
  uint32_t lo, hi;
  __device__ __forceinline__ void operator()(int, int64_t j0, int64_t j1, int64_t& s, int64_t& e) const {
    s = lower_bound_col(bcol, j0, j1, lo);
    e = lower_bound_col(bcol, s, j1, hi);
  }
};

// Dense-window insert: flag bit (structural entry) and, numeric, the value (warp-aggregated).
template <int PASS, typename V>
__device__ __forceinline__ void dense_insert(uint32_t* bits, V* dvals, uint32_t wlo, uint32_t col, V v, bool act) {
  const uint32_t c = col - wlo;
  if (PASS == 0) {
    if (act) atomicOr(&bits[c >> 5], 1u << (c & 31));
  } else {
    bool leader;
    const V sum = warp_key_sum(col, v, leader);
    if (act && leader) {
      atomicOr(&bits[c >> 5], 1u << (c & 31));
      atomicAdd(&dvals[c], sum);
    }
  }
}

// Coalesced, sorted write-out of a numeric dense window (values + flag bits): warp w owns a
// contiguous range of flag words; pass 1 counts, one block-level prefix over the warps, pass 2
// broadcasts each word and lane b writes the entry of bit b, so every store instruction
// writes up to 32 consecutive entries of C.  Returns the entries written (barriers inside).
template <int T, typename V>
__device__ int64_t dense_emit(const uint32_t* bits, const V* dvals, int nwords, uint32_t wlo, int64_t out,
                              int32_t* __restrict__ C_col, V* __restrict__ C_val, int64_t* part) {
  constexpr int NW = T / 32;
  const int lane = lane_id(), wp = warp_id();
  const int WW = ((nwords + NW - 1) / NW + 31) & ~31;
  const int w0 = min(nwords, wp * WW), w1 = min(nwords, w0 + WW);
  int cnt = 0;
  for (int i = w0 + lane; i < w1; i += 32) cnt += __popc(bits[i]);
  cnt = warp_sum(cnt);
  if (lane == 0) part[wp] = cnt;
  __syncthreads();
  int64_t base = out, total = 0;
  for (int w = 0; w < NW; ++w) {
    const int64_t c = part[w];
    if (w < wp) base += c;
    total += c;
  }
  for (int c0 = w0; c0 < w1; c0 += 32) {
    const int wi = c0 + lane;
    const uint32_t word = wi < w1 ? bits[wi] : 0u;
    const int pc = __popc(word);
    const int incl = warp_incl_scan(pc);
    const int excl = incl - pc;
    for (int j = 0; j < 32; ++j) {
      const uint32_t wj = __shfl_sync(0xffffffffu, word, j);
      if (!wj) continue;   // warp-uniform
      const int oj = __shfl_sync(0xffffffffu, excl, j);
      if ((wj >> lane) & 1u) {
        const int64_t o = base + oj + __popc(wj & ((1u << lane) - 1u));
        const uint32_t ci = (uint32_t)(c0 + j) * 32u + (uint32_t)lane;
        C_col[o] = (int32_t)(wlo + ci);
        C_val[o] = dvals[ci];
      }
    }
    base += __shfl_sync(0xffffffffu, incl, 31);
  }
  __syncthreads();   // part[] is reused by the caller
  return total;
}

// Per-SM resume scratch slot of multi-window dense rows.  The slot is private because such
// rows run only in the largest configuration, whose 225 KB of shared memory admits one CTA per
// SM (no other kernel of any launch can co-reside with it: the bitmap kernel needs the same
// 225 KB).  The buffer holds %nsmid slots (queried at speck_create; %smid < %nsmid, which may
// exceed the SM count), and an out-of-range id traps instead of writing past the buffer.
__device__ __forceinline__ unsigned smid() {
  unsigned r;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(r));
  return r;
}
__device__ __forceinline__ unsigned nsmid() {
  unsigned r;
  asm volatile("mov.u32 %0, %%nsmid;" : "=r"(r));
  return r;
}

// Warp-path write-out of a scrambled (or wrapped) map region: compact in place, then rank
// counting for <= kSmallSeg entries or a warp bitonic sort.  Out of line.
template <typename V>
__device__ __noinline__ void warp_row_sorted_write(uint32_t* rk, V* rv, uint32_t S, int64_t ob, int32_t* __restrict__ C_col,
                                                   V* __restrict__ C_val) {
  const int lane = lane_id();
  int pos = 0;
  for (uint32_t c0 = 0; c0 < S; c0 += 32) {
    const uint32_t s = c0 + lane;
    uint32_t kk = kEmptyKey;
    V vv = V(0);
    if (s < S) { kk = rk[s]; vv = rv[s]; }
    const uint32_t occ = __ballot_sync(0xffffffffu, kk != kEmptyKey);
    __syncwarp();
    if (kk != kEmptyKey) {
      const int o = pos + __popc(occ & ((1u << lane) - 1u));
      rk[o] = kk;
      rv[o] = vv;
    }
    pos += __popc(occ);
    __syncwarp();
  }
  const int cnt = pos;
  if (cnt <= kSmallSeg) {
    // all lanes read key j together (shared-memory broadcast)
    for (int e0 = 0; e0 < cnt; e0 += 32) {
      const int e = e0 + lane;
      const uint32_t key = e < cnt ? rk[e] : 0xffffffffu;
      const V val = e < cnt ? rv[e] : V(0);
      int rank = 0;
      for (int j = 0; j < cnt; ++j) rank += rk[j] < key;
      if (e < cnt) {
        C_col[ob + rank] = (int32_t)key;
        C_val[ob + rank] = val;
      }
    }
  } else {
    smem_bitonic_sort<32, V, true>(rk, rv, cnt);
    for (int e = lane; e < cnt; e += 32) {
      C_col[ob + e] = (int32_t)rk[e];
      C_val[ob + e] = rv[e];
    }
  }
}

// Block-path write-out of scrambled (or wrapped) maps: order-preserving compaction of all row
// regions, rank counting for short rows, bitonic sort for long ones.  Out of line.
template <int T, typename V>
__device__ __noinline__ void block_sorted_write(uint32_t* keys, V* vals, uint32_t capt, BlockMeta& bm,
                                                int32_t* __restrict__ C_col, V* __restrict__ C_val) {
  const int tid = threadIdx.x;
  const int nr = bm.nr;
  int64_t running = 0;
  for (uint32_t base = 0; base < capt; base += T) {
    const uint32_t s = base + tid;
    uint32_t kk = kEmptyKey;
    V vv = V(0);
    if (s < capt) { kk = keys[s]; vv = vals[s]; }
    const int64_t fl = kk != kEmptyKey;
    int64_t tot;
    const int64_t pos = block_excl_scan<T>(fl, bm.scan_part, &tot);
    if (fl) { keys[running + pos] = kk; vals[running + pos] = vv; }
    running += tot;
    __syncthreads();
  }
  const int ncnt = (int)bm.cnt;
  int rr = 0;
  for (int i = tid; i < ncnt; i += T) {
    while (i >= bm.cseg[rr + 1]) ++rr;
    const int s0 = bm.cseg[rr], s1 = bm.cseg[rr + 1];
    if (s1 - s0 > kSmallSeg) continue;
    const uint32_t key = keys[i];
    int rank = 0;
    for (int j = s0; j < s1; ++j) rank += keys[j] < key;
    const int64_t o = bm.cbase[rr] + rank;
    C_col[o] = (int32_t)key;
    C_val[o] = vals[i];
  }
  for (int r = 0; r < nr; ++r) {
    const int s0 = bm.cseg[r], s1 = bm.cseg[r + 1];
    if (s1 - s0 <= kSmallSeg) continue;
    __syncthreads();
    smem_bitonic_sort<T, V>(keys + s0, vals + s0, s1 - s0);
    const int64_t o = bm.cbase[r];
    for (int i = tid; i < s1 - s0; i += T) {
      C_col[o + i] = (int32_t)keys[s0 + i];
      C_val[o + i] = vals[s0 + i];
    }
  }
}

// One row of C by one warp in a private map region rk/rv[0, S) (cleared here): expand-balanced
// products, hash insert (symbolic: count new keys; numeric: equal keys of a warp step add in
// rounds — the region is private, so no atomics on values), then the sorted write-out
// (ordered map for rows > kSmallSeg entries, else rank counting).  Returns the symbolic count.
// MODE (numeric): 0 any row, 1 rows of <= kSmallSeg entries only, 2 larger rows only.
template <int PASS, typename V, int MODE = 0>
__device__ __forceinline__ int warp_row(const SpgemmArgs<V>& p, uint32_t* rk, V* rv, uint32_t S, int64_t a0, int alen,
                                        int32_t cmin, int32_t cmax, int32_t cnt, int64_t cbase,
                                        const PreBatch<V>* pre = nullptr, int64_t warp_row_prods = 0,
                                        int64_t warp_row_maxlen = 0) {
  const int lane = lane_id();
  for (uint32_t i = lane; i < S; i += 32) {
    rk[i] = kEmptyKey;
    if (PASS == 1) rv[i] = V(0);
  }
  __syncwarp();
  const uint32_t mlo = (uint32_t)cmin;
  const uint64_t mmult = bkt_mult((uint32_t)(cmax - cmin + 1), S);
  // long rows use the order-preserving map (sorted write-out without a sort network);
  // short rows keep the scrambled hash (robust to clustered columns) and rank counting
  constexpr int M = MODE & 7;
  const bool ordered = PASS == 1 && (M == 2 || (M == 0 && cnt > kSmallSeg));
  int newc = 0, wrapped = 0;
  // 2 products per lane per chunk (fewer registers, more resident warps) for numeric MODE 1/2 rows
  // (C5 numeric 379 -> 362 ms, C2 tiny rows at 40 warps/SM 2.56 -> 2.35 ms) and symbolic rows
  // (C2 symbolic A*P 1.38 -> 1.31 ms; 8 per lane spills: 1.72 ms); numeric MODE 0 rows 4
  // products: symbolic rows by expand_row (long B rows streamed, short ones balanced), numeric
  // rows by expand_esc (REDUX owner search, esc_kernels.cuh) with the first batch loaded ahead
  auto ins = [&](uint32_t col, V v, bool act) {
    if (PASS == 0) {
      if (act) newc += hash_insert_key(rk, S, col);
    } else {
      const uint32_t peers = __match_any_sync(0xffffffffu, col);
      const uint32_t lt = (1u << lane_id()) - 1u;
      uint32_t s = 0;
      if (act && !(peers & lt)) {
        s = ordered ? probe_insert_bkt(rk, S >> 3, bkt_home(col, mlo, mmult), col, &wrapped)
                    : probe_insert_mono(rk, S, hash_slot(col, S), col, &wrapped);
      }
      // equal keys of the warp step add in lane order, one round each: no atomics on values, and
      // the in-order, per-product-rounded sum of reading R15 (summing the peers in registers
      // first was tried: C2 numeric A*P 2.35 -> 2.52 ms, fp64 shuffles cost two instructions)
      s = __shfl_sync(0xffffffffu, s, __ffs(peers) - 1);   // the key's slot, from its first lane
      const int rank = __popc(peers & lt);
      const int maxg = (int)__reduce_max_sync(0xffffffffu, (unsigned)__popc(peers));
      for (int t = 0; t < maxg; ++t) {
        if (act && rank == t) rv[s] = add_rn(rv[s], v);
        __syncwarp();
      }
    }
  };
  if (MODE & 8) {
    // the paper's local load balancing (Fig. 13 ablation; own kernel instantiation, MODE | 8, so
    // its registers do not weigh on the default path): one warp = T threads, g per group
    int g = p.fixed_g;
    if (g < 0) g = local_group_size(32, alen, warp_row_prods, warp_row_maxlen);
    expand_grouped<PASS, V>(p, a0, alen, 0, 1, g, ins);
  } else if (PASS == 0) {
    // symbolic warp rows by expand_esc too (REDUX owner search; the streamed shuffle binary search
    // of expand_row measured slower once the probe was mask-based: C5 19.0 -> 18.3 ms, C2 A*P
    // 1.39 -> 1.37 ms, profiles/r02/r02as_*)
    expand_esc<PASS, V, SPECK_SYM_WARP_U>(p, a0, alen, 0, 1, ins);
  } else {
    expand_esc<PASS, V, SPECK_WARP_U>(p, a0, alen, 0, 1, ins, pre);
  }
  if (PASS == 0) {
    if (lane == 0) count_path(p.paths, SPECK_PATH_SYM_WARP);
    __syncwarp();   // the region's last probes complete before the next row clears it (racecheck)
    return warp_sum(newc);
  }
  if (M != 1 && ordered && !__any_sync(0xffffffffu, wrapped)) {
    // ordered map: every entry goes to (occupied slots before its run) + (rank in the run)
    if (lane == 0) count_path(p.paths, SPECK_PATH_NUM_WARP_ORDERED);
    warp_write_ordered<V>(rk, rv, S, 0u, S, cbase, 0, p.C_col, p.C_val);
  } else {
    if (lane == 0) count_path(p.paths, M == 1 || cnt <= kSmallSeg ? SPECK_PATH_NUM_TINY : SPECK_PATH_NUM_WARP_SORTED);
    warp_row_sorted_write<V>(rk, rv, S, cbase, p.C_col, p.C_val);
  }
  __syncwarp();
  return 0;
}

template <int CFG, int PASS, typename V>
__device__ __noinline__ void dense_row(const SpgemmArgs<V>& p, BlockMeta& bm, int b0, unsigned char* smem, int* chist,
                                       int64_t gidx);

// -----------------------------------------------------------------------------------
// The per-configuration kernel.  PASS 0 = symbolic, 1 = numeric.
// -----------------------------------------------------------------------------------
template <int CFG, int PASS, typename V>
__device__ __forceinline__ void spgemm_group(const SpgemmArgs<V>& p, const int64_t gidx, unsigned char* smem, BlockMeta& bm,
                                             int* chist) {
  constexpr int T = kCfgThreads[CFG];
  const int tid = threadIdx.x;

  const int64_t e0 = gidx * p.group_rows;
  const int ne = (int)(p.n_entries - e0 < p.group_rows ? p.n_entries - e0 : p.group_rows);
  if (ne <= 0) return;

  // ---- group: load rows and needs, block merge (Alg. 2) -------------------------------
  if (tid < 32) {
    int32_t row = -1;
    int64_t need = 0;
    if (tid < ne) {
      row = p.rows ? p.rows[e0 + tid] : (int32_t)(e0 + tid);
      need = PASS == 0 ? p.prods[row] : (p.C_rp[row + 1] - p.C_rp[row]);
      bm.row[tid] = row;
    }
    const uint32_t st = p.merge ? warp_block_merge(need, ne, p.merge_cap) : 1u;
    if (tid == 0) bm.starts = st;
  }
  __syncthreads();
  const uint32_t starts = bm.starts;

  for (int b0 = 0; b0 < ne;) {
    const uint32_t rest = b0 >= 31 ? 0u : (starts & ~((2u << b0) - 1u));
    const int b1 = rest ? __ffs(rest) - 1 : ne;
    const int nr = b1 - b0;

    // ---- block setup (warp 0) ------------------------------------------------------
    if (tid < 32) {
      const int l = tid;
      int64_t a0 = 0, alen = 0, pr = 0, ml = 0, c0 = 0, c = 0;
      int32_t cmn = 0x7fffffff, cmx = -1;
      int32_t row = -1;
      if (l < nr) {
        row = bm.row[b0 + l];
        a0 = p.A_rp[row];
        alen = p.A_rp[row + 1] - a0;
        pr = p.prods[row];
        ml = p.maxlen[row];
        cmn = p.colmin[row];
        cmx = p.colmax[row];
        if (PASS == 1) { c0 = p.C_rp[row]; c = p.C_rp[row + 1] - c0; }
      }
      const int64_t ainc = warp_incl_scan(alen);
      const int64_t cinc = warp_incl_scan(c);
      const int64_t pinc = warp_incl_scan(pr);
      int64_t mlx = ml;
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) mlx = max(mlx, __shfl_xor_sync(0xffffffffu, mlx, o));
      const int64_t tot_a = __shfl_sync(0xffffffffu, ainc, 31);
      const int64_t tot_c = __shfl_sync(0xffffffffu, cinc, 31);
      const int64_t tot_p = __shfl_sync(0xffffffffu, pinc, 31);
      // hash regions: proportional to the row's need (prods for symbolic, cnt numeric)
      const uint32_t cap = PASS == 0 ? sym_map_cap(CFG) : num_map_cap<V>(CFG);
      const int64_t need = PASS == 0 ? pr : c;
      const int64_t need_tot = PASS == 0 ? tot_p : tot_c;
      uint32_t rsz = 0;
      // (multiples of 4 slots so 4-slot probe groups stay 16-byte aligned: 4 + a share of the rest)
      // A single row gets a region sized to it (symbolic 4x products, numeric 2.5x entries:
      // <= 50% / 40% load), so clearing and the write-out scan touch only the slots the row can use
      // (C5: the write-out scan of the full map was over half of the numeric instructions).
      if (l < nr) {
        if (nr == 1) {
          const uint64_t want = PASS == 0 ? (uint64_t)need * SPECK_SYM_REGION_X2 / 2 : (uint64_t)need * 5 / 2;
          const uint64_t w32 = (want + 31) & ~(uint64_t)31;
          rsz = (uint32_t)(w32 < 64 ? 64 : (w32 > cap ? cap : w32));
        } else {
          rsz = 4u + (need_tot > 0 ? (uint32_t)((uint64_t)(cap - 4u * nr) * (uint64_t)need / (uint64_t)need_tot) & ~3u : 0u);
        }
      }
      const uint32_t rinc = warp_incl_scan(rsz);
      const bool any_small = __any_sync(0xffffffffu, l < nr && c <= kSmallSeg);
      if (l < nr) {
        bm.astart[l] = a0;
        bm.aoff[l + 1] = ainc;
        bm.cbase[l] = c0;
        bm.cseg[l + 1] = (int32_t)cinc;
        bm.rbase[l + 1] = rinc;
        bm.rcnt[l] = 0;
        bm.rlo[l] = cmn;
        bm.rhi[l] = cmx;
        bm.rwrap[l] = 0;
      }
      if (l == 0) {
        bm.aoff[0] = 0; bm.cseg[0] = 0; bm.rbase[0] = 0;
        bm.nr = nr;
        bm.ordered = PASS == 1 && !any_small;
        bm.nnzA = tot_a;
        bm.prods = tot_p;
        bm.maxlen = mlx;
        bm.cnt = tot_c;
        bm.colmin = cmn;
        bm.colmax = cmx;
        // ---- accumulator choice (per block) ----
        int dense = 0;
        const int64_t range = (int64_t)cmx - cmn + 1;
        if (nr == 1 && tot_p > 0) {
          if (PASS == 0) {
            const int64_t W = sym_dense_window(CFG);
            if (p.force_acc == 2) dense = 1;
            else if ((uint64_t)tot_p > (uint64_t)sym_map_fill(CFG)) dense = 1;         // beyond the map: P:1112-1113
            else if (p.force_acc != 1 && range <= W && range <= 16 * tot_p) dense = 1;  // bitmap cheaper than hashing
          } else {
            const int64_t W = num_dense_window<V>(CFG);
            const int64_t nwin = (range + W - 1) / W;
            if (p.force_acc == 2) dense = 1;
            else if ((uint64_t)tot_c > (uint64_t)num_map_fill<V>(CFG)) dense = 1;       // rows needing the largest kernel: P:1146-1148
            else if (p.force_acc != 1 && nwin <= (CFG == kNumCfg - 1 ? kDenseMaxWindows : 1) &&
                     tot_c * 100 > (int64_t)kDensePct * range) dense = 1;              // density > 18%: P:1127-1129
          }
          if (dense && CFG != kNumCfg - 1) {
            // smaller configurations only run single-window dense rows
            const int64_t W = PASS == 0 ? sym_dense_window(CFG) : num_dense_window<V>(CFG);
            int64_t Wc = (p.dense_window_cap > 0 && p.dense_window_cap < W) ? p.dense_window_cap : W;
            if (range > Wc) dense = 0;
          }
        }
        bm.dense = dense;
        // single-row hash blocks whose products are (almost) all distinct: bucket counting sort
        const int64_t ecap = esc_capacity<V>(PASS, kCfgMapBytes[CFG]);
        bm.esc = (nr == 1 && !dense && tot_p > 0 && tot_p <= ecap && tot_p <= 32 * T && CFG <= SPECK_ESC_MAX_CFG &&
                  p.esc >= (PASS == 0 ? 2 : 1) && (PASS == 0 || tot_p * 100 <= (int64_t)kEscRatioPct * tot_c)) ? 1 : 0;
      }
    }
    __syncthreads();
    constexpr int NW = T / 32;

    int esc_done = 0;
    if (bm.esc) {
      // ===================== BUCKET COUNTING SORT (esc_kernels.cuh) =====================
      const bool chunks = CFG == kNumCfg - 1 && PASS == 0 && p.chunk_cnt && bm.prods > p.long_thr;
      if (chunks) {
        for (int i = tid; i < p.nchunks; i += T) chist[i] = 0;
        __syncthreads();
      }
      const int c =
          (kEscStaged && !chunks && bm.prods <= esc_staged_capacity<V>(PASS, kCfgMapBytes[CFG]))
              ? esc_row_staged<NW, PASS, V>(p, smem, kCfgMapBytes[CFG], warp_id(), bm.astart[0], (int)bm.nnzA, (int)bm.prods, (int)bm.cnt,
                                      bm.colmin, bm.colmax, bm.cbase[0], reinterpret_cast<int*>(bm.scan_part))
              : esc_row<NW, PASS, V>(p, smem, kCfgMapBytes[CFG], warp_id(), bm.astart[0], (int)bm.nnzA,
                                     (int)bm.prods, (int)bm.cnt, bm.colmin, bm.colmax, bm.cbase[0],
                                     reinterpret_cast<int*>(bm.scan_part), chunks ? chist : nullptr,
                                     p.chunk_shift);
      if (c >= 0) {
        esc_done = 1;
        if (PASS == 0 && tid == 0) p.cnt[bm.row[b0]] = c;
        if (chunks) {
          __syncthreads();
          int32_t* dst = p.chunk_cnt + gidx * p.nchunks;
          for (int i = tid; i < p.nchunks; i += T) dst[i] = chist[i];
        }
      }
      __syncthreads();
    }
    if (esc_done) {
    } else if (!bm.dense && nr >= NW && nr > 1) {
      // ===================== HASH, WARP PER ROW (multi-row blocks) =====================
      if (tid == 0) count_path(p.paths, PASS == 0 ? SPECK_PATH_SYM_MERGED : SPECK_PATH_NUM_MERGED);
      // Each warp owns whole rows and their private map regions, so accumulation and the
      // sort/compaction epilogue need no block barrier; lanes whose key is unique within
      // the warp step update the value with a plain read-modify-write.
      uint32_t* keys = reinterpret_cast<uint32_t*>(smem);
      V* vals = reinterpret_cast<V*>(smem + (PASS == 0 ? 0u : num_val_offset<V>(CFG)));
      const int lane = lane_id();
      for (int r = warp_id(); r < nr; r += NW) {
        const uint32_t rb = bm.rbase[r], S = bm.rbase[r + 1] - rb;
        const int c = warp_row<PASS, V>(p, keys + rb, vals + rb, S, bm.astart[r], (int)(bm.aoff[r + 1] - bm.aoff[r]),
                                        bm.rlo[r], bm.rhi[r], bm.cseg[r + 1] - bm.cseg[r], bm.cbase[r]);
        if (PASS == 0 && lane == 0) p.cnt[bm.row[b0 + r]] = c;
        __syncwarp();
      }
    } else if (!bm.dense) {
      // ============================ HASH ACCUMULATOR ==============================
      uint32_t* keys = reinterpret_cast<uint32_t*>(smem);
      const uint32_t capt = bm.rbase[nr];
      V* vals = reinterpret_cast<V*>(smem + (PASS == 0 ? 0u : num_val_offset<V>(CFG)));
      for (uint32_t i = tid; i < capt; i += T) {
        keys[i] = kEmptyKey;
        if (PASS == 1) vals[i] = V(0);
      }
      __syncthreads();
      // all warps share each row: expand-balanced products, warp aggregation of equal keys,
      // one atomic per distinct key per warp step (other warps may hold the same key)
      for (int r = 0; r < nr; ++r) {
        const uint32_t rb = bm.rbase[r], S = bm.rbase[r + 1] - rb;
        uint32_t* rk = keys + rb;
        V* rv = vals + rb;
        const uint32_t mlo = (uint32_t)bm.rlo[r];
        const uint64_t mmult = bkt_mult((uint32_t)(bm.rhi[r] - bm.rlo[r] + 1), S);
        const bool ordered = bm.ordered;
        int newc = 0, wrapped = 0;
        auto ins = [&](uint32_t col, V v, bool act) {
                              if (PASS == 0) {
                                if (act) newc += hash_insert_key(rk, S, col);
                              } else {
                                uint32_t s = 0;
                                if (act)
                                  s = ordered ? probe_insert_bkt(rk, S >> 3, bkt_home(col, mlo, mmult), col, &wrapped)
                                              : probe_insert_mono(rk, S, hash_slot(col, S), col, &wrapped);
                                bool leader;
                                const V sum = warp_key_sum(col, v, leader);
                                if (act && leader) atomicAdd(&rv[s], sum);
                              }
                            };
        const int ralen = (int)(bm.aoff[r + 1] - bm.aoff[r]);
        if (p.fixed_g != 0) {
          // the paper's local load balancing (Fig. 13 ablation): T threads in groups of g
          const int g = p.fixed_g > 0 ? p.fixed_g
                                      : local_group_size(T, ralen, p.prods[bm.row[b0 + r]], p.maxlen[bm.row[b0 + r]]);
          expand_grouped<PASS, V>(p, bm.astart[r], ralen, warp_id(), NW, g, ins);
        } else {
          expand_esc<PASS, V, PASS == 0 ? 4 : 2>(p, bm.astart[r], ralen, warp_id(), NW, ins);
        }
        if (PASS == 0) {
          newc = warp_sum(newc);
          if (lane_id() == 0 && newc) atomicAdd(&bm.rcnt[r], newc);
        } else if (__any_sync(0xffffffffu, wrapped) && lane_id() == 0) {
          bm.rwrap[r] = 1;
        }
      }
      __syncthreads();
      int any_wrap = !bm.ordered;   // scrambled maps take the compaction + sort epilogue
      if (PASS == 1)
        for (int rr = 0; rr < nr; ++rr) any_wrap |= bm.rwrap[rr];
      if (tid == 0)
        count_path(p.paths, PASS == 0 ? SPECK_PATH_SYM_BLOCK_HASH : any_wrap ? SPECK_PATH_NUM_BLOCK_SORTED : SPECK_PATH_NUM_BLOCK_ORDERED);
      if (PASS == 0) {
        if (tid < nr) p.cnt[bm.row[b0 + tid]] = bm.rcnt[tid];
        if (CFG == kNumCfg - 1 && p.chunk_cnt && nr == 1 && bm.prods > p.long_thr) {
          // long-row candidate: distinct columns per 2^15-column chunk, for the numeric split
          for (int i = tid; i < p.nchunks; i += T) chist[i] = 0;
          __syncthreads();
          for (uint32_t s = tid; s < capt; s += T) {
            const uint32_t kk = keys[s];
            if (kk != kEmptyKey) atomicAdd(&chist[kk >> p.chunk_shift], 1);
          }
          __syncthreads();
          int32_t* dst = p.chunk_cnt + gidx * p.nchunks;
          for (int i = tid; i < p.nchunks; i += T) dst[i] = chist[i];
        }
      } else if (!any_wrap) {
        // ---- ordered maps: each entry goes to (occupied before its cluster) + (rank in it) ----
        for (int rr = 0; rr < nr; ++rr) {
          const uint32_t rb = bm.rbase[rr];
          block_write_ordered<T, V>(keys + rb, vals + rb, bm.rbase[rr + 1] - rb, bm.cbase[rr], p.C_col, p.C_val,
                                    bm.scan_part);
        }
      } else {
        block_sorted_write<T, V>(keys, vals, capt, bm, p.C_col, p.C_val);
      }
    } else {
      dense_row<CFG, PASS, V>(p, bm, b0, smem, chist, gidx);
    }
    __syncthreads();
    b0 = b1;
  }
}

// One CTA per group of entries (grid = groups).
template <int CFG, int PASS, typename V>
__global__ void __launch_bounds__(kCfgThreads[CFG], 1024 / kCfgThreads[CFG]) k_spgemm(const __grid_constant__ SpgemmArgs<V> p) {
  extern __shared__ __align__(16) unsigned char smem[];
  __shared__ BlockMeta bm;
  __shared__ int chist[(CFG == kNumCfg - 1 && PASS == 0) ? kMaxChunks : 1];
  spgemm_group<CFG, PASS, V>(p, (int64_t)blockIdx.x, smem, bm, chist);
}

// ============================ DENSE ACCUMULATOR (single row) =============================
// Windows over [colmin, colmax] (Fig. 5); kept out of line so the hash paths'
// hot loops stay compact in the instruction cache.
template <int CFG, int PASS, typename V>
__device__ __noinline__ void dense_row(const SpgemmArgs<V>& p, BlockMeta& bm, int b0, unsigned char* smem, int* chist,
                                       int64_t gidx) {
  constexpr int T = kCfgThreads[CFG];
  constexpr int NW = T / 32;
  const int tid = threadIdx.x;
  const int64_t nnzA = bm.nnzA;
  {
    {
      const int32_t row = bm.row[b0];
      // symbolic windows start 32-aligned so a bitmap word never straddles a 2^15 chunk
      const int64_t lo = PASS == 0 ? (bm.colmin & ~31) : bm.colmin, hi = bm.colmax;
      const bool chunks = CFG == kNumCfg - 1 && PASS == 0 && p.chunk_cnt && bm.prods > p.long_thr;
      if (chunks) {
        for (int i = tid; i < p.nchunks; i += T) chist[i] = 0;   // ordered by the window's barrier
      }
      const int64_t W0 = PASS == 0 ? sym_dense_window(CFG) : num_dense_window<V>(CFG);
      const int64_t W = (p.dense_window_cap > 0 && p.dense_window_cap < W0) ? p.dense_window_cap : W0;
      const int64_t nwin = (hi - lo + 1 + W - 1) / W;
      const int64_t astart = bm.astart[0];
      uint32_t* bits = reinterpret_cast<uint32_t*>(smem);                       // W bits
      V* dvals = reinterpret_cast<V*>(smem + (PASS == 0 ? 0 : (((W + 31) / 32) * 4 + 15) / 16 * 16));
      int32_t* res = nullptr;       // double-buffered resume offsets (cur, next)
      int32_t* res_next = nullptr;
      if (tid == 0)
        count_path(p.paths, PASS == 0 ? (nwin > 1 ? SPECK_PATH_SYM_DENSE_MULTI : SPECK_PATH_SYM_DENSE)
                                      : (nwin > 1 ? SPECK_PATH_NUM_DENSE_MULTI : SPECK_PATH_NUM_DENSE));
      if (nwin > 1) {
        const unsigned slot = smid();
        if (slot >= (unsigned)p.resume_slots) __trap();
        res = p.resume + (int64_t)slot * p.resume_stride;
        res_next = res + p.resume_stride / 2;
        for (int64_t f = tid; f < nnzA; f += T) res[f] = 0;
      }
      int64_t out = PASS == 1 ? bm.cbase[0] : 0;
      int64_t total = 0;
      if (tid == 0 && PASS == 1 && p.n_dense_rows) atomicAdd(p.n_dense_rows, 1ull);
      for (int64_t w = 0; w < nwin; ++w) {
        const int64_t wlo = lo + w * W, whi = min(wlo + W, hi + 1);
        // only the window's actual width is cleared and scanned (the last / only window of a
        // row is usually much narrower than the scratchpad)
        const int nwords = (int)((whi - wlo + 31) / 32);
        for (int i = tid; i < nwords; i += T) bits[i] = 0u;
        if (PASS == 1)
          for (int64_t i = tid; i < whi - wlo; i += T) dvals[i] = V(0);
        __syncthreads();
        // expand-balanced accumulation of the products falling into this window
        auto ins = [&](uint32_t col, V v, bool act) { dense_insert<PASS, V>(bits, dvals, (uint32_t)wlo, col, v, act); };
        // ALL mode (every warp reads every batch) only where references are long on average:
        // C4's 200k-NZ rows of A with ~20 products per reference paid 32x their A traffic
        if (nwin == 1 && bm.prods >= kAllAvgLen * nnzA) expand_row<PASS, V, PASS == 0, true>(p, astart, (int)nnzA, warp_id(), NW, ins);
        else if (nwin == 1) expand_row<PASS, V>(p, astart, (int)nnzA, warp_id(), NW, ins);
        else expand_row<PASS, V>(p, astart, (int)nnzA, warp_id(), NW, ins, WindowRange{res, res_next, p.B_col, (uint32_t)whi});
        __syncthreads();
        { int32_t* t_ = res; res = res_next; res_next = t_; }
        // ---- window epilogue: count (symbolic) / compact in column order (numeric) ----
        int64_t wtot = 0;
        if (PASS == 1) {
          wtot = dense_emit<T, V>(bits, dvals, nwords, (uint32_t)wlo, out, p.C_col, p.C_val, bm.scan_part);
        } else {
          int cw = 0;
          for (int wi = tid; wi < nwords; wi += T) {
            const uint32_t word = bits[wi];
            cw += __popc(word);
            if (chunks && word) atomicAdd(&chist[(wlo + (int64_t)wi * 32) >> p.chunk_shift], __popc(word));
          }
          cw = warp_sum(cw);
          if (lane_id() == 0) bm.scan_part[warp_id()] = cw;
          __syncthreads();
          for (int w = 0; w < NW; ++w) wtot += bm.scan_part[w];
        }
        out += wtot;
        total += wtot;
        __syncthreads();
      }
      if (PASS == 0 && tid == 0) p.cnt[row] = total;
      if (CFG == kNumCfg - 1 && PASS == 0 && chunks && p.bm_pool && nwin == 1 && total > p.long_thr) {
        // keep the bitmap (words relative to colmin & ~31, as k_long_bitmap lays it out)
        const int nwords = (int)((hi - lo + 1 + 31) / 32);
        __shared__ long long s_bmo;
        if (tid == 0) {
          const unsigned long long need = ((unsigned long long)nwords + 3ull) & ~3ull;
          const unsigned long long o = atomicAdd(p.bm_ctr, need);
          s_bmo = o + need <= p.bm_pool_words ? (long long)o : -1ll;
          p.bm_off[gidx] = s_bmo;
        }
        __syncthreads();
        const long long o = s_bmo;
        if (o >= 0) {
          uint32_t* dst = p.bm_pool + o;
          for (int i = tid; i < nwords; i += T) dst[i] = bits[i];
        }
      }
      if (chunks) {
        int32_t* dst = p.chunk_cnt + gidx * p.nchunks;
        for (int i = tid; i < p.nchunks; i += T) dst[i] = chist[i];
      }
    }
  }
}

// -----------------------------------------------------------------------------------
// Small rows, one warp each (B200 replacement of the paper's block merge of small rows,
// P:785-804): every warp owns a 7 KB region and pulls rows of the bin from a global counter
// one row ahead, so no warp ever waits at a block barrier for another warp's row (ncu: 33% of
// the stall samples of the merged-block kernel were barrier waits).  The region is sized to
// the row (symbolic: 4x products (capped at the region); numeric: 2.5x exact nnz), so clearing and the
// write-out scan only the slots a row can use.  Rows of the bin (p.rows) or, without global
// load balancing, every row of A (p.rows == nullptr).
// -----------------------------------------------------------------------------------
template <int PASS, typename V, int MODE>
__global__ void __launch_bounds__(kWarpRowThreads, wr_ctas_per_sm(PASS, MODE & 7))
    k_warp_rows(const __grid_constant__ SpgemmArgs<V> p, unsigned long long* __restrict__ counter) {
  // MODE & 7: numeric 0 any row, 1 rows of <= kTinyCnt entries, 2 larger rows; symbolic 0 hash,
  // 3 hash + bucket counting sort.  MODE & 8: the paper's grouped local load balancing (ablation).
  extern __shared__ __align__(16) unsigned char smem[];
  const int lane = lane_id();
  constexpr int M = MODE & 7;
  constexpr int kRegion = wr_region_bytes(PASS, M);
  unsigned char* region = smem + warp_id() * kRegion;
  uint32_t* rk = reinterpret_cast<uint32_t*>(region);
  V* rv = reinterpret_cast<V*>(region + (PASS == 0 ? 0u : wr_num_val_offset<V>(kRegion)));
  const uint32_t cap = PASS == 0 ? wr_sym_cap() : wr_num_cap<V>(kRegion);
  const int64_t esc_cap = esc_capacity<V>(PASS, kRegion);
  const int64_t n = p.n_entries;
  constexpr bool kRange = (PASS == 1 && M != 1) || M == 3;
  // row metadata, one field per lane: 0 A_rp[r], 1 A_rp[r+1], 2 prods[r] / C_rp[r], 3 C_rp[r+1],
  // 4 colmin[r], 5 colmax[r], 6 prods[r] (numeric) (one round trip instead of seven dependent loads)
  auto fetch = [&](int64_t e, int32_t& row, int64_t& mv) {
    row = -1;
    mv = 0;
    if (e < n) {
      row = p.rows ? p.rows[e] : (int32_t)e;
      if (lane == 0) mv = p.A_rp[row];
      else if (lane == 1) mv = p.A_rp[row + 1];
      else if (lane == 2) mv = PASS == 0 ? p.prods[row] : p.C_rp[row];
      else if (lane == 3 && PASS == 1) mv = p.C_rp[row + 1];
      else if (lane == 4 && kRange) mv = p.colmin[row];   // column range: ordered maps only
      else if (lane == 5 && kRange) mv = p.colmax[row];
      else if (lane == 6 && PASS == 1 && M != 1) mv = p.prods[row];
      else if (lane == 7 && (MODE & 8) && p.fixed_g < 0) mv = p.maxlen[row];   // dynamic g (paper's local LB)
    }
  };
  // rows are claimed kWarpRowChunk at a time (one same-address atomic per chunk: per-row
  // claims serialise at ~2-3 G/s in L2), the next chunk one chunk ahead
  unsigned long long e = 0, cend = 0, nxt = 0;
  if (lane == 0) {
    e = atomicAdd(counter, (unsigned long long)kWarpRowChunk);
    nxt = atomicAdd(counter, (unsigned long long)kWarpRowChunk);
  }
  e = __shfl_sync(0xffffffffu, e, 0);
  nxt = __shfl_sync(0xffffffffu, nxt, 0);
  cend = e + kWarpRowChunk;
  // the first batch of a row (A col/val -> B row start/length, two dependent round trips) is
  // loaded one row ahead, the metadata two rows ahead: a row's only exposed latency is its
  // B gathers
  auto fetch_batch = [&](int64_t a0, int alen, PreBatch<V>& bt) {
    bt.valid = true;
    bt.bst = 0;
    bt.blen = 0;
    bt.a = V(0);
    if (lane < alen) {
      const int32_t kc = p.A_col[a0 + lane];
      if (PASS == 1) bt.a = ldv(p.A_val + a0 + lane);
      bt.bst = p.B_rp[kc];
      bt.blen = (int)(p.B_rp[kc + 1] - bt.bst);
    }
  };
  auto next_index = [&](unsigned long long x) {
    unsigned long long y = x + 1;
    if (y == cend) {                                      // chunk done: move to the claimed one
      y = nxt;
      cend = nxt + kWarpRowChunk;
      if (lane == 0 && (int64_t)nxt < n) nxt = atomicAdd(counter, (unsigned long long)kWarpRowChunk);
      nxt = __shfl_sync(0xffffffffu, nxt, 0);
    }
    return y;
  };
  int32_t row;
  int64_t mv;
  fetch((int64_t)e, row, mv);
  PreBatch<V> bt;
  {
    const int64_t a0 = __shfl_sync(0xffffffffu, mv, 0);
    if (PASS == 1) fetch_batch(a0, (int)(__shfl_sync(0xffffffffu, mv, 1) - a0), bt);   // symbolic rows: no pre-batch
  }
  unsigned long long en = next_index(e);
  int32_t rown;
  int64_t mvn;
  fetch((int64_t)en, rown, mvn);
  while ((int64_t)e < n) {
    const int64_t a0 = __shfl_sync(0xffffffffu, mv, 0);
    const int alen = (int)(__shfl_sync(0xffffffffu, mv, 1) - a0);
    const int64_t m2 = __shfl_sync(0xffffffffu, mv, 2);
    const int64_t m3 = __shfl_sync(0xffffffffu, mv, 3);
    const int32_t cmn = (int32_t)__shfl_sync(0xffffffffu, mv, 4);
    const int32_t cmx = (int32_t)__shfl_sync(0xffffffffu, mv, 5);
    const int64_t mv_prev6 = mv;
    const int32_t cur = row;
    const int64_t need = PASS == 0 ? m2 : m3 - m2;       // products (symbolic) / exact nnz (numeric)
    // region: symbolic 4x products (<= 25% load below the cap), numeric 2.5x entries (<= 40% load), 32-slot multiples
    const uint64_t want = PASS == 0 ? (uint64_t)need * SPECK_SYM_REGION_X2 / 2 : (uint64_t)need * 5 / 2;
    const uint64_t w32 = (want + 31) & ~(uint64_t)31;
    const uint32_t S = (uint32_t)(w32 < 64 ? 64 : (w32 > cap ? cap : w32));
    const PreBatch<V> bcur = bt;
    // pipeline: next row's batch, the row after next's metadata
    const unsigned long long enn = (int64_t)en < n ? next_index(en) : en;
    if (PASS == 1 && (int64_t)en < n) {
      const int64_t a0n = __shfl_sync(0xffffffffu, mvn, 0);
      fetch_batch(a0n, (int)(__shfl_sync(0xffffffffu, mvn, 1) - a0n), bt);
    }
    row = rown;
    mv = mvn;
    fetch((int64_t)enn, rown, mvn);
    int c = -1;
    if (M != 1 && (PASS == 1 || M == 3) && !(MODE & 8)) {
      // rows whose products are (almost) all distinct columns: counting sort on column buckets
      // (esc_kernels.cuh); -1 = uneven buckets, the hash map below takes the row
      const int64_t np = PASS == 0 ? need : __shfl_sync(0xffffffffu, mv_prev6, 6);
      if (p.esc >= (PASS == 0 ? 2 : 1) && np > 0 && np <= esc_cap && (PASS == 0 || np * 100 <= (int64_t)kEscRatioPct * need))
        c = (kEscStaged && np <= esc_staged_capacity<V>(PASS, kRegion))
                ? esc_row_staged<1, PASS, V>(p, region, kRegion, 0, a0, alen, (int)np, (int)need, cmn, cmx, m2, nullptr, &bcur)
                : esc_row<1, PASS, V>(p, region, kRegion, 0, a0, alen, (int)np, (int)need, cmn, cmx, m2, nullptr, nullptr, 0);
    }
    if (c < 0)
      c = warp_row<PASS, V, MODE>(p, rk, rv, S, a0, alen, cmn, cmx, (int32_t)(m3 - m2), m2, &bcur,
                                  PASS == 0 ? need : __shfl_sync(0xffffffffu, mv_prev6, 6),
                                  __shfl_sync(0xffffffffu, mv_prev6, 7));
    if (PASS == 0 && lane == 0) p.cnt[cur] = c;
    e = en;
    en = enn;
  }
}

// -----------------------------------------------------------------------------------
// Direct referencing: a row of A with a single NZ a·B_k — C_i = a·B_k in
// B's (sorted) order, no accumulator.  GD lanes per row, grid-stride over the bin.
// -----------------------------------------------------------------------------------
template <typename V, int GD>
__global__ void __launch_bounds__(256) k_direct(const int32_t* __restrict__ rows, int64_t n_rows,
                                                const int64_t* __restrict__ A_rp, const int32_t* __restrict__ A_col,
                                                const V* __restrict__ A_val, const int64_t* __restrict__ B_rp,
                                                const int32_t* __restrict__ B_col, const V* __restrict__ B_val,
                                                const int64_t* __restrict__ C_rp, int32_t* __restrict__ C_col,
                                                V* __restrict__ C_val, unsigned long long* paths) {
  const int sub = threadIdx.x % GD;
  const int64_t stride = (int64_t)gridDim.x * (blockDim.x / GD);
  for (int64_t e = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) / GD; e < n_rows; e += stride) {
    const int32_t row = rows[e];
    const int64_t q = A_rp[row];
    const int32_t kc = A_col[q];
    const V a = A_val[q];
    const int64_t b0 = B_rp[kc], len = B_rp[kc + 1] - b0;
    const int64_t c0 = C_rp[row];
    if (sub == 0) count_path(paths, SPECK_PATH_NUM_DIRECT);
    for (int64_t j = sub; j < len; j += GD) {
      C_col[c0 + j] = B_col[b0 + j];
      C_val[c0 + j] = a * B_val[b0 + j];
    }
  }
}

}  // namespace speck
