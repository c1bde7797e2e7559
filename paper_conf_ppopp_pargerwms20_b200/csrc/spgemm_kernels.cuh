// spgemm_kernels.cuh — symbolic and numeric SpGEMM kernels (§4.3).
//
// One kernel template per configuration of the ladder (speck_internal.cuh) and pass.  A CTA
// takes a group of <= 32 consecutive entries of its bin (or of the identity row list when
// the global load balancer is off), splits the group into blocks with the
// block merge of Alg. 2 (merged small-row bin only), and for each block:
//   1. picks the accumulator: hash map, dense array; direct
//      rows have their own kernel below;
//   2. picks the local-load-balancer group size g and lets k = T/g groups of
//      g threads stream the referenced rows of B (coalesced within a group);
//   3. symbolic: counts the distinct columns per row;
//      numeric: accumulates values, then compacts and SORTS each row in shared memory
//      before writing it at its C row offset.
//
// B200 differences from the paper's Titan V design:
//   * merged rows use per-row regions of the map instead of a 5-bit row + 27-bit column
//     compound key, so blocks of up to 32 rows work for any column count;
//   * every hash row is sorted in shared memory (rank counting for short rows, a bitonic
//     network for long ones) — 227 KB per CTA makes a global radix-sort pass unnecessary;
//   * dense windows of rows needing several windows keep resume positions per referenced
//     B row in a per-SM global scratch slot.
#pragma once

#include "speck_internal.cuh"

namespace speck {

constexpr int kSmallSeg = 64;   // rows with <= this many C entries are ranked, not sorted

struct BlockMeta {
  int32_t row[kMaxGroupRows];
  int64_t astart[kMaxGroupRows];
  int64_t aoff[kMaxGroupRows + 1];   // prefix of nnz(A_r) over the block
  int64_t cbase[kMaxGroupRows];      // numeric: C_rp[row]
  int32_t cseg[kMaxGroupRows + 1];   // numeric: prefix of cnt_r over the block
  uint32_t rbase[kMaxGroupRows + 1]; // hash region start of each row
  int32_t rcnt[kMaxGroupRows];       // symbolic: distinct columns per row
  uint32_t starts;
  int nr, g, dense;
  int64_t nnzA, prods, maxlen, cnt;
  int32_t colmin, colmax;
  int64_t scan_part[33];
  int64_t total;
};

template <typename V>
__device__ __forceinline__ V ldv(const V* p) { return __ldg(p); }

// Linear probing from slot s (Fig. 4): find `key` or claim an empty slot for
// it with a CAS; returns the slot, *is_new tells whether this thread inserted the key.
__device__ __forceinline__ uint32_t probe_insert(uint32_t* keys, uint32_t S, uint32_t s, uint32_t key, bool* is_new) {
  while (true) {
    const uint32_t k = keys[s];
    if (k == key) { *is_new = false; return s; }
    if (k == kEmptyKey) {
      const uint32_t old = atomicCAS(&keys[s], kEmptyKey, key);
      if (old == kEmptyKey) { *is_new = true; return s; }
      if (old == key) { *is_new = false; return s; }
    }
    s = (s + 1 == S) ? 0u : s + 1;
  }
}

// symbolic insert: true if the key was new
__device__ __forceinline__ bool hash_insert_key(uint32_t* keys, uint32_t S, uint32_t col) {
  bool is_new;
  probe_insert(keys, S, hash_slot(col, S), col, &is_new);
  return is_new;
}

// numeric insert-or-accumulate
template <typename V>
__device__ __forceinline__ void hash_accumulate(uint32_t* keys, V* vals, uint32_t S, uint32_t col, V v) {
  bool is_new;
  const uint32_t s = probe_insert(keys, S, hash_slot(col, S), col, &is_new);
  atomicAdd(&vals[s], v);
}

// Bitonic sort of (keys, vals)[0, n) ascending in shared memory, any n: the "flip"
// formulation keeps all sub-sorts ascending, so comparisons with a partner index >= n
// (a virtual +inf) are no-ops and can be skipped.
template <int T, typename V>
__device__ void smem_bitonic_sort(uint32_t* keys, V* vals, int n) {
  if (n <= 1) return;
  int P = 1;
  while (P < n) P <<= 1;
  for (int k = 2; k <= P; k <<= 1) {
    const int hk = k >> 1;
    for (int t = threadIdx.x; t < P / 2; t += T) {
      const int blk = t / hk, off = t - blk * hk;
      const int i = blk * k + off, j = blk * k + k - 1 - off;
      if (j < n) {
        const uint32_t a = keys[i], b = keys[j];
        if (a > b) {
          keys[i] = b; keys[j] = a;
          const V va = vals[i]; vals[i] = vals[j]; vals[j] = va;
        }
      }
    }
    __syncthreads();
    for (int d = k >> 2; d >= 1; d >>= 1) {
      for (int t = threadIdx.x; t < P / 2; t += T) {
        const int blk = t / d, off = t - blk * d;
        const int i = blk * 2 * d + off, j = i + d;
        if (j < n) {
          const uint32_t a = keys[i], b = keys[j];
          if (a > b) {
            keys[i] = b; keys[j] = a;
            const V va = vals[i]; vals[i] = vals[j]; vals[j] = va;
          }
        }
      }
      __syncthreads();
    }
  }
}

// acquire a per-SM resume scratch slot (largest configuration: one CTA per SM)
__device__ __forceinline__ unsigned smid() {
  unsigned r;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(r));
  return r;
}

// -----------------------------------------------------------------------------------
// The per-configuration kernel.  PASS 0 = symbolic, 1 = numeric.
// -----------------------------------------------------------------------------------
template <int CFG, int PASS, typename V>
__global__ void __launch_bounds__(kCfgThreads[CFG], 1024 / kCfgThreads[CFG]) k_spgemm(SpgemmArgs<V> p) {
  constexpr int T = kCfgThreads[CFG];
  
  extern __shared__ __align__(16) unsigned char smem[];
  __shared__ BlockMeta bm;
  const int tid = threadIdx.x;

  const int64_t e0 = (int64_t)blockIdx.x * p.group_rows;
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
      if (l < nr) rsz = nr == 1 ? cap : (need_tot > 0 ? (uint32_t)((uint64_t)cap * (uint64_t)need / (uint64_t)need_tot) : 0u);
      const uint32_t rinc = warp_incl_scan(rsz);
      if (l < nr) {
        bm.astart[l] = a0;
        bm.aoff[l + 1] = ainc;
        bm.cbase[l] = c0;
        bm.cseg[l + 1] = (int32_t)cinc;
        bm.rbase[l + 1] = rinc;
        bm.rcnt[l] = 0;
      }
      if (l == 0) {
        bm.aoff[0] = 0; bm.cseg[0] = 0; bm.rbase[0] = 0;
        bm.nr = nr;
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
            else if ((uint64_t)tot_p > (uint64_t)cap) dense = 1;                       // cannot hash: P:1112-1113
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
        // ---- local load balancer ----
        int g = p.fixed_g > 0 ? min(p.fixed_g, T) : local_group_size(T, tot_a, tot_p, mlx);
        if (dense) {
          const int64_t W0 = PASS == 0 ? sym_dense_window(CFG) : num_dense_window<V>(CFG);
          const int64_t W = (p.dense_window_cap > 0 && p.dense_window_cap < W0) ? p.dense_window_cap : W0;
          if (range > W && g > 32) g = 32;  // multi-window rows: a group must fit a warp
        }
        bm.g = g;
      }
    }
    __syncthreads();
    const int g = bm.g;
    const int gid = tid / g, gl = tid - gid * g, k = T / g;
    const int64_t nnzA = bm.nnzA;

    if (!bm.dense) {
      // ============================ HASH ACCUMULATOR ==============================
      uint32_t* keys = reinterpret_cast<uint32_t*>(smem);
      const uint32_t capt = bm.rbase[nr];
      V* vals = reinterpret_cast<V*>(smem + (PASS == 0 ? 0u : num_val_offset<V>(CFG)));
      for (uint32_t i = tid; i < capt; i += T) {
        keys[i] = kEmptyKey;
        if (PASS == 1) vals[i] = V(0);
      }
      __syncthreads();
      int r = 0;
      for (int64_t f = gid; f < nnzA; f += k) {
        while (f >= bm.aoff[r + 1]) ++r;
        const int64_t q = bm.astart[r] + (f - bm.aoff[r]);
        const int32_t kc = p.A_col[q];
        const int64_t j0 = p.B_rp[kc], j1 = p.B_rp[kc + 1];
        const uint32_t rb = bm.rbase[r], S = bm.rbase[r + 1] - rb;
        if (PASS == 0) {
          int newc = 0;
          for (int64_t j = j0 + gl; j < j1; j += g) newc += hash_insert_key(keys + rb, S, (uint32_t)p.B_col[j]);
          if (newc) atomicAdd(&bm.rcnt[r], newc);
        } else {
          const V a = ldv(p.A_val + q);
          for (int64_t j = j0 + gl; j < j1; j += g)
            hash_accumulate<V>(keys + rb, vals + rb, S, (uint32_t)p.B_col[j], a * ldv(p.B_val + j));
        }
      }
      __syncthreads();
      if (PASS == 0) {
        if (tid < nr) p.cnt[bm.row[b0 + tid]] = bm.rcnt[tid];
      } else {
        // ---- compaction (order preserving -> row regions stay in row order) ----
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
        // ---- short rows: rank counting, written straight to C ----
        const int ncnt = (int)bm.cnt;
        {
          int rr = 0;
          for (int i = tid; i < ncnt; i += T) {
            while (i >= bm.cseg[rr + 1]) ++rr;
            const int s0 = bm.cseg[rr], s1 = bm.cseg[rr + 1];
            if (s1 - s0 > kSmallSeg) continue;
            const uint32_t key = keys[i];
            int rank = 0;
            for (int j = s0; j < s1; ++j) rank += keys[j] < key;
            const int64_t o = bm.cbase[rr] + rank;
            p.C_col[o] = (int32_t)key;
            p.C_val[o] = vals[i];
          }
        }
        // ---- long rows: bitonic sort in shared memory, then coalesced write ----
        for (int rr = 0; rr < nr; ++rr) {
          const int s0 = bm.cseg[rr], s1 = bm.cseg[rr + 1];
          if (s1 - s0 <= kSmallSeg) continue;
          __syncthreads();
          smem_bitonic_sort<T, V>(keys + s0, vals + s0, s1 - s0);
          const int64_t o = bm.cbase[rr];
          for (int i = tid; i < s1 - s0; i += T) {
            p.C_col[o + i] = (int32_t)keys[s0 + i];
            p.C_val[o + i] = vals[s0 + i];
          }
        }
      }
    } else {
      // ============================ DENSE ACCUMULATOR =============================
      // single row; windows over [colmin, colmax] (Fig. 5)
      const int32_t row = bm.row[b0];
      const int64_t lo = bm.colmin, hi = bm.colmax;
      const int64_t W0 = PASS == 0 ? sym_dense_window(CFG) : num_dense_window<V>(CFG);
      const int64_t W = (p.dense_window_cap > 0 && p.dense_window_cap < W0) ? p.dense_window_cap : W0;
      const int64_t nwin = (hi - lo + 1 + W - 1) / W;
      const int64_t astart = bm.astart[0];
      uint32_t* bits = reinterpret_cast<uint32_t*>(smem);                       // W bits
      V* dvals = reinterpret_cast<V*>(smem + (PASS == 0 ? 0 : (((W + 31) / 32) * 4 + 15) / 16 * 16));
      int32_t* res = nullptr;
      if (nwin > 1) {
        res = p.resume + (int64_t)smid() * p.resume_stride;
        for (int64_t f = tid; f < nnzA; f += T) res[f] = 0;
      }
      const int nwords = (int)((W + 31) / 32);
      const uint32_t gmask = g >= 32 ? 0xffffffffu : (((1u << g) - 1u) << (lane_id() & ~(g - 1)));
      int64_t out = PASS == 1 ? bm.cbase[0] : 0;
      int64_t total = 0;
      if (tid == 0 && PASS == 1 && p.n_dense_rows) atomicAdd(p.n_dense_rows, 1ull);
      for (int64_t w = 0; w < nwin; ++w) {
        const int64_t wlo = lo + w * W, whi = min(wlo + W, hi + 1);
        for (int i = tid; i < nwords; i += T) bits[i] = 0u;
        if (PASS == 1)
          for (int64_t i = tid; i < W; i += T) dvals[i] = V(0);
        __syncthreads();
        for (int64_t f = gid; f < nnzA; f += k) {
          const int64_t q = astart + f;
          const int32_t kc = p.A_col[q];
          const int64_t j0 = p.B_rp[kc], j1 = p.B_rp[kc + 1];
          V a = V(0);
          if (PASS == 1) a = ldv(p.A_val + q);
          if (nwin == 1) {
            for (int64_t j = j0 + gl; j < j1; j += g) {
              const uint32_t c = (uint32_t)(p.B_col[j] - wlo);
              atomicOr(&bits[c >> 5], 1u << (c & 31));
              if (PASS == 1) atomicAdd(&dvals[c], a * ldv(p.B_val + j));
            }
          } else {
            int64_t pos = j0 + res[f];
            while (pos < j1) {
              const int64_t j = pos + gl;
              const int32_t cj = j < j1 ? p.B_col[j] : 0x7fffffff;
              const bool in = cj < whi;
              if (in) {
                const uint32_t c = (uint32_t)(cj - wlo);
                atomicOr(&bits[c >> 5], 1u << (c & 31));
                if (PASS == 1) atomicAdd(&dvals[c], a * ldv(p.B_val + j));
              }
              const uint32_t bal = __ballot_sync(gmask, in);
              const int took = __popc(bal);
              pos += took;
              if (took < g) break;
            }
            if (gl == 0) res[f] = (int32_t)(pos - j0);
          }
        }
        __syncthreads();
        // ---- window epilogue: count (symbolic) / compact in column order (numeric) ----
        int64_t wtot = 0;
        for (int base = 0; base < nwords; base += T) {
          const int wi = base + tid;
          const uint32_t word = wi < nwords ? bits[wi] : 0u;
          const int64_t pc = __popc(word);
          int64_t tot;
          const int64_t pre = block_excl_scan<T>(pc, bm.scan_part, &tot);
          if (PASS == 1 && word) {
            uint32_t wd = word;
            int64_t o = out + wtot + pre;
            while (wd) {
              const int b = __ffs(wd) - 1;
              wd &= wd - 1;
              const int64_t ci = (int64_t)wi * 32 + b;
              p.C_col[o] = (int32_t)(wlo + ci);
              p.C_val[o] = dvals[ci];
              ++o;
            }
          }
          wtot += tot;
        }
        out += wtot;
        total += wtot;
        __syncthreads();
      }
      if (PASS == 0 && tid == 0) p.cnt[row] = total;
    }
    __syncthreads();
    b0 = b1;
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
                                                V* __restrict__ C_val) {
  const int sub = threadIdx.x % GD;
  const int64_t stride = (int64_t)gridDim.x * (blockDim.x / GD);
  for (int64_t e = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) / GD; e < n_rows; e += stride) {
    const int32_t row = rows[e];
    const int64_t q = A_rp[row];
    const int32_t kc = A_col[q];
    const V a = A_val[q];
    const int64_t b0 = B_rp[kc], len = B_rp[kc + 1] - b0;
    const int64_t c0 = C_rp[row];
    for (int64_t j = sub; j < len; j += GD) {
      C_col[c0 + j] = B_col[b0 + j];
      C_val[c0 + j] = a * B_val[b0 + j];
    }
  }
}

}  // namespace speck
