// det_kernels.cuh — deterministic-value mode (SPECK_OPT_DETERMINISTIC).
//
// Shared-memory atomics from several warps make the order of the additions into an entry of C
// run dependent (the paper's accumulators; reading R2).  In
// deterministic mode every row of C is accumulated by ONE warp that enumerates the row's
// products in the order of eq. (1)'s sum (row i of A in order, then each B_k in order) and adds
// the products of one column in that order: equal columns of a warp step are added in lane
// order ("rounds"), steps in order.  Each product is rounded before it is added
// (acc <- fl(acc + fl(a*b)), __fadd_rn: no contraction), so C_ij is bit-identical across runs
// and equal to a sequential sum in the inputs' precision (reading R15).
//   - rows that fit the 7 KB warp region: k_warp_rows (unchanged, already one warp per row);
//   - larger rows: k_det_rows below — one warp per row with a 54 KB region: the ordered hash map
//     of warp_row when the row fits it, else sequential dense column windows (each referenced B
//     row resumes where the previous window stopped) with the same in-order adds.
#pragma once

#include "spgemm_kernels.cuh"

namespace speck {

constexpr int kDetWarps = 4;                                   // warps (rows) per CTA
constexpr int kDetRegion = 55296;                              // bytes per warp (4 x 54 KB = 216 KB per CTA)

template <typename V>
__host__ __device__ inline uint32_t det_map_cap() { return (uint32_t)((kDetRegion - 16) / (4 + (int)sizeof(V))); }
template <typename V>
__host__ __device__ inline int64_t det_window() {              // columns of one dense window (values + flag bits)
  return ((int64_t)(kDetRegion - 16) * 8 / (8 * (int64_t)sizeof(V) + 1)) & ~int64_t(31);
}

// Warp-level sorted write-out of a dense window (flag bits + values) at C[out, ...).
template <typename V>
__device__ __forceinline__ int64_t warp_dense_emit(const uint32_t* bits, const V* dv, int nwords, uint32_t wlo, int64_t out,
                                                   int32_t* __restrict__ C_col, V* __restrict__ C_val) {
  const int lane = lane_id();
  int64_t base = out;
  for (int c0 = 0; c0 < nwords; c0 += 32) {
    const uint32_t word = c0 + lane < nwords ? bits[c0 + lane] : 0u;
    const int pc = __popc(word);
    const int incl = warp_incl_scan(pc);
    const int excl = incl - pc;
    for (int j = 0; j < 32; ++j) {
      const uint32_t wj = __shfl_sync(0xffffffffu, word, j);
      if (!wj) continue;
      const int oj = __shfl_sync(0xffffffffu, excl, j);
      if ((wj >> lane) & 1u) {
        const int64_t o = base + oj + __popc(wj & ((1u << lane) - 1u));
        const uint32_t ci = (uint32_t)(c0 + j) * 32u + (uint32_t)lane;
        C_col[o] = (int32_t)(wlo + ci);
        C_val[o] = dv[ci];
      }
    }
    base += __shfl_sync(0xffffffffu, incl, 31);
  }
  return base - out;
}

template <typename V>
__global__ void __launch_bounds__(32 * kDetWarps, 1) k_det_rows(const __grid_constant__ SpgemmArgs<V> p,
                                                                 unsigned long long* __restrict__ counter,
                                                                 int32_t* __restrict__ scratch) {
  extern __shared__ __align__(16) unsigned char smem[];
  const int lane = lane_id();
  unsigned char* region = smem + (size_t)warp_id() * kDetRegion;
  const uint32_t cap = det_map_cap<V>();
  const int64_t W = det_window<V>();
  // resume offsets of this warp (two buffers of max nnz(A_i)), one slot per resident warp
  const int64_t gw = (int64_t)blockIdx.x * kDetWarps + warp_id();
  int32_t* res = scratch + gw * p.resume_stride;
  int32_t* res_next = res + p.resume_stride / 2;
  while (true) {
    unsigned long long e = 0;
    if (lane == 0) e = atomicAdd(counter, 1ull);
    e = __shfl_sync(0xffffffffu, e, 0);
    if ((int64_t)e >= p.n_entries) break;
    const int32_t row = p.rows[e];
    const int64_t a0 = p.A_rp[row];
    const int alen = (int)(p.A_rp[row + 1] - a0);
    const int64_t cb = p.C_rp[row];
    const int32_t cnt = (int32_t)(p.C_rp[row + 1] - cb);
    const int32_t cmn = p.colmin[row], cmx = p.colmax[row];
    if (lane == 0) count_path(p.paths, SPECK_PATH_NUM_DET);
    if ((uint32_t)cnt * 2u <= cap) {
      // the ordered hash map of the warp-row path, sized to the row (rounds: in-order adds)
      uint32_t* rk = reinterpret_cast<uint32_t*>(region);
      V* rv = reinterpret_cast<V*>(region + (((size_t)cap * 4 + 15) & ~(size_t)15));
      const uint64_t w32 = ((uint64_t)cnt * 5 / 2 + 31) & ~(uint64_t)31;
      const uint32_t S = (uint32_t)(w32 < 64 ? 64 : (w32 > cap ? cap : w32));
      warp_row<1, V, 0>(p, rk, rv, S, a0, alen, cmn, cmx, cnt, cb);
      continue;
    }
    // dense windows over [colmin, colmax], products of every window in the order of eq. (1)
    const int64_t nwords_max = W / 32;
    uint32_t* bits = reinterpret_cast<uint32_t*>(region);
    V* dv = reinterpret_cast<V*>(region + ((nwords_max * 4 + 15) & ~(int64_t)15));
    for (int f = lane; f < alen; f += 32) res[f] = 0;
    __syncwarp();
    int64_t out = cb;
    for (int64_t wlo = cmn; wlo <= cmx; wlo += W) {
      const int64_t whi = min(wlo + W, (int64_t)cmx + 1);
      const int nwords = (int)((whi - wlo + 31) / 32);
      for (int i = lane; i < nwords; i += 32) bits[i] = 0u;
      for (int64_t i = lane; i < whi - wlo; i += 32) dv[i] = V(0);
      __syncwarp();
      expand_row<1, V, false, false, 1>(p, a0, alen, 0, 1, [&](uint32_t col, V v, bool act) {
        const uint32_t peers = __match_any_sync(0xffffffffu, col);
        const uint32_t c = col - (uint32_t)wlo;
        const int rank = __popc(peers & ((1u << lane) - 1u));
        const int maxg = (int)__reduce_max_sync(0xffffffffu, (unsigned)__popc(peers));
        if (act && rank == 0) atomicOr(&bits[c >> 5], 1u << (c & 31));
        for (int t = 0; t < maxg; ++t) {
          if (act && rank == t) dv[c] = add_rn(dv[c], v);
          __syncwarp();
        }
      }, WindowRange{res, res_next, p.B_col, (uint32_t)whi});
      __syncwarp();
      { int32_t* t_ = res; res = res_next; res_next = t_; }
      out += warp_dense_emit<V>(bits, dv, nwords, (uint32_t)wlo, out, p.C_col, p.C_val);
      __syncwarp();
    }
  }
}

}  // namespace speck
