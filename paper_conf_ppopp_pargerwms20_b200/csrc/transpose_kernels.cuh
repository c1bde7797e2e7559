// transpose_kernels.cuh — device CSR transpose.
//
// The paper multiplies rectangular matrices as A·Aᵀ "with Aᵀ precomputed", and
// the AMG Galerkin product needs R = Pᵀ.  T = Aᵀ in sorted CSR:
//   1. count the entries of every column of A (global atomics)          -> T row lengths
//   2. exclusive scan                                                    -> T row offsets
//   3. scatter every (row r, value) of column c to a slot of T row c (atomic cursor)
//   4. sort every row of T by its column index (the source row r; unique per row):
//        <= 32 entries: one warp, bitonic network over shuffles;
//        <= kTrSmemSort entries: one CTA, bitonic sort in shared memory;
//        longer rows: 16K-entry tiles sorted in shared memory, then merge rounds (merge path
//        per CTA) in global memory with a scratch buffer.
// The result is unique (T's rows sorted, values carried bit for bit), so it is compared
// bit-exactly with a host transpose.
#pragma once

#include "spgemm_kernels.cuh"

namespace speck {

constexpr int kTrThreads = 256;
constexpr int kTrSmemSort = 8192;   // entries a CTA sorts in shared memory (keys + fp64 values: 96 KB)

__global__ void __launch_bounds__(kTrThreads) k_tr_count(const int32_t* __restrict__ col, int64_t nnz,
                                                         unsigned long long* __restrict__ cnt) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nnz; i += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(&cnt[col[i]], 1ull);
}

template <typename V>
__global__ void __launch_bounds__(kTrThreads) k_tr_scatter(const int64_t* __restrict__ rp, const int32_t* __restrict__ col,
                                                           const V* __restrict__ val, int64_t rows,
                                                           unsigned long long* __restrict__ cursor,
                                                           int32_t* __restrict__ tcol, V* __restrict__ tval) {
  // one warp per row of A, lanes over its entries
  const int lane = lane_id();
  const int64_t w0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t ws = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t r = w0; r < rows; r += ws) {
    const int64_t a = rp[r], b = rp[r + 1];
    for (int64_t i = a + lane; i < b; i += 32) {
      const int32_t c = col[i];
      const unsigned long long pos = atomicAdd(&cursor[c], 1ull);
      tcol[pos] = (int32_t)r;
      if (val) tval[pos] = val[i];
    }
  }
}

// Rows of T with <= 32 entries: one warp per row, bitonic network over the lanes (ascending key).
template <typename V>
__global__ void __launch_bounds__(kTrThreads) k_tr_sort_warp(const int64_t* __restrict__ trp, int64_t trows,
                                                             int32_t* __restrict__ tcol, V* __restrict__ tval) {
  const int lane = lane_id();
  const int64_t w0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t ws = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t r = w0; r < trows; r += ws) {
    const int64_t a = trp[r], n = trp[r + 1] - a;
    if (n <= 1 || n > 32) continue;
    uint32_t k = lane < n ? (uint32_t)tcol[a + lane] : 0xffffffffu;
    V v = (lane < n && tval) ? tval[a + lane] : V(0);
#pragma unroll
    for (int size = 2; size <= 32; size <<= 1) {
#pragma unroll
      for (int stride = size >> 1; stride > 0; stride >>= 1) {
        const uint32_t ok = __shfl_xor_sync(0xffffffffu, k, stride);
        const V ov = __shfl_xor_sync(0xffffffffu, v, stride);
        const bool up = ((lane & size) == 0);          // ascending half of the bitonic step
        const bool lower = (lane & stride) == 0;
        const bool take_min = (up == lower);
        const bool swap = take_min ? (ok < k) : (ok > k);
        if (swap) { k = ok; v = ov; }
      }
    }
    if (lane < n) {
      tcol[a + lane] = (int32_t)k;
      if (tval) tval[a + lane] = v;
    }
  }
}

// Rows of T with 33 .. kTrSmemSort entries (list `rows`): one CTA each, bitonic sort in shared
// memory.  Rows longer than that: the CTA sorts tile `tile` (kTrSmemSort entries) of the row.
template <typename V>
__global__ void __launch_bounds__(1024) k_tr_sort_block(const int64_t* __restrict__ trp, const int32_t* __restrict__ rows,
                                                        const int64_t* __restrict__ tile_first, int64_t nrows,
                                                        int32_t* __restrict__ tcol, V* __restrict__ tval) {
  extern __shared__ __align__(16) unsigned char smem[];
  uint32_t* sk = reinterpret_cast<uint32_t*>(smem);
  V* sv = reinterpret_cast<V*>(smem + kTrSmemSort * 4);
  // block b -> (row, tile) via the per-row first-tile offsets (binary search)
  int64_t lo = 0, hi = nrows;
  while (hi - lo > 1) {
    const int64_t mid = (lo + hi) >> 1;
    if (tile_first[mid] <= (int64_t)blockIdx.x) lo = mid; else hi = mid;
  }
  const int32_t r = rows[lo];
  const int64_t tile = (int64_t)blockIdx.x - tile_first[lo];
  const int64_t a = trp[r] + tile * kTrSmemSort;
  const int n = (int)min((int64_t)kTrSmemSort, trp[r + 1] - a);
  for (int i = threadIdx.x; i < n; i += blockDim.x) {
    sk[i] = (uint32_t)tcol[a + i];
    sv[i] = tval ? tval[a + i] : V(0);
  }
  __syncthreads();
  smem_bitonic_sort<1024, V>(sk, sv, n);
  __syncthreads();
  for (int i = threadIdx.x; i < n; i += blockDim.x) {
    tcol[a + i] = (int32_t)sk[i];
    if (tval) tval[a + i] = sv[i];
  }
}

// One merge round over the long rows: runs of length L (sorted) are merged pairwise from src
// into dst.  Work item = (row, pair, part): every CTA merges kTrSmemSort outputs of one pair,
// its start found by merge-path binary search; each thread then merges its slice sequentially.
template <typename V>
__global__ void __launch_bounds__(256) k_tr_merge(const int64_t* __restrict__ trp, const int32_t* __restrict__ rows,
                                                  const int64_t* __restrict__ part_first, int64_t nrows, int64_t L,
                                                  const int32_t* __restrict__ scol, const V* __restrict__ sval,
                                                  int32_t* __restrict__ dcol, V* __restrict__ dval) {
  int64_t lo = 0, hi = nrows;
  while (hi - lo > 1) {
    const int64_t mid = (lo + hi) >> 1;
    if (part_first[mid] <= (int64_t)blockIdx.x) lo = mid; else hi = mid;
  }
  const int32_t r = rows[lo];
  const int64_t base = trp[r], n = trp[r + 1] - base;
  const int64_t part = (int64_t)blockIdx.x - part_first[lo];
  const int64_t out0 = part * kTrSmemSort;             // position in the row
  const int64_t pair0 = out0 / (2 * L) * (2 * L);      // the pair this part belongs to
  const int64_t a0 = pair0, a1 = min(pair0 + L, n), b0 = a1, b1 = min(pair0 + 2 * L, n);
  const int64_t out1 = min(out0 + kTrSmemSort, min(pair0 + 2 * L, n));
  // per thread: a slice [d0, d1) of the part's output diagonals
  const int64_t per = (out1 - out0 + blockDim.x - 1) / blockDim.x;
  const int64_t d0 = min(out1, out0 + (int64_t)threadIdx.x * per), d1 = min(out1, d0 + per);
  if (d0 >= d1) return;
  // merge path: i elements from A, d - i from B, for diagonal d (relative to pair0)
  auto split = [&](int64_t d) {
    const int64_t dd = d - pair0;
    int64_t l = max((int64_t)0, dd - (b1 - b0)), h = min(dd, a1 - a0);
    while (l < h) {
      const int64_t i = (l + h) >> 1;
      // take more from A while A[i] <= B[dd - i - 1] (keys are unique: < suffices)
      if ((uint32_t)scol[base + a0 + i] < (uint32_t)scol[base + b0 + dd - i - 1]) l = i + 1; else h = i;
    }
    return l;
  };
  int64_t i = split(d0), j = (d0 - pair0) - i;
  for (int64_t d = d0; d < d1; ++d) {
    const bool takeA = i < a1 - a0 && (j >= b1 - b0 || (uint32_t)scol[base + a0 + i] < (uint32_t)scol[base + b0 + j]);
    const int64_t src = takeA ? a0 + i : b0 + j;
    dcol[base + d] = scol[base + src];
    if (sval) dval[base + d] = sval[base + src];
    if (takeA) ++i; else ++j;
  }
}

// rows of T longer than `lo` entries -> list (any order) with their kTrSmemSort-tile counts
__global__ void k_tr_list(const int64_t* __restrict__ trp, int64_t trows, int64_t lo, int32_t* __restrict__ list,
                          int64_t* __restrict__ tiles, unsigned long long* __restrict__ n) {
  for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < trows; r += (int64_t)gridDim.x * blockDim.x) {
    const int64_t len = trp[r + 1] - trp[r];
    if (len > lo) {
      const unsigned long long i = atomicAdd(n, 1ull);
      list[i] = (int32_t)r;
      tiles[i] = (len + kTrSmemSort - 1) / kTrSmemSort;
    }
  }
}

}  // namespace speck
