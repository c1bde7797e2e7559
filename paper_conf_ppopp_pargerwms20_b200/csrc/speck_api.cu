// speck_api.cu — C ABI (include/speck.h), handle/workspace management and the host-side
// plan of the spECK pipeline (Fig. 2) on B200.
//
// Host decisions follow §5: the global load balancer runs for a step when
// m_max/m_avg and rows_C exceed the Table 2 thresholds, with the "*" set when
// the longest row needs one of the largest kernels; otherwise rows are processed in fixed
// groups of consecutive rows by one configuration big enough for the longest row
// (P:806-818).
#include <algorithm>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

#include "plan_kernels.cuh"
#include "spgemm_kernels.cuh"
#include "segment_kernels.cuh"
#include "transpose_kernels.cuh"
#include "det_kernels.cuh"

#define SPECK_VERSION "speck-b200 0.1.0 (sm_100a)"

namespace speck {

// Table 2 thresholds: {ratio, rows} for all kernels and for the largest ones.
// The paper's Titan V values were {39.2, 28000, 6.0, 5431} (symbolic) and {10.5, 23006, 1.3, 1238}
// (numeric).  B200 re-tuning (tools/ablation.py --lb-sweep,
// profiles/r02/r02r_ablation_c3_lbsweep.jsonl): on R-MAT families of scale 12-18 and uniform
// matrices, global balancing wins from ~64k rows on at any skew above ~4 (scale 18, a = .35,
// ratio 12: 8.33 ms off, 3.06 ms on — the Titan V threshold 39.2 left the symbolic step
// unbalanced, 3.66 ms) and loses below ~16k rows (scale 12: 0.26 off vs 0.74 on: the binning
// launches cost more than the imbalance), so both steps use {4.0, 32768}; rows that need the
// largest configuration still force it on (long rows are only handled by the binned path).
struct LbThresholds { double ratio, rows, ratio_big, rows_big; int big_from_cfg; };
static const LbThresholds kLbSym = {4.0, 32768, 4.0, 32768, 2};  // "*" = three largest (caption, reading R11)
static const LbThresholds kLbNum = {4.0, 32768, 4.0, 32768, 3};  // "*" = two largest

struct Buf {
  void* p = nullptr;
  size_t cap = 0;
};

constexpr int kMaxTimed = 64;      // timed launches per analyze/spgemm pair (SPECK_OPT_KERNEL_TIMING)
constexpr int kPinnedWords = 256;  // pinned readback words
// pinned readback layout (u64 words)
constexpr int kPinSymCat = 16;     // [CAT_COUNT + 1] bin offsets
constexpr int kPinBinSums = 64;    // [2][CAT_COUNT][3] per-bin sums (nnzA, products, nnzC)
// `small` device scratch layout (bytes)
constexpr int kSmallBinSums = 3072;   // unsigned long long [2][CAT_COUNT][3]
constexpr int kSmallRange = 3584;     // int64 [2 CAT_COUNT + 1] (speck_spgemm_rows)
constexpr int kPinRange = 128;        // pinned words for the same

}  // namespace speck

using namespace speck;

struct speck_handle_s {
  int device = 0;
  int num_sms = 148;
  int num_smid = 148;   // %nsmid: bound of %smid (sizes the per-SM resume scratch)
  std::string err;
  // options
  int64_t opt_lb_sym = -1, opt_lb_num = -1, opt_force_acc = 0, opt_dense_window = 0, opt_timing = 0, opt_validate = 0,
          opt_disable_direct = 0, opt_fixed_g = 0, opt_streams = 4, opt_esc = 1, opt_det = 0;
  // workspace
  Buf prods, maxlen, colmin, colmax, cnt, hist, hist_off, bins, stats, scan_status, resume, small, ana_long, binfo;
  unsigned long long* h_pinned = nullptr;  // pinned readback area (kPinnedWords x u64)
  cudaStream_t streams[kMaxStreams] = {};
  cudaEvent_t ev_fork = nullptr, ev_join[kMaxStreams] = {};
  cudaEvent_t ev_t[8] = {};
  // plan state of the last analyze
  bool analyzed = false;
  const int64_t* A_rp = nullptr; const int32_t* A_col = nullptr; int64_t A_rows = 0, A_cols = 0, A_nnz = 0;
  const int64_t* B_rp = nullptr; const int32_t* B_col = nullptr; int64_t B_rows = 0, B_cols = 0, B_nnz = 0;
  speck_dtype_t dtype = SPECK_F32;
  int64_t nnz_c = 0, max_cnt = 0, max_nnza = 0;
  int64_t num_cat_start[CAT_COUNT + 1] = {};
  speck_stats_t st = {};
  int lb_num = 0;
  bool numeric_pending = false;
  bool num_binned = false;   // numeric bins of the current analysis scattered (speck_spgemm_rows)
  int64_t launches = 0;  // kernels launched by this handle (cumulative)
  // long-row segments
  int64_t opt_segments = 1;
  int64_t opt_warp_rows = 1;
  int64_t opt_long_bitmap = 1;
  int64_t opt_bitmap_reuse = 1;
  bool bm_enabled = false;
  unsigned long long bm_pool_words = 0;
  Buf bm_pool, bm_off;
  bool seg_enabled = false;
  int seg_shift = 15, nchunks = 0;
  int64_t long_thr = INT64_MAX, n_cand = 0, n_segs = 0, cand_start = 0;
  Buf chunk_cnt, cand, nseg, seg_off, segs, chunks, tr_cnt, tr_list, tr_col, tr_val, det_scratch;
  // SPECK_OPT_KERNEL_TIMING: one event pair per launch of the current analyze/spgemm pair
  int64_t opt_ktime = 0, opt_paths = 0;
  cudaEvent_t kt_ev[2 * kMaxTimed] = {};
  int kt_n = 0;
  int32_t kt_id[kMaxTimed] = {}, kt_bin[kMaxTimed] = {};
  float kt_ms[kMaxTimed] = {};
  bool kt_pending = false;
  Buf paths;   // SPECK_OPT_PATH_COUNTERS: unsigned long long [SPECK_PATH_COUNT]
  // user workspace allocator (speck_set_allocator)
  speck_alloc_fn ualloc = nullptr;
  speck_release_fn urelease = nullptr;
  void* uctx = nullptr;
};

namespace {

speck_status_t fail(speck_handle_t h, speck_status_t s, const char* fmt, ...) {
  if (h) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    h->err = buf;
  }
  return s;
}

#define CK(call)                                                                                      \
  do {                                                                                                \
    cudaError_t e_ = (call);                                                                          \
    if (e_ != cudaSuccess)                                                                            \
      return fail(h, e_ == cudaErrorMemoryAllocation ? SPECK_ERR_OUT_OF_MEMORY : SPECK_ERR_CUDA,      \
                  "%s failed: %s (%s:%d)", #call, cudaGetErrorString(e_), __FILE__, __LINE__);        \
  } while (0)

#define CKL()                                                                                         \
  do {                                                                                                \
    ++h->launches;                                                                                    \
    cudaError_t e_ = cudaGetLastError();                                                              \
    if (e_ != cudaSuccess)                                                                            \
      return fail(h, SPECK_ERR_CUDA, "kernel launch failed: %s (%s:%d)", cudaGetErrorString(e_),      \
                  __FILE__, __LINE__);                                                                \
  } while (0)

void release_buf(speck_handle_t h, Buf& b, cudaStream_t s) {
  if (b.p) {
    if (h->urelease) h->urelease(b.p, static_cast<speck_stream_t>(s), h->uctx);
    else cudaFreeAsync(b.p, s);
  }
  b.p = nullptr;
  b.cap = 0;
}

speck_status_t ensure(speck_handle_t h, Buf& b, size_t bytes, cudaStream_t s, bool exact = false) {
  if (bytes <= b.cap) return SPECK_OK;
  release_buf(h, b, s);
  size_t want = std::max<size_t>(exact ? bytes : bytes + bytes / 4, 4096);
  if (h->ualloc) {
    b.p = h->ualloc(want, static_cast<speck_stream_t>(s), h->uctx);
    if (!b.p) return fail(h, SPECK_ERR_OUT_OF_MEMORY, "workspace allocation of %zu bytes failed (user allocator)", want);
    b.cap = want;
    return SPECK_OK;
  }
  cudaError_t e = cudaMallocAsync(&b.p, want, s);
  if (e != cudaSuccess) {
    (void)cudaGetLastError();
    return fail(h, SPECK_ERR_OUT_OF_MEMORY, "workspace allocation of %zu bytes failed: %s", want,
                cudaGetErrorString(e));
  }
  b.cap = want;
  return SPECK_OK;
}

// SPECK_OPT_KERNEL_TIMING: bracket a launch with events on the stream it runs on.
int kt_begin(speck_handle_t h, cudaStream_t s, int kind, int cfg, int bin) {
  if (!h->opt_ktime || h->kt_n >= kMaxTimed) return -1;
  const int i = h->kt_n++;
  h->kt_id[i] = kind * 16 + cfg;
  h->kt_bin[i] = bin;
  cudaEventRecord(h->kt_ev[2 * i], s);
  h->kt_pending = true;
  return i;
}
void kt_end(speck_handle_t h, cudaStream_t s, int i) {
  if (i >= 0) cudaEventRecord(h->kt_ev[2 * i + 1], s);
}

int64_t ws_bytes(speck_handle_t h) {
  return (int64_t)(h->prods.cap + h->maxlen.cap + h->colmin.cap + h->colmax.cap + h->cnt.cap + h->hist.cap +
                   h->hist_off.cap + h->bins.cap + h->stats.cap + h->scan_status.cap + h->resume.cap + h->small.cap +
                   h->ana_long.cap + h->chunk_cnt.cap + h->cand.cap + h->nseg.cap + h->seg_off.cap + h->segs.cap +
                   h->bm_pool.cap + h->bm_off.cap + h->binfo.cap + h->paths.cap + h->chunks.cap +
                   h->tr_cnt.cap + h->tr_list.cap + h->tr_col.cap + h->tr_val.cap + h->det_scratch.cap);
}

speck_status_t check_csr(speck_handle_t h, const speck_csr_t* M, const char* name, bool need_values) {
  if (!M) return fail(h, SPECK_ERR_INVALID_ARGUMENT, "%s is NULL", name);
  if (M->rows < 0 || M->cols < 0 || M->nnz < 0) return fail(h, SPECK_ERR_INVALID_ARGUMENT, "%s has negative dims", name);
  if (M->cols >= 0x7fffffffLL || M->rows >= 0x7fffffffLL)
    return fail(h, SPECK_ERR_UNSUPPORTED, "%s: rows/cols must be < 2^31-1", name);
  if (!M->row_ptr && M->rows > 0) return fail(h, SPECK_ERR_INVALID_ARGUMENT, "%s.row_ptr is NULL", name);
  if (M->nnz > 0 && !M->col_idx) return fail(h, SPECK_ERR_INVALID_ARGUMENT, "%s.col_idx is NULL", name);
  if (need_values && M->nnz > 0 && !M->values) return fail(h, SPECK_ERR_INVALID_ARGUMENT, "%s.values is NULL", name);
  if (M->dtype != SPECK_F32 && M->dtype != SPECK_F64) return fail(h, SPECK_ERR_INVALID_ARGUMENT, "%s.dtype invalid", name);
  return SPECK_OK;
}

int pow2_clamp(double x, int lo, int hi) {
  int p = lo;
  while (p * 2 <= hi && (double)(p * 2) <= x) p *= 2;
  return p;
}

// Row analysis (Alg. 1): GA lanes per row (GA x kAnaU ~ average row length of A), rows longer than
// kAnaLong deferred to one CTA each.  `st` may be null (no statistics).
speck_status_t run_analysis(speck_handle_t h, const speck_csr_t* A, const speck_csr_t* B, int64_t* prods,
                            int32_t* maxlen, int32_t* colmin, int32_t* colmax, AnalysisStats* st, cudaStream_t s) {
  const int64_t m = A->rows;
  speck_status_t r;
  if ((r = ensure(h, h->ana_long, (size_t)(A->nnz / kAnaLong + 1) * 4, s))) return r;
  if ((r = ensure(h, h->small, 4096, s))) return r;
  unsigned* nlong = reinterpret_cast<unsigned*>(static_cast<char*>(h->small.p) + 640);
  int32_t* lrows = static_cast<int32_t*>(h->ana_long.p);
  CK(cudaMemsetAsync(nlong, 0, 4, s));
  const int kt = kt_begin(h, s, SPECK_KERNEL_ANALYSIS, 0, -1);
  // rows of B referenced several times on average: one 16-byte record per row of B
  const int4* binfo = nullptr;
  if (B->rows > 0 && A->nnz > 4 * B->rows && B->rows < ((int64_t)1 << 31)) {
    if ((r = ensure(h, h->binfo, (size_t)B->rows * 16, s))) return r;
    binfo = static_cast<const int4*>(h->binfo.p);
    const unsigned bg = (unsigned)std::max<int64_t>(1, std::min<int64_t>((B->rows + 255) / 256, (int64_t)h->num_sms * 16));
    k_brow_info<<<bg, 256, 0, s>>>(B->row_ptr, B->col_idx, B->rows, const_cast<int4*>(binfo));
    CKL();
  }
  const int ga = pow2_clamp(m > 0 ? (double)A->nnz / (double)m / kAnaU : 1.0, 1, 32);   // GA*kAnaU ~ avg row
  const unsigned agrid = (unsigned)std::max<int64_t>(1, std::min<int64_t>((m * ga + 255) / 256, (int64_t)h->num_sms * 8));
#define SPECK_ANA(GA)                                                                                        \
  k_analysis<GA><<<agrid, 256, 0, s>>>(A->row_ptr, A->col_idx, B->row_ptr, B->col_idx, m, prods, maxlen, colmin, \
                                       colmax, st, lrows, nlong, binfo)
  switch (ga) {
    case 1: SPECK_ANA(1); break;
    case 2: SPECK_ANA(2); break;
    case 4: SPECK_ANA(4); break;
    case 8: SPECK_ANA(8); break;
    case 16: SPECK_ANA(16); break;
    default: SPECK_ANA(32); break;
  }
#undef SPECK_ANA
  CKL();
  k_analysis_long<<<(unsigned)h->num_sms * 2, 256, 0, s>>>(A->row_ptr, A->col_idx, B->row_ptr, B->col_idx, prods, maxlen,
                                                           colmin, colmax, st, lrows, nlong);
  CKL();
  kt_end(h, s, kt);
  return SPECK_OK;
}

// kernel function pointer for (cfg, pass, V)
template <typename V>
void* spgemm_fn(int cfg, int pass) {
  switch (cfg * 2 + pass) {
    case 0: return (void*)k_spgemm<0, 0, V>;
    case 1: return (void*)k_spgemm<0, 1, V>;
    case 2: return (void*)k_spgemm<1, 0, V>;
    case 3: return (void*)k_spgemm<1, 1, V>;
    case 4: return (void*)k_spgemm<2, 0, V>;
    case 5: return (void*)k_spgemm<2, 1, V>;
    case 6: return (void*)k_spgemm<3, 0, V>;
    case 7: return (void*)k_spgemm<3, 1, V>;
    case 8: return (void*)k_spgemm<4, 0, V>;
    default: return (void*)k_spgemm<4, 1, V>;
  }
}

template <typename V>
speck_status_t launch_spgemm(speck_handle_t h, int cfg, int pass, const SpgemmArgs<V>& a, cudaStream_t s, int bin) {
  if (a.n_entries <= 0) return SPECK_OK;
  const int64_t grid = (a.n_entries + a.group_rows - 1) / a.group_rows;
  // (persistent CTAs pulling groups from a counter were tried: C5 336 -> 350 ms, the resident
  // grid keeps the other bins' kernels from overlapping; one CTA per group it is)
  const int kt = kt_begin(h, s, pass == 0 ? SPECK_KERNEL_SYM_BLOCK : SPECK_KERNEL_NUM_BLOCK, cfg, bin);
  void* args[] = {(void*)&a};
  CK(cudaLaunchKernel(spgemm_fn<V>(cfg, pass), dim3((unsigned)grid), dim3(kCfgThreads[cfg]), args,
                      (size_t)kCfgMapBytes[cfg], s));
  kt_end(h, s, kt);
  ++h->launches;
  return SPECK_OK;
}

template <typename V>
speck_status_t set_smem_attrs(speck_handle_t h) {
  for (int c = 0; c < kNumCfg; ++c)
    for (int pass = 0; pass < 2; ++pass)
      CK(cudaFuncSetAttribute(spgemm_fn<V>(c, pass), cudaFuncAttributeMaxDynamicSharedMemorySize, kCfgMapBytes[c]));
  CK(cudaFuncSetAttribute(k_segments<V>, cudaFuncAttributeMaxDynamicSharedMemorySize, kCfgMapBytes[kSegCfg]));
  CK(cudaFuncSetAttribute(k_tr_sort_block<V>, cudaFuncAttributeMaxDynamicSharedMemorySize, kTrSmemSort * (4 + (int)sizeof(V))));
  CK(cudaFuncSetAttribute(k_det_rows<V>, cudaFuncAttributeMaxDynamicSharedMemorySize, kDetRegion * kDetWarps));
  CK(cudaFuncSetAttribute(k_long_bitmap<V>, cudaFuncAttributeMaxDynamicSharedMemorySize, kCfgMapBytes[kNumCfg - 1]));
  CK(cudaFuncSetAttribute(k_warp_rows<0, V, 0>, cudaFuncAttributeMaxDynamicSharedMemorySize, kWarpRegionBytesSym * (kWarpRowThreads / 32)));
  CK(cudaFuncSetAttribute(k_warp_rows<0, V, 3>, cudaFuncAttributeMaxDynamicSharedMemorySize, kWarpRegionBytesSym * (kWarpRowThreads / 32)));
  CK(cudaFuncSetAttribute(k_warp_rows<0, V, 8>, cudaFuncAttributeMaxDynamicSharedMemorySize, kWarpRegionBytesSym * (kWarpRowThreads / 32)));
  CK(cudaFuncSetAttribute(k_warp_rows<1, V, 8>, cudaFuncAttributeMaxDynamicSharedMemorySize, kWarpRegionBytes * (kWarpRowThreads / 32)));
  CK(cudaFuncSetAttribute(k_warp_rows<1, V, 9>, cudaFuncAttributeMaxDynamicSharedMemorySize, kWarpRegionBytesTiny * (kWarpRowThreads / 32)));
  CK(cudaFuncSetAttribute(k_warp_rows<1, V, 10>, cudaFuncAttributeMaxDynamicSharedMemorySize, kWarpRegionBytes * (kWarpRowThreads / 32)));
  CK(cudaFuncSetAttribute(k_warp_rows<1, V, 0>, cudaFuncAttributeMaxDynamicSharedMemorySize, kWarpRegionBytes * (kWarpRowThreads / 32)));
  CK(cudaFuncSetAttribute(k_warp_rows<1, V, 1>, cudaFuncAttributeMaxDynamicSharedMemorySize, kWarpRegionBytesTiny * (kWarpRowThreads / 32)));
  CK(cudaFuncSetAttribute(k_warp_rows<1, V, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize, kWarpRegionBytes * (kWarpRowThreads / 32)));
  return SPECK_OK;
}

speck_status_t launch_scan(speck_handle_t h, const int64_t* in, int64_t n, int64_t* out, unsigned long long* max_out,
                           cudaStream_t s) {
  const int64_t tiles = n / kScanTile + 1;
  speck_status_t st = ensure(h, h->scan_status, (size_t)tiles * 8 + 64, s);
  if (st) return st;
  CK(cudaMemsetAsync(h->scan_status.p, 0, (size_t)tiles * 8 + 64, s));
  unsigned int* counter = reinterpret_cast<unsigned int*>(static_cast<char*>(h->scan_status.p) + tiles * 8);
  k_scan<<<(unsigned)tiles, kScanThreads, 0, s>>>(in, n, out, static_cast<unsigned long long*>(h->scan_status.p), counter,
                                                 max_out);
  CKL();
  return SPECK_OK;
}

// fork: internal streams wait for the user stream
speck_status_t fork(speck_handle_t h, cudaStream_t s, int n) {
  CK(cudaEventRecord(h->ev_fork, s));
  for (int i = 0; i < n; ++i) CK(cudaStreamWaitEvent(h->streams[i], h->ev_fork, 0));
  return SPECK_OK;
}
speck_status_t join(speck_handle_t h, cudaStream_t s, int n) {
  for (int i = 0; i < n; ++i) {
    CK(cudaEventRecord(h->ev_join[i], h->streams[i]));
    CK(cudaStreamWaitEvent(s, h->ev_join[i], 0));
  }
  return SPECK_OK;
}

int64_t warp_row_fill(speck_handle_t h, int pass) {
  if (pass == 0) return wr_sym_fill();
  return h->dtype == SPECK_F64 ? wr_num_fill<double>() : wr_num_fill<float>();
}

// Small-row kernel: persistent CTAs of 8 warps pulling rows from a counter (zeroed here).
// mode (numeric): 0 any row, 1 rows of <= kTinyCnt entries, 2 larger rows (k_warp_rows MODE).
template <typename V>
speck_status_t launch_warp_rows(speck_handle_t h, int pass, const SpgemmArgs<V>& a, cudaStream_t s, int mode, int bin) {
  if (a.n_entries <= 0) return SPECK_OK;
  unsigned long long* ctr =
      reinterpret_cast<unsigned long long*>(static_cast<char*>(h->small.p) + 1024 + 8 * (pass == 0 ? 0 : 1 + mode));
  CK(cudaMemsetAsync(ctr, 0, 8, s));
  const int md = pass == 0 ? 0 : mode;
  const int64_t grid = std::min<int64_t>((a.n_entries + 7) / 8, (int64_t)h->num_sms * wr_ctas_per_sm(pass, md));
  const size_t smem = (size_t)wr_region_bytes(pass, md) * (kWarpRowThreads / 32);
  const int kt = kt_begin(h, s, pass == 0 ? SPECK_KERNEL_SYM_WARP : md == 1 ? SPECK_KERNEL_NUM_TINY : SPECK_KERNEL_NUM_WARP,
                          md, bin);
  if (a.fixed_g != 0) {   // the paper's grouped local load balancing (ablation instantiations)
    if (pass == 0) k_warp_rows<0, V, 8><<<(unsigned)grid, kWarpRowThreads, smem, s>>>(a, ctr);
    else if (mode == 1) k_warp_rows<1, V, 9><<<(unsigned)grid, kWarpRowThreads, smem, s>>>(a, ctr);
    else if (mode == 2) k_warp_rows<1, V, 10><<<(unsigned)grid, kWarpRowThreads, smem, s>>>(a, ctr);
    else k_warp_rows<1, V, 8><<<(unsigned)grid, kWarpRowThreads, smem, s>>>(a, ctr);
  } else if (pass == 0 && a.esc >= 2) k_warp_rows<0, V, 3><<<(unsigned)grid, kWarpRowThreads, smem, s>>>(a, ctr);
  else if (pass == 0) k_warp_rows<0, V, 0><<<(unsigned)grid, kWarpRowThreads, smem, s>>>(a, ctr);
  else if (mode == 1) k_warp_rows<1, V, 1><<<(unsigned)grid, kWarpRowThreads, smem, s>>>(a, ctr);
  else if (mode == 2) k_warp_rows<1, V, 2><<<(unsigned)grid, kWarpRowThreads, smem, s>>>(a, ctr);
  else k_warp_rows<1, V, 0><<<(unsigned)grid, kWarpRowThreads, smem, s>>>(a, ctr);
  CKL();
  kt_end(h, s, kt);
  return SPECK_OK;
}

BinParams make_bin_params(speck_handle_t h, int pass) {
  BinParams bp{};
  bp.pass = pass;
  bp.use_direct = h->opt_disable_direct ? 0 : 1;
  bp.long_thr = INT64_MAX;
  bp.tiny_cap = (pass == 1 && h->opt_warp_rows) ? kTinyCnt : -1;
  for (int c = 0; c < kNumCfg; ++c) {
    if (pass == 0) bp.cap[c] = sym_map_fill(c);
    else bp.cap[c] = h->dtype == SPECK_F64 ? num_map_fill<double>(c) : num_map_fill<float>(c);
  }
  // smallest bin = rows of one warp (k_warp_rows) instead of merged blocks of configuration 0
  if (h->opt_warp_rows) bp.cap[0] = warp_row_fill(h, pass);
  if (h->seg_enabled) {
    // every row that may exceed the largest numeric map is a symbolic cfg4 row, so that the
    // symbolic pass records its per-chunk counts; such rows become numeric segments
    if (pass == 0) bp.cap[kNumCfg - 2] = std::min<int64_t>(bp.cap[kNumCfg - 2], h->long_thr);
    else bp.long_thr = h->long_thr;
  }
  if (h->opt_force_acc == 2) {  // dense everywhere: every non-trivial row is a single-row block of the largest cfg
    for (int c = 0; c < kNumCfg - 1; ++c) bp.cap[c] = -1;
  }
  return bp;
}

// Segment geometry for long numeric rows (segment_kernels.cuh); decided before the analysis.
template <typename V>
void plan_segments(speck_handle_t h, int64_t ncols) {
  h->long_thr = num_map_fill<V>(kNumCfg - 1);
  int s = 0;
  while ((int64_t)1 << (s + 1) <= num_dense_window<V>(kSegCfg)) ++s;
  h->seg_shift = s;
  h->nchunks = (int)((ncols + ((int64_t)1 << s) - 1) >> s);
  h->seg_enabled = h->opt_force_acc != 2 && h->opt_segments != 0 && !h->opt_det && h->nchunks >= 1 && h->nchunks <= kMaxChunks;
  h->n_cand = 0;
  h->n_segs = 0;
}

// Table 2 decision.  need_max / need_avg per row; returns 1 = balance.
int decide_lb(const LbThresholds& t, int64_t opt, double need_max, double need_sum, int64_t rows, int cfg_of_max,
              bool forced) {
  if (forced) return 1;
  if (opt >= 0) return opt ? 1 : 0;
  if (rows <= 0 || need_sum <= 0) return 0;
  const double ratio = need_max / (need_sum / (double)rows);
  if (cfg_of_max >= t.big_from_cfg) return (ratio > t.ratio_big && rows > t.rows_big) ? 1 : 0;
  return (ratio > t.ratio && rows > t.rows) ? 1 : 0;
}

int cfg_for(const BinParams& bp, int64_t need) {
  for (int c = 0; c < kNumCfg; ++c)
    if (need <= bp.cap[c]) return c;
  return kNumCfg;  // does not fit any hash configuration
}

template <typename V>
SpgemmArgs<V> base_args(speck_handle_t h, const speck_csr_t* A, const speck_csr_t* B) {
  SpgemmArgs<V> a{};
  a.A_rp = A->row_ptr; a.A_col = A->col_idx; a.A_val = static_cast<const V*>(A->values);
  a.B_rp = B->row_ptr; a.B_col = B->col_idx; a.B_val = static_cast<const V*>(B->values);
  a.m = A->rows; a.n = B->cols;
  a.prods = static_cast<const int64_t*>(h->prods.p);
  a.maxlen = static_cast<const int32_t*>(h->maxlen.p);
  a.colmin = static_cast<const int32_t*>(h->colmin.p);
  a.colmax = static_cast<const int32_t*>(h->colmax.p);
  a.force_acc = (int)h->opt_force_acc;
  a.dense_window_cap = h->opt_dense_window;
  a.fixed_g = (int)h->opt_fixed_g;
  a.esc = h->opt_det ? 0 : (int)h->opt_esc;          // deterministic: one warp per row, in-order adds
  if (h->opt_det) a.fixed_g = 0;
  a.paths = h->opt_paths ? static_cast<unsigned long long*>(h->paths.p) : nullptr;
  a.row_lo = 0;
  a.row_hi = INT64_MAX;
  a.cnt = static_cast<int64_t*>(h->cnt.p);
  a.resume = static_cast<int32_t*>(h->resume.p);
  a.resume_stride = 2 * std::max<int64_t>(h->max_nnza, 1);   // two buffers (cur / next) per SM slot
  a.resume_slots = h->num_smid;
  a.n_dense_rows = reinterpret_cast<unsigned long long*>(static_cast<char*>(h->small.p) + 256);
  return a;
}

template <typename V>
SegPlanArgs seg_plan_args(speck_handle_t h, const int64_t* C_rp) {
  SegPlanArgs s{};
  s.cand = static_cast<const int32_t*>(h->cand.p);
  s.ncand = h->n_cand;
  s.C_rp = C_rp;
  s.A_rp = h->A_rp;
  s.prods = static_cast<const int64_t*>(h->prods.p);
  s.colmin = static_cast<const int32_t*>(h->colmin.p);
  s.colmax = static_cast<const int32_t*>(h->colmax.p);
  s.chunk_cnt = static_cast<const int32_t*>(h->chunk_cnt.p);
  s.nchunks = h->nchunks;
  s.shift = h->seg_shift;
  s.limit = h->long_thr;
  s.dense_window = num_dense_window<V>(kSegCfg);
  s.map_slots = num_map_cap<V>(kSegCfg);
  s.seg_limit = num_map_fill<V>(kSegCfg);
  // few candidates: split every long row so its work spreads over the SMs — unless rows of A
  // are very long: every column segment binary-searches each referenced B row, so a segment
  // costs O(nnz(A_i)) before its first product (C4: 200k-NZ rows, 32 segments each; the bitmap
  // CTA per row took the numeric step 32.6 -> 16.5 ms)
  s.prefer_parallel = (h->n_cand < 4 * (int64_t)h->num_sms && h->max_nnza < kSegMaxNnzA) ? 1 : 0;
  // many long rows: one bitmap CTA per row whose column range fits (no column segments)
  s.bitmap_cols = (h->opt_long_bitmap == 2 || (h->opt_long_bitmap && !s.prefer_parallel)) ? kBitmapMaxCols : 0;
  s.bm_pool = (h->bm_enabled && s.bitmap_cols > 0) ? static_cast<const uint32_t*>(h->bm_pool.p) : nullptr;
  s.bm_off = static_cast<const int64_t*>(h->bm_off.p);
  s.split_max = 1;
  return s;
}

// Launch one pass (symbolic pass=0 / numeric pass=1) either over the bins (LB on) or over
// fixed groups of consecutive rows (LB off).
template <typename V>
speck_status_t run_pass(speck_handle_t h, int pass, int lb, const int64_t* cat_beg, const int64_t* cat_end,
                        SpgemmArgs<V> a, int64_t need_max, const BinParams& bp, cudaStream_t s) {
  const int64_t m = a.m;
  if (!lb) {
    // no load balancing: one configuration with room for R rows of the longest size.
    // Capacities are the maps' own (the long-row cap adjustment of the binned path does not
    // apply: without balancing every row already fits below it).
    BinParams own = bp;
    for (int c = 0; c < kNumCfg; ++c)
      own.cap[c] = pass == 0 ? (int64_t)sym_map_fill(c) : (int64_t)num_map_fill<V>(c);
    a.rows = nullptr;
    a.n_entries = m;
    if (h->opt_warp_rows && need_max <= warp_row_fill(h, pass))
      return launch_warp_rows<V>(h, pass, a, s, pass == 1 && need_max <= kTinyCnt ? 1 : 0, -1);
    int cfg = -1, R = 1;
    for (int c = 0; c < kNumCfg; ++c)
      if (need_max * kMaxGroupRows <= own.cap[c]) { cfg = c; R = kMaxGroupRows; break; }
    if (cfg < 0) {
      cfg = cfg_for(own, need_max);
      if (cfg >= kNumCfg) cfg = kNumCfg - 1;
      R = (int)std::max<int64_t>(1, std::min<int64_t>(kMaxGroupRows, own.cap[cfg] / std::max<int64_t>(need_max, 1)));
    }
    a.rows = nullptr;
    a.n_entries = m;
    a.group_rows = R;
    a.merge = 0;
    return launch_spgemm<V>(h, cfg, pass, a, s, -1);
  }
  const int ns = (int)std::max<int64_t>(1, std::min<int64_t>(h->opt_streams, kMaxStreams));
  speck_status_t st;
  const bool segs = pass == 1 && h->seg_enabled && h->n_segs > 0;
  if (segs) {
    // segment descriptors of the long rows (offsets were scanned during analyze)
    if ((st = ensure(h, h->segs, (size_t)h->n_segs * sizeof(Seg), s))) return st;
    const int64_t nc = h->n_cand;
    const int kt = kt_begin(h, s, SPECK_KERNEL_SEG_PLAN, 1, -1);
    k_seg_emit<<<(unsigned)((nc + 127) / 128), 128, 0, s>>>(seg_plan_args<V>(h, a.C_rp),
                                                           static_cast<const int64_t*>(h->seg_off.p),
                                                           static_cast<Seg*>(h->segs.p));
    CKL();
    kt_end(h, s, kt);
  }
  // few long rows with kept bitmaps: split them over several CTAs (zero C.val first, on the
  // user stream, before any kernel of this pass writes it)
  SegPlanArgs sa0{};
  if (pass == 1 && h->seg_enabled && h->n_cand > 0) {
    sa0 = seg_plan_args<V>(h, a.C_rp);
    if (sa0.bitmap_cols > 0 && sa0.bm_pool && h->n_cand <= kSplitMaxCand) {
      sa0.split_max = kSplitPieces;
      // zero the C.val ranges of the rows that will be split over several CTAs (only those)
      k_zero_split_rows<V><<<(unsigned)h->n_cand, 256, 0, s>>>(a, sa0);
      CKL();
    }
  }
  if ((st = fork(h, s, ns))) return st;
  int si = 0;
  const int32_t* bins = static_cast<const int32_t*>(h->bins.p);
  if (pass == 1 && h->seg_enabled && h->n_cand > 0) {
    const SegPlanArgs sa = sa0;
    if (sa.bitmap_cols > 0) {
      const int kt = kt_begin(h, h->streams[si], SPECK_KERNEL_LONG_BITMAP, 0, 16 + CAT_LONG);
      k_long_bitmap<V><<<(unsigned)(h->n_cand * sa.split_max), kBitmapThreads, kCfgMapBytes[kNumCfg - 1], h->streams[si]>>>(a, sa);
      CKL();
      kt_end(h, h->streams[si], kt);
      si = (si + 1) % ns;
    }
  }
  if (segs) {
    const int kt = kt_begin(h, h->streams[si], SPECK_KERNEL_SEGMENTS, kSegCfg, 16 + CAT_LONG);
    k_segments<V><<<(unsigned)h->n_segs, kCfgThreads[kSegCfg], kCfgMapBytes[kSegCfg], h->streams[si]>>>(
        a, static_cast<const Seg*>(h->segs.p));
    CKL();
    kt_end(h, h->streams[si], kt);
    si = (si + 1) % ns;
  }
  // largest configurations first so long rows start early
  for (int c = kNumCfg - 1; c >= 0; --c) {
    const int cat = CAT_CFG0 + c;
    const int64_t n = cat_end[cat] - cat_beg[cat];
    if (n <= 0) continue;
    SpgemmArgs<V> b = a;
    b.rows = bins + cat_beg[cat];
    b.n_entries = n;
    if (pass == 1 && h->opt_det && (c > 0 || !h->opt_warp_rows)) {
      // deterministic mode: rows beyond the warp region -> one warp per row (det_kernels.cuh)
      const int64_t slots = (int64_t)h->num_sms * kDetWarps;
      if ((st = ensure(h, h->det_scratch, (size_t)slots * (size_t)a.resume_stride * 4, h->streams[si]))) return st;
      unsigned long long* ctr = reinterpret_cast<unsigned long long*>(static_cast<char*>(h->small.p) + 1280 + 8 * c);
      CK(cudaMemsetAsync(ctr, 0, 8, h->streams[si]));
      const int kt = kt_begin(h, h->streams[si], SPECK_KERNEL_NUM_BLOCK, c, 16 + cat);
      k_det_rows<V><<<(unsigned)std::min<int64_t>(h->num_sms, (n + kDetWarps - 1) / kDetWarps), 32 * kDetWarps,
                      (size_t)kDetRegion * kDetWarps, h->streams[si]>>>(b, ctr, static_cast<int32_t*>(h->det_scratch.p));
      CKL();
      kt_end(h, h->streams[si], kt);
      si = (si + 1) % ns;
      continue;
    }
    if (c == 0 && h->opt_warp_rows) {
      st = launch_warp_rows<V>(h, pass, b, h->streams[si], pass == 1 ? 2 : 0, pass * 16 + cat);
      if (st) return st;
      si = (si + 1) % ns;
      continue;
    }
    if (c == 0) {
      b.group_rows = kMaxGroupRows;
      b.merge = 1;
      b.merge_cap = bp.cap[0] + 1;  // merge while the sum stays <= cap (strict < cap+1)
    } else {
      b.group_rows = 1;
      b.merge = 0;
    }
    if (pass == 0 && c == kNumCfg - 1 && h->seg_enabled && h->n_cand > 0) {
      b.chunk_cnt = static_cast<int32_t*>(h->chunk_cnt.p);   // entry e of this bin -> chunk_cnt[e]
      b.nchunks = h->nchunks;
      b.chunk_shift = h->seg_shift;
      b.long_thr = h->long_thr;
      if (h->bm_enabled) {
        b.bm_pool = static_cast<uint32_t*>(h->bm_pool.p);
        b.bm_pool_words = h->bm_pool_words;
        b.bm_ctr = reinterpret_cast<unsigned long long*>(static_cast<char*>(h->small.p) + 2048);
        b.bm_off = static_cast<int64_t*>(h->bm_off.p);
      }
    }
    st = launch_spgemm<V>(h, c, pass, b, h->streams[si], pass * 16 + cat);
    if (st) return st;
    si = (si + 1) % ns;
  }
  if (pass == 1 && cat_end[CAT_TINY] > cat_beg[CAT_TINY]) {
    SpgemmArgs<V> b = a;
    b.rows = bins + cat_beg[CAT_TINY];
    b.n_entries = cat_end[CAT_TINY] - cat_beg[CAT_TINY];
    st = launch_warp_rows<V>(h, pass, b, h->streams[si], 1, 16 + CAT_TINY);
    if (st) return st;
    si = (si + 1) % ns;
  }
  if (pass == 1) {
    const int64_t n = cat_end[CAT_DIRECT] - cat_beg[CAT_DIRECT];
    if (n > 0) {
      // GD lanes per row: average length of B rows
      const double avg = h->B_rows > 0 ? (double)h->B_nnz / (double)h->B_rows : 1.0;
      const int gd = pow2_clamp(avg, 1, 32);
      const int64_t rows_per_cta = 256 / gd;
      const unsigned grid = (unsigned)std::min<int64_t>((n + rows_per_cta - 1) / rows_per_cta, (int64_t)h->num_sms * 16);
      const int32_t* rows = bins + cat_beg[CAT_DIRECT];
      cudaStream_t ds = h->streams[si];
      const int kt = kt_begin(h, ds, SPECK_KERNEL_DIRECT, 0, 16 + CAT_DIRECT);
#define SPECK_DIRECT(GD)                                                                                   \
  k_direct<V, GD><<<grid, 256, 0, ds>>>(rows, n, a.A_rp, a.A_col, a.A_val, a.B_rp, a.B_col, a.B_val, a.C_rp, \
                                        a.C_col, a.C_val, a.paths)
      switch (gd) {
        case 1: SPECK_DIRECT(1); break;
        case 2: SPECK_DIRECT(2); break;
        case 4: SPECK_DIRECT(4); break;
        case 8: SPECK_DIRECT(8); break;
        case 16: SPECK_DIRECT(16); break;
        default: SPECK_DIRECT(32); break;
      }
#undef SPECK_DIRECT
      CKL();
      kt_end(h, ds, kt);
    }
  }
  return join(h, s, ns);
}

speck_status_t timing_mark(speck_handle_t h, int i, cudaStream_t s) {
  if (h->opt_timing) CK(cudaEventRecord(h->ev_t[i], s));
  return SPECK_OK;
}

float elapsed(speck_handle_t h, int a, int b) {
  float ms = 0.f;
  if (cudaEventElapsedTime(&ms, h->ev_t[a], h->ev_t[b]) != cudaSuccess) {
    (void)cudaGetLastError();
    return -1.f;
  }
  return ms;
}

template <typename V>
speck_status_t analyze_impl(speck_handle_t h, const speck_csr_t* A, const speck_csr_t* B, int64_t* C_rp, int64_t* nnz_c,
                            cudaStream_t s) {
  const int64_t m = A->rows;
  speck_status_t st;
  h->analyzed = false;
  h->dtype = A->dtype;
  h->A_rp = A->row_ptr; h->A_col = A->col_idx; h->A_rows = A->rows; h->A_cols = A->cols; h->A_nnz = A->nnz;
  h->B_rp = B->row_ptr; h->B_col = B->col_idx; h->B_rows = B->rows; h->B_cols = B->cols; h->B_nnz = B->nnz;
  {
    int64_t keep[SPECK_PATH_COUNT];   // path counters are cumulative
    std::memcpy(keep, h->st.path_rows, sizeof keep);
    std::memset(&h->st, 0, sizeof h->st);
    std::memcpy(h->st.path_rows, keep, sizeof keep);
  }
  h->kt_n = 0;
  h->kt_pending = false;
  plan_segments<V>(h, B->cols);
  if (m == 0) {
    if (C_rp) CK(cudaMemsetAsync(C_rp, 0, sizeof(int64_t), s));
    *nnz_c = 0;
    h->nnz_c = 0;
    h->analyzed = true;
    return SPECK_OK;
  }
  const int64_t tiles = (m + kBinTile - 1) / kBinTile;
  if ((st = ensure(h, h->prods, (size_t)m * 8, s))) return st;
  if ((st = ensure(h, h->maxlen, (size_t)m * 4, s))) return st;
  if ((st = ensure(h, h->colmin, (size_t)m * 4, s))) return st;
  if ((st = ensure(h, h->colmax, (size_t)m * 4, s))) return st;
  if ((st = ensure(h, h->cnt, (size_t)m * 8, s))) return st;
  if ((st = ensure(h, h->bins, (size_t)m * 4, s))) return st;
  if ((st = ensure(h, h->hist, (size_t)tiles * CAT_COUNT * 8, s))) return st;
  if ((st = ensure(h, h->hist_off, ((size_t)tiles * CAT_COUNT + 1) * 8, s))) return st;
  if ((st = ensure(h, h->small, 4096, s))) return st;

  if (h->opt_validate) {
    int* bad = reinterpret_cast<int*>(static_cast<char*>(h->small.p) + 512);
    CK(cudaMemsetAsync(bad, 0, 8, s));
    k_validate<<<(unsigned)std::min<int64_t>((A->rows + 255) / 256, 4096), 256, 0, s>>>(A->row_ptr, A->col_idx, A->rows, A->cols, bad);
    k_validate<<<(unsigned)std::min<int64_t>((B->rows + 255) / 256, 4096), 256, 0, s>>>(B->row_ptr, B->col_idx, B->rows, B->cols, bad + 1);
    CKL();
    int hb[2];
    CK(cudaMemcpyAsync(hb, bad, 8, cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    if (hb[0] || hb[1]) return fail(h, SPECK_ERR_INVALID_INPUT, "input CSR %s has unsorted/duplicate/out-of-range columns", hb[0] ? "A" : "B");
  }

  // ---- 1. row analysis (Alg. 1) ---------------------------------------------------------
  if ((st = timing_mark(h, 0, s))) return st;
  AnalysisStats* dstats = static_cast<AnalysisStats*>(h->small.p);
  CK(cudaMemsetAsync(h->small.p, 0, 4096, s));
  if ((st = run_analysis(h, A, B, static_cast<int64_t*>(h->prods.p), static_cast<int32_t*>(h->maxlen.p),
                         static_cast<int32_t*>(h->colmin.p), static_cast<int32_t*>(h->colmax.p), dstats, s)))
    return st;
  // symbolic classification histogram per tile (global LB step 1), computed unconditionally
  const BinParams bps = make_bin_params(h, 0);
  unsigned long long* bin_sums = reinterpret_cast<unsigned long long*>(static_cast<char*>(h->small.p) + kSmallBinSums);
  int kt = kt_begin(h, s, SPECK_KERNEL_BINNING, 0, -1);
  k_classify<<<(unsigned)tiles, kBinTile, 0, s>>>(A->row_ptr, static_cast<int64_t*>(h->prods.p), nullptr, m, bps,
                                                 static_cast<int64_t*>(h->hist.p), tiles, bin_sums);
  CKL();
  if ((st = launch_scan(h, static_cast<int64_t*>(h->hist.p), tiles * CAT_COUNT, static_cast<int64_t*>(h->hist_off.p),
                        nullptr, s)))
    return st;
  kt_end(h, s, kt);
  // read back the stats and the bin boundaries (sync #1)
  {
    unsigned long long* hp = h->h_pinned;
    CK(cudaMemcpyAsync(hp, dstats, sizeof(AnalysisStats), cudaMemcpyDeviceToHost, s));
    for (int c = 0; c <= CAT_COUNT; ++c)
      CK(cudaMemcpyAsync(hp + kPinSymCat + c, static_cast<int64_t*>(h->hist_off.p) + (int64_t)c * tiles, 8,
                         cudaMemcpyDeviceToHost, s));
    CK(cudaMemcpyAsync(hp + kPinBinSums, bin_sums, CAT_COUNT * 3 * 8, cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
  }
  AnalysisStats hs;
  std::memcpy(&hs, h->h_pinned, sizeof hs);
  int64_t sym_cat[CAT_COUNT + 1];
  for (int c = 0; c <= CAT_COUNT; ++c) sym_cat[c] = (int64_t)h->h_pinned[kPinSymCat + c];
  for (int c = 0; c < CAT_COUNT; ++c) {
    h->st.bin_rows[0][c] = sym_cat[c + 1] - sym_cat[c];
    h->st.bin_nnza[0][c] = (int64_t)h->h_pinned[kPinBinSums + 3 * c];
    h->st.bin_products[0][c] = (int64_t)h->h_pinned[kPinBinSums + 3 * c + 1];
  }
  h->max_nnza = (int64_t)hs.max_nnza;
  h->st.products = (int64_t)hs.sum_prods;
  h->st.max_row_products = (int64_t)hs.max_prods;
  h->st.rows_direct = (int64_t)hs.n_direct;
  h->st.rows_empty = (int64_t)hs.n_empty;
  for (int c = 0; c < CAT_TINY; ++c) h->st.rows_per_bin_symbolic[c] = sym_cat[c + 1] - sym_cat[c];
  if ((st = timing_mark(h, 1, s))) return st;

  // resume scratch for multi-window dense rows (largest configuration, one CTA per SM)
  if ((st = ensure(h, h->resume, (size_t)h->num_smid * 2 * (size_t)std::max<int64_t>(h->max_nnza, 1) * 4, s))) return st;

  // ---- 2. symbolic global load balancing decision + binning --------------------------
  const int cfg_max_sym = cfg_for(bps, (int64_t)hs.max_prods);
  const int lb_sym = decide_lb(kLbSym, h->opt_lb_sym, (double)hs.max_prods, (double)hs.sum_prods, m, cfg_max_sym,
                               cfg_max_sym >= kNumCfg - 1 || h->opt_force_acc == 2);
  h->st.lb_symbolic = lb_sym;
  if (h->seg_enabled && lb_sym) {
    // long-row candidates = the symbolic bin of the largest configuration
    h->cand_start = sym_cat[CAT_CFG0 + kNumCfg - 1];
    h->n_cand = sym_cat[CAT_CFG0 + kNumCfg] - h->cand_start;
    const size_t bytes = (size_t)h->n_cand * (size_t)h->nchunks * 4;
    if (h->n_cand > 0 && (bytes > ((size_t)4 << 30) || ensure(h, h->chunk_cnt, bytes, s) != SPECK_OK)) {
      (void)cudaGetLastError();
      h->seg_enabled = false;   // too many candidates for the chunk table: dense windows instead
      h->n_cand = 0;
    }
  } else {
    h->n_cand = 0;
  }
  // bitmap reuse: will the numeric long rows go to k_long_bitmap (seg_plan_args), and does every
  // row's column range fit its bitmap?  Then the symbolic dense rows keep their bitmaps.
  h->bm_enabled = false;
  if (h->seg_enabled && h->n_cand > 0 && h->opt_bitmap_reuse && h->opt_long_bitmap && B->cols <= kBitmapMaxCols &&
      (h->opt_long_bitmap == 2 || !(h->n_cand < 4 * (int64_t)h->num_sms && h->max_nnza < kSegMaxNnzA))) {
    const size_t per_row = ((size_t)(B->cols + 31) / 32 + 4) * 4;
    size_t want = ((size_t)h->n_cand * per_row + 15) & ~(size_t)15;
    if (want > h->bm_pool.cap) {
      // growing: cap the pool at a quarter of the free memory (C is allocated after analyze);
      // the query is slow, so it only happens when the pool grows
      size_t free_b = 0, tot_b = 0;
      CK(cudaMemGetInfo(&free_b, &tot_b));
      want = std::min<size_t>(want, (free_b + h->bm_pool.cap) / 4) & ~(size_t)15;
      if (want < h->bm_pool.cap) want = h->bm_pool.cap;
    }
    if (want >= ((size_t)1 << 20) && ensure(h, h->bm_pool, want, s, true) == SPECK_OK &&
        ensure(h, h->bm_off, (size_t)h->n_cand * 8, s) == SPECK_OK) {
      CK(cudaMemsetAsync(h->bm_off.p, 0xFF, (size_t)h->n_cand * 8, s));
      CK(cudaMemsetAsync(static_cast<char*>(h->small.p) + 2048, 0, 8, s));
      h->bm_pool_words = h->bm_pool.cap / 4;
      h->bm_enabled = true;
    } else {
      (void)cudaGetLastError();
    }
  }
  SpgemmArgs<V> a = base_args<V>(h, A, B);
  if (lb_sym) {
    kt = kt_begin(h, s, SPECK_KERNEL_BINNING, 1, -1);
    k_bin_scatter<<<(unsigned)tiles, kBinTile, 0, s>>>(A->row_ptr, static_cast<int64_t*>(h->prods.p), nullptr, m, bps,
                                                      static_cast<int64_t*>(h->hist_off.p), tiles,
                                                      static_cast<int32_t*>(h->bins.p), static_cast<int64_t*>(h->cnt.p));
    CKL();
    kt_end(h, s, kt);
  }
  if ((st = timing_mark(h, 2, s))) return st;
  // ---- 3. symbolic SpGEMM -------------------------------------------------------------
  if ((st = run_pass<V>(h, 0, lb_sym, sym_cat, sym_cat + 1, a, (int64_t)hs.max_prods, bps, s))) return st;
  if ((st = timing_mark(h, 3, s))) return st;
  // ---- 4. prefix sum -> C row offsets; numeric classification -------------------------
  unsigned long long* dmax = reinterpret_cast<unsigned long long*>(static_cast<char*>(h->small.p) + 128);
  kt = kt_begin(h, s, SPECK_KERNEL_SCAN, 0, -1);
  if ((st = launch_scan(h, static_cast<int64_t*>(h->cnt.p), m, C_rp, dmax, s))) return st;
  kt_end(h, s, kt);
  if ((st = timing_mark(h, 4, s))) return st;
  const BinParams bpn = make_bin_params(h, 1);
  kt = kt_begin(h, s, SPECK_KERNEL_BINNING, 2, -1);
  k_classify<<<(unsigned)tiles, kBinTile, 0, s>>>(A->row_ptr, static_cast<int64_t*>(h->prods.p), C_rp, m, bpn,
                                                 static_cast<int64_t*>(h->hist.p), tiles, bin_sums + CAT_COUNT * 3);
  CKL();
  if ((st = launch_scan(h, static_cast<int64_t*>(h->hist.p), tiles * CAT_COUNT, static_cast<int64_t*>(h->hist_off.p),
                        nullptr, s)))
    return st;
  kt_end(h, s, kt);
  // numeric long rows: segments per candidate (exact sizes from the symbolic chunk counts)
  if (h->seg_enabled && h->n_cand > 0) {
    const int64_t nc = h->n_cand;
    if ((st = ensure(h, h->cand, (size_t)nc * 4, s))) return st;
    if ((st = ensure(h, h->nseg, (size_t)nc * 8, s))) return st;
    if ((st = ensure(h, h->seg_off, (size_t)(nc + 1) * 8, s))) return st;
    CK(cudaMemcpyAsync(h->cand.p, static_cast<int32_t*>(h->bins.p) + h->cand_start, (size_t)nc * 4,
                       cudaMemcpyDeviceToDevice, s));
    kt = kt_begin(h, s, SPECK_KERNEL_SEG_PLAN, 0, -1);
    k_seg_count<<<(unsigned)((nc + 127) / 128), 128, 0, s>>>(seg_plan_args<V>(h, C_rp),
                                                            static_cast<int64_t*>(h->nseg.p));
    CKL();
    if ((st = launch_scan(h, static_cast<int64_t*>(h->nseg.p), nc, static_cast<int64_t*>(h->seg_off.p), nullptr, s)))
      return st;
    kt_end(h, s, kt);
  }
  {
    unsigned long long* hp = h->h_pinned;
    CK(cudaMemcpyAsync(hp, C_rp + m, 8, cudaMemcpyDeviceToHost, s));
    CK(cudaMemcpyAsync(hp + 1, dmax, 8, cudaMemcpyDeviceToHost, s));
    hp[2] = 0;
    if (h->seg_enabled && h->n_cand > 0)
      CK(cudaMemcpyAsync(hp + 2, static_cast<int64_t*>(h->seg_off.p) + h->n_cand, 8, cudaMemcpyDeviceToHost, s));
    for (int c = 0; c <= CAT_COUNT; ++c)
      CK(cudaMemcpyAsync(hp + kPinSymCat + c, static_cast<int64_t*>(h->hist_off.p) + (int64_t)c * tiles, 8,
                         cudaMemcpyDeviceToHost, s));
    CK(cudaMemcpyAsync(hp + kPinBinSums + CAT_COUNT * 3, bin_sums + CAT_COUNT * 3, CAT_COUNT * 3 * 8,
                       cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));  // sync #2
  }
  h->nnz_c = (int64_t)h->h_pinned[0];
  h->max_cnt = (int64_t)h->h_pinned[1];
  h->n_segs = (int64_t)h->h_pinned[2];
  h->st.segments = h->n_segs;
  for (int c = 0; c <= CAT_COUNT; ++c) h->num_cat_start[c] = (int64_t)h->h_pinned[kPinSymCat + c];
  for (int c = 0; c < CAT_COUNT; ++c) {
    h->st.bin_rows[1][c] = h->num_cat_start[c + 1] - h->num_cat_start[c];
    h->st.bin_nnza[1][c] = (int64_t)h->h_pinned[kPinBinSums + CAT_COUNT * 3 + 3 * c];
    h->st.bin_products[1][c] = (int64_t)h->h_pinned[kPinBinSums + CAT_COUNT * 3 + 3 * c + 1];
    h->st.bin_nnzc[c] = (int64_t)h->h_pinned[kPinBinSums + CAT_COUNT * 3 + 3 * c + 2];
  }
  for (int c = 0; c < CAT_TINY; ++c) h->st.rows_per_bin_numeric[c] = h->num_cat_start[c + 1] - h->num_cat_start[c];
  // the stats keep one smallest-configuration count (tiny rows included)
  h->st.rows_per_bin_numeric[CAT_CFG0] += h->num_cat_start[CAT_TINY + 1] - h->num_cat_start[CAT_TINY];
  *nnz_c = h->nnz_c;
  h->st.nnz_c = h->nnz_c;
  if (h->opt_timing) {
    h->st.ms_analysis = elapsed(h, 0, 1);
    h->st.ms_symbolic_lb = elapsed(h, 1, 2);
    h->st.ms_symbolic = elapsed(h, 2, 3);
    h->st.ms_scan = elapsed(h, 3, 4);
  }
  h->analyzed = true;
  h->num_binned = false;
  return SPECK_OK;
}

// Numeric phase of the rows [r0, r1) only (speck_spgemm_rows): the numeric bins (scattered once
// per analysis) are cut to the chunk's rows by binary search, C pointers are shifted so that the
// kernels' absolute C offsets land in the caller's chunk buffers, and long-row jobs of other
// rows exit immediately.  The global load balancer is always on in this mode.
template <typename V>
speck_status_t spgemm_rows_impl(speck_handle_t h, const speck_csr_t* A, const speck_csr_t* B, const int64_t* C_rp,
                                int64_t r0, int64_t r1, int32_t* C_col, V* C_val, cudaStream_t s) {
  const int64_t m = A->rows;
  if (r1 <= r0 || h->nnz_c == 0) return SPECK_OK;
  const int64_t tiles = (m + kBinTile - 1) / kBinTile;
  const BinParams bpn = make_bin_params(h, 1);
  h->st.lb_numeric = 1;
  if (!h->num_binned) {
    const int kt = kt_begin(h, s, SPECK_KERNEL_BINNING, 3, -1);
    k_bin_scatter<<<(unsigned)tiles, kBinTile, 0, s>>>(A->row_ptr, static_cast<int64_t*>(h->prods.p), C_rp, m, bpn,
                                                      static_cast<int64_t*>(h->hist_off.p), tiles,
                                                      static_cast<int32_t*>(h->bins.p), nullptr);
    CKL();
    kt_end(h, s, kt);
    h->num_binned = true;
  }
  CatStarts cs;
  for (int c = 0; c <= CAT_COUNT; ++c) cs.s[c] = h->num_cat_start[c];
  int64_t* d_out = reinterpret_cast<int64_t*>(static_cast<char*>(h->small.p) + kSmallRange);
  k_bin_range<<<1, 32, 0, s>>>(static_cast<const int32_t*>(h->bins.p), cs, r0, r1, C_rp, d_out);
  CKL();
  unsigned long long* hp = h->h_pinned + kPinRange;
  CK(cudaMemcpyAsync(hp, d_out, (2 * CAT_COUNT + 2) * 8, cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  int64_t beg[CAT_COUNT], end[CAT_COUNT];
  for (int c = 0; c < CAT_COUNT; ++c) { beg[c] = (int64_t)hp[2 * c]; end[c] = (int64_t)hp[2 * c + 1]; }
  const int64_t off = (int64_t)hp[2 * CAT_COUNT];
  unsigned long long* ndense = reinterpret_cast<unsigned long long*>(static_cast<char*>(h->small.p) + 256);
  CK(cudaMemsetAsync(ndense, 0, 8, s));
  SpgemmArgs<V> a = base_args<V>(h, A, B);
  a.C_rp = C_rp;
  a.C_col = C_col - off;     // the kernels write C[C_rp[row] + t]; the chunk buffer starts at C_rp[r0]
  a.C_val = C_val - off;
  a.row_lo = r0;
  a.row_hi = r1;
  return run_pass<V>(h, 1, 1, beg, end, a, h->max_cnt, bpn, s);
}

// Device CSR transpose (transpose_kernels.cuh).
template <typename V>
speck_status_t transpose_impl(speck_handle_t h, const speck_csr_t* A, int64_t* T_rp, int32_t* T_col, V* T_val,
                              cudaStream_t s) {
  const int64_t n = A->cols, nnz = A->nnz;
  speck_status_t st;
  if ((st = ensure(h, h->small, 4096, s))) return st;
  if ((st = ensure(h, h->tr_cnt, (size_t)(n + 1) * 8, s))) return st;
  unsigned long long* cnt = static_cast<unsigned long long*>(h->tr_cnt.p);
  CK(cudaMemsetAsync(cnt, 0, (size_t)(n + 1) * 8, s));
  const unsigned grid = (unsigned)std::max<int64_t>(1, std::min<int64_t>((nnz + kTrThreads - 1) / kTrThreads, (int64_t)h->num_sms * 16));
  if (nnz > 0) {
    k_tr_count<<<grid, kTrThreads, 0, s>>>(A->col_idx, nnz, cnt);
    CKL();
  }
  unsigned long long* dmax = reinterpret_cast<unsigned long long*>(static_cast<char*>(h->small.p) + 3968);
  CK(cudaMemsetAsync(dmax, 0, 8, s));
  if ((st = launch_scan(h, reinterpret_cast<const int64_t*>(cnt), n, T_rp, dmax, s))) return st;
  if (nnz == 0) return SPECK_OK;
  CK(cudaMemcpyAsync(cnt, T_rp, (size_t)n * 8, cudaMemcpyDeviceToDevice, s));   // cursors
  const unsigned wgrid = (unsigned)std::max<int64_t>(1, std::min<int64_t>((A->rows * 32 + kTrThreads - 1) / kTrThreads, (int64_t)h->num_sms * 16));
  k_tr_scatter<V><<<wgrid, kTrThreads, 0, s>>>(A->row_ptr, A->col_idx, static_cast<const V*>(A->values), A->rows, cnt,
                                               T_col, T_val);
  CKL();
  const unsigned tgrid = (unsigned)std::max<int64_t>(1, std::min<int64_t>((n * 32 + kTrThreads - 1) / kTrThreads, (int64_t)h->num_sms * 16));
  k_tr_sort_warp<V><<<tgrid, kTrThreads, 0, s>>>(T_rp, n, T_col, T_val);
  CKL();
  // longer rows: list them with their tile counts (two lists: > 32 entries, > one tile)
  unsigned long long hmax = 0;
  CK(cudaMemcpyAsync(h->h_pinned + kPinRange, dmax, 8, cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  hmax = h->h_pinned[kPinRange];
  for (int stage = 0; stage < 2; ++stage) {
    const int64_t lo = stage == 0 ? 32 : kTrSmemSort;
    if ((int64_t)hmax <= lo) break;
    if ((st = ensure(h, h->tr_list, (size_t)n * 4 + (size_t)(n + 1) * 8 + 64, s))) return st;
    int32_t* list = static_cast<int32_t*>(h->tr_list.p);
    int64_t* tiles = reinterpret_cast<int64_t*>(static_cast<char*>(h->tr_list.p) + (((size_t)n * 4 + 15) & ~(size_t)15));
    int64_t* first = reinterpret_cast<int64_t*>(cnt);   // cursors are no longer needed: tile prefix
    unsigned long long* nl = dmax + 1;
    CK(cudaMemsetAsync(nl, 0, 8, s));
    k_tr_list<<<tgrid, kTrThreads, 0, s>>>(T_rp, n, lo, list, tiles, nl);
    CKL();
    CK(cudaMemcpyAsync(h->h_pinned + kPinRange + 1, nl, 8, cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    const int64_t nrows = (int64_t)h->h_pinned[kPinRange + 1];
    if ((st = launch_scan(h, tiles, nrows, first, nullptr, s))) return st;
    CK(cudaMemcpyAsync(h->h_pinned + kPinRange + 2, first + nrows, 8, cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    const int64_t ntiles = (int64_t)h->h_pinned[kPinRange + 2];
    if (stage == 0) {
      const size_t sm = (size_t)kTrSmemSort * (4 + sizeof(V));
      k_tr_sort_block<V><<<(unsigned)ntiles, 1024, sm, s>>>(T_rp, list, first, nrows, T_col, T_val);
      CKL();
      continue;
    }
    // rows longer than a tile: merge rounds, ping-pong with a scratch copy of T
    if ((st = ensure(h, h->tr_col, (size_t)nnz * 4, s))) return st;
    if ((st = ensure(h, h->tr_val, (size_t)nnz * sizeof(V), s))) return st;
    int32_t* c0 = T_col; V* v0 = T_val;
    int32_t* c1 = static_cast<int32_t*>(h->tr_col.p); V* v1 = T_val ? static_cast<V*>(h->tr_val.p) : nullptr;
    int rounds = 0;
    for (int64_t L = kTrSmemSort; L < (int64_t)hmax; L *= 2, ++rounds) {
      k_tr_merge<V><<<(unsigned)ntiles, 256, 0, s>>>(T_rp, list, first, nrows, L, c0, v0, c1, v1);
      CKL();
      std::swap(c0, c1);
      std::swap(v0, v1);
    }
    if (rounds & 1) {   // result in the scratch copy: one copying round (a single run per pair) back
      k_tr_merge<V><<<(unsigned)ntiles, 256, 0, s>>>(T_rp, list, first, nrows, (int64_t)1 << 40, c0, v0, c1, v1);
      CKL();
    }
  }
  return SPECK_OK;
}

template <typename V>
speck_status_t spgemm_impl(speck_handle_t h, const speck_csr_t* A, const speck_csr_t* B, const int64_t* C_rp,
                           int32_t* C_col, V* C_val, cudaStream_t s) {
  const int64_t m = A->rows;
  if (m == 0 || h->nnz_c == 0) return SPECK_OK;
  speck_status_t st;
  const int64_t tiles = (m + kBinTile - 1) / kBinTile;
  const BinParams bpn = make_bin_params(h, 1);
  const int cfg_max = cfg_for(bpn, h->max_cnt);
  const int lb = decide_lb(kLbNum, h->opt_lb_num, (double)h->max_cnt, (double)h->nnz_c, m, cfg_max,
                           cfg_max >= kNumCfg - 1 || h->opt_force_acc == 2 || h->opt_det);
  h->st.lb_numeric = lb;
  h->lb_num = lb;
  if ((st = timing_mark(h, 5, s))) return st;
  unsigned long long* ndense = reinterpret_cast<unsigned long long*>(static_cast<char*>(h->small.p) + 256);
  CK(cudaMemsetAsync(ndense, 0, 8, s));
  if (lb) {
    const int kt = kt_begin(h, s, SPECK_KERNEL_BINNING, 3, -1);
    k_bin_scatter<<<(unsigned)tiles, kBinTile, 0, s>>>(A->row_ptr, static_cast<int64_t*>(h->prods.p), C_rp, m, bpn,
                                                      static_cast<int64_t*>(h->hist_off.p), tiles,
                                                      static_cast<int32_t*>(h->bins.p), nullptr);
    CKL();
    kt_end(h, s, kt);
  }
  if ((st = timing_mark(h, 6, s))) return st;
  SpgemmArgs<V> a = base_args<V>(h, A, B);
  a.C_rp = C_rp;
  a.C_col = C_col;
  a.C_val = C_val;
  if ((st = run_pass<V>(h, 1, lb, h->num_cat_start, h->num_cat_start + 1, a, h->max_cnt, bpn, s))) return st;
  if ((st = timing_mark(h, 7, s))) return st;
  // numeric-stage times and counters are read lazily by speck_get_stats (no sync here)
  if (h->opt_timing) CK(cudaMemcpyAsync(h->h_pinned + 40, ndense, 8, cudaMemcpyDeviceToHost, s));
  h->numeric_pending = h->opt_timing != 0;
  return SPECK_OK;
}

bool same_problem(speck_handle_t h, const speck_csr_t* A, const speck_csr_t* B) {
  return h->analyzed && h->A_rp == A->row_ptr && h->A_col == A->col_idx && h->A_rows == A->rows && h->A_cols == A->cols &&
         h->A_nnz == A->nnz && h->B_rp == B->row_ptr && h->B_col == B->col_idx && h->B_rows == B->rows &&
         h->B_cols == B->cols && h->B_nnz == B->nnz && h->dtype == A->dtype;
}

// component kernels -------------------------------------------------------------------
__global__ void k_block_merge_groups(const int64_t* needs, int64_t n, int64_t cap, uint8_t* flags) {
  const int64_t g0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) / 32 * 32;
  if (g0 >= n) return;
  const int ne = (int)(n - g0 < 32 ? n - g0 : 32);
  const int l = lane_id();
  const int64_t need = l < ne ? needs[g0 + l] : 0;
  const uint32_t st = warp_block_merge(need, ne, cap);
  if (l < ne) flags[g0 + l] = (st >> l) & 1u;
}

__global__ void k_query_nsmid(int* out) { *out = (int)nsmid(); }


__global__ void k_group_size(int32_t T, const int64_t* nnzA, const int64_t* prods, const int64_t* maxlen, int64_t n,
                             int32_t* g) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) g[i] = local_group_size(T, nnzA[i], prods[i], maxlen[i]);
}

__global__ void k_hash_probe(const uint32_t* keys, const uint32_t* homes, int64_t n, int32_t size, uint32_t* out_keys,
                             uint32_t* out_counts) {
  extern __shared__ uint32_t sm[];
  uint32_t* sk = sm;
  uint32_t* sc = sm + size;
  for (int i = threadIdx.x; i < size; i += blockDim.x) { sk[i] = kEmptyKey; sc[i] = 0; }
  __syncthreads();
  if (threadIdx.x == 0) {
    // the pipeline's probe_insert_mono (numeric maps of scrambled rows) with the home slot
    // injected instead of hash_slot()
    int wrapped = 0;
    for (int64_t i = 0; i < n; ++i) {
      const uint32_t s = probe_insert_mono(sk, (uint32_t)size, homes[i] % (uint32_t)size, keys[i], &wrapped);
      atomicAdd(&sc[s], 1u);
    }
  }
  __syncthreads();
  for (int i = threadIdx.x; i < size; i += blockDim.x) { out_keys[i] = sk[i]; out_counts[i] = sc[i]; }
}

}  // namespace

// ======================================================================================
// C ABI
// ======================================================================================
extern "C" {

const char* speck_version(void) { return SPECK_VERSION; }

const char* speck_status_string(speck_status_t s) {
  switch (s) {
    case SPECK_OK: return "SPECK_OK";
    case SPECK_ERR_INVALID_ARGUMENT: return "SPECK_ERR_INVALID_ARGUMENT";
    case SPECK_ERR_DIMENSION_MISMATCH: return "SPECK_ERR_DIMENSION_MISMATCH";
    case SPECK_ERR_DTYPE_MISMATCH: return "SPECK_ERR_DTYPE_MISMATCH";
    case SPECK_ERR_UNSUPPORTED: return "SPECK_ERR_UNSUPPORTED";
    case SPECK_ERR_OUT_OF_MEMORY: return "SPECK_ERR_OUT_OF_MEMORY";
    case SPECK_ERR_CUDA: return "SPECK_ERR_CUDA";
    case SPECK_ERR_NOT_ANALYZED: return "SPECK_ERR_NOT_ANALYZED";
    case SPECK_ERR_INVALID_INPUT: return "SPECK_ERR_INVALID_INPUT";
  }
  return "SPECK_ERR_UNKNOWN";
}

const char* speck_last_error(speck_handle_t h) { return h ? h->err.c_str() : "null handle"; }

speck_status_t speck_create(speck_handle_t* out, int device) {
  if (!out) return SPECK_ERR_INVALID_ARGUMENT;
  *out = nullptr;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev) {
    (void)cudaGetLastError();
    return SPECK_ERR_CUDA;
  }
  speck_handle_t h = new (std::nothrow) speck_handle_s();
  if (!h) return SPECK_ERR_OUT_OF_MEMORY;
  h->device = device;
  int prev = 0;
  cudaGetDevice(&prev);
  if (cudaSetDevice(device) != cudaSuccess) { delete h; return SPECK_ERR_CUDA; }
  cudaDeviceGetAttribute(&h->num_sms, cudaDevAttrMultiProcessorCount, device);
  bool ok = cudaHostAlloc(&h->h_pinned, kPinnedWords * 8, cudaHostAllocDefault) == cudaSuccess;
  for (int i = 0; i < kMaxStreams && ok; ++i) ok = cudaStreamCreateWithFlags(&h->streams[i], cudaStreamNonBlocking) == cudaSuccess;
  ok = ok && cudaEventCreateWithFlags(&h->ev_fork, cudaEventDisableTiming) == cudaSuccess;
  for (int i = 0; i < kMaxStreams && ok; ++i) ok = cudaEventCreateWithFlags(&h->ev_join[i], cudaEventDisableTiming) == cudaSuccess;
  for (int i = 0; i < 8 && ok; ++i) ok = cudaEventCreate(&h->ev_t[i]) == cudaSuccess;
  for (int i = 0; i < 2 * kMaxTimed && ok; ++i) ok = cudaEventCreate(&h->kt_ev[i]) == cudaSuccess;
  if (ok) ok = set_smem_attrs<float>(h) == SPECK_OK && set_smem_attrs<double>(h) == SPECK_OK;
  if (ok) {
    // %nsmid bounds %smid (it may exceed the SM count): it sizes the per-SM resume slots
    int* d = nullptr;
    ok = cudaMalloc(&d, sizeof(int)) == cudaSuccess;
    if (ok) {
      k_query_nsmid<<<1, 1>>>(d);
      int v = 0;
      ok = cudaMemcpy(&v, d, sizeof(int), cudaMemcpyDeviceToHost) == cudaSuccess;
      if (ok) h->num_smid = std::max(v, h->num_sms);
      cudaFree(d);
    }
  }
  cudaSetDevice(prev);
  if (!ok) {
    (void)cudaGetLastError();
    speck_destroy(h);
    return SPECK_ERR_CUDA;
  }
  *out = h;
  return SPECK_OK;
}

speck_status_t speck_destroy(speck_handle_t h) {
  if (!h) return SPECK_ERR_INVALID_ARGUMENT;
  int prev = 0;
  cudaGetDevice(&prev);
  cudaSetDevice(h->device);
  cudaDeviceSynchronize();
  Buf* bufs[] = {&h->prods, &h->maxlen, &h->colmin, &h->colmax, &h->cnt, &h->hist, &h->hist_off, &h->bins, &h->stats,
                 &h->scan_status, &h->resume, &h->small, &h->ana_long, &h->chunk_cnt, &h->cand, &h->nseg,
                 &h->seg_off, &h->segs, &h->bm_pool, &h->bm_off, &h->binfo, &h->paths, &h->chunks, &h->tr_cnt,
                 &h->tr_list, &h->tr_col, &h->tr_val, &h->det_scratch};
  for (Buf* b : bufs) {
    if (!b->p) continue;
    if (h->urelease) h->urelease(b->p, nullptr, h->uctx);
    else cudaFree(b->p);
  }
  if (h->h_pinned) cudaFreeHost(h->h_pinned);
  for (int i = 0; i < kMaxStreams; ++i) {
    if (h->streams[i]) cudaStreamDestroy(h->streams[i]);
    if (h->ev_join[i]) cudaEventDestroy(h->ev_join[i]);
  }
  if (h->ev_fork) cudaEventDestroy(h->ev_fork);
  for (int i = 0; i < 8; ++i)
    if (h->ev_t[i]) cudaEventDestroy(h->ev_t[i]);
  for (int i = 0; i < 2 * kMaxTimed; ++i)
    if (h->kt_ev[i]) cudaEventDestroy(h->kt_ev[i]);
  (void)cudaGetLastError();
  cudaSetDevice(prev);
  delete h;
  return SPECK_OK;
}

speck_status_t speck_set_option(speck_handle_t h, int option, int64_t v) {
  if (!h) return SPECK_ERR_INVALID_ARGUMENT;
  // every option except these shapes the plan speck_analyze builds (bins, long-row jobs,
  // bitmap pool): changing it invalidates the analysis, so a following speck_spgemm fails with
  // SPECK_ERR_NOT_ANALYZED instead of running kernels on a stale plan
  if (option != SPECK_OPT_STAGE_TIMING && option != SPECK_OPT_CONCURRENT_STREAMS &&
      option != SPECK_OPT_GLOBAL_LB_NUMERIC && option != SPECK_OPT_VALIDATE && option != SPECK_OPT_KERNEL_TIMING &&
      option != SPECK_OPT_PATH_COUNTERS)
    h->analyzed = false;
  switch (option) {
    case SPECK_OPT_GLOBAL_LB_SYMBOLIC: h->opt_lb_sym = v; break;
    case SPECK_OPT_GLOBAL_LB_NUMERIC: h->opt_lb_num = v; break;
    case SPECK_OPT_FORCE_ACCUMULATOR:
      if (v < 0 || v > 2) return fail(h, SPECK_ERR_INVALID_ARGUMENT, "FORCE_ACCUMULATOR must be 0..2");
      h->opt_force_acc = v; break;
    case SPECK_OPT_DENSE_WINDOW:
      if (v < 0) return fail(h, SPECK_ERR_INVALID_ARGUMENT, "DENSE_WINDOW must be >= 0");
      h->opt_dense_window = v; break;
    case SPECK_OPT_STAGE_TIMING: h->opt_timing = v; break;
    case SPECK_OPT_VALIDATE: h->opt_validate = v; break;
    case SPECK_OPT_DISABLE_DIRECT: h->opt_disable_direct = v; break;
    case SPECK_OPT_FIXED_GROUP_SIZE:
      if (v < -1 || v > 1024 || (v > 0 && (v & (v - 1))))
        return fail(h, SPECK_ERR_INVALID_ARGUMENT, "FIXED_GROUP_SIZE must be -1, 0 or a power of two <= 1024");
      h->opt_fixed_g = v; break;
    case SPECK_OPT_CONCURRENT_STREAMS:
      if (v < 1 || v > kMaxStreams) return fail(h, SPECK_ERR_INVALID_ARGUMENT, "CONCURRENT_STREAMS must be 1..8");
      h->opt_streams = v; break;
    case SPECK_OPT_SEGMENTS: h->opt_segments = v; break;
    case SPECK_OPT_WARP_ROWS: h->opt_warp_rows = v; break;
    case SPECK_OPT_LONG_BITMAP: h->opt_long_bitmap = v; break;
    case SPECK_OPT_BITMAP_REUSE: h->opt_bitmap_reuse = v; break;
    case SPECK_OPT_KERNEL_TIMING: h->opt_ktime = v; break;
    case SPECK_OPT_DETERMINISTIC: h->opt_det = v ? 1 : 0; break;
    case SPECK_OPT_BUCKET_SORT:
      if (v < 0 || v > 2) return fail(h, SPECK_ERR_INVALID_ARGUMENT, "BUCKET_SORT must be 0..2");
      h->opt_esc = v; break;
    case SPECK_OPT_PATH_COUNTERS: {
      h->opt_paths = v;
      std::memset(h->st.path_rows, 0, sizeof h->st.path_rows);
      if (v) {
        speck_status_t r = ensure(h, h->paths, SPECK_PATH_COUNT * 8, nullptr);
        if (r) return r;
        if (cudaMemset(h->paths.p, 0, SPECK_PATH_COUNT * 8) != cudaSuccess)
          return fail(h, SPECK_ERR_CUDA, "cannot clear the path counters");
      }
      break;
    }
    default: return fail(h, SPECK_ERR_INVALID_ARGUMENT, "unknown option %d", option);
  }
  return SPECK_OK;
}

speck_status_t speck_analyze(speck_handle_t h, const speck_csr_t* A, const speck_csr_t* B, int64_t* C_rp, int64_t* nnz_c,
                             speck_stream_t stream) {
  if (!h) return SPECK_ERR_INVALID_ARGUMENT;
  h->err.clear();
  speck_status_t st;
  if ((st = check_csr(h, A, "A", false)) || (st = check_csr(h, B, "B", false))) return st;
  if (!nnz_c) return fail(h, SPECK_ERR_INVALID_ARGUMENT, "nnz_c is NULL");
  if (!C_rp) return fail(h, SPECK_ERR_INVALID_ARGUMENT, "C_row_ptr is NULL");
  if (A->cols != B->rows) return fail(h, SPECK_ERR_DIMENSION_MISMATCH, "A.cols (%lld) != B.rows (%lld)", (long long)A->cols, (long long)B->rows);
  if (A->dtype != B->dtype) return fail(h, SPECK_ERR_DTYPE_MISMATCH, "A and B value types differ");
  int prev = 0;
  cudaGetDevice(&prev);
  if (cudaSetDevice(h->device) != cudaSuccess) return fail(h, SPECK_ERR_CUDA, "cudaSetDevice failed");
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  st = A->dtype == SPECK_F64 ? analyze_impl<double>(h, A, B, C_rp, nnz_c, s) : analyze_impl<float>(h, A, B, C_rp, nnz_c, s);
  cudaSetDevice(prev);
  return st;
}

speck_status_t speck_spgemm(speck_handle_t h, const speck_csr_t* A, const speck_csr_t* B, const int64_t* C_rp,
                            int32_t* C_col, void* C_val, speck_stream_t stream) {
  if (!h) return SPECK_ERR_INVALID_ARGUMENT;
  h->err.clear();
  speck_status_t st;
  if ((st = check_csr(h, A, "A", true)) || (st = check_csr(h, B, "B", true))) return st;
  if (A->cols != B->rows) return fail(h, SPECK_ERR_DIMENSION_MISMATCH, "A.cols != B.rows");
  if (A->dtype != B->dtype) return fail(h, SPECK_ERR_DTYPE_MISMATCH, "A and B value types differ");
  if (!same_problem(h, A, B)) return fail(h, SPECK_ERR_NOT_ANALYZED, "speck_spgemm without a matching speck_analyze");
  if (h->nnz_c > 0 && (!C_rp || !C_col || !C_val)) return fail(h, SPECK_ERR_INVALID_ARGUMENT, "C arrays are NULL");
  int prev = 0;
  cudaGetDevice(&prev);
  if (cudaSetDevice(h->device) != cudaSuccess) return fail(h, SPECK_ERR_CUDA, "cudaSetDevice failed");
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  st = A->dtype == SPECK_F64 ? spgemm_impl<double>(h, A, B, C_rp, C_col, static_cast<double*>(C_val), s)
                             : spgemm_impl<float>(h, A, B, C_rp, C_col, static_cast<float*>(C_val), s);
  cudaSetDevice(prev);
  return st;
}

speck_status_t speck_spgemm_rows(speck_handle_t h, const speck_csr_t* A, const speck_csr_t* B, const int64_t* C_rp,
                                 int64_t r0, int64_t r1, int32_t* C_col_part, void* C_val_part, speck_stream_t stream) {
  if (!h) return SPECK_ERR_INVALID_ARGUMENT;
  h->err.clear();
  speck_status_t st;
  if ((st = check_csr(h, A, "A", true)) || (st = check_csr(h, B, "B", true))) return st;
  if (A->cols != B->rows) return fail(h, SPECK_ERR_DIMENSION_MISMATCH, "A.cols != B.rows");
  if (A->dtype != B->dtype) return fail(h, SPECK_ERR_DTYPE_MISMATCH, "A and B value types differ");
  if (!same_problem(h, A, B)) return fail(h, SPECK_ERR_NOT_ANALYZED, "speck_spgemm_rows without a matching speck_analyze");
  if (r0 < 0 || r1 < r0 || r1 > A->rows) return fail(h, SPECK_ERR_INVALID_ARGUMENT, "row range [%lld, %lld) outside [0, %lld)",
                                                       (long long)r0, (long long)r1, (long long)A->rows);
  if (!C_rp || (h->nnz_c > 0 && r1 > r0 && (!C_col_part || !C_val_part)))
    return fail(h, SPECK_ERR_INVALID_ARGUMENT, "C arrays are NULL");
  int prev = 0;
  cudaGetDevice(&prev);
  if (cudaSetDevice(h->device) != cudaSuccess) return fail(h, SPECK_ERR_CUDA, "cudaSetDevice failed");
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  st = A->dtype == SPECK_F64 ? spgemm_rows_impl<double>(h, A, B, C_rp, r0, r1, C_col_part, static_cast<double*>(C_val_part), s)
                             : spgemm_rows_impl<float>(h, A, B, C_rp, r0, r1, C_col_part, static_cast<float*>(C_val_part), s);
  cudaSetDevice(prev);
  return st;
}

speck_status_t speck_transpose(speck_handle_t h, const speck_csr_t* A, int64_t* T_row_ptr, int32_t* T_col_idx,
                               void* T_values, speck_stream_t stream) {
  if (!h) return SPECK_ERR_INVALID_ARGUMENT;
  h->err.clear();
  speck_status_t st;
  if ((st = check_csr(h, A, "A", false))) return st;
  if (!T_row_ptr || (A->nnz > 0 && !T_col_idx)) return fail(h, SPECK_ERR_INVALID_ARGUMENT, "T arrays are NULL");
  if (A->nnz > 0 && !T_values != !A->values)
    return fail(h, SPECK_ERR_INVALID_ARGUMENT, "T_values must be given exactly when A.values is");
  int prev = 0;
  cudaGetDevice(&prev);
  if (cudaSetDevice(h->device) != cudaSuccess) return fail(h, SPECK_ERR_CUDA, "cudaSetDevice failed");
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  st = A->dtype == SPECK_F64 ? transpose_impl<double>(h, A, T_row_ptr, T_col_idx, static_cast<double*>(T_values), s)
                             : transpose_impl<float>(h, A, T_row_ptr, T_col_idx, static_cast<float*>(T_values), s);
  cudaSetDevice(prev);
  return st;
}

speck_status_t speck_row_chunks(speck_handle_t h, const int64_t* C_rp, int64_t rows, int64_t max_nnz, int64_t* bounds,
                                int64_t max_parts, int64_t* n_parts) {
  if (!h || !C_rp || !bounds || !n_parts || rows < 0 || max_parts < 1) return SPECK_ERR_INVALID_ARGUMENT;
  h->err.clear();
  if (!h->analyzed || rows != h->A_rows) return fail(h, SPECK_ERR_NOT_ANALYZED, "speck_row_chunks needs the analysis of C_row_ptr");
  const int64_t step = max_nnz - h->max_cnt;
  if (step <= 0)
    return fail(h, SPECK_ERR_INVALID_ARGUMENT, "max_nnz %lld does not exceed the longest row of C (%lld entries)",
                (long long)max_nnz, (long long)h->max_cnt);
  const int64_t parts = std::max<int64_t>(1, (h->nnz_c + step - 1) / step);
  if (parts > max_parts) return fail(h, SPECK_ERR_INVALID_ARGUMENT, "%lld chunks needed, bounds holds %lld", (long long)parts, (long long)max_parts);
  int prev = 0;
  cudaGetDevice(&prev);
  cudaSetDevice(h->device);
  speck_status_t st;
  if ((st = ensure(h, h->chunks, (size_t)(parts + 1) * 8, nullptr))) { cudaSetDevice(prev); return st; }
  k_chunk_bounds<<<(unsigned)((parts + 1 + 127) / 128), 128>>>(C_rp, rows, step, parts, static_cast<int64_t*>(h->chunks.p));
  cudaError_t e = cudaMemcpy(bounds, h->chunks.p, (size_t)(parts + 1) * 8, cudaMemcpyDeviceToHost);
  cudaSetDevice(prev);
  if (e != cudaSuccess) return fail(h, SPECK_ERR_CUDA, "speck_row_chunks: %s", cudaGetErrorString(e));
  *n_parts = parts;
  return SPECK_OK;
}

speck_status_t speck_row_analysis(speck_handle_t h, const speck_csr_t* A, const speck_csr_t* B, int64_t* prods,
                                  int32_t* maxlen, int32_t* colmin, int32_t* colmax, speck_stream_t stream) {
  if (!h) return SPECK_ERR_INVALID_ARGUMENT;
  h->err.clear();
  speck_status_t st;
  if ((st = check_csr(h, A, "A", false)) || (st = check_csr(h, B, "B", false))) return st;
  if (A->cols != B->rows) return fail(h, SPECK_ERR_DIMENSION_MISMATCH, "A.cols != B.rows");
  const int64_t m = A->rows;
  if (m == 0) return SPECK_OK;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  int prev = 0;
  cudaGetDevice(&prev);
  cudaSetDevice(h->device);
  int64_t* pr = prods;
  if (!pr) {
    if ((st = ensure(h, h->prods, (size_t)m * 8, s))) { cudaSetDevice(prev); return st; }
    pr = static_cast<int64_t*>(h->prods.p);
  }
  st = run_analysis(h, A, B, pr, maxlen, colmin, colmax, nullptr, s);
  cudaSetDevice(prev);
  return st;
}

speck_status_t speck_row_products(speck_handle_t h, const speck_csr_t* A, const speck_csr_t* B, int64_t* prods,
                                  speck_stream_t stream) {
  if (!h) return SPECK_ERR_INVALID_ARGUMENT;
  if (!prods && A && A->rows > 0) return fail(h, SPECK_ERR_INVALID_ARGUMENT, "prods is NULL");
  return speck_row_analysis(h, A, B, prods, nullptr, nullptr, nullptr, stream);
}

speck_status_t speck_set_allocator(speck_handle_t h, speck_alloc_fn alloc, speck_release_fn release, void* ctx) {
  if (!h) return SPECK_ERR_INVALID_ARGUMENT;
  if ((alloc == nullptr) != (release == nullptr))
    return fail(h, SPECK_ERR_INVALID_ARGUMENT, "alloc and release must both be set or both be NULL");
  int prev = 0;
  cudaGetDevice(&prev);
  cudaSetDevice(h->device);
  cudaDeviceSynchronize();   // no kernel may still use the workspace being released
  Buf* bufs[] = {&h->prods, &h->maxlen, &h->colmin, &h->colmax, &h->cnt, &h->hist, &h->hist_off, &h->bins, &h->stats,
                 &h->scan_status, &h->resume, &h->small, &h->ana_long, &h->chunk_cnt, &h->cand, &h->nseg,
                 &h->seg_off, &h->segs, &h->bm_pool, &h->bm_off, &h->binfo, &h->paths, &h->chunks, &h->tr_cnt,
                 &h->tr_list, &h->tr_col, &h->tr_val, &h->det_scratch};
  for (Buf* b : bufs) release_buf(h, *b, nullptr);
  cudaStreamSynchronize(nullptr);
  h->ualloc = alloc;
  h->urelease = release;
  h->uctx = ctx;
  h->analyzed = false;
  cudaSetDevice(prev);
  return SPECK_OK;
}

speck_status_t speck_get_stats(speck_handle_t h, speck_stats_t* out) {
  if (!h || !out) return SPECK_ERR_INVALID_ARGUMENT;
  if (h->numeric_pending) {
    if (cudaEventSynchronize(h->ev_t[7]) != cudaSuccess) {
      (void)cudaGetLastError();
      return fail(h, SPECK_ERR_CUDA, "stage timing event failed");
    }
    h->st.ms_numeric_lb = elapsed(h, 5, 6);
    h->st.ms_numeric = elapsed(h, 6, 7);
    h->st.rows_dense_numeric = (int64_t)h->h_pinned[40];
    h->numeric_pending = false;
  }
  if (h->kt_pending) {
    for (int i = 0; i < h->kt_n; ++i) {
      float ms = -1.f;
      if (cudaEventSynchronize(h->kt_ev[2 * i + 1]) != cudaSuccess ||
          cudaEventElapsedTime(&ms, h->kt_ev[2 * i], h->kt_ev[2 * i + 1]) != cudaSuccess) {
        (void)cudaGetLastError();
        ms = -1.f;
      }
      h->kt_ms[i] = ms;
    }
    h->kt_pending = false;
  }
  h->st.n_kernels = h->kt_n;
  for (int i = 0; i < h->kt_n; ++i) {
    h->st.kernel_id[i] = h->kt_id[i];
    h->st.kernel_bin[i] = h->kt_bin[i];
    h->st.kernel_ms[i] = h->kt_ms[i];
  }
  if (h->opt_paths && h->paths.p) {
    unsigned long long pc[SPECK_PATH_COUNT];
    if (cudaMemcpy(pc, h->paths.p, sizeof pc, cudaMemcpyDeviceToHost) != cudaSuccess) {
      (void)cudaGetLastError();
      return fail(h, SPECK_ERR_CUDA, "cannot read the path counters");
    }
    for (int i = 0; i < SPECK_PATH_COUNT; ++i) h->st.path_rows[i] = (int64_t)pc[i];
  }
  h->st.workspace_bytes = ws_bytes(h);
  h->st.kernel_launches = h->launches;
  *out = h->st;
  return SPECK_OK;
}

speck_status_t speck_block_merge(speck_handle_t h, const int64_t* needs, int64_t n, int64_t cap, uint8_t* flags,
                                 speck_stream_t stream) {
  if (!h || (n > 0 && (!needs || !flags)) || n < 0) return SPECK_ERR_INVALID_ARGUMENT;
  if (n == 0) return SPECK_OK;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  const int64_t groups = (n + 31) / 32;
  k_block_merge_groups<<<(unsigned)((groups * 32 + 255) / 256), 256, 0, s>>>(needs, n, cap, flags);
  CKL();
  return SPECK_OK;
}

speck_status_t speck_group_size(speck_handle_t h, int32_t T, const int64_t* nnzA, const int64_t* prods, const int64_t* maxlen,
                                int64_t n, int32_t* g, speck_stream_t stream) {
  if (!h || n < 0 || T <= 0 || (n > 0 && (!nnzA || !prods || !maxlen || !g))) return SPECK_ERR_INVALID_ARGUMENT;
  if (n == 0) return SPECK_OK;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  k_group_size<<<(unsigned)((n + 255) / 256), 256, 0, s>>>(T, nnzA, prods, maxlen, n, g);
  CKL();
  return SPECK_OK;
}

speck_status_t speck_hash_probe(speck_handle_t h, const uint32_t* keys, const uint32_t* homes, int64_t n, int32_t size,
                                uint32_t* slot_keys, uint32_t* slot_counts, speck_stream_t stream) {
  if (!h || size <= 0 || size > 8192 || n < 0 || (n > 0 && (!keys || !homes)) || !slot_keys || !slot_counts)
    return SPECK_ERR_INVALID_ARGUMENT;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  k_hash_probe<<<1, 128, (size_t)size * 8, s>>>(keys, homes, n, size, slot_keys, slot_counts);
  CKL();
  return SPECK_OK;
}

speck_status_t speck_exclusive_scan(speck_handle_t h, const int64_t* in, int64_t n, int64_t* out, speck_stream_t stream) {
  if (!h || n < 0 || (n > 0 && !in) || !out) return SPECK_ERR_INVALID_ARGUMENT;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  return launch_scan(h, in, n, out, nullptr, s);
}

}  // extern "C"
