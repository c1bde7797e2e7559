/*
 * speck.h — C ABI of the B200-native spECK SpGEMM library (libspeck.so).
 *
 * Computes C = A·B for sparse matrices in CSR format (Parger et al., PPoPP'20; citations
 * "P:a-b" are lines of the paper text PAPER.md):
 *   C_ij = Σ_k A_ik · B_kj                                   eq. (1)
 * CSR stores "the NZ elements sorted row-major and column-minor ... a sorted array of
 * row offsets indicates the beginning of each row".  The output C is sorted
 * CSR as well.  Every stored (structural) product counts:
 * entries whose value cancels to 0.0 are kept (the symbolic pass counts "without
 * calculating their values"; reading R1).
 *
 * The call sequence follows the paper's pipeline (Fig. 2):
 *   speck_analyze  = row analysis (Alg. 1) -> symbolic global load balancing
 *                     -> symbolic SpGEMM -> prefix sum of the
 *                    row sizes.  Returns nnz(C); the CALLER allocates C
 *                    (allocation of C is outside the paper's timing).
 *   speck_spgemm   = numeric global load balancing -> numeric SpGEMM with
 *                    direct / hash / dense accumulators and in-scratchpad sorting
 *                    (P:1121-1148).
 *
 * Conventions (all functions):
 *   - Matrix pointers are DEVICE pointers on the handle's device.  row_ptr is int64
 *     [rows+1] with row_ptr[0] == 0, col_idx is int32 [nnz], values fp32 or fp64 [nnz].
 *     A, B and C share one value type.
 *   - Inputs are borrowed and never written; C arrays are caller-owned.  Workspace is
 *     owned by the handle, grown on demand and reused across calls; speck_destroy frees it.
 *   - Work is issued on the caller's `stream` (0 = legacy default stream).  The library
 *     forks internal streams for concurrent kernels and joins them back onto `stream`.
 *   - No exception crosses the ABI.  Every function returns a speck_status_t; the text of
 *     the last error of a handle is available from speck_last_error().
 *   - A handle is bound to one device and is not thread-safe.
 *   - Input rows must be sorted with unique columns.  Unsorted or duplicate
 *     columns are undefined behaviour unless SPECK_OPT_VALIDATE is set, which turns them
 *     into SPECK_ERR_INVALID_INPUT.
 *   - Column indices must be < 2^31 - 1.  nnz(C) and per-matrix nnz are int64.
 */
#ifndef SPECK_H_
#define SPECK_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct speck_handle_s* speck_handle_t;
typedef void* speck_stream_t; /* a cudaStream_t */

typedef enum {
  SPECK_OK = 0,
  SPECK_ERR_INVALID_ARGUMENT = 1,  /* null pointer with nnz > 0, negative dims, bad option */
  SPECK_ERR_DIMENSION_MISMATCH = 2,/* A.cols != B.rows */
  SPECK_ERR_DTYPE_MISMATCH = 3,    /* A and B value types differ */
  SPECK_ERR_UNSUPPORTED = 4,       /* e.g. cols >= 2^31 - 1 */
  SPECK_ERR_OUT_OF_MEMORY = 5,     /* workspace allocation failed */
  SPECK_ERR_CUDA = 6,              /* any CUDA runtime / launch error; see speck_last_error */
  SPECK_ERR_NOT_ANALYZED = 7,      /* speck_spgemm without a matching speck_analyze */
  SPECK_ERR_INVALID_INPUT = 8      /* validation (SPECK_OPT_VALIDATE) found unsorted/duplicate/out-of-range columns */
} speck_status_t;

typedef enum { SPECK_F32 = 0, SPECK_F64 = 1 } speck_dtype_t;

/* A borrowed CSR matrix.  values may be NULL for speck_analyze /
 * speck_row_analysis (structure only). */
typedef struct {
  int64_t rows;
  int64_t cols;
  int64_t nnz;
  const int64_t* row_ptr; /* device, [rows+1] */
  const int32_t* col_idx; /* device, [nnz], sorted ascending per row */
  const void* values;     /* device, [nnz] fp32 or fp64 */
  speck_dtype_t dtype;
} speck_csr_t;

/* Options (speck_set_option).  Defaults in brackets.  All are plan/test knobs: none of
 * them changes the result, only which accumulator / load-balancing path produces it. */
typedef enum {
  SPECK_OPT_GLOBAL_LB_SYMBOLIC = 0, /* -1 auto by Table 2 thresholds, 0 off, 1 on [-1] */
  SPECK_OPT_GLOBAL_LB_NUMERIC = 1,  /* same for the numeric step [-1] */
  SPECK_OPT_FORCE_ACCUMULATOR = 2,  /* 0 auto; 1 hash wherever it fits; 2 dense for every non-direct row [0] */
  SPECK_OPT_DENSE_WINDOW = 3,       /* >0: cap the dense accumulator window (columns) — Fig. 5 tests [0] */
  SPECK_OPT_STAGE_TIMING = 4,       /* 1: record per-stage times with CUDA events (syncs) [0] */
  SPECK_OPT_VALIDATE = 5,           /* 1: validate input CSR (sorted, unique, in range) [0] */
  SPECK_OPT_DISABLE_DIRECT = 6,     /* 1: route single-NZ rows through the accumulators [0] */
  SPECK_OPT_FIXED_GROUP_SIZE = 7,   /* local load balancing of hash rows: 0 expand-balanced (every lane
                                       the same number of products, B200 default); >0 the paper's groups of g
                                       threads per referenced B row with this fixed g (power of two, clamped to the
                                       row's threads); -1 the paper's dynamic g (reading R9) [0] */
  SPECK_OPT_CONCURRENT_STREAMS = 8, /* number of internal streams for concurrent bins, 1..8 [4] */
  SPECK_OPT_SEGMENTS = 9,           /* 1: split rows beyond the largest map into column segments; 0: windowed dense [1] */
  SPECK_OPT_WARP_ROWS = 10,         /* 1: smallest bin = one warp per row (k_warp_rows); 0: merged blocks (Alg. 2) [1] */
  SPECK_OPT_LONG_BITMAP = 11,       /* 1: many long rows -> one bitmap+rank CTA per row when the column range fits; 2: always [1] */
  SPECK_OPT_BITMAP_REUSE = 12,      /* 1: the symbolic step keeps the dense bitmaps of numeric long rows (workspace
                                       <= 1/4 of free memory) so the numeric step does not rebuild them [1] */
  SPECK_OPT_KERNEL_TIMING = 13,     /* 1: time every kernel launch with CUDA events on the stream it runs on; read
                                       by speck_get_stats (kernel_id / kernel_bin / kernel_ms) [0] */
  SPECK_OPT_PATH_COUNTERS = 14,     /* 1: count the rows each accumulator path processes (path_rows); costs a few
                                       atomics per row — tests and diagnostics only [0] */
  SPECK_OPT_BUCKET_SORT = 15,       /* rows whose products are mostly distinct columns use a counting sort on
                                       column buckets instead of the hash map: 0 off, 1 numeric rows, 2 numeric
                                       and symbolic rows [1] */
  SPECK_OPT_DETERMINISTIC = 16      /* 1: every row of C accumulated by one warp in the order of eq. (1)'s sum, each
                                       product rounded before it is added: values bit-identical across runs and
                                       equal to a sequential sum in the inputs' precision (reading R15); slower
                                       for large rows [0] */
} speck_option_t;
/* Changing any option except STAGE_TIMING, CONCURRENT_STREAMS, GLOBAL_LB_NUMERIC, VALIDATE,
 * KERNEL_TIMING and PATH_COUNTERS after speck_analyze invalidates the analysis: the next
 * speck_spgemm returns SPECK_ERR_NOT_ANALYZED until speck_analyze runs again. */

/* Kernel identities reported by SPECK_OPT_KERNEL_TIMING: id = kind * 16 + configuration. */
typedef enum {
  SPECK_KERNEL_ANALYSIS = 1,     /* row analysis (Alg. 1) */
  SPECK_KERNEL_BINNING = 2,      /* classification + bin scatter (global load balancer) */
  SPECK_KERNEL_SCAN = 3,         /* prefix sum of the C row sizes */
  SPECK_KERNEL_SYM_WARP = 4,     /* symbolic, one warp per row (smallest bin) */
  SPECK_KERNEL_SYM_BLOCK = 5,    /* symbolic, one CTA per row or merged block (+ configuration 0..4) */
  SPECK_KERNEL_NUM_TINY = 6,     /* numeric rows of <= 64 entries, one warp per row (rank counting) */
  SPECK_KERNEL_NUM_WARP = 7,     /* numeric, one warp per row (ordered map) */
  SPECK_KERNEL_NUM_BLOCK = 8,    /* numeric, one CTA per row or merged block (+ configuration 0..4) */
  SPECK_KERNEL_DIRECT = 9,       /* numeric single-NZ rows (direct referencing) */
  SPECK_KERNEL_SEGMENTS = 10,    /* numeric long rows: column segments / windows */
  SPECK_KERNEL_LONG_BITMAP = 11, /* numeric long rows: bitmap + rank CTAs */
  SPECK_KERNEL_SEG_PLAN = 12     /* long-row job planning */
} speck_kernel_kind_t;

/* Accumulator paths counted by SPECK_OPT_PATH_COUNTERS (rows per path, path_rows[]). */
typedef enum {
  SPECK_PATH_SYM_WARP = 0,        /* symbolic warp-per-row hash */
  SPECK_PATH_SYM_BLOCK_HASH = 1,  /* symbolic hash shared by the warps of a CTA */
  SPECK_PATH_SYM_MERGED = 2,      /* symbolic merged block (Alg. 2), warp per row */
  SPECK_PATH_SYM_DENSE = 3,       /* symbolic dense bitmap, one window */
  SPECK_PATH_SYM_DENSE_MULTI = 4, /* symbolic dense bitmap, several windows (resume positions) */
  SPECK_PATH_NUM_TINY = 5,        /* numeric scrambled hash + rank counting (<= 64 entries) */
  SPECK_PATH_NUM_WARP_ORDERED = 6,/* numeric warp-per-row ordered map */
  SPECK_PATH_NUM_WARP_SORTED = 7, /* numeric warp-per-row compaction + sort (scrambled / wrapped map) */
  SPECK_PATH_NUM_BLOCK_ORDERED = 8,/* numeric CTA ordered map */
  SPECK_PATH_NUM_BLOCK_SORTED = 9,/* numeric CTA compaction + sort */
  SPECK_PATH_NUM_MERGED = 10,     /* numeric merged block (Alg. 2), warp per row */
  SPECK_PATH_NUM_DENSE = 11,      /* numeric dense window, one window */
  SPECK_PATH_NUM_DENSE_MULTI = 12,/* numeric dense, several windows */
  SPECK_PATH_NUM_DIRECT = 13,     /* numeric direct referencing */
  SPECK_PATH_SEG_HASH = 14,       /* long row column segment, ordered hash (per segment) */
  SPECK_PATH_SEG_DENSE = 15,      /* long row column segment, dense (per segment) */
  SPECK_PATH_SEG_WINDOWS = 16,    /* long row, sequential dense windows (per job) */
  SPECK_PATH_LONG_BITMAP = 17,    /* long row, bitmap + rank CTA */
  SPECK_PATH_LONG_BITMAP_SPLIT = 18,/* long row, bitmap kept by the symbolic step, split over CTAs (per CTA) */
  SPECK_PATH_SYM_ESC = 19,        /* symbolic bucket counting sort (esc_kernels.cuh) */
  SPECK_PATH_NUM_ESC = 20,        /* numeric bucket counting sort, no repeated column */
  SPECK_PATH_NUM_ESC_DUP = 21,    /* numeric bucket counting sort with repeated columns */
  SPECK_PATH_ESC_FALLBACK = 22,   /* bucket counting sort abandoned (uneven buckets): hash map instead */
  SPECK_PATH_NUM_DET = 23,        /* deterministic mode: one warp per large row (k_det_rows) */
  SPECK_PATH_COUNT = 24
} speck_path_t;

/* Statistics of the last analyze/spgemm pair (speck_get_stats). */
typedef struct {
  int64_t products;          /* Σ_i prods_i (Alg. 1 line 10); FLOP = 2·products */
  int64_t max_row_products;  /* prod_max (Alg. 1 line 11) */
  int64_t nnz_c;             /* nnz(C) */
  int64_t rows_direct;       /* rows with a single NZ in A */
  int64_t rows_empty;        /* rows without products */
  int32_t lb_symbolic;       /* 1 if the global load balancer ran for the symbolic step */
  int32_t lb_numeric;        /* 1 if it ran for the numeric step */
  int64_t rows_per_bin_symbolic[8]; /* [0]=empty [1]=direct [2..6]=configs 0..4 [7]=unused */
  int64_t rows_per_bin_numeric[8];  /* [7]=long rows split into column segments */
  int64_t rows_dense_numeric;    /* rows accumulated with the dense accumulator in the numeric step */
  int64_t segments;              /* column segments the long numeric rows were split into */
  int64_t workspace_bytes;       /* workspace currently held by the handle */
  int64_t kernel_launches;       /* kernels this handle has launched since speck_create (cumulative) */
  float ms_analysis, ms_symbolic_lb, ms_symbolic, ms_scan, ms_numeric_lb, ms_numeric; /* SPECK_OPT_STAGE_TIMING */
  /* Per bin of the last analyze/spgemm: [pass 0 symbolic / 1 numeric][category], categories
   * 0 empty, 1 direct, 2..6 configurations 0..4, 7 long (numeric), 8 tiny (numeric <= 64
   * entries), 9 unused.  Rows, Σ nnz(A_i), Σ products and (numeric) Σ nnz(C_i) of the rows in
   * the bin — the per-kernel algorithmic byte model of bench.py is built from them. */
  int64_t bin_rows[2][10];
  int64_t bin_nnza[2][10];
  int64_t bin_products[2][10];
  int64_t bin_nnzc[10];
  /* SPECK_OPT_KERNEL_TIMING: the launches of the last analyze/spgemm pair in issue order:
   * kernel id (speck_kernel_kind_t * 16 + configuration), the bin it processed (pass * 16 +
   * category; -1: all rows / not a bin) and its CUDA-event time on its own stream (ms). */
  int32_t n_kernels;
  int32_t kernel_id[64];
  int32_t kernel_bin[64];
  float kernel_ms[64];
  /* SPECK_OPT_PATH_COUNTERS: rows (or segments / CTAs, see speck_path_t) per path since the
   * option was set (cumulative over calls). */
  int64_t path_rows[SPECK_PATH_COUNT];
} speck_stats_t;

/* Create a handle on `device` (CUDA ordinal). */
speck_status_t speck_create(speck_handle_t* handle, int device);

/* Release all workspace and the handle.  Synchronises the handle's device. */
speck_status_t speck_destroy(speck_handle_t handle);

/* Set a plan option (speck_option_t). */
speck_status_t speck_set_option(speck_handle_t handle, int option, int64_t value);

/* Symbolic phase: rows analysis (Alg. 1), global load balancing, symbolic SpGEMM and the
 * exclusive prefix sum of the C row sizes.
 *   C_row_ptr : device int64 [A.rows + 1], caller-owned, written with C's row offsets
 *   nnz_c     : host out, nnz(C) = C_row_ptr[A.rows]
 * Synchronises `stream` twice (the analysis statistics and nnz(C) are read back).
 * A.values / B.values are not read. */
speck_status_t speck_analyze(speck_handle_t handle, const speck_csr_t* A, const speck_csr_t* B,
                             int64_t* C_row_ptr, int64_t* nnz_c, speck_stream_t stream);

/* Numeric phase: writes C_col_idx [nnz_c] and C_values [nnz_c] (caller-allocated, device)
 * for the A, B of the preceding speck_analyze on this handle (same pointers and shapes,
 * else SPECK_ERR_NOT_ANALYZED).  Rows come out sorted by column.  Asynchronous. */
speck_status_t speck_spgemm(speck_handle_t handle, const speck_csr_t* A, const speck_csr_t* B,
                            const int64_t* C_row_ptr, int32_t* C_col_idx, void* C_values,
                            speck_stream_t stream);

/* Memory-bounded numeric phase (the paper's future work "partial
 * multiplications of large matrices on single GPUs"): after speck_analyze, the
 * numeric phase of the rows [r0, r1) only.  C_row_ptr is the full array speck_analyze wrote;
 * C_col_part / C_val_part (device, caller-owned) hold the chunk's C_row_ptr[r1] - C_row_ptr[r0]
 * entries: entry t of row i goes to index C_row_ptr[i] - C_row_ptr[r0] + t.  Calls for different
 * ranges may follow one speck_analyze in any order; together they produce exactly the entries
 * speck_spgemm would.  One small D2H synchronisation per call (the chunk's bin ranges); the
 * numeric work is asynchronous.  Invalid ranges -> SPECK_ERR_INVALID_ARGUMENT. */
speck_status_t speck_spgemm_rows(speck_handle_t handle, const speck_csr_t* A, const speck_csr_t* B,
                                 const int64_t* C_row_ptr, int64_t r0, int64_t r1, int32_t* C_col_part,
                                 void* C_val_part, speck_stream_t stream);

/* Device CSR transpose: T = Aᵀ in sorted CSR, for the paper's A·Aᵀ protocol
 * ("rectangular matrices ... multiplied with their transpose", Aᵀ precomputed) and
 * the AMG restriction R = Pᵀ.  T is A.cols x A.rows: T_row_ptr device int64 [A.cols + 1],
 * T_col_idx int32 [A.nnz], T_values [A.nnz] of A's dtype (NULL exactly when A.values is NULL),
 * all caller-owned.  Values are moved bit for bit; every row of T is sorted.  Synchronises
 * `stream` (row-length statistics are read back to size the sort). */
speck_status_t speck_transpose(speck_handle_t handle, const speck_csr_t* A, int64_t* T_row_ptr, int32_t* T_col_idx,
                               void* T_values, speck_stream_t stream);

/* Row chunks for a memory budget: splits [0, rows) of the analysed C (C_row_ptr, device) into
 * consecutive ranges of fewer than max_nnz entries each (some may be empty).  Writes
 * bounds[0..n] (host, int64, n <= max_parts) and *n_parts = n.  max_nnz must exceed the longest
 * row of C (else SPECK_ERR_INVALID_ARGUMENT).  Synchronous. */
speck_status_t speck_row_chunks(speck_handle_t handle, const int64_t* C_row_ptr, int64_t rows, int64_t max_nnz,
                                int64_t* bounds, int64_t max_parts, int64_t* n_parts);

/* Row analysis only (Alg. 1).  Per row i of A (device arrays, [A.rows]):
 *   prods[i]  = Σ_{k ∈ A_i} |B_k|           maxlen[i] = max_k |B_k|
 *   colmin[i] = min over non-empty B_k of the first column (INT32_MAX if none)
 *   colmax[i] = max over non-empty B_k of the last column  (-1 if none)
 * Any output pointer may be NULL.  Used by the multi-GPU row partitioner (balanced
 * product split).  Asynchronous. */
speck_status_t speck_row_analysis(speck_handle_t handle, const speck_csr_t* A, const speck_csr_t* B,
                                  int64_t* prods, int32_t* maxlen, int32_t* colmin, int32_t* colmax,
                                  speck_stream_t stream);

/* Row analysis restricted to the product counts (Alg. 1 line 10):
 *   prods[i] = Σ_{k ∈ A_i} |B_k|, device int64 [A.rows], caller-owned.
 * The multi-GPU partitioner's balanced row split.  Asynchronous. */
speck_status_t speck_row_products(speck_handle_t handle, const speck_csr_t* A, const speck_csr_t* B, int64_t* prods,
                                  speck_stream_t stream);

/* Workspace allocator hooks (e.g. the PyTorch caching allocator): alloc(bytes, stream, ctx)
 * returns device memory usable on `stream` (NULL on failure -> SPECK_ERR_OUT_OF_MEMORY),
 * release(p, stream, ctx) gives it back.  Without hooks the handle uses cudaMallocAsync /
 * cudaFreeAsync.  Setting (or clearing, with NULLs) the hooks first releases the handle's
 * current workspace, so call it before speck_analyze; a pending speck_spgemm must be complete. */
typedef void* (*speck_alloc_fn)(size_t bytes, speck_stream_t stream, void* ctx);
typedef void (*speck_release_fn)(void* ptr, speck_stream_t stream, void* ctx);
speck_status_t speck_set_allocator(speck_handle_t handle, speck_alloc_fn alloc, speck_release_fn release, void* ctx);

/* Statistics of the last analyze/spgemm (host struct). */
speck_status_t speck_get_stats(speck_handle_t handle, speck_stats_t* out);

/* Static text for a status code. */
const char* speck_status_string(speck_status_t status);

/* Detail text of the last error on this handle ("" if none).  Valid until the next call. */
const char* speck_last_error(speck_handle_t handle);

/* Library version string. */
const char* speck_version(void);

/* ----------------------------------------------------------------------------------
 * Component entry points: each runs, on device buffers, a device function the pipeline
 * itself calls (warp_block_merge in the merged-block kernels, local_group_size in the
 * SPECK_OPT_FIXED_GROUP_SIZE = -1 expansion, probe_insert_mono in the numeric maps of
 * scrambled rows, the look-back scan of the C row offsets), so the paper's worked examples can
 * be checked against the oracle in isolation.  All asynchronous on `stream`.
 * ---------------------------------------------------------------------------------- */

/* Block merge (Alg. 2; Fig. 3), reading R10: for each aligned group
 * of 32 entries of needs[n] (int64, device), neighbouring blocks are merged level by level
 * (5 levels) while their sum stays strictly below `cap`.  Writes block_start_flag[n]
 * (uint8, device): 1 where a block starts. */
speck_status_t speck_block_merge(speck_handle_t handle, const int64_t* needs, int64_t n, int64_t cap,
                                 uint8_t* block_start_flag, speck_stream_t stream);

/* Local load balancer group size g (reading R9) for n blocks described by
 * device arrays nnzA[n], prods[n], maxlen[n] (int64) and T threads; writes g[n] (int32). */
speck_status_t speck_group_size(speck_handle_t handle, int32_t T, const int64_t* nnzA, const int64_t* prods,
                                const int64_t* maxlen, int64_t n, int32_t* g, speck_stream_t stream);

/* Scratchpad linear-probing hash (Fig. 4) with injected home slots: inserts
 * keys[n] (uint32, device) at homes[n] (uint32) into a map of `size` slots (<= 8192) held
 * in shared memory by one CTA, counting duplicates; copies the map out to
 * slot_keys[size] (uint32, 0xFFFFFFFF = empty) and slot_counts[size] (uint32).
 * Inserts are issued in order (one thread) so the final layout is deterministic. */
speck_status_t speck_hash_probe(speck_handle_t handle, const uint32_t* keys, const uint32_t* homes, int64_t n,
                                int32_t size, uint32_t* slot_keys, uint32_t* slot_counts, speck_stream_t stream);

/* Exclusive prefix sum of int64 in[n] into out[n+1] (out[n] = total) with the library's
 * single-pass decoupled look-back scan (the C row-offset step). */
speck_status_t speck_exclusive_scan(speck_handle_t handle, const int64_t* in, int64_t n, int64_t* out,
                                    speck_stream_t stream);

#ifdef __cplusplus
}
#endif
#endif /* SPECK_H_ */
