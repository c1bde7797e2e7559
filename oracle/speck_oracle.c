/*
 * speck_oracle.c — plain, slow, obviously-correct CPU reference for the spECK hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  The product path
 * (paper_conf_ppopp_pargerwms20_b200/) never imports, links or calls it, and it shares
 * no code, header, constant or helper with the CUDA path.
 *
 * Paper: Parger, Winter, Mlakar, Steinberger, "spECK: Accelerating GPU Sparse
 * Matrix-Matrix Multiplication through Lightweight Analysis", PPoPP'20.
 * Citations "P:a-b" are lines of /root/reference/PAPER.md.
 *
 * What each function follows:
 *   oracle_row_analysis   Algorithm 1 + the text P:651-656
 *   oracle_symbolic       structural nnz per C row (eq. (1))
 *   oracle_numeric        C = A·B, eq. (1), rows sorted by column (P:98-103,
 *                         P:1121-1123); structural zeros kept (R1)
 *   oracle_numeric_sequential  the same sums left to right in the inputs' precision
 *                         (deterministic-value mode, R15)
 *   oracle_block_merge    Algorithm 2 + Fig. 3, reading R10
 *   oracle_group_iters    Fig. 1 iteration model
 *   oracle_group_size     local load balancer g, reading R9
 *   oracle_hash_insert    linear-probing hash map (Fig. 4)
 *   oracle_dense_windows  windowed dense accumulator (Fig. 5)
 *
 * Pins (tests/test_oracle_*.py): brute-force dense products, closed forms (identity,
 * permutation, diagonal scaling, squared 5-point Laplacian, Galerkin Kronecker form),
 * invariants, the transposition identity and the paper's worked examples (golden files).
 * Parity unpinned: none of the functions above.
 *
 * Precision: products and sums are formed in long double (x87 80-bit); the value
 * returned is rounded to double.  The scale s_ij = Σ|A_ik·B_kj| is returned beside it
 * for the tolerance test |c - r| <= tol·s (north_star).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define ORACLE_OK 0
#define ORACLE_ERR_ALLOC 1
#define ORACLE_ERR_ARG 2
#define ORACLE_ERR_UNSORTED 3

static long double load_val(const void *v, int is_f64, int64_t i) {
    if (is_f64) return (long double)((const double *)v)[i];
    return (long double)((const float *)v)[i];
}

int oracle_num_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

void oracle_set_threads(int n) {
#ifdef _OPENMP
    if (n > 0) omp_set_num_threads(n);
#else
    (void)n;
#endif
}

/* Check the CSR contract of P:98-103: columns strictly ascending inside each row and
 * inside [0, ncols).  Returns the first offending row or -1. */
int64_t oracle_check_csr(int64_t rows, int64_t ncols, const int64_t *rp, const int32_t *col) {
    for (int64_t i = 0; i < rows; ++i) {
        if (rp[i + 1] < rp[i]) return i;
        for (int64_t p = rp[i]; p < rp[i + 1]; ++p) {
            if (col[p] < 0 || col[p] >= ncols) return i;
            if (p > rp[i] && col[p] <= col[p - 1]) return i;
        }
    }
    return -1;
}

/* ---------------------------------------------------------------- Algorithm 1 ---
 * For each row of A:
 *   a) prod_r      = total number of products        (Alg.1 line 8)
 *   b) prod_r,max  = products of the longest referenced B row (line 9)
 *   c) colmin/colmax over all referenced rows of B   (lines 6-7; "minimum and maximum
 *      column index of all referenced rows", P:654-655 — empty B rows reference no
 *      column; a row with no products gets colmin = INT32_MAX, colmax = -1, reading R6)
 * and globally prod = Σ prod_r (line 10), prod_max = max prod_r (line 11).
 * stats_out[0] = prod, stats_out[1] = prod_max. */
int oracle_row_analysis(int64_t m, const int64_t *A_rp, const int32_t *A_col,
                        const int64_t *B_rp, const int32_t *B_col,
                        int64_t *prods, int32_t *maxlen, int32_t *colmin, int32_t *colmax,
                        int64_t *stats_out) {
    int64_t prod = 0, prod_max = 0;
    for (int64_t r = 0; r < m; ++r) {
        int64_t prod_r = 0, prod_r_max = 0;
        int32_t cmin = INT32_MAX, cmax = -1;
        for (int64_t p = A_rp[r]; p < A_rp[r + 1]; ++p) {
            int32_t colA = A_col[p];
            int64_t id0 = B_rp[colA], idn = B_rp[colA + 1];
            if (idn > id0) {
                if (B_col[id0] < cmin) cmin = B_col[id0];
                if (B_col[idn - 1] > cmax) cmax = B_col[idn - 1];
            }
            prod_r += idn - id0;
            if (idn - id0 > prod_r_max) prod_r_max = idn - id0;
        }
        prods[r] = prod_r;
        maxlen[r] = (int32_t)prod_r_max;
        colmin[r] = cmin;
        colmax[r] = cmax;
        prod += prod_r;
        if (prod_r > prod_max) prod_max = prod_r;
    }
    stats_out[0] = prod;
    stats_out[1] = prod_max;
    return ORACLE_OK;
}

/* ------------------------------------------------------- Gustavson accumulator ---
 * Row-wise SpGEMM: row i of C accumulates the rows of B that row i of A
 * references.  `mark[j] == i` tells whether column j was touched in row i. */
typedef struct {
    int64_t *mark;
    long double *acc;
    long double *sc;
    int32_t *touched;
} scratch_t;

static int scratch_init(scratch_t *s, int64_t ncols) {
    s->mark = (int64_t *)malloc(sizeof(int64_t) * (size_t)(ncols > 0 ? ncols : 1));
    s->acc = (long double *)malloc(sizeof(long double) * (size_t)(ncols > 0 ? ncols : 1));
    s->sc = (long double *)malloc(sizeof(long double) * (size_t)(ncols > 0 ? ncols : 1));
    s->touched = (int32_t *)malloc(sizeof(int32_t) * (size_t)(ncols > 0 ? ncols : 1));
    if (!s->mark || !s->acc || !s->sc || !s->touched) return ORACLE_ERR_ALLOC;
    for (int64_t j = 0; j < ncols; ++j) s->mark[j] = -1;
    return ORACLE_OK;
}

static void scratch_free(scratch_t *s) {
    free(s->mark); free(s->acc); free(s->sc); free(s->touched);
}

static int cmp_i32(const void *a, const void *b) {
    int32_t x = *(const int32_t *)a, y = *(const int32_t *)b;
    return (x > y) - (x < y);
}

/* Structural count of row i of C: |∪_{k∈S(A_i)} S(B_k)| (every stored
 * entry counts, whatever its value — reading R1). */
int oracle_symbolic(const int64_t *A_rp, const int32_t *A_col, const int64_t *B_rp,
                    const int32_t *B_col, int64_t ncols, int64_t r0, int64_t r1, int64_t *cnt) {
    int err = ORACLE_OK;
#pragma omp parallel
    {
        scratch_t s;
        int my = scratch_init(&s, ncols);
        if (my != ORACLE_OK) {
#pragma omp atomic write
            err = my;
        }
#pragma omp for schedule(dynamic, 1024)
        for (int64_t i = r0; i < r1; ++i) {
            if (my != ORACLE_OK) continue;
            int64_t n = 0;
            for (int64_t p = A_rp[i]; p < A_rp[i + 1]; ++p) {
                int32_t k = A_col[p];
                for (int64_t q = B_rp[k]; q < B_rp[k + 1]; ++q) {
                    int32_t j = B_col[q];
                    if (s.mark[j] != i) { s.mark[j] = i; ++n; }
                }
            }
            cnt[i - r0] = n;
        }
        scratch_free(&s);
    }
    return err;
}

/* Numeric rows [r0, r1): C_ij = Σ_{k ∈ S(A_i), (k,j) ∈ S(B)} A_ik·B_kj  (eq. (1)),
 * written sorted by column at out_rp[i-r0] .. out_rp[i-r0+1] (relative to
 * the first row of the range; out_rp[0] is usually 0).  out_scale = Σ|A_ik·B_kj|. */
int oracle_numeric(const int64_t *A_rp, const int32_t *A_col, const void *A_val,
                   const int64_t *B_rp, const int32_t *B_col, const void *B_val, int is_f64,
                   int64_t ncols, int64_t r0, int64_t r1, const int64_t *out_rp,
                   int32_t *out_col, double *out_val, double *out_scale) {
    int err = ORACLE_OK;
#pragma omp parallel
    {
        scratch_t s;
        int my = scratch_init(&s, ncols);
        if (my != ORACLE_OK) {
#pragma omp atomic write
            err = my;
        }
#pragma omp for schedule(dynamic, 1024)
        for (int64_t i = r0; i < r1; ++i) {
            if (my != ORACLE_OK) continue;
            int64_t n = 0;
            for (int64_t p = A_rp[i]; p < A_rp[i + 1]; ++p) {
                int32_t k = A_col[p];
                long double a = load_val(A_val, is_f64, p);
                for (int64_t q = B_rp[k]; q < B_rp[k + 1]; ++q) {
                    int32_t j = B_col[q];
                    long double ab = a * load_val(B_val, is_f64, q);
                    if (s.mark[j] != i) {
                        s.mark[j] = i;
                        s.acc[j] = 0.0L;
                        s.sc[j] = 0.0L;
                        s.touched[n++] = j;
                    }
                    s.acc[j] += ab;
                    s.sc[j] += fabsl(ab);
                }
            }
            qsort(s.touched, (size_t)n, sizeof(int32_t), cmp_i32);
            int64_t base = out_rp[i - r0];
            if (out_rp[i - r0 + 1] - base != n) {
#pragma omp atomic write
                err = ORACLE_ERR_ARG;
                continue;
            }
            for (int64_t t = 0; t < n; ++t) {
                int32_t j = s.touched[t];
                out_col[base + t] = j;
                out_val[base + t] = (double)s.acc[j];
                if (out_scale) out_scale[base + t] = (double)s.sc[j];
            }
        }
        scratch_free(&s);
    }
    return err;
}

/* Sequential working-precision values (deterministic-value mode; DESIGN.md
 * reading R15): C_ij accumulated left to right in the order of eq. (1)'s sum — k in the order
 * of row i of A, then the entries of B_k in order — in the inputs' own precision, every
 * product rounded before it is added:  acc <- fl(acc + fl(A_ik * B_kj)), acc starting at the
 * first product.  (The library's deterministic mode promises exactly these bits.)  Structure as
 * oracle_numeric; out_val is the float / double result widened to double. */
int oracle_numeric_sequential(const int64_t *A_rp, const int32_t *A_col, const void *A_val,
                              const int64_t *B_rp, const int32_t *B_col, const void *B_val, int is_f64,
                              int64_t ncols, int64_t r0, int64_t r1, const int64_t *out_rp,
                              int32_t *out_col, double *out_val) {
    int err = ORACLE_OK;
#pragma omp parallel
    {
        int64_t *mark = (int64_t *)malloc(sizeof(int64_t) * (size_t)(ncols > 0 ? ncols : 1));
        double *accd = (double *)malloc(sizeof(double) * (size_t)(ncols > 0 ? ncols : 1));
        float *accf = (float *)malloc(sizeof(float) * (size_t)(ncols > 0 ? ncols : 1));
        int32_t *touched = (int32_t *)malloc(sizeof(int32_t) * (size_t)(ncols > 0 ? ncols : 1));
        int my = (mark && accd && accf && touched) ? ORACLE_OK : ORACLE_ERR_ALLOC;
        if (my != ORACLE_OK) {
#pragma omp atomic write
            err = my;
        } else {
            for (int64_t j = 0; j < ncols; ++j) mark[j] = -1;
        }
#pragma omp for schedule(dynamic, 1024)
        for (int64_t i = r0; i < r1; ++i) {
            if (my != ORACLE_OK) continue;
            int64_t n = 0;
            for (int64_t p = A_rp[i]; p < A_rp[i + 1]; ++p) {
                int32_t k = A_col[p];
                for (int64_t q = B_rp[k]; q < B_rp[k + 1]; ++q) {
                    int32_t j = B_col[q];
                    if (is_f64) {
                        volatile double prod = ((const double *)A_val)[p] * ((const double *)B_val)[q];
                        if (mark[j] != i) { mark[j] = i; accd[j] = prod; touched[n++] = j; }
                        else accd[j] = accd[j] + prod;
                    } else {
                        volatile float prod = ((const float *)A_val)[p] * ((const float *)B_val)[q];
                        if (mark[j] != i) { mark[j] = i; accf[j] = prod; touched[n++] = j; }
                        else accf[j] = accf[j] + prod;
                    }
                }
            }
            qsort(touched, (size_t)n, sizeof(int32_t), cmp_i32);
            int64_t base = out_rp[i - r0];
            if (out_rp[i - r0 + 1] - base != n) {
#pragma omp atomic write
                err = ORACLE_ERR_ARG;
                continue;
            }
            for (int64_t t = 0; t < n; ++t) {
                int32_t j = touched[t];
                out_col[base + t] = j;
                out_val[base + t] = is_f64 ? accd[j] : (double)accf[j];
            }
        }
        free(mark); free(accd); free(accf); free(touched);
    }
    return err;
}

/* ---------------------------------------------------------------- Algorithm 2 ---
 * Block merge (Fig. 3), reading R10 of DESIGN.md:
 * a binary tree over the sequence of per-row needs b[0..n); at level s = 0..levels-1
 * every aligned group of 2^(s+1) rows consists of a left and a right half, each
 * already partitioned into blocks; the LAST block of the left half and the FIRST
 * block of the right half are merged when their sum is strictly below `cap`.
 * levels = 5 (blocks of at most 32 rows).
 * Output: block_start[nb], block_len[nb]; returns nb. */
int64_t oracle_block_merge(int64_t n, const int64_t *b, int64_t cap, int levels,
                           int64_t *block_start, int64_t *block_len) {
    /* start[i] = 1 if a block starts at position i; blocks are maximal runs. */
    char *start = (char *)malloc((size_t)(n > 0 ? n : 1));
    int64_t *sum = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    if (!start || !sum) { free(start); free(sum); return -1; }
    for (int64_t i = 0; i < n; ++i) { start[i] = 1; sum[i] = b[i]; }
    for (int s = 0; s < levels; ++s) {
        int64_t half = (int64_t)1 << s;
        for (int64_t g = 0; g + half < n; g += 2 * half) {
            int64_t mid = g + half;              /* first position of the right half */
            int64_t left = mid - 1;              /* find the start of the left half's last block */
            while (!start[left]) --left;
            /* the right half's first block starts at mid */
            if (sum[left] + sum[mid] < cap) {
                sum[left] += sum[mid];
                start[mid] = 0;
            }
        }
    }
    int64_t nb = 0;
    for (int64_t i = 0; i < n; ++i) {
        if (start[i]) {
            int64_t j = i + 1;
            while (j < n && !start[j]) ++j;
            block_start[nb] = i;
            block_len[nb] = j - i;
            ++nb;
        }
    }
    free(start); free(sum);
    return nb;
}

/* ------------------------------------------------------------- Fig. 1 model ---
 * T threads split into k = T/g groups; groups are assigned successively to the
 * referenced B rows (group j takes rows j, j+k, j+2k, ...); a group needs
 * ceil(len/g) iterations per row; the block needs the maximum over groups. */
int64_t oracle_group_iters(int64_t nrows, const int64_t *lens, int64_t T, int64_t g) {
    if (g <= 0 || T <= 0) return -1;
    int64_t k = T / g;
    if (k < 1) k = 1;
    int64_t best = 0;
    for (int64_t j = 0; j < k; ++j) {
        int64_t it = 0;
        for (int64_t r = j; r < nrows; r += k) it += (lens[r] + g - 1) / g;
        if (it > best) best = it;
    }
    return best;
}

static int64_t round_pow2(double x) {
    /* "we also round g to the closest power of two": of the two powers of two
     * p <= x < 2p, the one at the smaller |x - p| distance; a tie goes to 2p (reading R9). */
    if (x <= 1.0) return 1;
    int64_t p = 1;
    while ((double)(2 * p) <= x) p *= 2;
    return (x - (double)p < (double)(2 * p) - x) ? p : 2 * p;
}

/* Local load balancer, reading R9:
 *   g0 = average referenced-B-row length (prods / nnzA), rounded to a power of two;
 *   iter_max = ceil(maxlen / g), n_rows = nnzA / k with k = T/g;
 *   if iter_max > 2 n_rows: g <- g·sqrt(iter_max / (2 n_rows));
 *   else if n_rows > 2 iter_max: g <- g·sqrt(iter_max / n_rows);
 *   round to the closest power of two and clamp to [1, T];
 *   finally if k = T/g > nnzA, reduce k to the largest power of two <= nnzA so every
 *   group gets at least one NZ of A and all groups keep one power-of-two size.
 *   Returns g. */
int64_t oracle_group_size(int64_t T, int64_t nnzA, int64_t prods, int64_t maxlen) {
    if (nnzA <= 0 || prods <= 0) return T;
    double g = (double)round_pow2((double)prods / (double)nnzA);
    if (g > (double)T) g = (double)T;
    double k = (double)T / g;
    double iter_max = ceil((double)maxlen / g);
    double n_rows = (double)nnzA / k;
    if (iter_max > 2.0 * n_rows) g = g * sqrt(iter_max / (2.0 * n_rows));
    else if (n_rows > 2.0 * iter_max) g = g * sqrt(iter_max / n_rows);
    int64_t gi = round_pow2(g);
    if (gi > T) gi = T;
    if (gi < 1) gi = 1;
    int64_t kk = T / gi;
    if (kk > nnzA) {
        int64_t p = 1;
        while (p * 2 <= nnzA) p <<= 1;  /* largest power of two <= nnzA: every group gets >= 1 NZ */
        gi = T / p;
        if (gi < 1) gi = 1;
    }
    return gi;
}

/* ------------------------------------------------------------- Fig. 4 hash ---
 * Linear-probing insert-or-accumulate (Fig. 4): a key goes to slot h(key);
 * if that slot holds another key, probe the next slot (mod size).  `home` gives h(id)
 * per insert (the hash function is injected).  Slots are EMPTY (-1) initially.
 * Returns 0, or -1 if the map overflowed. */
int oracle_hash_insert(int64_t n, const int64_t *keys, const int64_t *home, int64_t size,
                       int64_t *slot_key, int64_t *slot_count) {
    for (int64_t s = 0; s < size; ++s) { slot_key[s] = -1; slot_count[s] = 0; }
    for (int64_t i = 0; i < n; ++i) {
        int64_t h = home[i] % size, probes = 0;
        while (slot_key[h] != -1 && slot_key[h] != keys[i]) {
            h = (h + 1) % size;
            if (++probes >= size) return -1;
        }
        slot_key[h] = keys[i];
        slot_count[h] += 1;
    }
    return 0;
}

/* ------------------------------------------------------------ Fig. 5 dense ---
 * Windowed dense accumulation over [colmin, colmax] with a window of W columns
 * (P:1071-1078): window w covers [colmin + w·W, colmin + (w+1)·W); in each window the
 * products falling into it are summed per column and the touched columns are emitted
 * in ascending order.  Emits (window, col, value) triples; returns the
 * number emitted. */
int64_t oracle_dense_windows(int64_t n, const int32_t *cols, const double *vals, int32_t colmin,
                             int32_t colmax, int64_t W, int64_t *out_window, int32_t *out_col,
                             double *out_val) {
    int64_t ne = 0;
    int64_t range = (int64_t)colmax - colmin + 1;
    double *acc = (double *)calloc((size_t)W, sizeof(double));
    char *hit = (char *)calloc((size_t)W, 1);
    if (!acc || !hit) { free(acc); free(hit); return -1; }
    for (int64_t w = 0; w * W < range; ++w) {
        int64_t lo = colmin + w * W, hi = lo + W;
        memset(acc, 0, sizeof(double) * (size_t)W);
        memset(hit, 0, (size_t)W);
        for (int64_t i = 0; i < n; ++i) {
            if (cols[i] >= lo && cols[i] < hi) {
                acc[cols[i] - lo] += vals[i];
                hit[cols[i] - lo] = 1;
            }
        }
        for (int64_t c = 0; c < W; ++c) {
            if (hit[c]) {
                out_window[ne] = w;
                out_col[ne] = (int32_t)(lo + c);
                out_val[ne] = acc[c];
                ++ne;
            }
        }
    }
    free(acc); free(hit);
    return ne;
}
