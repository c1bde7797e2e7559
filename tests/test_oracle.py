"""Pins for the CPU oracle (oracle/speck_oracle.c) against things other than itself.

Each test fixes the oracle to mathematics or to the paper: brute-force dense products,
closed forms (identity, permutation, diagonal scaling, the squared 5-point Laplacian,
the Galerkin Kronecker form), invariants, the transposition identity, a library
cross-check on pattern matrices, and the paper's worked examples (tests/golden/).
No expected value here comes from the CUDA path.
"""
import numpy as np
import pytest
import torch

import oracle
import workloads as W
from conftest import golden


def dense(M):
    rp, col, val = M.numpy()
    D = np.zeros((M.rows, M.cols), np.float64)
    P = np.zeros((M.rows, M.cols), np.int64)
    for i in range(M.rows):
        for p in range(rp[i], rp[i + 1]):
            D[i, col[p]] = val[p]
            P[i, col[p]] = 1
    return D, P


def csr_dense(rp, col, val, rows, cols):
    D = np.zeros((rows, cols), np.float64)
    P = np.zeros((rows, cols), np.int64)
    for i in range(rows):
        for p in range(rp[i], rp[i + 1]):
            D[i, col[p]] = val[p]
            P[i, col[p]] += 1
    return D, P


def assert_sorted_csr(rp, col, rows, cols):
    assert rp[0] == 0 and np.all(np.diff(rp) >= 0)
    assert oracle.check_csr(rows, cols, rp, col) == -1


CASES = [
    # rows, inner, cols, density A, density B, empty_rows, zero_frac, int_values, dtype
    (17, 23, 19, 0.2, 0.25, 0.2, 0.0, False, torch.float64),
    (40, 33, 51, 0.1, 0.3, 0.1, 0.3, False, torch.float64),
    (64, 64, 64, 0.05, 0.05, 0.0, 0.0, True, torch.float64),
    (31, 45, 8, 0.5, 0.6, 0.3, 0.2, True, torch.float32),
    (9, 60, 57, 0.9, 0.02, 0.0, 0.0, False, torch.float32),
    (50, 7, 61, 0.3, 0.9, 0.0, 0.5, False, torch.float64),
    (1, 64, 64, 1.0, 0.5, 0.0, 0.0, False, torch.float64),   # one full row of A
]


@pytest.mark.parametrize("case", range(len(CASES)))
def test_bruteforce_dense(case):
    """Oracle == dense fp64 product (values) and boolean pattern product (structure)."""
    m, k, n, da, db, er, zf, iv, dt = CASES[case]
    A = W.random_sparse(m, k, da, seed=10 + case, dtype=dt, empty_rows=er, zero_frac=zf, int_values=iv)
    B = W.random_sparse(k, n, db, seed=50 + case, dtype=dt, empty_rows=er, zero_frac=zf, int_values=iv)
    DA, PA = dense(A)
    DB, PB = dense(B)
    rp, col, val, scale = oracle.spgemm(A, B)
    assert_sorted_csr(rp, col, m, n)
    DC, PC = csr_dense(rp, col, val, m, n)
    # structure: stored entries of C are exactly the structural product pattern (zeros kept)
    assert np.array_equal(PC, (PA @ PB > 0).astype(np.int64))
    # values: dense product; scale = Σ|a·b|
    ref = DA @ DB
    S = np.abs(DA) @ np.abs(DB)
    if iv:
        assert np.array_equal(DC, ref)
    else:
        assert np.all(np.abs(DC - ref) <= 4e-16 * S + 1e-300)
    DS, _ = csr_dense(rp, col, scale, m, n)
    assert np.allclose(DS, S, rtol=1e-14, atol=0)


def test_bruteforce_rectangular_not_transposed():
    """A (3x5) · B (5x2): a transposed operand would not even conform; pin the orientation."""
    rows = np.array([0, 2, 3, 5], np.int64)
    A = W.CSR(3, 5, torch.tensor(rows), torch.tensor([0, 4, 2, 1, 3], dtype=torch.int32),
              torch.tensor([1., 2., 3., 4., 5.], dtype=torch.float64))
    B = W.CSR(5, 2, torch.tensor([0, 1, 2, 2, 4, 5]), torch.tensor([1, 0, 0, 1, 0], dtype=torch.int32),
              torch.tensor([10., 20., 30., 40., 50.], dtype=torch.float64))
    rp, col, val, _ = oracle.spgemm(A, B)
    # row0 = 1*B0 + 2*B4 = [2*50, 1*10] ; row1 = 3*B2 = [] ; row2 = 4*B1 + 5*B3 = [4*20+5*30, 5*40]
    assert rp.tolist() == [0, 2, 2, 4]
    assert col.tolist() == [0, 1, 0, 1]
    assert val.tolist() == [100., 10., 230., 200.]


def _eye(n, dtype=torch.float64):
    return W.CSR(n, n, torch.arange(n + 1, dtype=torch.int64), torch.arange(n, dtype=torch.int32),
                 torch.ones(n, dtype=dtype))


@pytest.mark.parametrize("dt", [torch.float32, torch.float64])
def test_identity(dt):
    A = W.random_sparse(37, 41, 0.15, seed=3, dtype=dt, empty_rows=0.1, zero_frac=0.2)
    for L, R in ((A, _eye(41, dt)), (_eye(37, dt), A)):
        rp, col, val, _ = oracle.spgemm(L, R)
        arp, acol, aval = A.numpy()
        assert np.array_equal(rp, arp) and np.array_equal(col, acol)
        assert np.array_equal(val, aval.astype(np.float64))      # bit-exact, zeros kept


def test_permutation_and_diagonal_scaling():
    n = 45
    A = W.random_sparse(n, n, 0.12, seed=4, dtype=torch.float64, empty_rows=0.1)
    perm = np.random.default_rng(0).permutation(n)
    Pi = W.CSR(n, n, torch.arange(n + 1), torch.tensor(perm, dtype=torch.int32), torch.ones(n, dtype=torch.float64))
    DA, _ = dense(A)
    # Π·A: row i of the product is row perm[i] of A
    rp, col, val, _ = oracle.spgemm(Pi, A)
    D, _ = csr_dense(rp, col, val, n, n)
    assert np.array_equal(D, DA[perm])
    # A·Π: column j of the product collects column with Π[j', j] = 1, i.e. relabel col perm->idx
    rp, col, val, _ = oracle.spgemm(A, Pi)
    assert_sorted_csr(rp, col, n, n)
    D, _ = csr_dense(rp, col, val, n, n)
    DP = np.zeros((n, n)); DP[np.arange(n), perm] = 1
    assert np.array_equal(D, DA @ DP)
    # D·A and A·D with arbitrary diagonal: one product per entry -> exact
    d = W.uniform_pm1(9, 1, torch.arange(n), torch.float64)
    Dg = W.CSR(n, n, torch.arange(n + 1), torch.arange(n, dtype=torch.int32), d)
    dn = d.numpy()
    rp, col, val, _ = oracle.spgemm(Dg, A)
    arp, acol, aval = A.numpy()
    assert np.array_equal(col, acol)
    rows = np.repeat(np.arange(n), np.diff(arp))
    assert np.array_equal(val, dn[rows] * aval)
    rp, col, val, _ = oracle.spgemm(A, Dg)
    assert np.array_equal(val, aval * dn[acol])


def test_poisson_squared_closed_form():
    """C1: A = 5-point Laplacian 64x64 (4 diag, -1 neighbours). (A^2)_ii = 16 + deg(i),
    -8 at Manhattan distance 1, +1 at distance 2 along an axis, +2 diagonally; nnz is the
    count of in-grid offsets with |dx|+|dy| <= 2; products = Σ_k len(A_k)^2."""
    nx = 64
    A = W.poisson2d(nx)
    rp, col, val, _ = oracle.spgemm(A, A)
    prods, maxlen, cmin, cmax, (sp, pmax) = oracle.row_analysis(A, A)
    lens = np.diff(A.row_ptr.numpy())
    assert sp == int((lens.astype(np.int64) ** 2).sum()) == 100104
    nnz = 0
    for y in range(nx):
        for x in range(nx):
            nnz += sum(1 for dy in range(-2, 3) for dx in range(-2, 3)
                       if abs(dx) + abs(dy) <= 2 and 0 <= x + dx < nx and 0 <= y + dy < nx)
    assert rp[-1] == nnz == 51972
    for i in range(nx * nx):
        x, y = i % nx, i // nx
        deg = sum(1 for dx, dy in ((1, 0), (-1, 0), (0, 1), (0, -1)) if 0 <= x + dx < nx and 0 <= y + dy < nx)
        for p in range(rp[i], rp[i + 1]):
            j = col[p]
            dx, dy = j % nx - x, j // nx - y
            d1 = abs(dx) + abs(dy)
            want = 16 + deg if d1 == 0 else -8 if d1 == 1 else (1 if dx == 0 or dy == 0 else 2)
            assert val[p] == want, (i, j)


@pytest.mark.parametrize("nf", [8, 16])
def test_galerkin_kronecker_closed_form(nf):
    """C2: A27 = 27I - T3^(x3), P = P1^(x3) =>  AP = 27P - (T3 P1)^(x3) and
    R·AP = 27 (P1^T P1)^(x3) - (P1^T T3 P1)^(x3); structural nnz(AP) = nnz(T3P1)^3."""
    A, P, R = W.amg27(nf)
    nc = nf // 2
    T3 = np.eye(nf) + np.eye(nf, k=1) + np.eye(nf, k=-1)
    P1 = np.zeros((nf, nc))
    for J in range(nc):
        P1[2 * J, J] = 1.0
        P1[2 * J + 1, J] = 0.5
        if 2 * J - 1 >= 0:
            P1[2 * J - 1, J] = 0.5

    def k3(M):
        return np.kron(np.kron(M, M), M)

    rp, col, val, _ = oracle.spgemm(A, P)
    D, PAT = csr_dense(rp, col, val, nf ** 3, nc ** 3)
    assert np.array_equal(D, 27 * k3(P1) - k3(T3 @ P1))
    assert np.array_equal(PAT, k3((T3 @ P1 != 0).astype(np.int64)))
    assert rp[-1] == int((T3 @ P1 != 0).sum()) ** 3
    assert (np.asarray(val) == 0).sum() > 0            # structural zeros are kept (reading R1)
    AP = W.CSR(nf ** 3, nc ** 3, torch.tensor(rp), torch.tensor(col), torch.tensor(val))
    rp2, col2, val2, _ = oracle.spgemm(R, AP)
    D2, _ = csr_dense(rp2, col2, val2, nc ** 3, nc ** 3)
    assert np.array_equal(D2, 27 * k3(P1.T @ P1) - k3(P1.T @ T3 @ P1))


def test_analysis_and_invariants_rmat():
    A = W.rmat(10, 8, seed=5, dtype=torch.float32)
    B = W.rmat(10, 8, seed=6, dtype=torch.float32)
    arp, acol, aval = A.numpy()
    brp, bcol, bval = B.numpy()
    prods, maxlen, cmin, cmax, (sp, pmax) = oracle.row_analysis(A, B)
    blen = np.diff(brp)
    # brute force Alg. 1 per row
    for i in range(A.rows):
        ks = acol[arp[i]:arp[i + 1]]
        assert prods[i] == blen[ks].sum()
        assert maxlen[i] == (blen[ks].max() if ks.size else 0)
        ne = [k for k in ks if blen[k] > 0]
        assert cmin[i] == (min(bcol[brp[k]] for k in ne) if ne else np.iinfo(np.int32).max)
        assert cmax[i] == (max(bcol[brp[k + 1] - 1] for k in ne) if ne else -1)
    # Σ prods by a second, independent formula: Σ_k colcount_A(k) · len(B_k)
    colcount = np.bincount(acol, minlength=A.cols)
    assert sp == int((colcount * blen).sum()) and pmax == prods.max()
    rp, col, val, scale = oracle.spgemm(A, B)
    assert_sorted_csr(rp, col, A.rows, B.cols)
    cnt = np.diff(rp)
    assert np.array_equal(cnt, oracle.symbolic(A, B))
    assert np.all(cnt >= maxlen) and np.all(cnt <= prods)
    has = cnt > 0
    assert np.all(cnt[has] <= (cmax - cmin + 1)[has])
    for i in np.nonzero(has)[0][:200]:
        assert col[rp[i]] == cmin[i] and col[rp[i + 1] - 1] == cmax[i]
    # single-NZ rows of A: C_i = a·B_k, bit exact, structure of B_k
    single = np.nonzero(np.diff(arp) == 1)[0]
    assert single.size > 0
    for i in single:
        k = acol[arp[i]]
        a = np.float64(aval[arp[i]])
        assert np.array_equal(col[rp[i]:rp[i + 1]], bcol[brp[k]:brp[k + 1]])
        assert np.array_equal(val[rp[i]:rp[i + 1]], a * bval[brp[k]:brp[k + 1]].astype(np.float64))


def test_transposition_identity():
    """S((A·B)^T) = S(B^T·A^T), values bit-identical (same k order)."""
    A = W.random_sparse(53, 47, 0.1, seed=21, dtype=torch.float64, empty_rows=0.1, zero_frac=0.1)
    B = W.random_sparse(47, 61, 0.1, seed=22, dtype=torch.float64, empty_rows=0.1)
    rp, col, val, _ = oracle.spgemm(A, B)
    C = W.CSR(53, 61, torch.tensor(rp), torch.tensor(col), torch.tensor(val))
    Ct = W.transpose(C)
    rp2, col2, val2, _ = oracle.spgemm(W.transpose(B), W.transpose(A))
    assert np.array_equal(rp2, Ct.row_ptr.numpy()) and np.array_equal(col2, Ct.col.numpy())
    assert np.array_equal(val2, Ct.val.numpy())


def test_scipy_pattern_crosscheck():
    """Library cross-check on pattern (all-positive) matrices: no cancellation, so scipy's
    zero-dropping cannot hide structure."""
    sp = pytest.importorskip("scipy.sparse")
    A = W.rmat(11, 8, seed=31, dtype=torch.float64)
    A.val = A.val.abs() + 0.5
    arp, acol, aval = A.numpy()
    S = sp.csr_matrix((aval, acol, arp), shape=(A.rows, A.cols))
    ref = (S @ S).tocsr()
    ref.sort_indices()
    rp, col, val, _ = oracle.spgemm(A, A)
    assert np.array_equal(rp, ref.indptr) and np.array_equal(col, ref.indices)
    assert np.allclose(val, ref.data, rtol=1e-13)


def test_row_blocks_streaming_matches_full():
    A = W.rmat(10, 8, seed=8, dtype=torch.float32)
    rp, col, val, _ = oracle.spgemm(A, A)
    r0, r1 = 300, 777
    rpb, colb, valb, _ = oracle.spgemm(A, A, r0, r1)
    assert np.array_equal(rpb, rp[r0:r1 + 1] - rp[r0])
    assert np.array_equal(colb, col[rp[r0]:rp[r1]]) and np.array_equal(valb, val[rp[r0]:rp[r1]])


# ----------------------------------------------------------------- worked examples
def test_fig1_group_iterations():
    kv, rows = golden("fig1_group_iters.txt")
    lens = [int(x) for x in kv["lens"].split()]
    T = int(kv["T"])
    for g, it in rows:
        assert oracle.group_iters(lens, T, int(g)) == int(it)


def test_fig3_block_merge():
    kv, _ = golden("fig3_block_merge.txt")
    needs = [int(x) for x in kv["needs"].split()]
    cap = int(kv["cap"])
    for lv, key in ((1, "level1"), (2, "level2"), (3, "level3")):
        bs, bl = oracle.block_merge(needs, cap, levels=lv)
        sums = [sum(needs[s:s + l]) for s, l in zip(bs, bl)]
        assert sums == [int(x) for x in kv[key].split()], key
    bs, bl = oracle.block_merge(needs, cap)
    sums = [sum(needs[s:s + l]) for s, l in zip(bs, bl)]
    assert sums == [int(x) for x in kv["final"].split()]
    assert all(s < cap or l == 1 for s, l in zip(sums, bl))
    assert int(kv["optimal_blocks"]) < len(sums)


def test_block_merge_properties():
    rng = np.random.default_rng(1)
    for trial in range(50):
        n = int(rng.integers(1, 300))
        cap = int(rng.integers(2, 100))
        needs = rng.integers(0, cap, n)
        bs, bl = oracle.block_merge(needs, cap)
        assert bs[0] == 0 and np.array_equal(np.cumsum(bl)[:-1], bs[1:]) and bl.sum() == n
        assert bl.max() <= 32
        for s, l in zip(bs, bl):
            assert l == 1 or needs[s:s + l].sum() < cap
        # within-50% guarantee: two neighbouring blocks inside one 32-row group
        # could not be merged -> their sum is >= cap
        for j in range(len(bs) - 1):
            if bs[j] // 32 == bs[j + 1] // 32:
                assert needs[bs[j]:bs[j] + bl[j]].sum() + needs[bs[j + 1]:bs[j + 1] + bl[j + 1]].sum() >= cap


def test_fig4_hash_linear_probing():
    kv, _ = golden("fig4_hash.txt")
    size = int(kv["size"])
    enc = lambda s: int(s[1]) * 2 + int(s[3])       # "rXcY" -> row*2 + col
    keys, homes = [], []
    for tok in kv["inserts"].split():
        name, h = tok.split(":")
        keys.append(enc(name)); homes.append(int(h))
    sk, sc = oracle.hash_insert(keys, homes, size)
    want = kv["final"].split()
    for s, w in enumerate(want):
        if w == "-":
            assert sk[s] == -1
        else:
            name, c = w.split("|")
            assert sk[s] == enc(name) and sc[s] == int(c)


def test_fig5_dense_windows():
    kv, _ = golden("fig5_dense.txt")
    Wd = int(kv["window"]); n = int(kv["ncols"])
    cols = [int(x) for x in kv["products"].split()]
    w, c, v = oracle.dense_windows(cols, [1.0] * len(cols), 0, n - 1, Wd)
    got = [f"{a}:{b}:{int(x)}" for a, b, x in zip(w, c, v)]
    assert got == kv["out"].split()


def test_group_size_properties():
    rng = np.random.default_rng(2)
    for _ in range(500):
        T = int(2 ** rng.integers(5, 11))
        nnzA = int(rng.integers(1, 5000))
        maxlen = int(rng.integers(1, 10000))
        prods = int(rng.integers(maxlen, maxlen * nnzA + 1))
        g = oracle.group_size(T, nnzA, prods, maxlen)
        assert 1 <= g <= T and (g & (g - 1)) == 0
        assert T // g <= max(nnzA, 1) or g == T
    # Fig. 1 situation: avg len 3 -> g starts at 4; iter_max = 2, n_rows = 4/2 = 2 -> keep 4
    assert oracle.group_size(8, 4, 12, 7) == 4


def test_group_size_sqrt_branches_hand_derived():
    """Reading R9, both sqrt branches and the final k <= NNZ_A clamp, each value
    derived by hand from the formula (not by calling the oracle):
    (a) T=256, nnzA=64, maxlen=4288, prods=4351: avg 67.98 -> g=64, k=4, iter_max=ceil(4288/64)=67,
        n_rows=16; 67 > 2*16 -> g = 64*sqrt(67/32) = 92.6 -> closest power of two in linear
        distance: 64 (28.6 < 35.4).  Dropping the sqrt gives 134 -> 128; log-distance rounding
        gives 128; dropping the factor 2 gives 64*sqrt(67/16) = 131 -> 128.
    (b) T=256, nnzA=1024, maxlen=16, prods=4096: avg 4 -> g=4, k=64, iter_max=4, n_rows=16;
        16 > 2*4 -> g = 4*sqrt(4/16) = 2.  Without the sqrt: 4*4/16 = 1.
    (c) T=1024, nnzA=3, maxlen=2, prods=6: g=2, k=512, iter_max=1, n_rows=3/512; first branch
        -> 2*sqrt(1/(2*3/512)) = 18.5 -> 16; k = 64 > nnzA = 3 -> k = 2 (largest pow2 <= 3),
        g = 1024/2 = 512."""
    assert oracle.group_size(256, 64, 4351, 4288) == 64
    assert oracle.group_size(256, 1024, 4096, 16) == 2
    assert oracle.group_size(1024, 3, 6, 2) == 512
    # neither branch: (T=256, nnzA=64, maxlen=64, prods=4096): g=64, k=4, iter_max=1, n_rows=16
    # -> 16 > 2 -> g = 64*sqrt(1/16) = 16
    assert oracle.group_size(256, 64, 4096, 64) == 16


def test_check_csr_rejects_each_violation():
    """oracle_check_csr (columns strictly ascending inside a row, in [0, ncols)) returns
    the first offending row for each kind of violation and -1 only for valid CSR."""
    rp = np.array([0, 2, 4, 6], np.int64)
    ok = np.array([0, 3, 1, 2, 0, 4], np.int32)
    assert oracle.check_csr(3, 5, rp, ok) == -1
    assert oracle.check_csr(3, 5, rp, np.array([0, 3, 2, 1, 0, 4], np.int32)) == 1     # unsorted row 1
    assert oracle.check_csr(3, 5, rp, np.array([0, 3, 1, 2, 4, 4], np.int32)) == 2     # duplicate in row 2
    assert oracle.check_csr(3, 5, rp, np.array([0, 5, 1, 2, 0, 4], np.int32)) == 0     # column == ncols
    assert oracle.check_csr(3, 5, rp, np.array([0, 3, -1, 2, 0, 4], np.int32)) == 1    # negative column
    assert oracle.check_csr(3, 5, np.array([0, 2, 1, 6], np.int64), ok) == 1           # decreasing row_ptr
    assert oracle.check_csr(0, 5, np.array([0], np.int64), np.zeros(0, np.int32)) == -1


# ----------------------------------------------------------------- the comparator itself
def _cmp_case():
    rp = np.array([0, 2, 3], np.int64)
    col = np.array([1, 4, 0], np.int32)
    val = np.array([1.0, -2.0, 0.0])
    scale = np.array([1.0, 2.0, 0.0])
    return rp, col, val, scale


def test_compare_accepts_exact_and_within_tolerance():
    rp, col, val, scale = _cmp_case()
    assert oracle.compare(rp, col, val, rp, col, val, scale, 1e-5)["ok"]
    g = val.copy(); g[0] += 0.5e-5 * scale[0]; g[2] = -0.0        # half of tol·s; -0 where s = 0
    assert oracle.compare(rp + 7, col, g, rp, col, val, scale, 1e-5)["ok"]   # offsets compared relative


@pytest.mark.parametrize("kind", ["nan", "inf", "ulp_past_tol", "nonzero_where_s0", "swapped_col",
                                  "off_by_one_rowptr", "short_arrays"])
def test_compare_rejects(kind):
    """Every parity claim rests on oracle.compare: each plausible GPU error must fail it."""
    rp, col, val, scale = _cmp_case()
    g_rp, g_col, g_val = rp.copy(), col.copy(), val.copy()
    if kind == "nan":
        g_val[1] = np.nan
    elif kind == "inf":
        g_val[0] = np.inf
    elif kind == "ulp_past_tol":
        g_val = np.array([0.0, -2.0, 0.0]); r = np.array([0.0, -2.0, 0.0]); s = np.array([1.0, 2.0, 0.0])
        g_val[0] = np.nextafter(1e-5, 1.0)                          # one ulp beyond tol·s = 1e-5
        res = oracle.compare(rp, col, g_val, rp, col, r, s, 1e-5)
        assert not res["ok"] and res["n_viol"] == 1 and res["first_bad"] == 0
        return
    elif kind == "nonzero_where_s0":
        g_val[2] = 1e-300
    elif kind == "swapped_col":
        g_col[[0, 1]] = g_col[[1, 0]]
    elif kind == "off_by_one_rowptr":
        g_rp[1] += 1
    elif kind == "short_arrays":
        g_col, g_val = g_col[:2], g_val[:2]
    res = oracle.compare(g_rp, g_col, g_val, rp, col, val, scale, 1e-5)
    assert not res["ok"], (kind, res)
    if kind in ("nan", "inf"):
        assert res["n_nonfinite"] == 1


def test_compare_nan_even_with_huge_tolerance():
    rp, col, val, scale = _cmp_case()
    g = val.copy(); g[0] = np.nan
    assert not oracle.compare(rp, col, g, rp, col, val, scale, 1e300)["ok"]


# ----------------------------------------------------------------- sequential (deterministic) values
def test_sequential_sum_order_and_precision_pin():
    """oracle.spgemm_sequential adds left to right in the inputs' precision (reading R15): for
    fp32, 1e8 + 1 - 1e8 in that order is 0 (1e8 + 1 rounds to 1e8 in float), 1 in exact
    arithmetic; reordered as 1e8 - 1e8 + 1 it is 1.  fp64 keeps the 1 (53-bit significand)."""
    for dt, want in ((torch.float32, 0.0), (torch.float64, 1.0)):
        A = W.CSR(1, 3, torch.tensor([0, 3]), torch.tensor([0, 1, 2], dtype=torch.int32), torch.ones(3, dtype=dt))
        B = W.CSR(3, 2, torch.tensor([0, 1, 2, 3]), torch.tensor([1, 1, 1], dtype=torch.int32),
                  torch.tensor([1e8, 1.0, -1e8], dtype=dt))
        rp, col, val = oracle.spgemm_sequential(A, B)
        assert col.tolist() == [1] and val.tolist() == [want]
        B2 = W.CSR(3, 2, torch.tensor([0, 1, 2, 3]), torch.tensor([1, 1, 1], dtype=torch.int32),
                   torch.tensor([1e8, -1e8, 1.0], dtype=dt))
        assert oracle.spgemm_sequential(A, B2)[2].tolist() == [1.0]
        # the exact oracle keeps the 1 either way
        assert oracle.spgemm(A, B)[2].tolist() == [1.0]


def test_sequential_equals_exact_on_integer_values():
    """With small-integer values every order gives the exact result (C1 closed form)."""
    A = W.poisson2d(32)
    rp, col, val = oracle.spgemm_sequential(A, A)
    rp2, col2, val2, _ = oracle.spgemm(A, A)
    assert np.array_equal(rp, rp2) and np.array_equal(col, col2) and np.array_equal(val, val2)
    # single product per entry (diagonal scaling): fl(a*b) exactly
    D = W.CSR(50, 50, torch.arange(51), torch.arange(50, dtype=torch.int32), torch.linspace(0.1, 5, 50, dtype=torch.float32))
    B = W.random_sparse(50, 40, 0.2, seed=9, dtype=torch.float32)
    _, _, v = oracle.spgemm_sequential(D, B)
    Bd = B.val.numpy()
    want = np.concatenate([(np.float32(D.val[i].item()) * Bd[B.row_ptr[i]:B.row_ptr[i + 1]]).astype(np.float32)
                           for i in range(50)])
    assert np.array_equal(v, want.astype(np.float64))
