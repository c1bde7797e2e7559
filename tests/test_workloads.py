"""The seeded input generators: determinism, shapes and closed-form sizes of the workloads
(SURVEY.md §8.0 / §8(d)).  No method arithmetic lives in workloads/."""
import numpy as np
import torch

import oracle
import workloads as W


def test_counter_rng_is_deterministic_and_uniform():
    idx = torch.arange(200_000)
    a = W.uniform01(5, 3, idx)
    b = W.uniform01(5, 3, idx)
    assert torch.equal(a, b)
    assert not torch.equal(a, W.uniform01(6, 3, idx)) and not torch.equal(a, W.uniform01(5, 4, idx))
    assert 0.0 <= float(a.min()) and float(a.max()) < 1.0
    assert abs(float(a.mean()) - 0.5) < 5e-3
    f = W.uniform_pm1(1, 1, idx, torch.float32)
    assert f.dtype == torch.float32 and -1.0 <= float(f.min()) and float(f.max()) < 1.0


def test_amg27_closed_form_sizes():
    for nf in (8, 16):
        A, P, R = W.amg27(nf)
        nc = nf // 2
        assert A.nnz == (3 * nf - 2) ** 3                  # 27-point stencil without boundary modification
        nnz_p1 = nc + nc + (nc - 1)                         # P1[2J,J], P1[2J+1,J], P1[2J-1,J] (J>=1)
        assert P.nnz == nnz_p1 ** 3 and set(P.row_lengths().unique().tolist()) <= {1, 2, 4, 8}
        assert (P.rows, P.cols, R.rows, R.cols) == (nf ** 3, nc ** 3, nc ** 3, nf ** 3)
        # R is exactly P^T
        Pd = np.zeros((P.rows, P.cols)); Rd = np.zeros((R.rows, R.cols))
        prp, pc, pv = P.numpy(); rrp, rc, rv = R.numpy()
        for i in range(P.rows):
            Pd[i, pc[prp[i]:prp[i + 1]]] = pv[prp[i]:prp[i + 1]]
        for i in range(R.rows):
            Rd[i, rc[rrp[i]:rrp[i + 1]]] = rv[rrp[i]:rrp[i + 1]]
        assert np.array_equal(Pd.T, Rd)
        assert oracle.check_csr(A.rows, A.cols, *A.numpy()[:2]) == -1
    # full-size sizes of config[1] by the same closed forms
    assert (3 * 128 - 2) ** 3 == 55_742_968 and (64 + 64 + 63) ** 3 == 6_967_871


def test_rmat_and_mixed():
    A = W.rmat(10, 8, seed=3)
    B = W.rmat(10, 8, seed=3)
    assert torch.equal(A.col, B.col) and torch.equal(A.val, B.val) and torch.equal(A.row_ptr, B.row_ptr)
    assert A.nnz <= 8 * 1024 and oracle.check_csr(A.rows, A.cols, *A.numpy()[:2]) == -1
    M = W.mixed(1 << 12, 8, 3, 500, seed=7)
    lens = M.row_lengths().numpy()
    assert M.nnz == 3 * 500 + ((1 << 12) - 3) * 8
    assert sorted(set(lens.tolist())) == [8, 500] and (lens == 500).sum() == 3
    assert oracle.check_csr(M.rows, M.cols, *M.numpy()[:2]) == -1


def test_transpose_roundtrip():
    A = W.random_sparse(37, 53, 0.1, seed=2, zero_frac=0.2)
    T = W.transpose(W.transpose(A))
    assert torch.equal(T.row_ptr, A.row_ptr) and torch.equal(T.col, A.col) and torch.equal(T.val, A.val)


def test_uniform_rows():
    A = W.uniform_rows(500, 100_000, 3, 40, seed=5)
    B = W.uniform_rows(500, 100_000, 3, 40, seed=5)
    assert torch.equal(A.row_ptr, B.row_ptr) and torch.equal(A.col, B.col) and torch.equal(A.val, B.val)
    lens = (A.row_ptr[1:] - A.row_ptr[:-1])
    assert int(lens.min()) >= 1 and int(lens.max()) <= 40 and abs(float(lens.double().mean()) - 21.5) < 2
    for i in range(0, 500, 50):                    # sorted, distinct, in range
        c = A.col[A.row_ptr[i]:A.row_ptr[i + 1]]
        assert bool((c[1:] > c[:-1]).all()) and int(c.min()) >= 0 and int(c.max()) < 100_000
