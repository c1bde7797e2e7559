"""Seeded synthetic inputs shared by the oracle tests, the CUDA-path tests and bench.py.

This module holds NONE of the SpGEMM method's arithmetic.  It only builds input
matrices (CSR triples) with the shapes and structure of the workloads named in
BASELINE.json / SURVEY.md §8(d):

  C1  2-D 5-point Poisson Laplacian on a 64x64 grid (A·A, fp64)
  C2  3-D 27-point stencil on 128^3 with trilinear prolongation P and R = P^T
      (the AMG Galerkin chain A·P then R·(AP), fp64)
  C3  R-MAT Graph500 (a,b,c,d) = (.57,.19,.19,.05), scale 20, edge factor 16 (fp32)
  C4  mixed: uniform 8 nnz/row plus 64 rows of 200k nnz, n = 2^20 (fp32)
  C5  R-MAT (.45,.15,.15,.25), scale 24, edge factor 16 (fp32) — SURVEY §0 finding 2

Randomness is a counter-based generator (splitmix64 of (seed, stream, index)) written
with torch int64 tensor ops, so the same seed gives bit-identical matrices on CPU and
on CUDA: tests build small cases on the CPU, bench.py builds the big ones on the GPU,
and the oracle always receives a host copy of exactly what the CUDA path multiplied.

The CSR convention is the paper's (§1): row_ptr int64 [rows+1], col int32
sorted strictly ascending within a row, values fp32 or fp64.  A CSR transpose lives
here too, but only to *prepare inputs* (R = P^T is precomputed and untimed, like the
paper's A^T).
"""
from __future__ import annotations

import dataclasses
from typing import Optional

import numpy as np
import torch

__all__ = [
    "CSR", "splitmix64", "uniform01", "uniform_pm1", "csr_from_coo", "transpose",
    "poisson2d", "amg27", "rmat", "mixed", "random_sparse", "config", "CONFIGS",
]

_MASK = {k: (1 << (64 - k)) - 1 for k in range(1, 64)}


def _s64(x: int) -> int:
    """Python int in [0, 2^64) -> the int64 with the same bit pattern."""
    x &= (1 << 64) - 1
    return x - (1 << 64) if x >= (1 << 63) else x


_GOLDEN = _s64(0x9E3779B97F4A7C15)
_M1 = _s64(0xBF58476D1CE4E5B9)
_M2 = _s64(0x94D049BB133111EB)


def _srl(x: torch.Tensor, k: int) -> torch.Tensor:
    """Logical right shift of int64 bit patterns (torch >> is arithmetic)."""
    return (x >> k) & _MASK[k]


def splitmix64(seed: int, stream: int, idx: torch.Tensor) -> torch.Tensor:
    """splitmix64 finaliser of (seed, stream, idx): int64 tensor of 64 random bits.

    Wrapping int64 multiply is used on both devices, so results are device-independent.
    """
    base = _s64(seed * 0x632BE59BD9B4E019 + stream * 0xD1B54A32D192ED03)
    z = idx.to(torch.int64) * _GOLDEN + base
    z = (z ^ _srl(z, 30)) * _M1
    z = (z ^ _srl(z, 27)) * _M2
    return z ^ _srl(z, 31)


def uniform01(seed: int, stream: int, idx: torch.Tensor, dtype=torch.float64) -> torch.Tensor:
    """U[0,1) from the top 53 (fp64) or 24 (fp32) random bits — exact in that dtype."""
    r = splitmix64(seed, stream, idx)
    if dtype == torch.float32:
        return _srl(r, 40).to(torch.float32) * (1.0 / (1 << 24))
    return _srl(r, 11).to(torch.float64) * (1.0 / (1 << 53))


def uniform_pm1(seed: int, stream: int, idx: torch.Tensor, dtype) -> torch.Tensor:
    """U[-1,1) in `dtype` (exact dyadic values; 2u-1 is exact)."""
    return uniform01(seed, stream, idx, dtype) * 2 - 1


@dataclasses.dataclass
class CSR:
    """A CSR triple.  Tensors may live on CPU or CUDA."""
    rows: int
    cols: int
    row_ptr: torch.Tensor   # int64 [rows+1]
    col: torch.Tensor       # int32 [nnz]
    val: torch.Tensor       # float32 / float64 [nnz]

    @property
    def nnz(self) -> int:
        return int(self.col.numel())

    @property
    def dtype(self):
        return self.val.dtype

    @property
    def device(self):
        return self.col.device

    def to(self, device) -> "CSR":
        return CSR(self.rows, self.cols, self.row_ptr.to(device), self.col.to(device), self.val.to(device))

    def numpy(self):
        """(row_ptr, col, val) as contiguous numpy arrays on the host."""
        return (self.row_ptr.cpu().contiguous().numpy(), self.col.cpu().contiguous().numpy(),
                self.val.cpu().contiguous().numpy())

    def row_lengths(self) -> torch.Tensor:
        return self.row_ptr[1:] - self.row_ptr[:-1]

    def nbytes(self) -> int:
        return self.row_ptr.numel() * 8 + self.col.numel() * 4 + self.val.numel() * self.val.element_size()


def csr_from_coo(rows: int, cols: int, r: torch.Tensor, c: torch.Tensor, v: Optional[torch.Tensor],
                 dtype=torch.float64, dedup: bool = True, seed: int = 0, stream: int = 7) -> CSR:
    """Sort (r, c) row-major/column-minor, drop duplicate coordinates, build CSR.

    If v is None the values are U[-1,1) drawn by final entry index (so they do not
    depend on the duplicate pattern's history).
    """
    dev = r.device
    key = r.to(torch.int64) * cols + c.to(torch.int64)
    if dedup:
        if v is not None:
            key, inv = torch.unique(key, sorted=True, return_inverse=True)
            vv = torch.zeros(key.numel(), dtype=v.dtype, device=dev)
            vv.index_add_(0, inv, v)   # duplicates merged by summation (inputs only)
            v = vv
        else:
            key = torch.unique(key, sorted=True)
    else:
        key, order = torch.sort(key, stable=True)
        if v is not None:
            v = v[order]
    rr = torch.div(key, cols, rounding_mode="floor")
    cc = (key - rr * cols).to(torch.int32)
    counts = torch.bincount(rr, minlength=rows) if rr.numel() else torch.zeros(rows, dtype=torch.int64, device=dev)
    row_ptr = torch.zeros(rows + 1, dtype=torch.int64, device=dev)
    row_ptr[1:] = torch.cumsum(counts, 0)
    if v is None:
        v = uniform_pm1(seed, stream, torch.arange(key.numel(), device=dev), dtype)
    return CSR(rows, cols, row_ptr, cc, v.to(dtype))


def transpose(A: CSR) -> CSR:
    """Explicit CSR transpose (input preparation only: R = P^T, A^T for A·A^T)."""
    dev = A.col.device
    r = torch.repeat_interleave(torch.arange(A.rows, device=dev, dtype=torch.int64), A.row_lengths())
    return csr_from_coo(A.cols, A.rows, A.col.to(torch.int64), r, A.val, dtype=A.dtype, dedup=False)


# ----------------------------------------------------------------------------- C1
def poisson2d(nx: int = 64, ny: Optional[int] = None, dtype=torch.float64, device="cpu") -> CSR:
    """2-D 5-point Laplacian, Dirichlet: 4 on the diagonal, -1 to grid neighbours.

    A = I (x) T + T (x) I with T = tridiag(-1, 2, -1); node index i = y*nx + x.
    """
    ny = nx if ny is None else ny
    n = nx * ny
    idx = torch.arange(n, device=device, dtype=torch.int64)
    x, y = idx % nx, idx // nx
    rs, cs, vs = [], [], []
    for dy, dx, w in ((-1, 0, -1.0), (0, -1, -1.0), (0, 0, 4.0), (0, 1, -1.0), (1, 0, -1.0)):
        ok = (x + dx >= 0) & (x + dx < nx) & (y + dy >= 0) & (y + dy < ny)
        rs.append(idx[ok]); cs.append(idx[ok] + dy * nx + dx)
        vs.append(torch.full((int(ok.sum()),), w, dtype=dtype, device=device))
    return csr_from_coo(n, n, torch.cat(rs), torch.cat(cs), torch.cat(vs), dtype=dtype)


# ----------------------------------------------------------------------------- C2
def _p1(nf: int, dtype, device):
    """1-D linear-interpolation prolongation P1 (nf x nf/2): P1[2J,J]=1, P1[2J±1,J]=1/2."""
    nc = nf // 2
    J = torch.arange(nc, device=device, dtype=torch.int64)
    r = torch.cat([2 * J, 2 * J + 1, 2 * J - 1])
    c = torch.cat([J, J, J])
    v = torch.cat([torch.ones(nc, dtype=dtype, device=device), torch.full((nc,), 0.5, dtype=dtype, device=device),
                   torch.full((nc,), 0.5, dtype=dtype, device=device)])
    ok = (r >= 0) & (r < nf)
    return r[ok], c[ok], v[ok], nc


def amg27(nf: int = 128, dtype=torch.float64, device="cpu"):
    """AMG Galerkin inputs on an nf^3 grid: (A27, P, R=P^T).

    A27 = 27 I - T3 (x) T3 (x) T3, T3 = tridiag(1,1,1): 26 on the diagonal, -1 to the
    26 neighbours (no boundary modification).  P = P1 (x) P1 (x) P1 (rows 1/2/4/8 nnz).
    Node index i = (z*nf + y)*nf + x.
    """
    n = nf ** 3
    idx = torch.arange(n, device=device, dtype=torch.int64)
    x, y, z = idx % nf, (idx // nf) % nf, idx // (nf * nf)
    rs, cs, vs = [], [], []
    for dz in (-1, 0, 1):
        for dy in (-1, 0, 1):
            for dx in (-1, 0, 1):
                ok = ((x + dx >= 0) & (x + dx < nf) & (y + dy >= 0) & (y + dy < nf) & (z + dz >= 0) & (z + dz < nf))
                w = 26.0 if (dx, dy, dz) == (0, 0, 0) else -1.0
                rs.append(idx[ok]); cs.append(idx[ok] + (dz * nf + dy) * nf + dx)
                vs.append(torch.full((int(ok.sum()),), w, dtype=dtype, device=device))
    A = csr_from_coo(n, n, torch.cat(rs), torch.cat(cs), torch.cat(vs), dtype=dtype)
    pr, pc, pv, nc = _p1(nf, dtype, device)
    # Kronecker product P1 (x) P1 (x) P1 by broadcasting the 1-D entries
    e = pr.numel()
    iz, iy, ix = torch.meshgrid(torch.arange(e, device=device), torch.arange(e, device=device),
                                torch.arange(e, device=device), indexing="ij")
    iz, iy, ix = iz.reshape(-1), iy.reshape(-1), ix.reshape(-1)
    R3 = (pr[iz] * nf + pr[iy]) * nf + pr[ix]
    C3 = (pc[iz] * nc + pc[iy]) * nc + pc[ix]
    V3 = pv[iz] * pv[iy] * pv[ix]
    P = csr_from_coo(n, nc ** 3, R3, C3, V3, dtype=dtype)
    return A, P, transpose(P)


# ----------------------------------------------------------------------------- C3 / C5
def rmat(scale: int, edge_factor: int = 16, abcd=(0.57, 0.19, 0.19, 0.05), seed: int = 42,
         dtype=torch.float32, device="cpu", permute: bool = True) -> CSR:
    """R-MAT graph (Chakrabarti et al.; Graph500 generator without per-level noise).

    2^scale vertices, edge_factor*2^scale generated directed edges, self loops kept,
    duplicates merged, ids relabelled by one seeded random permutation applied to rows
    and columns, values U[-1,1).
    """
    n = 1 << scale
    E = edge_factor * n
    a, b, c, _ = abcd
    t1, t2, t3 = a, a + b, a + b + c
    e = torch.arange(E, device=device, dtype=torch.int64)
    r = torch.zeros(E, dtype=torch.int64, device=device)
    cc = torch.zeros(E, dtype=torch.int64, device=device)
    for lvl in range(scale):
        u = uniform01(seed, 100 + lvl, e, torch.float64)
        rbit = (u >= t2).to(torch.int64)
        cbit = (((u >= t1) & (u < t2)) | (u >= t3)).to(torch.int64)
        r = r * 2 + rbit
        cc = cc * 2 + cbit
        del u, rbit, cbit
    del e
    if permute:
        perm_keys = splitmix64(seed, 99, torch.arange(n, device=device, dtype=torch.int64))
        perm = torch.argsort(perm_keys, stable=True)
        del perm_keys
        r = perm[r]
        cc = perm[cc]
        del perm
    return csr_from_coo(n, n, r, cc, None, dtype=dtype, seed=seed, stream=7)


# ----------------------------------------------------------------------------- C4
def mixed(n: int = 1 << 20, per_row: int = 8, n_long: int = 64, long_len: int = 200_000, seed: int = 7,
          dtype=torch.float32, device="cpu") -> CSR:
    """Uniform random rows of `per_row` distinct columns plus `n_long` rows of `long_len`
    distinct uniform columns (rows chosen uniformly without replacement)."""
    long_rows = torch.argsort(splitmix64(seed, 1, torch.arange(n, device=device)), stable=True)[:n_long]
    is_long = torch.zeros(n, dtype=torch.bool, device=device)
    is_long[long_rows] = True
    short = torch.nonzero(~is_long).reshape(-1)
    # short rows: draw 2*per_row candidates per row, keep the first per_row distinct ones (draw order)
    k = 2 * per_row
    ci = torch.arange(short.numel() * k, device=device, dtype=torch.int64)
    cand = (splitmix64(seed, 2, ci) & ((1 << 62) - 1)) % n
    cand = cand.view(-1, k)
    srt, order = torch.sort(cand, dim=1, stable=True)
    dup = torch.zeros_like(srt, dtype=torch.bool)
    dup[:, 1:] = srt[:, 1:] == srt[:, :-1]
    first = torch.ones_like(cand, dtype=torch.bool)
    first.scatter_(1, order, ~dup)          # True for the first (in draw order) copy of each column
    rank = torch.cumsum(first.to(torch.int64), dim=1)
    keep = first & (rank <= per_row)
    assert bool((keep.sum(1) == per_row).all()), "mixed(): not enough distinct candidates"
    rs = [short.view(-1, 1).expand(-1, k)[keep]]
    cs = [cand[keep]]
    # long rows: first long_len entries of a seeded permutation of the columns
    for j in range(n_long):
        p = torch.argsort(splitmix64(seed, 1000 + j, torch.arange(n, device=device)), stable=True)[:long_len]
        rs.append(torch.full((long_len,), int(long_rows[j]), dtype=torch.int64, device=device))
        cs.append(p)
    return csr_from_coo(n, n, torch.cat(rs), torch.cat(cs), None, dtype=dtype, seed=seed, stream=8)


# ----------------------------------------------------------------------------- tests
def random_sparse(rows: int, cols: int, density: float, seed: int, dtype=torch.float64, device="cpu",
                  empty_rows: float = 0.0, int_values: bool = False, zero_frac: float = 0.0) -> CSR:
    """Uniform random pattern with optional empty rows, small-integer values or explicit zeros."""
    tot = rows * cols
    idx = torch.arange(tot, device=device, dtype=torch.int64)
    keep = uniform01(seed, 1, idx) < density
    if empty_rows > 0:
        er = uniform01(seed, 2, torch.arange(rows, device=device)) < empty_rows
        keep &= ~er.repeat_interleave(cols)
    sel = idx[keep]
    r, c = sel // cols, sel % cols
    if int_values:
        v = ((splitmix64(seed, 3, sel) & 7) - 3).to(dtype)        # {-3..4}, exact in any order
    else:
        v = uniform_pm1(seed, 3, sel, dtype)
    if zero_frac > 0:
        v = torch.where(uniform01(seed, 4, sel) < zero_frac, torch.zeros_like(v), v)
    return csr_from_coo(rows, cols, r, c, v, dtype=dtype, dedup=False)


def uniform_rows(rows: int, cols: int, lmin: int, lmax: int, seed: int, dtype=torch.float32, device="cpu") -> CSR:
    """Rows of lmin..lmax uniform random columns (row length uniform in [lmin, lmax]; columns drawn
    with replacement, repeated draws merged, so a row may come out slightly shorter)."""
    span = lmax - lmin + 1
    L = lmin + (splitmix64(seed, 1, torch.arange(rows, device=device)) & ((1 << 62) - 1)) % span
    r = torch.repeat_interleave(torch.arange(rows, device=device), L)
    c = (splitmix64(seed, 2, torch.arange(r.numel(), device=device)) & ((1 << 62) - 1)) % cols
    return csr_from_coo(rows, cols, r, c, None, dtype=dtype, seed=seed, stream=3)


CONFIGS = {
    "c1": "2D 5-point Poisson 64x64, A*A, fp64",
    "c2": "3D 27-point 128^3 AMG Galerkin R*(A*P), fp64",
    "c3": "R-MAT Graph500 scale 20 ef16, A*A, fp32",
    "c4": "mixed 2^20: 8/row + 64 rows x 200k, A*A, fp32",
    "c5": "R-MAT (.45,.15,.15,.25) scale 24 ef16, A*A, fp32",
}


def config(name: str, device="cpu", small: bool = False):
    """Return the list of SpGEMM problems [(label, A, B), ...] of a named workload.

    `small=True` gives the same structure at reduced size (for oracle-speed tests).
    C2 returns the two products of the Galerkin chain: AP = A·P, then Ac = R·AP; the
    second B is produced by the first product, so the caller supplies it (see
    bench.py/tests); here B of the second problem is None.
    """
    if name == "c1":
        A = poisson2d(16 if small else 64, device=device)
        return [("A*A", A, A)]
    if name == "c2":
        A, P, R = amg27(16 if small else 128, device=device)
        return [("A*P", A, P), ("R*(AP)", R, None)]
    if name == "c3":
        A = rmat(12 if small else 20, 16, (0.57, 0.19, 0.19, 0.05), seed=42, device=device)
        return [("A*A", A, A)]
    if name == "c4":
        A = mixed(1 << 14, 8, 4, 3000, seed=7, device=device) if small else mixed(device=device)
        return [("A*A", A, A)]
    if name == "c5":
        A = rmat(14 if small else 24, 16, (0.45, 0.15, 0.15, 0.25), seed=42, device=device)
        return [("A*A", A, A)]
    raise KeyError(name)
