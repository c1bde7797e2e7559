"""CPU oracle for the spECK hot path — TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / `--impl reference`
legs may import this package.  The product package (paper_conf_ppopp_pargerwms20_b200)
never imports it and shares no code with it; see oracle/speck_oracle.c for what each
function follows in the paper (P:line = /root/reference/PAPER.md).

This module is argument marshalling (numpy <-> ctypes) around the plain C oracle plus
the comparison rule of north_star (structure bit-exact; |c - r| <= tol·Σ|a·b|).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from typing import Optional, Tuple

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "speck_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

TOL = {np.dtype(np.float32): 1e-5, np.dtype(np.float64): 1e-12}   # north_star tolerances


def build(force: bool = False) -> str:
    """Compile the C oracle (gcc -O2 -fopenmp).  Building the checker is not using it."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-shared", "-fPIC", "-std=c11", "-Wall",
                               "-o", _LIB, _SRC, "-lm"])
    return _LIB


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        P = ctypes.c_void_p
        I64 = ctypes.c_int64
        L.oracle_row_analysis.argtypes = [I64, P, P, P, P, P, P, P, P, P]
        L.oracle_symbolic.argtypes = [P, P, P, P, I64, I64, I64, P]
        L.oracle_numeric.argtypes = [P, P, P, P, P, P, ctypes.c_int, I64, I64, I64, P, P, P, P]
        L.oracle_numeric_sequential.argtypes = [P, P, P, P, P, P, ctypes.c_int, I64, I64, I64, P, P, P]
        L.oracle_block_merge.argtypes = [I64, P, I64, ctypes.c_int, P, P]
        L.oracle_block_merge.restype = I64
        L.oracle_group_iters.argtypes = [I64, P, I64, I64]
        L.oracle_group_iters.restype = I64
        L.oracle_group_size.argtypes = [I64, I64, I64, I64]
        L.oracle_group_size.restype = I64
        L.oracle_hash_insert.argtypes = [I64, P, P, I64, P, P]
        L.oracle_dense_windows.argtypes = [I64, P, P, ctypes.c_int32, ctypes.c_int32, I64, P, P, P]
        L.oracle_dense_windows.restype = I64
        L.oracle_check_csr.argtypes = [I64, I64, P, P]
        L.oracle_check_csr.restype = I64
        L.oracle_num_threads.restype = ctypes.c_int
        L.oracle_set_threads.argtypes = [ctypes.c_int]
        _lib = L
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def _host(M):
    """Accept a workloads.CSR (any device) or a (rows, cols, rp, col, val) tuple."""
    if hasattr(M, "numpy"):
        rp, col, val = M.numpy()
        return M.rows, M.cols, np.ascontiguousarray(rp, np.int64), np.ascontiguousarray(col, np.int32), np.ascontiguousarray(val)
    rows, cols, rp, col, val = M
    return rows, cols, np.ascontiguousarray(rp, np.int64), np.ascontiguousarray(col, np.int32), np.ascontiguousarray(val)


def num_threads() -> int:
    return int(lib().oracle_num_threads())


def set_threads(n: int) -> None:
    lib().oracle_set_threads(int(n))


def check_csr(rows, cols, rp, col) -> int:
    rp = np.ascontiguousarray(rp, np.int64); col = np.ascontiguousarray(col, np.int32)
    return int(lib().oracle_check_csr(rows, cols, _p(rp), _p(col)))


def row_analysis(A, B):
    """Algorithm 1: per-row (prods, maxlen, colmin, colmax) + (Σprods, max prods)."""
    m, k, arp, acol, _ = _host(A)
    kb, n, brp, bcol, _ = _host(B)
    assert k == kb
    prods = np.empty(m, np.int64); maxlen = np.empty(m, np.int32)
    cmin = np.empty(m, np.int32); cmax = np.empty(m, np.int32); stats = np.zeros(2, np.int64)
    lib().oracle_row_analysis(m, _p(arp), _p(acol), _p(brp), _p(bcol), _p(prods), _p(maxlen), _p(cmin), _p(cmax), _p(stats))
    return prods, maxlen, cmin, cmax, (int(stats[0]), int(stats[1]))


def symbolic(A, B, r0: int = 0, r1: Optional[int] = None) -> np.ndarray:
    """Structural nnz of rows [r0, r1) of C = A·B."""
    m, k, arp, acol, _ = _host(A)
    kb, n, brp, bcol, _ = _host(B)
    assert k == kb
    r1 = m if r1 is None else r1
    cnt = np.empty(r1 - r0, np.int64)
    err = lib().oracle_symbolic(_p(arp), _p(acol), _p(brp), _p(bcol), n, r0, r1, _p(cnt))
    if err:
        raise RuntimeError(f"oracle_symbolic error {err}")
    return cnt


def spgemm(A, B, r0: int = 0, r1: Optional[int] = None, with_scale: bool = True):
    """C = A·B rows [r0, r1) (eq. (1)), sorted CSR with structural zeros kept.

    Returns (row_ptr int64 [r1-r0+1] starting at 0, col int32, val float64, scale float64).
    """
    m, k, arp, acol, aval = _host(A)
    kb, n, brp, bcol, bval = _host(B)
    assert k == kb, "dimension mismatch"
    assert aval.dtype == bval.dtype, "dtype mismatch"
    is64 = 1 if aval.dtype == np.float64 else 0
    r1 = m if r1 is None else r1
    cnt = symbolic((m, k, arp, acol, aval), (kb, n, brp, bcol, bval), r0, r1)
    rp = np.zeros(r1 - r0 + 1, np.int64)
    np.cumsum(cnt, out=rp[1:])
    nnz = int(rp[-1])
    col = np.empty(nnz, np.int32); val = np.empty(nnz, np.float64)
    scale = np.empty(nnz, np.float64) if with_scale else None
    err = lib().oracle_numeric(_p(arp), _p(acol), _p(aval), _p(brp), _p(bcol), _p(bval), is64, n, r0, r1,
                               _p(rp), _p(col), _p(val), _p(scale) if with_scale else None)
    if err:
        raise RuntimeError(f"oracle_numeric error {err}")
    return rp, col, val, scale


def spgemm_sequential(A, B, r0: int = 0, r1: Optional[int] = None):
    """C = A·B rows [r0, r1) with every sum taken left to right in the inputs' precision, each
    product rounded before it is added (reading R15; the deterministic mode's exact bits).
    Returns (row_ptr, col, val as float64 holding the fp32/fp64 results)."""
    m, k, arp, acol, aval = _host(A)
    kb, n, brp, bcol, bval = _host(B)
    assert k == kb and aval.dtype == bval.dtype
    is64 = 1 if aval.dtype == np.float64 else 0
    r1 = m if r1 is None else r1
    cnt = symbolic((m, k, arp, acol, aval), (kb, n, brp, bcol, bval), r0, r1)
    rp = np.zeros(r1 - r0 + 1, np.int64)
    np.cumsum(cnt, out=rp[1:])
    col = np.empty(int(rp[-1]), np.int32); val = np.empty(int(rp[-1]), np.float64)
    err = lib().oracle_numeric_sequential(_p(arp), _p(acol), _p(aval), _p(brp), _p(bcol), _p(bval), is64, n, r0, r1,
                                          _p(rp), _p(col), _p(val))
    if err:
        raise RuntimeError(f"oracle_numeric_sequential error {err}")
    return rp, col, val


def block_merge(needs, cap: int, levels: int = 5):
    """Algorithm 2 under reading R10 -> (block_start, block_len)."""
    b = np.ascontiguousarray(needs, np.int64)
    n = b.size
    bs = np.empty(max(n, 1), np.int64); bl = np.empty(max(n, 1), np.int64)
    nb = lib().oracle_block_merge(n, _p(b), cap, levels, _p(bs), _p(bl))
    if nb < 0:
        raise MemoryError
    return bs[:nb].copy(), bl[:nb].copy()


def group_iters(lens, T: int, g: int) -> int:
    """Fig. 1 iteration model."""
    l = np.ascontiguousarray(lens, np.int64)
    return int(lib().oracle_group_iters(l.size, _p(l), T, g))


def group_size(T: int, nnzA: int, prods: int, maxlen: int) -> int:
    """Local load balancer group size g (reading R9)."""
    return int(lib().oracle_group_size(T, nnzA, prods, maxlen))


def hash_insert(keys, homes, size: int):
    """Linear-probing insert-or-count with injected home slots (Fig. 4)."""
    k = np.ascontiguousarray(keys, np.int64); h = np.ascontiguousarray(homes, np.int64)
    sk = np.empty(size, np.int64); sc = np.empty(size, np.int64)
    if lib().oracle_hash_insert(k.size, _p(k), _p(h), size, _p(sk), _p(sc)) != 0:
        raise OverflowError("hash map full")
    return sk, sc


def dense_windows(cols, vals, colmin: int, colmax: int, W: int):
    """Windowed dense accumulation (Fig. 5) -> (window, col, val) arrays."""
    c = np.ascontiguousarray(cols, np.int32); v = np.ascontiguousarray(vals, np.float64)
    cap = c.size
    ow = np.empty(max(cap, 1), np.int64); oc = np.empty(max(cap, 1), np.int32); ov = np.empty(max(cap, 1), np.float64)
    ne = lib().oracle_dense_windows(c.size, _p(c), _p(v), colmin, colmax, W, _p(ow), _p(oc), _p(ov))
    return ow[:ne].copy(), oc[:ne].copy(), ov[:ne].copy()


def compare(rp_gpu, col_gpu, val_gpu, rp_ref, col_ref, val_ref, scale_ref, tol: float):
    """north_star parity rule on one row block.

    row_ptr and col must be bit-exact; |c - r| <= tol·s per entry, and c == ±0 when s == 0.
    A non-finite GPU value (NaN, ±Inf) always fails: inputs are finite by contract (reading
    R14), so every reference value and scale is finite.  The test is written as
    `not (rel <= tol)` so that a NaN anywhere in the arithmetic counts as a violation.
    Returns dict(ok, rp_ok, col_mismatch, first_bad, max_rel, n_viol, n_nonfinite).
    """
    rp_gpu = np.asarray(rp_gpu, np.int64); rp_ref = np.asarray(rp_ref, np.int64)
    rp_ok = rp_gpu.shape == rp_ref.shape and rp_gpu.size > 0 and \
        bool(np.array_equal(rp_gpu - rp_gpu[0], rp_ref - rp_ref[0]))
    out = {"rp_ok": rp_ok, "col_mismatch": None, "first_bad": None, "max_rel": 0.0, "n_viol": 0, "n_nonfinite": 0}
    if not rp_ok:
        out["ok"] = False
        return out
    n = int(rp_ref[-1] - rp_ref[0])
    col_gpu = np.asarray(col_gpu); col_ref = np.asarray(col_ref)
    c = np.asarray(val_gpu, np.float64); r = np.asarray(val_ref, np.float64); s = np.asarray(scale_ref, np.float64)
    if not (col_gpu.size == col_ref.size == c.size == r.size == s.size == n):
        out["ok"] = False
        out["col_mismatch"] = -1           # array lengths disagree with row_ptr
        return out
    neq = np.nonzero(col_gpu != col_ref)[0]
    out["col_mismatch"] = int(neq.size)
    if neq.size:
        out["first_bad"] = int(neq[0])
        out["ok"] = False
        return out
    err = np.abs(c - r)
    with np.errstate(divide="ignore", invalid="ignore"):
        rel = np.where(s > 0, err / np.where(s > 0, s, 1.0), np.where(err == 0, 0.0, np.inf))
    nonfinite = ~np.isfinite(c)
    bad = ~(rel <= tol) | nonfinite
    out["n_nonfinite"] = int(nonfinite.sum())
    out["n_viol"] = int(bad.sum())
    out["max_rel"] = float(np.max(np.where(np.isnan(rel), np.inf, rel))) if rel.size else 0.0
    if out["n_viol"]:
        out["first_bad"] = int(np.nonzero(bad)[0][0])
    out["ok"] = out["n_viol"] == 0
    return out
