"""Thin Python binding of libspeck.so (include/speck.h) — argument marshalling only.

Every step of the SpGEMM path runs in the CUDA kernels of libspeck.so; this module only
turns torch CUDA tensors into the C ABI's device pointers and back.  There is no CPU or
library fallback: if the extension is missing or no CUDA device is present, calls raise.

    import paper_conf_ppopp_pargerwms20_b200 as speck
    C = speck.spgemm(A, B)            # A, B: objects with rows, cols, row_ptr, col, val (cuda)
"""
from __future__ import annotations

import ctypes
import dataclasses
import os
from typing import Optional

import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libspeck.so")

SPECK_F32, SPECK_F64 = 0, 1
OPT = {
    "global_lb_symbolic": 0, "global_lb_numeric": 1, "force_accumulator": 2, "dense_window": 3,
    "stage_timing": 4, "validate": 5, "disable_direct": 6, "fixed_group_size": 7, "concurrent_streams": 8,
    "segments": 9, "warp_rows": 10, "long_bitmap": 11, "bitmap_reuse": 12, "kernel_timing": 13,
    "path_counters": 14, "bucket_sort": 15, "deterministic": 16,
}
# speck_kernel_kind_t (kernel id = kind * 16 + configuration)
KERNEL_KINDS = {1: "analysis", 2: "binning", 3: "scan", 4: "sym_warp", 5: "sym_block", 6: "num_tiny", 7: "num_warp",
                8: "num_block", 9: "direct", 10: "segments", 11: "long_bitmap", 12: "seg_plan"}
# speck_path_t
PATHS = ["sym_warp", "sym_block_hash", "sym_merged", "sym_dense", "sym_dense_multi", "num_tiny", "num_warp_ordered",
         "num_warp_sorted", "num_block_ordered", "num_block_sorted", "num_merged", "num_dense", "num_dense_multi",
         "num_direct", "seg_hash", "seg_dense", "seg_windows", "long_bitmap", "long_bitmap_split", "sym_esc", "num_esc",
         "num_esc_dup", "esc_fallback", "num_det"]
PATH_COUNT = 24
# bin categories of speck_stats_t.bin_* (per pass)
CATEGORIES = ["empty", "direct", "cfg0", "cfg1", "cfg2", "cfg3", "cfg4", "long", "tiny", "unused"]
STATUS = {
    0: "SPECK_OK", 1: "SPECK_ERR_INVALID_ARGUMENT", 2: "SPECK_ERR_DIMENSION_MISMATCH", 3: "SPECK_ERR_DTYPE_MISMATCH",
    4: "SPECK_ERR_UNSUPPORTED", 5: "SPECK_ERR_OUT_OF_MEMORY", 6: "SPECK_ERR_CUDA", 7: "SPECK_ERR_NOT_ANALYZED",
    8: "SPECK_ERR_INVALID_INPUT",
}
# every symbol include/speck.h declares
EXPORTS = [
    "speck_create", "speck_destroy", "speck_set_option", "speck_analyze", "speck_spgemm", "speck_row_analysis",
    "speck_get_stats", "speck_status_string", "speck_last_error", "speck_version", "speck_block_merge",
    "speck_group_size", "speck_hash_probe", "speck_exclusive_scan", "speck_row_products", "speck_set_allocator",
    "speck_spgemm_rows", "speck_row_chunks", "speck_transpose",
]
_ALLOC_FN = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_void_p)
_RELEASE_FN = ctypes.CFUNCTYPE(None, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p)


class SpeckError(RuntimeError):
    def __init__(self, status: int, detail: str = ""):
        self.status = status
        super().__init__(f"{STATUS.get(status, status)}: {detail}")


class _Csr(ctypes.Structure):
    _fields_ = [("rows", ctypes.c_int64), ("cols", ctypes.c_int64), ("nnz", ctypes.c_int64),
                ("row_ptr", ctypes.c_void_p), ("col_idx", ctypes.c_void_p), ("values", ctypes.c_void_p),
                ("dtype", ctypes.c_int)]


class Stats(ctypes.Structure):
    _fields_ = [("products", ctypes.c_int64), ("max_row_products", ctypes.c_int64), ("nnz_c", ctypes.c_int64),
                ("rows_direct", ctypes.c_int64), ("rows_empty", ctypes.c_int64), ("lb_symbolic", ctypes.c_int32),
                ("lb_numeric", ctypes.c_int32), ("rows_per_bin_symbolic", ctypes.c_int64 * 8),
                ("rows_per_bin_numeric", ctypes.c_int64 * 8), ("rows_dense_numeric", ctypes.c_int64),
                ("segments", ctypes.c_int64),
                ("workspace_bytes", ctypes.c_int64), ("kernel_launches", ctypes.c_int64), ("ms_analysis", ctypes.c_float), ("ms_symbolic_lb", ctypes.c_float),
                ("ms_symbolic", ctypes.c_float), ("ms_scan", ctypes.c_float), ("ms_numeric_lb", ctypes.c_float),
                ("ms_numeric", ctypes.c_float),
                ("bin_rows", (ctypes.c_int64 * 10) * 2), ("bin_nnza", (ctypes.c_int64 * 10) * 2),
                ("bin_products", (ctypes.c_int64 * 10) * 2), ("bin_nnzc", ctypes.c_int64 * 10),
                ("n_kernels", ctypes.c_int32), ("kernel_id", ctypes.c_int32 * 64), ("kernel_bin", ctypes.c_int32 * 64),
                ("kernel_ms", ctypes.c_float * 64), ("path_rows", ctypes.c_int64 * PATH_COUNT)]

    def as_dict(self):
        def conv(v):
            return [conv(x) for x in v] if hasattr(v, "__len__") else v
        d = {name: conv(getattr(self, name)) for name, _ in self._fields_}
        n = d["n_kernels"]
        d["kernels"] = [{"kind": KERNEL_KINDS.get(i >> 4, str(i >> 4)), "cfg": i & 15, "bin": b, "ms": ms}
                        for i, b, ms in zip(d["kernel_id"][:n], d["kernel_bin"][:n], d["kernel_ms"][:n])]
        d["paths"] = dict(zip(PATHS, d["path_rows"]))
        return d


_lib = None


def load() -> ctypes.CDLL:
    """Load the in-tree libspeck.so.  Raises if it has not been built (no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} not built: run `python -m paper_conf_ppopp_pargerwms20_b200.build`")
        L = ctypes.CDLL(LIB_PATH)
        P, I64, I32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32
        L.speck_create.argtypes = [ctypes.POINTER(P), ctypes.c_int]
        L.speck_destroy.argtypes = [P]
        L.speck_set_option.argtypes = [P, ctypes.c_int, I64]
        L.speck_analyze.argtypes = [P, ctypes.POINTER(_Csr), ctypes.POINTER(_Csr), P, ctypes.POINTER(I64), P]
        L.speck_spgemm.argtypes = [P, ctypes.POINTER(_Csr), ctypes.POINTER(_Csr), P, P, P, P]
        L.speck_row_analysis.argtypes = [P, ctypes.POINTER(_Csr), ctypes.POINTER(_Csr), P, P, P, P, P]
        L.speck_get_stats.argtypes = [P, ctypes.POINTER(Stats)]
        L.speck_status_string.argtypes = [ctypes.c_int]
        L.speck_status_string.restype = ctypes.c_char_p
        L.speck_last_error.argtypes = [P]
        L.speck_last_error.restype = ctypes.c_char_p
        L.speck_version.restype = ctypes.c_char_p
        L.speck_block_merge.argtypes = [P, P, I64, I64, P, P]
        L.speck_group_size.argtypes = [P, I32, P, P, P, I64, P, P]
        L.speck_hash_probe.argtypes = [P, P, P, I64, I32, P, P, P]
        L.speck_exclusive_scan.argtypes = [P, P, I64, P, P]
        L.speck_row_products.argtypes = [P, ctypes.POINTER(_Csr), ctypes.POINTER(_Csr), P, P]
        L.speck_set_allocator.argtypes = [P, _ALLOC_FN, _RELEASE_FN, P]
        L.speck_spgemm_rows.argtypes = [P, ctypes.POINTER(_Csr), ctypes.POINTER(_Csr), P, I64, I64, P, P, P]
        L.speck_row_chunks.argtypes = [P, P, I64, I64, P, I64, ctypes.POINTER(I64)]
        L.speck_transpose.argtypes = [P, ctypes.POINTER(_Csr), P, P, P, P]
        for f in EXPORTS:
            if f not in ("speck_status_string", "speck_last_error", "speck_version"):
                getattr(L, f).restype = ctypes.c_int
        _lib = L
    return _lib


def version() -> str:
    return load().speck_version().decode()


@dataclasses.dataclass
class CSR:
    """Result matrix C (device tensors): row_ptr int64 [rows+1], col int32, val fp32/fp64."""
    rows: int
    cols: int
    row_ptr: torch.Tensor
    col: torch.Tensor
    val: torch.Tensor

    @property
    def nnz(self) -> int:
        return int(self.col.numel())


def _dtype_code(t: torch.Tensor) -> int:
    if t.dtype == torch.float32:
        return SPECK_F32
    if t.dtype == torch.float64:
        return SPECK_F64
    raise TypeError(f"values must be float32 or float64, got {t.dtype}")


def _csr(M) -> _Csr:
    for name in ("row_ptr", "col", "val"):
        t = getattr(M, name)
        if not t.is_cuda:
            raise ValueError(f"{name} must be a CUDA tensor")
        if not t.is_contiguous():
            raise ValueError(f"{name} must be contiguous")
    if M.row_ptr.dtype != torch.int64 or M.col.dtype != torch.int32:
        raise TypeError("row_ptr must be int64 and col int32")
    return _Csr(M.rows, M.cols, M.col.numel(), M.row_ptr.data_ptr(), M.col.data_ptr(),
                M.val.data_ptr() if M.val.numel() else None, _dtype_code(M.val))


def _stream(stream) -> int:
    if stream is None:
        stream = torch.cuda.current_stream()
    return stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream)


def _ptr(t: Optional[torch.Tensor]):
    return None if t is None else t.data_ptr()


class Handle:
    """A libspeck handle (workspace + plan state), bound to one CUDA device."""

    def __init__(self, device: Optional[int] = None, torch_allocator: bool = True, **options):
        self._L = load()
        self.device = torch.cuda.current_device() if device is None else int(device)
        h = ctypes.c_void_p()
        st = self._L.speck_create(ctypes.byref(h), self.device)
        if st != 0:
            raise SpeckError(st, "speck_create failed (is a CUDA device available?)")
        self._h = h
        if torch_allocator:
            self.use_torch_allocator()
        for k, v in options.items():
            self.set_option(k, v)

    def use_torch_allocator(self):
        """Route the handle's workspace through PyTorch's caching allocator (speck_set_allocator)."""
        dev = self.device

        def _alloc(nbytes, stream, ctx):
            try:
                return torch.cuda.caching_allocator_alloc(int(nbytes), dev, stream or 0)
            except RuntimeError:
                return None

        def _release(ptr, stream, ctx):
            torch.cuda.caching_allocator_delete(ptr)

        self._alloc_cb, self._release_cb = _ALLOC_FN(_alloc), _RELEASE_FN(_release)   # keep alive
        self._check(self._L.speck_set_allocator(self._h, self._alloc_cb, self._release_cb, None))

    def close(self):
        if getattr(self, "_h", None):
            import sys
            if getattr(self, "_alloc_cb", None) is not None and sys.is_finalizing():
                self._h = None   # interpreter teardown: torch's allocator may be gone; the process frees all
                return
            self._L.speck_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def _check(self, st: int):
        if st != 0:
            raise SpeckError(st, self._L.speck_last_error(self._h).decode())

    def set_option(self, name, value: int):
        self._check(self._L.speck_set_option(self._h, OPT[name] if isinstance(name, str) else int(name), int(value)))

    # -- the pipeline ----------------------------------------------------------------------
    def analyze(self, A, B, C_row_ptr: Optional[torch.Tensor] = None, stream=None):
        """Symbolic phase -> (C_row_ptr, nnz_C)."""
        if C_row_ptr is None:
            C_row_ptr = torch.empty(A.rows + 1, dtype=torch.int64, device=A.row_ptr.device)
        self._A, self._B = _csr(A), _csr(B)
        nnz = ctypes.c_int64(0)
        self._check(self._L.speck_analyze(self._h, ctypes.byref(self._A), ctypes.byref(self._B), C_row_ptr.data_ptr(),
                                          ctypes.byref(nnz), _stream(stream)))
        return C_row_ptr, int(nnz.value)

    def numeric(self, A, B, C_row_ptr: torch.Tensor, C_col: torch.Tensor, C_val: torch.Tensor, stream=None):
        """Numeric phase into caller-allocated C_col / C_val (asynchronous)."""
        a, b = _csr(A), _csr(B)
        self._check(self._L.speck_spgemm(self._h, ctypes.byref(a), ctypes.byref(b), C_row_ptr.data_ptr(),
                                         _ptr(C_col), _ptr(C_val), _stream(stream)))

    def spgemm(self, A, B, stream=None) -> CSR:
        """C = A·B (analyze, allocate C with torch.empty, numeric)."""
        rp, nnz = self.analyze(A, B, stream=stream)
        dev = A.row_ptr.device
        col = torch.empty(nnz, dtype=torch.int32, device=dev)
        val = torch.empty(nnz, dtype=A.val.dtype, device=dev)
        self.numeric(A, B, rp, col, val, stream=stream)
        return CSR(A.rows, B.cols, rp, col, val)

    def numeric_rows(self, A, B, C_row_ptr: torch.Tensor, r0: int, r1: int, C_col: torch.Tensor, C_val: torch.Tensor,
                     stream=None):
        """Numeric phase of rows [r0, r1) into chunk buffers of C_row_ptr[r1] - C_row_ptr[r0] entries."""
        a, b = _csr(A), _csr(B)
        self._check(self._L.speck_spgemm_rows(self._h, ctypes.byref(a), ctypes.byref(b), C_row_ptr.data_ptr(), int(r0),
                                              int(r1), _ptr(C_col), _ptr(C_val), _stream(stream)))

    def row_chunks(self, C_row_ptr: torch.Tensor, max_nnz: int, max_parts: int = 1 << 16):
        """Row bounds [0, ..., rows] of consecutive chunks holding < max_nnz entries each."""
        import numpy as np
        bounds = np.zeros(max_parts + 1, np.int64)
        n = ctypes.c_int64(0)
        self._check(self._L.speck_row_chunks(self._h, C_row_ptr.data_ptr(), C_row_ptr.numel() - 1, int(max_nnz),
                                             bounds.ctypes.data, int(max_parts), ctypes.byref(n)))
        return [int(x) for x in bounds[:n.value + 1]]

    def spgemm_chunks(self, A, B, max_nnz: int, stream=None):
        """Memory-bounded C = A·B: analyze once, then yield (r0, r1, row_ptr_slice, col, val) for
        consecutive row chunks of < max_nnz entries; only one chunk's C is allocated at a time
        (the caller consumes it before asking for the next)."""
        rp, nnz = self.analyze(A, B, stream=stream)
        dev = A.row_ptr.device
        bounds = self.row_chunks(rp, max_nnz)
        for r0, r1 in zip(bounds[:-1], bounds[1:]):
            if r1 <= r0:
                continue
            off = rp[r0:r1 + 1] - rp[r0]
            n = int(off[-1])
            col = torch.empty(n, dtype=torch.int32, device=dev)
            val = torch.empty(n, dtype=A.val.dtype, device=dev)
            self.numeric_rows(A, B, rp, r0, r1, col, val, stream=stream)
            yield r0, r1, off, col, val

    def transpose(self, A, stream=None) -> CSR:
        """T = Aᵀ (sorted CSR) on the device (speck_transpose)."""
        dev = A.row_ptr.device
        rp = torch.empty(A.cols + 1, dtype=torch.int64, device=dev)
        col = torch.empty(A.col.numel(), dtype=torch.int32, device=dev)
        val = torch.empty(A.col.numel(), dtype=A.val.dtype, device=dev)
        self._check(self._L.speck_transpose(self._h, ctypes.byref(_csr(A)), rp.data_ptr(), _ptr(col),
                                            val.data_ptr() if A.val.numel() else None, _stream(stream)))
        return CSR(A.cols, A.rows, rp, col, val)

    def row_products(self, A, B, stream=None) -> torch.Tensor:
        """Alg. 1 line 10 per row: products int64 device tensor (speck_row_products)."""
        prods = torch.empty(A.rows, dtype=torch.int64, device=A.row_ptr.device)
        self._check(self._L.speck_row_products(self._h, ctypes.byref(_csr(A)), ctypes.byref(_csr(B)),
                                               prods.data_ptr(), _stream(stream)))
        return prods

    def row_analysis(self, A, B, stream=None):
        """Alg. 1 per row: (prods int64, maxlen int32, colmin int32, colmax int32) device tensors."""
        dev = A.row_ptr.device
        m = A.rows
        prods = torch.empty(m, dtype=torch.int64, device=dev)
        maxlen = torch.empty(m, dtype=torch.int32, device=dev)
        cmin = torch.empty(m, dtype=torch.int32, device=dev)
        cmax = torch.empty(m, dtype=torch.int32, device=dev)
        a, b = _csr(A), _csr(B)
        self._check(self._L.speck_row_analysis(self._h, ctypes.byref(a), ctypes.byref(b), _ptr(prods), _ptr(maxlen),
                                               _ptr(cmin), _ptr(cmax), _stream(stream)))
        return prods, maxlen, cmin, cmax

    def stats(self) -> dict:
        s = Stats()
        self._check(self._L.speck_get_stats(self._h, ctypes.byref(s)))
        return s.as_dict()

    # -- component entry points ------------------------------------------------------------
    def block_merge(self, needs: torch.Tensor, cap: int, stream=None) -> torch.Tensor:
        needs = needs.to(torch.int64).contiguous()
        flags = torch.empty(needs.numel(), dtype=torch.uint8, device=needs.device)
        self._check(self._L.speck_block_merge(self._h, needs.data_ptr(), needs.numel(), int(cap), flags.data_ptr(),
                                              _stream(stream)))
        return flags

    def group_size(self, T: int, nnzA: torch.Tensor, prods: torch.Tensor, maxlen: torch.Tensor, stream=None):
        n = nnzA.numel()
        nnzA, prods, maxlen = (x.to(torch.int64).contiguous() for x in (nnzA, prods, maxlen))
        g = torch.empty(n, dtype=torch.int32, device=nnzA.device)
        self._check(self._L.speck_group_size(self._h, int(T), nnzA.data_ptr(), prods.data_ptr(), maxlen.data_ptr(), n,
                                             g.data_ptr(), _stream(stream)))
        return g

    def hash_probe(self, keys: torch.Tensor, homes: torch.Tensor, size: int, stream=None):
        keys = keys.to(torch.int32).contiguous()
        homes = homes.to(torch.int32).contiguous()
        sk = torch.empty(size, dtype=torch.int32, device=keys.device)
        sc = torch.empty(size, dtype=torch.int32, device=keys.device)
        self._check(self._L.speck_hash_probe(self._h, keys.data_ptr(), homes.data_ptr(), keys.numel(), int(size),
                                             sk.data_ptr(), sc.data_ptr(), _stream(stream)))
        return sk, sc

    def exclusive_scan(self, x: torch.Tensor, stream=None) -> torch.Tensor:
        x = x.to(torch.int64).contiguous()
        out = torch.empty(x.numel() + 1, dtype=torch.int64, device=x.device)
        self._check(self._L.speck_exclusive_scan(self._h, x.data_ptr(), x.numel(), out.data_ptr(), _stream(stream)))
        return out


_default_handles = {}


def default_handle(device: Optional[int] = None) -> Handle:
    d = torch.cuda.current_device() if device is None else int(device)
    if d not in _default_handles:
        _default_handles[d] = Handle(d)
    return _default_handles[d]


def spgemm(A, B, stream=None, handle: Optional[Handle] = None) -> CSR:
    """C = A·B on the GPU (sorted CSR, structural zeros kept)."""
    return (handle or default_handle(A.row_ptr.device.index)).spgemm(A, B, stream=stream)
