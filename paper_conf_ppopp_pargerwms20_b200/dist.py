"""Row-block multi-GPU partitioner (the paper names multi-GPU as future work,
P:2026-2028).

Rows of A are independent units of row-wise SpGEMM, so A's rows are
split into contiguous blocks of balanced product count and B is replicated.  Every rank:
  1. has the replicated B (and A) — broadcast from rank 0 with `broadcast_csr` (NCCL over
     NVLink) or regenerated deterministically;
  2. computes the split with `partition_rows` from the per-row products of Alg. 1
     (identical on every rank, so no communication is needed to agree on it);
  3. multiplies its row block locally (libspeck.so);
  4. all-gathers the per-rank nnz (8 B per rank) and turns its local row offsets into
     global ones: global row_ptr = local row_ptr + off_p (exclusive scan of nnz_p).
C stays row-sharded; `allgather_csr` assembles the full C where a later step needs it
(e.g. the second product of the Galerkin chain R·(A·P) needs all of A·P as its B).

The local multiply is a parameter so the host-side logic can be exercised with the gloo
backend on CPU; the default is the CUDA path.
"""
from __future__ import annotations

import dataclasses
from typing import Callable, List, Optional

import torch
import torch.distributed as dist


@dataclasses.dataclass
class RowBlock:
    """Rows [r0, r1) of a row-sharded CSR matrix; entries [off, off + nnz) of the global C."""
    rows: int
    cols: int
    row_ptr: torch.Tensor      # int64 [r1-r0+1], LOCAL offsets (start at 0)
    col: torch.Tensor
    val: torch.Tensor
    r0: int
    r1: int
    off: int                   # global offset of the block's first entry
    total_nnz: int             # nnz of the whole (global) matrix

    @property
    def nnz(self) -> int:
        return int(self.col.numel())

    def global_row_ptr(self) -> torch.Tensor:
        return self.row_ptr + self.off


def partition_rows(prods: torch.Tensor, parts: int) -> List[int]:
    """Contiguous row blocks with ~equal products: boundary j = first row whose inclusive
    product prefix reaches j·Σprods/parts.  Deterministic; returns [r_0=0, ..., r_parts=m]."""
    m = int(prods.numel())
    if parts <= 1 or m == 0:
        return [0, m]
    pre = torch.cumsum(prods.to(torch.int64).cpu(), 0)
    total = int(pre[-1]) if m else 0
    bounds = [0]
    for j in range(1, parts):
        target = (total * j + parts - 1) // parts
        r = int(torch.searchsorted(pre, torch.tensor([target], dtype=torch.int64), right=False)[0]) + 1
        bounds.append(min(max(r, bounds[-1]), m))
    bounds.append(m)
    return bounds


def row_slice(A, r0: int, r1: int):
    """Rows [r0, r1) of a CSR matrix as a CSR matrix (row_ptr rebased; col/val are views)."""
    a0 = int(A.row_ptr[r0])
    a1 = int(A.row_ptr[r1])
    rp = (A.row_ptr[r0:r1 + 1] - a0).contiguous()
    return type("CSRSlice", (), dict(rows=r1 - r0, cols=A.cols, row_ptr=rp, col=A.col[a0:a1], val=A.val[a0:a1]))()


def _default_local(A, B):
    from .speck import spgemm
    return spgemm(A, B)


def _default_prods(A, B):
    from .speck import default_handle
    return default_handle(A.row_ptr.device.index).row_products(A, B)


def broadcast_csr(M, src: int = 0, group=None, device=None):
    """Replicate a CSR matrix from `src` to every rank (NCCL broadcast of row_ptr/col/val).
    Non-source ranks pass M=None; `device` defaults to the current CUDA device."""
    rank = dist.get_rank(group)
    if M is not None:
        dev = M.row_ptr.device
    else:
        dev = torch.device(device) if device is not None else torch.device("cuda", torch.cuda.current_device())
    meta = torch.tensor([M.rows, M.cols, M.col.numel(), 1 if M.val.dtype == torch.float64 else 0] if rank == src
                        else [0, 0, 0, 0], dtype=torch.int64, device=dev)
    dist.broadcast(meta, src, group=group)
    rows, cols, nnz, is64 = (int(x) for x in meta.tolist())
    if rank != src:
        dt = torch.float64 if is64 else torch.float32
        M = type("CSRB", (), dict(rows=rows, cols=cols, row_ptr=torch.empty(rows + 1, dtype=torch.int64, device=dev),
                                  col=torch.empty(nnz, dtype=torch.int32, device=dev),
                                  val=torch.empty(nnz, dtype=dt, device=dev)))()
    for t in (M.row_ptr, M.col, M.val):
        dist.broadcast(t, src, group=group)
    return M


def spgemm_rowsharded(A, B, group=None, local: Optional[Callable] = None, prods: Optional[torch.Tensor] = None,
                      bounds: Optional[List[int]] = None) -> RowBlock:
    """This rank's row block of C = A·B (A and B replicated on every rank)."""
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    local = local or _default_local
    if bounds is None:
        if prods is None:
            prods = _default_prods(A, B)
        bounds = partition_rows(prods, world)
    r0, r1 = bounds[rank], bounds[rank + 1]
    C = local(row_slice(A, r0, r1), B)
    nnz = torch.tensor([C.col.numel()], dtype=torch.int64, device=C.row_ptr.device)
    all_nnz = [torch.zeros_like(nnz) for _ in range(world)]
    dist.all_gather(all_nnz, nnz, group=group)            # 8 B per rank
    sizes = [int(x) for x in torch.cat(all_nnz).tolist()]
    off = sum(sizes[:rank])
    return RowBlock(r1 - r0, C.cols if hasattr(C, "cols") else B.cols, C.row_ptr, C.col, C.val, r0, r1, off, sum(sizes))


def allgather_csr(blk: RowBlock, m: int, group=None):
    """Assemble the full row-sharded matrix on every rank (all_gather of the row blocks)."""
    world = dist.get_world_size(group)
    dev = blk.row_ptr.device
    meta = torch.tensor([blk.r0, blk.r1, blk.nnz], dtype=torch.int64, device=dev)
    metas = [torch.zeros_like(meta) for _ in range(world)]
    dist.all_gather(metas, meta, group=group)
    metas = [tuple(int(v) for v in x.tolist()) for x in metas]
    max_rows = max(r1 - r0 for r0, r1, _ in metas)
    max_nnz = max(n for _, _, n in metas)

    def gather(t: torch.Tensor, length: int, max_len: int):
        buf = torch.zeros(max_len, dtype=t.dtype, device=dev)
        buf[:length] = t[:length]
        outs = [torch.empty(max_len, dtype=t.dtype, device=dev) for _ in range(world)]
        dist.all_gather(outs, buf, group=group)
        return outs

    cnts = gather(blk.row_ptr[1:] - blk.row_ptr[:-1], blk.r1 - blk.r0, max(max_rows, 1))
    cols = gather(blk.col, blk.nnz, max(max_nnz, 1))
    vals = gather(blk.val, blk.nnz, max(max_nnz, 1))
    row_counts = torch.cat([c[:r1 - r0] for c, (r0, r1, _) in zip(cnts, metas)])
    row_ptr = torch.zeros(m + 1, dtype=torch.int64, device=dev)
    row_ptr[1:] = torch.cumsum(row_counts, 0)
    col = torch.cat([c[:n] for c, (_, _, n) in zip(cols, metas)])
    val = torch.cat([v[:n] for v, (_, _, n) in zip(vals, metas)])
    return type("CSRG", (), dict(rows=m, cols=blk.cols, row_ptr=row_ptr, col=col, val=val))()


# ------------------------------------------------------------------------------ 2-D grid
# multi-GPU without full replication of B ("shared matrix storage in multi-GPU
# setups").  Ranks form a pr x pc grid; rank (i, j) holds the row block A_i of A
# and the column block B_:j of B (columns [c_j, c_{j+1}) renumbered from 0), so each GPU stores
# 1/pc of B instead of all of it.  C_ij = A_i · B_:j is the (i, j) tile of C with local columns;
# the row block C_i is the concatenation, row by row, of C_i0, C_i1, ... with columns shifted by
# c_j (column blocks are disjoint and ordered, so the rows stay sorted).


def column_block(B, c0: int, c1: int):
    """Columns [c0, c1) of B renumbered from 0 (rows kept; the CSR slice rank (i, j) stores)."""
    rows = torch.repeat_interleave(torch.arange(B.rows, device=B.col.device), B.row_ptr[1:] - B.row_ptr[:-1])
    keep = (B.col >= c0) & (B.col < c1)
    counts = torch.bincount(rows[keep], minlength=B.rows)
    rp = torch.zeros(B.rows + 1, dtype=torch.int64, device=B.col.device)
    rp[1:] = torch.cumsum(counts, 0)
    return type("CSRCol", (), dict(rows=B.rows, cols=c1 - c0, row_ptr=rp, col=(B.col[keep] - c0).to(torch.int32),
                                   val=B.val[keep]))()


def column_bounds(ncols: int, parts: int) -> List[int]:
    return [ncols * j // parts for j in range(parts + 1)]


def grid_coords(rank: int, pc: int):
    return divmod(rank, pc)


def spgemm_2d_tile(A_i, B_j, local: Optional[Callable] = None):
    """This rank's tile C_ij = A_i · B_:j (local columns)."""
    return (local or _default_local)(A_i, B_j)


def assemble_row_block(tile, c0: int, row_group, n_cols: int):
    """Concatenate the tiles of one row block (all ranks of `row_group`, in column order) into
    the rows of C_i with global columns; every rank of the row group receives C_i."""
    world = dist.get_world_size(row_group)
    dev = tile.row_ptr.device
    m = tile.row_ptr.numel() - 1
    meta = torch.tensor([c0, tile.col.numel()], dtype=torch.int64, device=dev)
    metas = [torch.zeros_like(meta) for _ in range(world)]
    dist.all_gather(metas, meta, group=row_group)
    metas = [tuple(int(v) for v in x.tolist()) for x in metas]
    lens = [torch.empty(m, dtype=torch.int64, device=dev) for _ in range(world)]
    dist.all_gather(lens, (tile.row_ptr[1:] - tile.row_ptr[:-1]).contiguous(), group=row_group)
    mx = max(n for _, n in metas)
    cols, vals = [], []
    for t, src in ((tile.col, cols), (tile.val, vals)):
        buf = torch.zeros(max(mx, 1), dtype=t.dtype, device=dev)
        buf[:t.numel()] = t
        outs = [torch.empty(max(mx, 1), dtype=t.dtype, device=dev) for _ in range(world)]
        dist.all_gather(outs, buf, group=row_group)
        src.extend(outs)
    order = sorted(range(world), key=lambda q: metas[q][0])       # column order
    total = sum(lens)
    rp = torch.zeros(m + 1, dtype=torch.int64, device=dev)
    rp[1:] = torch.cumsum(total, 0)
    nnz = int(rp[-1])
    col = torch.empty(nnz, dtype=torch.int32, device=dev)
    val = torch.empty(nnz, dtype=tile.val.dtype, device=dev)
    before = torch.zeros(m, dtype=torch.int64, device=dev)        # entries of earlier column blocks per row
    for q in order:
        c0q, nq = metas[q]
        lq = lens[q]
        rows = torch.repeat_interleave(torch.arange(m, device=dev), lq)
        start = torch.zeros(m + 1, dtype=torch.int64, device=dev)
        start[1:] = torch.cumsum(lq, 0)
        t_in_row = torch.arange(nq, device=dev) - start[rows]
        dst = rp[rows] + before[rows] + t_in_row
        col[dst] = cols[q][:nq] + c0q
        val[dst] = vals[q][:nq]
        before += lq
    return type("CSRRow", (), dict(rows=m, cols=n_cols, row_ptr=rp, col=col, val=val))()
