"""Multi-process (world_size 2, gloo, CPU) tests of the row-block partitioner's host logic:
balanced product split, per-rank nnz all-gather -> global offsets, CSR all-gather, B
broadcast.  The local multiply is injected (the oracle, test-side) because the CUDA path
needs a GPU; on the GPU box the same code runs with libspeck.so and NCCL."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import workloads as W
from paper_conf_ppopp_pargerwms20_b200 import dist as sdist


def _oracle_local(A, B):
    tup = lambda M: (M.rows, M.cols, M.row_ptr.numpy(), M.col.numpy(), M.val.numpy())
    rp, col, val, _ = oracle.spgemm(tup(A), tup(B), with_scale=False)
    return W.CSR(A.rows, B.cols, torch.from_numpy(rp), torch.from_numpy(col),
                 torch.from_numpy(val).to(A.val.dtype))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        A = W.rmat(10, 16, seed=5, dtype=torch.float64)
        # B replicated from rank 0 (the NCCL protocol, here over gloo on CPU tensors)
        B = sdist.broadcast_csr(A if rank == 0 else None, src=0, device="cpu")
        prods = torch.from_numpy(oracle.row_analysis(A, A)[0])
        blk = sdist.spgemm_rowsharded(A, B, local=_oracle_local, prods=prods)
        full = sdist.allgather_csr(blk, A.rows)
        q.put((rank, blk.r0, blk.r1, blk.off, blk.total_nnz, blk.global_row_ptr().numpy(),
               full.row_ptr.numpy(), full.col.numpy(), full.val.numpy()))
    except Exception as e:        # report instead of leaving the peer blocked in a collective
        q.put((rank, repr(e)))
        raise
    finally:
        dist.destroy_process_group()


def test_rowsharded_two_ranks_gloo():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted([q.get(timeout=300) for _ in range(world)], key=lambda x: x[0])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    A = W.rmat(10, 16, seed=5, dtype=torch.float64)
    rp, col, val, _ = oracle.spgemm(A, A)
    # contiguous cover of the rows, offsets = exclusive scan of per-rank nnz
    assert res[0][1] == 0 and res[0][2] == res[1][1] and res[1][2] == A.rows
    assert res[0][3] == 0 and res[1][3] == rp[res[1][1]] and res[0][4] == res[1][4] == rp[-1]
    for r in res:
        r0, r1 = r[1], r[2]
        assert np.array_equal(r[5], rp[r0:r1 + 1])              # global row_ptr of the block
        assert np.array_equal(r[6], rp) and np.array_equal(r[7], col) and np.array_equal(r[8], val)


def test_partition_rows_balanced():
    rng = np.random.default_rng(0)
    prods = torch.tensor(rng.integers(0, 1000, 10000))
    for parts in (1, 2, 3, 4, 8):
        b = sdist.partition_rows(prods, parts)
        assert b[0] == 0 and b[-1] == 10000 and all(x <= y for x, y in zip(b, b[1:]))
        tot = int(prods.sum())
        loads = [int(prods[b[j]:b[j + 1]].sum()) for j in range(parts)]
        assert max(loads) <= tot / parts + 1000      # within one row of perfect balance
    # skewed: one huge row
    p = torch.ones(100, dtype=torch.int64); p[50] = 10**6
    b = sdist.partition_rows(p, 4)
    assert b[0] == 0 and b[-1] == 100


def _bcast_worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        A = W.random_sparse(50, 40, 0.1, seed=3) if rank == 0 else None
        M = sdist.broadcast_csr(A, src=0, device="cpu")
        q.put((rank, M.rows, M.cols, M.row_ptr.numpy(), M.col.numpy(), M.val.numpy()))
    finally:
        dist.destroy_process_group()


def test_broadcast_protocol_gloo():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_bcast_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted([q.get(timeout=300) for _ in range(world)], key=lambda x: x[0])
    for p in procs:
        p.join(timeout=60)
    assert res[0][1:3] == res[1][1:3]
    for a, b in zip(res[0][3:], res[1][3:]):
        assert np.array_equal(a, b)


def _grid_worker(rank, world, port, q, pr, pc):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        A = W.rmat(10, 16, seed=9, dtype=torch.float64)
        i, j = sdist.grid_coords(rank, pc)
        groups = [dist.new_group([ii * pc + jj for jj in range(pc)]) for ii in range(pr)]
        prods = torch.from_numpy(oracle.row_analysis(A, A)[0])
        rb = sdist.partition_rows(prods, pr)
        cb = sdist.column_bounds(A.cols, pc)
        A_i = sdist.row_slice(A, rb[i], rb[i + 1])
        B_j = sdist.column_block(A, cb[j], cb[j + 1])
        tile = sdist.spgemm_2d_tile(A_i, B_j, local=_oracle_local)
        Ci = sdist.assemble_row_block(tile, cb[j], groups[i], A.cols)
        q.put((rank, rb[i], rb[i + 1], int(B_j.col.numel()), A.nnz, Ci.row_ptr.numpy(), Ci.col.numpy(), Ci.val.numpy()))
    except Exception as e:
        q.put((rank, repr(e)))
        raise
    finally:
        dist.destroy_process_group()


def test_2d_grid_without_b_replication():
    """2 x 2 grid: rank (i, j) holds A's row block i and B's column block j only;
    the tiles C_ij assembled per row block equal the oracle's rows, and no rank stores more than
    ~half of B."""
    world, pr, pc = 4, 2, 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_grid_worker, args=(r, world, port, q, pr, pc)) for r in range(world)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(world):
        item = q.get(timeout=300)
        assert len(item) > 2, f"rank {item[0]} failed: {item[1]}"
        res[item[0]] = item
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    A = W.rmat(10, 16, seed=9, dtype=torch.float64)
    rp, col, val, _ = oracle.spgemm(A, A)
    for r, (_, r0, r1, bnnz, annz, crp, ccol, cval) in res.items():
        assert bnnz < 0.75 * annz                       # B is partitioned, not replicated
        assert np.array_equal(crp, rp[r0:r1 + 1] - rp[r0])
        assert np.array_equal(ccol, col[rp[r0]:rp[r1]])
        assert np.allclose(cval, val[rp[r0]:rp[r1]], rtol=1e-12, atol=0)
