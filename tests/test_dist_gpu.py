"""Multi-GPU row partitioner with the REAL kernels: two processes share cuda:0
(the round's boxes have one GPU) with the gloo backend; B is replicated from rank 0 with
`broadcast_csr`, every rank multiplies its balanced row block through libspeck.so
(`spgemm_rowsharded`'s default local multiply) and the row blocks are assembled with
`allgather_csr`.  Rank 0 compares the assembled C with the CPU oracle, element by element."""
import os
import socket

import numpy as np
import pytest
import torch

import oracle
import workloads as W

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q, dtype_name):
    import torch.distributed as dist
    from paper_conf_ppopp_pargerwms20_b200 import dist as sdist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        dt = getattr(torch, dtype_name)
        A = W.rmat(12, 16, seed=77, dtype=dt)
        Ad = A.to("cuda")
        B = sdist.broadcast_csr(Ad if rank == 0 else None, src=0, device="cuda:0")
        blk = sdist.spgemm_rowsharded(Ad, B)            # libspeck.so local multiply
        full = sdist.allgather_csr(blk, A.rows)
        torch.cuda.synchronize()
        q.put((rank, blk.r0, blk.r1, blk.nnz, blk.off, full.row_ptr.cpu().numpy(), full.col.cpu().numpy(),
               full.val.cpu().numpy().astype(np.float64)))
    except Exception as e:
        q.put((rank, repr(e)))
        raise
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("dtype_name", ["float32", "float64"])
def test_rowsharded_real_kernels_two_ranks(dtype_name):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import torch.multiprocessing as mp
    from paper_conf_ppopp_pargerwms20_b200 import build
    build.build()
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q, dtype_name)) for r in range(world)]
    for p in procs:
        p.start()
    outs = {}
    for _ in range(world):
        item = q.get(timeout=600)
        assert len(item) > 2, f"rank {item[0]} failed: {item[1]}"
        outs[item[0]] = item
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    A = W.rmat(12, 16, seed=77, dtype=getattr(torch, dtype_name))
    rp, col, val, scale = oracle.spgemm(A, A)
    # the two row blocks tile the rows; offsets are the exclusive scan of the per-rank nnz
    (_, r0a, r1a, nza, offa, *_), (_, r0b, r1b, nzb, offb, *_) = outs[0], outs[1]
    assert (r0a, r1b) == (0, A.rows) and r1a == r0b and offa == 0 and offb == nza
    assert nza + nzb == int(rp[-1])
    tol = oracle.TOL[np.dtype(np.float32 if dtype_name == "float32" else np.float64)]
    for r in (0, 1):
        _, _, _, _, _, grp, gcol, gval = outs[r]
        res = oracle.compare(grp, gcol, gval, rp, col, val, scale, tol)
        assert res["ok"], (r, res)


def _grid_worker(rank, world, port, q):
    import torch.distributed as dist
    from paper_conf_ppopp_pargerwms20_b200 import dist as sdist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        A = W.rmat(12, 16, seed=78, dtype=torch.float32).to("cuda")
        group = dist.new_group([0, 1])
        cb = sdist.column_bounds(A.cols, world)                 # 1 x 2 grid: B split by columns
        B_j = sdist.column_block(A, cb[rank], cb[rank + 1])
        tile = sdist.spgemm_2d_tile(A, B_j)                     # libspeck.so
        C = sdist.assemble_row_block(tile, cb[rank], group, A.cols)
        torch.cuda.synchronize()
        q.put((rank, int(B_j.col.numel()), A.nnz, C.row_ptr.cpu().numpy(), C.col.cpu().numpy(),
               C.val.cpu().numpy().astype(np.float64)))
    except Exception as e:
        q.put((rank, repr(e)))
        raise
    finally:
        dist.destroy_process_group()


def test_2d_grid_real_kernels():
    """1 x 2 grid on one GPU: each rank keeps half of B's columns, multiplies with
    libspeck.so, and the assembled rows equal the oracle's."""
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import torch.multiprocessing as mp
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_grid_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    outs = {}
    for _ in range(world):
        item = q.get(timeout=600)
        assert len(item) > 2, f"rank {item[0]} failed: {item[1]}"
        outs[item[0]] = item
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    A = W.rmat(12, 16, seed=78, dtype=torch.float32)
    rp, col, val, scale = oracle.spgemm(A, A)
    for r in (0, 1):
        _, bnnz, annz, grp, gcol, gval = outs[r]
        assert bnnz < 0.75 * annz
        res = oracle.compare(grp, gcol, gval, rp, col, val, scale, 1e-5)
        assert res["ok"], (r, res)
