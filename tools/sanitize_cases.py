"""Small SpGEMM cases for compute-sanitizer (memcheck / racecheck / synccheck / initcheck):
every accumulator path on inputs small enough for the tools' slowdown, each checked against
the oracle.  Run on the GPU box:

    compute-sanitizer --tool memcheck --error-exitcode 9 python tools/sanitize_cases.py
"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
import workloads as W  # noqa: E402
import paper_conf_ppopp_pargerwms20_b200 as sp  # noqa: E402


def check(A, B, **opts):
    h = sp.Handle(0, **opts)
    C = h.spgemm(A.to("cuda"), B.to("cuda"))
    torch.cuda.synchronize()
    tol = oracle.TOL[np.dtype(np.float64 if A.dtype == torch.float64 else np.float32)]
    rp, col, val, sc = oracle.spgemm(A, B)
    res = oracle.compare(C.row_ptr.cpu().numpy(), C.col.cpu().numpy(), C.val.cpu().numpy().astype(np.float64),
                         rp, col, val, sc, tol)
    h.close()
    assert res["ok"], (opts, res)


def main():
    cases = [(W.poisson2d(32), None, {}),
             (W.rmat(10, 16, seed=1, dtype=torch.float32), None, {}),
             (W.rmat(10, 16, seed=2, dtype=torch.float32), None, dict(bucket_sort=2)),
             (W.rmat(10, 16, seed=3, dtype=torch.float32), None, dict(bucket_sort=0, warp_rows=0)),
             (W.rmat(10, 16, seed=4, dtype=torch.float64), None, dict(force_accumulator=2, dense_window=64)),
             (W.rmat(10, 16, seed=5, dtype=torch.float32), None, dict(bucket_sort=0, fixed_group_size=-1)),
             (W.random_sparse(4, 1500, 0.5, seed=31, dtype=torch.float32),
              W.random_sparse(1500, 60_000, 0.01, seed=32, dtype=torch.float32), {}),
             (W.random_sparse(4, 1500, 0.5, seed=33, dtype=torch.float64),
              W.random_sparse(1500, 60_000, 0.01, seed=34, dtype=torch.float64), dict(segments=0))]
    A, P, R = W.amg27(16)
    cases.append((A, P, {}))
    for A, B, opts in cases:
        check(A, A if B is None else B, **opts)
    # transpose and chunked rows
    h = sp.Handle(0)
    Ad = W.rmat(10, 16, seed=6, dtype=torch.float32).to("cuda")
    T = h.transpose(Ad)
    chunks = list(h.spgemm_chunks(Ad, Ad, max_nnz=20000))
    torch.cuda.synchronize()
    print("sanitize cases ok:", len(cases), "spgemm,", len(chunks), "chunks, transpose", T.nnz)


if __name__ == "__main__":
    main()
