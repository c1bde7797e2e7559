"""Row-size histogram of a workload on the GPU: rows / products / nnz(C) / nnz(A) per
power-of-two bucket of nnz(C_i), plus the library's bin counts.  Diagnostic only.

    python tools/binstats.py c5
"""
import json
import sys

import torch

sys.path.insert(0, ".")
import workloads as W  # noqa: E402
import paper_conf_ppopp_pargerwms20_b200 as sp  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "c5"
dev = torch.device("cuda", 0)
probs = W.config(cfg, device=dev)
for name, A, B in probs[:1] if cfg != "c2" else [(p[0], p[1], p[2]) for p in probs[:1]]:
    h = sp.Handle(0, stage_timing=1)
    C = h.spgemm(A, B)
    torch.cuda.synchronize()
    st = h.stats()
    prods = h.row_analysis(A, B)[0].double()
    cnt = (C.row_ptr[1:] - C.row_ptr[:-1]).double()
    nnza = (A.row_ptr[1:] - A.row_ptr[:-1]).double()
    b = torch.where(cnt > 0, torch.floor(torch.log2(cnt.clamp(min=1))), torch.full_like(cnt, -1)).long()
    print(json.dumps({k: st[k] for k in ("rows_per_bin_symbolic", "rows_per_bin_numeric", "rows_dense_numeric",
                                          "segments", "products", "nnz_c")}))
    print(f"{'cnt bucket':>14s} {'rows':>10s} {'prods':>14s} {'nnzC':>14s} {'nnzA':>12s} {'prod%':>6s} {'avgA':>6s}")
    P = prods.sum().item()
    for k in range(-1, int(b.max().item()) + 1):
        m = b == k
        n = int(m.sum().item())
        if n == 0:
            continue
        pk = prods[m].sum().item()
        lo, hi = (0, 0) if k < 0 else (1 << k, (2 << k) - 1)
        print(f"{lo:>6d}-{hi:<7d} {n:10d} {pk:14.0f} {cnt[m].sum().item():14.0f} {nnza[m].sum().item():12.0f} "
              f"{100 * pk / P:6.2f} {nnza[m].mean().item():6.1f}")
