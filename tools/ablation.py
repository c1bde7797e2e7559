"""B200 ablations of the paper's design choices (Figs. 12-14) and
the data for re-tuning Table 2's load-balancing thresholds — GPU box only.

    python tools/ablation.py [--configs c2,c3,c4,c5] [--steps 3] > gpurun_out/ablation.json

Every variant is the same pipeline with plan options (include/speck.h); every result is checked
against the one of the default plan (row_ptr and col_idx identical, values within tolerance), so
an ablation never measures a wrong answer.  Times: CUDA events around analyze + spgemm
(C allocation outside), median of `steps` after 2 warm-ups.
"""
import argparse
import json
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import workloads as W  # noqa: E402
import paper_conf_ppopp_pargerwms20_b200 as sp  # noqa: E402

VARIANTS = {
    # Fig. 12 (accumulators): hash only -> + dense -> + direct -> + B200 bucket counting sort
    "fig12_hash_only": dict(force_accumulator=1, bucket_sort=0, disable_direct=1),
    "fig12_hash_dense": dict(bucket_sort=0, disable_direct=1),
    "fig12_hash_dense_direct": dict(bucket_sort=0),
    "fig12_b200_default": dict(),
    # Fig. 13 (local load balancing of hash rows): fixed g = 32, the paper's dynamic g, B200 expand-balanced
    "fig13_fixed_g32": dict(bucket_sort=0, fixed_group_size=32),
    "fig13_dynamic_g": dict(bucket_sort=0, fixed_group_size=-1),
    "fig13_expand_balanced": dict(bucket_sort=0, fixed_group_size=0),
    # Fig. 14 (global load balancing): off / always / Table 2 decision
    "fig14_lb_off": dict(global_lb_symbolic=0, global_lb_numeric=0),
    "fig14_lb_on": dict(global_lb_symbolic=1, global_lb_numeric=1),
    "fig14_lb_auto": dict(),
    # B200 extras
    "bucket_sort_symbolic_too": dict(bucket_sort=2),
    "one_stream": dict(concurrent_streams=1),
}


def timed(probs, opts, steps):
    hs = [sp.Handle(0, **opts) for _ in probs]
    outs = None

    def step():
        nonlocal outs
        outs = None                      # the previous step's C must not coexist with this one
        res, prev = [], None
        for (label, A, B), h in zip(probs, hs):
            C = h.spgemm(A, B if B is not None else prev)
            res.append(C)
            prev = C
        outs = res

    for _ in range(2):
        step()
    ts = []
    for _ in range(steps):
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        step()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    st = [h.stats() for h in hs]
    for h in hs:
        h.close()
    return statistics.median(ts), outs, st


def signature(outs):
    """Exact structure (row_ptr, a position-weighted column checksum) and the value sum of every
    product's result — the full C of C3/C5 (70-90 GB) cannot be kept twice on the device."""
    sig = []
    for C in outs:
        ck, vs, va = 0, 0.0, 0.0
        for o in range(0, C.col.numel(), 1 << 27):          # bounded temporaries
            c = C.col[o:o + (1 << 27)].long()
            pos = (torch.arange(o, o + c.numel(), device=c.device, dtype=torch.int64) % 1000003) + 1
            ck = (ck + int((c * pos).sum())) & ((1 << 63) - 1)
            v = C.val[o:o + (1 << 27)].double()
            vs += float(v.sum())
            va += float(v.abs().sum())
        sig.append((C.row_ptr.cpu(), ck, vs, va))
    return sig


def same(sa, sb, tol):
    return all(torch.equal(a[0], b[0]) and a[1] == b[1] and abs(a[2] - b[2]) <= tol * 64 * a[3] + 1e-30
               for a, b in zip(sa, sb))


def lb_sweep(steps):
    """Table 2 re-tuning data: global LB on vs off on R-MAT families of varying skew and size
    and on uniform rows (m_max/m_avg and rows span the thresholds of P:1198-1206)."""
    out = []
    fams = []
    for scale in (12, 14, 16, 18):
        for a in (0.35, 0.45, 0.57):
            b = (1 - a) / 3
            fams.append((f"rmat s{scale} a{a}", lambda s=scale, a=a, b=b: W.rmat(s, 16, (a, b, b, 1 - a - 2 * b), seed=5,
                                                                                 dtype=torch.float32, device="cuda")))
    for n, d in ((1 << 14, 8e-4), (1 << 16, 2e-4), (1 << 18, 5e-5)):
        fams.append((f"uniform n{n}", lambda n=n, d=d: W.random_sparse(n, n, d, seed=3, dtype=torch.float32).to("cuda")))
    for name, gen in fams:
        A = gen()
        probs = [("A*A", A, A)]
        row = {"family": name, "rows": A.rows}
        for tag, o in (("off", dict(global_lb_symbolic=0, global_lb_numeric=0)),
                       ("on", dict(global_lb_symbolic=1, global_lb_numeric=1)), ("auto", {})):
            ms, _, st = timed(probs, o, steps)
            row[tag] = round(ms, 4)
            if tag == "auto":
                row["products"] = st[0]["products"]
                row["max_row_products"] = st[0]["max_row_products"]
                row["nnz_c"] = st[0]["nnz_c"]
                row["auto_choice"] = [st[0]["lb_symbolic"], st[0]["lb_numeric"]]
        row["ratio_prods"] = row["max_row_products"] / max(row["products"] / A.rows, 1e-9)
        out.append(row)
        print(json.dumps({"lb_sweep": row}), flush=True)
        del A, probs
        torch.cuda.empty_cache()
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="c2,c3,c4,c5", help="'' for none")
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--variants", default=",".join(VARIANTS))
    ap.add_argument("--lb-sweep", action="store_true")
    args = ap.parse_args()
    from paper_conf_ppopp_pargerwms20_b200 import build
    build.build()
    res = {"variants": {k: VARIANTS[k] for k in args.variants.split(",")}, "configs": {}}
    for cfg in [c for c in args.configs.split(",") if c]:
        probs = W.config(cfg, device="cuda")
        tol = 1e-5 if probs[0][1].dtype == torch.float32 else 1e-12
        base_ms, ref, st = timed(probs, {}, args.steps)
        ref = signature(ref)
        prods = sum(s["products"] for s in st)
        row = {"products": prods, "default_ms": round(base_ms, 4)}
        for name in args.variants.split(","):
            ms, outs, _ = timed(probs, VARIANTS[name], args.steps)
            ok = same(signature(outs), ref, tol)
            row[name] = {"ms": round(ms, 4), "gflops": round(2 * prods / ms / 1e6, 2), "same_result": ok}
            print(cfg, name, row[name], file=sys.stderr, flush=True)
            del outs
            torch.cuda.empty_cache()
        res["configs"][cfg] = row
        print(json.dumps({"config": cfg, **row}), flush=True)      # one line per config (a kill keeps the rest)
        del probs, ref
        torch.cuda.empty_cache()
    if args.lb_sweep:
        res["lb_sweep"] = lb_sweep(args.steps)


if __name__ == "__main__":
    main()
