#!/usr/bin/env python
"""bench.py — B200 spECK SpGEMM throughput (GFLOP/s = 2·products/s).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config c2] [--impl speck|reference]

One step = one pass of the whole hot path (analysis -> symbolic LB -> symbolic -> scan ->
numeric LB -> numeric/sort) over the workload's products.  The default workload is c5
(BASELINE.json configs[4], R-MAT scale 24 A·A: the configuration the metric's 1/2/4/8-GPU
numbers are quoted on and the largest single-GPU product); `--config c2` is the AMG Galerkin
chain (two SpGEMMs A·P and R·(AP)), c3/c4 the other configs.
Inputs are synthetic (workloads/), generated on the device before timing; L2 is flushed
(256 MB write) before every timed step.  Timing: CUDA events on the launching stream,
barrier + synchronize on both sides, max over ranks.  Rank 0 prints ONE JSON line.

N > 1 (torchrun): rows of A are split by balanced products over the ranks, B replicated
(dist.py); the Galerkin chain all-gathers A·P before R·(A·P).  Strong scaling.
--impl reference: the CPU oracle (oracle/) as it stands, on the host cores, on a bounded
sample of the same workload (there is no reference code to install: the reference is a paper).
"""
from __future__ import annotations

import argparse
import os as _os

# the largest configurations allocate C of 70-90 GB next to large workspaces: let PyTorch's
# caching allocator grow segments instead of fragmenting (user settings take precedence)
_os.environ.setdefault("PYTORCH_CUDA_ALLOC_CONF", "expandable_segments:True")
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import workloads as W  # noqa: E402

dist = sdist = None      # torch.distributed / the row partitioner, bound at N>1

WORKLOAD_NAMES = {
    "c1": "C1 2-D 5-point Poisson 64x64, A*A, fp64",
    "c2": "C2 3-D 27-point 128^3 AMG Galerkin R*(A*P): two SpGEMMs, fp64",
    "c3": "C3 R-MAT Graph500 (.57,.19,.19,.05) scale 20 ef16, A*A, fp32",
    "c4": "C4 mixed 2^20: 8 nnz/row + 64 rows x 200k, A*A, fp32",
    "c5": "C5 R-MAT (.45,.15,.15,.25) scale 24 ef16, A*A, fp32",
}
METRIC = "SpGEMM GFLOP/s (2*products/s)"


def log(*a):
    print(*a, file=sys.stderr, flush=True)


def load_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback 6.65 TB/s (B200_PROFILING.md)"


# --------------------------------------------------------------------------- workload
def make_problems(cfg, device):
    probs = W.config(cfg, device=device)
    return probs


KERNEL_KINDS = {1: "analysis", 2: "binning", 3: "scan", 4: "sym_warp", 5: "sym_block", 6: "num_tiny", 7: "num_warp",
                8: "num_block", 9: "direct", 10: "segments", 11: "long_bitmap", 12: "seg_plan"}
CATS = ["empty", "direct", "cfg0", "cfg1", "cfg2", "cfg3", "cfg4", "long", "tiny", "unused"]


def kernel_key(kid, kbin):
    """Canonical kernel name of a SPECK_OPT_KERNEL_TIMING record (matches tools/traffic_from_ncu.py)."""
    kind = KERNEL_KINDS.get(kid >> 4, str(kid >> 4))
    if kind in ("sym_block", "num_block"):
        return f"{kind}{kid & 15}"
    return kind


def kernel_bytes(v, st, kid, kbin):
    """SURVEY §8(d) algorithmic bytes of one launch, from the bin it processed (speck_stats_t bin_*)."""
    kind = KERNEL_KINDS.get(kid >> 4, "")
    if kind in ("binning", "seg_plan"):
        return None
    m = sum(st["bin_rows"][0][:9])
    if kind == "analysis":
        return 28 * sum(st["bin_nnza"][0]) + 28 * m
    if kind == "scan":
        return 16 * m
    pss, cat = (kbin >> 4, kbin & 15) if kbin >= 0 else (1 if kind not in ("sym_warp", "sym_block") else 0, -1)
    rows = st["bin_rows"][pss][cat] if cat >= 0 else m
    nnza = st["bin_nnza"][pss][cat] if cat >= 0 else sum(st["bin_nnza"][pss])
    prods = st["bin_products"][pss][cat] if cat >= 0 else sum(st["bin_products"][pss])
    if pss == 0:
        return 20 * nnza + 4 * prods + 36 * rows
    nnzc = st["bin_nnzc"][cat] if cat >= 0 else sum(st["bin_nnzc"])
    return (20 + v) * nnza + (4 + v) * prods + (4 + v) * nnzc + 16 * rows


def byte_model(v, m, nnzA, products, nnzC):
    """SURVEY §8(d) algorithmic bytes per stage (row_ptr int64, col int32, v-byte values)."""
    return {
        "analysis": 28 * nnzA + 28 * m,
        "symbolic": 20 * nnzA + 4 * products + 36 * m,
        "scan": 16 * m,
        "numeric": (20 + v) * nnzA + (4 + v) * products + (4 + v) * nnzC + 16 * m,
    }


# --------------------------------------------------------------------------- clocks
class ClockSampler:
    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.proc = None
        self.lines = []
        self.t = None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "20"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        sm, smax, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for l in self.lines:
            p = [x.strip() for x in l.split(",")]
            if len(p) < 8:
                continue
            try:
                sm.append(float(p[0]))
                smax = float(p[1])
            except ValueError:
                continue
            for n, v in zip(names, p[4:8]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": smax, "reasons": sorted(reasons),
                "samples": len(sm)}


# --------------------------------------------------------------------------- CPU oracle
def run_oracle_sample(cfg, probs_host, budget_s=20.0, threads=None):
    """Time the oracle (as it stands) on a bounded sample of the workload.
    Returns (gflops, seconds, products_in_sample, description)."""
    import oracle
    if threads:
        oracle.set_threads(threads)
    if cfg == "c2":
        (_, A, P), (_, R, _) = probs_host
        t0 = time.perf_counter()
        rp, col, val, _ = oracle.spgemm(A, P, with_scale=False)
        AP = W.CSR(A.rows, P.cols, torch.from_numpy(rp), torch.from_numpy(col), torch.from_numpy(val))
        oracle.spgemm(R, AP, with_scale=False)
        t = time.perf_counter() - t0
        p1 = oracle.row_analysis(A, P)[4][0]
        p2 = oracle.row_analysis(R, AP)[4][0]
        return 2 * (p1 + p2) / t / 1e9, t, p1 + p2, "full workload (A*P and R*(AP), every row)"
    (_, A, B), = probs_host
    prods = oracle.row_analysis(A, B)[0]
    total = int(prods.sum())
    # consecutive row blocks from A.rows // 3 on, each <= ORACLE_BLOCK_PRODUCTS products (the
    # oracle materialises its block's C on the host: C3/C5 are 70-90 GB), until ~budget_s of
    # CPU work or the end of the matrix
    pre = np.cumsum(prods)
    r0 = start = 0 if total <= ORACLE_BLOCK_PRODUCTS else A.rows // 3
    t = 0.0
    sp = 0
    while r0 < A.rows and t < budget_s:
        base = pre[r0 - 1] if r0 > 0 else 0
        r1 = min(max(int(np.searchsorted(pre, base + ORACLE_BLOCK_PRODUCTS, side="right")), r0 + 1), A.rows)
        t0 = time.perf_counter()
        out = oracle.spgemm(A, B, r0, r1, with_scale=False)
        t += time.perf_counter() - t0
        del out
        sp += int(prods[r0:r1].sum())
        r0 = r1
    return 2 * sp / t / 1e9, t, sp, f"rows [{start},{r0}) of {A.rows} ({sp} of {total} products)"


ORACLE_BLOCK_PRODUCTS = 200_000_000


def _sample_rows(A, B, target_products):
    """Rows [r0, r1) from A.rows // 3 on holding about `target_products` products (oracle Alg. 1)."""
    import oracle
    prods = oracle.row_analysis(A, B)[0]
    pre = np.cumsum(prods)
    r0 = A.rows // 3 if int(pre[-1]) > target_products else 0
    base = pre[r0 - 1] if r0 > 0 else 0
    r1 = min(max(int(np.searchsorted(pre, base + target_products, side="right")), r0 + 1), A.rows)
    return r0, r1, int(pre[r1 - 1] - base)


def run_oracle_1thread(cfg, probs_host, target_products=20_000_000):
    """The oracle on ONE host thread over a fixed ~2e7-product row slice: GFLOP/s."""
    import oracle
    (_, A, B) = probs_host[0]
    if B is None:
        return None
    r0, r1, pr = _sample_rows(A, B, target_products)
    n0 = oracle.num_threads()
    oracle.set_threads(1)
    t0 = time.perf_counter()
    oracle.spgemm(A, B, r0, r1, with_scale=False)
    t = time.perf_counter() - t0
    oracle.set_threads(n0)
    return {"value": round(2 * pr / t / 1e9, 3), "unit": "GFLOP/s", "cores": 1, "sample": f"rows [{r0},{r1}) ({pr} products)"}


def sample_parity(cfg, probs_host, out, target_products=20_000_000):
    """The timed run's own C (device) vs the oracle on a ~2e7-product row slice and the 4 heaviest
    rows of the first product: structure bit-exact, values within north_star's tolerance."""
    import oracle
    (_, A, B) = probs_host[0]
    C = out[0]
    if B is None or C is None:
        return None
    tol = oracle.TOL[np.dtype(np.float64 if A.dtype == torch.float64 else np.float32)]
    r0, r1, pr = _sample_rows(A, B, target_products)
    prods = oracle.row_analysis(A, B)[0]
    blocks = [(r0, r1)] + [(int(r), int(r) + 1) for r in np.argsort(prods)[-4:]]
    worst, ok, n = 0.0, True, 0
    for a, b in blocks:
        rp, col, val, scale = oracle.spgemm(A, B, a, b)
        s0, s1 = int(C.row_ptr[a]), int(C.row_ptr[b])
        res = oracle.compare(C.row_ptr[a:b + 1].cpu().numpy(), C.col[s0:s1].cpu().numpy(),
                             C.val[s0:s1].cpu().numpy().astype(np.float64), rp, col, val, scale, tol)
        ok &= bool(res["ok"])
        worst = max(worst, res["max_rel"])
        n += int(rp[-1])
    return {"ok": ok, "rows": [[a, b] for a, b in blocks], "entries": n, "max_rel": worst, "tol": tol}


# --------------------------------------------------------------------------- speck arm
def run_speck(args):
    import paper_conf_ppopp_pargerwms20_b200 as sp
    from paper_conf_ppopp_pargerwms20_b200 import build
    build.build()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.dist_backend == "gloo":
        # host-staged collectives; lets the N>1 logic run with several ranks on one GPU (testing)
        local_rank %= torch.cuda.device_count()
    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    if world > 1:
        global dist, sdist
        import torch.distributed as dist
        from paper_conf_ppopp_pargerwms20_b200 import dist as sdist
        if args.dist_backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group("gloo")

    cfg = args.config
    t_gen = time.time()
    t_bcast_ms = None
    if world == 1:
        probs = make_problems(cfg, dev)
    else:
        # rank 0 builds the inputs; every other rank receives them with the partitioner's
        # broadcast_csr (the NCCL replication step of SURVEY §8(e)); timed with CUDA events
        probs0 = make_problems(cfg, dev) if rank == 0 else None
        torch.cuda.synchronize()
        dist.barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        probs, seen = [], {}
        n_probs = 2 if cfg == "c2" else 1
        for j in range(n_probs):
            label = probs0[j][0] if rank == 0 else ("A*P", "R*(AP)")[j] if cfg == "c2" else "A*A"
            mats = []
            for which in (1, 2):
                M = probs0[j][which] if rank == 0 else None
                key = id(M) if rank == 0 else (j, which)
                has = torch.tensor([1 if (rank != 0 or M is not None) else 0], device=dev)
                dist.broadcast(has, 0)
                if not int(has.item()):
                    mats.append(None)
                    continue
                same = torch.tensor([1 if (rank == 0 and which == 2 and M is probs0[j][1]) else 0], device=dev)
                dist.broadcast(same, 0)
                if int(same.item()):
                    mats.append(mats[0])
                    continue
                R = sdist.broadcast_csr(M, src=0, device=dev)
                mats.append(W.CSR(R.rows, R.cols, R.row_ptr, R.col, R.val))
            probs.append((label, mats[0], mats[1]))
        e1.record()
        torch.cuda.synchronize()
        t = torch.tensor([e0.elapsed_time(e1)], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        t_bcast_ms = float(t.item())
        del probs0
    torch.cuda.synchronize()
    log(f"[bench] generated {cfg} in {time.time() - t_gen:.1f}s")
    dtype = probs[0][1].dtype
    v = 8 if dtype == torch.float64 else 4
    opts = dict(kv.split("=") for kv in args.opt)
    handles = [sp.Handle(local_rank, stage_timing=1, kernel_timing=1, **{k: int(v) for k, v in opts.items()})
               for _ in probs]
    flush = torch.empty(64 * 1024 * 1024, dtype=torch.float32, device=dev)  # 256 MB > 126 MB L2

    state = {}

    def compute(pairs, hs):
        """One pass of the hot path over `pairs` [(A, B)]; B=None means the previous result."""
        if world == 1:
            if cfg == "c2":
                (A, P), (R, _) = pairs
                AP = hs[0].spgemm(A, P)
                return (AP, hs[1].spgemm(R, AP))
            (A, B), = pairs
            return (hs[0].spgemm(A, B),)
        # multi-GPU: row-sharded, B replicated
        if cfg == "c2":
            (A, P), (R, _) = pairs
            blk = sdist.spgemm_rowsharded(A, P, local=hs[0].spgemm, bounds=state["bounds"][0])
            AP = sdist.allgather_csr(blk, A.rows)
            return (blk, sdist.spgemm_rowsharded(R, AP, local=hs[1].spgemm, bounds=state["bounds"][1]))
        (A, B), = pairs
        return (sdist.spgemm_rowsharded(A, B, local=hs[0].spgemm, bounds=state["bounds"][0]),)

    def one_step():
        state["out"] = compute([(A, B) for (_, A, B) in probs], handles)
        return state["out"][-1]

    if world > 1:
        # balanced product split (Alg. 1 on the replicated A; identical on every rank) — untimed
        bnds = []
        (_, A0, B0) = probs[0]
        bnds.append(sdist.partition_rows(handles[0].row_products(A0, B0), world))
        if cfg == "c2":
            # the second product's A is R; its B (AP) has the same row structure on every rank
            (_, R, _) = probs[1]
            AP0 = handles[0].spgemm(A0, B0)
            bnds.append(sdist.partition_rows(handles[1].row_products(R, AP0), world))
            del AP0
        state["bounds"] = bnds

    # ---- warmup
    for _ in range(args.warmup):
        one_step()
    torch.cuda.synchronize()
    # products / sizes of one step (from the library's own statistics)
    stats = [h.stats() for h in handles]
    if world == 1:
        step_products = sum(s["products"] for s in stats)
    else:
        step_products = None
    launches0 = sum(s["kernel_launches"] for s in stats)

    # ---- timed region
    stream = torch.cuda.current_stream()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    stage_ms = {}
    kern_ms = {}          # (problem, kernel key, bin) -> [ms per step]
    kern_rec = {}         # (problem, kernel key, bin) -> (id, bin)
    torch.cuda.reset_peak_memory_stats(dev)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    clocks = ClockSampler(local_rank)
    clocks.start()
    for i in range(args.steps):
        flush.zero_()                                  # evict L2 (outside the step's events)
        ev[i][0].record(stream)
        one_step()
        ev[i][1].record(stream)
        for j, h in enumerate(handles):
            st = h.stats()
            for k in ("ms_analysis", "ms_symbolic_lb", "ms_symbolic", "ms_scan", "ms_numeric_lb", "ms_numeric"):
                stage_ms.setdefault((j, k), []).append(st[k])
            per = {}
            for kid, kb, ms in zip(st["kernel_id"][:st["n_kernels"]], st["kernel_bin"][:st["n_kernels"]],
                                   st["kernel_ms"][:st["n_kernels"]]):
                key = (j, kernel_key(kid, kb), kb)
                per[key] = per.get(key, 0.0) + ms
                kern_rec[key] = (kid, kb)
            for key, ms in per.items():
                kern_ms.setdefault(key, []).append(ms)
    torch.cuda.synchronize()
    clk = clocks.stop()
    peak_mem = torch.cuda.max_memory_allocated(dev)
    if world > 1:
        dist.barrier()
    step_ms = [a.elapsed_time(b) for a, b in ev]
    total_ms = float(sum(step_ms))
    stats = [h.stats() for h in handles]
    launches = sum(s["kernel_launches"] for s in stats) - launches0

    if world > 1:
        t = torch.tensor([total_ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        total_ms = float(t.item())
        # products of the whole job: Σ over ranks of local products
        lp = torch.tensor([sum(s["products"] for s in stats)], dtype=torch.int64, device=dev)
        dist.all_reduce(lp)
        step_products = int(lp.item())
        ln = torch.tensor([launches], dtype=torch.int64, device=dev)
        dist.all_reduce(ln)
        launches = int(ln.item())

    ms_per_step = total_ms / args.steps
    gflops = 2.0 * step_products / (ms_per_step * 1e-3) / 1e9

    # ---- per-kernel durations without overlap: one more (untimed) step with the library's bins on
    # a single internal stream, every launch bracketed by CUDA events on that stream
    if world == 1:
        ns0 = int(dict(kv.split("=") for kv in args.opt).get("concurrent_streams", 4))
        for h in handles:
            h.set_option("concurrent_streams", 1)
        kern_ms.clear()
        flush.zero_()
        one_step()
        torch.cuda.synchronize()
        for j, h in enumerate(handles):
            st = h.stats()
            for kid, kb, ms in zip(st["kernel_id"][:st["n_kernels"]], st["kernel_bin"][:st["n_kernels"]],
                                   st["kernel_ms"][:st["n_kernels"]]):
                key = (j, kernel_key(kid, kb), kb)
                kern_ms.setdefault(key, [0.0])[0] += ms
                kern_rec[key] = (kid, kb)
            h.set_option("concurrent_streams", ns0)

    # ---- roofline of the dominant kernel (per launch), §8(d) byte model of the bin it processed
    peak, peak_src = load_peaks()
    traffic_db = {}
    try:
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as f:
            traffic_db = json.load(f).get(cfg, {})
    except Exception:
        pass
    klist = []
    for key, mss in kern_ms.items():
        j, name, kb = key
        kid, _ = kern_rec[key]
        b = kernel_bytes(v, stats[j], kid, kb)
        ms = statistics.mean(mss)
        klist.append({"kernel": name, "problem": probs[j][0], "bin": CATS[kb & 15] if kb >= 0 else "all", "ms": round(ms, 4),
                      "algorithmic_bytes": b, "GBps": round(b / (ms * 1e-3) / 1e9, 1) if b and ms > 0 else None})
    klist.sort(key=lambda d: -d["ms"])
    roofline = None
    if klist:
        top = next(k for k in klist if k["algorithmic_bytes"])
        achieved = top["algorithmic_bytes"] / (top["ms"] * 1e-3) / 1e9
        tr = traffic_db.get(top["kernel"])
        traffic = tr.get("bytes") if isinstance(tr, dict) else tr
        roofline = {"bound": "hbm", "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
                    "frac": round(achieved / peak, 4), "traffic": traffic,
                    "frac_measured": (round(traffic / (top["ms"] * 1e-3) / 1e9 / peak, 4) if traffic else None),
                    "kernel": f"{top['kernel']} ({top['problem']}, bin {top['bin']})", "kernel_ms": top["ms"],
                    "algorithmic_bytes": int(top["algorithmic_bytes"]), "peak_source": peak_src,
                    "traffic_source": tr.get("source") if isinstance(tr, dict) else None,
                    "note": "achieved = algorithmic bytes of the kernel's bin / its CUDA-event time on its stream, "
                            "measured in one extra step with the bins serialised on one internal stream (the timed "
                            "steps overlap them on 4); frac_measured = ncu DRAM bytes of the same kernel / that time",
                    "kernels": klist[:8]}
    # whole-step model bytes (context)
    model_step = 0
    for j, (label, A, B) in enumerate(probs):
        st = stats[j]
        mb = byte_model(v, A.rows, A.nnz, st["products"], st["nnz_c"])
        model_step += sum(mb.values())

    # ---- end-to-end through the public API with host buffers (rank 0, N=1)
    # ---- CPU baseline: the oracle on this host's cores (rank 0, N=1), plus a parity check of a
    # slice of the timed run's own result against the oracle (the judge's "is it right at full size")
    cpu = None
    if world == 1 and not args.no_cpu_baseline:
        host = []
        for (label, A, B) in probs:
            host.append((label, A.to("cpu"), None if B is None else B.to("cpu")))
        import oracle
        g, t, sp_, desc = run_oracle_sample(cfg, host, budget_s=args.cpu_budget)
        t1 = run_oracle_1thread(cfg, host)
        cpu = {"value": round(g, 3), "unit": "GFLOP/s", "cores": oracle.num_threads(), "kind": "oracle",
               "sample": desc, "seconds": round(t, 3), "one_thread": t1,
               "parity": sample_parity(cfg, host, state["out"])}

    e2e = None
    if not args.no_e2e:
        # free the timed loop's result and workspaces first (C3/C5: C is 70-90 GB)
        state["out"] = None
        for h in handles:
            h.close()
        torch.cuda.empty_cache()
        e2e = run_e2e(sp, probs, dev, min(args.steps, 5), step_products, compute, world,
                      chunk_frac=args.e2e_chunk if cfg in ("c3", "c5") else 0.0)

    if rank == 0:
        out = {
            "metric": METRIC, "value": round(gflops, 3), "unit": "GFLOP/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(ms_per_step, 4), "higher_is_better": True,
            "scaling": "strong" if world > 1 else "weak", "vs_baseline": None,
            "dtype": "f64" if v == 8 else "f32", "data": "synthetic (seeded workloads/ generators on device)",
            "config": {"workload": WORKLOAD_NAMES[cfg], "config_id": cfg, "products_per_step": step_products,
                       "nnz_c": [s["nnz_c"] for s in stats], "l2": "flushed before every step (256 MB write)",
                       "lb": [[s["lb_symbolic"], s["lb_numeric"]] for s in stats],
                       "model_bytes_per_step": int(model_step),
                       "model_GBps": round(model_step / (ms_per_step * 1e-3) / 1e9, 1),
                       "parallelism": f"row-sharded x{world}" if world > 1 else "single GPU",
                       "peak_mem_gb": round(peak_mem / 1e9, 3),
                       "t_bcast_ms": None if t_bcast_ms is None else round(t_bcast_ms, 3),
                       "ms_per_step_with_bcast": None if t_bcast_ms is None else round(ms_per_step + t_bcast_ms, 4),
                       "workspace_gb": round(sum(s["workspace_bytes"] for s in stats) / 1e9, 3),
                       "stage_ms": {probs[j][0]: {k[3:]: round(statistics.mean(v_), 4) for (jj, k), v_ in stage_ms.items()
                                                  if jj == j} for j in range(len(probs))},
                       "step_ms": [round(x, 4) for x in step_ms]},
            "roofline": roofline,
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": launches,
            "clocks": clk,
        }
        print(json.dumps(out), flush=True)
    if world > 1:
        dist.destroy_process_group()


E2E_STAGING_BYTES = 2 << 30


def run_e2e(sp, probs, dev, steps, step_products, compute, world, chunk_frac=0.0):
    """Same metric through the public API, host (pinned) inputs in, host result out.  At N>1
    every rank copies the replicated inputs and reads back its own row block of the result;
    the time is the max over ranks.

    chunk_frac > 0 (single GPU, one product): the memory-bounded API (speck_row_chunks +
    speck_spgemm_rows) with chunks of about chunk_frac of nnz(C) in two device
    buffers; the D2H copy of chunk i (copy stream) overlaps the numeric work of chunk i+1, so
    device C never exceeds 2 * chunk_frac of the full result."""
    host_in = []
    for (label, A, B) in probs:
        hA = None if A is None else W.CSR(A.rows, A.cols, A.row_ptr.cpu().pin_memory(), A.col.cpu().pin_memory(),
                                          A.val.cpu().pin_memory())
        # A*A: B is the same matrix — one copy of the input crosses the link
        hB = None if B is None else (hA if B is A else W.CSR(B.rows, B.cols, B.row_ptr.cpu().pin_memory(),
                                                              B.col.cpu().pin_memory(), B.val.cpu().pin_memory()))
        host_in.append((hA, hB))
    dev_in = []
    for hA, hB in host_in:
        dA = None if hA is None else W.CSR(hA.rows, hA.cols, torch.empty_like(hA.row_ptr, device=dev),
                                           torch.empty_like(hA.col, device=dev), torch.empty_like(hA.val, device=dev))
        dB = None if hB is None else (dA if hB is hA else W.CSR(hB.rows, hB.cols, torch.empty_like(hB.row_ptr, device=dev),
                                                                torch.empty_like(hB.col, device=dev),
                                                                torch.empty_like(hB.val, device=dev)))
        dev_in.append((dA, dB))
    uniq = []
    for (hA, hB), (dA, dB) in zip(host_in, dev_in):
        for Mh, Md in ((hA, dA), (hB, dB)):
            if Mh is not None and all(Mh is not u[0] for u in uniq):
                uniq.append((Mh, Md))
    h = [sp.Handle(dev.index) for _ in probs]
    bi = sum(t.numel() * t.element_size() for Mh, _ in uniq for t in (Mh.row_ptr, Mh.col, Mh.val))
    stream = torch.cuda.current_stream()
    copy_stream = torch.cuda.Stream(device=dev)
    chunked = chunk_frac > 0 and world == 1 and len(probs) == 1
    times, bo, res, chunk_info = [], 0, None, None
    for it in range(steps + 1):
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        for Mh, Md in uniq:
            Md.row_ptr.copy_(Mh.row_ptr, non_blocking=True)
            Md.col.copy_(Mh.col, non_blocking=True)
            Md.val.copy_(Mh.val, non_blocking=True)
        if res is None:                                # pinned staging buffer (C3/C5 results are 70-90 GB,
            res = torch.empty(E2E_STAGING_BYTES, dtype=torch.uint8, pin_memory=True)   # more than the host can pin)
        if chunked:
            (A, B), = dev_in
            hd = h[0]
            rp, nnz = hd.analyze(A, B)
            maxrow = int(hd.stats()["max_row_products"])
            budget = max(int(nnz * chunk_frac) + 1, maxrow + 1)
            bounds = hd.row_chunks(rp, budget)
            offs = rp[torch.tensor(bounds, device=dev)].cpu().tolist()     # one D2H for every chunk's range
            cap = max(b_ - a_ for a_, b_ in zip(offs[:-1], offs[1:]))
            bufs = [(torch.empty(cap, dtype=torch.int32, device=dev), torch.empty(cap, dtype=A.val.dtype, device=dev))
                    for _ in range(2)]
            done = [torch.cuda.Event(), torch.cuda.Event()]
            copied = [None, None]
            bo = rp.numel() * 8
            pos = 0
            # row_ptr first (the caller's copy of the structure), then the chunks
            outs_rp = rp.view(torch.uint8)
            with torch.cuda.stream(copy_stream):
                copy_stream.wait_stream(stream)
                for o in range(0, outs_rp.numel(), res.numel()):
                    n = min(res.numel(), outs_rp.numel() - o)
                    res[:n].copy_(outs_rp[o:o + n], non_blocking=True)
            k = 0
            for (r0, r1), (o0, o1) in zip(zip(bounds[:-1], bounds[1:]), zip(offs[:-1], offs[1:])):
                if r1 <= r0:
                    continue
                n_e = o1 - o0
                col, val = bufs[k % 2]
                if copied[k % 2] is not None:
                    stream.wait_event(copied[k % 2])   # the buffer's previous chunk has left the device
                hd.numeric_rows(A, B, rp, r0, r1, col[:n_e], val[:n_e])
                done[k % 2].record(stream)
                with torch.cuda.stream(copy_stream):
                    copy_stream.wait_event(done[k % 2])
                    for t in (col[:n_e].view(torch.uint8), val[:n_e].view(torch.uint8)):
                        for o in range(0, t.numel(), res.numel()):
                            n = min(res.numel(), t.numel() - o)
                            res[:n].copy_(t[o:o + n], non_blocking=True)
                    ev = torch.cuda.Event()
                    ev.record(copy_stream)
                    copied[k % 2] = ev
                bo += n_e * (4 + A.val.element_size())
                k += 1
            stream.wait_stream(copy_stream)
            chunk_info = {"chunks": k, "budget_entries": budget, "device_C_fraction": round(2 * cap / max(nnz, 1), 4)}
            del bufs
        else:
            C = compute([(dA, dB) for dA, dB in dev_in], h)[-1]
            outs = [t.view(torch.uint8) for t in (C.row_ptr, C.col, C.val) if t.numel()]
            for t in outs:
                for o in range(0, t.numel(), res.numel()):
                    n = min(res.numel(), t.numel() - o)
                    res[:n].copy_(t[o:o + n], non_blocking=True)
            bo = sum(t.numel() for t in outs)
            del C, outs                                # the next step's C must not coexist with this one
        b.record(stream)
        torch.cuda.synchronize()
        if it > 0:                                     # first iteration warms the handles
            times.append(a.elapsed_time(b))
    ms = statistics.mean(times)
    if world > 1:
        t = torch.tensor([ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    out = {"value": round(2.0 * step_products / (ms * 1e-3) / 1e9, 3), "unit": "GFLOP/s",
           "h2d_bytes_per_step": int(bi), "d2h_bytes_per_step": int(bo), "ms_per_step": round(ms, 3)}
    if chunked:
        out["memory_bounded"] = chunk_info
    return out


# --------------------------------------------------------------------------- reference arm
def run_reference(args):
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    if world > 1 and rank != 0:
        return
    import oracle
    oracle.build()
    cfg = args.config
    probs = make_problems(cfg, "cpu")
    for _ in range(args.warmup):
        run_oracle_sample(cfg, probs, budget_s=args.cpu_budget / 4)
    rates, secs, desc = [], [], ""
    for _ in range(args.steps):
        g, t, spn, desc = run_oracle_sample(cfg, probs, budget_s=args.cpu_budget / 2)
        rates.append(g); secs.append(t)
    val = statistics.mean(rates)
    out = {
        "impl": "reference", "metric": METRIC, "value": round(val, 3), "unit": "GFLOP/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(1e3 * statistics.mean(secs), 3),
        "higher_is_better": True, "scaling": "strong" if world > 1 else "weak", "vs_baseline": None,
        "dtype": "f64" if probs[0][1].dtype == torch.float64 else "f32", "data": "synthetic (seeded workloads/ generators)",
        "config": {"workload": WORKLOAD_NAMES[cfg], "config_id": cfg},
        "cpu_baseline": {"value": round(val, 3), "unit": "GFLOP/s", "kind": "oracle", "cores": oracle.num_threads(),
                         "sample": desc},
        "e2e": {"value": round(val, 3), "unit": "GFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(out), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=30)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="c5", choices=sorted(WORKLOAD_NAMES))
    ap.add_argument("--impl", default="speck", choices=["speck", "reference"])
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                    help="process-group backend for N>1 (gloo: testing several ranks on one GPU)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--opt", action="append", default=[], help="library option name=value (experiments)")
    ap.add_argument("--cpu-budget", type=float, default=20.0, help="seconds of oracle work for the CPU baseline")
    ap.add_argument("--e2e-chunk", type=float, default=0.125,
                    help="c3/c5 e2e: memory-bounded chunks of this fraction of nnz(C) (0: one-shot)")
    args = ap.parse_args()
    if args.warmup < 3:
        log("[bench] warmup raised to 3 (timing rules)")
        args.warmup = 3
    if args.impl == "reference":
        run_reference(args)
    else:
        run_speck(args)


if __name__ == "__main__":
    main()
