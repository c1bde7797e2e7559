"""Per-SASS-opcode breakdown of an ncu report: executed warp instructions and stall samples.

    python tools/ncu_sass.py report.ncu-rep [launch]
"""
import collections
import csv
import io
import subprocess
import sys


def main(rep, launch=0):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass",
                          "--launch-skip", str(launch), "--launch-count", "1"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hi = next(i for i, r in enumerate(rows) if "Source" in r)
    h = rows[hi]
    si = h.index("Source")
    ii = next(i for i, k in enumerate(h) if k.startswith("Instructions Executed"))
    wi = next((i for i, k in enumerate(h) if k.startswith("Warp Stall Sampling (All")), None)
    by_op = collections.Counter()
    st_op = collections.Counter()
    lines = []
    for r in rows[hi + 1:]:
        if len(r) <= ii:
            continue
        src = r[si].strip()
        try:
            n = int(float(r[ii] or 0))
            w = int(float(r[wi] or 0)) if wi is not None else 0
        except ValueError:
            continue
        toks = src.split()
        if not toks:
            continue
        op = toks[0]
        if op.startswith("@"):
            op = toks[1] if len(toks) > 1 else op
        op = op.split(".")[0]
        by_op[op] += n
        st_op[op] += w
        lines.append((n, w, src[:90]))
    tot = sum(by_op.values()) or 1
    stot = sum(st_op.values()) or 1
    print(f"total warp instructions {tot}, stall samples {stot}")
    for op, n in by_op.most_common(30):
        print(f"  {op:10s} {100 * n / tot:5.1f}% inst  {100 * st_op[op] / stot:5.1f}% stalls")
    print("top SASS instructions:")
    for n, w, s in sorted(lines, reverse=True)[:40]:
        print(f"  {100 * n / tot:5.2f}% {100 * w / stot:5.2f}%  {s}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 0)
