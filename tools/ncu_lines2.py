"""Per-source-line instruction counts of an ncu report (cuda source view), with average active
threads per instruction (divergence) and stall samples.   python tools/ncu_lines2.py rep [N]"""
import csv, io, subprocess, sys
rep = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 40
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"], capture_output=True, text=True).stdout
cur, hdr, out = None, None, []
for r in csv.reader(io.StringIO(txt)):
    if len(r) >= 2 and r[0] in ("File Path", "File Name"):
        cur = r[1].split("/")[-1]; continue
    if r and r[0] == "Line No":
        hdr = r; continue
    if hdr and r and r[0].isdigit():
        ix = {k: i for i, k in reversed(list(enumerate(hdr)))}
        try:
            g = lambda k: r[ix[k]] if ix[k] < len(r) else ""
            out.append((int(g("Instructions Executed") or 0), float(g("Avg. Threads Executed") or 0),
                        int(g("Warp Stall Sampling (All Samples)") or 0), cur, r[0], r[1].strip()[:80]))
        except (ValueError, KeyError):
            pass
ti = sum(o[0] for o in out) or 1
ts = sum(o[2] for o in out) or 1
acc = 0
print(f"total warp instructions {ti:.4g}, stall samples {ts}")
for o in sorted(out, reverse=True)[:n]:
    acc += o[0]
    print(f"{100*o[0]/ti:5.1f}% (cum {100*acc/ti:5.1f}%) thr {o[1]:4.1f} stall {100*o[2]/ts:4.1f}%  {o[3]}:{o[4]}  {o[5]}")
