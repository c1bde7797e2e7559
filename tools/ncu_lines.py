"""Aggregate an `ncu --page source --csv` export by CUDA source line (top stall lines)."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
cur = None; hdr = None; out = []
for r in rows:
    if len(r) >= 2 and r[0] == 'File Path':
        cur = r[1].split('/')[-1]; continue
    if r and r[0] == 'Line No':
        hdr = r; continue
    if hdr and r and r[0].isdigit():
        try:
            s = int(r[4] or 0); i = int(r[7] or 0)
        except ValueError:
            continue
        out.append((s, i, cur, r[0], r[1][:110]))
tot = sum(o[0] for o in out) or 1; ti = sum(o[1] for o in out) or 1
print("stall samples", tot, "warp instructions", ti)
for o in sorted(out, reverse=True)[:top]:
    print(f"{100*o[0]/tot:5.1f}%s {100*o[1]/ti:5.1f}%i {o[2]}:{o[3]}  {o[4]}")
