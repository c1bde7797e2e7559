"""Summarise an `ncu --metrics gpu__time_duration.sum --csv` launch list by kernel."""
import csv, collections, sys
rows = list(csv.reader(open(sys.argv[1])))
hi = [i for i, r in enumerate(rows) if 'Kernel Name' in r][0]
h = rows[hi]; data = rows[hi + 1:]
ki, vi = h.index('Kernel Name'), h.index('Metric Value')
agg = collections.OrderedDict(); tot = 0.0; mine = 0.0
for r in data:
    name = r[ki]
    v = float(r[vi].replace(',', ''))
    a = agg.setdefault(name[:100], [0.0, 0]); a[0] += v; a[1] += 1; tot += v
    if 'speck' in name or 'k_' in name[:30]:
        mine += v
print(f"total {tot/1e6:.3f} ms over {len(data)} launches; speck kernels {mine/1e6:.3f} ms")
for k, (v, n) in sorted(agg.items(), key=lambda x: -x[1][0])[:int(sys.argv[2]) if len(sys.argv) > 2 else 25]:
    print(f"{v/1e6:10.3f} ms {n:5d}  {k}")
