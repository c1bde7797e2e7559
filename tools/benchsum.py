"""Compact view of bench.py JSON lines: python tools/benchsum.py file.json [...]"""
import json
import sys

for fn in sys.argv[1:]:
    try:
        d = json.loads([l for l in open(fn).read().splitlines() if l.startswith("{")][-1])
    except Exception as e:
        print(fn, "no JSON line:", e)
        continue
    c = d["config"]
    print(f"{fn}: {c.get('config_id')} {d['ms_per_step']:.2f} ms/step  {d['value']} {d['unit']}  "
          f"peak_mem {c.get('peak_mem_gb')} GB  clocks {d.get('clocks', {}).get('sm_mhz')}")
    for prob, st in c.get("stage_ms", {}).items():
        print("   ", prob, {k: round(v, 2) for k, v in st.items()})
    r = d.get("roofline") or {}
    if r:
        print(f"    roofline: {r.get('kernel')} {r.get('kernel_ms')} ms  frac {r.get('frac')}  measured {r.get('frac_measured')}")
        for k in r.get("kernels", []):
            print(f"      {k['kernel']:12s} {k['problem']:8s} {k['bin']:6s} {k['ms']:9.3f} ms  {k['GBps']} GB/s")
    if d.get("cpu_baseline"):
        print("    cpu:", d["cpu_baseline"])
    if d.get("e2e"):
        print("    e2e:", d["e2e"])
