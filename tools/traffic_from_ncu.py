"""Write profiles/traffic.json from `ncu --set full` reports (never edited by hand).

    python tools/traffic_from_ncu.py CFG TAG report1.ncu-rep [report2.ncu-rep ...]
    python tools/traffic_from_ncu.py --ingest CFG TAG gpurun_out/<tag>_<cfg>_traffic.txt   (lines printed by --dry)

For every launch in the reports: DRAM bytes (dram__bytes_read.sum + dram__bytes_write.sum) and
the ncu duration, keyed by the same canonical kernel name bench.py derives from the library's
SPECK_OPT_KERNEL_TIMING records (sym_block1, num_warp, segments, ...).  bench.py reports the
entry of its dominant kernel as roofline.traffic.  TAG names the capture (e.g. r02d) so a
reader can find the summary under profiles/.
"""
import csv
import io
import json
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def key_of(name: str):
    m = re.search(r"k_spgemm<\(?int\)?(\d+), \(?int\)?(\d+),", name) or re.search(r"k_spgemm<(\d+), (\d+),", name)
    if m:
        return ("sym_block" if m.group(2) == "0" else "num_block") + m.group(1)
    m = re.search(r"k_warp_rows<\(?int\)?(\d+), \w+, \(?int\)?(\d+)>", name) or re.search(r"k_warp_rows<(\d+), \w+, (\d+)>", name)
    if m:
        return "sym_warp" if m.group(1) == "0" else ("num_tiny" if m.group(2) == "1" else "num_warp")
    for pat, key in (("k_segments", "segments"), ("k_long_bitmap", "long_bitmap"), ("k_analysis", "analysis"),
                     ("k_direct", "direct"), ("k_scan", "scan"), ("k_classify", "binning"), ("k_bin_scatter", "binning")):
        if pat in name:
            return key
    return None


def metrics(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, units, data = rows[0], rows[1], rows[2:]
    res = []
    for d in data:
        name = d[h.index("Kernel Name")]

        def val(k):
            i = h.index(k)
            x = float(d[i].replace(",", ""))
            u = units[i]
            return x * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12, "ns": 1e-6, "us": 1e-3,
                        "usecond": 1e-3, "msecond": 1, "ms": 1, "nsecond": 1e-6, "second": 1e3}.get(u, 1)
        res.append((name, val("dram__bytes_read.sum") + val("dram__bytes_write.sum"), val("gpu__time_duration.sum")))
    return res


def ingest(cfg, tag, txt_files):
    """Merge `--dry` lines printed on the GPU box (gpurun_out/*_traffic.txt) into traffic.json."""
    head = subprocess.run(["git", "rev-parse", "--short=12", "HEAD"], capture_output=True, text=True, cwd=ROOT).stdout.strip()
    path = os.path.join(ROOT, "profiles", "traffic.json")
    db = {}
    if os.path.exists(path):
        with open(path) as f:
            db = json.load(f)
    db = {k: v for k, v in db.items() if isinstance(v, dict) and all(isinstance(x, dict) for x in v.values())}
    ent = db.setdefault(cfg, {})
    for fn in txt_files:
        for line in open(fn):
            t = line.split()
            if len(t) < 7 or t[0] != cfg:
                continue
            ent[t[1]] = {"bytes": int(t[6]), "ncu_ms": float(t[4]), "kernel": " ".join(t[7:])[:120],
                         "source": f"{tag}: {os.path.basename(fn)} (ncu --set full; committed at {head})"}
    with open(path, "w") as f:
        json.dump(db, f, indent=1, sort_keys=True)


def main():
    if sys.argv[1] == "--ingest":
        ingest(sys.argv[2], sys.argv[3], sys.argv[4:])
        return
    dry = "--dry" in sys.argv
    args = [a for a in sys.argv[1:] if a != "--dry"]
    cfg, tag, reps = args[0], args[1], args[2:]
    head = subprocess.run(["git", "rev-parse", "--short=12", "HEAD"], capture_output=True, text=True, cwd=ROOT).stdout.strip()
    path = os.path.join(ROOT, "profiles", "traffic.json")
    db = {}
    if os.path.exists(path):
        with open(path) as f:
            db = json.load(f)
    db = {k: v for k, v in db.items() if isinstance(v, dict) and all(isinstance(x, dict) for x in v.values())}
    ent = db.setdefault(cfg, {})
    for rep in reps:
        for name, b, ms in metrics(rep):
            k = key_of(name)
            if k is None:
                continue
            ent[k] = {"bytes": int(b), "ncu_ms": round(ms, 4), "kernel": name[:120],
                      "source": f"{tag}: {os.path.basename(rep)} (ncu --set full, built from {head})"}
            print(f"{cfg} {k:14s} {b / 1e9:9.3f} GB  {ms:9.3f} ms  {int(b)} {name[:80]}")
    if dry:   # print only (GPU side); profiles/traffic.json is written from the printed lines
        return
    with open(path, "w") as f:
        json.dump(db, f, indent=1, sort_keys=True)


if __name__ == "__main__":
    main()
